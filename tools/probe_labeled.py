"""Count candidate labeled queries on a config graph (choosing golden cases): python tools/probe_labeled.py c4"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import stmgen
from paper_conf_sc_weij22_b200 import stm
g = stmgen.config_graph(sys.argv[1])
G = stm.Graph.from_stmgen(g)
cands = [("c6", (0, 1, 2, 0, 1, 2)), ("c6", (0, 1, 2, 3, 4, 5)), ("prism", (0, 0, 0, 1, 1, 1)), ("prism", (0, 1, 2, 0, 1, 2)),
         ("w5", (0, 1, 1, 1, 1, 1)), ("w5", (0, 1, 2, 1, 2, 1)), ("octahedron", (0, 0, 1, 1, 2, 2)),
         ("k6_minus_e", (0, 0, 1, 1, 1, 1)), ("c7", (0, 1, 2, 3, 4, 5, 6)), ("c7", (0, 1, 0, 1, 0, 1, 2)),
         ("w6", (0, 1, 1, 1, 1, 1, 1)), ("w6", (0, 1, 2, 1, 2, 1, 2)), ("w6", (0, 1, 1, 2, 2, 1, 1)),
         ("k7_minus_e", (0, 0, 0, 0, 0, 1, 1)), ("w6", (1, 0, 0, 0, 0, 0, 0))]
for name, lab in cands:
    p = stmgen.CATALOG[name]
    plan = stm.Plan(p.k, p.edges, lab, graph=G)
    t = time.perf_counter(); c = stm.count(G, plan); dt = time.perf_counter() - t
    print(f"{name:12} {lab} count {c:>14} {dt*1e3:9.1f} ms", flush=True)
