"""Run query launches for ncu: one warm-up launch then one measured launch per query."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import stmgen
from paper_conf_sc_weij22_b200 import stm
cfg = sys.argv[1]
g = stmgen.config_graph(cfg)
G = stm.Graph.from_stmgen(g)
for spec in sys.argv[2].split(","):
    name, _, mode = spec.partition(":")
    p = stmgen.CATALOG[name]
    plan = stm.Plan(p.k, p.edges, vertex_induced=(mode == "vi"))
    for _ in range(2):
        c = stm.count(G, plan)
    print(cfg, spec, c, flush=True)
