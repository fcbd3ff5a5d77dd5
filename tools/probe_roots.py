"""Per-root match counts of a query (which roots carry the work): python tools/probe_roots.py c5 k6_minus_e"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import stmgen
from paper_conf_sc_weij22_b200 import stm
g = stmgen.config_graph(sys.argv[1])
G = stm.Graph.from_stmgen(g)
p = stmgen.CATALOG[sys.argv[2]]
plan = stm.Plan(p.k, p.edges)
tot, pr = stm.stm_match_count_per_root(G.handle, plan.handle, stm.stm_tuning_default())
deg = g.degrees()
rank = np.empty(g.n, np.int64); rank[np.lexsort((np.arange(g.n), deg))] = np.arange(g.n)
o = np.argsort(-pr.astype(np.float64))
print("total", tot, "roots with matches", np.count_nonzero(pr))
for v in o[:25]:
    print(f"root {v} rank {rank[v]} (n-{g.n - rank[v]}) deg {deg[v]} count {pr[v]} share {pr[v] / tot:.4f}")
