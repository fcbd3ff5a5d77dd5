import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import stmgen
from paper_conf_sc_weij22_b200 import stm
g = stmgen.rmat(8, 900, 0.57, 0.19, 0.19, 3)
G = stm.Graph.from_stmgen(g)
p = stmgen.CATALOG["k4"]
pl = stm.Plan(p.k, p.edges)
for label, fn in [("list-first", lambda: stm.stm_match_list(G.handle, pl.handle, p.k, None, capacity=10)[1]),
                  ("instr", lambda: stm.stm_match_count_ex(G.handle, pl.handle, stm.stm_tuning_default(instrument=1))),
                  ("count", lambda: stm.count(G, pl)),
                  ("list-after", lambda: stm.stm_match_list(G.handle, pl.handle, p.k, None, capacity=10)[1]),
                  ("list-occ2", lambda: stm.stm_match_list(G.handle, pl.handle, p.k, stm.stm_tuning_default(occupancy=2), capacity=10)[1])]:
    try:
        print(label, fn(), flush=True)
    except Exception as e:
        print(label, "ERR", e, flush=True)
