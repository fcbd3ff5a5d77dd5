import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import stmgen, oracle
from paper_conf_sc_weij22_b200 import stm
g = stmgen.er(300, 2500, 7); G = stm.Graph.from_stmgen(g)
for name in sys.argv[1].split(","):
    p = stmgen.CATALOG[name]
    t = stm.stm_tuning_default(**{k: int(v) for k, v in (a.split("=") for a in sys.argv[2:])})
    c = stm.count(G, stm.Plan(p.k, p.edges), t)
    print(name, c, oracle.count(g, p.k, p.edges, restrictions=oracle.gk_restrictions(p.k, p.edges)), flush=True)
