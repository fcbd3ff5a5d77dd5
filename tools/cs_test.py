import sys; sys.path.insert(0, '.')
import stmgen
from paper_conf_sc_weij22_b200 import stm
g = stmgen.er(60, 200, 3)
G = stm.Graph.from_stmgen(g)
import sys
print(stm.stm_motif_census(G.handle, 3, 0, tuning=stm.stm_tuning_default(**dict(a.split("=") for a in sys.argv[1:]))))
