import os, sys, time
sys.path.insert(0, os.getcwd())
import torch, stmgen
from paper_conf_sc_weij22_b200 import stm, dist as sdist
g = stmgen.config_graph("c5")
G = stm.Graph.from_stmgen(g)
plans = [stm.Plan(stmgen.CATALOG[p].k, stmgen.CATALOG[p].edges, None, graph=G) for p in ("k5", "k6_minus_e")]
layer = sdist.MultiGPUCounter(G, device=torch.device("cuda", 0))
for pl in plans:
    layer.count(pl)
import time as _t
orig = stm.stm_graph_load
def timed_load(*a, **k):
    t = _t.perf_counter(); h = orig(*a, **k); print(f"  load {1e3*(_t.perf_counter()-t):.1f} ms", flush=True); return h
stm.stm_graph_load = timed_load
for i in range(3):
    r = layer.e2e(g, plans, steps=1)
    print("e2e step", f"{r['seconds_per_step']*1e3:.1f} ms", flush=True)
