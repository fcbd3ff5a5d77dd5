import os, sys, time
sys.path.insert(0, os.getcwd())
import torch, stmgen
from paper_conf_sc_weij22_b200 import stm
from paper_conf_sc_weij22_b200.dist import MultiGPUCounter
g = stmgen.config_graph("c2"); G = stm.Graph.from_stmgen(g, device=0)
p = stmgen.CATALOG["c4"]; plan = stm.Plan(p.k, p.edges)
for wd in (1, 5, 20):
    t = stm.stm_tuning_default(watchdog_ms=wd)
    layer = MultiGPUCounter(G, tuning=t, device=torch.device("cuda", 0))
    d = layer.new_results(1)
    t0 = time.perf_counter(); layer.count_async(plan, d[0]); layer.reduce_counts(d)
    row = d.cpu().tolist()[0]; print("async wd", wd, row, f"{(time.perf_counter()-t0)*1e3:.1f} ms", flush=True)
    try:
        t0 = time.perf_counter(); c = stm.count(G, plan, t); print("sync", c, f"{(time.perf_counter()-t0)*1e3:.1f} ms")
    except Exception as e:
        print("sync raised", e)
