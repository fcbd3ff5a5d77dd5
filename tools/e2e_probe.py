"""Break the bench's end-to-end step into its parts: python tools/e2e_probe.py [cfg]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import stmgen  # noqa: E402
from paper_conf_sc_weij22_b200 import stm  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "c5"
g = stmgen.config_graph(cfg)
plans = [stm.Plan(stmgen.CATALOG[p].k, stmgen.CATALOG[p].edges) for p in ("k5", "k6_minus_e")]
G0 = stm.Graph.from_stmgen(g)
for pl in plans:
    stm.count(G0, pl)  # JIT warm
for rep in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    gh = stm.stm_graph_load(g.n, g.row_ptr, g.col_idx, g.labels, 0)
    t1 = time.perf_counter()
    c = [stm.stm_match_count(gh, pl.handle) for pl in plans]
    t2 = time.perf_counter()
    stm.stm_graph_free(gh)
    print(f"load {1e3 * (t1 - t0):.1f} ms, counts (first launches on the new graph) {1e3 * (t2 - t1):.1f} ms {c}",
          flush=True)
