"""Motif census timing (NEXT-3): python tools/census.py c2:4 c5:4 ... -- greedy vs cost orders."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("STM_WATCHDOG_S", "120")
import stmgen
from paper_conf_sc_weij22_b200 import stm
for spec in sys.argv[1:]:
    cfg, k = spec.split(":")[:2]
    k = int(k)
    flags = stm.STM_VERTEX_INDUCED if ":vi" in spec else 0
    g = stmgen.config_graph(cfg)
    G = stm.Graph.from_stmgen(g)
    stats = stm.stm_graph_stats_host(g.n, g.row_ptr, g.labels)
    for name, st in (("greedy", None), ("cost", stats)):
        stm.stm_motif_census(G.handle, k, flags, st)  # warm-up
        t0 = time.perf_counter()
        c = stm.stm_motif_census(G.handle, k, flags, st)
        dt = time.perf_counter() - t0
        print(f"{spec:10} {name:6} {len(c)} motifs {dt * 1e3:10.2f} ms  total {sum(c)}  counts {c}", flush=True)
    G.close()
