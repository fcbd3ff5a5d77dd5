"""Probe counts/times of candidate workloads on the GPU (one line per query)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("STM_WATCHDOG_S", "120")
import stmgen
from paper_conf_sc_weij22_b200 import stm
cfgs = sys.argv[1].split(",")
pats = sys.argv[2].split(",")
out = open(sys.argv[3], "a") if len(sys.argv) > 3 else sys.stdout
for cfg in cfgs:
    t = time.time(); g = stmgen.config_graph(cfg); tg = time.time() - t
    t = time.time(); G = stm.Graph.from_stmgen(g); tl = time.time() - t
    print(cfg, g.stats(), f"gen {tg:.1f}s load {tl:.1f}s", file=out, flush=True)
    for spec in pats:
        name, _, mode = spec.partition(":")
        vi = mode == "vi"
        p = stmgen.CATALOG[name]
        lab = None
        if g.labels is not None:
            lab = stmgen.pattern_labels(p.k, 8, 7)
        plan = stm.Plan(p.k, p.edges, lab, vertex_induced=vi)
        for rep in range(2):
            try:
                t = time.time(); c = stm.count(G, plan); dt = time.time() - t
                info = stm.stm_last_launch()
                print(cfg, spec, lab, "count", c, f"time {dt:.4f}s", f"{c/dt:.3e} m/s", info, file=out, flush=True)
            except Exception as e:
                print(cfg, spec, "ERR", e, file=out, flush=True)
                break
