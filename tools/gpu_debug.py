"""Quick GPU sanity sweep: one case per line, flushed, so a hang is localised."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import sys, time
os.environ.setdefault("STM_WATCHDOG_S", "5")
import numpy as np
import oracle, stmgen
from stmgen import CATALOG
from paper_conf_sc_weij22_b200 import stm

out = open(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/dbg.log", "w")
def log(*a):
    print(*a, file=out, flush=True); print(*a, flush=True)

graphs = {"er": stmgen.er(300, 2500, 7), "rmat": stmgen.rmat(10, 4000, 0.57, 0.19, 0.19, 17)}
tunings = [dict(local_steal=0, global_steal=0), dict(local_steal=1, global_steal=0), dict()]
for gname, g in graphs.items():
    G = stm.Graph.from_stmgen(g)
    for name in ["edge", "triangle", "wedge", "k4", "c4", "diamond", "house", "c5", "k5"]:
        for vi in (False, True):
            p = CATALOG[name]
            t0 = time.time()
            want = oracle.count(g, p.k, p.edges, vertex_induced=vi, restrictions=oracle.gk_restrictions(p.k, p.edges))
            to = time.time() - t0
            for tk in tunings:
                plan = stm.Plan(p.k, p.edges, vertex_induced=vi)
                t1 = time.time()
                try:
                    got = stm.count(G, plan, stm.stm_tuning_default(**tk))
                except Exception as ex:
                    got = repr(ex)
                tg = time.time() - t1
                log(gname, name, "vi" if vi else "ei", tk, "want", want, "got", got, "OK" if got == want else "MISMATCH",
                    f"oracle {to:.2f}s gpu {tg:.3f}s", stm.stm_last_launch())
