"""Per-motif greedy vs cost-order timing with the model's predicted cost ratio:
python tools/census_permotif.py c1:6:vi ..."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("STM_WATCHDOG_S", "60")
import stmgen
from paper_conf_sc_weij22_b200 import stm


def best_of(G, plan, reps=3):
    b = 1e9
    for _ in range(reps):
        t0 = time.perf_counter(); c = stm.count(G, plan); b = min(b, time.perf_counter() - t0)
    return c, b


for spec in sys.argv[1:]:
    cfg, k = spec.split(":")[:2]
    k = int(k)
    vi = ":vi" in spec
    g = stmgen.config_graph(cfg)
    G = stm.Graph.from_stmgen(g)
    st = stm.stm_graph_stats_host(g.n, g.row_ptr)
    fl = (stm.STM_VERTEX_INDUCED if vi else 0) | stm.STM_AUTO_RESTRICT
    for i, e in enumerate(stm.stm_motif_catalog(k)):
        pg = stm.Plan(k, e, vertex_induced=vi, auto_order=True)
        gr = [int(x) for x in pg.describe().split("order=[")[1].split("]")[0].split(",")]
        # the unthresholded optimum: minimum over connected orders of the model cost
        best, bc = None, None
        import itertools
        for perm in itertools.permutations(range(k)):
            try:
                c, _ = stm.stm_order_cost(k, e, None, None, fl, st, list(perm))
            except stm.StmError:
                continue
            if bc is None or c < bc * (1 - 1e-9):
                best, bc = list(perm), c
        gc, _ = stm.stm_order_cost(k, e, None, None, fl, st, gr)
        if best == gr or bc >= gc * (1 - 1e-9):
            continue
        pc = stm.Plan(k, e, vertex_induced=vi, order=best)
        try:
            c1, t1 = best_of(G, pg)
            c2, t2 = best_of(G, pc)
        except stm.StmError as ex:
            print(f"{spec} motif {i:3d} pred {bc / gc:.3f} ERR {ex}", flush=True)
            continue
        assert c1 == c2
        print(f"{spec} motif {i:3d} pred {bc / gc:.3f} measured {t2 / t1:.3f}  greedy {t1 * 1e3:8.2f} ms  "
              f"cost {t2 * 1e3:8.2f} ms  count {c1}", flush=True)
    G.close()
