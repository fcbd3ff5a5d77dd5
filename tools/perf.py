"""Min-of-N timing of single queries through the C ABI: python tools/perf.py c2:k4,c2:c4,c5:k5 [key=val tuning...]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import stmgen
from paper_conf_sc_weij22_b200 import stm
specs = sys.argv[1].split(",")
tk = dict(a.split("=") for a in sys.argv[2:] if "=" in a)
reps = int(tk.pop("reps", 3))
tk.setdefault("watchdog_ms", "60000")  # failure detection: a hung launch reports STM_ETIMEOUT
graphs = {}
for spec in specs:
    cfg, name = spec.split(":")[:2]
    vi = ":vi" in spec
    nocm = ":nocm" in spec
    lazy = ":lazy" in spec
    cost = ":cost" in spec  # cost-based matching order (stm_order_optimize, NEXT-2)
    if cfg not in graphs:
        g = stmgen.config_graph(cfg)
        graphs[cfg] = (g, stm.Graph.from_stmgen(g))
    g, G = graphs[cfg]
    p = stmgen.CATALOG[name]
    lab = stmgen.pattern_labels(p.k, 8, 7) if g.labels is not None else None
    stats = stm.stm_graph_stats_host(g.n, g.row_ptr, g.labels) if cost else None
    plan = stm.Plan(p.k, p.edges, lab, vertex_induced=vi, code_motion=not nocm, lazy_unbounded=lazy,
                    cost_stats=stats)
    if cost:
        print(f"   {spec}: model cost {plan.model_cost:.3e}, est count {plan.model_count:.3e}, "
              + plan.describe().split(chr(10))[0], flush=True)
    t = stm.stm_tuning_default(**{k: int(v) for k, v in tk.items()})
    best = 1e9
    try:
        for _ in range(reps):
            t0 = time.perf_counter(); c = stm.count(G, plan, t); best = min(best, time.perf_counter() - t0)
        info = stm.stm_last_launch()
        prof = stm.stm_last_profile()
        if prof["lifetime_cycles"]:
            L = prof.pop("lifetime_cycles")
            tail = prof.pop("tail")
            lv = prof.pop("levels")
            mt = prof.pop("max_task_cycles")
            tl = prof.pop("timeline_busy_warps")
            last = max([i for i, x in enumerate(tl) if x > 0] or [0])
            print("   busy warps per 0.5 ms: " + " ".join(f"{x:.0f}" for x in tl[:last + 1]), flush=True)
            print(f"   longest busy interval between work-sharing checks (indivisible unit): {mt / 1.9e6:.2f} ms", flush=True)
            nw = info["grid"] * info["block_threads"] // 32
            print(f"   tail: mean lifetime {L / nw / 1.9e6:.2f} ms, max {tail['max_lifetime'] / 1.9e6:.2f} ms, "
                  f"cursors dry at mean {tail['sum_dry'] / nw / 1.9e6:.2f} ms / max {tail['max_dry'] / 1.9e6:.2f} ms "
                  f"(1.9 GHz)", flush=True)
            print("   profile: " + "  ".join(f"{k}={100.0 * v['cycles'] / L:.1f}%/{v['calls']}/{v['items']}"
                                           for k, v in prof.items() if v["calls"]), flush=True)
            print("   levels: " + "  ".join(f"{k}={100.0 * v['cycles'] / L:.1f}%/{v['ops']}/{v['elements']}"
                                          for k, v in lv.items()), flush=True)
        print(f"{spec:16} {tk} count {c:>16} best {best*1e3:9.2f} ms  {c/best:.3e} m/s  ls={info['local_steals']} gs={info['global_steals']} grid={info['grid']} smem={info['smem_bytes']}", flush=True)
    except Exception as e:
        print(f"{spec:16} {tk} ERR {e}", flush=True)
