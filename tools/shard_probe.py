"""Scaling probe on ONE GPU: time each rank's share of the root space (stm_shard rank r of W,
own cursor only, no cross-GPU stealing) for W = 1, 2, 4, 8.  max over ranks approximates the
W-GPU step time without cross stealing; the counts of the W shares must sum to the total.
usage: python tools/shard_probe.py c5 k5,k6_minus_e [key=val tuning...]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import stmgen  # noqa: E402
from paper_conf_sc_weij22_b200 import stm  # noqa: E402

cfg, pats = sys.argv[1], sys.argv[2].split(",")
tk = dict(a.split("=") for a in sys.argv[3:] if "=" in a)
WS = tuple(int(x) for x in tk.pop("ws", "1,2,4,8").split(","))
g = stmgen.config_graph(cfg)
G = stm.Graph.from_stmgen(g)
t = stm.stm_tuning_default(**{k: int(v) for k, v in tk.items()})
cur = torch.zeros(64 * max(WS), dtype=torch.int64, device="cuda")
for name in pats:
    p = stmgen.CATALOG[name]
    plan = stm.Plan(p.k, p.edges, None)
    total = None
    t1 = None
    for W in WS:
        times, cnt = [], 0
        for r in range(W):
            ptrs = [None] * 8
            ptrs[r] = cur.data_ptr() + 64 * r  # own cursor only (no cross-GPU stealing)
            sh = stm.make_shard(r, W, 0, ptrs)  # chunk 0: the launch's root_chunk (as dist.py)
            best = 1e9
            for _ in range(2):
                cur.zero_()
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                c = stm.stm_match_count_ex(G.handle, plan.handle, t, sh)
                best = min(best, time.perf_counter() - t0)
            times.append(best)
            cnt += c
            if r == 0 and W > 1 and os.environ.get("STM_LIB_PATH", "").endswith("prof.so"):
                prof = stm.stm_last_profile()
                tl = prof["timeline_busy_warps"]
                last = max([i for i, x in enumerate(tl) if x > 0] or [0])
                print(f"   W={W} rank 0 busy warps per 0.5 ms: " + " ".join(f"{x:.0f}" for x in tl[:last + 1]), flush=True)
                print(f"   tail: cursors dry at max {prof['tail']['max_dry'] / 1.9e6:.2f} ms, "
                      f"indivisible {prof['max_task_cycles'] / 1.9e6:.2f} ms", flush=True)
        if total is None:
            total, t1 = cnt, max(times)
        ok = "ok" if cnt == total else f"MISMATCH {cnt} != {total}"
        print(f"{cfg}:{name} W={W} max {max(times) * 1e3:8.2f} ms  min {min(times) * 1e3:8.2f} ms  "
              f"speedup {t1 / max(times):5.2f} (ideal {W})  count {ok}", flush=True)
