#!/usr/bin/env python3
"""Benchmark of the STMatch counting hot path on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--workload c5|c2|...]

One *step* is one pass of the whole hot path over the workload: every query of the
workload counted once on the (already device-resident) graph -- root partition,
one persistent kernel per query, and (N > 1) the NCCL all-reduce of the per-rank
partial counts.  `value` = matches counted per second over the whole job
(BASELINE.json metric: query time and matches/s per pattern x graph).

Workload: BASELINE.json configs[4] -- the config the
metric is quoted on at 1/2/4/8 B200 -- a LiveJournal-shaped R-MAT (scale 23, 46M
edge draws, isolated vertices compacted) with the 5-clique and a size-6 pattern,
edge-induced, unlabeled, complete symmetry-breaking restrictions.  The graph
(~368 MB CSR) is larger than the 126 MB L2, which is how L2 reuse across steps is
excluded (an L2 flush is also written between steps).

--impl reference times the oracle (oracle/, the plain CPU backtracking matcher)
on a bounded sample of roots of the same workload: there is no runnable reference
implementation.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

WORKLOADS = {
    # name: (config graph, [(pattern, vertex_induced, labels)], description)
    "c5": ("c5", [("k5", False, None), ("k6_minus_e", False, None)],
           "configs[4]: 5-clique + K6-e (size 6) on LiveJournal-shaped R-MAT s23 (5.45M v, 46M e)"),
    "c2": ("c2", [("k4", False, None), ("c4", False, None)],
           "configs[1]: 4-clique + 4-cycle on R-MAT s16 (65k v, 0.9M e)"),
    "c3": ("c3", [("k5", False, None), ("house", False, None), ("c5", False, None)],
           "configs[2]: 5-clique, house, 5-cycle on com-Youtube-shaped Chung-Lu (1.13M v, 3M e)"),
    "c4": ("c4", [("k6_minus_e", False, (0, 1, 2, 3, 4, 5)), ("w5", False, (0, 1, 1, 2, 2, 3))],
           "configs[3]: labeled size-6 patterns (8 labels) on MiCo-shaped R-MAT s17"),
    "c1": ("c1", [("triangle", False, None)], "configs[0]: triangles on ER(1000, 10k)"),
}


def log(msg):
    print(f"[bench] {msg}", file=sys.stderr, flush=True)


def env_int(name, default):
    try:
        return int(os.environ.get(name, default))
    except ValueError:
        return default


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.lines:
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


# ---------------------------------------------------------------- oracle baseline
def oracle_sample(g, queries, plans, budget_s: float, seed: int = 0):
    """Time the oracle (as it stands) on a bounded random sample of roots."""
    import oracle
    import stmgen
    threads = os.cpu_count() or 1
    rng = np.random.default_rng(seed)
    per_q_budget = budget_s / max(1, len(queries))
    tot_matches, tot_time, roots_used = 0, 0.0, []
    for (pname, vi, lab), plan in zip(queries, plans):
        p = stmgen.CATALOG[pname]
        R = oracle.gk_restrictions(p.k, p.edges, lab)
        size = max(16, g.n // 20000)
        spent = 0.0
        while True:
            roots = np.sort(rng.choice(g.n, size=min(size, g.n), replace=False))
            t = time.perf_counter()
            c = oracle.count(g, p.k, p.edges, plabels=lab, vertex_induced=vi, restrictions=R,
                             root_u=plan.first_vertex, roots=roots, threads=threads)
            dt = time.perf_counter() - t
            spent += dt
            if dt >= per_q_budget / 4 or size >= g.n or spent >= per_q_budget:
                tot_matches += c
                tot_time += dt
                roots_used.append(int(roots.size))
                break
            size = min(g.n, size * 4)
    return {"value": tot_matches / tot_time if tot_time > 0 else None, "unit": "matches/s", "cores": threads,
            "kind": "oracle", "matches": int(tot_matches), "seconds": round(tot_time, 3),
            "sample": f"uniform random sample of {roots_used} roots (of {g.n}) per query, seeded; "
                      f"matches attributed to f(order[0]) as on the GPU"}


# ---------------------------------------------------------------- reference arm
def run_reference(args):
    rank = env_int("RANK", 0)
    if rank != 0:
        return
    import stmgen
    from types import SimpleNamespace
    cfg, queries, desc = WORKLOADS[args.workload]
    g = stmgen.config_graph(cfg)
    # the oracle's own root vertex choice is irrelevant for a sample; use pattern vertex 0
    plans = [SimpleNamespace(first_vertex=0) for _ in queries]
    for _ in range(args.warmup):
        oracle_sample(g, queries, plans, budget_s=2.0, seed=99)
    vals, secs = [], []
    for s in range(args.steps):
        r = oracle_sample(g, queries, plans, budget_s=args.ref_step_budget, seed=s)
        vals.append(r)
        secs.append(r["seconds"])
    matches = sum(r["matches"] for r in vals)
    t = sum(secs)
    value = matches / t if t else None
    line = {"impl": "reference", "metric": "query time (s) and matches/s per pattern×graph at 1/2/4/8 B200",
            "value": value, "unit": "matches/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000.0 * t / max(1, args.steps), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": desc, "graph": cfg, "queries": [q[0] for q in queries],
                       "mode": "edge-induced", "restrictions": "auto (GK)"},
            "cpu_baseline": {"value": value, "unit": "matches/s", "cores": vals[0]["cores"], "kind": "oracle",
                             "sample": vals[0]["sample"]},
            "e2e": {"value": value, "unit": "matches/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default=os.environ.get("STM_BENCH_WORKLOAD", "c5"), choices=sorted(WORKLOADS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=20.0)
    ap.add_argument("--ref-step-budget", type=float, default=15.0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cross-steal", action="store_true")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl == "ours" else args.warmup
    if args.impl == "reference":
        run_reference(args)
        return

    import torch
    import torch.distributed as dist
    import stmgen
    from paper_conf_sc_weij22_b200 import stm, dist as sdist

    world = env_int("WORLD_SIZE", 1)
    rank = env_int("RANK", 0)
    local = env_int("LOCAL_RANK", 0)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("nccl", device_id=dev)

    cfg, queries, desc = WORKLOADS[args.workload]
    t_start = time.time()
    g = stmgen.config_graph(cfg)
    log(f"graph {cfg} generated in {time.time() - t_start:.1f}s (n={g.n}, nnz={g.row_ptr[-1]})")
    G = stm.Graph.from_stmgen(g, device=local)
    log(f"graph loaded ({time.time() - t_start:.1f}s)")
    plans = [stm.Plan(stmgen.CATALOG[p].k, stmgen.CATALOG[p].edges, lab, vertex_induced=vi)
             for p, vi, lab in queries]
    stream = torch.cuda.current_stream(dev)
    sp = stream.cuda_stream
    tuning = stm.stm_tuning_default()
    layer = sdist.MultiGPUCounter(G, tuning=tuning, rank=rank, world=world, device=dev,
                                  cross_steal=not args.no_cross_steal)

    # ---- reference counts + algorithmic bytes (one instrumented, untimed launch per query)
    counts, alg, merge, jobs, idle, ranked = [], [], [], [], [], []
    for pl in plans:
        c, info = layer.count_instrumented(pl)
        counts.append(c)
        alg.append(info["alg_bytes"])
        merge.append(info["merge_bytes"])
        jobs.append(info["jobs"])
        idle.append(info["idle_cycles"] / info["warp_cycles"] if info["warp_cycles"] else None)
        ranked.append(bool(info["ranked"]))

    log(f"instrumented launches done ({time.time() - t_start:.1f}s): counts {counts}")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    d_counts = torch.zeros(len(plans), dtype=torch.int64, device=dev)

    def step(timed_events=None):
        for qi, pl in enumerate(plans):
            if timed_events is not None:
                timed_events[qi][0].record(stream)
            layer.count_async(pl, d_counts[qi:qi + 1])
            if timed_events is not None:
                timed_events[qi][1].record(stream)
        layer.reduce_counts(d_counts)

    for _ in range(args.warmup):
        flush.fill_(1)
        step()
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()

    step_ms, launch_ms = [], [[] for _ in plans]
    with ClockSampler(local) as clk:
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
        for s in range(args.steps):
            flush.fill_(s & 0xFF)  # L2 flush between timed steps (not timed)
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in plans]
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            step(ev)
            e1.record(stream)
            e1.synchronize()
            step_ms.append(e0.elapsed_time(e1))
            for qi in range(len(plans)):
                launch_ms[qi].append(ev[qi][0].elapsed_time(ev[qi][1]))
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()
    got = [int(x) for x in d_counts.cpu().tolist()]
    for qi in range(len(plans)):
        if (got[qi] & ((1 << 64) - 1)) != counts[qi]:
            raise SystemExit(f"count mismatch between timed and reference runs for query {qi}: {got[qi]} vs {counts[qi]}")
    total_ms = float(sum(step_ms))
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    matches_per_step = sum(counts)
    value = matches_per_step * args.steps / (total_ms / 1000.0)

    # ---- roofline of the dominant kernel (the query launch with the largest mean time):
    # its algorithmic bytes W (one instrumented launch) / its mean
    # CUDA-event launch time over the timed steps
    import json as _json
    peaks_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    peak, peak_src = 6650.0, "fallback (B200_PROFILING.md)"
    if os.path.exists(peaks_path):
        pk = _json.load(open(peaks_path))
        peak = float(pk.get("hbm_gbs_sustained", pk["hbm_gbs"]))
        peak_src = "measured (MEASURED_PEAKS.json " + ("hbm_gbs_sustained" if "hbm_gbs_sustained" in pk else "hbm_gbs") + ")"
    avg_launch_s = [statistics.mean(x) / 1000.0 for x in launch_ms]
    dom = max(range(len(plans)), key=lambda i: avg_launch_s[i])
    W_step = float(sum(alg))
    achieved = alg[dom] / avg_launch_s[dom] / 1e9
    traffic, traffic_src, ncu_ev = None, None, None
    prof = os.path.join(ROOT, "profiles", f"ncu_traffic_{args.workload}_{queries[dom][0]}.json")
    if os.path.exists(prof):
        try:
            pj = _json.load(open(prof))
            traffic, traffic_src = pj.get("dram_bytes_per_launch"), os.path.relpath(prof, ROOT)
            ncu_ev = {k: pj[k] for k in ("warp_execution_efficiency", "dram_read_gbs", "l2_gbs", "l1_hit_pct",
                                         "l2_hit_pct", "warps_active_pct") if k in pj}
        except Exception:
            traffic = None

    # ---- end-to-end through the public API from pinned host buffers
    e2e = None
    if not args.no_e2e:
        e2e = layer.e2e(g, plans, steps=max(1, min(args.steps, 3)))
        e2e["value"] = matches_per_step / e2e.pop("seconds_per_step")
        e2e["unit"] = "matches/s"

    log(f"timed + e2e done ({time.time() - t_start:.1f}s)")
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = oracle_sample(g, queries, plans, budget_s=args.cpu_budget)

    if rank == 0:
        per_q = []
        for qi, (p, vi, lab) in enumerate(queries):
            tq = statistics.mean(launch_ms[qi]) / 1000.0
            per_q.append({"pattern": p, "mode": "vertex" if vi else "edge", "labels": lab, "count": counts[qi],
                          "query_time_s": round(tq, 6), "matches_per_s": counts[qi] / tq if tq else None,
                          "alg_bytes": alg[qi], "merge_bytes": merge[qi], "set_ops": jobs[qi],
                          "idle_steal_fraction": idle[qi], "degree_ranked": ranked[qi]})
        info = stm.stm_last_launch()
        line = {
            "metric": "query time (s) and matches/s per pattern×graph at 1/2/4/8 B200",
            "value": value, "unit": "matches/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "int32", "data": "synthetic",
            "config": {"workload": desc, "graph": cfg, "n": g.n, "m": g.m, "max_degree": int(g.degrees().max()),
                       "queries": [q[0] for q in queries], "mode": "edge-induced", "restrictions": "auto (GK)",
                       "parallelism": f"root-partition x{world}" + ("" if world == 1 else " + cross-GPU stealing"),
                       "l2": "inputs (368 MB CSR) larger than L2 + 256 MB L2 flush between steps",
                       "grid": info["grid"], "block_threads": info["block_threads"]},
            "per_query": per_q,
            "gpu_launches": args.steps * len(plans),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "traffic_source": traffic_src,
                         "ncu": ncu_ev,
                         "kernel": ("stm_count_kernel_occ" if info.get("variant") == 2 else "stm_count_kernel")
                                   + f" ({queries[dom][0]} launch, unroll {info.get('unroll')})",
                         "algorithmic_bytes_per_launch": alg[dom], "algorithmic_bytes_per_step": W_step,
                         "peak_source": peak_src,
                         "note": "achieved = SURVEY.md 8(d) W of the dominant launch (instrumented launch) / "
                                 "its mean CUDA-event launch time; traffic = ncu dram read+write bytes of "
                                 "that launch (--set full capture, committed under profiles/)"},
            "clocks": clk.summary(),
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
