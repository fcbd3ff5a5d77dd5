#!/usr/bin/env python3
"""Benchmark of the STMatch counting hot path on B200 (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--workload c5|c2|...]

One *step* is one pass of the whole hot path over the workload: every query of the
workload counted once on the (already device-resident) graph -- root partition,
one persistent kernel per query, and (N > 1) the all-reduce of the per-rank
partial counts.  `value` = matches counted per second over the whole job
(BASELINE.json metric: query time and matches/s per pattern x graph).

Workload: BASELINE.json configs[4] -- the config the
metric is quoted on at 1/2/4/8 B200 -- a LiveJournal-shaped R-MAT (scale 23, 46M
edge draws, isolated vertices compacted) with the 5-clique and a size-6 pattern,
edge-induced, unlabeled, complete symmetry-breaking restrictions.  The graph
(~368 MB CSR) is larger than the 126 MB L2 (an L2 flush is also written between
steps).  Every timed count is checked against the ORACLE's stored full-graph count
(tests/golden/config_counts.json, written by tools/make_golden.py): "parity":
"golden" per query.  At N = 1 the line also carries `per_config`: the queries of
configs[0..3] timed the same way, each checked against its golden count.

--impl reference times the oracle (oracle/, the plain CPU backtracking matcher) on
the same deterministic, degree-stratified root sample the `cpu_baseline` leg uses:
there is no runnable reference implementation.
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

METRIC = "query time (s) and matches/s per pattern×graph at 1/2/4/8 B200"
WORKLOADS = {
    # name: (config graph, [(pattern, vertex_induced, labels)], description)
    "c5": ("c5", [("k5", False, None), ("k6_minus_e", False, None)],
           "configs[4]: 5-clique + K6-e (size 6) on LiveJournal-shaped R-MAT s23 (5.45M v, 46M e)"),
    "c2": ("c2", [("k4", False, None), ("c4", False, None)],
           "configs[1]: 4-clique + 4-cycle on R-MAT s16 (65k v, 0.9M e)"),
    "c3": ("c3", [("k5", False, None), ("c5", False, None)],
           "configs[2]: 5-clique, 5-cycle on com-Youtube-shaped Chung-Lu (1.13M v, 3M e)"),
    "c4": ("c4", [("c6", False, (0, 1, 2, 0, 1, 2)), ("c7", False, (0, 1, 2, 3, 0, 1, 2))],
           "configs[3]: labeled size-6/7 patterns (8 labels) on MiCo-shaped R-MAT s17"),
    "c1": ("c1", [("triangle", False, None)], "configs[0]: triangles on ER(1000, 10k)"),
}
# per_config block (N = 1): configs[0..3], every query with an oracle golden count
PER_CONFIG = [
    ("c1", "triangle", False, None),
    ("c2", "k4", False, None), ("c2", "c4", False, None), ("c2", "c4", True, None),
    ("c3", "k5", False, None), ("c3", "k5", True, None), ("c3", "c5", False, None),
    ("c4", "c6", False, (0, 1, 2, 0, 1, 2)), ("c4", "c6", False, (0, 1, 2, 3, 4, 5)),
    ("c4", "c6", True, (0, 1, 2, 0, 1, 2)), ("c4", "c7", True, (0, 1, 2, 3, 0, 1, 2)),
]
# The oracle counts K6-e through an isomorphic labelling whose non-adjacent pair is (4, 5):
# its own BFS order then starts with the K4 (0, 1, 2, 3) instead of enumerating the
# non-adjacent pair from a degree-5 vertex.  Same pattern, same count of distinct
# subgraphs (GK restrictions of the relabelled pattern; tests/test_oracle.py pins
# relabel/order invariance); tools/make_golden.py uses the same edge list.
ORACLE_EDGES = {"k6_minus_e": tuple((i, j) for i in range(6) for j in range(i + 1, 6) if (i, j) != (4, 5))}
GOLDEN = os.path.join(ROOT, "tests", "golden", "config_counts.json")


def log(msg):
    print(f"[bench] {msg}", file=sys.stderr, flush=True)


def env_int(name, default):
    try:
        return int(os.environ.get(name, default))
    except ValueError:
        return default


def golden_count(cfg, fingerprint, pname, vi, labels):
    """The oracle's stored full-graph count for this exact query and graph, or None."""
    if not os.path.exists(GOLDEN):
        return None
    for d in json.load(open(GOLDEN)).values():
        if (d["config"] == cfg and d["pattern"] == pname and bool(d["vertex_induced"]) == bool(vi)
                and (d["labels"] or None) == (list(labels) if labels else None)):
            if d["fingerprint"] != fingerprint:
                raise SystemExit(f"golden {cfg}/{pname}: graph fingerprint mismatch")
            return int(d["count"])
    return None


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """SM clocks and throttle reasons sampled DURING the timed region: NVML polled every 2 ms by
    a thread (a 5-step region lasts only ~0.25 s, too short for `nvidia-smi -lms`, whose first
    line arrives after it); `nvidia-smi -lms 100` only if NVML is unavailable."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.proc = None
        self.lines = []
        self.samples = []  # (sm_mhz, max_mhz, reasons) from NVML
        self.stop = threading.Event()
        self.t = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.gpu)
            bits = {"hw_slowdown": pynvml.nvmlClocksEventReasonHwSlowdown,
                    "hw_thermal_slowdown": pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                    "sw_thermal_slowdown": pynvml.nvmlClocksEventReasonSwThermalSlowdown,
                    "sw_power_cap": pynvml.nvmlClocksEventReasonSwPowerCap}
            mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)

            def poll():
                while not self.stop.is_set():
                    sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                    r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                    self.samples.append((float(sm), float(mx), {n for n, b in bits.items() if r & b}))
                    self.stop.wait(0.002)
            self.t = threading.Thread(target=poll, daemon=True)
            self.t.start()
            return self
        except Exception:
            self.samples = []
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
        self.stop.set()
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        elif self.t:
            self.t.join(timeout=1)

    def summary(self):
        sm, mx, reasons = [], [], set()
        for a, b, r in self.samples:
            sm.append(a)
            mx.append(b)
            reasons |= r
        for line in self.lines:
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(self.NAMES, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm), "source": "nvml" if self.samples else "nvidia-smi"}


# ---------------------------------------------------------------- oracle baseline
def degree_ranked(g):
    """g renumbered in (degree, id) order -- the numbering the GPU counts order-free plans on."""
    import stmgen
    deg = g.degrees()
    rank2orig = np.lexsort((np.arange(g.n), deg))
    perm = np.empty(g.n, np.int64)
    perm[rank2orig] = np.arange(g.n)
    return stmgen.permute(g, perm)


SAMPLE_SIZES = (1024, 16, 2, 2)


def stratified_sample(n, seed=2024):
    """Deterministic degree-stratified root sample of a degree-ranked graph (vertex i = i-th
    lowest degree): strata of ranks [0, n-4096), [n-4096, n-256), [n-256, n-16), [n-16, n)
    -- the 16 highest-degree hubs are their own stratum -- with fixed sample sizes
    SAMPLE_SIZES.  Returns [(stratum size N_s, sampled root ids)]."""
    rng = np.random.default_rng(seed)
    cuts = [0, max(0, n - 4096), max(0, n - 256), max(0, n - 16), n]
    out = []
    for (a, b), k in zip(zip(cuts[:-1], cuts[1:]), SAMPLE_SIZES):
        if b <= a:
            continue
        take = np.sort(rng.choice(np.arange(a, b), size=min(k, b - a), replace=False))
        out.append((b - a, take))
    return out


def oracle_baseline(gr, queries, cores=None, seed=2024, parts=1, part=0):
    """The oracle (as it stands) on the deterministic stratified root sample of the same
    workload, timed on the host cores.  Every sampled root is one single-threaded oracle call
    (part `part` of `parts`: every parts-th root of each stratum, so that `parts` calls cover
    the sample once; the light bulk in groups of 64 roots), run `cores` at a time; its wall
    time is those roots' CPU time.  The
    whole-workload throughput is the stratified ratio estimate
    sum_s (N_s/n_s) m_s / (sum_s (N_s/n_s) sum_r t_r / C)  (m_s matches of stratum s, t_r the
    time of root r, C = cores): independent of how the sample is split into calls, so both
    bench arms measure the same quantity on the same roots."""
    import oracle
    import stmgen
    from concurrent.futures import ThreadPoolExecutor
    cores = cores or os.cpu_count() or 1
    strata = stratified_sample(gr.n, seed)
    tasks = []
    for qi, (pname, vi, lab) in enumerate(queries):
        p = stmgen.CATALOG[pname]
        edges = ORACLE_EDGES.get(pname, p.edges)
        R = oracle.gk_restrictions(p.k, edges, lab)
        for si, (N_s, roots_all) in enumerate(strata):
            mine = roots_all[part::parts]
            step = 64 if si == 0 else 1  # the light bulk in groups of 64 roots (call overhead)
            for i in range(0, mine.size, step):
                tasks.append((qi, si, p.k, edges, lab, vi, R, mine[i:i + step]))

    def one(task):
        qi, si, k, edges, lab, vi, R, roots = task
        t = time.perf_counter()
        m = oracle.count(gr, k, edges, plabels=lab, vertex_induced=vi, restrictions=R,
                         roots=np.ascontiguousarray(roots, np.int64), threads=1)
        return qi, si, m, time.perf_counter() - t, roots.size

    t_wall = time.perf_counter()
    with ThreadPoolExecutor(max_workers=cores) as ex:  # (ctypes releases the GIL in the oracle)
        res = list(ex.map(one, tasks))
    t_wall = time.perf_counter() - t_wall
    acc = {}
    for qi, si, m, dt, nr in res:
        a = acc.setdefault((qi, si), [0, 0.0, 0])
        a[0] += m
        a[1] += dt
        a[2] += nr
    M = T = 0.0
    raw_m, detail = 0, []
    for (qi, si), (m, dt, nr) in sorted(acc.items()):
        N_s, roots_all = strata[si]
        w = N_s / roots_all.size
        M += w * m
        T += w * dt / cores
        raw_m += m
        detail.append([queries[qi][0], int(N_s), int(nr), int(m), round(dt, 4)])
    return {"value": M / T if T > 0 else None, "unit": "matches/s", "cores": cores, "kind": "oracle",
            "sample_matches": raw_m, "sample_seconds": round(t_wall, 3), "est_matches": M, "est_seconds": T,
            "strata": detail,
            "sample": f"deterministic degree-stratified root sample (seed {seed}) of the degree-ranked graph: "
                      f"{SAMPLE_SIZES[0]} roots of the low-degree bulk, {SAMPLE_SIZES[1]} of ranks n-4096..n-256, "
                      f"{SAMPLE_SIZES[2]} of n-256..n-16, {SAMPLE_SIZES[3]} of the 16 top hubs, per query; one "
                      f"single-threaded oracle call per root (bulk: per 64 roots), {cores} at a time; stratified "
                      "ratio estimate of "
                      "whole-workload matches/s from the per-root times (bench.py oracle_baseline)"}


# ---------------------------------------------------------------- reference arm
def run_reference(args):
    rank = env_int("RANK", 0)
    if rank != 0:
        return
    import stmgen
    cfg, queries, desc = WORKLOADS[args.workload]
    gr = degree_ranked(stmgen.config_graph(cfg))
    for _ in range(args.warmup):  # warm-up: a small slice of the bulk stratum
        oracle_baseline(gr, queries[:1], parts=64, part=0)
    # the K steps together cover the deterministic sample exactly once (step i times the
    # i-th slice of every stratum), so the run stays within minutes for any K
    vals = [oracle_baseline(gr, queries, parts=args.steps, part=i) for i in range(args.steps)]
    est_m = sum(v["est_matches"] for v in vals)
    est_t = sum(v["est_seconds"] for v in vals)
    value = est_m / est_t if est_t else None
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "matches/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000.0 * sum(v["sample_seconds"] for v in vals) / max(1, args.steps),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic",
            "config": {"workload": desc, "graph": cfg, "queries": [q[0] for q in queries],
                       "mode": "edge-induced", "restrictions": "auto (GK)"},
            "cpu_baseline": {"value": value, "unit": "matches/s", "cores": vals[0]["cores"], "kind": "oracle",
                             "sample": vals[0]["sample"] + f"; split over the {args.steps} timed steps",
                             "sample_matches": sum(v["sample_matches"] for v in vals),
                             "sample_seconds": round(sum(v["sample_seconds"] for v in vals), 3)},
            "e2e": {"value": value, "unit": "matches/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- per-config block
def per_config_block(dev, reps=3):
    """configs[0..3] at N = 1: each query counted (mean CUDA-event time of `reps` launches after
    one warm-up) and checked against its oracle golden count."""
    import torch
    import stmgen
    from paper_conf_sc_weij22_b200 import stm
    from paper_conf_sc_weij22_b200.dist import MultiGPUCounter
    out = []
    graphs = {}
    stream = torch.cuda.current_stream(dev)
    for cfg, pname, vi, lab in PER_CONFIG:
        if cfg not in graphs:
            graphs.clear()
            g = stmgen.config_graph(cfg)
            graphs[cfg] = (g, stm.Graph.from_stmgen(g, device=dev.index))
        g, G = graphs[cfg]
        p = stmgen.CATALOG[pname]
        plan = stm.Plan(p.k, p.edges, lab, vertex_induced=vi, graph=G)  # cost-based order from G's statistics
        layer = MultiGPUCounter(G, device=dev)
        d = layer.new_results(1)
        layer.count_async(plan, d[0])
        ms = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            layer.count_async(plan, d[0])
            e1.record(stream)
            e1.synchronize()
            ms.append(e0.elapsed_time(e1))
        c = layer.check(d)[0]
        want = golden_count(cfg, g.fingerprint(), pname, vi, lab)
        if want is not None and c != want:
            raise SystemExit(f"per_config {cfg}/{pname}/vi={vi}: count {c} != oracle golden {want}")
        t = statistics.mean(ms) / 1000.0
        out.append({"config": cfg, "pattern": pname, "mode": "vertex" if vi else "edge",
                    "labels": list(lab) if lab else None, "count": c, "query_time_s": round(t, 6),
                    "matches_per_s": c / t if t else None,
                    "parity": "golden" if want is not None else "no golden"})
        log(f"per_config {cfg} {pname} vi={vi}: {c} in {t * 1e3:.2f} ms ({out[-1]['parity']})")
    return out


# ---------------------------------------------------------------- our arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default=os.environ.get("STM_BENCH_WORKLOAD", "c5"), choices=sorted(WORKLOADS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-per-config", action="store_true")
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
    # compiled for the loaded graph: its statistics pick the cost-based order (NEXT-2)
    plans = [stm.Plan(stmgen.CATALOG[p].k, stmgen.CATALOG[p].edges, lab, vertex_induced=vi, graph=G)
             for p, vi, lab in queries]
    stream = torch.cuda.current_stream(dev)
    tuning = stm.stm_tuning_default()
    layer = sdist.MultiGPUCounter(G, tuning=tuning, rank=rank, world=world, device=dev,
                                  cross_steal=not args.no_cross_steal)
    goldens = [golden_count(cfg, g.fingerprint(), p, vi, lab) for p, vi, lab in queries]

    # ---- algorithmic bytes (one instrumented, untimed launch per query)
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
    d_res = layer.new_results(len(plans))

    def step(timed_events=None):
        for qi, pl in enumerate(plans):
            if timed_events is not None:
                timed_events[qi][0].record(stream)
            layer.count_async(pl, d_res[qi])
            if timed_events is not None:
                timed_events[qi][1].record(stream)
        layer.reduce_counts(d_res)

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
    got = layer.check(d_res)  # raises if any rank's launch reported a failure status
    main_info = stm.stm_last_launch()  # the last timed launch (the workload's last query)
    parity = []
    for qi in range(len(plans)):
        if got[qi] != counts[qi]:
            raise SystemExit(f"query {qi}: timed count {got[qi]} != instrumented count {counts[qi]}")
        if goldens[qi] is not None and got[qi] != goldens[qi]:
            raise SystemExit(f"query {qi}: count {got[qi]} != oracle golden {goldens[qi]}")
        parity.append("golden" if goldens[qi] is not None else "no golden")
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
    peaks_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    peak, peak_src = 6650.0, "fallback (B200_PROFILING.md)"
    if os.path.exists(peaks_path):
        pk = json.load(open(peaks_path))
        key = "hbm_gbs_sustained" if "hbm_gbs_sustained" in pk else "hbm_gbs"
        peak = float(pk[key])
        peak_src = f"measured (MEASURED_PEAKS.json {key})"
    avg_launch_s = [statistics.mean(x) / 1000.0 for x in launch_ms]
    dom = max(range(len(plans)), key=lambda i: avg_launch_s[i])
    W_step = float(sum(alg))
    achieved = alg[dom] / avg_launch_s[dom] / 1e9
    traffic, traffic_src, ncu_ev = None, None, None
    prof = os.path.join(ROOT, "profiles", f"ncu_traffic_{args.workload}_{queries[dom][0]}.json")
    if os.path.exists(prof):
        try:
            pj = json.load(open(prof))
            traffic, traffic_src = pj.get("dram_bytes_per_launch"), os.path.relpath(prof, ROOT)
            ncu_ev = {k: pj[k] for k in ("warp_execution_efficiency", "dram_read_gbs", "l2_gbs", "l1_hit_pct",
                                         "l2_hit_pct", "warps_active_pct", "kernel_ms") if k in pj}
        except Exception:
            traffic = None

    # ---- end-to-end through the public API from host buffers
    e2e = None
    if not args.no_e2e:
        e2e = layer.e2e(g, plans, steps=2)
        if e2e.pop("counts") != counts:
            raise SystemExit("e2e counts differ from the timed counts")
        e2e["value"] = matches_per_step / e2e.pop("seconds_per_step")
        e2e["unit"] = "matches/s"
    log(f"timed + e2e done ({time.time() - t_start:.1f}s)")

    per_config = None
    if rank == 0 and world == 1 and not args.no_per_config:
        per_config = per_config_block(dev)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = oracle_baseline(degree_ranked(g), queries)
    log(f"done ({time.time() - t_start:.1f}s)")

    if rank == 0:
        per_q = []
        for qi, (p, vi, lab) in enumerate(queries):
            tq = statistics.mean(launch_ms[qi]) / 1000.0
            per_q.append({"pattern": p, "mode": "vertex" if vi else "edge", "labels": lab, "count": counts[qi],
                          "parity": parity[qi], "query_time_s": round(tq, 6),
                          "matches_per_s": counts[qi] / tq if tq else None,
                          "alg_bytes": alg[qi], "merge_bytes": merge[qi], "set_ops": jobs[qi],
                          "idle_steal_fraction": idle[qi], "degree_ranked": ranked[qi]})
        info = main_info
        line = {
            "metric": METRIC,
            "value": value, "unit": "matches/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "int32", "data": "synthetic",
            "config": {"workload": desc, "graph": cfg, "n": g.n, "m": g.m, "max_degree": int(g.degrees().max()),
                       "queries": [q[0] for q in queries], "mode": "edge-induced", "restrictions": "auto (GK)",
                       "parallelism": f"root-partition x{world}" + (
                           "" if world == 1 else (" + cross-GPU stealing (CUDA IPC cursors)" if layer.cross_steal
                                                  else " static (no cross-GPU stealing)")),
                       "cross_steal": layer.cross_steal if world > 1 else None,
                       "l2": "inputs (368 MB CSR) larger than L2 + 256 MB L2 flush between steps",
                       "grid": info["grid"], "block_threads": info["block_threads"]},
            "per_query": per_q,
            "gpu_launches": args.steps * len(plans),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "traffic_source": traffic_src,
                         "ncu": ncu_ev,
                         "kernel": ("stm_count_kernel_occ" if info.get("variant") == 2 else "stm_count_kernel")
                                   + f" ({queries[dom][0]} launch, unroll {info.get('unroll')}, "
                                   f"{'plan-specialised' if info.get('jit') else 'generic'} kernel)",
                         "algorithmic_bytes_per_launch": alg[dom], "algorithmic_bytes_per_step": W_step,
                         "peak_source": peak_src,
                         "note": "achieved = SURVEY.md 8(d) W of the dominant launch (instrumented launch) / "
                                 "its mean CUDA-event launch time; traffic = ncu dram read+write bytes of "
                                 "that launch (--set full capture, committed under profiles/)"},
            "clocks": clk.summary(),
            "e2e": e2e,
            "per_config": per_config,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    layer.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
