"""Thin ctypes binding over libstm.so (include/stm.h).  Argument marshalling only:
every step of the counting path runs inside the library's CUDA kernel.  There is
no CPU fallback: importing this module without the built library raises.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, fields
from typing import Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("STM_LIB_PATH") or os.path.join(_HERE, "libstm.so")  # override: A/B experiments only

STM_OK, STM_EINVAL, STM_ENOMEM, STM_ECUDA, STM_EUNSUPPORTED, STM_EOVERFLOW, STM_ETIMEOUT = range(7)
STM_EDGE_INDUCED, STM_VERTEX_INDUCED, STM_NO_CODE_MOTION, STM_AUTO_RESTRICT, STM_AUTO_ORDER = 0, 1, 2, 4, 8
STM_LAZY_UNBOUNDED = 16
STM_CENSUS_PER_MOTIF = 32
STM_DIRECTED = 64
_NAMES = {1: "STM_EINVAL", 2: "STM_ENOMEM", 3: "STM_ECUDA", 4: "STM_EUNSUPPORTED", 5: "STM_EOVERFLOW",
          6: "STM_ETIMEOUT"}
STM_IPC_HANDLE_BYTES = 64

EXPORTS = ["stm_match_list", "stm_graph_load", "stm_graph_load_device", "stm_graph_info", "stm_graph_free",
           "stm_pattern_compile", "stm_plan_describe", "stm_plan_info", "stm_plan_free",
           "stm_plan_first_vertex", "stm_tuning_default", "stm_match_count", "stm_match_count_ex",
           "stm_match_count_async", "stm_match_count_per_root", "stm_last_launch", "stm_last_profile", "stm_last_error",
           "stm_graph_stats_host", "stm_order_cost", "stm_order_optimize", "stm_motif_catalog",
           "stm_motif_census", "stm_cursors_alloc", "stm_cursors_open", "stm_cursors_close", "stm_cursors_free",
           "stm_cursors_reset", "stm_graph_get_stats", "stm_motif_census_launches", "stm_motif_merge_stats",
           "stm_plan_raw", "stm_graph_load_directed"]


class StmError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_NAMES.get(status, status)}: {msg}")
        self.status = status


class stm_tuning(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in ("local_steal", "global_steal", "stop_level", "detect_level",
                                               "unroll", "root_chunk", "block_warps", "blocks_per_sm",
                                               "instrument", "hash_slots", "vertex_order",
                                               "bitmap_min_degree", "bitmap_budget_mb", "occupancy", "root_order",
                                               "l2_persist_mb", "drive_ratio", "narrow_split", "watchdog_ms",
                                               "backoff_max", "carveout_pct", "root_split", "chunk_cost", "jit")]


class stm_shard(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("world", ctypes.c_int32), ("chunk", ctypes.c_int32),
                ("reserved", ctypes.c_int32), ("d_cursors", ctypes.c_void_p * 8)]


class stm_launch_info(ctypes.Structure):
    _fields_ = [("grid", ctypes.c_int32), ("block_threads", ctypes.c_int32), ("smem_bytes", ctypes.c_int32),
                ("cap", ctypes.c_int32), ("arena_bytes", ctypes.c_int64), ("local_steals", ctypes.c_int64),
                ("global_steals", ctypes.c_int64), ("chunks", ctypes.c_int64), ("alg_bytes", ctypes.c_int64),
                ("merge_bytes", ctypes.c_int64), ("jobs", ctypes.c_int64), ("ranked", ctypes.c_int32),
                ("jit", ctypes.c_int32), ("idle_cycles", ctypes.c_int64), ("warp_cycles", ctypes.c_int64),
                ("hubs", ctypes.c_int64), ("variant", ctypes.c_int32), ("unroll", ctypes.c_int32),
                ("peer_chunks", ctypes.c_int64)]


class stm_async_result(ctypes.Structure):
    """Device-side result record of stm_match_count_async (4 x uint64)."""
    _fields_ = [("count", ctypes.c_uint64), ("status", ctypes.c_uint64), ("chunks", ctypes.c_uint64),
                ("peer_chunks", ctypes.c_uint64)]


ASYNC_WORDS = 4  # uint64 words of stm_async_result


STM_STATS_MOMENTS, STM_STATS_LABELS = 9, 256


class stm_graph_stats(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("moment", ctypes.c_double * STM_STATS_MOMENTS),
                ("n_labels", ctypes.c_int32), ("reserved", ctypes.c_int32),
                ("label_value", ctypes.c_int32 * STM_STATS_LABELS),
                ("label_freq", ctypes.c_double * STM_STATS_LABELS)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_sc_weij22_b200.build` "
                          "(there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    vp, i32, i64, u32, sz = ctypes.c_void_p, ctypes.c_int, ctypes.c_int64, ctypes.c_uint32, ctypes.c_size_t
    P64 = ctypes.POINTER(ctypes.c_int64)
    sig = {
        "stm_graph_load": [i64, vp, vp, vp, i32, ctypes.POINTER(vp)],
        "stm_graph_load_directed": [i64, vp, vp, vp, i32, ctypes.POINTER(vp)],
        "stm_graph_load_device": [i64, i64, vp, vp, vp, i32, ctypes.POINTER(vp)],
        "stm_graph_info": [vp, P64, P64, P64],
        "stm_graph_free": [vp],
        "stm_pattern_compile": [i32, i32, vp, vp, vp, i32, vp, u32, ctypes.POINTER(vp)],
        "stm_plan_describe": [vp, ctypes.c_char_p, sz],
        "stm_plan_info": [vp, ctypes.POINTER(i32), ctypes.POINTER(i32), P64],
        "stm_plan_free": [vp],
        "stm_plan_raw": [vp, vp, sz, ctypes.POINTER(sz)],
        "stm_plan_first_vertex": [vp, ctypes.POINTER(i32)],
        "stm_match_count": [vp, vp, vp, ctypes.POINTER(ctypes.c_uint64)],
        "stm_match_count_ex": [vp, vp, vp, vp, vp, ctypes.POINTER(ctypes.c_uint64)],
        "stm_match_count_async": [vp, vp, vp, vp, vp, vp],
        "stm_match_count_per_root": [vp, vp, vp, vp, vp, ctypes.POINTER(ctypes.c_uint64)],
        "stm_match_list": [vp, vp, vp, i64, i64, vp, vp, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64),
                           ctypes.POINTER(ctypes.c_uint64)],
        "stm_last_launch": [ctypes.POINTER(stm_launch_info)],
        "stm_motif_catalog": [i32, i32, vp, vp, ctypes.POINTER(i32)],
        "stm_motif_census": [vp, i32, u32, vp, vp, vp, i32, vp, ctypes.POINTER(i32)],
        "stm_motif_census_launches": [ctypes.POINTER(i32)],
        "stm_motif_merge_stats": [i32, u32, vp, ctypes.POINTER(i32), ctypes.POINTER(i32)],
        "stm_graph_stats_host": [i64, vp, vp, ctypes.POINTER(stm_graph_stats)],
        "stm_graph_get_stats": [vp, ctypes.POINTER(stm_graph_stats)],
        "stm_cursors_alloc": [i32, i32, ctypes.POINTER(vp), vp],
        "stm_cursors_open": [i32, vp, ctypes.POINTER(vp)],
        "stm_cursors_close": [i32, vp],
        "stm_cursors_free": [i32, vp],
        "stm_cursors_reset": [i32, vp, i32, i32, vp],
        "stm_order_cost": [i32, i32, vp, vp, i32, vp, u32, ctypes.POINTER(stm_graph_stats), vp,
                           ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)],
        "stm_order_optimize": [i32, i32, vp, vp, i32, vp, u32, ctypes.POINTER(stm_graph_stats), vp,
                               ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)],
    }
    for name, args in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = ctypes.c_int
    lib.stm_tuning_default.argtypes = [ctypes.POINTER(stm_tuning)]
    lib.stm_tuning_default.restype = None
    lib.stm_last_error.argtypes = []
    lib.stm_last_error.restype = ctypes.c_char_p
    return lib


lib = _load()


def _check(status: int) -> None:
    if status != STM_OK:
        raise StmError(status, lib.stm_last_error().decode())


def _arr(a, dtype):
    return None if a is None else np.ascontiguousarray(np.asarray(a, dtype=dtype))


def _p(a):
    return None if a is None else a.ctypes.data


# ---------------------------------------------------------------- same-name wrappers
def stm_graph_load(n: int, row_ptr, col_idx, labels=None, device: int = 0) -> int:
    rp, ci, lb = _arr(row_ptr, np.int64), _arr(col_idx, np.int32), _arr(labels, np.int32)
    h = ctypes.c_void_p()
    _check(lib.stm_graph_load(n, _p(rp), _p(ci), _p(lb), device, ctypes.byref(h)))
    return h.value


def stm_graph_load_directed(n: int, row_ptr, col_idx, labels=None, device: int = 0) -> int:
    """Directed graph from its out-neighbour rows (NEXT-4)."""
    rp, ci, lb = _arr(row_ptr, np.int64), _arr(col_idx, np.int32), _arr(labels, np.int32)
    h = ctypes.c_void_p()
    _check(lib.stm_graph_load_directed(n, _p(rp), _p(ci), _p(lb), device, ctypes.byref(h)))
    return h.value


def stm_graph_load_device(n: int, nnz: int, d_row_ptr: int, d_col_idx: int, d_labels: Optional[int],
                          device: int = 0) -> int:
    h = ctypes.c_void_p()
    _check(lib.stm_graph_load_device(n, nnz, d_row_ptr, d_col_idx, d_labels, device, ctypes.byref(h)))
    return h.value


def stm_graph_info(g: int) -> Tuple[int, int, int]:
    n, nnz, md = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
    _check(lib.stm_graph_info(g, ctypes.byref(n), ctypes.byref(nnz), ctypes.byref(md)))
    return n.value, nnz.value, md.value


def stm_graph_free(g: int) -> None:
    _check(lib.stm_graph_free(g))


def stm_pattern_compile(k: int, edges, labels=None, order=None, restrictions=None, flags: int = 0) -> int:
    e = _arr(edges, np.int32).reshape(-1)
    lb = _arr(labels, np.int32)
    od = _arr(order, np.int32)
    rs = _arr(restrictions, np.int32).reshape(-1) if restrictions is not None and len(restrictions) else None
    nr = 0 if rs is None else rs.size // 2
    h = ctypes.c_void_p()
    _check(lib.stm_pattern_compile(k, e.size // 2, _p(e), _p(lb), _p(od), nr, _p(rs), flags, ctypes.byref(h)))
    return h.value


def stm_graph_stats_host(n: int, row_ptr, labels=None) -> stm_graph_stats:
    rp = _arr(row_ptr, np.int64)
    lb = _arr(labels, np.int32)
    st = stm_graph_stats()
    _check(lib.stm_graph_stats_host(n, _p(rp), _p(lb), ctypes.byref(st)))
    return st


def stm_graph_get_stats(g: int) -> stm_graph_stats:
    st = stm_graph_stats()
    _check(lib.stm_graph_get_stats(g, ctypes.byref(st)))
    return st


def _pattern_args(edges, labels, restrictions):
    e = _arr(edges, np.int32).reshape(-1)
    lb = _arr(labels, np.int32)
    rs = _arr(restrictions, np.int32).reshape(-1) if restrictions is not None and len(restrictions) else None
    return e, lb, rs, 0 if rs is None else rs.size // 2


def stm_order_cost(k: int, edges, labels, restrictions, flags: int, stats: stm_graph_stats,
                   order) -> Tuple[float, float]:
    e, lb, rs, nr = _pattern_args(edges, labels, restrictions)
    od = _arr(order, np.int32)
    c, est = ctypes.c_double(), ctypes.c_double()
    _check(lib.stm_order_cost(k, e.size // 2, _p(e), _p(lb), nr, _p(rs), flags, ctypes.byref(stats), _p(od),
                              ctypes.byref(c), ctypes.byref(est)))
    return c.value, est.value


def stm_order_optimize(k: int, edges, labels, restrictions, flags: int,
                       stats: stm_graph_stats) -> Tuple[list, float, float]:
    e, lb, rs, nr = _pattern_args(edges, labels, restrictions)
    od = np.zeros(k, np.int32)
    c, est = ctypes.c_double(), ctypes.c_double()
    _check(lib.stm_order_optimize(k, e.size // 2, _p(e), _p(lb), nr, _p(rs), flags, ctypes.byref(stats), _p(od),
                                  ctypes.byref(c), ctypes.byref(est)))
    return od.tolist(), c.value, est.value


def stm_motif_catalog(k: int) -> list:
    """[(n_edges, [(a, b), ...]), ...] in catalog order."""
    n = ctypes.c_int()
    _check(lib.stm_motif_catalog(k, 0, None, None, ctypes.byref(n)))
    ne = np.zeros(n.value, np.int32)
    ed = np.zeros(n.value * k * (k - 1), np.int32)
    _check(lib.stm_motif_catalog(k, n.value, _p(ne), _p(ed), ctypes.byref(n)))
    s = k * (k - 1)
    return [[(int(ed[i * s + 2 * e]), int(ed[i * s + 2 * e + 1])) for e in range(ne[i])] for i in range(n.value)]


def stm_motif_census(g: int, k: int, flags: int = 0, stats: Optional[stm_graph_stats] = None,
                     tuning: Optional[stm_tuning] = None, stream: Optional[int] = None) -> list:
    n = ctypes.c_int()
    cap = 112
    out = np.zeros(cap, np.uint64)
    sp = None if stats is None else ctypes.cast(ctypes.pointer(stats), ctypes.c_void_p)
    _check(lib.stm_motif_census(g, k, flags, sp, _tp(tuning), stream, cap, _p(out), ctypes.byref(n)))
    return [int(x) for x in out[: n.value]]


def stm_motif_census_launches() -> int:
    n = ctypes.c_int()
    _check(lib.stm_motif_census_launches(ctypes.byref(n)))
    return n.value


def stm_motif_merge_stats(k: int, flags: int = 0) -> dict:
    per = np.zeros(k, np.int32)
    nn, nr = ctypes.c_int(), ctypes.c_int()
    _check(lib.stm_motif_merge_stats(k, flags, _p(per), ctypes.byref(nn), ctypes.byref(nr)))
    return {"verts_per_depth": per.tolist(), "pool_nodes": nn.value, "regions": nr.value}


def stm_plan_describe(p: int) -> str:
    buf = ctypes.create_string_buffer(1 << 16)
    _check(lib.stm_plan_describe(p, buf, len(buf)))
    return buf.value.decode()


def stm_plan_info(p: int) -> Tuple[int, int, int]:
    k, ns, aut = ctypes.c_int(), ctypes.c_int(), ctypes.c_int64()
    _check(lib.stm_plan_info(p, ctypes.byref(k), ctypes.byref(ns), ctypes.byref(aut)))
    return k.value, ns.value, aut.value


def stm_plan_first_vertex(p: int) -> int:
    u = ctypes.c_int()
    _check(lib.stm_plan_first_vertex(p, ctypes.byref(u)))
    return u.value


def stm_plan_raw(p: int) -> bytes:
    """The compiled device plan record (plan.h StmPlan) as bytes."""
    n = ctypes.c_size_t()
    _check(lib.stm_plan_raw(p, None, 0, ctypes.byref(n)))
    buf = ctypes.create_string_buffer(n.value)
    _check(lib.stm_plan_raw(p, buf, n.value, ctypes.byref(n)))
    return buf.raw


def stm_plan_free(p: int) -> None:
    _check(lib.stm_plan_free(p))


def stm_tuning_default(**overrides) -> stm_tuning:
    t = stm_tuning()
    lib.stm_tuning_default(ctypes.byref(t))
    for k, v in overrides.items():
        setattr(t, k, int(v))
    return t


def _tp(t: Optional[stm_tuning]):
    return None if t is None else ctypes.cast(ctypes.pointer(t), ctypes.c_void_p)


def make_shard(rank: int, world: int, chunk: int, cursor_ptrs: Sequence[Optional[int]]) -> stm_shard:
    s = stm_shard()
    s.rank, s.world, s.chunk = rank, world, chunk
    for i, p in enumerate(cursor_ptrs):
        s.d_cursors[i] = p
    return s


def stm_match_count(g: int, p: int, stream: Optional[int] = None) -> int:
    c = ctypes.c_uint64()
    _check(lib.stm_match_count(g, p, stream, ctypes.byref(c)))
    return c.value


def stm_match_count_ex(g: int, p: int, tuning: Optional[stm_tuning] = None, shard: Optional[stm_shard] = None,
                       stream: Optional[int] = None) -> int:
    c = ctypes.c_uint64()
    sp = None if shard is None else ctypes.cast(ctypes.pointer(shard), ctypes.c_void_p)
    _check(lib.stm_match_count_ex(g, p, _tp(tuning), sp, stream, ctypes.byref(c)))
    return c.value


def stm_match_count_async(g: int, p: int, d_result: int, tuning: Optional[stm_tuning] = None,
                          shard: Optional[stm_shard] = None, stream: Optional[int] = None) -> None:
    """d_result: device address of an stm_async_result (4 x uint64, e.g. a torch int64[4] tensor)."""
    sp = None if shard is None else ctypes.cast(ctypes.pointer(shard), ctypes.c_void_p)
    _check(lib.stm_match_count_async(g, p, _tp(tuning), sp, stream, d_result))


def async_status_message(status: int) -> str:
    return _NAMES.get(int(status), str(status))


def stm_cursors_alloc(device: int, n_slots: int) -> Tuple[int, bytes]:
    """n_slots zeroed device cursors (64 bytes apart) + their CUDA IPC handle bytes."""
    d = ctypes.c_void_p()
    h = ctypes.create_string_buffer(STM_IPC_HANDLE_BYTES)
    _check(lib.stm_cursors_alloc(device, n_slots, ctypes.byref(d), h))
    return d.value, h.raw


def stm_cursors_open(device: int, handle: bytes) -> int:
    d = ctypes.c_void_p()
    h = ctypes.create_string_buffer(bytes(handle), STM_IPC_HANDLE_BYTES)
    _check(lib.stm_cursors_open(device, h, ctypes.byref(d)))
    return d.value


def stm_cursors_close(device: int, d_peer: int) -> None:
    _check(lib.stm_cursors_close(device, d_peer))


def stm_cursors_reset(device: int, d_base: int, first_slot: int, n_slots: int, stream: Optional[int]) -> None:
    _check(lib.stm_cursors_reset(device, d_base, first_slot, n_slots, stream))


def stm_cursors_free(device: int, d_base: int) -> None:
    _check(lib.stm_cursors_free(device, d_base))


def stm_match_list(g: int, p: int, k: int, tuning: Optional[stm_tuning] = None, root_begin: int = 0,
                   root_end: Optional[int] = None, capacity: int = 0, stream: Optional[int] = None):
    """Enumerate embeddings of the root page [root_begin, root_end): returns (rows, count)
    with rows an int32 [min(count, capacity), k] array (pattern-vertex order, caller's ids)."""
    if root_end is None:
        n = ctypes.c_int64()
        _check(lib.stm_graph_info(g, ctypes.byref(n), None, None))
        root_end = n.value
    buf = np.zeros((max(capacity, 1), k), dtype=np.int32)
    nl, c = ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib.stm_match_list(g, p, _tp(tuning), root_begin, root_end, stream,
                              buf.ctypes.data if capacity else None, capacity, ctypes.byref(nl), ctypes.byref(c)))
    return buf[:nl.value], c.value


def stm_match_count_per_root(g: int, p: int, tuning: Optional[stm_tuning] = None,
                             stream: Optional[int] = None) -> Tuple[int, np.ndarray]:
    n, _, _ = stm_graph_info(g)
    out = np.zeros(max(n, 1), dtype=np.uint64)
    c = ctypes.c_uint64()
    _check(lib.stm_match_count_per_root(g, p, _tp(tuning), stream, out.ctypes.data, ctypes.byref(c)))
    return c.value, out[:n]


PROF_PHASES = ["gather_roots", "root_sibling", "gather_batch", "build_nodes", "frame_count", "fused_count",
               "donate", "acquire_work", "next_sibling", "descend", "jobs_setup", "jobs_loop"]


def stm_last_profile() -> dict:
    N = 3 * len(PROF_PHASES) + 4
    NL = 3 * 3 * 8 + 2
    NT = 64  # timeline buckets (kernel.h STM_PROF_TL, 0.5 ms each)
    out = (ctypes.c_uint64 * (N + NL + NT))()
    _check(lib.stm_last_profile(out, N + NL + NT))
    d = {ph: {"cycles": out[3 * i], "calls": out[3 * i + 1], "items": out[3 * i + 2]}
         for i, ph in enumerate(PROF_PHASES)}
    d["lifetime_cycles"] = out[N - 4]
    d["tail"] = {"max_lifetime": out[N - 3], "sum_dry": out[N - 2], "max_dry": out[N - 1]}
    lv = {}
    for kind, kn in enumerate(["pretest", "build", "count"]):
        for lvl in range(8):
            c, j, e = out[N + 3 * (8 * kind + lvl):N + 3 * (8 * kind + lvl) + 3]
            if j:
                lv[f"{kn}@L{lvl}"] = {"cycles": c, "ops": j, "elements": e}
    d["levels"] = lv
    d["max_task_cycles"] = out[N + NL - 2]
    d["timeline_busy_warps"] = [out[N + NL + i] / 5e5 for i in range(NT)]  # mean busy warps per 0.5 ms
    return d


def stm_last_launch() -> dict:
    info = stm_launch_info()
    _check(lib.stm_last_launch(ctypes.byref(info)))
    return {f[0]: getattr(info, f[0]) for f in info._fields_}


# ---------------------------------------------------------------- convenience objects
class Graph:
    """Device-resident data graph (owns the stm_graph handle)."""

    def __init__(self, n: int, row_ptr, col_idx, labels=None, device: int = 0, directed: bool = False):
        """directed: row_ptr / col_idx are out-neighbour rows of a digraph (stm_graph_load_directed)."""
        self.handle = (stm_graph_load_directed if directed else stm_graph_load)(n, row_ptr, col_idx, labels, device)
        self.n, self.nnz, self.max_degree = stm_graph_info(self.handle)
        self.device = device
        self.directed = directed

    @classmethod
    def from_stmgen(cls, g, device: int = 0) -> "Graph":
        return cls(g.n, g.row_ptr, g.col_idx, g.labels, device)

    def close(self):
        if self.handle:
            stm_graph_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Plan:
    """Compiled pattern (owns the stm_plan handle)."""

    def __init__(self, k: int, edges, labels=None, order=None, restrictions=None, vertex_induced=False,
                 code_motion=True, auto_restrict=None, auto_order=False, lazy_unbounded=False,
                 cost_stats: Optional[stm_graph_stats] = None, graph: Optional["Graph"] = None,
                 directed: bool = False):
        """cost_stats: graph statistics (stm_graph_stats_host) -> the cost-optimal order (NEXT-2)
        replaces `order`.  graph: compile for this loaded graph -- its statistics (stm_graph_get_stats)
        give the cost-based order unless `order` or `cost_stats` is given.  directed: `edges` are arcs
        (a, b) = a -> b (STM_DIRECTED; graphs from Graph(..., directed=True)); greedy order only."""
        directed = directed or bool(graph is not None and getattr(graph, "directed", False))
        if graph is not None and cost_stats is None and order is None and not auto_order and not directed:
            cost_stats = stm_graph_get_stats(graph.handle)
        if auto_restrict is None:
            auto_restrict = restrictions is None
        flags = (STM_VERTEX_INDUCED if vertex_induced else 0) | (0 if code_motion else STM_NO_CODE_MOTION)
        flags |= STM_AUTO_RESTRICT if auto_restrict else 0
        flags |= STM_LAZY_UNBOUNDED if lazy_unbounded else 0
        flags |= STM_DIRECTED if directed else 0
        if cost_stats is not None and not directed:
            order, self.model_cost, self.model_count = stm_order_optimize(k, edges, labels, restrictions, flags,
                                                                          cost_stats)
        flags |= STM_AUTO_ORDER if auto_order else 0
        self.handle = stm_pattern_compile(k, edges, labels, order, restrictions, flags)
        self.k, self.n_sets, self.aut = stm_plan_info(self.handle)
        self.first_vertex = stm_plan_first_vertex(self.handle)

    @classmethod
    def from_pattern(cls, p, **kw) -> "Plan":
        return cls(p.k, p.edges, p.labels, **kw)

    def describe(self) -> str:
        return stm_plan_describe(self.handle)

    def close(self):
        if self.handle:
            stm_plan_free(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def count(graph: Graph, plan: Plan, tuning: Optional[stm_tuning] = None, stream: Optional[int] = None) -> int:
    return stm_match_count_ex(graph.handle, plan.handle, tuning, None, stream)
