"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

INPUT GENERATION ONLY: this package holds none of the matching method's
arithmetic.  It builds data graphs (CSR: ``row_ptr`` int64[n+1], ``col_idx``
int32[2m], rows sorted, undirected and simple), vertex labels, and the pattern
catalog.  Both ``oracle/`` (via the tests) and ``paper_conf_sc_weij22_b200``
consume these arrays; neither imports the other.

Workload recipe: the paper evaluates on
SNAP graphs (Table I at 170-209) that are not available here, so
each BASELINE.json config is replaced by a seeded generator of the same shape.
"""
from __future__ import annotations

import ctypes
import hashlib
import os
from dataclasses import dataclass
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libstmgen.so")
_lib = None


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        import subprocess
        subprocess.check_call(
            ["gcc", "-O2", "-shared", "-fPIC", "-o", _LIB_PATH, os.path.join(_HERE, "gen.c"),
             "-lpthread", "-lm"])
    lib = ctypes.CDLL(_LIB_PATH)
    vp, i64, u64, i32, dbl = ctypes.c_void_p, ctypes.c_int64, ctypes.c_uint64, ctypes.c_int32, ctypes.c_double
    lib.stmgen_er.restype = vp
    lib.stmgen_er.argtypes = [i64, i64, u64]
    lib.stmgen_rmat.restype = vp
    lib.stmgen_rmat.argtypes = [ctypes.c_int, i64, dbl, dbl, dbl, u64, ctypes.c_int, ctypes.c_int]
    lib.stmgen_chung_lu.restype = vp
    lib.stmgen_chung_lu.argtypes = [i64, i64, dbl, dbl, dbl, u64, ctypes.c_int]
    lib.stmgen_from_edges.restype = vp
    lib.stmgen_from_edges.argtypes = [i64, i64, vp, vp, u64, ctypes.c_int]
    lib.stmgen_sizes.argtypes = [vp, ctypes.POINTER(i64), ctypes.POINTER(i64)]
    lib.stmgen_copy.argtypes = [vp, vp, vp]
    lib.stmgen_free.argtypes = [vp]
    lib.stmgen_labels.argtypes = [i64, i32, u64, vp]
    _lib = lib
    return lib


@dataclass
class Graph:
    """Undirected simple graph in CSR form with optional int32 vertex labels."""
    n: int
    row_ptr: np.ndarray  # int64[n+1]
    col_idx: np.ndarray  # int32[2m]
    labels: Optional[np.ndarray] = None  # int32[n]
    name: str = ""

    @property
    def m(self) -> int:
        return int(self.col_idx.shape[0] // 2)

    def degrees(self) -> np.ndarray:
        return np.diff(self.row_ptr)

    def neighbors(self, v: int) -> np.ndarray:
        return self.col_idx[self.row_ptr[v]:self.row_ptr[v + 1]]

    def fingerprint(self) -> str:
        h = hashlib.sha256()
        h.update(np.int64(self.n).tobytes())
        h.update(np.ascontiguousarray(self.row_ptr).tobytes())
        h.update(np.ascontiguousarray(self.col_idx).tobytes())
        if self.labels is not None:
            h.update(np.ascontiguousarray(self.labels).tobytes())
        return h.hexdigest()[:16]

    def with_labels(self, nlabels: int, seed: int) -> "Graph":
        return Graph(self.n, self.row_ptr, self.col_idx, labels(self.n, nlabels, seed), self.name)

    def stats(self) -> Dict[str, float]:
        d = self.degrees()
        nz = d[d > 0]
        return {"n": self.n, "m": self.m, "non_isolated": int(nz.size),
                "max_degree": int(d.max()) if d.size else 0,
                "median_degree": float(np.median(nz)) if nz.size else 0.0,
                "deg_gt_4096": int((d > 4096).sum()),
                "sum_d2": float((d.astype(np.float64) ** 2).sum())}


def _take(h, name: str) -> Graph:
    lib = _load()
    n, nnz = ctypes.c_int64(), ctypes.c_int64()
    lib.stmgen_sizes(h, ctypes.byref(n), ctypes.byref(nnz))
    rp = np.empty(n.value + 1, dtype=np.int64)
    ci = np.empty(max(nnz.value, 0), dtype=np.int32)
    lib.stmgen_copy(h, rp.ctypes.data, ci.ctypes.data)
    lib.stmgen_free(h)
    return Graph(int(n.value), rp, ci, None, name)


def from_edges(n: int, edges: Sequence[Tuple[int, int]] | np.ndarray, perm_seed: int = 0,
               compact: bool = False, name: str = "edges") -> Graph:
    """Canonicalise an arbitrary edge list (self-loops and duplicates dropped)."""
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    u = np.ascontiguousarray(e[:, 0])
    v = np.ascontiguousarray(e[:, 1])
    h = _load().stmgen_from_edges(n, e.shape[0], u.ctypes.data, v.ctypes.data, perm_seed, int(compact))
    return _take(h, name)


def er(n: int, m: int, seed: int) -> Graph:
    """Erdos-Renyi G(n, m)."""
    return _take(_load().stmgen_er(n, m, seed), f"er_{n}_{m}_s{seed}")


def rmat(scale: int, ndraws: int, a: float, b: float, c: float, seed: int, compact: bool = False,
         threads: int = 0) -> Graph:
    """R-MAT with 2^scale vertices and ndraws edge draws (Graph500-style), IDs permuted."""
    threads = threads or min(32, os.cpu_count() or 1)
    h = _load().stmgen_rmat(scale, ndraws, a, b, c, seed, int(compact), threads)
    return _take(h, f"rmat_s{scale}_d{ndraws}_s{seed}")


def chung_lu(n: int, m: int, gamma: float, wmax: float, seed: int, draw_factor: float = 1.04,
             compact: bool = False) -> Graph:
    """Chung-Lu power-law graph with max weight wmax and expected ~m edges."""
    h = _load().stmgen_chung_lu(n, m, gamma, wmax, draw_factor, seed, int(compact))
    return _take(h, f"chunglu_{n}_{m}_s{seed}")


def labels(n: int, nlabels: int, seed: int) -> np.ndarray:
    out = np.empty(n, dtype=np.int32)
    if n:
        _load().stmgen_labels(n, nlabels, seed, out.ctypes.data)
    return out


# ---------------------------------------------------------------- small graphs
def complete(n: int) -> Graph:
    e = [(i, j) for i in range(n) for j in range(i + 1, n)]
    return from_edges(n, e if e else np.zeros((0, 2), np.int64), name=f"K{n}")


def cycle(n: int) -> Graph:
    return from_edges(n, [(i, (i + 1) % n) for i in range(n)], name=f"C{n}")


def grid(a: int, b: int) -> Graph:
    e = []
    for i in range(a):
        for j in range(b):
            v = i * b + j
            if j + 1 < b:
                e.append((v, v + 1))
            if i + 1 < a:
                e.append((v, v + b))
    return from_edges(a * b, e if e else np.zeros((0, 2), np.int64), name=f"grid{a}x{b}")


def disjoint_union(g1: Graph, g2: Graph) -> Graph:
    def edges(g):
        src = np.repeat(np.arange(g.n, dtype=np.int64), np.diff(g.row_ptr))
        return np.stack([src, g.col_idx.astype(np.int64)], 1)
    e = np.concatenate([edges(g1), edges(g2) + g1.n], 0)
    g = from_edges(g1.n + g2.n, e, name=f"{g1.name}+{g2.name}")
    if g1.labels is not None and g2.labels is not None:
        g.labels = np.concatenate([g1.labels, g2.labels]).astype(np.int32)
    return g


def relabel(g: Graph, perm_seed: int) -> Graph:
    """Same graph with vertex IDs randomly permuted (labels carried along)."""
    src = np.repeat(np.arange(g.n, dtype=np.int64), np.diff(g.row_ptr))
    e = np.stack([src, g.col_idx.astype(np.int64)], 1)
    rng = np.random.default_rng(perm_seed)
    p = rng.permutation(g.n)
    out = from_edges(g.n, p[e], name=g.name + f"_perm{perm_seed}")
    if g.labels is not None:
        lab = np.empty(g.n, np.int32)
        lab[p] = g.labels
        out.labels = lab
    return out


def permute(g: Graph, p: np.ndarray) -> Graph:
    """Same graph with vertex v renamed p[v] (labels carried along)."""
    src = np.repeat(np.arange(g.n, dtype=np.int64), np.diff(g.row_ptr))
    e = np.stack([src, g.col_idx.astype(np.int64)], 1)
    p = np.asarray(p, dtype=np.int64)
    out = from_edges(g.n, p[e], name=g.name + "_permuted")
    if g.labels is not None:
        lab = np.empty(g.n, np.int32)
        lab[p] = g.labels
        out.labels = lab
    return out


def empty(n: int) -> Graph:
    return from_edges(n, np.zeros((0, 2), np.int64), name=f"empty{n}")


# ---------------------------------------------------------------- patterns
@dataclass(frozen=True)
class Pattern:
    name: str
    k: int
    edges: Tuple[Tuple[int, int], ...]
    labels: Optional[Tuple[int, ...]] = None

    def with_labels(self, labs: Sequence[int]) -> "Pattern":
        return Pattern(self.name + "_L" + "".join(str(x) for x in labs), self.k, self.edges,
                       tuple(int(x) for x in labs))


def _cyc(k):
    return tuple((i, (i + 1) % k) if i < (i + 1) % k else ((i + 1) % k, i) for i in range(k))


def _clique(k):
    return tuple((i, j) for i in range(k) for j in range(i + 1, k))


def _wheel(k):  # hub 0 + rim cycle 1..k-1
    rim = k - 1
    e = [(0, i) for i in range(1, k)]
    for i in range(rim):
        a, b = 1 + i, 1 + (i + 1) % rim
        e.append((min(a, b), max(a, b)))
    return tuple(e)


# Our own catalog (the paper's q1-q24 shapes are lost in extraction, PAPER.md:151;
# SURVEY.md 8(c) reading c23).  The diamond follows Fig. 2: u0
# adjacent to u1, u2, u3; u3 adjacent to u1, u2; u1, u2 not adjacent.
CATALOG: Dict[str, Pattern] = {}
for _p in [
    Pattern("edge", 2, ((0, 1),)),
    Pattern("wedge", 3, ((0, 1), (0, 2))),
    Pattern("triangle", 3, _clique(3)),
    Pattern("path4", 4, ((0, 1), (1, 2), (2, 3))),
    Pattern("star4", 4, ((0, 1), (0, 2), (0, 3))),
    Pattern("c4", 4, _cyc(4)),
    Pattern("diamond", 4, ((0, 1), (0, 2), (0, 3), (1, 3), (2, 3))),
    Pattern("tailed_triangle", 4, ((0, 1), (0, 2), (1, 2), (2, 3))),
    Pattern("k4", 4, _clique(4)),
    Pattern("k5", 5, _clique(5)),
    Pattern("house", 5, ((0, 1), (0, 2), (1, 3), (2, 3), (2, 4), (3, 4))),
    Pattern("c5", 5, _cyc(5)),
    Pattern("k6", 6, _clique(6)),
    Pattern("k6_minus_e", 6, tuple(e for e in _clique(6) if e != (0, 1))),
    Pattern("octahedron", 6, tuple(e for e in _clique(6) if e not in ((0, 1), (2, 3), (4, 5)))),
    Pattern("w5", 6, _wheel(6)),
    Pattern("prism", 6, ((0, 1), (1, 2), (0, 2), (3, 4), (4, 5), (3, 5), (0, 3), (1, 4), (2, 5))),
    Pattern("c6", 6, _cyc(6)),
    Pattern("k7", 7, _clique(7)),
    Pattern("k7_minus_e", 7, tuple(e for e in _clique(7) if e != (0, 1))),
    Pattern("w6", 7, _wheel(7)),
    Pattern("c7", 7, _cyc(7)),
    Pattern("k8", 8, _clique(8)),
]:
    CATALOG[_p.name] = _p


def pattern(name: str, labels: Optional[Sequence[int]] = None) -> Pattern:
    p = CATALOG[name]
    return p.with_labels(labels) if labels is not None else p


def pattern_labels(k: int, nlabels: int, seed: int) -> Tuple[int, ...]:
    rng = np.random.default_rng(seed)
    return tuple(int(x) for x in rng.integers(0, nlabels, size=k))


# ---------------------------------------------------------------- configs
# The five BASELINE.json configs.
def config_graph(cfg: str, small: bool = False) -> Graph:
    if cfg == "c1":  # ER, 1,000 vertices, ~10k edges
        return er(1000, 10_000, 101)
    if cfg == "c2":  # R-MAT scale 16, edge factor 16, Graph500 (0.57, 0.19, 0.19, 0.05)
        return rmat(16, 1 << 20, 0.57, 0.19, 0.19, 102)
    if cfg == "c3":  # com-Youtube-shaped Chung-Lu power law
        return chung_lu(1_134_890, 2_987_624, 2.2, 28_754.0, 103)
    if cfg == "c4":  # MiCo-shaped R-MAT scale 17 + 8 labels
        g = rmat(17, 1_150_000, 0.45, 0.22, 0.22, 104)
        g.labels = labels(g.n, 8, 1040)
        g.name += "_L8"
        return g
    if cfg == "c4p":  # Patents-shaped R-MAT scale 22 + 8 labels
        g = rmat(22, 17_000_000, 0.40, 0.25, 0.25, 105)
        g.labels = labels(g.n, 8, 1050)
        g.name += "_L8"
        return g
    if cfg == "c5":  # LiveJournal-shaped R-MAT scale 23, isolated vertices compacted
        return rmat(23, 46_000_000, 0.50, 0.20, 0.20, 106, compact=True)
    raise KeyError(cfg)
