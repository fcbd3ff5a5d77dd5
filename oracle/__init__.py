"""oracle -- TEST INFRASTRUCTURE ONLY (never imported by the product path).

Plain, slow, obviously correct CPU reference for the STMatch counting hot path.
Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with
``paper_conf_sc_weij22_b200`` (no common headers, helpers, tables or
pre/post-processing); the only shared module is ``stmgen`` (seeded inputs).

Functions and the passage each follows:

* ``count``            -- C backtracking matcher (oracle.c), Alg. 1
                          and the Fig. 1 nested loop applied to the
                          plain definition.
* ``brute_force_count`` -- the definition written out literally: every injective
                          map V_Q -> V is tested (tiny graphs only).
* ``automorphisms``    -- label-preserving automorphism group of Q by brute force
                          over all k! permutations (Definition 1, PAPER.md:46,
                          applied to Q itself).
* ``gk_restrictions``  -- symmetry-breaking restriction pairs (not in the paper;
                          BASELINE.json north_star): Grochow-Kellis stabiliser chain.
                          SURVEY.md 8(c) "Restriction generation".

Pins (tests/test_oracle.py): brute force on tiny graphs, closed forms on K_n,
C_n, grids, tr(A^3)/6, degree sums, the C4 trace formula, networkx VF2, known
|Aut| values, and the invariants restricted x |Aut_L| = unrestricted,
label-sum, order invariance, relabel invariance and disjoint-union additivity.
Every function here is pinned; none is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import itertools
import os
import subprocess
from typing import List, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build() -> str:
    subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", _LIB_PATH,
                           os.path.join(_HERE, "oracle.c"), "-lpthread"])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        src = os.path.join(_HERE, "oracle.c")
        if not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
            build()
        lib = ctypes.CDLL(_LIB_PATH)
        vp = ctypes.c_void_p
        lib.oracle_count.restype = ctypes.c_int
        lib.oracle_count.argtypes = [ctypes.c_int64, vp, vp, vp, ctypes.c_int, ctypes.c_int, vp, vp,
                                     ctypes.c_int, ctypes.c_int, vp, ctypes.c_int, vp, ctypes.c_int64,
                                     ctypes.c_int, vp, ctypes.POINTER(ctypes.c_uint64)]
        lib.oracle_count_directed.restype = ctypes.c_int
        lib.oracle_count_directed.argtypes = [ctypes.c_int64, vp, vp, vp, vp, vp, ctypes.c_int, ctypes.c_int, vp,
                                              vp, ctypes.c_int, ctypes.c_int, vp, ctypes.c_int, vp,
                                              ctypes.c_int64, ctypes.c_int, vp, ctypes.POINTER(ctypes.c_uint64)]
        lib.oracle_list.restype = ctypes.c_int
        lib.oracle_list.argtypes = [ctypes.c_int64, vp, vp, vp, ctypes.c_int, ctypes.c_int, vp, vp,
                                    ctypes.c_int, ctypes.c_int, vp, ctypes.c_int, vp, ctypes.c_int64,
                                    ctypes.c_int, vp, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64),
                                    ctypes.POINTER(ctypes.c_uint64)]
        _lib = lib
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data


def check_graph(n: int, row_ptr: np.ndarray, col_idx: np.ndarray) -> None:
    """Reject anything that is not an undirected simple graph with sorted rows."""
    assert row_ptr.shape == (n + 1,) and row_ptr[0] == 0 and row_ptr[-1] == col_idx.shape[0]
    assert np.all(np.diff(row_ptr) >= 0)
    for v in range(n) if n <= 5000 else []:
        nb = col_idx[row_ptr[v]:row_ptr[v + 1]]
        assert np.all(np.diff(nb) > 0) and not np.any(nb == v)


def count(g, k: int, edges: Sequence[Tuple[int, int]], plabels: Optional[Sequence[int]] = None,
          vertex_induced: bool = False, restrictions: Sequence[Tuple[int, int]] = (),
          root_u: int = -1, roots: Optional[np.ndarray] = None, threads: int = 0,
          per_root: bool = False):
    """Count embeddings of Q in g (stmgen.Graph-like: n, row_ptr, col_idx, labels).

    Returns the uint64 count (Python int), or (count, per_root_counts) if per_root.
    ``roots`` restricts level 0 to those data vertices (matches attributed to
    f(root_u)); ``root_u`` picks the oracle's first pattern vertex (-1 = default).
    """
    lib = _load()
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(g.col_idx, dtype=np.int32)
    lab = None
    if plabels is not None:
        if g.labels is None:
            raise ValueError("labeled pattern on an unlabeled graph")
        lab = np.ascontiguousarray(g.labels, dtype=np.int32)
    e = np.ascontiguousarray(np.asarray(edges, dtype=np.int32).reshape(-1, 2))
    pl = None if plabels is None else np.ascontiguousarray(np.asarray(plabels, dtype=np.int32))
    r = np.ascontiguousarray(np.asarray(restrictions, dtype=np.int32).reshape(-1, 2))
    ro = None if roots is None else np.ascontiguousarray(np.asarray(roots, dtype=np.int64))
    nr = 0 if ro is None else ro.shape[0]
    pr = np.zeros(nr if ro is not None else g.n, dtype=np.uint64) if per_root else None
    out = ctypes.c_uint64(0)
    threads = threads or (os.cpu_count() or 1)
    rc = lib.oracle_count(g.n, _ptr(rp), _ptr(ci), _ptr(lab), k, e.shape[0], _ptr(e), _ptr(pl),
                          int(vertex_induced), r.shape[0], _ptr(r), root_u, _ptr(ro), nr, threads,
                          _ptr(pr), ctypes.byref(out))
    if rc != 0:
        raise ValueError("oracle_count rejected its input")
    return (int(out.value), pr) if per_root else int(out.value)


def list_embeddings(g, k: int, edges: Sequence[Tuple[int, int]], plabels: Optional[Sequence[int]] = None,
                    vertex_induced: bool = False, restrictions: Sequence[Tuple[int, int]] = (),
                    threads: int = 0, capacity: Optional[int] = None) -> np.ndarray:
    """Every embedding f of Q in g as the rows of an int32 [count, k] array (row = f(0..k-1),
    in pattern-vertex order), sorted lexicographically (Output(C, iter) at the
    last level).  Counts first to size the buffer unless ``capacity`` is given."""
    lib = _load()
    if capacity is None:
        capacity = count(g, k, edges, plabels, vertex_induced, restrictions, threads=threads)
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(g.col_idx, dtype=np.int32)
    lab = None if plabels is None else np.ascontiguousarray(g.labels, dtype=np.int32)
    e = np.ascontiguousarray(np.asarray(edges, dtype=np.int32).reshape(-1, 2))
    pl = None if plabels is None else np.ascontiguousarray(np.asarray(plabels, dtype=np.int32))
    r = np.ascontiguousarray(np.asarray(restrictions, dtype=np.int32).reshape(-1, 2))
    buf = np.zeros((max(int(capacity), 1), k), dtype=np.int32)
    out, nl = ctypes.c_uint64(0), ctypes.c_uint64(0)
    rc = lib.oracle_list(g.n, _ptr(rp), _ptr(ci), _ptr(lab), k, e.shape[0], _ptr(e), _ptr(pl),
                         int(vertex_induced), r.shape[0], _ptr(r), -1, None, 0, threads or (os.cpu_count() or 1),
                         _ptr(buf), int(capacity), ctypes.byref(nl), ctypes.byref(out))
    if rc != 0:
        raise ValueError("oracle_list rejected its input")
    got = buf[:min(int(nl.value), int(capacity))]
    return got[np.lexsort(got.T[::-1])] if got.shape[0] else got


def transpose(n: int, row_ptr: np.ndarray, col_idx: np.ndarray):
    """In-neighbour rows of a digraph given by its out-neighbour rows (sorted ascending)."""
    rp = np.asarray(row_ptr, dtype=np.int64)
    ci = np.asarray(col_idx, dtype=np.int64)
    src = np.repeat(np.arange(n, dtype=np.int64), np.diff(rp))
    o = np.lexsort((src, ci))  # by destination, then source
    in_rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(ci, minlength=n), out=in_rp[1:])
    return in_rp, np.ascontiguousarray(src[o], dtype=np.int32)


def count_directed(g, k: int, arcs: Sequence[Tuple[int, int]], plabels: Optional[Sequence[int]] = None,
                   vertex_induced: bool = False, restrictions: Sequence[Tuple[int, int]] = (),
                   root_u: int = -1, roots: Optional[np.ndarray] = None, threads: int = 0,
                   per_root: bool = False):
    """count() for a directed data graph (g.row_ptr / g.col_idx = sorted out-neighbour rows)
    and a pattern given by arcs (a, b) = a -> b (oracle.c oracle_count_directed)."""
    lib = _load()
    rp = np.ascontiguousarray(g.row_ptr, dtype=np.int64)
    ci = np.ascontiguousarray(g.col_idx, dtype=np.int32)
    irp, ici = transpose(g.n, rp, ci)
    lab = None
    if plabels is not None:
        if g.labels is None:
            raise ValueError("labeled pattern on an unlabeled graph")
        lab = np.ascontiguousarray(g.labels, dtype=np.int32)
    e = np.ascontiguousarray(np.asarray(arcs, dtype=np.int32).reshape(-1, 2))
    pl = None if plabels is None else np.ascontiguousarray(np.asarray(plabels, dtype=np.int32))
    r = np.ascontiguousarray(np.asarray(restrictions, dtype=np.int32).reshape(-1, 2))
    ro = None if roots is None else np.ascontiguousarray(np.asarray(roots, dtype=np.int64))
    nr = 0 if ro is None else ro.shape[0]
    pr = np.zeros(nr if ro is not None else g.n, dtype=np.uint64) if per_root else None
    out = ctypes.c_uint64(0)
    rc = lib.oracle_count_directed(g.n, _ptr(rp), _ptr(ci), _ptr(irp), _ptr(ici), _ptr(lab), k, e.shape[0],
                                   _ptr(e), _ptr(pl), int(vertex_induced), r.shape[0], _ptr(r), root_u,
                                   _ptr(ro), nr, threads or (os.cpu_count() or 1), _ptr(pr), ctypes.byref(out))
    if rc != 0:
        raise ValueError("oracle_count_directed rejected its input")
    return (int(out.value), pr) if per_root else int(out.value)


def brute_force_count_directed(g, k: int, arcs, plabels=None, vertex_induced=False, restrictions=()) -> int:
    """The directed definition tested literally on every injective map f: V_Q -> V: every
    pattern arc a -> b an arc f(a) -> f(b) of g, [vertex-induced] every pattern non-arc a
    non-arc.  Tiny graphs only."""
    A = _adj_sets(g)
    E = {(a, b) for a, b in arcs}
    non = [(a, b) for a in range(k) for b in range(k) if a != b and (a, b) not in E]
    c = 0
    for f in itertools.permutations(range(g.n), k):
        if any(f[b] not in A[f[a]] for a, b in E):
            continue
        if vertex_induced and any(f[b] in A[f[a]] for a, b in non):
            continue
        if plabels is not None and any(int(g.labels[f[u]]) != int(plabels[u]) for u in range(k)):
            continue
        if any(not f[a] < f[b] for a, b in restrictions):
            continue
        c += 1
    return c % (1 << 64)


def automorphisms_directed(k: int, arcs, plabels=None) -> List[Tuple[int, ...]]:
    """All label- and arc-preserving permutations of a directed pattern (brute force)."""
    E = {(a, b) for a, b in arcs}
    out = []
    for p in itertools.permutations(range(k)):
        if plabels is not None and any(plabels[p[u]] != plabels[u] for u in range(k)):
            continue
        if all((p[a], p[b]) in E for a, b in E):
            out.append(p)
    return out


def gk_restrictions_directed(k: int, arcs, plabels=None) -> List[Tuple[int, int]]:
    """gk_restrictions over the automorphism group of a directed pattern."""
    group = automorphisms_directed(k, arcs, plabels)
    R: List[Tuple[int, int]] = []
    while len(group) > 1:
        for u in range(k):
            orbit = sorted({p[u] for p in group})
            if len(orbit) > 1:
                break
        R.extend((u, w) for w in orbit if w != u)
        group = [p for p in group if p[u] == u]
    return R


# ---------------------------------------------------------------- brute force
def _adj_sets(g):
    return [set(int(x) for x in g.col_idx[g.row_ptr[v]:g.row_ptr[v + 1]]) for v in range(g.n)]


def brute_force_count(g, k: int, edges, plabels=None, vertex_induced=False, restrictions=()) -> int:
    """The definition tested literally on every
    injective map f: V_Q -> V.  n!/(n-k)! maps: tiny graphs only."""
    A = _adj_sets(g)
    E = {(min(a, b), max(a, b)) for a, b in edges}
    non_edges = [(a, b) for a in range(k) for b in range(a + 1, k) if (a, b) not in E]
    c = 0
    for f in itertools.permutations(range(g.n), k):
        if any(f[b] not in A[f[a]] for a, b in E):
            continue
        if vertex_induced and any(f[b] in A[f[a]] for a, b in non_edges):
            continue
        if plabels is not None and any(int(g.labels[f[u]]) != int(plabels[u]) for u in range(k)):
            continue
        if any(not f[a] < f[b] for a, b in restrictions):
            continue
        c += 1
    return c % (1 << 64)


def brute_force_list(g, k: int, edges, plabels=None, vertex_induced=False, restrictions=()) -> np.ndarray:
    """brute_force_count's maps themselves, as a lexicographically sorted int32 [count, k] array."""
    A = _adj_sets(g)
    E = {(min(a, b), max(a, b)) for a, b in edges}
    non_edges = [(a, b) for a in range(k) for b in range(a + 1, k) if (a, b) not in E]
    rows = []
    for f in itertools.permutations(range(g.n), k):
        if any(f[b] not in A[f[a]] for a, b in E):
            continue
        if vertex_induced and any(f[b] in A[f[a]] for a, b in non_edges):
            continue
        if plabels is not None and any(int(g.labels[f[u]]) != int(plabels[u]) for u in range(k)):
            continue
        if any(not f[a] < f[b] for a, b in restrictions):
            continue
        rows.append(f)
    return np.array(sorted(rows), dtype=np.int32).reshape(-1, k)


# ---------------------------------------------------------------- symmetry
def automorphisms(k: int, edges, plabels=None) -> List[Tuple[int, ...]]:
    """All label-preserving automorphisms of Q (brute force over k! permutations)."""
    E = {(min(a, b), max(a, b)) for a, b in edges}
    out = []
    for p in itertools.permutations(range(k)):
        if plabels is not None and any(plabels[p[u]] != plabels[u] for u in range(k)):
            continue
        if all((min(p[a], p[b]), max(p[a], p[b])) in E for a, b in E):
            out.append(p)
    return out


def gk_restrictions(k: int, edges, plabels=None) -> List[Tuple[int, int]]:
    """Grochow-Kellis symmetry breaking: while the group is non-trivial, take the
    smallest u whose orbit is larger than {u}, add (u, w) for every other w in the
    orbit, and replace the group by the stabiliser of u."""
    group = automorphisms(k, edges, plabels)
    R: List[Tuple[int, int]] = []
    while len(group) > 1:
        for u in range(k):
            orbit = sorted({p[u] for p in group})
            if len(orbit) > 1:
                break
        R.extend((u, w) for w in orbit if w != u)
        group = [p for p in group if p[u] == u]
    return R
