"""Pins of the directed oracle (oracle.count_directed; "supports both directed and
undirected graphs") against things other than itself: the definition
tested literally on tiny digraphs (brute force over every injective map), tournament closed
forms, the undirected oracle on symmetric digraphs, and the restriction invariant."""
import itertools

import numpy as np
import pytest

import oracle


class DG:
    def __init__(self, n, arcs, labels=None):
        arcs = sorted(set(arcs))
        self.n = n
        out = [[] for _ in range(n)]
        for a, b in arcs:
            assert a != b
            out[a].append(b)
        self.row_ptr = np.zeros(n + 1, dtype=np.int64)
        self.row_ptr[1:] = np.cumsum([len(x) for x in out])
        self.col_idx = np.array([y for x in out for y in sorted(x)], dtype=np.int32)
        self.labels = labels


def rand_dg(n, p, seed, labels=0):
    rng = np.random.default_rng(seed)
    arcs = [(a, b) for a in range(n) for b in range(n) if a != b and rng.random() < p]
    lab = rng.integers(0, labels, n).astype(np.int32) if labels else None
    return DG(n, arcs, lab)


PATTERNS = {
    "cycle3": (3, [(0, 1), (1, 2), (2, 0)]),
    "transitive3": (3, [(0, 1), (1, 2), (0, 2)]),
    "mutual_path": (3, [(0, 1), (1, 0), (1, 2)]),
    "out_star": (4, [(0, 1), (0, 2), (0, 3)]),
    "in_star": (4, [(1, 0), (2, 0), (3, 0)]),
    "cycle4": (4, [(0, 1), (1, 2), (2, 3), (3, 0)]),
    "feed_forward4": (4, [(0, 1), (0, 2), (1, 3), (2, 3)]),
    "bifan": (4, [(0, 2), (0, 3), (1, 2), (1, 3)]),
    "mutual_triangle": (3, [(0, 1), (1, 0), (1, 2), (2, 1), (0, 2), (2, 0)]),
}


@pytest.mark.parametrize("name", sorted(PATTERNS))
@pytest.mark.parametrize("vi", [False, True])
def test_directed_brute_force(name, vi):
    k, arcs = PATTERNS[name]
    for seed in (1, 2):
        g = rand_dg(7, 0.35, seed)
        R = oracle.gk_restrictions_directed(k, arcs)
        for restr in (R, []):
            assert oracle.count_directed(g, k, arcs, vertex_induced=vi, restrictions=restr, threads=2) == \
                oracle.brute_force_count_directed(g, k, arcs, vertex_induced=vi, restrictions=restr)


def test_directed_labeled_brute_force():
    g = rand_dg(8, 0.4, 5, labels=2)
    for name in ("cycle3", "transitive3", "feed_forward4"):
        k, arcs = PATTERNS[name]
        pl = [u % 2 for u in range(k)]
        R = oracle.gk_restrictions_directed(k, arcs, pl)
        for vi in (False, True):
            assert oracle.count_directed(g, k, arcs, pl, vi, R) == oracle.brute_force_count_directed(g, k, arcs, pl, vi, R)


def test_transitive_tournament():
    """i -> j for every i < j: every 3-set is one transitive triangle, none is cyclic."""
    n = 12
    g = DG(n, [(i, j) for i in range(n) for j in range(i + 1, n)])
    k, arcs = PATTERNS["transitive3"]
    assert oracle.count_directed(g, k, arcs, restrictions=oracle.gk_restrictions_directed(k, arcs)) == 220
    k, arcs = PATTERNS["cycle3"]
    assert oracle.count_directed(g, k, arcs, restrictions=oracle.gk_restrictions_directed(k, arcs)) == 0


@pytest.mark.parametrize("n", [7, 9, 13])
def test_regular_tournament(n):
    """Circulant tournament i -> i+1..i+m (n = 2m+1): n(n^2-1)/24 cyclic triangles (Kendall &
    Babington Smith); the other C(n,3) - that are transitive."""
    m = n // 2
    g = DG(n, [(i, (i + d) % n) for i in range(n) for d in range(1, m + 1)])
    cyc = n * (n * n - 1) // 24
    k, arcs = PATTERNS["cycle3"]
    assert oracle.count_directed(g, k, arcs, restrictions=oracle.gk_restrictions_directed(k, arcs)) == cyc
    k, arcs = PATTERNS["transitive3"]
    assert oracle.count_directed(g, k, arcs) == n * (n - 1) * (n - 2) // 6 - cyc


def test_symmetric_digraph_equals_undirected():
    """A digraph with both arcs of every undirected edge, and a pattern all of whose edges are
    mutual, count exactly what the (independently pinned) undirected oracle counts."""
    import stmgen
    g = stmgen.er(60, 300, 4)
    dg = DG(g.n, [(int(a), int(b)) for a in range(g.n) for b in g.col_idx[g.row_ptr[a]:g.row_ptr[a + 1]]])
    for name in ("triangle", "c4", "diamond", "house"):
        p = stmgen.CATALOG[name]
        arcs = [(a, b) for a, b in p.edges] + [(b, a) for a, b in p.edges]
        for vi in (False, True):
            R = oracle.gk_restrictions(p.k, p.edges)
            assert oracle.gk_restrictions_directed(p.k, arcs) == R
            assert oracle.count_directed(dg, p.k, arcs, vertex_induced=vi, restrictions=R) == \
                oracle.count(g, p.k, p.edges, vertex_induced=vi, restrictions=R)


@pytest.mark.parametrize("name", sorted(PATTERNS))
def test_directed_restrictions_times_aut(name):
    k, arcs = PATTERNS[name]
    g = rand_dg(30, 0.15, 9)
    A = len(oracle.automorphisms_directed(k, arcs))
    R = oracle.gk_restrictions_directed(k, arcs)
    for vi in (False, True):
        assert oracle.count_directed(g, k, arcs, vertex_induced=vi, restrictions=R) * A == \
            oracle.count_directed(g, k, arcs, vertex_induced=vi)
