"""Pins for the oracle (CPU only, -m "not gpu").

The oracle (oracle/) must be checked against something other than itself before
it may judge the CUDA path.  Each test below names what pins it:
brute force over all injective maps, closed forms, an independent library
(networkx VF2, scipy sparse products), known group orders, and invariants.
"""
import itertools
import math

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
import stmgen
from stmgen import CATALOG

SMALL_PATTERNS = ["edge", "wedge", "triangle", "path4", "star4", "c4", "diamond",
                  "tailed_triangle", "k4", "house", "c5", "k5"]


def adj_matrix(g):
    return sp.csr_matrix((np.ones(g.col_idx.size, dtype=np.float64), g.col_idx, g.row_ptr),
                         shape=(g.n, g.n))


def ocount(g, p, mode="edge", restr=None, plabels=None, **kw):
    if restr == "auto":
        restr = oracle.gk_restrictions(p.k, p.edges, plabels)
    return oracle.count(g, p.k, p.edges, plabels=plabels, vertex_induced=(mode == "vertex"),
                        restrictions=restr or (), **kw)


# ------------------------------------------------------------------ brute force
@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("mode", ["edge", "vertex"])
def test_brute_force_small_graphs(seed, mode):
    """Pin: the definition tested literally on every injective map."""
    rng = np.random.default_rng(seed)
    n = 7 + seed % 2
    g = stmgen.er(n, int(rng.integers(8, 16)), 1000 + seed)
    g.labels = stmgen.labels(n, 2, 77 + seed)
    for name in SMALL_PATTERNS:
        p = CATALOG[name]
        if p.k > 5:
            continue
        pl = tuple(int(x) for x in rng.integers(0, 2, p.k))
        for restr in (None, "auto"):
            for lab in (None, pl):
                R = oracle.gk_restrictions(p.k, p.edges, lab) if restr == "auto" else []
                want = oracle.brute_force_count(g, p.k, p.edges, lab, mode == "vertex", R)
                got = ocount(g, p, mode, R, lab, threads=2)
                assert got == want, (name, mode, restr, lab)


def test_brute_force_random_restrictions():
    """Pin: caller-given (non-automorphism) restriction pairs, brute force."""
    rng = np.random.default_rng(5)
    g = stmgen.er(8, 16, 4242)
    for name in ["path4", "c4", "diamond", "house"]:
        p = CATALOG[name]
        for _ in range(3):
            perm = rng.permutation(p.k)
            R = [(int(perm[i]), int(perm[j])) for i in range(p.k) for j in range(i + 1, p.k)
                 if rng.random() < 0.4]
            for mode in ("edge", "vertex"):
                want = oracle.brute_force_count(g, p.k, p.edges, None, mode == "vertex", R)
                assert ocount(g, p, mode, R, threads=3) == want


# ------------------------------------------------------------------ closed forms
@pytest.mark.parametrize("name", SMALL_PATTERNS + ["k6", "octahedron", "prism", "w5", "c6"])
def test_complete_graph_closed_forms(name):
    """Pin: in K_n every injective map is an edge-induced embedding -> n!/(n-k)!;
    AUTO restrictions give the number of copies C(n,k) k!/|Aut|; vertex-induced
    non-cliques never occur."""
    p = CATALOG[name]
    n = 8
    g = stmgen.complete(n)
    aut = len(oracle.automorphisms(p.k, p.edges))
    assert ocount(g, p) == math.perm(n, p.k)
    assert ocount(g, p, restr="auto") == math.comb(n, p.k) * math.factorial(p.k) // aut
    clique = len(p.edges) == p.k * (p.k - 1) // 2
    want_vi = math.perm(n, p.k) if clique else 0
    assert ocount(g, p, "vertex") == want_vi


@pytest.mark.parametrize("n", [5, 6, 7])
def test_cycle_graph(n):
    """Pin: C_n contains exactly one n-cycle (2n embeddings) and no shorter cycle."""
    g = stmgen.cycle(n)
    for k in (5, 6, 7):
        p = CATALOG[f"c{k}"]
        assert ocount(g, p, restr="auto") == (1 if k == n else 0)
        assert ocount(g, p) == (2 * n if k == n else 0)
    assert ocount(g, CATALOG["triangle"]) == 0


@pytest.mark.parametrize("a,b", [(3, 3), (3, 4), (4, 5)])
def test_grid_closed_forms(a, b):
    """Pin: a x b grid: C4 = (a-1)(b-1) both modes; C6 = (a-2)(b-1)+(a-1)(b-2)
    edge-induced, 0 vertex-induced; no odd cycles (bipartite)."""
    g = stmgen.grid(a, b)
    for mode in ("edge", "vertex"):
        assert ocount(g, CATALOG["c4"], mode, "auto") == (a - 1) * (b - 1)
        assert ocount(g, CATALOG["c5"], mode, "auto") == 0
        assert ocount(g, CATALOG["triangle"], mode, "auto") == 0
    assert ocount(g, CATALOG["c6"], "edge", "auto") == (a - 2) * (b - 1) + (a - 1) * (b - 2)
    assert ocount(g, CATALOG["c6"], "vertex", "auto") == 0


def _degree_forms(g):
    A = adj_matrix(g)
    d = np.asarray(A.sum(1)).ravel().astype(np.int64)
    A2 = (A @ A).tocsr()
    tri = int(round(A2.multiply(A).sum() / 6))
    wedges = int(sum(int(x) * (int(x) - 1) // 2 for x in d))
    # edge-induced 4-cycles: 1/2 sum_{i<j} C(codeg(i,j), 2), codeg from A^2 off-diagonal
    A2.setdiag(0)
    A2.eliminate_zeros()
    cod = A2.data.astype(np.int64)
    c4 = int((cod * (cod - 1) // 2).sum() // 2 // 2)
    return d, tri, wedges, c4


@pytest.mark.parametrize("gen", ["c1", "rmat12"])
def test_degree_and_trace_closed_forms(gen):
    """Pin: triangles = tr(A^3)/6 (scipy), wedges = sum C(d,2), induced wedges =
    sum C(d,2) - 3T, k-stars = sum C(d,k-1), 4-cycles = 1/2 sum_{i<j} C(codeg,2),
    single edges = m (AUTO) / 2m."""
    g = stmgen.config_graph("c1") if gen == "c1" else stmgen.rmat(12, 20000, 0.57, 0.19, 0.19, 9)
    d, tri, wedges, c4 = _degree_forms(g)
    assert ocount(g, CATALOG["triangle"], restr="auto") == tri
    assert ocount(g, CATALOG["wedge"], restr="auto") == wedges
    assert ocount(g, CATALOG["wedge"], "vertex", "auto") == wedges - 3 * tri
    assert ocount(g, CATALOG["star4"], restr="auto") == int(sum(math.comb(int(x), 3) for x in d))
    assert ocount(g, CATALOG["c4"], restr="auto") == c4
    assert ocount(g, CATALOG["edge"], restr="auto") == g.m
    assert ocount(g, CATALOG["edge"]) == 2 * g.m


# ------------------------------------------------------------------ networkx VF2
def test_networkx_vf2_labeled():
    """Pin: an independent matcher (networkx VF2; monomorphisms = edge-induced,
    isomorphisms = vertex-induced, categorical node match for labels)."""
    nx = pytest.importorskip("networkx")
    from networkx.algorithms import isomorphism as iso
    g = stmgen.er(40, 120, 31)
    g.labels = stmgen.labels(g.n, 3, 32)
    G = nx.Graph()
    G.add_nodes_from((v, {"label": int(g.labels[v])}) for v in range(g.n))
    for v in range(g.n):
        for w in g.neighbors(v):
            if v < w:
                G.add_edge(v, int(w))
    rng = np.random.default_rng(3)
    for name in ["c4", "diamond", "house", "c5", "tailed_triangle"]:
        p = CATALOG[name]
        pl = tuple(int(x) for x in rng.integers(0, 3, p.k))
        Q = nx.Graph()
        Q.add_nodes_from((u, {"label": pl[u]}) for u in range(p.k))
        Q.add_edges_from(p.edges)
        nm = iso.categorical_node_match("label", None)
        mono = sum(1 for _ in iso.GraphMatcher(G, Q, node_match=nm).subgraph_monomorphisms_iter())
        isom = sum(1 for _ in iso.GraphMatcher(G, Q, node_match=nm).subgraph_isomorphisms_iter())
        assert ocount(g, p, "edge", None, pl) == mono
        assert ocount(g, p, "vertex", None, pl) == isom
        mono_u = sum(1 for _ in iso.GraphMatcher(G, Q).subgraph_monomorphisms_iter())
        assert ocount(g, p, "edge") == mono_u


# ------------------------------------------------------------------ symmetry
KNOWN_AUT = {"triangle": 6, "k4": 24, "c4": 8, "c5": 10, "house": 2, "diamond": 4, "c6": 12,
             "prism": 12, "octahedron": 48, "w5": 10, "w6": 12, "k6_minus_e": 48,
             "k7_minus_e": 240, "k5": 120, "k6": 720, "c7": 14, "star4": 6, "path4": 2}


@pytest.mark.parametrize("name", sorted(KNOWN_AUT))
def test_known_automorphism_orders(name):
    """Pin: textbook automorphism group orders (|Aut(C_n)| = 2n, |Aut(K_n)| = n!,
    |Aut(W_n)| = 2(n-1) for rim >= 4, K_{2,2,2}: 48, prism: 12, ...)."""
    p = CATALOG[name]
    assert len(oracle.automorphisms(p.k, p.edges)) == KNOWN_AUT[name]


@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "house", "c5", "k4", "path4",
                                  "star4", "tailed_triangle", "prism", "w5"])
def test_restricted_times_aut_equals_unrestricted(name):
    """Invariant: (count with GK restrictions) x |Aut_L(Q)| = unrestricted count,
    labeled and unlabeled, both modes."""
    p = CATALOG[name]
    g = stmgen.er(60, 400, 11)
    g.labels = stmgen.labels(g.n, 2, 12)
    for pl in (None, tuple([0, 1] * 4)[:p.k]):
        aut = len(oracle.automorphisms(p.k, p.edges, pl))
        for mode in ("edge", "vertex"):
            assert ocount(g, p, mode, "auto", pl) * aut == ocount(g, p, mode, None, pl)


def test_gk_restrictions_match_survey_derivation():
    """Pin: the GK restriction sets SURVEY.md 8(c) derived independently (networkx
    automorphism groups) for the same vertex numbering."""
    want = {"triangle": [(0, 1), (0, 2), (1, 2)], "c4": [(0, 1), (0, 2), (0, 3), (1, 3)],
            "c5": [(0, 1), (0, 2), (0, 3), (0, 4), (1, 4)], "house": [(0, 1)],
            "diamond": [(0, 3), (1, 2)]}
    for name, R in want.items():
        p = CATALOG[name]
        assert oracle.gk_restrictions(p.k, p.edges) == R, name


def test_label_sum_invariant():
    """Invariant: summing the unrestricted labeled count over all L^k pattern
    labelings gives the unlabeled count."""
    g = stmgen.er(30, 90, 5)
    g.labels = stmgen.labels(g.n, 2, 6)
    for name in ["triangle", "c4", "diamond"]:
        p = CATALOG[name]
        for mode in ("edge", "vertex"):
            tot = sum(ocount(g, p, mode, None, pl, threads=2)
                      for pl in itertools.product(range(2), repeat=p.k))
            assert tot == ocount(g, p, mode)


def test_order_invariance_and_relabel_invariance():
    """Invariant: the count does not depend on the matching order (every root
    pattern vertex) nor, with complete restrictions, on the vertex numbering."""
    g = stmgen.rmat(10, 6000, 0.57, 0.19, 0.19, 21)
    g2 = stmgen.relabel(g, 99)
    for name in ["diamond", "house", "c5", "k4"]:
        p = CATALOG[name]
        for mode in ("edge", "vertex"):
            ref = ocount(g, p, mode, "auto")
            for u in range(p.k):
                assert ocount(g, p, mode, "auto", root_u=u) == ref
            assert ocount(g2, p, mode, "auto") == ref


def test_disjoint_union_additivity():
    """Invariant: for connected Q, count(G1 + G2) = count(G1) + count(G2)."""
    g1 = stmgen.er(50, 300, 1)
    g2 = stmgen.rmat(7, 700, 0.57, 0.19, 0.19, 2)
    g = stmgen.disjoint_union(g1, g2)
    for name in ["triangle", "c4", "house"]:
        p = CATALOG[name]
        assert ocount(g, p, restr="auto") == ocount(g1, p, restr="auto") + ocount(g2, p, restr="auto")


def test_per_root_and_root_subsets():
    """Per-root attribution sums to the total; a root subset counts only its roots."""
    g = stmgen.er(200, 1200, 8)
    p = CATALOG["diamond"]
    R = oracle.gk_restrictions(p.k, p.edges)
    tot, pr = oracle.count(g, p.k, p.edges, restrictions=R, root_u=0, per_root=True)
    assert int(pr.sum()) == tot
    roots = np.arange(0, g.n, 7)
    sub, prs = oracle.count(g, p.k, p.edges, restrictions=R, root_u=0, roots=roots, per_root=True)
    assert sub == int(pr[roots].sum()) and np.array_equal(prs, pr[roots])


def test_degenerate_inputs():
    """Empty graph, k > n, isolated vertices: count 0; rejects invalid patterns."""
    p = CATALOG["triangle"]
    assert ocount(stmgen.empty(10), p) == 0
    assert ocount(stmgen.complete(2), p) == 0
    assert ocount(stmgen.empty(0), p) == 0
    with pytest.raises(ValueError):
        oracle.count(stmgen.complete(4), 4, [(0, 1), (2, 3)])  # disconnected pattern


# ------------------------------------------------------------------ listing (NEXT-1)
@pytest.mark.parametrize("seed", range(3))
@pytest.mark.parametrize("mode", ["edge", "vertex"])
def test_listing_equals_brute_force(seed, mode):
    """Pin: the oracle's listing (PAPER.md:75 Output(C, iter)) is exactly the set of
    maps that satisfy the definition, found by brute force over all injective maps."""
    rng = np.random.default_rng(40 + seed)
    n = 7
    g = stmgen.er(n, int(rng.integers(9, 15)), 2000 + seed)
    g.labels = stmgen.labels(n, 2, 88 + seed)
    for name in ["triangle", "path4", "c4", "diamond", "house", "star4"]:
        p = CATALOG[name]
        pl = tuple(int(x) for x in rng.integers(0, 2, p.k))
        for lab in (None, pl):
            for R in ([], oracle.gk_restrictions(p.k, p.edges, lab)):
                want = oracle.brute_force_list(g, p.k, p.edges, lab, mode == "vertex", R)
                got = oracle.list_embeddings(g, p.k, p.edges, lab, mode == "vertex", R, threads=2)
                assert np.array_equal(got, want), (name, mode, lab, R)


def test_listing_orbits_cover_unrestricted():
    """Invariant: the automorphism images of the restricted (distinct-subgraph) listing
    are exactly the unrestricted listing, each embedding once (|Aut| * restricted =
    unrestricted, element by element) -- on a graph too large for brute force."""
    g = stmgen.er(60, 420, 31)
    for name in ["c4", "diamond", "house", "k4", "c5"]:
        p = CATALOG[name]
        R = oracle.gk_restrictions(p.k, p.edges)
        res = oracle.list_embeddings(g, p.k, p.edges, restrictions=R)
        full = oracle.list_embeddings(g, p.k, p.edges)
        aut = oracle.automorphisms(p.k, p.edges)
        imgs = np.concatenate([res[:, [a.index(u) for u in range(p.k)]] for a in aut]) if res.size else res
        imgs = imgs[np.lexsort(imgs.T[::-1])] if imgs.size else imgs
        assert imgs.shape[0] == full.shape[0] == res.shape[0] * len(aut)
        assert np.array_equal(imgs, full), name


def test_listing_truncates_at_capacity():
    g = stmgen.er(40, 200, 5)
    p = CATALOG["triangle"]
    full = oracle.list_embeddings(g, p.k, p.edges)
    part = oracle.list_embeddings(g, p.k, p.edges, capacity=5)
    assert part.shape == (5, 3) and all(tuple(r) in {tuple(x) for x in full} for r in part)
