"""GPU parity: the CUDA path (through the C ABI) vs the oracle, bit-exact.

Every count here is an exact integer; the bar is equality.
"""
import itertools

import numpy as np
import pytest

import oracle
import stmgen
from stmgen import CATALOG

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU container
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_sc_weij22_b200 import stm  # noqa: E402  (fails loudly if libstm.so is missing)

SMALL = ["edge", "wedge", "triangle", "path4", "star4", "c4", "diamond", "tailed_triangle", "k4",
         "house", "c5", "k5"]
BIG = ["k6", "k6_minus_e", "octahedron", "w5", "prism", "c6", "k7_minus_e", "w6", "c7"]


def ocount(g, p, vi, labels=None, restr="auto", threads=0):
    R = oracle.gk_restrictions(p.k, p.edges, labels) if restr == "auto" else restr
    return oracle.count(g, p.k, p.edges, plabels=labels, vertex_induced=vi, restrictions=R,
                        threads=threads)


def gcount(G, p, vi, labels=None, restr="auto", tuning=None, **kw):
    if restr == "auto":
        plan = stm.Plan(p.k, p.edges, labels, vertex_induced=vi, **kw)
    else:
        plan = stm.Plan(p.k, p.edges, labels, restrictions=restr, auto_restrict=False, vertex_induced=vi, **kw)
    return stm.count(G, plan, tuning)


@pytest.fixture(scope="module")
def er_small():
    g = stmgen.er(300, 2500, 7)
    g.labels = stmgen.labels(g.n, 3, 8)
    return g, stm.Graph.from_stmgen(g)


@pytest.fixture(scope="module")
def er_sparse():
    g = stmgen.er(300, 1500, 9)
    return g, stm.Graph.from_stmgen(g)


@pytest.fixture(scope="module")
def rmat_small():
    # hubs (max degree ~250 of 1024 vertices) so that stealing and long/short operands mix
    g = stmgen.rmat(10, 4000, 0.57, 0.19, 0.19, 17)
    g.labels = stmgen.labels(g.n, 4, 18)
    return g, stm.Graph.from_stmgen(g)


@pytest.mark.parametrize("name", SMALL)
@pytest.mark.parametrize("vi", [False, True])
def test_small_patterns_er(er_small, name, vi):
    g, G = er_small
    p = CATALOG[name]
    assert gcount(G, p, vi) == ocount(g, p, vi)


@pytest.mark.parametrize("name", SMALL + ["k6", "k6_minus_e", "k7_minus_e", "octahedron"])
@pytest.mark.parametrize("vi", [False, True])
def test_patterns_rmat_hubs(rmat_small, name, vi):
    g, G = rmat_small
    p = CATALOG[name]
    assert gcount(G, p, vi) == ocount(g, p, vi)


@pytest.mark.parametrize("name", ["w5", "prism", "c6", "c7", "w6", "k8"])
@pytest.mark.parametrize("vi", [False, True])
def test_size6_8_sparse(er_sparse, name, vi):
    g, G = er_sparse
    p = CATALOG[name]
    assert gcount(G, p, vi) == ocount(g, p, vi)


def test_size6_7_hubs_vertex_induced(rmat_small):
    g, G = rmat_small
    for name in ["w5", "prism", "c6"]:
        p = CATALOG[name]
        assert gcount(G, p, True) == ocount(g, p, True), name


@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "house", "c5", "k4", "tailed_triangle"])
@pytest.mark.parametrize("vi", [False, True])
def test_labeled(rmat_small, name, vi):
    g, G = rmat_small
    p = CATALOG[name]
    rng = np.random.default_rng(hash(name) % 1000)
    for _ in range(3):
        pl = tuple(int(x) for x in rng.integers(0, 4, p.k))
        assert gcount(G, p, vi, pl) == ocount(g, p, vi, pl)


@pytest.mark.parametrize("name", ["c4", "house", "diamond", "path4", "c5"])
def test_unrestricted_and_custom_restrictions(er_small, name):
    g, G = er_small
    p = CATALOG[name]
    for vi in (False, True):
        assert gcount(G, p, vi, restr=[]) == ocount(g, p, vi, restr=[])
        R = [(1, 0)] if p.k > 1 else []
        assert gcount(G, p, vi, restr=R) == ocount(g, p, vi, restr=R)


TUNINGS = [
    dict(local_steal=0, global_steal=0),
    dict(local_steal=1, global_steal=0),
    dict(local_steal=1, global_steal=1),
    dict(local_steal=0, global_steal=1),
    dict(unroll=1), dict(unroll=2), dict(unroll=16),
    dict(root_chunk=1, stop_level=3, detect_level=3),
    dict(block_warps=4), dict(block_warps=32, blocks_per_sm=1),
    dict(vertex_order=1), dict(vertex_order=1, unroll=1, local_steal=0, global_steal=0),
    dict(root_chunk=32), dict(root_chunk=7, unroll=3),
    dict(bitmap_min_degree=1), dict(bitmap_min_degree=-1), dict(bitmap_min_degree=1, vertex_order=1),
    dict(bitmap_min_degree=40, unroll=1),
    dict(narrow_split=1), dict(narrow_split=1, vertex_order=1, bitmap_min_degree=-1),
    dict(occupancy=2), dict(occupancy=2, unroll=32, vertex_order=1), dict(occupancy=1, unroll=32),
    dict(occupancy=2, unroll=5, root_chunk=1, stop_level=3, detect_level=3),
    dict(root_order=1), dict(root_order=2, vertex_order=1), dict(root_order=2, root_chunk=3, occupancy=2),
    dict(l2_persist_mb=8, occupancy=2),
    dict(root_split=-1), dict(root_split=1), dict(root_split=3, root_chunk=5, stop_level=3),
    dict(root_split=2, vertex_order=1, root_order=2), dict(root_split=4, root_chunk=1, unroll=2),
    dict(backoff_max=1, carveout_pct=-1), dict(backoff_max=12, carveout_pct=50),
    # donation at every frame (split kinds 2 and 3 below frame 1), small batches, one big block
    dict(stop_level=8, root_chunk=1, unroll=2), dict(stop_level=8, detect_level=8, unroll=1, root_split=1),
    dict(stop_level=8, block_warps=32, blocks_per_sm=1, root_chunk=1),
    # work-balanced chunks: off, one position per chunk, descending, one huge chunk
    dict(chunk_cost=-1), dict(chunk_cost=1), dict(chunk_cost=64, root_order=2, root_chunk=3),
    dict(chunk_cost=1 << 30, root_split=-1), dict(chunk_cost=40, vertex_order=1, root_split=-1),
]


@pytest.mark.parametrize("name", SMALL + ["k6_minus_e", "octahedron", "w5"])
@pytest.mark.parametrize("vi", [False, True])
def test_hub_bitmaps(rmat_small, name, vi):
    """Hub bitmaps (every vertex, caller's and degree-ranked numbering, labeled and not)
    change only how membership is probed, never the count."""
    g, G = rmat_small
    p = CATALOG[name]
    want = ocount(g, p, vi)
    for vo in (0, 1):
        t = stm.stm_tuning_default(bitmap_min_degree=1, vertex_order=vo)
        assert gcount(G, p, vi, tuning=t) == want, (name, vi, vo)
        assert stm.stm_last_launch()["hubs"] > 0
    pl = tuple(int(x) for x in np.random.default_rng(p.k).integers(0, 4, p.k))
    t = stm.stm_tuning_default(bitmap_min_degree=8)
    assert gcount(G, p, vi, pl, tuning=t) == ocount(g, p, vi, pl)


@pytest.mark.parametrize("tk", range(len(TUNINGS)))
def test_tuning_invariance(rmat_small, tk):
    """Every scheduler switch (ablation of Fig. 12) leaves the count unchanged."""
    g, G = rmat_small
    t = stm.stm_tuning_default(**TUNINGS[tk])
    for name, vi in [("k4", False), ("house", True), ("c5", False), ("diamond", True), ("triangle", False)]:
        p = CATALOG[name]
        assert gcount(G, p, vi, tuning=t) == ocount(g, p, vi), (name, vi, TUNINGS[tk])


@pytest.mark.parametrize("name", ["house", "diamond", "c5", "k5", "prism"])
def test_code_motion_and_order_invariance(rmat_small, name):
    g, G = rmat_small
    p = CATALOG[name]
    for vi in (False, True):
        want = ocount(g, p, vi)
        assert gcount(G, p, vi, code_motion=False) == want
        for perm in list(itertools.permutations(range(p.k)))[:: max(1, len(list(itertools.permutations(range(p.k)))) // 6)]:
            adj = {u: set() for u in range(p.k)}
            for a, b in p.edges:
                adj[a].add(b)
                adj[b].add(a)
            if all(any(perm[j] in adj[perm[i]] for j in range(i)) for i in range(1, p.k)):
                assert gcount(G, p, vi, order=list(perm)) == want


def test_golden_config_counts():
    """Full-size config graphs against stored oracle counts (tools/make_golden.py,
    fingerprints checked so the very same graph is compared)."""
    import json, os
    path = os.path.join(os.path.dirname(__file__), "golden", "config_counts.json")
    data = json.load(open(path))
    graphs = {}
    for cid, d in sorted(data.items()):
        if d["config"] not in graphs:
            g = stmgen.config_graph(d["config"])
            graphs[d["config"]] = (g, stm.Graph.from_stmgen(g))
        g, G = graphs[d["config"]]
        assert g.fingerprint() == d["fingerprint"], cid
        plan = stm.Plan(d["k"], d["edges"], d["labels"], restrictions=d["restrictions"], auto_restrict=False,
                        vertex_induced=d["vertex_induced"])
        assert stm.count(G, plan) == d["count"], cid
        # the product default: the plan-specialised kernel (jit.cpp) of the compiler's own plan
        plan2 = stm.Plan(d["k"], d["edges"], d["labels"], vertex_induced=d["vertex_induced"])
        assert stm.count(G, plan2, stm.stm_tuning_default(jit=1)) == d["count"], cid + " (specialised kernel)"
        assert stm.stm_last_launch()["jit"] == 1


def stratified_roots(n, sizes, seed=5):
    """Degree-stratified root sample of a degree-ranked graph (vertex i = i-th lowest degree):
    `sizes` roots from ranks [0, n-4096), [n-4096, n-256), [n-256, n-16), [n-16, n)."""
    rng = np.random.default_rng(seed)
    cuts = [0, max(0, n - 4096), max(0, n - 256), max(0, n - 16), n]
    out = [rng.choice(np.arange(a, b), size=min(k, b - a), replace=False)
           for (a, b), k in zip(zip(cuts[:-1], cuts[1:]), sizes) if b > a and k]
    return np.unique(np.concatenate(out))


@pytest.mark.parametrize("cfg,name,sizes", [
    ("c5", "k5", (24, 8, 4, 2)), ("c5", "k6_minus_e", (24, 8, 1, 0)),
    ("c3", "house", (24, 2, 0, 0)), ("c3", "c5", (24, 2, 0, 0)), ("c3", "k5", (24, 8, 4, 2)),
    ("c2", "c4", (24, 8, 2, 0)), ("c2", "k4", (24, 8, 4, 2))])
def test_config_scale_sampled_roots(cfg, name, sizes):
    """At full size, in the bench's launch configuration (degree-ranked copy, default
    tuning): GPU per-root counts on a degree-stratified sample of roots -- the bulk, the
    high-degree strata where the work concentrates, and (where the oracle can afford them)
    the top hubs -- equal the oracle's, run on the same graph renumbered in (degree, id)
    order with matches attributed to f(order[0]) as on the GPU.  The sample must hold
    matches (no zero-versus-zero pass)."""
    g = stmgen.config_graph(cfg)
    G = stm.Graph.from_stmgen(g)
    p = CATALOG[name]
    plan = stm.Plan(p.k, p.edges)
    R = oracle.gk_restrictions(p.k, p.edges)
    tot, pr = stm.stm_match_count_per_root(G.handle, plan.handle, stm.stm_tuning_default(jit=1))
    assert stm.stm_last_launch()["ranked"] == 1 and stm.stm_last_launch()["jit"] == 1
    assert int(pr.sum(dtype=np.uint64)) == tot
    rank2orig, gr = degree_ranked(g)
    roots = stratified_roots(g.n, sizes)
    oc, opr = oracle.count(gr, p.k, p.edges, restrictions=R, root_u=plan.first_vertex, roots=roots, per_root=True)
    assert np.array_equal(pr[rank2orig[roots]], opr)
    assert int(opr.sum()) > 0 and np.count_nonzero(opr) >= 2, "sample holds no matches"


def degree_ranked(g):
    """(rank2orig, g renumbered so that vertex i is the i-th in (degree, id) order)."""
    deg = g.degrees()
    rank2orig = np.lexsort((np.arange(g.n), deg))
    perm = np.empty(g.n, np.int64)
    perm[rank2orig] = np.arange(g.n)
    return rank2orig, stmgen.permute(g, perm)


def test_degenerate_graphs():
    for g in [stmgen.complete(8), stmgen.cycle(7), stmgen.grid(4, 5), stmgen.empty(5)]:
        G = stm.Graph.from_stmgen(g)
        for name in ["triangle", "c4", "k4", "c6", "c7", "house"]:
            p = CATALOG[name]
            for vi in (False, True):
                assert gcount(G, p, vi) == ocount(g, p, vi), (g.name, name, vi)


def test_per_root_histogram(rmat_small):
    """Localisation: GPU per-root counts equal the oracle's, attributed to f(order[0])."""
    g, G = rmat_small
    for name, vi in [("diamond", False), ("house", True), ("k4", False)]:
        p = CATALOG[name]
        plan = stm.Plan(p.k, p.edges, vertex_induced=vi)
        R = oracle.gk_restrictions(p.k, p.edges)
        tot, pr = stm.stm_match_count_per_root(G.handle, plan.handle,
                                               stm.stm_tuning_default(root_chunk=1, vertex_order=1))
        otot, opr = oracle.count(g, p.k, p.edges, vertex_induced=vi, restrictions=R,
                                 root_u=plan.first_vertex, per_root=True)
        assert tot == otot
        assert np.array_equal(pr, opr)
        # degree-ranked (default): attribution to the (degree, id)-minimal root
        tot2, pr2 = stm.stm_match_count_per_root(G.handle, plan.handle, stm.stm_tuning_default(root_chunk=1))
        rank2orig, gr = degree_ranked(g)
        otot2, opr2 = oracle.count(gr, p.k, p.edges, vertex_induced=vi, restrictions=R,
                                   root_u=plan.first_vertex, per_root=True)
        assert tot2 == otot2 == otot
        assert np.array_equal(pr2[rank2orig], opr2)


@pytest.mark.parametrize("name", SMALL + ["k6", "k6_minus_e", "octahedron", "w5", "prism", "c6"])
@pytest.mark.parametrize("vi", [False, True])
def test_lazy_unbounded_code_motion(rmat_small, name, vi):
    """STM_LAZY_UNBOUNDED (bound-split code motion) changes where sets are computed,
    never the count: labeled and unlabeled, both vertex numberings."""
    g, G = rmat_small
    p = CATALOG[name]
    want = ocount(g, p, vi)
    assert gcount(G, p, vi, lazy_unbounded=True) == want, (name, vi)
    t = stm.stm_tuning_default(vertex_order=1, unroll=3)
    assert gcount(G, p, vi, tuning=t, lazy_unbounded=True) == want, (name, vi)
    if p.k <= 6:
        pl = tuple(int(x) for x in np.random.default_rng(p.k + 1).integers(0, 4, p.k))
        assert gcount(G, p, vi, pl, lazy_unbounded=True) == ocount(g, p, vi, pl)


@pytest.mark.parametrize("world", [2, 3, 8])
@pytest.mark.parametrize("peers", [False, True])
@pytest.mark.parametrize("chunk", [0, 3])
def test_sharded_ranks_on_one_gpu(rmat_small, world, peers, chunk):
    """The multi-GPU root partition through the C ABI: `world` ranks'
    launches share one device's cursor array (peer pointers = the other ranks' cursors,
    as torch symmetric memory maps them over NVLink).  Static partition (no peers) and
    cross-rank stealing (peers: the first launch drains every cursor) both cover every
    root chunk exactly once: the partial counts sum to the oracle's count."""
    g, G = rmat_small
    for name, vi in [("k4", False), ("house", True), ("c5", False)]:
        p = CATALOG[name]
        plan = stm.Plan(p.k, p.edges, vertex_induced=vi)
        want = ocount(g, p, vi)
        cur = torch.zeros(world * 8, dtype=torch.int64, device="cuda")
        ptrs = [cur.data_ptr() + 64 * r for r in range(world)]
        parts = []
        for r in range(world):
            sh = stm.make_shard(r, world, chunk, [ptrs[q] if (peers or q == r) else None for q in range(world)])
            parts.append(stm.stm_match_count_ex(G.handle, plan.handle, None, sh, None))
        assert sum(parts) % (1 << 64) == want, (name, world, peers, chunk, parts)
        if peers:
            assert parts[0] == want and all(x == 0 for x in parts[1:])


# ---------------------------------------------------------------- listing (NEXT-1)
def _sorted_rows(a):
    return a[np.lexsort(a.T[::-1])] if a.shape[0] else a


def _canon(rows, aut):
    """Orbit representative of every row: the lexicographically smallest automorphism image."""
    if rows.shape[0] == 0:
        return rows
    imgs = np.stack([rows[:, [a.index(u) for u in range(rows.shape[1])]] for a in aut])  # [|Aut|, m, k]
    best = imgs[0].copy()
    for im in imgs[1:]:
        for i in range(best.shape[0]):
            if tuple(im[i]) < tuple(best[i]):
                best[i] = im[i]
    return _sorted_rows(best)


@pytest.mark.parametrize("name", ["triangle", "c4", "diamond", "house", "k4", "c5", "tailed_triangle", "path4"])
@pytest.mark.parametrize("vi", [False, True])
def test_listing_matches_oracle(er_small, name, vi):
    """stm_match_list rows (caller ids, pattern-vertex order) are exactly the oracle's
    embeddings: caller numbering element by element; degree-ranked numbering (different
    symmetry-breaking representatives of the same subgraphs) orbit by orbit."""
    g, G = er_small
    p = CATALOG[name]
    R = oracle.gk_restrictions(p.k, p.edges)
    want = oracle.list_embeddings(g, p.k, p.edges, vertex_induced=vi, restrictions=R)
    plan = stm.Plan(p.k, p.edges, vertex_induced=vi)
    rows, c = stm.stm_match_list(G.handle, plan.handle, p.k, stm.stm_tuning_default(vertex_order=1),
                                 capacity=want.shape[0] + 5)
    assert c == want.shape[0] and np.array_equal(_sorted_rows(rows), want)
    rows2, c2 = stm.stm_match_list(G.handle, plan.handle, p.k, None, capacity=want.shape[0] + 5)
    assert stm.stm_last_launch()["ranked"] == 1
    aut = oracle.automorphisms(p.k, p.edges)
    assert c2 == c and np.array_equal(_canon(rows2, aut), _canon(want, aut))
    # labeled and unrestricted
    pl = tuple(int(x) for x in np.random.default_rng(p.k).integers(0, 3, p.k))
    want3 = oracle.list_embeddings(g, p.k, p.edges, pl, vi)
    plan3 = stm.Plan(p.k, p.edges, pl, restrictions=[], auto_restrict=False, vertex_induced=vi)
    rows3, c3 = stm.stm_match_list(G.handle, plan3.handle, p.k, None, capacity=want3.shape[0])
    assert c3 == want3.shape[0] and np.array_equal(_sorted_rows(rows3), want3)


def test_listing_pages_and_capacity(rmat_small):
    """Pages of the root space partition the embeddings; a short buffer returns a valid
    subset and the full count (paging by splitting the root range)."""
    g, G = rmat_small
    p = CATALOG["diamond"]
    R = oracle.gk_restrictions(p.k, p.edges)
    want = oracle.list_embeddings(g, p.k, p.edges, restrictions=R)
    plan = stm.Plan(p.k, p.edges)
    t = stm.stm_tuning_default(vertex_order=1)
    cuts = [0, 1, 100, 333, 334, 800, g.n]
    parts, tot = [], 0
    for b, e in zip(cuts[:-1], cuts[1:]):
        rows, c = stm.stm_match_list(G.handle, plan.handle, p.k, t, b, e, capacity=want.shape[0])
        assert rows.shape[0] == c
        if c:
            assert np.all(rows[:, plan.first_vertex] >= b) and np.all(rows[:, plan.first_vertex] < e)
        parts.append(rows)
        tot += c
    assert tot == want.shape[0] and np.array_equal(_sorted_rows(np.concatenate(parts)), want)
    rows, c = stm.stm_match_list(G.handle, plan.handle, p.k, t, capacity=7)
    wanted = {tuple(r) for r in want}
    assert c == want.shape[0] and rows.shape[0] == 7 and all(tuple(r) in wanted for r in rows)
    rows, c = stm.stm_match_list(G.handle, plan.handle, p.k, t, capacity=0)
    assert c == want.shape[0] and rows.shape[0] == 0


def test_compiled_out_options_fail_loudly(er_small):
    """Options whose code path is compiled out of the product build are refused, never ignored."""
    g, G = er_small
    p = CATALOG["triangle"]
    with pytest.raises(stm.StmError, match="STM_EUNSUPPORTED"):
        gcount(G, p, False, tuning=stm.stm_tuning_default(drive_ratio=4))


@pytest.mark.parametrize("name", ["path4", "c4", "tailed_triangle", "house", "c5", "w5", "c6", "prism", "w6"])
@pytest.mark.parametrize("vi", [False, True])
def test_cost_order_counts(rmat_small, name, vi):
    """NEXT-2: the cost-optimal matching order (stm_order_optimize) changes the work,
    never the count -- bit-exact against the oracle, unlabeled and labeled."""
    g, G = rmat_small
    p = CATALOG[name]
    stats = stm.stm_graph_stats_host(g.n, g.row_ptr, g.labels)
    for lab in (None, stmgen.pattern_labels(p.k, 4, 3)):
        plan = stm.Plan(p.k, p.edges, lab, vertex_induced=vi, cost_stats=stats)
        assert stm.count(G, plan) == ocount(g, p, vi, labels=lab)


@pytest.mark.parametrize("k", [3, 4, 5])
@pytest.mark.parametrize("vi", [False, True])
def test_motif_census(rmat_small, k, vi):
    """NEXT-3: every motif of the size-k catalog, bit-exact against the oracle -- merged
    (pattern merging: one launch of the trie plan) and per motif, greedy and
    cost-based orders, with stealing off and forced (root chunk 1, deep stop level)."""
    g, G = rmat_small
    flags = stm.STM_VERTEX_INDUCED if vi else 0
    got = stm.stm_motif_census(G.handle, k, flags)
    if k >= 3:
        assert stm.stm_motif_census_launches() == 1
    cat = stm.stm_motif_catalog(k)
    assert len(got) == len(cat)
    for edges, c in zip(cat, got):
        assert c == oracle.count(g, k, edges, vertex_induced=vi, restrictions=oracle.gk_restrictions(k, edges))
    assert stm.stm_motif_census(G.handle, k, flags | stm.STM_CENSUS_PER_MOTIF) == got
    assert stm.stm_motif_census_launches() == len(cat)
    assert stm.stm_motif_census(G.handle, k, flags | stm.STM_AUTO_ORDER) == got
    stats = stm.stm_graph_stats_host(g.n, g.row_ptr)
    assert stm.stm_motif_census(G.handle, k, flags, stats) == got
    for tk in (dict(local_steal=0, global_steal=0), dict(root_chunk=1, stop_level=4, detect_level=4, unroll=3),
               dict(vertex_order=1, block_warps=4)):
        assert stm.stm_motif_census(G.handle, k, flags, tuning=stm.stm_tuning_default(**tk)) == got, tk


@pytest.mark.parametrize("vi", [False, True])
def test_motif_census_k6_merged(vi):
    """The 112-motif size-6 census in one merged launch, bit-exact against the oracle."""
    g = stmgen.er(90, 330, 31)
    G = stm.Graph.from_stmgen(g)
    flags = stm.STM_VERTEX_INDUCED if vi else 0
    got = stm.stm_motif_census(G.handle, 6, flags)
    assert stm.stm_motif_census_launches() == 1
    cat = stm.stm_motif_catalog(6)
    want = [oracle.count(g, 6, e, vertex_induced=vi, restrictions=oracle.gk_restrictions(6, e)) for e in cat]
    assert got == want
    assert sum(got) > 0


def test_motif_census_sums_to_connected_subsets():
    """Induced motif frequencies partition the connected induced k-vertex subsets
    (brute force over all k-subsets of a small graph)."""
    g = stmgen.er(30, 80, 21)
    G = stm.Graph.from_stmgen(g)
    adj = [set(g.neighbors(v).tolist()) for v in range(g.n)]
    for k in (3, 4, 5, 6):
        want = 0
        for S in itertools.combinations(range(g.n), k):
            seen, stack = {S[0]}, [S[0]]
            while stack:
                u = stack.pop()
                for w in S:
                    if w not in seen and w in adj[u]:
                        seen.add(w)
                        stack.append(w)
            want += len(seen) == k
        assert sum(stm.stm_motif_census(G.handle, k, stm.STM_VERTEX_INDUCED)) == want
