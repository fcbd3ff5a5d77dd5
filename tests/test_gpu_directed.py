"""Directed graphs (NEXT-4; "supports both directed and undirected graphs") on the
GPU through the C ABI: stm_graph_load_directed + STM_DIRECTED plans vs the directed oracle
(oracle.count_directed, pinned in tests/test_oracle_directed.py), bit-exact: directed patterns
with one-way and mutual arcs, both induced modes, labels, scheduler switches, both kernels."""
import numpy as np
import pytest

import oracle
import stmgen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU container
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_sc_weij22_b200 import stm  # noqa: E402

from test_oracle_directed import PATTERNS  # noqa: E402


class DG:
    pass


def orient(g, seed, p_both=0.2):
    """A digraph from an undirected graph: each edge becomes a -> b, b -> a, or both (p_both)."""
    rng = np.random.default_rng(seed)
    out = [[] for _ in range(g.n)]
    for a in range(g.n):
        for b in g.col_idx[g.row_ptr[a]:g.row_ptr[a + 1]]:
            b = int(b)
            if b <= a:
                continue
            r = rng.random()
            if r < p_both:
                out[a].append(b)
                out[b].append(a)
            elif r < (1 + p_both) / 2:
                out[a].append(b)
            else:
                out[b].append(a)
    d = DG()
    d.n = g.n
    d.row_ptr = np.zeros(g.n + 1, dtype=np.int64)
    d.row_ptr[1:] = np.cumsum([len(x) for x in out])
    d.col_idx = np.array([y for x in out for y in sorted(x)], dtype=np.int32)
    d.labels = g.labels
    return d


@pytest.fixture(scope="module")
def dg_hubs():
    g = stmgen.rmat(10, 5000, 0.57, 0.19, 0.19, 23)
    g.labels = stmgen.labels(g.n, 3, 4)
    d = orient(g, 7)
    return d, stm.Graph(d.n, d.row_ptr, d.col_idx, d.labels, directed=True)


def _gpu(G, k, arcs, vi=False, lab=None, **tk):
    plan = stm.Plan(k, arcs, lab, vertex_induced=vi, directed=True)
    return stm.count(G, plan, stm.stm_tuning_default(**tk))


def _orc(d, k, arcs, vi=False, lab=None):
    return oracle.count_directed(d, k, arcs, lab, vi, oracle.gk_restrictions_directed(k, arcs, lab))


@pytest.mark.parametrize("name", sorted(PATTERNS))
@pytest.mark.parametrize("vi", [False, True])
def test_directed_patterns(dg_hubs, name, vi):
    d, G = dg_hubs
    k, arcs = PATTERNS[name]
    want = _orc(d, k, arcs, vi)
    assert _gpu(G, k, arcs, vi) == want
    assert _gpu(G, k, arcs, vi, jit=1) == want  # the plan-specialised kernel
    assert stm.stm_last_launch()["jit"] == 1


def test_directed_labeled(dg_hubs):
    d, G = dg_hubs
    for name in ("cycle3", "feed_forward4", "mutual_path", "bifan"):
        k, arcs = PATTERNS[name]
        lab = tuple(u % 3 for u in range(k))
        for vi in (False, True):
            assert _gpu(G, k, arcs, vi, lab) == _orc(d, k, arcs, vi, lab), (name, vi)


@pytest.mark.parametrize("tk", [dict(local_steal=0, global_steal=0), dict(stop_level=8, root_chunk=1, unroll=2),
                                dict(occupancy=2), dict(occupancy=1, unroll=32), dict(chunk_cost=1),
                                dict(block_warps=32, blocks_per_sm=1), dict(narrow_split=1)])
def test_directed_tunings(dg_hubs, tk):
    d, G = dg_hubs
    for name, vi in (("cycle3", False), ("feed_forward4", True), ("cycle4", False)):
        k, arcs = PATTERNS[name]
        assert _gpu(G, k, arcs, vi, **tk) == _orc(d, k, arcs, vi), (name, vi, tk)


def test_directed_custom_restrictions(dg_hubs):
    d, G = dg_hubs
    k, arcs = PATTERNS["cycle4"]
    for R in ([], [(0, 2)], [(0, 1), (0, 2), (0, 3)]):
        plan = stm.Plan(k, arcs, restrictions=R, directed=True)
        assert stm.count(G, plan) == oracle.count_directed(d, k, arcs, restrictions=R), R


def test_symmetric_digraph_matches_undirected():
    """Both arcs of every edge + a pattern of mutual arcs = the undirected count (GPU both ways)."""
    g = stmgen.rmat(9, 2000, 0.57, 0.19, 0.19, 5)
    G = stm.Graph.from_stmgen(g)
    D = stm.Graph(g.n, g.row_ptr, g.col_idx, directed=True)  # a symmetric CSR read as out-rows
    for name in ("triangle", "c4", "diamond", "house"):
        p = stmgen.CATALOG[name]
        arcs = list(p.edges) + [(b, a) for a, b in p.edges]
        for vi in (False, True):
            assert stm.count(D, stm.Plan(p.k, arcs, vertex_induced=vi, directed=True)) == \
                stm.count(G, stm.Plan(p.k, p.edges, vertex_induced=vi)), (name, vi)


def test_directed_mismatch_rejected(dg_hubs):
    d, G = dg_hubs
    with pytest.raises(stm.StmError):
        stm.count(G, stm.Plan(3, [(0, 1), (1, 2), (0, 2)]))  # undirected plan on a directed graph


@pytest.mark.parametrize("rows,why", [
    ([[1], []], "not symmetric"),                  # 0 -> 1 without 1 -> 0
    ([[0, 1], [0]], "self-loop"),
    ([[2, 1], [0], [0]], "strictly increasing"),
    ([[1, 7], [0]], "out of range"),
])
def test_graph_validation(rows, why):
    """stm_graph_load rejects what is not an undirected simple graph (entry checks on the device);
    stm_graph_load_directed accepts one-way arcs but rejects the rest."""
    n = len(rows)
    rp = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int64)
    ci = np.array([x for r in rows for x in r], dtype=np.int32)
    with pytest.raises(stm.StmError) as ei:
        stm.Graph(n, rp, ci)
    assert ei.value.status == stm.STM_EINVAL and why in str(ei.value)
    if why == "not symmetric":
        stm.Graph(n, rp, ci, directed=True).close()
    else:
        with pytest.raises(stm.StmError):
            stm.Graph(n, rp, ci, directed=True)
