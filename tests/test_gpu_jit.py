"""Plan-specialised kernels (jit.cpp, stm_tuning.jit): the counting kernel compiled once more per
plan with the plan and the frame as compile-time constants must count exactly what the oracle
counts -- every pattern shape (fused and frame count modes, k = 3..7), both induced modes,
labels, custom restrictions, both register variants, stealing on and off.  The kernel source is
the generic one; what changes is only constant folding, so these cases pin the specialisation
(frame dispatch per level, folded plan lookups) against the oracle."""
import pytest

import oracle
import stmgen
from stmgen import CATALOG

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover - CPU container
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_sc_weij22_b200 import stm  # noqa: E402  (fails loudly if libstm.so is missing)


@pytest.fixture(scope="module")
def er_small():
    g = stmgen.er(300, 2500, 7)
    return g, stm.Graph.from_stmgen(g)


@pytest.fixture(scope="module")
def rmat_small():
    g = stmgen.rmat(10, 4000, 0.57, 0.19, 0.19, 17)
    g.labels = stmgen.labels(g.n, 4, 18)
    return g, stm.Graph.from_stmgen(g)


def _count(G, p, vi, lab=None, **tk):
    plan = stm.Plan(p.k, p.edges, lab, vertex_induced=vi)
    c = stm.count(G, plan, stm.stm_tuning_default(jit=1, **tk))
    assert stm.stm_last_launch()["jit"] == 1
    return c


def _oracle(g, p, vi, lab=None):
    return oracle.count(g, p.k, p.edges, plabels=lab, vertex_induced=vi,
                        restrictions=oracle.gk_restrictions(p.k, p.edges, lab))


@pytest.mark.parametrize("name,vi", [("triangle", False), ("k4", False), ("c4", True), ("diamond", True),
                                     ("house", False), ("k5", False), ("c5", True), ("k6_minus_e", False),
                                     ("prism", True), ("c6", False), ("w6", False)])
def test_jit_patterns(rmat_small, name, vi):
    g, G = rmat_small
    p = CATALOG[name]
    assert _count(G, p, vi) == _oracle(g, p, vi)


@pytest.mark.parametrize("tk", [dict(occupancy=1), dict(occupancy=2), dict(local_steal=0, global_steal=0),
                                dict(stop_level=8, root_chunk=1, unroll=2), dict(vertex_order=1),
                                dict(chunk_cost=1, root_split=3)])
def test_jit_tunings(rmat_small, tk):
    g, G = rmat_small
    for name, vi in [("k4", False), ("house", True), ("c5", False)]:
        p = CATALOG[name]
        assert _count(G, p, vi, **tk) == _oracle(g, p, vi), (name, vi, tk)


def test_jit_labeled(rmat_small):
    g, G = rmat_small
    for name, lab in [("c4", (0, 1, 0, 2)), ("diamond", (1, 0, 0, 1)), ("house", (0, 1, 2, 0, 1))]:
        p = CATALOG[name]
        for vi in (False, True):
            assert _count(G, p, vi, lab) == _oracle(g, p, vi, lab), (name, lab, vi)


def test_jit_custom_restrictions(er_small):
    g, G = er_small
    p = CATALOG["c4"]
    for R in ([], [(0, 2)], [(0, 1), (0, 2), (0, 3), (1, 3)]):
        plan = stm.Plan(p.k, p.edges, restrictions=R)
        got = stm.count(G, plan, stm.stm_tuning_default(jit=1))
        assert stm.stm_last_launch()["jit"] == 1
        assert got == oracle.count(g, p.k, p.edges, restrictions=R), R


def test_jit_off_runs_generic(rmat_small):
    g, G = rmat_small
    p = CATALOG["k4"]
    plan = stm.Plan(p.k, p.edges)
    assert stm.count(G, plan, stm.stm_tuning_default(jit=-1)) == _oracle(g, p, False)
    assert stm.stm_last_launch()["jit"] == 0
