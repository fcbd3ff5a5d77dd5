"""Motif catalog on the CPU: the connected graphs on k vertices
up to isomorphism.  Pinned by counts known independently of this code: 1, 2, 6, 21, 112
unlabeled connected graphs on k = 2..6 vertices (OEIS A001349), and the orbit-stabiliser
identity sum_motifs k!/|Aut| = number of labeled connected graphs on k vertices
(1, 4, 38, 728, 26704; OEIS A001187).  The census itself is GPU parity
(tests/test_gpu_parity.py::test_motif_census)."""
import itertools
import math

import pytest


@pytest.fixture(scope="module")
def stm():
    from paper_conf_sc_weij22_b200 import build
    build.build()
    from paper_conf_sc_weij22_b200 import stm as m
    return m


def canon(k, edges):
    return min(tuple(sorted(tuple(sorted((p[a], p[b]))) for a, b in edges)) for p in itertools.permutations(range(k)))


def aut(k, edges):
    E = {tuple(sorted(e)) for e in edges}
    return sum(all(tuple(sorted((p[a], p[b]))) in E for a, b in E) for p in itertools.permutations(range(k)))


def is_connected(k, edges):
    seen, stack = {0}, [0]
    while stack:
        u = stack.pop()
        for a, b in edges:
            for x, y in ((a, b), (b, a)):
                if x == u and y not in seen:
                    seen.add(y)
                    stack.append(y)
    return len(seen) == k


@pytest.mark.parametrize("k,n_unlabeled,n_labeled", [(2, 1, 1), (3, 2, 4), (4, 6, 38), (5, 21, 728),
                                                      (6, 112, 26704)])
def test_catalog_counts(stm, k, n_unlabeled, n_labeled):
    cat = stm.stm_motif_catalog(k)
    assert len(cat) == n_unlabeled
    assert all(is_connected(k, m) for m in cat)
    assert all(a < b for m in cat for a, b in m)
    assert [len(m) for m in cat] == sorted(len(m) for m in cat)
    if k <= 5:  # pairwise non-isomorphic (k = 6 is implied by the labeled count below)
        assert len({canon(k, m) for m in cat}) == n_unlabeled
    assert sum(math.factorial(k) // aut(k, m) for m in cat) == n_labeled


def test_catalog_k4_shapes(stm):
    # star, path, triangle+tail, 4-cycle, diamond, K4
    assert sorted(len(m) for m in stm.stm_motif_catalog(4)) == [3, 3, 4, 4, 5, 6]


def test_errors(stm):
    with pytest.raises(stm.StmError):
        stm.stm_motif_catalog(7)
    with pytest.raises(stm.StmError):
        stm.stm_motif_catalog(1)
    with pytest.raises(stm.StmError):
        stm.stm_motif_census(None, 4)
