"""C ABI (libstm.so) on the CPU: the library loads, exports every symbol that
include/stm.h declares, and its host-only pattern compiler behaves as the paper
and SURVEY.md 8(b)/(c) specify.  No CUDA device is needed for anything here."""
import ctypes
import os
import re

import pytest

import oracle
import stmgen
from stmgen import CATALOG

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def stm():
    from paper_conf_sc_weij22_b200 import build
    build.build()
    from paper_conf_sc_weij22_b200 import stm as m
    return m


def declared_functions():
    src = open(os.path.join(ROOT, "include", "stm.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?[\w]+\s*\*?\s*(stm_\w+)\s*\(", src, flags=re.M)))


def test_exports_every_declared_symbol(stm):
    names = declared_functions()
    assert len(names) >= 15, names
    lib = ctypes.CDLL(stm.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), f"libstm.so does not export {n}"
    assert set(names) <= set(stm.EXPORTS) | {"stm_tuning_default"}


def _plan_lines(stm, k, edges, **kw):
    p = stm.Plan(k, edges, **kw)
    return p, p.describe().splitlines()


def _strip(line):
    return re.sub(r" lab=.*$", "", line)


def test_golden_diamond_plan(stm):
    """Fig. 1 / Fig. 9a worked example -> tests/golden/diamond_plan.txt."""
    sections, cur = {}, None
    for line in open(os.path.join(ROOT, "tests", "golden", "diamond_plan.txt")):
        line = line.rstrip("\n")
        if not line or line.startswith("#"):
            continue
        if line.startswith("["):
            cur = line.strip("[]")
            sections[cur] = []
        else:
            sections[cur].append(line)
    d = CATALOG["diamond"]
    for sec, kw in [("vertex", dict(vertex_induced=True)), ("edge", dict(vertex_induced=False)),
                    ("vertex_no_code_motion", dict(vertex_induced=True, code_motion=False))]:
        _, lines = _plan_lines(stm, d.k, d.edges, order=[0, 1, 2, 3], **kw)
        got = [_strip(x) for x in lines if re.match(r"(S\d|cand|count)", x)]
        for want in sections[sec]:
            assert want in got, (sec, want, got)


def test_house_plan_exclusion(stm):
    """edge-induced house counts N(v1) & N(v3) excluding {v0, v2}
    with lower bound v3 (v0 really is in N(v1) & N(v3))."""
    h = CATALOG["house"]
    _, lines = _plan_lines(stm, h.k, h.edges)
    assert "order=[2,3,4,0,1]" in lines
    cnt = [x for x in lines if x.startswith("count")][0]
    assert "N(v1) & N(v3)" in cnt and "lo={v3}" in cnt and "excl={v0,v2}" in cnt


def test_clique_plan_one_set_per_level(stm):
    k5 = CATALOG["k5"]
    p, lines = _plan_lines(stm, k5.k, k5.edges)
    assert p.n_sets == 2
    # v0 < v1 < v2 already holds, so only the dominant lower bound v2 is kept
    assert "S1: level 3 stage 0 = S0 & N(v2) lab=any lo={v2} hi={}" in lines


KNOWN_AUT = {"triangle": 6, "k4": 24, "c4": 8, "c5": 10, "house": 2, "diamond": 4, "c6": 12,
             "prism": 12, "octahedron": 48, "w5": 10, "w6": 12, "k6_minus_e": 48, "k7_minus_e": 240,
             "k8": 40320, "c7": 14}


@pytest.mark.parametrize("name", sorted(KNOWN_AUT))
def test_compiler_automorphisms_and_restrictions(stm, name):
    """|Aut| (textbook values) and a complete restriction set: on K_n the restricted
    count must be C(n,k) k!/|Aut| -- checked through the plan's restriction list
    with the ORACLE, i.e. the compiler's restrictions are pinned independently."""
    p = CATALOG[name]
    plan = stm.Plan(p.k, p.edges)
    assert plan.aut == KNOWN_AUT[name]
    if p.k <= 6:
        txt = plan.describe()
        R = [tuple(map(int, x)) for x in re.findall(r"\((\d+),(\d+)\)", txt.split("restrictions=")[1].split("\n")[0])]
        import math
        g = stmgen.complete(7)
        got = oracle.count(g, p.k, p.edges, restrictions=R)
        assert got == math.comb(7, p.k) * math.factorial(p.k) // KNOWN_AUT[name]


def test_labeled_automorphisms(stm):
    c4 = CATALOG["c4"]
    assert stm.Plan(c4.k, c4.edges, labels=[0, 1, 0, 1]).aut == 4
    assert stm.Plan(c4.k, c4.edges, labels=[0, 1, 2, 3]).aut == 1
    assert stm.Plan(c4.k, c4.edges, labels=[5, 5, 5, 5]).aut == 8


@pytest.mark.parametrize("bad", [
    dict(k=1, edges=[(0, 0)]),
    dict(k=3, edges=[(0, 1)]),                   # disconnected (vertex 2 isolated)
    dict(k=4, edges=[(0, 1), (2, 3)]),           # disconnected
    dict(k=3, edges=[(0, 0), (0, 1), (1, 2)]),   # self-loop
    dict(k=3, edges=[(0, 5)]),                   # out of range
    dict(k=3, edges=[(0, 1), (1, 2)], order=[0, 2, 1]),      # order violates PAPER.md:52
    dict(k=3, edges=[(0, 1), (1, 2)], order=[0, 0, 1]),      # not a permutation
    dict(k=3, edges=[(0, 1), (1, 2)], restrictions=[(0, 1), (1, 0)]),  # cyclic
    dict(k=3, edges=[(0, 1), (1, 2)], restrictions=[(1, 1)]),
    dict(k=3, edges=[(0, 1), (1, 2)], labels=[0, -2, 1]),
])
def test_compile_rejects_invalid(stm, bad):
    kw = dict(bad)
    k, edges = kw.pop("k"), kw.pop("edges")
    if "restrictions" in kw:
        kw["auto_restrict"] = False
    with pytest.raises(stm.StmError) as ei:
        stm.Plan(k, edges, **kw)
    assert ei.value.status == stm.STM_EINVAL
    assert stm.lib.stm_last_error()


def test_k_too_large(stm):
    e = [(i, i + 1) for i in range(8)]
    with pytest.raises(stm.StmError) as ei:
        stm.Plan(9, e)
    assert ei.value.status == stm.STM_EUNSUPPORTED


def test_plan_describe_buffer_too_small(stm):
    p = stm.Plan(3, CATALOG["triangle"].edges)
    buf = ctypes.create_string_buffer(8)
    assert stm.lib.stm_plan_describe(p.handle, buf, 8) == stm.STM_EINVAL


def test_greedy_order_is_connected(stm):
    for name, p in CATALOG.items():
        plan = stm.Plan(p.k, p.edges)
        txt = plan.describe()
        order = [int(x) for x in txt.split("order=[")[1].split("]")[0].split(",")]
        assert sorted(order) == list(range(p.k))
        adj = {u: set() for u in range(p.k)}
        for a, b in p.edges:
            adj[a].add(b)
            adj[b].add(a)
        for i in range(1, p.k):
            assert any(order[j] in adj[order[i]] for j in range(i)), (name, order)
        assert plan.first_vertex == order[0]


def test_no_code_motion_keeps_all_work_at_the_consumer_level(stm):
    h = CATALOG["house"]
    _, lines = _plan_lines(stm, h.k, h.edges, vertex_induced=True, code_motion=False)
    assert "code_motion=off" in lines[0]
    for x in lines:
        m = re.match(r"S\d+: level (\d) .*= (\S+) ", x)
        if m:  # without code motion a set is only built at the level that consumes it
            assert int(m.group(1)) >= 2


def test_lazy_unbounded_plan_k6_minus_e(stm):
    """STM_LAZY_UNBOUNDED: the bounded chain that enumerates the K4 (v0 < v1 < v2 < v3)
    stays hoisted; the unbounded common neighbourhood of the K4, needed only by the two
    last pattern vertices, is built at level 4 as one staged chain and shared by both."""
    p = CATALOG["k6_minus_e"]
    _, lines = _plan_lines(stm, p.k, p.edges, lazy_unbounded=True)
    sets = [_strip(x) for x in lines if x.startswith("S")]
    assert sets == ["S0: level 2 stage 0 = N(v0) & N(v1)", "S1: level 3 stage 0 = S0 & N(v2)",
                    "S2: level 4 stage 0 = N(v0) & N(v1)", "S3: level 4 stage 1 = S2 & N(v2)",
                    "S4: level 4 stage 2 = S3 & N(v3)"]
    assert any(x.startswith("S0:") and "lo={v1}" in x for x in lines)
    assert any(x.startswith("cand 4: S4") for x in lines) and any(x.startswith("count 5: S4") for x in lines)
    # cliques are bounded at every level: lazy changes nothing
    k5 = CATALOG["k5"]
    assert _plan_lines(stm, k5.k, k5.edges, lazy_unbounded=True)[1][2:] == _plan_lines(stm, k5.k, k5.edges)[1][2:]


def test_directed_plan_compile():
    """STM_DIRECTED plans (NEXT-4): raw operands name out-rows N+(v) or in-rows N-(v); the directed
    3-cycle counts N-(v0) & N+(v1) at its last level, with |Aut| = 3 (rotations only)."""
    from paper_conf_sc_weij22_b200 import stm
    p = stm.Plan(3, [(0, 1), (1, 2), (2, 0)], directed=True)
    d = p.describe()
    assert "directed" in d and p.aut == 3
    assert "count 2: N-(v0) & N+(v1)" in d
    assert stm.Plan(3, [(0, 1), (1, 2), (0, 2)], directed=True).aut == 1
    # an undirected plan never carries in-rows
    assert "N-(" not in stm.Plan(3, [(0, 1), (1, 2), (0, 2)]).describe()
