"""Write tests/golden/config_counts.json: full-graph expected counts from the ORACLE only.

Every value in that file is produced here by calling oracle.count on a graph from
stmgen (seeded, machine-independent); the graph fingerprint is stored next to
each value so a test can prove it compares the same input.  Nothing here touches
the CUDA path.  Usage: python tools/make_golden.py [case ...] (default: all).

Two speed-only input choices, both invariances pinned in tests/test_oracle.py
(relabel and order invariance of the count of distinct subgraphs):
  * "ranked": the oracle runs on the graph renumbered in (degree, id) order (the
    stored fingerprint is the caller's graph; the count does not depend on ids);
  * "edges": an isomorphic labelling of the pattern (K6-e with its non-adjacent pair
    at (4, 5), so the oracle's own BFS order starts with the K4).
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import stmgen  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "config_counts.json")

K6ME_45 = tuple((i, j) for i in range(6) for j in range(i + 1, 6) if (i, j) != (4, 5))

# (case id, config graph, pattern, vertex_induced, pattern labels or None[, options])
CASES = [
    ("c1_triangle_ei", "c1", "triangle", False, None),
    ("c1_triangle_vi", "c1", "triangle", True, None),
    ("c1_c4_ei", "c1", "c4", False, None),
    ("c1_house_vi", "c1", "house", True, None),
    ("c2_triangle_ei", "c2", "triangle", False, None),
    ("c2_k4_ei", "c2", "k4", False, None),
    ("c4_k4_L_ei", "c4", "k4", False, (0, 1, 2, 3)),
    ("c3_k5_ei", "c3", "k5", False, None),
    ("c4_diamond_L_ei", "c4", "diamond", False, (0, 1, 1, 2)),
    ("c2_c4_ei", "c2", "c4", False, None),
    ("c4_k6me_L_ei", "c4", "k6_minus_e", False, (0, 1, 2, 3, 4, 5)),
    ("c4_w5_L_ei", "c4", "w5", False, (0, 1, 1, 2, 2, 3)),
    ("c4_c6_L_vi", "c4", "c6", True, (0, 1, 2, 0, 1, 2)),
    ("c4_w6_L_ei", "c4", "w6", False, (0, 1, 2, 1, 2, 1, 2)),
    ("c4_c7_L_vi", "c4", "c7", True, (0, 1, 2, 3, 0, 1, 2)),
    ("c5_k5_ei", "c5", "k5", False, None, {"ranked": True}),
    ("c5_k6me_ei", "c5", "k6_minus_e", False, None, {"ranked": True, "edges": K6ME_45}),
    ("c3_k5_vi", "c3", "k5", True, None, {"ranked": True}),
    ("c2_c4_vi", "c2", "c4", True, None),
    ("c4_c6_L012012_ei", "c4", "c6", False, (0, 1, 2, 0, 1, 2)),
    ("c4_c6_L012345_ei", "c4", "c6", False, (0, 1, 2, 3, 4, 5)),
    ("c4_c7_L0123456_ei", "c4", "c7", False, (0, 1, 2, 3, 4, 5, 6)),
    ("c4_c7_L0101012_ei", "c4", "c7", False, (0, 1, 0, 1, 0, 1, 2)),
    ("c3_c5_ei", "c3", "c5", False, None, {"ranked": True}),
    ("c3_house_ei", "c3", "house", False, None, {"ranked": True}),
]


def degree_ranked(g):
    """g renumbered so that vertex i is the i-th in (degree, id) order (labels carried)."""
    import numpy as np
    deg = g.degrees()
    rank2orig = np.lexsort((np.arange(g.n), deg))
    perm = np.empty(g.n, np.int64)
    perm[rank2orig] = np.arange(g.n)
    return stmgen.permute(g, perm)


def main(argv):
    want = set(argv) if argv else None
    data = json.load(open(OUT)) if os.path.exists(OUT) else {}
    graphs = {}
    threads = int(os.environ.get("GOLDEN_THREADS", os.cpu_count() or 1))
    for case in CASES:
        cid, cfg, pname, vi, plab = case[:5]
        opt = case[5] if len(case) > 5 else {}
        if want is not None and cid not in want:
            continue
        if cid in data:
            continue
        if cfg not in graphs:
            graphs.clear()
            graphs[cfg] = stmgen.config_graph(cfg)
        g = graphs[cfg]
        gin = degree_ranked(g) if opt.get("ranked") else g
        p = stmgen.CATALOG[pname]
        edges = opt.get("edges", p.edges)
        R = oracle.gk_restrictions(p.k, edges, plab)
        t = time.time()
        c = oracle.count(gin, p.k, edges, plabels=plab, vertex_induced=vi, restrictions=R, threads=threads)
        dt = time.time() - t
        data[cid] = {"config": cfg, "fingerprint": g.fingerprint(), "pattern": pname, "k": p.k,
                     "edges": [list(e) for e in edges], "labels": list(plab) if plab else None,
                     "vertex_induced": vi, "restrictions": [list(r) for r in R], "count": c,
                     "oracle_seconds": round(dt, 2), "oracle_threads": threads,
                     "oracle_input": "degree-ranked relabelling" if opt.get("ranked") else "caller ids"}
        print(cid, c, f"{dt:.1f}s", flush=True)
        json.dump(data, open(OUT, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main(sys.argv[1:])
