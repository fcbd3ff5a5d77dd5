"""Write tests/golden/config_counts.json: full-graph expected counts from the ORACLE only.

Every value in that file is produced here by calling oracle.count on a graph from
stmgen (seeded, machine-independent); the graph fingerprint is stored next to
each value so a test can prove it compares the same input.  Nothing here touches
the CUDA path.  Usage: python tools/make_golden.py [case ...] (default: all).
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

# (case id, config graph, pattern, vertex_induced, pattern labels or None)
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
    ("c3_house_ei", "c3", "house", False, None),
    ("c3_c5_ei", "c3", "c5", False, None),
]


def main(argv):
    want = set(argv) if argv else None
    data = json.load(open(OUT)) if os.path.exists(OUT) else {}
    graphs = {}
    threads = int(os.environ.get("GOLDEN_THREADS", os.cpu_count() or 1))
    for cid, cfg, pname, vi, plab in CASES:
        if want is not None and cid not in want:
            continue
        if cid in data:
            continue
        if cfg not in graphs:
            graphs[cfg] = stmgen.config_graph(cfg)
        g = graphs[cfg]
        p = stmgen.CATALOG[pname]
        R = oracle.gk_restrictions(p.k, p.edges, plab)
        t = time.time()
        c = oracle.count(g, p.k, p.edges, plabels=plab, vertex_induced=vi, restrictions=R, threads=threads)
        dt = time.time() - t
        data[cid] = {"config": cfg, "fingerprint": g.fingerprint(), "pattern": pname, "k": p.k,
                     "edges": [list(e) for e in p.edges], "labels": list(plab) if plab else None,
                     "vertex_induced": vi, "restrictions": [list(r) for r in R], "count": c,
                     "oracle_seconds": round(dt, 2), "oracle_threads": threads}
        print(cid, c, f"{dt:.1f}s", flush=True)
        json.dump(data, open(OUT, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main(sys.argv[1:])
