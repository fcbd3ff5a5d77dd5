"""Small counts for compute-sanitizer (memcheck / racecheck / synccheck): every stealing
path forced on a small hub graph, results checked against the oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import stmgen, oracle
from paper_conf_sc_weij22_b200 import stm
g = stmgen.rmat(8, 900, 0.57, 0.19, 0.19, 3)
G = stm.Graph.from_stmgen(g)
ok = True
mode = sys.argv[1] if len(sys.argv) > 1 else "count"
TUNE = [dict(), dict(block_warps=4, blocks_per_sm=1, root_chunk=1, stop_level=3, detect_level=3),
        dict(occupancy=2, unroll=3, bitmap_min_degree=1)]
if mode == "nosteal":
    TUNE = [dict(local_steal=0, global_steal=0), dict(local_steal=0, global_steal=0, occupancy=2, unroll=3)]
for name, vi in [("k4", False), ("house", True), ("c5", False)]:
    p = stmgen.CATALOG[name]
    want = oracle.count(g, p.k, p.edges, vertex_induced=vi, restrictions=oracle.gk_restrictions(p.k, p.edges))
    for tk in TUNE if mode != "list" else []:
        got = stm.count(G, stm.Plan(p.k, p.edges, vertex_induced=vi), stm.stm_tuning_default(**tk))
        print(name, vi, tk, got, want, flush=True)
        ok &= got == want
    if mode == "list":
        plan = stm.Plan(p.k, p.edges, vertex_induced=vi)  # keep the handle's owner alive
        rows, c = stm.stm_match_list(G.handle, plan.handle, p.k, None, capacity=50)
        print(name, vi, "list", c, want, flush=True)
        ok &= c == want
print("SANITIZE_COUNTS_OK" if ok else "SANITIZE_COUNTS_MISMATCH")
