"""Motif census timing (NEXT-3): python tools/census.py c1:6:vi c2:4 ... -- merged (one launch of the
pattern-merging trie) vs one launch per motif, cost-based orders from the graph's statistics."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import stmgen
from paper_conf_sc_weij22_b200 import stm
tk = dict(a.split("=") for a in sys.argv[1:] if "=" in a)
tuning = stm.stm_tuning_default(**{k: int(v) for k, v in tk.items()}) if tk else None
for spec in [a for a in sys.argv[1:] if "=" not in a]:
    cfg, k = spec.split(":")[:2]
    k = int(k)
    flags = (stm.STM_VERTEX_INDUCED if ":vi" in spec else 0) | (stm.STM_AUTO_ORDER if ":greedy" in spec else 0)
    g = stmgen.config_graph(cfg)
    G = stm.Graph.from_stmgen(g)
    res = {}
    for name, f in (("merged", flags), ("per-motif", flags | stm.STM_CENSUS_PER_MOTIF)):
        stm.stm_motif_census(G.handle, k, f, tuning=tuning)  # warm-up
        best = 1e9
        for _ in range(3):
            t0 = time.perf_counter()
            c = stm.stm_motif_census(G.handle, k, f, tuning=tuning)
            best = min(best, time.perf_counter() - t0)
        res[name] = c
        print(f"{spec:10} {name:9} {len(c)} motifs in {stm.stm_motif_census_launches()} launch(es) "
              f"{best * 1e3:10.2f} ms  total {sum(c)}", flush=True)
    assert res["merged"] == res["per-motif"], "merged and per-motif censuses differ"
    G.close()
