"""Multi-GPU layer on ONE GPU: two ranks (processes) run dist.MultiGPUCounter against
each other on cuda:0 (gloo process group for the plumbing; the chunk cursors are
shared through libstm's CUDA IPC handles exactly as across GPUs).
(duplicate the graph, divide the outermost loop) + north_star (cross-GPU stealing,
one all-reduce).  Expected counts are the ORACLE's full-graph goldens
(tests/golden/config_counts.json, tools/make_golden.py).

Also: failure reporting of the asynchronous path (a watchdog-aborted launch is
reported through stm_async_result.status, never counted).
"""
import json
import os
import socket
import tempfile
import time

import pytest

pytestmark = pytest.mark.gpu

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "config_counts.json")))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_main(rank, world, port, out_dir, cross_steal):
    import torch
    import torch.distributed as dist
    import stmgen
    from paper_conf_sc_weij22_b200 import stm
    from paper_conf_sc_weij22_b200.dist import MultiGPUCounter

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = stmgen.config_graph("c2")
    G = stm.Graph.from_stmgen(g, device=0)
    layer = MultiGPUCounter(G, rank=rank, world=world, device=torch.device("cuda", 0), cross_steal=cross_steal)
    names = ["k4", "c4"]
    plans = [stm.Plan(stmgen.CATALOG[p].k, stmgen.CATALOG[p].edges) for p in names]
    rec = {"fingerprint": g.fingerprint(), "cross_steal": layer.cross_steal, "steps": []}
    # step i: rank slow[i] enqueues its kernels late (host sleep), so the other rank's
    # persistent kernel drains its own cursor and then the slow rank's (cross-steal);
    # every step reuses the slot-set protocol (dist.py docstring)
    for slow in [1, 0, 1, 0, -1]:
        d = layer.new_results(len(plans))
        torch.cuda.synchronize()
        dist.barrier()
        if rank == slow:
            time.sleep(0.4)
        for qi, pl in enumerate(plans):
            layer.count_async(pl, d[qi])
        layer.reduce_counts(d)
        counts = layer.check(d)
        local = layer.last_local.cpu().tolist()
        rec["steps"].append({"slow": slow, "counts": counts, "chunks": [r[2] for r in local],
                             "peer_chunks": [r[3] for r in local]})
    rec["count_api"] = layer.count(plans[0])
    e = layer.e2e(g, plans, steps=1)
    rec["e2e_counts"] = e["counts"]
    layer.close()
    with open(os.path.join(out_dir, f"r{rank}.json"), "w") as f:
        json.dump(rec, f)
    dist.destroy_process_group()


def _run(cross_steal):
    import torch.multiprocessing as mp
    with tempfile.TemporaryDirectory() as d:
        mp.spawn(_rank_main, args=(2, _port(), d, cross_steal), nprocs=2, join=True)
        return [json.load(open(os.path.join(d, f"r{r}.json"))) for r in range(2)]


def test_two_ranks_one_gpu_cross_steal():
    r0, r1 = _run(True)
    want = [GOLD["c2_k4_ei"]["count"], GOLD["c2_c4_ei"]["count"]]
    assert r0["fingerprint"] == GOLD["c2_k4_ei"]["fingerprint"]
    assert r0["cross_steal"] and r1["cross_steal"]
    for a, b in zip(r0["steps"], r1["steps"]):
        assert a["counts"] == b["counts"] == want, (a, b)
        # all-reduced partials: every chunk processed exactly once
        for q in range(2):
            assert a["chunks"][q] >= 0 and b["chunks"][q] >= 0
    assert r0["count_api"] == r1["count_api"] == want[0]
    assert r0["e2e_counts"] == r1["e2e_counts"] == want
    # both ranks took chunks, and each stole from the other when the other was late
    steps = list(zip(r0["steps"], r1["steps"]))
    assert sum(sum(a["chunks"]) for a, _ in steps) > 0 and sum(sum(b["chunks"]) for _, b in steps) > 0
    stolen_by_0 = sum(sum(a["peer_chunks"]) for a, b in steps if a["slow"] == 1)
    stolen_by_1 = sum(sum(b["peer_chunks"]) for a, b in steps if a["slow"] == 0)
    assert stolen_by_0 > 0 and stolen_by_1 > 0, (stolen_by_0, stolen_by_1)


def test_two_ranks_one_gpu_static_partition():
    r0, r1 = _run(False)
    want = [GOLD["c2_k4_ei"]["count"], GOLD["c2_c4_ei"]["count"]]
    assert not r0["cross_steal"] and not r1["cross_steal"]
    for a, b in zip(r0["steps"], r1["steps"]):
        assert a["counts"] == b["counts"] == want
        assert a["peer_chunks"] == [0, 0] and b["peer_chunks"] == [0, 0]
        assert min(a["chunks"]) > 0 and min(b["chunks"]) > 0


def test_async_watchdog_is_reported_not_counted():
    """A launch aborted by the watchdog (stm_tuning.watchdog_ms) reports STM_ETIMEOUT through
    stm_async_result.status (count withheld); the synchronous call raises it."""
    import torch
    import stmgen
    from paper_conf_sc_weij22_b200 import stm
    from paper_conf_sc_weij22_b200.dist import MultiGPUCounter

    g = stmgen.config_graph("c2")
    G = stm.Graph.from_stmgen(g, device=0)
    p = stmgen.CATALOG["c4"]
    plan = stm.Plan(p.k, p.edges)
    t = stm.stm_tuning_default(watchdog_ms=1)
    layer = MultiGPUCounter(G, tuning=t, device=torch.device("cuda", 0))
    d = layer.new_results(1)
    layer.count_async(plan, d[0])
    layer.reduce_counts(d)
    row = d.cpu().tolist()[0]
    assert row[1] == stm.STM_ETIMEOUT and row[0] == 0
    with pytest.raises(stm.StmError) as ei:
        layer.check(d)
    assert "STM_ETIMEOUT" in str(ei.value)
    with pytest.raises(stm.StmError) as ei:
        stm.count(G, plan, t)
    assert ei.value.status == stm.STM_ETIMEOUT
    # the same launch without the watchdog is counted (and bit-exact)
    layer.tuning = stm.stm_tuning_default()
    assert layer.count(plan) == GOLD["c2_c4_ei"]["count"]
