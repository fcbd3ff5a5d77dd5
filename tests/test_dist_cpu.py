"""Multi-GPU layer, host logic, on CPU with world_size-2 gloo process groups.

The GPU side (libstm.so try_chunk + peer cursors, dist.MultiGPUCounter) cannot run
here; these tests pin what it relies on: the chunk partition covers every root
exactly once, the cursor protocol (own cursor first, then peers', exhausted
cursors skipped) hands out every chunk exactly once however the ranks interleave,
and one int64 SUM all-reduce of per-rank partial counts (each computed by the
ORACLE over that rank's roots) equals the single-process count.
"""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import stmgen
from paper_conf_sc_weij22_b200.dist import chunk_roots, cursor_chunk, shard_chunks, steal_order


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("n,chunk,world", [(0, 4, 2), (1, 32, 8), (1000, 32, 3), (1001, 7, 8), (64, 64, 2)])
def test_static_partition_covers_roots_once(n, chunk, world):
    seen = np.zeros(n, np.int64)
    for r in range(world):
        for c in shard_chunks(n, chunk, r, world):
            b, e = chunk_roots(c, chunk, n)
            seen[b:e] += 1
    assert (seen == 1).all()


def _worker(rank, world, port, out, steal):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = stmgen.rmat(9, 3000, 0.57, 0.19, 0.19, 23)
    chunk = 16
    nchunks = (g.n + chunk - 1) // chunk
    p = stmgen.CATALOG["house"]
    R = oracle.gk_restrictions(p.k, p.edges)
    mine = []
    if not steal:
        mine = shard_chunks(g.n, chunk, rank, world)
    else:
        # emulate the kernel's cursor protocol on cursors shared through the process
        # group: every take is an atomic fetch-add on the owner's cursor (done here
        # by the owner's lock-step turn), skipping exhausted cursors
        cursors = torch.zeros(world, dtype=torch.int64)
        exhausted = set()
        while len(exhausted) < world:
            # one round: every rank asks for one chunk from its next live cursor
            want = torch.tensor([next((o for o in steal_order(rank, world) if o not in exhausted), -1)])
            asks = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
            dist.all_gather(asks, want)
            got = -1
            for r in range(world):  # fetch-adds in rank order (any order is valid)
                o = int(asks[r])
                if o < 0:
                    continue
                idx = int(cursors[o])
                cursors[o] += 1
                c = cursor_chunk(o, idx, world)
                if r == rank:
                    got = c if c < nchunks else -1
                    if c >= nchunks:
                        exhausted.add(o)
            if got >= 0:
                mine.append(got)
            done = torch.tensor([1 if len(exhausted) == world else 0])
            dist.all_reduce(done, op=dist.ReduceOp.MIN)
            if int(done) == 1:
                break
    roots = np.concatenate([np.arange(*chunk_roots(c, chunk, g.n)) for c in mine]) if mine else np.zeros(0, np.int64)
    part = oracle.count(g, p.k, p.edges, restrictions=R, roots=roots, threads=1) if roots.size else 0
    t = torch.tensor([part], dtype=torch.int64)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    lists = [None] * world
    dist.all_gather_object(lists, mine)
    if rank == 0:
        allc = sorted(c for l in lists for c in l)
        whole = oracle.count(g, p.k, p.edges, restrictions=R, threads=1)
        with open(out, "w") as f:
            f.write(f"{int(t)} {whole} {int(allc == list(range(nchunks)))}")
    dist.destroy_process_group()


@pytest.mark.parametrize("steal", [False, True])
def test_gloo_world2_partial_counts_all_reduce(steal):
    with tempfile.TemporaryDirectory() as d:
        out = os.path.join(d, "r.txt")
        mp.spawn(_worker, args=(2, _port(), out, steal), nprocs=2, join=True)
        total, whole, exact_once = open(out).read().split()
    assert int(total) == int(whole) > 0
    assert exact_once == "1"
