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


# ---------------------------------------------------------------- cursor protocol
def _simulate(world, nchunks, steps, seed, protocol):
    """Discrete-event model of MultiGPUCounter's per-rank streams.  Each rank's stream is
    [kernel(step) ; all-reduce(step) ; zero(own cursors of the step's set)] per step
    ("new" protocol, dist.SlotSchedule), or [zero(own slot) ; kernel ; all-reduce] (the
    round-1 protocol).  A kernel is a sequence of atomic fetch-adds, own cursor first then
    the peers' (kernel try_chunk); an all-reduce completes on a rank only once every rank
    has entered it.  The scheduler interleaves ranks at random.  Returns, per step, the
    sorted list of chunks handed out."""
    from paper_conf_sc_weij22_b200.dist import SlotSchedule
    rng = np.random.default_rng(seed)
    sched = [SlotSchedule(slots=1, sets=2) for _ in range(world)]
    cursors = np.zeros((world, 2), np.int64)  # [owner, slot]
    taken = [[] for _ in range(steps)]
    # per-rank program counter: (step, phase, state)
    ops = []
    for r in range(world):
        prog = []
        for s in range(steps):
            slot = sched[r].next_slot() if protocol == "new" else 0  # round 1: slot 0 every step
            if protocol == "old":
                prog.append(("zero", s, slot))
            prog.append(("kernel", s, slot))
            prog.append(("ar", s, slot))
            if protocol == "new":
                first, n = sched[r].end_step()
                prog.append(("zero", s, first))
        ops.append(prog)
    pc = [0] * world
    kstate = [None] * world  # exhausted set of the running kernel
    entered_ar = [set() for _ in range(steps)]
    speed = rng.random(world) ** 4 + 1e-3  # per-rank speed: some ranks far faster than others
    while any(pc[r] < len(ops[r]) for r in range(world)):
        def blocked(r):  # waiting inside an all-reduce that not every rank has entered
            kind, s, _ = ops[r][pc[r]]
            return kind == "ar" and r in entered_ar[s] and len(entered_ar[s]) < world
        live = [r for r in range(world) if pc[r] < len(ops[r]) and not blocked(r)]
        r = int(rng.choice(live, p=speed[live] / speed[live].sum()))  # skewed ranks
        kind, s, slot = ops[r][pc[r]]
        if kind == "zero":
            cursors[r, slot] = 0
            pc[r] += 1
        elif kind == "ar":
            entered_ar[s].add(r)
            if len(entered_ar[s]) == world:  # completes for this rank only when all entered
                pc[r] += 1
        else:
            if kstate[r] is None:
                kstate[r] = set()
            o = next((o for o in steal_order(r, world) if o not in kstate[r]), None)
            if o is None:
                kstate[r] = None
                pc[r] += 1
                continue
            idx = int(cursors[o, slot])
            cursors[o, slot] += 1
            c = cursor_chunk(o, idx, world)
            if c < nchunks:
                taken[s].append(c)
            else:
                kstate[r].add(o)
    return [sorted(t) for t in taken]


@pytest.mark.parametrize("world", [2, 3, 8])
def test_cursor_protocol_hands_out_every_chunk_once_per_step(world):
    """dist.py's slot-set protocol: under any interleaving of the ranks' streams, every
    step hands out every chunk exactly once (no chunk recounted after a reset, none lost)."""
    for seed in range(60):
        for t in _simulate(world, nchunks=23, steps=5, seed=seed, protocol="new"):
            assert t == list(range(23))


def test_cursor_protocol_round1_reset_race_is_caught():
    """The round-1 order (each rank zeroes its own cursor right before its launch) recounts
    chunks when a fast rank drains a slow rank's cursor first -- the model detects it."""
    bad = 0
    for seed in range(60):
        bad += any(t != list(range(23)) for t in _simulate(2, nchunks=23, steps=5, seed=seed, protocol="old"))
    assert bad > 0


def test_slot_schedule_alternates_sets():
    from paper_conf_sc_weij22_b200.dist import SlotSchedule
    s = SlotSchedule(slots=4, sets=2)
    assert [s.next_slot() for _ in range(3)] == [0, 1, 2]
    assert s.end_step() == (0, 4)
    assert s.next_slot() == 4
    assert s.end_step() == (4, 4)
    assert s.next_slot() == 0
    with pytest.raises(RuntimeError):
        for _ in range(5):
            s.next_slot()
