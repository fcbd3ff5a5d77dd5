"""1..8 GPU layer ("duplicating the input graph and dividing the
outermost loop iterations across GPUs"; north_star: cross-GPU stealing of root
ranges and one NCCL all-reduce of the per-rank counts).

One process per GPU (torchrun).  Every rank holds a full replica of the graph.
The root space [0, n) is cut into chunks of `root_chunk` roots; chunk c belongs to
rank c % world and each rank owns one device-resident uint64 cursor per query
slot (libstm ``stm_cursors_alloc``).  Every rank maps every peer's cursors through
CUDA IPC (``stm_cursors_open``), so a kernel whose own cursor is exhausted takes
chunks from the peers' cursors with atomics on peer memory over NVLink: every chunk
is processed exactly once.  The partial counts are summed with ONE ``all_reduce``
(int64, SUM) per step.  PyTorch is plumbing only: the counting runs in libstm.so.

Cursor protocol (why a count is never double-counted).  Cursors are never reset
while a peer may still take chunks from them: the cursors of a step live in one of
two slot SETS used on alternate steps, and a rank zeroes its own cursors of set s
in stream order right after the all-reduce that closes the step using set s.  That
all-reduce completes on a rank only after every rank's kernels of the step have
finished, so no kernel of that step can still touch them; and a peer can start its
next step on set s only after the following step's all-reduce, which this rank
enters after the zeroing (stream order).  A peer that reads a cursor of the other
set early sees it exhausted (stale) and simply does not steal from it.
"""
from __future__ import annotations

import time
from typing import List, Optional, Sequence

import torch
import torch.distributed as dist

from . import stm

SLOTS = 16  # query slots per step (cursor set size)
SETS = 2    # cursor sets, used on alternate steps


def shard_chunks(n: int, chunk: int, rank: int, world: int) -> List[int]:
    """Chunk ids owned by `rank` before any stealing (c % world == rank)."""
    nchunks = (n + chunk - 1) // chunk
    return list(range(rank, nchunks, world))


def chunk_roots(c: int, chunk: int, n: int):
    """Root-ID range [b, e) of chunk c (empty past the end)."""
    b = min(n, c * chunk)
    return b, min(n, b + chunk)


def cursor_chunk(owner: int, idx: int, world: int) -> int:
    """Chunk handed out by the idx-th atomicAdd on rank `owner`'s cursor (kernel try_chunk)."""
    return owner + world * idx


def steal_order(rank: int, world: int) -> List[int]:
    """Cursors a rank's kernel draws from: its own first, then the peers' in ring order."""
    return [(rank + i) % world for i in range(world)]


class SlotSchedule:
    """Host-side bookkeeping of the cursor protocol (pure Python, tested on CPU):
    which slot a query of the current step uses, and which slots must be zeroed
    after the step's all-reduce."""

    def __init__(self, slots: int = SLOTS, sets: int = SETS):
        self.slots, self.sets = slots, sets
        self.set = 0
        self.used = 0

    def next_slot(self) -> int:
        if self.used >= self.slots:
            raise RuntimeError(f"more than {self.slots} queries in one step")
        s = self.set * self.slots + self.used
        self.used += 1
        return s

    def end_step(self):
        """Returns (first_slot, n_slots) to zero after the all-reduce, then flips the set."""
        z = (self.set * self.slots, self.slots)
        self.set = (self.set + 1) % self.sets
        self.used = 0
        return z


class MultiGPUCounter:
    """Counts on this rank's GPU; combines ranks with one all-reduce per step.

    ``count_async`` enqueues one query writing an stm_async_result (int64[4]:
    count, status, chunks, peer_chunks) into a device tensor; ``reduce_counts``
    closes the step (all-reduce of the result rows, cursor zeroing)."""

    def __init__(self, graph: stm.Graph, tuning: Optional[stm.stm_tuning] = None, rank: int = 0, world: int = 1,
                 device: Optional[torch.device] = None, cross_steal: bool = True, group=None):
        self.G = graph
        self.tuning = tuning if tuning is not None else stm.stm_tuning_default()
        self.rank, self.world = rank, world
        self.device = device or torch.device("cuda", torch.cuda.current_device())
        self.dev = self.device.index if self.device.index is not None else torch.cuda.current_device()
        self.group = group
        self.cross_steal = False
        self.chunk = int(self.tuning.root_chunk)
        self.sched = SlotSchedule()
        self.own_base: Optional[int] = None
        self.peer_base: List[Optional[int]] = [None] * 8
        self._opened: List[int] = []
        self.last_local: Optional[torch.Tensor] = None  # this rank's result rows of the last step, pre-reduce
        if world > 1:
            self.backend = dist.get_backend(group)
            self._init_cursors(cross_steal)

    # -- cursors ---------------------------------------------------------------------------
    def _init_cursors(self, cross_steal: bool):
        base, handle = stm.stm_cursors_alloc(self.dev, SLOTS * SETS)
        self.own_base = base
        handles: List[Optional[bytes]] = [None] * self.world
        dist.all_gather_object(handles, handle, group=self.group)
        self.peer_base = [None] * self.world
        self.peer_base[self.rank] = base
        if cross_steal:
            # Loud: a rank that cannot map its peers' cursors must not silently fall back to
            # the static partition (the caller asked for cross-GPU stealing).
            for r, h in enumerate(handles):
                if r != self.rank:
                    p = stm.stm_cursors_open(self.dev, h)
                    self._opened.append(p)
                    self.peer_base[r] = p
            self.cross_steal = True
        torch.cuda.synchronize(self.device)
        dist.barrier(group=self.group)

    def close(self):
        if self.world > 1 and self.own_base is not None:
            torch.cuda.synchronize(self.device)
            dist.barrier(group=self.group)  # no peer still maps my cursors after this
            for p in self._opened:
                stm.stm_cursors_close(self.dev, p)
            self._opened = []
            dist.barrier(group=self.group)
            stm.stm_cursors_free(self.dev, self.own_base)
            self.own_base = None

    def _shard(self, slot: int) -> stm.stm_shard:
        ptrs = []
        for r in range(self.world):
            b = self.peer_base[r]
            ptrs.append(None if b is None else b + slot * 64)
        return stm.make_shard(self.rank, self.world, self.chunk, ptrs)

    # -- counting --------------------------------------------------------------------------
    def new_results(self, nq: int) -> torch.Tensor:
        """Device tensor of nq stm_async_result rows (int64[nq, 4])."""
        return torch.zeros((nq, stm.ASYNC_WORDS), dtype=torch.int64, device=self.device)

    def count_async(self, plan: stm.Plan, d_out: torch.Tensor, graph_handle: Optional[int] = None) -> None:
        """Enqueue one query on the current stream; d_out (one int64[4] result row on this
        GPU) gets this rank's partial count, status and chunk counters."""
        assert d_out.dtype == torch.int64 and d_out.numel() >= stm.ASYNC_WORDS and d_out.is_contiguous()
        gh = graph_handle or self.G.handle
        sp = torch.cuda.current_stream(self.device).cuda_stream
        shard = None if self.world == 1 else self._shard(self.sched.next_slot())
        stm.stm_match_count_async(gh, plan.handle, d_out.data_ptr(), self.tuning, shard, sp)

    def reduce_counts(self, d_results: torch.Tensor) -> None:
        """Close the step: the single all-reduce (int64 SUM over the result rows: counts
        exact below 2^63, statuses non-zero iff some rank failed), then zero this rank's
        cursors of the step's slot set in stream order (module docstring)."""
        if self.world == 1:
            self.last_local = d_results
            return
        self.last_local = d_results.clone()
        if self.backend == "gloo":
            host = d_results.cpu()
            dist.all_reduce(host, op=dist.ReduceOp.SUM, group=self.group)
            d_results.copy_(host)
        else:
            dist.all_reduce(d_results, op=dist.ReduceOp.SUM, group=self.group)
        first, n = self.sched.end_step()
        stm.stm_cursors_reset(self.dev, self.own_base, first, n, torch.cuda.current_stream(self.device).cuda_stream)

    @staticmethod
    def check(results: torch.Tensor) -> List[int]:
        """Host check of reduced result rows: raises on any failed launch, returns the counts."""
        r = results.cpu().tolist()
        out = []
        for row in r:
            if row[1] != 0:
                raise stm.StmError(int(row[1]) if 0 < row[1] < 8 else stm.STM_ECUDA,
                                   f"a rank's launch failed with status {stm.async_status_message(row[1])}")
            out.append(int(row[0]) & ((1 << 64) - 1))
        return out

    def count(self, plan: stm.Plan) -> int:
        d = self.new_results(1)
        self.count_async(plan, d[0])
        self.reduce_counts(d)
        return self.check(d)[0]

    def count_instrumented(self, plan: stm.Plan):
        """Untimed synchronous launch that also measures the algorithmic bytes."""
        t = stm.stm_tuning_default(**{f[0]: getattr(self.tuning, f[0]) for f in self.tuning._fields_})
        t.instrument = 1
        if self.world == 1:
            c = stm.stm_match_count_ex(self.G.handle, plan.handle, t, None, None)
            return c, stm.stm_last_launch()
        part = stm.stm_match_count_ex(self.G.handle, plan.handle, t, self._shard(self.sched.next_slot()), None)
        info = stm.stm_last_launch()
        d = self.new_results(1)
        d[0, 0] = part if part < (1 << 63) else part - (1 << 64)
        self.reduce_counts(d)
        return self.check(d)[0], info

    # -- end to end ------------------------------------------------------------------------
    def e2e(self, g, plans: Sequence[stm.Plan], steps: int = 3):
        """Public-API end to end, per step: stm_graph_load from the HOST CSR arrays (the
        validating entry: O(m log d) CSR checks, H2D copies, degree-ranked copy) -> count
        every query -> all-reduce -> read the result rows back (D2H) -> stm_graph_free.
        Wall clock per step, max over ranks."""
        h2d = g.row_ptr.nbytes + g.col_idx.nbytes + (g.labels.nbytes if g.labels is not None else 0)
        times = []
        counts = None
        for _ in range(steps):
            torch.cuda.synchronize(self.device)
            if self.world > 1:
                dist.barrier(group=self.group)
            t0 = time.perf_counter()
            gh = stm.stm_graph_load(g.n, g.row_ptr, g.col_idx, g.labels, self.dev)
            out = self.new_results(len(plans))
            for qi, pl in enumerate(plans):
                self.count_async(pl, out[qi], graph_handle=gh)
            self.reduce_counts(out)
            counts = self.check(out)  # D2H of the step's result rows
            dt = time.perf_counter() - t0
            stm.stm_graph_free(gh)
            if self.world > 1:
                t = torch.tensor([dt], dtype=torch.float64)
                if self.backend != "gloo":
                    t = t.to(self.device)
                dist.all_reduce(t, op=dist.ReduceOp.MAX, group=self.group)
                dt = float(t.item())
            times.append(dt)
        return {"seconds_per_step": sum(times) / len(times), "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": 8 * stm.ASYNC_WORDS * len(plans), "counts": counts,
                "path": "host CSR -> stm_graph_load (validation + H2D + degree-ranked copy) -> "
                        "stm_match_count_async per query -> all_reduce -> D2H of the result rows "
                        "(wall clock, max over ranks; graph free untimed)"}
