"""1..8 GPU layer ("duplicating the input graph and dividing the
outermost loop iterations across GPUs"; north_star: cross-GPU stealing of root
ranges and one NCCL all-reduce of the per-rank counts).

One process per GPU (torchrun).  Every rank holds a full replica of the graph.
The root space [0, n) is cut into chunks of `root_chunk` roots; chunk c belongs to
rank c % world and each rank owns one device-resident uint64 cursor per query
slot.  When a rank's cursor runs dry its kernel takes chunks from the peers'
cursors with atomics on peer memory over NVLink (pointers from torch symmetric
memory), so every chunk is processed exactly once.  The partial counts are summed
with ONE ``all_reduce`` (int64, SUM) on the NCCL backend.  PyTorch is plumbing
only: the counting itself runs in libstm.so.
"""
from __future__ import annotations

import time
from typing import List, Optional, Sequence

import torch
import torch.distributed as dist

from . import stm

SLOTS = 32  # cursor slots (one per query of a step)


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


class MultiGPUCounter:
    """Counts on this rank's GPU; combines ranks with one NCCL all-reduce."""

    def __init__(self, graph: stm.Graph, tuning: Optional[stm.stm_tuning] = None, rank: int = 0, world: int = 1,
                 device: Optional[torch.device] = None, cross_steal: bool = True, group=None):
        self.G = graph
        self.tuning = tuning if tuning is not None else stm.stm_tuning_default()
        self.rank, self.world = rank, world
        self.device = device or torch.device("cuda", torch.cuda.current_device())
        self.group = group
        self.cross_steal = False
        self.chunk = int(self.tuning.root_chunk)
        self._slot = 0
        self.peer_ptrs: List[Optional[int]] = [None] * 8
        if world > 1:
            self._init_cursors(cross_steal)

    # -- cursors ---------------------------------------------------------------------------
    def _init_cursors(self, cross_steal: bool):
        self.cursors = None
        if cross_steal:
            try:  # peer-mapped cursors over NVLink (torch symmetric memory)
                import torch.distributed._symmetric_memory as symm_mem
                buf = symm_mem.empty(SLOTS * 8, dtype=torch.int64, device=self.device)
                hdl = symm_mem.rendezvous(buf, self.group or dist.group.WORLD)
                ptrs = list(hdl.buffer_ptrs)
                if len(ptrs) == self.world:
                    self.cursors = buf
                    self.peer_base = [int(p) for p in ptrs]
                    self.cross_steal = True
            except Exception:
                self.cursors = None
        if self.cursors is None:
            self.cursors = torch.zeros(SLOTS * 8, dtype=torch.int64, device=self.device)
            self.peer_base = [None] * self.world
            self.peer_base[self.rank] = self.cursors.data_ptr()
        self.cursors.zero_()
        torch.cuda.synchronize(self.device)
        dist.barrier(group=self.group)

    def _shard(self, slot: int) -> stm.stm_shard:
        ptrs = []
        for r in range(self.world):
            b = self.peer_base[r]
            ptrs.append(None if b is None else b + slot * 64)
        return stm.make_shard(self.rank, self.world, self.chunk, ptrs)

    # -- counting --------------------------------------------------------------------------
    def count_async(self, plan: stm.Plan, d_out: torch.Tensor, graph_handle: Optional[int] = None,
                    slot: Optional[int] = None) -> None:
        """Enqueue one query on the current stream; d_out (1 x int64 on this GPU) gets
        this rank's partial count (the whole count when world == 1)."""
        gh = graph_handle or self.G.handle
        sp = torch.cuda.current_stream(self.device).cuda_stream
        if self.world == 1:
            stm.stm_match_count_async(gh, plan.handle, d_out.data_ptr(), self.tuning, None, sp)
            return
        if slot is None:
            slot = self._slot % SLOTS
            self._slot += 1
        self.cursors[slot * 8].zero_()  # stream-ordered reset of my cursor for this slot
        stm.stm_match_count_async(gh, plan.handle, d_out.data_ptr(), self.tuning, self._shard(slot), sp)

    def reduce_counts(self, d_counts: torch.Tensor) -> None:
        """The single NCCL all-reduce of the step (int64 SUM; exact below 2^63)."""
        self._slot = 0
        if self.world > 1:
            dist.all_reduce(d_counts, op=dist.ReduceOp.SUM, group=self.group)

    def count(self, plan: stm.Plan) -> int:
        d = torch.zeros(1, dtype=torch.int64, device=self.device)
        self.count_async(plan, d)
        self.reduce_counts(d)
        return int(d.item()) & ((1 << 64) - 1)

    def count_instrumented(self, plan: stm.Plan):
        """Untimed launch that also measures the algorithmic bytes."""
        t = stm.stm_tuning_default(**{f[0]: getattr(self.tuning, f[0]) for f in self.tuning._fields_})
        t.instrument = 1
        if self.world == 1:
            c = stm.stm_match_count_ex(self.G.handle, plan.handle, t, None, None)
            return c, stm.stm_last_launch()
        slot = SLOTS - 1
        self.cursors[slot * 8].zero_()
        torch.cuda.synchronize(self.device)
        dist.barrier(group=self.group)
        part = stm.stm_match_count_ex(self.G.handle, plan.handle, t, self._shard(slot), None)
        info = stm.stm_last_launch()
        d = torch.tensor([part if part < (1 << 63) else part - (1 << 64)], dtype=torch.int64, device=self.device)
        dist.all_reduce(d, group=self.group)
        torch.cuda.synchronize(self.device)
        dist.barrier(group=self.group)
        return int(d.item()) & ((1 << 64) - 1), info

    # -- end to end ------------------------------------------------------------------------
    def e2e(self, g, plans: Sequence[stm.Plan], steps: int = 3):
        """Public-API end-to-end: pinned host CSR -> device (timed) -> stm_graph_load_device ->
        count every query -> (all-reduce) -> 8-byte read-backs.  Wall-clock per step."""
        rp = torch.from_numpy(g.row_ptr).pin_memory()
        ci = torch.from_numpy(g.col_idx).pin_memory()
        lb = torch.from_numpy(g.labels).pin_memory() if g.labels is not None else None
        h2d = rp.numel() * 8 + ci.numel() * 4 + (lb.numel() * 4 if lb is not None else 0)
        times = []
        for _ in range(steps):
            torch.cuda.synchronize(self.device)
            if self.world > 1:
                dist.barrier(group=self.group)
            t0 = time.perf_counter()
            d_rp = rp.to(self.device, non_blocking=True)
            d_ci = ci.to(self.device, non_blocking=True)
            d_lb = lb.to(self.device, non_blocking=True) if lb is not None else None
            torch.cuda.current_stream(self.device).synchronize()
            gh = stm.stm_graph_load_device(g.n, int(ci.numel()), d_rp.data_ptr(), d_ci.data_ptr(),
                                           d_lb.data_ptr() if d_lb is not None else None, self.device.index)
            out = torch.zeros(len(plans), dtype=torch.int64, device=self.device)
            for qi, pl in enumerate(plans):
                self.count_async(pl, out[qi:qi + 1], graph_handle=gh)
            self.reduce_counts(out)
            host = out.cpu()  # D2H of the step's result
            stm.stm_graph_free(gh)
            dt = time.perf_counter() - t0
            if self.world > 1:
                t = torch.tensor([dt], dtype=torch.float64, device=self.device)
                dist.all_reduce(t, op=dist.ReduceOp.MAX, group=self.group)
                dt = float(t.item())
            times.append(dt)
            del d_rp, d_ci, d_lb, host
        return {"seconds_per_step": sum(times) / len(times), "h2d_bytes_per_step": int(h2d),
                "d2h_bytes_per_step": 8 * len(plans),
                "path": "pinned host CSR -> torch H2D -> stm_graph_load_device -> stm_match_count_async "
                        "-> all_reduce -> D2H (wall clock, max over ranks)"}
