"""Pattern-sharded likelihood across GPUs (one process per GPU).

Site patterns are independent ("each character ... can be computed
autonomously, and subsequently combined", §I), so rank r of R owns
the contiguous pattern slice [r*ceil(p/R), min(p, (r+1)*ceil(p/R))) of every
tip, partials and scale buffer.  The tree, the reroot/schedule (a deterministic
host routine, identical on every rank, so nothing is broadcast) and the
transition matrices are replicated.  The only collective is the all-reduce of
the per-rank fp64 sum of wt_i lnL_i, performed in place on the device buffer
the library's K4 writes (NCCL over NVLink for CUDA tensors; gloo works for the
CPU-side tests of this wiring).
"""
from __future__ import annotations

import hashlib
import math

import numpy as np


def pattern_slice(p: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous slice of rank `rank` (the last rank may be shorter; a rank
    may be empty when world > p)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    chunk = math.ceil(p / world)
    lo = min(p, rank * chunk)
    return lo, min(p, lo + chunk)


def schedule_digest(sched: dict) -> str:
    """Hash of a schedule (ops + offsets + rerooted tree) -- equal on every rank."""
    h = hashlib.sha256()
    for k in ("parent", "blen", "ops", "set_offsets"):
        h.update(np.ascontiguousarray(sched[k]).tobytes())
    return h.hexdigest()


def allreduce_sum_(tensor, group=None, deterministic=False):
    """In-place SUM all-reduce of a 1-element fp64 tensor: on the device with
    NCCL; through a host copy with gloo (the CPU-side wiring tests and
    several ranks sharing one GPU, where NCCL refuses).

    deterministic=True: every rank writes its value into its
    own slot of a zero R-vector, the vector is all-reduced (x + 0 = x, so the
    reduction order cannot change a bit) and every rank folds the R slots in
    rank order -- the same bits on every rank and in every run, whatever
    order the collective adds in."""
    import torch.distributed as dist
    if not dist.is_initialized():  # a single process: the local sum is the global one
        return tensor
    if deterministic:
        import torch
        world, rank = dist.get_world_size(group), dist.get_rank(group)
        v = torch.zeros(world, dtype=tensor.dtype, device=tensor.device)
        v[rank] = tensor.reshape(())
        allreduce_sum_(v, group)
        acc = v[0].clone()
        for r in range(1, world):
            acc += v[r]
        tensor.copy_(acc.reshape(tensor.shape))
        return tensor
    if tensor.is_cuda and dist.get_backend(group) != "nccl":
        h = tensor.cpu()
        dist.all_reduce(h, op=dist.ReduceOp.SUM, group=group)
        tensor.copy_(h)
        return tensor
    dist.all_reduce(tensor, op=dist.ReduceOp.SUM, group=group)
    return tensor


class ShardedTreeLikelihood:
    """One rank's share of a pattern-sharded likelihood (wraps TreeLikelihood)."""

    def __init__(self, n: int, p_total: int, s: int, c: int, rank: int, world: int,
                 precision: int = 32, device: int = 0, cuda_graph: bool = True,
                 stream_ptr: int | None = None, group=None, buffer_count: int | None = None,
                 deterministic_reduce: bool = False):
        import torch

        from .engine import TreeLikelihood
        self.lo, self.hi = pattern_slice(p_total, rank, world)
        if self.hi <= self.lo:
            raise ValueError("empty pattern slice: use fewer ranks than patterns")
        self.group = group
        if stream_ptr is None:
            # the collective runs on torch's current stream: the library must
            # enqueue K4 on that same stream so all_reduce is ordered after it
            stream_ptr = torch.cuda.current_stream(device).cuda_stream
        self.tl = TreeLikelihood(n, self.hi - self.lo, s, c, precision=precision, device=device,
                                 cuda_graph=cuda_graph, stream_ptr=stream_ptr, buffer_count=buffer_count)
        self.stream_ptr = stream_ptr
        self.deterministic = deterministic_reduce
        self.device = device
        self.d_out = torch.zeros(1, dtype=torch.float64, device=f"cuda:{device}")

    def set_model_params(self, mp, rates, cat_weights):
        return self.tl.set_model_params(mp, rates, cat_weights)

    def set_tips(self, tips_full: np.ndarray):
        self.tl.set_tips(np.ascontiguousarray(tips_full[:, self.lo:self.hi]))

    def set_tips_local(self, tips_slice: np.ndarray):
        """This rank's columns [lo, hi) only (no full alignment on every rank)."""
        if tips_slice.shape[1] != self.hi - self.lo:
            raise ValueError(f"expected {self.hi - self.lo} pattern columns, got {tips_slice.shape[1]}")
        self.tl.set_tips(tips_slice)

    def set_pattern_weights(self, w_full):
        self.tl.set_pattern_weights(np.ascontiguousarray(w_full[self.lo:self.hi]))

    def set_tree(self, parent, blen, mode="reroot", reuse_buffers=False):
        return self.tl.set_tree(parent, blen, mode, reuse_buffers=reuse_buffers)

    def loglik_device(self):
        """Local pass + in-place all-reduce; returns the device tensor."""
        self.tl.update()
        self.tl.root_loglik_device(self.d_out.data_ptr())
        import torch
        if torch.cuda.current_stream(self.device).cuda_stream != self.stream_ptr:
            # the collective is enqueued on torch's current stream, not the
            # library's: K4 must have written d_out first
            from . import rrl as R
            R.rrl_synchronize(self.tl.inst)
        allreduce_sum_(self.d_out, self.group, deterministic=self.deterministic)
        return self.d_out

    def loglik(self) -> float:
        return float(self.loglik_device().item())

    def close(self):
        self.tl.close()
