"""Host orchestration of one likelihood pass through the C ABI (no arithmetic here).

``TreeLikelihood`` is the public entry point a user calls: it owns one
instance of the library (one GPU, one stream), loads a model / alignment /
tree, and runs the hot path of SURVEY.md §8(a):

  a1+a2  rrl_reroot_and_schedule      (C++ host, once per tree)
  a3     rrl_update_transition_matrices (K1)
  a4     rrl_update_partials            (one K2/K3 launch per level set)
  a5     scale accumulation             (fused into a4 by default, or K5)
  a6     rrl_calculate_root_log_likelihoods(_device) (K4)
  a7     all-reduce of the fp64 sum      (torch.distributed, see parallel.py)

Every numeric step runs in librrl.so; this module only marshals arguments.
"""
from __future__ import annotations

import numpy as np

from . import rrl as R


def model_param_vector(name: str, kappa: float = 1.0, omega: float = 1.0, exch=None) -> list[float]:
    if name == "jc69":
        return []
    if name == "hky":
        return [float(kappa)]
    if name == "gtr":
        return [float(x) for x in exch]
    if name == "gy94":
        return [float(kappa), float(omega)]
    raise ValueError(name)


class TreeLikelihood:
    """One instance: n tips, p patterns, s states, c categories, fp32|fp64."""

    def __init__(self, n: int, p: int, s: int, c: int, precision: int = 32, device: int = 0,
                 cumulative_scaling: bool = True, cuda_graph: bool = False,
                 buffer_count: int | None = None, stream_ptr: int | None = None,
                 codon_simt: bool = False, partitions: int = 1, fused_pass: bool = False):
        self.n, self.p, self.s, self.c, self.precision = n, p, s, c, precision
        self.cumulative = cumulative_scaling
        nbuf = buffer_count if buffer_count is not None else 2 * n - 1
        n_scale = nbuf - n + (0 if cumulative_scaling else 1)
        flags = (R.FLAG_SCALE_CUMULATIVE if cumulative_scaling else 0) | \
                (R.FLAG_CUDA_GRAPH if cuda_graph else 0) | (R.FLAG_CODON_SIMT if codon_simt else 0) | \
                (R.FLAG_FUSED_PASS if fused_pass else 0)
        self.nbuf = nbuf
        self.n_scale = n_scale
        self.partitions = partitions
        self.ranges = None
        self.inst = R.rrl_create_instance(n, nbuf, s, p, c, partitions * (2 * n - 1), partitions, n_scale,
                                          device, precision, flags)
        if stream_ptr is not None:
            R.rrl_set_stream(self.inst, stream_ptr)
        self.sched = None

    # ---------------------------------------------------------------- inputs
    def set_model(self, name: str, pi, rates, cat_weights, kappa=1.0, omega=1.0, exch=None):
        prm = model_param_vector(name, kappa, omega, exch)
        Q, V, Vi, lam = R.rrl_model_eigensystem(name, pi, prm)
        R.rrl_set_eigen_decomposition(self.inst, 0, V, Vi, lam)
        R.rrl_set_state_frequencies(self.inst, 0, pi)
        R.rrl_set_category_rates(self.inst, rates)
        R.rrl_set_category_weights(self.inst, 0, cat_weights)
        self.Q = Q
        return Q

    def set_model_params(self, mp, rates, cat_weights):
        """Convenience for any object with name/pi/kappa/omega/exch attributes."""
        return self.set_model(mp.name, mp.pi, rates, cat_weights, getattr(mp, "kappa", 1.0),
                              getattr(mp, "omega", 1.0), getattr(mp, "exch", None))

    def set_partition_model(self, k: int, mp, rates, cat_weights):
        """Model of partition k (independent parameters per data
        subset): eigensystem, frequencies, category weights and rates in slot k."""
        prm = model_param_vector(mp.name, getattr(mp, "kappa", 1.0), getattr(mp, "omega", 1.0),
                                 getattr(mp, "exch", None))
        _, V, Vi, lam = R.rrl_model_eigensystem(mp.name, mp.pi, prm)
        R.rrl_set_eigen_decomposition(self.inst, k, V, Vi, lam)
        R.rrl_set_state_frequencies(self.inst, k, mp.pi)
        R.rrl_set_category_rates_idx(self.inst, k, rates)
        R.rrl_set_category_weights(self.inst, k, cat_weights)

    def set_partition_ranges(self, ranges):
        """[(begin, end)] per partition; begins multiples of RRL_PATTERN_RANGE_ALIGN."""
        assert len(ranges) == self.partitions
        self.ranges = [(int(b), int(e)) for b, e in ranges]

    def set_tips(self, tips_u8: np.ndarray):
        R.rrl_set_tip_states_u8(self.inst, 0, tips_u8, self.p)

    def set_pattern_weights(self, w):
        R.rrl_set_pattern_weights(self.inst, w)

    # NEXT-4 cost model parameters (rrl_schedule_cost): fixed cost of one
    # level-set launch and sustained HBM bandwidth, fitted to the measured
    # 1,024-pectinate sweep (DESIGN.md §9 "NEXT-4"); L2 size of the device.
    launch_us = 2.0
    hbm_gbs = 6225.0
    l2_bytes = 126e6

    def predicted_us(self, sch) -> float:
        return R.rrl_schedule_cost(self.n, sch["ops"], sch["set_offsets"], self.p, self.s, self.c,
                                   self.precision, self.launch_us, self.hbm_gbs, self.l2_bytes)

    def set_tree(self, parent, blen, mode: str = "auto", reuse_buffers: bool = False):
        """mode: "sequential" | "level" | "reroot" | "auto" (default) -- auto
        reroots only when the cost model predicts the rerooted schedule to be
        faster (NEXT-4): every measured point of the
        1,024-pectinate sweep below 10^6 fp32 patterns, not that one
        (profiles/r02_reroot_sweep.json)."""
        if reuse_buffers and not self.cumulative:
            # recycled buffers recycle their scale buffers too: per-node exponents
            # of consumed children would be overwritten before K5 sums them
            raise ValueError("reuse_buffers needs cumulative_scaling=True")
        if mode == "auto":
            cand = [R.rrl_reroot_and_schedule(self.n, parent, blen, m, reuse_buffers) for m in ("reroot", "level")]
            cost = [self.predicted_us(c) for c in cand]
            self.auto_choice = {"reroot_us": cost[0], "level_us": cost[1],
                                "mode": "reroot" if cost[0] <= cost[1] else "level"}
            mode = self.auto_choice["mode"]
        sch = R.rrl_reroot_and_schedule(self.n, parent, blen, mode, reuse_buffers)
        if sch["buffer_count"] > self.nbuf:
            raise ValueError(f"schedule needs {sch['buffer_count']} buffers, instance has {self.nbuf}")
        par = sch["parent"]
        self.root = int(np.flatnonzero(par < 0)[0])
        nonroot = np.flatnonzero(par >= 0).astype(np.int32)
        self.matrix_idx = nonroot
        self.t = sch["blen"][nonroot].copy()
        ops = sch["ops"]
        # physical buffer holding the root (last op of the last set)
        self.root_buffer = int(ops["dest"][-1])
        self.sched = sch
        self.reuse = reuse_buffers
        self.tree_parent, self.tree_blen = par.copy(), sch["blen"].copy()
        self.ops = ops
        self.offsets = sch["set_offsets"]
        self._pops = None
        return sch

    def update_tree(self, parent, blen, reroot: bool = False) -> dict:
        """Bring the stored partials up to date for a changed tree (topology
        moves, branch lengths; NEXT-2): only the nodes whose
        rooted subtree changed are recomputed (rrl_schedule_update, reading
        A28), level-batched, optionally on the rooting that minimises this
        update's sets.  K1 refreshes every matrix (one launch).  Needs identity
        buffers and a previous full pass.  Returns the update schedule."""
        if self.sched is None or self.reuse or self.partitions > 1:
            raise ValueError("update_tree needs a full pass on identity buffers first")
        sch = R.rrl_schedule_update(self.n, self.tree_parent, self.tree_blen, parent, blen, reroot)
        par = sch["parent"]
        nonroot = np.flatnonzero(par >= 0).astype(np.int32)
        self.matrix_idx = nonroot
        self.t = sch["blen"][nonroot].copy()
        R.rrl_update_transition_matrices(self.inst, 0, self.matrix_idx, self.t)
        if sch["op_count"] > 0:
            R.rrl_update_partials(self.inst, sch["ops"], sch["set_offsets"])
        if not self.cumulative:  # per-node exponents: re-sum every internal node's
            cum = self.n_scale - 1
            R.rrl_reset_scale_factors(self.inst, cum)
            R.rrl_accumulate_scale_factors(self.inst, np.arange(self.n - 1, dtype=np.int32), cum)
        self.root = int(np.flatnonzero(par < 0)[0])
        self.root_buffer = self.root
        self.tree_parent, self.tree_blen = par.copy(), sch["blen"].copy()
        # later full passes run the level sets of the tree as it now stands
        full = R.rrl_reroot_and_schedule(self.n, par, sch["blen"], "level")
        self.sched = full
        self.ops = full["ops"]
        self.offsets = full["set_offsets"]
        self._pops = None
        return sch

    # ---------------------------------------------------------------- pass
    def _partitioned_ops(self):
        """Every level set of every partition in ONE set: partition k's copy of
        an op uses matrices k*(2n-1)+node and its own pattern range."""
        N = 2 * self.n - 1
        ops, ranges, offs = [], [], [0]
        for a, b in zip(self.offsets[:-1], self.offsets[1:]):
            for k, (pb, pe) in enumerate(self.ranges):
                o = self.ops[a:b].copy()
                o["matrix1"] += k * N
                o["matrix2"] += k * N
                ops.append(o)
                ranges += [(pb, pe)] * (b - a)
            offs.append(offs[-1] + (b - a) * self.partitions)
        return np.concatenate(ops), np.array(ranges, np.int32), np.array(offs, np.int32)

    def update(self):
        """K1 + all level-set launches (+ K5 when not cumulative)."""
        if self.partitions > 1:
            N = 2 * self.n - 1
            for k in range(self.partitions):
                R.rrl_update_transition_matrices(self.inst, k, self.matrix_idx + k * N, self.t)
            if getattr(self, "_pops", None) is None or self._pops_key is not self.ops:
                self._pops = self._partitioned_ops()
                self._pops_key = self.ops
            R.rrl_update_partials_ranged(self.inst, self._pops[0], self._pops[1], self._pops[2])
        else:
            R.rrl_update_transition_matrices(self.inst, 0, self.matrix_idx, self.t)
            R.rrl_update_partials(self.inst, self.ops, self.offsets)
        if not self.cumulative:
            cum = self.n_scale - 1
            R.rrl_reset_scale_factors(self.inst, cum)
            R.rrl_accumulate_scale_factors(self.inst, self.ops["dest_scale_write"], cum)

    @property
    def cumulative_idx(self) -> int:
        return (self.root_buffer - self.n) if self.cumulative else self.n_scale - 1

    def root_loglik(self) -> float:
        return R.rrl_calculate_root_log_likelihoods(self.inst, self.root_buffer, 0, 0,
                                                    self.cumulative_idx)

    def root_loglik_device(self, d_out_ptr: int):
        R.rrl_calculate_root_log_likelihoods_device(self.inst, self.root_buffer, 0, 0,
                                                    self.cumulative_idx, d_out_ptr)

    def partition_logliks(self) -> list[float]:
        """Root log-likelihood of each partition (its model slot, its range)."""
        return [R.rrl_calculate_root_log_likelihoods_range(self.inst, self.root_buffer, k, k,
                                                           self.cumulative_idx, b, e)
                for k, (b, e) in enumerate(self.ranges)]

    def loglik(self) -> float:
        self.update()
        return self.root_loglik()

    def site_logliks(self) -> np.ndarray:
        return R.rrl_get_site_log_likelihoods(self.inst, self.p)

    def partials(self, buffer: int) -> np.ndarray:
        return R.rrl_get_partials(self.inst, buffer, self.c, self.p, self.s)

    def scale(self, idx: int) -> np.ndarray:
        return R.rrl_get_scale_factors(self.inst, idx, self.p)

    def close(self):
        if getattr(self, "inst", None) is not None:
            R.rrl_finalize_instance(self.inst)
            self.inst = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
