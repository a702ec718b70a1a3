"""Multi-process (gloo, world_size 2, CPU) tests of the pattern-sharding wiring.

No GPU here: each rank computes its shard's sum of site log-likelihoods with
the oracle and the all-reduce must reproduce the unsharded oracle value; the
C++ schedule must be bit-identical on both ranks (no broadcast is needed).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_ayresc18_b200.parallel import allreduce_sum_, pattern_slice, schedule_digest


def test_pattern_slice_covers_exactly():
    for p in (1, 7, 10_000, 4_194_304):
        for world in (1, 2, 3, 4, 8):
            spans = [pattern_slice(p, r, world) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == p
            for (a, b), (c, d) in zip(spans, spans[1:]):
                assert b == c and a <= b
    with pytest.raises(ValueError):
        pattern_slice(10, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import model as om, pruning
        from paper_conf_ipps_ayresc18_b200 import build
        build.build()
        from paper_conf_ipps_ayresc18_b200 import rrl as R
        from workloads import make_workload
        w = make_workload(tree_kind="random", n=30, p=501, model="gtr", c=4, seed=3)
        lo, hi = pattern_slice(w.p, rank, world)
        sched = R.rrl_reroot_and_schedule(w.n, w.tree.parent, w.tree.blen, "reroot")
        dig = schedule_digest(sched)
        digs = [None] * world
        dist.all_gather_object(digs, dig)
        Q = om.rate_matrix(w.model)
        part = pruning.prune(w.tree, Q, w.model.pi, w.rates, w.cat_weights, w.tips[:, lo:hi],
                             w.pattern_weights[lo:hi])
        t = torch.tensor([part.lnl], dtype=torch.float64)
        allreduce_sum_(t)
        full = pruning.prune(w.tree, Q, w.model.pi, w.rates, w.cat_weights, w.tips,
                             w.pattern_weights).lnl
        q.put((rank, float(t.item()), full, len(set(digs))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_sharded_sum_equals_unsharded(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, got, full, ndig in res:
        assert ndig == 1                      # identical schedule on every rank
        assert abs(got - full) <= 1e-12 * abs(full)


def _det_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        vals = [0.1, 1e16, -1e16, 0.3][:world]   # order-sensitive in floating point
        t = torch.tensor([vals[rank]], dtype=torch.float64)
        allreduce_sum_(t, deterministic=True)
        ref = 0.0
        for v in vals:
            ref += v
        q.put((rank, float(t.item()), ref))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_deterministic_allreduce_folds_in_rank_order(world):
    """one-hot R-vector all-reduce -- every rank gets the rank-order
    fold of the per-rank values, bit for bit."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_det_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, got, ref in res:
        assert got == ref
