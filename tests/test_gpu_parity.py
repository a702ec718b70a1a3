"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Tolerances (BASELINE.json north_star): reroot schedules bit-exact (CPU tests);
lnL fp64 relative <= 1e-10, fp32 relative <= 1e-4; per-node partials fp32
<= 1e-5 relative after scaling (per pattern, max over (c, z), reading A19),
fp64 <= 1e-12.
"""
import math

import numpy as np
import pytest

from oracle import model as om, pruning, reroot as orr
from workloads import Tree, config_workload, make_workload, with_blen

from ._util import gpu_setup, node_partial_error, oracle_run, rel, rooted

pytestmark = pytest.mark.gpu

LNL_TOL = {64: 1e-10, 32: 1e-4}
NODE_TOL = {64: 1e-12, 32: 1e-5}


@pytest.fixture(scope="module", autouse=True)
def _built():
    from paper_conf_ipps_ayresc18_b200 import build
    build.build()


# ------------------------------------------------------------------ K1
@pytest.mark.parametrize("precision", [64, 32])
@pytest.mark.parametrize("model", ["jc69", "hky", "gtr"])
def test_transition_matrices_vs_expm(precision, model):
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="random", n=40, p=10, model=model, c=4, seed=3)
    tl = gpu_setup(w, "level", precision)
    tl.update()
    Q = om.rate_matrix(w.model)
    tol = 2e-14 if precision == 64 else 2e-7
    for m in tl.matrix_idx[:20]:
        got = R.rrl_get_transition_matrix(tl.inst, int(m), w.c, w.s)
        for k in range(w.c):
            exp = pruning.transition_matrix(Q, w.rates[k] * w.tree.blen[m])
            np.testing.assert_allclose(got[k], exp, atol=tol, rtol=0)
    tl.close()


# ------------------------------------------------------------------ lnL parity, configs
CASES = [
    ("c0_jc", 64, {}),
    ("c0_hky", 64, {}),
    ("c1", 64, {}),
    ("c1", 32, {}),
    ("c2", 32, dict(p=20_000)),
    ("c2", 64, dict(p=20_000)),
    ("c2_paper", 32, dict(p=5_000)),
]


@pytest.mark.parametrize("name,precision,over", CASES)
@pytest.mark.parametrize("mode", ["reroot", "level"])
def test_loglik_matches_oracle(name, precision, over, mode):
    w = config_workload(name, seed=1, **over)
    tl = gpu_setup(w, mode, precision)
    got = tl.loglik()
    ora = oracle_run(w)                       # ORIGINAL rooting: reroot invariance
    assert rel(got, ora.lnl) <= LNL_TOL[precision], (got, ora.lnl)
    site = tl.site_logliks()
    np.testing.assert_allclose(site, ora.site_lnl, rtol=10 * LNL_TOL[precision])
    tl.close()


def test_c2_full_size_fp32_and_fp64():
    """BASELINE configs[2] at full size (1,024-tip Yule, 100,000 patterns)."""
    w = config_workload("c2", seed=1)
    ora = oracle_run(w)
    for precision in (32, 64):
        tl = gpu_setup(w, "reroot", precision)
        got = tl.loglik()
        assert rel(got, ora.lnl) <= LNL_TOL[precision], (precision, got, ora.lnl)
        tl.close()


# ------------------------------------------------------------------ per-node partials
@pytest.mark.parametrize("precision", [64, 32])
@pytest.mark.parametrize("kind,n,p", [("pectinate", 128, 2_000), ("yule", 300, 777),
                                      ("random", 64, 1_001), ("yule", 40, 17_001)])
def test_per_node_partials(precision, kind, n, p):
    w = make_workload(tree_kind=kind, n=n, p=p, model="gtr", c=4, seed=2, missing_frac=0.05)
    tl = gpu_setup(w, "reroot", precision)
    tl.update()
    ora = oracle_run(w, tree=rooted(tl), keep_partials=True)
    worst = 0.0
    for v, L in ora.partials.items():
        g = tl.partials(v)
        ge = tl.scale(v - n)                  # cumulative exponents (RRL_FLAG_SCALE_CUMULATIVE)
        err = node_partial_error(g, ge, L, ora.cum_exponent[v])
        worst = max(worst, float(err.max()))
    assert worst <= NODE_TOL[precision], worst
    tl.close()


# ------------------------------------------------------------------ schedules / modes
def test_schedule_invariance_fp64():
    w = make_workload(tree_kind="random", n=200, p=3_000, model="gtr", c=4, seed=4)
    vals = {}
    for mode in ("sequential", "level", "reroot"):
        tl = gpu_setup(w, mode, 64)
        vals[mode] = tl.loglik()
        tl.close()
    assert vals["sequential"] == vals["level"]          # same ops, same rooting: bit-identical
    assert rel(vals["reroot"], vals["level"]) <= 1e-12


def test_greedy_batching_and_graph_and_determinism():
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="yule", n=150, p=4_000, model="gtr", c=4, seed=5)
    tl = gpu_setup(w, "reroot", 32)
    a = tl.loglik()
    b = tl.loglik()
    assert a == b                                        # deterministic
    R.rrl_update_partials(tl.inst, tl.ops, None)          # greedy sets
    c = tl.root_loglik()
    assert c == a
    tl.close()
    tg = gpu_setup(w, "reroot", 32, graph=True)
    assert tg.loglik() == a and tg.loglik() == a         # graph capture, then replay
    prof = R.rrl_get_profile(tg.inst)
    assert prof["graph_launches"] == 2
    R.rrl_set_profiling(tg.inst, True)                   # per-set events inside the graph
    R.rrl_reset_profile(tg.inst)
    assert tg.loglik() == a and tg.loglik() == a
    prof = R.rrl_get_profile(tg.inst)
    assert prof["graph_launches"] == 2 and prof["partials_ms"] > 0
    assert prof["partials_launches"] == 2 * tg.sched["set_count"]
    tg.close()


def test_dependent_ops_in_one_set_rejected():
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="pectinate", n=8, p=64, model="gtr", c=4, seed=1)
    tl = gpu_setup(w, "level", 32)
    with pytest.raises(R.RRLError):
        R.rrl_update_partials(tl.inst, tl.ops, np.array([0, len(tl.ops)], np.int32))
    tl.close()


@pytest.mark.parametrize("precision", [64, 32])
def test_per_node_scaling_with_accumulate(precision):
    """Non-cumulative mode: own exponents per node + K5 accumulation."""
    w = make_workload(tree_kind="random", n=90, p=1_500, model="hky", c=4, seed=7)
    tl = gpu_setup(w, "reroot", precision, cumulative=False)
    got = tl.loglik()
    ora = oracle_run(w, tree=rooted(tl), keep_partials=True)
    assert rel(got, ora.lnl) <= LNL_TOL[precision]
    tl.close()
    w = make_workload(tree_kind="random", n=30, p=20_000, model="hky", c=4, seed=7)   # bulk path
    tl = gpu_setup(w, "reroot", precision, cumulative=False)
    got = tl.loglik()
    ora = oracle_run(w, tree=rooted(tl), keep_partials=True)
    assert rel(got, ora.lnl) <= LNL_TOL[precision]
    if precision == 64:
        tot = sum(tl.scale(v - w.n).astype(np.int64) for v in ora.partials)
        np.testing.assert_array_equal(tot, tl.scale(tl.n_scale - 1))
    tl.close()


def test_buffer_reuse_same_result():
    w = make_workload(tree_kind="pectinate", n=500, p=2_000, model="gtr", c=4, seed=3)
    a = gpu_setup(w, "reroot", 32)
    b = gpu_setup(w, "reroot", 32, reuse=True)
    assert b.nbuf < a.nbuf
    la, lb = a.loglik(), b.loglik()
    assert la == lb
    a.close()
    b.close()


# ------------------------------------------------------------------ edge cases
@pytest.mark.parametrize("precision", [64, 32])
@pytest.mark.parametrize("n,p", [(2, 1), (3, 5), (2, 1000), (5, 129), (17, 257)])
def test_tiny_and_ragged(precision, n, p):
    w = make_workload(tree_kind="random", n=n, p=p, model="gtr", c=4, seed=n + p)
    tl = gpu_setup(w, "reroot", precision)
    got = tl.loglik()
    assert rel(got, oracle_run(w).lnl) <= LNL_TOL[precision]
    tl.close()


@pytest.mark.parametrize("c,p", [(1, 500), (2, 500), (8, 500), (1, 70_001), (2, 33_333),
                                 (8, 8_200)])
def test_category_counts(c, p):
    """Latency path (few patterns) and bulk-copy path (>= 64K items per op)."""
    w = make_workload(tree_kind="yule", n=40, p=p, model="gtr", c=c, seed=c)
    tl = gpu_setup(w, "reroot", 64)
    assert rel(tl.loglik(), oracle_run(w).lnl) <= 1e-10
    tl.close()


@pytest.mark.parametrize("precision", [64, 32])
def test_long_branches_need_scaling(precision):
    """t = 50 on every branch of a 600-tip tree: lnL_i = sum ln pi_x exactly;
    the unscaled product underflows fp64, so this exercises the exponents."""
    w = make_workload(tree_kind="random", n=600, p=300, model="gtr", c=1, seed=8,
                      missing_frac=0.1)
    tree = with_blen(w.tree, 50.0)  # c = 1: rate 1, so every P is at its t -> inf limit
    tl = gpu_setup(w, "reroot", precision, tree=tree)
    got = tl.loglik()
    pi = w.model.pi
    exp = math.fsum(math.log(pi[x]) for x in w.tips.ravel() if x < 4)
    assert rel(got, exp) <= LNL_TOL[precision]
    tl.close()


def test_all_missing_and_zero_branch():
    w = make_workload(tree_kind="yule", n=30, p=50, model="gtr", c=4, seed=9)
    w.tips[:, 0] = 4
    for x in range(4):
        w.tips[:, 1 + x] = x
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    tl = gpu_setup(w, "reroot", 64)
    tl.loglik()
    site = tl.site_logliks()
    assert abs(site[0]) < 1e-13
    tl.close()
    tree = with_blen(w.tree, 0.0)          # non-constant patterns get L = 0 -> lnL = -inf
    tl = gpu_setup(w, "reroot", 64, tree=tree)
    tl.update()
    total = R.rrl_calculate_root_log_likelihoods(tl.inst, tl.root_buffer, 0, 0, tl.cumulative_idx,
                                                 allow_nonfinite=True)
    assert not np.isfinite(total)   # -inf (oracle) or NaN: P(0) = V Vinv is I only to ~1e-16
    site = tl.site_logliks()
    for x in range(4):
        assert abs(site[1 + x] - math.log(w.model.pi[x])) < 1e-13
    tl.close()


def test_tip_partials_equal_tip_states():
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="random", n=20, p=300, model="gtr", c=4, seed=10, missing_frac=0.1)
    tl = gpu_setup(w, "reroot", 64)
    a = tl.loglik()
    for tip in (0, 3, 7):
        L = pruning.tip_partials(w.tips[tip], 4)
        R.rrl_set_tip_partials(tl.inst, tip, L)
    b = tl.loglik()
    assert rel(b, a) <= 1e-13
    tl.close()


def test_tip_states_u8_validation_and_switch_back():
    """Device-side code check of rrl_set_tip_states_u8 (code > s fails with
    OUT_OF_RANGE, tips left all-missing); switching tips from partials back to
    states re-resolves the cached descriptors."""
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="random", n=20, p=300, model="gtr", c=4, seed=10, missing_frac=0.1)
    tl = gpu_setup(w, "reroot", 64)
    a = tl.loglik()
    for tip in (0, 3):
        R.rrl_set_tip_partials(tl.inst, tip, pruning.tip_partials(w.tips[tip], 4))
    tl.set_tips(w.tips)                       # back to states for every tip
    assert rel(tl.loglik(), a) <= 1e-13
    bad = w.tips.copy()
    bad[5, 299] = 5                           # > s = 4
    with pytest.raises(R.RRLError) as ei:
        tl.set_tips(bad)
    assert ei.value.code == R.ERROR_OUT_OF_RANGE
    assert abs(tl.loglik()) <= 1e-9           # every tip left all-missing: lnL = 0
    tl.set_tips(w.tips)
    assert rel(tl.loglik(), a) <= 1e-13
    tl.close()


def test_pattern_weights():
    w = make_workload(tree_kind="random", n=25, p=400, model="gtr", c=4, seed=11)
    w.pattern_weights = np.random.default_rng(0).integers(1, 5, 400).astype(np.float64)
    tl = gpu_setup(w, "reroot", 64)
    assert rel(tl.loglik(), oracle_run(w).lnl) <= 1e-10
    tl.close()


def test_edge_loglik_pulley():
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="balanced", n=32, p=500, model="gtr", c=4, seed=12)
    tl = gpu_setup(w, "level", 64)
    root_l = tl.loglik()
    t = w.tree
    ch = pruning.children_of(t.parent)
    a, b = ch[t.root]
    # matrix for branch a with length t_a + t_b
    R.rrl_update_transition_matrices(tl.inst, 0, np.array([a], np.int32),
                                     np.array([t.blen[a] + t.blen[b]]))
    e = R.rrl_calculate_edge_log_likelihoods(tl.inst, b, a, a, 0, 0, b - w.n, a - w.n)
    assert rel(e, root_l) <= 1e-12
    tl.close()


# ------------------------------------------------------------------ codon (61 states)
@pytest.mark.parametrize("precision", [64, 32])
def test_codon_transition_matrices(precision):
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="random", n=10, p=10, model="gy94", c=4, seed=3)
    tl = gpu_setup(w, "level", precision)
    tl.update()
    Q = om.rate_matrix(w.model)
    tol = 1e-12 if precision == 64 else 2e-7
    for m in tl.matrix_idx[:6]:
        got = R.rrl_get_transition_matrix(tl.inst, int(m), w.c, w.s)
        for k in range(w.c):
            exp = pruning.transition_matrix(Q, w.rates[k] * w.tree.blen[m])
            np.testing.assert_allclose(got[k], exp, atol=tol, rtol=0)
    tl.close()


@pytest.mark.parametrize("precision,simt", [(64, True), (32, True), (32, False)])
@pytest.mark.parametrize("mode", ["reroot", "level"])
def test_codon_loglik_c3(precision, simt, mode):
    """BASELINE configs[3] (256-tip random tree, GY94+G4) at 2,000 patterns;
    fp32 on both the SIMT kernel and the tcgen05 3xTF32 kernel."""
    w = config_workload("c3", seed=1, p=2_000)
    tl = gpu_setup(w, mode, precision, codon_simt=simt)
    got = tl.loglik()
    ora = oracle_run(w)
    assert rel(got, ora.lnl) <= LNL_TOL[precision], (got, ora.lnl)
    tl.close()


@pytest.mark.parametrize("precision,simt", [(64, True), (32, True), (32, False)])
@pytest.mark.parametrize("c,p", [(4, 130), (1, 64), (2, 65), (4, 1000), (8, 300)])
@pytest.mark.parametrize("matrices", ["oracle_expm", "gpu_k1"])
def test_codon_per_node_partials(precision, simt, c, p, matrices):
    """Per-node codon partials.  With the oracle's own expm matrices loaded
    through rrl_set_transition_matrix the K3 arithmetic is checked at the
    fp64 node tolerance.  With the GPU's eigen-route K1 matrices, codon P has
    entries down to ~1e-9 whose fp64 values differ from expm's by ~1e-16
    absolute (~1e-7 relative); partials dominated by such entries inherit that
    (reading "codon node tolerance"), so fp64 is held to 1e-6 there."""
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="yule", n=24, p=p, model="gy94", c=c, seed=5, missing_frac=0.05)
    tl = gpu_setup(w, "reroot", precision, codon_simt=simt)
    rt = rooted(tl)
    if matrices == "gpu_k1":
        tl.update()
        tol = NODE_TOL[precision] if precision == 32 else 1e-6
    else:
        Q = om.rate_matrix(w.model)
        for v in tl.matrix_idx:
            P = np.stack([pruning.transition_matrix(Q, r * rt.blen[v]) for r in w.rates])
            R.rrl_set_transition_matrix(tl.inst, int(v), P)
        R.rrl_update_partials(tl.inst, tl.ops, tl.offsets)
        tol = NODE_TOL[precision]
    ora = oracle_run(w, tree=rt, keep_partials=True)
    worst = 0.0
    for v, L in ora.partials.items():
        err = node_partial_error(tl.partials(v), tl.scale(v - w.n), L, ora.cum_exponent[v])
        worst = max(worst, float(err.max()))
    assert worst <= tol, worst
    assert rel(tl.root_loglik(), ora.lnl) <= LNL_TOL[precision]
    tl.close()


def test_codon_edge_pulley():
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="balanced", n=8, p=100, model="gy94", c=4, seed=12)
    tl = gpu_setup(w, "level", 64)
    root_l = tl.loglik()
    t = w.tree
    a, b = pruning.children_of(t.parent)[t.root]
    R.rrl_update_transition_matrices(tl.inst, 0, np.array([a], np.int32),
                                     np.array([t.blen[a] + t.blen[b]]))
    e = R.rrl_calculate_edge_log_likelihoods(tl.inst, b, a, a, 0, 0, b - w.n, a - w.n)
    assert rel(e, root_l) <= 1e-12
    tl.close()


# ------------------------------------------------------------------ sharding / full size
def test_emulated_pattern_sharding_sum():
    """R instances on contiguous pattern slices (one GPU): the sum of their
    root log-likelihoods equals the unsharded value (the all-reduce payload)."""
    from paper_conf_ipps_ayresc18_b200.parallel import pattern_slice
    w = make_workload(tree_kind="random", n=100, p=20_011, model="gtr", c=4, seed=21)
    full = gpu_setup(w, "reroot", 64)
    ref = full.loglik()
    full.close()
    tot = 0.0
    for r in range(3):
        lo, hi = pattern_slice(w.p, r, 3)
        ws = make_workload(tree_kind="random", n=100, p=20_011, model="gtr", c=4, seed=21)
        ws.tips = np.ascontiguousarray(ws.tips[:, lo:hi])
        ws.pattern_weights = ws.pattern_weights[lo:hi]
        tl = gpu_setup(ws, "reroot", 64)
        tot += tl.loglik()
        tl.close()
    assert rel(tot, ref) <= 1e-12


def test_sharded_engine_nccl_world1():
    import os
    import socket

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_ayresc18_b200.parallel import ShardedTreeLikelihood
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        w = make_workload(tree_kind="yule", n=64, p=3_000, model="gtr", c=4, seed=2)
        torch.cuda.set_stream(torch.cuda.Stream())
        sh = ShardedTreeLikelihood(w.n, w.p, w.s, w.c, 0, 1, precision=64,
                                   stream_ptr=torch.cuda.current_stream().cuda_stream)
        sh.set_model_params(w.model, w.rates, w.cat_weights)
        sh.set_tips(w.tips)
        sh.set_pattern_weights(w.pattern_weights)
        sh.set_tree(w.tree.parent, w.tree.blen)
        got = sh.loglik()
        sh.close()
    finally:
        dist.destroy_process_group()
    assert rel(got, oracle_run(w).lnl) <= 1e-10


@pytest.mark.slow
def test_c4_full_size_sampled_patterns():
    """BASELINE configs[4] at full size on one GPU (4,096-tip pectinate,
    4,194,304 patterns, fp32, rerooted, liveness buffer reuse, the launch
    configuration bench.py --config c4 times): strided per-pattern lnL against
    the oracle computed on just those columns."""
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = config_workload("c4", seed=1, p=1)
    p = 1 << 22
    rng = np.random.default_rng(np.random.SeedSequence([1, 7919, 0]))
    w.tips = rng.integers(0, 4, size=(w.n, p), dtype=np.uint8)
    w.pattern_weights = np.ones(p)
    tl = gpu_setup(w, "reroot", 32, reuse=True)
    assert tl.nbuf <= w.n + 8
    total = tl.loglik()
    site = tl.site_logliks()
    idx = np.arange(0, p, p // 256)
    sub = make_workload(tree_kind="pectinate", n=w.n, p=1, model="gtr", c=4, seed=1)
    sub.tips = np.ascontiguousarray(w.tips[:, idx])
    sub.pattern_weights = np.ones(idx.size)
    ora = oracle_run(sub)
    np.testing.assert_allclose(site[idx], ora.site_lnl, rtol=1e-4)
    assert np.isfinite(total)
    tl.close()


# ------------------------------------------------------------------ partial updates (NEXT-2)
@pytest.mark.parametrize("precision", [64, 32])
def test_partial_update_equals_full_recompute(precision):
    """Change one branch length, recompute only the path to the root
    (rrl_schedule_partial): bit-identical to a full pass."""
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="random", n=150, p=5_000, model="gtr", c=4, seed=31)
    tl = gpu_setup(w, "reroot", precision)
    tl.loglik()
    rt = rooted(tl)
    rng = np.random.default_rng(3)
    for _ in range(3):
        v = int(rng.choice(tl.matrix_idx))
        new_t = float(rng.uniform(0.01, 0.3))
        pos = int(np.flatnonzero(tl.matrix_idx == v)[0])
        tl.t[pos] = new_t
        R.rrl_update_transition_matrices(tl.inst, 0, np.array([v], np.int32), np.array([new_t]))
        sch = R.rrl_schedule_partial(w.n, rt.parent, np.array([rt.parent[v]], np.int32))
        R.rrl_update_partials(tl.inst, sch["ops"], sch["set_offsets"])
        partial = tl.root_loglik()
        full = tl.loglik()                    # K1 for all branches + every level set
        assert partial == full
        blen = rt.blen.copy()
        blen[v] = new_t
        rt = Tree(rt.n, rt.parent, blen)
        ora = oracle_run(w, tree=rt)
        assert rel(full, ora.lnl) <= LNL_TOL[precision]
    tl.close()


# ------------------------------------------------------------------ stored-factor rescaling (A6)
@pytest.mark.parametrize("kind,p,model,precision", [("yule", 3_000, "gtr", 32), ("yule", 20_000, "gtr", 64),
                                                    ("random", 300, "gy94", 32), ("random", 200, "gy94", 64)])
def test_dest_scale_read_reuses_factors(kind, p, model, precision):
    """The paper's timed regime computes new factors once per 1,000 passes and
    reuses them otherwise (reading A6).  Per-node mode:
    pass 1 writes own exponents; pass 2 applies them (dest_scale_read) and must
    reproduce every node bit for bit."""
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind=kind, n=40, p=p, model=model, c=4, seed=17)
    tl = gpu_setup(w, "reroot", precision, cumulative=False)
    first = tl.loglik()
    nodes = [int(d) for d in tl.ops["dest"]]
    before = {v: tl.partials(v) for v in nodes[::7]}
    ops2 = tl.ops.copy()
    ops2["dest_scale_read"] = ops2["dest_scale_write"]
    ops2["dest_scale_write"] = -1
    R.rrl_update_partials(tl.inst, ops2, tl.offsets)
    for v, L in before.items():
        np.testing.assert_array_equal(tl.partials(v), L)
    assert tl.root_loglik() == first
    tl.close()


@pytest.mark.parametrize("precision", [64, 32])
def test_unscaled_bulk_pass_with_tip_pairs(precision):
    """Bulk-path operations with two tip children read their whole output from a
    per-operation table of the 5 x 5 state pairs (missing included); with no
    rescaling at all (dest_scale_write = dest_scale_read = -1) the pass must
    still match the oracle (small tree: nothing underflows)."""
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind="yule", n=30, p=20_000, model="gtr", c=4, seed=23, missing_frac=0.1)
    tl = gpu_setup(w, "reroot", precision, cumulative=False)
    R.rrl_update_transition_matrices(tl.inst, 0, tl.matrix_idx, tl.t)
    ops = tl.ops.copy()
    ops["dest_scale_write"] = -1
    ops["dest_scale_read"] = -1
    R.rrl_update_partials(tl.inst, ops, tl.offsets)
    got = R.rrl_calculate_root_log_likelihoods(tl.inst, tl.root_buffer, 0, 0, tl.n_scale - 1)  # zeros
    ora = oracle_run(w)
    assert rel(got, ora.lnl) <= LNL_TOL[precision], (got, ora.lnl)
    tl.close()


# ------------------------------------------------------------------ pattern partitions (NEXT-3)
@pytest.mark.parametrize("precision,s_model", [(64, "gtr"), (32, "gtr"), (32, "gy94"), (64, "gy94"),
                                               (32, "gtr_bulk"), (64, "gtr_bulk")])
def test_pattern_partitions_one_launch_per_set(precision, s_model):
    """PAPER.md:75-79 §IV-A: partitions with independent models computed
    concurrently by the multi-operation kernel -- every level set of all
    partitions is ONE launch; each partition matches the oracle run on its
    own columns with its own model."""
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R
    from workloads import random_model, discrete_gamma_rates
    codon = s_model == "gy94"
    bulk = s_model == "gtr_bulk"           # >= 64 K items per op: the bulk-copy kernel
    s_model = "gtr" if bulk else s_model
    p = 1200 if codon else (40_000 if bulk else 2600)
    ranges = ([(0, 512), (512, 1024), (1024, p)] if codon else
              [(0, 20_480), (20_480, 33_280), (33_280, p)] if bulk else [(0, 1024), (1024, 2048), (2048, p)])
    w = make_workload(tree_kind="random", n=30, p=p, model=s_model, c=4, seed=41, missing_frac=0.05)
    rng = np.random.default_rng(5)
    names = ["gy94"] * 3 if codon else ["gtr", "hky", "gtr"]
    models = [random_model(nm, rng) for nm in names]
    rates = [discrete_gamma_rates(a, 4) for a in (0.3, 0.9, 1.7)]
    cw = np.full(4, 0.25)
    tl = TreeLikelihood(w.n, p, w.s, 4, precision=precision, partitions=3)
    for k in range(3):
        tl.set_partition_model(k, models[k], rates[k], cw)
    tl.set_partition_ranges(ranges)
    tl.set_tips(w.tips)
    tl.set_tree(w.tree.parent, w.tree.blen, "reroot")
    R.rrl_reset_profile(tl.inst)
    tl.update()
    prof = R.rrl_get_profile(tl.inst)
    assert prof["partials_launches"] == tl.sched["set_count"]   # not 3x
    got = tl.partition_logliks()
    for k, (b, e) in enumerate(ranges):
        sub = make_workload(tree_kind="random", n=30, p=1, model=s_model, c=4, seed=41,
                            model_params=models[k], alpha=1.0)
        sub.rates = rates[k]
        sub.tips = np.ascontiguousarray(w.tips[:, b:e])
        sub.pattern_weights = np.ones(e - b)
        assert rel(got[k], oracle_run(sub).lnl) <= LNL_TOL[precision], k
    tl.close()


# ------------------------------------------------------------------ fused pass (RRL_FLAG_FUSED_PASS)
FUSED_CASES = [  # (kind, n, p, c, precision, mode, cumulative, reuse)
    ("pectinate", 128, 10_000, 4, 32, "reroot", True, False),    # configs[1]
    ("pectinate", 128, 10_000, 4, 32, "level", True, False),
    ("pectinate", 128, 10_000, 4, 64, "reroot", True, False),
    ("yule", 300, 777, 4, 32, "reroot", True, False),
    ("yule", 300, 777, 4, 64, "sequential", True, False),
    ("random", 64, 1_001, 1, 32, "reroot", False, False),
    ("random", 64, 1_001, 2, 64, "reroot", False, False),
    ("random", 90, 3_333, 8, 32, "reroot", True, False),
    ("pectinate", 500, 2_000, 4, 32, "reroot", True, True),     # liveness buffer reuse
    ("yule", 40, 17_001, 4, 64, "reroot", True, False),        # bulk path when not fused
    ("random", 3, 5, 4, 32, "reroot", True, False),
    ("random", 2, 1, 4, 64, "reroot", True, False),
]


@pytest.mark.parametrize("kind,n,p,c,precision,mode,cumulative,reuse", FUSED_CASES)
def test_fused_pass_bit_identical_to_level_sets(kind, n, p, c, precision, mode, cumulative, reuse):
    """One launch per pass (each thread owns its items across all level sets)
    gives the per-set launches' results bit for bit, and the oracle's lnL."""
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    w = make_workload(tree_kind=kind, n=n, p=p, model="gtr", c=c, seed=n + p + c, missing_frac=0.05)
    a = gpu_setup(w, mode, precision, cumulative=cumulative, reuse=reuse)
    b = gpu_setup(w, mode, precision, cumulative=cumulative, reuse=reuse, fused=True)
    la, lb = a.loglik(), b.loglik()
    assert la == lb, (la, lb)
    assert rel(lb, oracle_run(w).lnl) <= LNL_TOL[precision]
    if not reuse:
        for v in range(n, 2 * n - 1):
            np.testing.assert_array_equal(a.partials(v), b.partials(v))
    for k in range(b.n_scale):
        np.testing.assert_array_equal(a.scale(k), b.scale(k))
    R.rrl_reset_profile(b.inst)
    b.loglik()
    assert R.rrl_get_profile(b.inst)["partials_launches"] == 1
    a.close()
    b.close()


def test_fused_pass_graph_replay():
    w = make_workload(tree_kind="yule", n=150, p=4_000, model="gtr", c=4, seed=5)
    a = gpu_setup(w, "reroot", 32)
    g = gpu_setup(w, "reroot", 32, graph=True, fused=True)
    ref = a.loglik()
    assert g.loglik() == ref and g.loglik() == ref         # capture, then replay
    a.close()
    g.close()
