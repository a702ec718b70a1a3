"""CPU tests of the C-ABI library's host code (no GPU needed).

* every symbol include/rrl.h declares is exported by librrl.so;
* the C++ O(n) reroot + schedule (rrl_reroot_and_schedule) is bit-exact
  against the oracle's exhaustive search and its level sets;
* the C++ model builder + Jacobi eigensystem reproduces the oracle's Q.
"""
import ctypes
import math
import os
import re

import numpy as np
import pytest

from oracle import model as om, reroot as orr
from workloads import make_tree, random_model

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def R():
    from paper_conf_ipps_ayresc18_b200 import build
    build.build()
    from paper_conf_ipps_ayresc18_b200 import rrl
    return rrl


def test_header_symbols_exported(R):
    hdr = open(os.path.join(ROOT, "include", "rrl.h")).read()
    names = set(re.findall(r"\b(rrl_[a-z0-9_]+)\s*\(", hdr))
    assert len(names) >= 30
    lib = ctypes.CDLL(R.LIB_PATH)
    for n in sorted(names):
        assert hasattr(lib, n), n
    assert set(R.EXPORTED) == names


def test_error_strings(R):
    assert R.rrl_error_string(R.ERROR_INVALID_TREE) == "invalid tree"
    assert "sm_100a" in R.rrl_version()


def _ops_tuple(ops):
    return [tuple(int(x) for x in o) for o in ops.tolist()]


@pytest.mark.parametrize("kind", ["pectinate", "random", "yule", "balanced"])
@pytest.mark.parametrize("n", [2, 3, 4, 7, 8, 33, 64, 150])
def test_reroot_schedule_bit_exact_vs_oracle(R, kind, n):
    for seed in (1, 2, 3):
        t = make_tree(kind, n, seed=seed)
        for mode in ("sequential", "level", "reroot"):
            rt, ops, offs, key = orr.reroot_and_schedule(t, mode)
            got = R.rrl_reroot_and_schedule(n, t.parent, t.blen, mode)
            assert got["root_edge"] == key, (mode, seed)
            assert np.array_equal(got["parent"], rt.parent)
            assert np.array_equal(got["blen"], rt.blen)          # bit-exact fp64
            assert _ops_tuple(got["ops"]) == ops
            assert got["set_offsets"].tolist() == offs
            assert got["buffer_count"] == 2 * n - 1


@pytest.mark.parametrize("kind", ["random", "yule", "pectinate"])
def test_edge_table_matches_exhaustive(R, kind):
    t = make_tree(kind, 120, seed=5)
    key, sets, imb = R.rrl_reroot_edge_table(120, t.parent)
    _, _, table = orr.best_rooting(t, with_table=True)
    exp = sorted((k, s, i) for s, _, i, k in table)
    assert list(zip(key.tolist(), sets.tolist(), imb.tolist())) == exp


def test_large_trees_closed_form(R):
    """n up to 4096: rerooted set count = ceil((D+1)/2) (survey identity) and
    the pectinate formulas of PAPER.md:96."""
    for n in (406, 1024, 4096):
        t = make_tree("pectinate", n, seed=1)
        assert R.rrl_reroot_and_schedule(n, t.parent, t.blen, "level")["set_count"] == n - 1
        g = R.rrl_reroot_and_schedule(n, t.parent, t.blen, "reroot")
        assert g["set_count"] == math.ceil(n / 2)
        w = np.diff(g["set_offsets"])
        assert w.max() == 2 and w.sum() == n - 1
    for seed in range(1, 6):
        t = make_tree("random", 1024, seed=seed)
        g = R.rrl_reroot_and_schedule(1024, t.parent, t.blen, "reroot")
        assert g["set_count"] == math.ceil((orr.unrooted_diameter(t) + 1) / 2)


def test_reuse_buffers_is_a_valid_allocation(R):
    for kind, n in (("pectinate", 300), ("random", 200), ("yule", 257)):
        t = make_tree(kind, n, seed=2)
        full = R.rrl_reroot_and_schedule(n, t.parent, t.blen, "reroot")
        re_ = R.rrl_reroot_and_schedule(n, t.parent, t.blen, "reroot", reuse_buffers=True)
        assert re_["buffer_count"] < full["buffer_count"]
        assert re_["set_offsets"].tolist() == full["set_offsets"].tolist()
        # simulate: logical node -> physical buffer must hold the value until read
        phys_of = {}
        holder = {}
        offs = re_["set_offsets"]
        for k in range(len(offs) - 1):
            lo, hi = offs[k], offs[k + 1]
            logical = full["ops"][lo:hi]
            physical = re_["ops"][lo:hi]
            for lo_op, ph_op in zip(logical, physical):
                for cl, cp in ((lo_op["child1"], ph_op["child1"]), (lo_op["child2"], ph_op["child2"])):
                    if cl < n:
                        assert cp == cl
                    else:
                        assert holder[cp] == cl      # still holds the child's value
                assert ph_op["matrix1"] == lo_op["matrix1"]
                assert ph_op["dest_scale_write"] == ph_op["dest"] - n
            dests = set(int(x) for x in physical["dest"])
            reads = set(int(x) for x in physical["child1"]) | set(int(x) for x in physical["child2"])
            assert not (dests & reads)
            for lo_op, ph_op in zip(logical, physical):
                holder[int(ph_op["dest"])] = int(lo_op["dest"])
                phys_of[int(lo_op["dest"])] = int(ph_op["dest"])
        # pectinate rerooted needs only a handful of internal buffers
        if kind == "pectinate":
            assert re_["buffer_count"] - n <= 6


def test_invalid_trees_rejected(R):
    t = make_tree("random", 10, seed=1)
    bad = t.parent.copy()
    bad[3] = 3
    with pytest.raises(R.RRLError) as e:
        R.rrl_reroot_and_schedule(10, bad, t.blen)
    assert e.value.code == R.ERROR_INVALID_TREE
    bad = t.parent.copy()
    bad[bad < 0] = 12          # no root -> cycle
    with pytest.raises(R.RRLError):
        R.rrl_reroot_and_schedule(10, bad, t.blen)
    with pytest.raises(R.RRLError):
        R.rrl_reroot_and_schedule(1, np.array([-1]), np.array([0.0]))


@pytest.mark.parametrize("name", ["jc69", "hky", "gtr", "gy94"])
def test_model_eigensystem_vs_oracle(R, name):
    from paper_conf_ipps_ayresc18_b200.engine import model_param_vector
    mp = random_model(name, np.random.default_rng(17))
    Q, V, Vi, lam = R.rrl_model_eigensystem(name, mp.pi, model_param_vector(
        name, mp.kappa, mp.omega, mp.exch))
    Qo = om.rate_matrix(mp)
    np.testing.assert_allclose(Q, Qo, atol=1e-14, rtol=1e-12)
    s = mp.states
    np.testing.assert_allclose(V @ Vi, np.eye(s), atol=1e-12)
    np.testing.assert_allclose(V @ np.diag(lam) @ Vi, Qo, atol=1e-12)
    assert abs(np.sort(lam)[-1]) < 1e-12     # one zero eigenvalue, rest negative
    assert np.all(np.sort(lam)[:-1] < 0)


@pytest.mark.parametrize("kind", ["random", "yule", "pectinate", "balanced"])
def test_partial_schedule_matches_oracle(R, kind):
    rng = np.random.default_rng(1)
    for n in (3, 10, 64, 200):
        t = make_tree(kind, n, seed=n)
        for _ in range(5):
            k = int(rng.integers(1, 4))
            nodes = rng.integers(n, 2 * n - 1, size=k)
            exp_ops, exp_offs = orr.schedule_partial(t, nodes.tolist())
            got = R.rrl_schedule_partial(n, t.parent, nodes)
            assert _ops_tuple(got["ops"]) == exp_ops
            assert got["set_offsets"].tolist() == exp_offs
    with pytest.raises(R.RRLError):
        R.rrl_schedule_partial(5, make_tree("random", 5, seed=1).parent, np.array([2]))


def test_exhaustive_cpp_equals_dp(R):
    """The paper's O(n^2) search (C++) and the O(n) DP choose the same edge."""
    for kind in ("random", "yule", "pectinate"):
        for seed in range(1, 6):
            t = make_tree(kind, 300, seed=seed)
            key, sets = R.rrl_reroot_exhaustive(300, t.parent, t.blen)
            g = R.rrl_reroot_and_schedule(300, t.parent, t.blen, "reroot")
            assert key == g["root_edge"] and sets == g["set_count"]


# ------------------------------------------------------------------ NEXT-2: moves + update schedules
def _random_move_pair(R, t, rng):
    """One random legal SPR or NNI, applied by the oracle and by the C++."""
    from oracle import moves
    from oracle.pruning import children_of
    n = t.n
    while True:
        if rng.random() < 0.5:
            x = int(rng.integers(0, 2 * n - 1))
            if x == t.root or t.parent[x] == t.root:
                continue
            r = int(rng.integers(0, 2 * n - 1))
            if r in moves._subtree_nodes(t, x) | {int(t.parent[x]), t.root}:
                continue
            return moves.spr(t, x, r), R.rrl_tree_spr(n, t.parent, t.blen, x, r)
        keys = [k for k, u, v, _ in orr.unrooted_edges(t) if u >= n and v >= n]
        k, which = keys[int(rng.integers(0, len(keys)))], int(rng.integers(0, 2))
        return moves.nni(t, k, which), R.rrl_tree_nni(n, t.parent, t.blen, k, which)


@pytest.mark.parametrize("kind,n", [("random", 40), ("pectinate", 33), ("yule", 64), ("balanced", 32)])
def test_moves_and_update_schedule_bit_exact_vs_oracle(R, kind, n):
    from oracle import moves
    for seed in (1, 2, 3):
        t0 = make_tree(kind, n, seed=seed)
        stored = orr.RTree(n, t0.parent.copy(), t0.blen.copy())
        rng = np.random.default_rng(seed)
        new = stored
        for step in range(4):
            o, (cp, cb) = _random_move_pair(R, new, rng)
            assert np.array_equal(o.parent, cp) and np.array_equal(o.blen, cb)   # bit-exact fp64
            new = o
            if rng.random() < 0.3:  # a branch-length change too
                v = int(rng.integers(0, 2 * n - 1))
                if v != new.root:
                    new.blen[v] *= 1.25
            for reroot in (False, True):
                rt, ops, offs, key, _ = moves.schedule_update(stored, new, reroot=reroot)
                got = R.rrl_schedule_update(n, stored.parent, stored.blen, new.parent, new.blen, reroot)
                assert got["root_edge"] == key, (seed, step, reroot)
                assert np.array_equal(got["parent"], rt.parent)
                assert np.array_equal(got["blen"], rt.blen)
                assert _ops_tuple(got["ops"]) == ops
                assert got["set_offsets"].tolist() == offs


def test_update_schedule_no_change_and_errors(R):
    t = make_tree("random", 30, seed=4)
    got = R.rrl_schedule_update(30, t.parent, t.blen, t.parent, t.blen, True)
    assert got["op_count"] == 0 and got["set_count"] == 0
    root = t.root
    a = int(np.flatnonzero(t.parent == root)[0])
    with pytest.raises(R.RRLError):
        R.rrl_tree_spr(30, t.parent, t.blen, a, 0 if a != 0 else 1)   # parent of prune node is the root
    with pytest.raises(R.RRLError):
        R.rrl_tree_nni(30, t.parent, t.blen, 3, 0)                     # a tip is no internal edge


# ------------------------------------------------------------------ NEXT-4 cost model (host only)
def test_schedule_cost_closed_forms(R):
    """rrl_schedule_cost against closed forms of a pectinate tree (PAPER.md:270,
    :288; DESIGN.md §9 "NEXT-4"): with no L2 credit the pass costs every set's
    launch plus every byte once -- n-1 outputs, n-2 internal children, n tip
    children; with infinite bandwidth it is the set count times the launch."""
    n, p, c, s = 64, 1000, 4, 4
    t = make_tree("pectinate", n, seed=3)
    for prec in (32, 64):
        v = c * s * prec // 8
        for mode, sets in (("level", n - 1), ("reroot", n // 2)):
            sch = R.rrl_reroot_and_schedule(n, t.parent, t.blen, mode)
            assert sch["set_count"] == sets
            bytes_ = p * ((n - 1) * (v + 4) + (n - 2) * (v + 4) + n * 1)
            got = R.rrl_schedule_cost(n, sch["ops"], sch["set_offsets"], p, s, c, prec, 2.0, 1000.0, 0.0)
            assert got == pytest.approx(sets * 2.0 + bytes_ / 1e12 * 1e6, rel=1e-12)
            got = R.rrl_schedule_cost(n, sch["ops"], sch["set_offsets"], p, s, c, prec, 3.0, 1e300, 0.0)
            assert got == pytest.approx(sets * 3.0, rel=1e-12)


def test_schedule_cost_l2_credit(R):
    """A chain (one op per set) whose outputs fit in L2 reads every internal
    child from L2: the credit removes exactly those reads; outputs bigger than
    L2 get none."""
    n, p, c, s = 32, 1000, 4, 4
    t = make_tree("pectinate", n, seed=1)
    sch = R.rrl_reroot_and_schedule(n, t.parent, t.blen, "level")
    v = c * s * 4 + 4
    full = R.rrl_schedule_cost(n, sch["ops"], sch["set_offsets"], p, s, c, 32, 0.0, 1000.0, 0.0)
    huge = R.rrl_schedule_cost(n, sch["ops"], sch["set_offsets"], p, s, c, 32, 0.0, 1000.0, 1e30)
    tiny = R.rrl_schedule_cost(n, sch["ops"], sch["set_offsets"], p, s, c, 32, 0.0, 1000.0, v * p / 2)
    assert huge == pytest.approx(full - (n - 2) * v * p / 1e6, rel=1e-9)
    assert tiny == pytest.approx(full, rel=1e-12)


def test_schedule_cost_predicts_measured_crossover(R):
    """The B200 parameters the engine's auto mode uses (engine.py) pick the
    rerooted 1,024-pectinate schedule where it measured faster and the original
    chain at 10^6 fp32 patterns, where it measured 0.88x
    (profiles/r02_reroot_sweep.json)."""
    n = 1024
    t = make_tree("pectinate", n, seed=1)
    lv = R.rrl_reroot_and_schedule(n, t.parent, t.blen, "level", True)
    rr = R.rrl_reroot_and_schedule(n, t.parent, t.blen, "reroot", True)

    def cost(sch, p):
        return R.rrl_schedule_cost(n, sch["ops"], sch["set_offsets"], p, 4, 4, 32, 2.0, 6225.0, 126e6)
    for p in (512, 4096, 10_000, 100_000):
        assert cost(rr, p) < cost(lv, p), p
    assert cost(lv, 1_000_000) < cost(rr, 1_000_000)


def test_schedule_cost_rejects_bad_input(R):
    t = make_tree("random", 10, seed=1)
    sch = R.rrl_reroot_and_schedule(10, t.parent, t.blen, "level")
    bad = sch["set_offsets"].copy()
    bad[-1] -= 1
    with pytest.raises(RuntimeError):
        R.rrl_schedule_cost(10, sch["ops"], bad, 100, 4, 4, 32)
    with pytest.raises(RuntimeError):
        R.rrl_schedule_cost(10, sch["ops"], sch["set_offsets"], 100, 4, 4, 16)
