"""Pins for oracle/moves.py and oracle.reroot.schedule_partial (CPU).

NEXT-2 (PAPER.md:258 §VII-D, :268, :282 §VIII-A): partial recomputation after
a topology change.  What fixes the oracle here, independently of itself:
  * textbook facts about the moves: an unrooted binary tree with n tips has
    exactly 2(n-3) NNI neighbours, each differing from it in exactly one split
    (Robinson 1971); the two NNIs of an edge are the two SPRs moving one of
    v's children onto the sibling's branch; an SPR back onto the old sibling
    restores the unrooted topology;
  * the full pruning oracle: running only the scheduled operations on top of
    the stored partials of the old tree must reproduce a full prune of the new
    tree (bit for bit on the same rooting, 1e-12 across rootings)
    -- a node missing from a schedule, or a child read before it is
    recomputed, changes the result.
"""
import numpy as np
import pytest

from oracle import model as om, moves, pruning, reroot as rr
from workloads import make_workload


def _w(kind, n, seed, p=40, c=2):
    return make_workload(tree_kind=kind, n=n, p=p, model="gtr", c=c, seed=seed, missing_frac=0.05)


def _full(w, tree, keep=False):
    Q = om.rate_matrix(w.model)
    return pruning.prune(tree, Q, w.model.pi, w.rates, w.cat_weights, w.tips, w.pattern_weights,
                         keep_partials=keep)


def _apply(w, tree, ops, stored):
    Q = om.rate_matrix(w.model)
    return moves.apply_ops(tree, ops, stored, Q, w.model.pi, w.rates, w.cat_weights, w.tips,
                           w.pattern_weights)


def _internal_edges(tree):
    """Keys of the unrooted internal edges (both ends internal)."""
    return [k for k, u, v, _ in rr.unrooted_edges(tree) if u >= tree.n and v >= tree.n]


# ------------------------------------------------------------------ moves (A26, A27)
@pytest.mark.parametrize("kind,n,seed", [("random", 6, 1), ("random", 13, 2), ("random", 25, 3),
                                         ("pectinate", 9, 1), ("balanced", 16, 1), ("yule", 20, 4)])
def test_nni_neighbourhood_is_2n_minus_6(kind, n, seed):
    t = _w(kind, n, seed).tree
    base = moves.unrooted_splits(t)
    assert len(base) == n - 3
    keys = _internal_edges(t)
    assert len(keys) == n - 3
    nb = set()
    for k in keys:
        for which in (0, 1):
            s = moves.unrooted_splits(moves.nni(t, k, which))
            assert len(s) == n - 3
            assert len(base - s) == 1 and len(s - base) == 1  # exactly one split replaced
            nb.add(s)
    assert len(nb) == 2 * (n - 3)


@pytest.mark.parametrize("seed", range(1, 6))
def test_nni_pair_equals_spr_pair(seed):
    t = _w("random", 30, seed).tree
    ch = pruning.children_of(t.parent)
    checked = 0
    for v in range(t.n, 2 * t.n - 1):
        u = int(t.parent[v])
        if u < 0 or u == t.root:
            continue
        w_ = [c for c in ch[u] if c != v][0]
        a = {moves.unrooted_splits(moves.nni(t, v, k)) for k in (0, 1)}
        b = {moves.unrooted_splits(moves.spr(t, ch[v][k], w_)) for k in (0, 1)}
        assert a == b
        checked += 1
    assert checked > 10


@pytest.mark.parametrize("seed", range(1, 6))
def test_spr_back_to_sibling_restores_topology(seed):
    t = _w("random", 30, seed).tree
    rng = np.random.default_rng(seed)
    base = moves.unrooted_splits(t)
    done = 0
    while done < 20:
        x = int(rng.integers(0, 2 * t.n - 1))
        if x == t.root or t.parent[x] == t.root:
            continue
        p = int(t.parent[x])
        sib = [c for c in pruning.children_of(t.parent)[p] if c != x][0]
        bad = moves._subtree_nodes(t, x) | {p, t.root}
        r = int(rng.integers(0, 2 * t.n - 1))
        if r in bad:
            continue
        t2 = moves.spr(t, x, r)
        assert sorted(np.flatnonzero(np.asarray(t2.parent) < 0)) == [t.root]
        assert moves.unrooted_splits(moves.spr(t, x, sib)) == base
        assert moves.unrooted_splits(moves.spr(t2, x, sib)) == base
        done += 1


# ------------------------------------------------------------------ schedule_partial
@pytest.mark.parametrize("kind,n,seed", [("random", 40, 1), ("pectinate", 24, 2), ("yule", 50, 3)])
def test_schedule_partial_reproduces_full_prune(kind, n, seed):
    """Verdict pin for oracle.reroot.schedule_partial: change branch lengths,
    run only the partial schedule on top of the stored partials: bit-identical
    to a full prune of the changed tree."""
    w = _w(kind, n, seed)
    t = w.tree
    stored = _full(w, t, keep=True)
    rng = np.random.default_rng(seed)
    for trial in range(6):
        k = 1 + trial % 3
        changed = rng.choice([v for v in range(2 * n - 1) if v != t.root], size=k, replace=False)
        blen = np.asarray(t.blen).copy()
        blen[changed] *= 1.7
        t2 = rr.RTree(n, t.parent.copy(), blen)
        lows = sorted({int(t.parent[v]) for v in changed})
        ops, offs = rr.schedule_partial(t2, lows)
        # exactly the changed branches' parents and their ancestors
        want = set()
        for v in lows:
            while v >= 0:
                want.add(v)
                v = int(t.parent[v])
        assert {o[0] for o in ops} == want
        # every recomputed child finished in an earlier set
        setof = {o[0]: s for s in range(len(offs) - 1) for o in ops[offs[s]:offs[s + 1]]}
        for o in ops:
            for ch in (o[3], o[5]):
                if ch in setof:
                    assert setof[ch] < setof[o[0]]
        got = _apply(w, t2, ops, stored)
        ref = _full(w, t2)
        np.testing.assert_array_equal(got.site_lnl, ref.site_lnl)


# ------------------------------------------------------------------ schedule_update (A28)
def _random_move(t, rng):
    while True:
        if rng.random() < 0.5:
            x = int(rng.integers(0, 2 * t.n - 1))
            if x == t.root or t.parent[x] == t.root:
                continue
            r = int(rng.integers(0, 2 * t.n - 1))
            if r in moves._subtree_nodes(t, x) | {int(t.parent[x]), t.root}:
                continue
            return moves.spr(t, x, r)
        keys = _internal_edges(t)
        return moves.nni(t, keys[int(rng.integers(0, len(keys)))], int(rng.integers(0, 2)))


@pytest.mark.parametrize("kind,n,seed", [("random", 40, 1), ("pectinate", 30, 2), ("yule", 36, 3),
                                         ("balanced", 32, 4)])
@pytest.mark.parametrize("nmoves", [1, 3])
@pytest.mark.parametrize("reroot", [False, True])
def test_schedule_update_reproduces_full_prune(kind, n, seed, nmoves, reroot):
    w = _w(kind, n, seed)
    stored_tree = rr.RTree(n, w.tree.parent.copy(), w.tree.blen.copy())
    stored = _full(w, stored_tree, keep=True)
    rng = np.random.default_rng(100 + seed)
    new = stored_tree
    for _ in range(nmoves):
        new = _random_move(new, rng)
    rt, ops, offs, key, table = moves.schedule_update(stored_tree, new, reroot=reroot)
    got = _apply(w, rt, ops, stored)
    np.testing.assert_array_equal(got.site_lnl, _full(w, rt).site_lnl)   # same rooting: bit for bit
    ref = _full(w, new)
    assert abs(got.lnl - ref.lnl) <= 1e-12 * abs(ref.lnl)                   # reroot invariance
    # reused nodes really are unchanged subtrees; recomputed ones are ancestor-closed
    dest = {o[0] for o in ops}
    for v in dest:
        u = int(rt.parent[v])
        assert u < 0 or u in dest
    if reroot:
        cur = [r for r in table if r[2] == 0][0]
        assert len(offs) - 1 <= cur[0]


def test_partial_reroot_beats_current_rooting_on_pectinate():
    """A move deep in a pectinate tree recomputes a long chain on the current
    rooting; rerooting the update halves its sets."""
    w = _w("pectinate", 64, 5)
    t = rr.RTree(64, w.tree.parent.copy(), w.tree.blen.copy())
    tips = [v for v in range(64)]
    depth = {v: 0 for v in range(2 * 64 - 1)}
    for v in pruning.postorder(t.parent)[::-1]:
        for c in pruning.children_of(t.parent)[v]:
            depth[c] = depth[v] + 1
    deep = max(tips, key=lambda v: depth[v])
    blen = np.asarray(t.blen).copy()
    blen[deep] *= 2.0
    new = rr.RTree(64, t.parent.copy(), blen)
    _, _, offs0, _, _ = moves.schedule_update(t, new, reroot=False)
    rt, ops, offs1, key, _ = moves.schedule_update(t, new, reroot=True)
    assert len(offs0) - 1 == 63
    assert len(offs1) - 1 <= 33
    stored = _full(w, t, keep=True)
    got = _apply(w, rt, ops, stored)
    assert abs(got.lnl - _full(w, new).lnl) <= 1e-12 * abs(got.lnl)
