"""Pins for oracle/pruning.py (CPU): closed forms, brute force, invariants.

Each test pins the oracle to something other than itself: the Jukes-Cantor
closed forms (independent algebra), brute-force summation over ancestral
states (oracle/brute.py, the textbook definition), exact limits (t -> inf,
t = 0, all-missing), and the reroot invariance of PAPER.md:94 §V-A.
"""
import math

import numpy as np
import pytest

from oracle import brute, model as om, pruning, reroot
from workloads import Tree, make_tree, make_workload, random_model, with_blen


def _run(w, tree=None, **kw):
    Q = om.rate_matrix(w.model)
    return pruning.prune(tree or w.tree, Q, w.model.pi, w.rates, w.cat_weights, w.tips,
                         w.pattern_weights, **kw)


# ---------------------------------------------------------------- JC closed forms

def _jc_p(t):
    e = math.exp(-4.0 * t / 3.0)
    return 0.25 + 0.75 * e, 0.25 - 0.25 * e


@pytest.mark.parametrize("c", [1, 4])
def test_jc_two_taxon_closed_form(c):
    w = make_workload(tree_kind="pectinate", n=2, p=16, model="jc69", c=c, seed=11)
    w.tips[:] = np.array([[a for a in range(4) for _ in range(4)],
                          [b for _ in range(4) for b in range(4)]], dtype=np.uint8)
    res = _run(w)
    T = w.tree.blen[0] + w.tree.blen[1]
    for i in range(16):
        a, b = int(w.tips[0, i]), int(w.tips[1, i])
        L = 0.0
        for k in range(c):
            same, diff = _jc_p(w.rates[k] * T)
            L += w.cat_weights[k] * 0.25 * (same if a == b else diff)
        assert abs(res.site_lnl[i] - math.log(L)) < 1e-13


def _jc3_class_form(x, t):
    """Survey §8(c3) / textbook JC 3-taxon forms by pattern class."""
    (eq1, ne1), (eq2, ne2), (eq3, ne3) = (_jc_p(ti) for ti in t)
    a, b, c = x
    if a == b == c:
        return 0.25 * (eq1 * eq2 * eq3 + 3 * ne1 * ne2 * ne3)
    if a != b and b != c and a != c:
        return 0.25 * (eq1 * ne2 * ne3 + ne1 * eq2 * ne3 + ne1 * ne2 * eq3 + ne1 * ne2 * ne3)
    # exactly two equal: put the odd tip last
    if a == b:
        p = ((eq1, ne1), (eq2, ne2), (eq3, ne3))
    elif a == c:
        p = ((eq1, ne1), (eq3, ne3), (eq2, ne2))
    else:
        p = ((eq2, ne2), (eq3, ne3), (eq1, ne1))
    (e1, n1), (e2, n2), (e3, n3) = p
    return 0.25 * (e1 * e2 * n3 + n1 * n2 * e3 + 2 * n1 * n2 * n3)


@pytest.mark.parametrize("kind", ["pectinate", "balanced"])
@pytest.mark.parametrize("c", [1, 4])
def test_jc_three_taxon_closed_form(kind, c):
    w = make_workload(tree_kind=kind, n=3, p=64, model="jc69", c=c, seed=5)
    pats = [(a, b, d) for a in range(4) for b in range(4) for d in range(4)]
    w.tips[:] = np.array(pats, dtype=np.uint8).T
    res = _run(w)
    t = w.tree
    # central node = the internal non-root node; its three branches
    ch = pruning.children_of(t.parent)
    root = t.root
    u = [v for v in ch[root] if v >= 3][0]
    other = [v for v in ch[root] if v != u][0]
    tt = [0.0, 0.0, 0.0]
    for v in ch[u]:
        tt[v] = t.blen[v]
    tt[other] = t.blen[u] + t.blen[other]
    for i, x in enumerate(pats):
        L = sum(w.cat_weights[k] * _jc3_class_form(x, [w.rates[k] * q for q in tt])
                for k in range(c))
        assert abs(res.site_lnl[i] - math.log(L)) < 1e-13, x


# ---------------------------------------------------------------- brute force

@pytest.mark.parametrize("kind", ["pectinate", "random", "balanced", "yule"])
@pytest.mark.parametrize("n", [4, 5, 6])
def test_brute_force_gtr_gamma(kind, n):
    w = make_workload(tree_kind=kind, n=n, p=6, model="gtr", c=4, seed=n * 13,
                      missing_frac=0.15)
    Q = om.rate_matrix(w.model)
    res = _run(w)
    bf = brute.site_likelihoods(w.tree, Q, w.model.pi, w.rates, w.cat_weights, w.tips)
    np.testing.assert_allclose(res.site_lnl, np.log(bf), rtol=1e-13, atol=1e-13)


def test_brute_force_hky_c1():
    w = make_workload(tree_kind="random", n=6, p=8, model="hky", c=1, seed=2)
    Q = om.rate_matrix(w.model)
    bf = brute.site_likelihoods(w.tree, Q, w.model.pi, w.rates, w.cat_weights, w.tips)
    np.testing.assert_allclose(_run(w).site_lnl, np.log(bf), rtol=1e-13)


def test_brute_force_codon_three_taxa():
    w = make_workload(tree_kind="random", n=3, p=3, model="gy94", c=2, seed=9)
    Q = om.rate_matrix(w.model)
    bf = brute.site_likelihoods(w.tree, Q, w.model.pi, w.rates, w.cat_weights, w.tips)
    np.testing.assert_allclose(_run(w).site_lnl, np.log(bf), rtol=1e-12)


# ---------------------------------------------------------------- invariants

@pytest.mark.parametrize("model,n,p", [("gtr", 20, 40), ("hky", 13, 30), ("gy94", 6, 4)])
def test_reroot_invariance_all_edges(model, n, p):
    """PAPER.md:94 §V-A: for time-reversible models the likelihood does not
    depend on the root.  Every one of the 2n-3 rootings, 1e-12 relative."""
    w = make_workload(tree_kind="random", n=n, p=p, model=model, c=4, seed=n)
    base = _run(w).lnl
    edges = reroot.unrooted_edges(w.tree)
    assert len(edges) == 2 * n - 3
    for key, *_ in edges:
        rt = reroot.reroot_at(w.tree, key)
        l2 = _run(w, tree=Tree(rt.n, rt.parent, rt.blen)).lnl
        assert abs(l2 - base) <= 1e-12 * abs(base), (key, l2, base)


def test_long_branch_limit_exercises_scaling():
    """t -> inf: P -> 1 pi^T, so lnL_i = sum_tips ln pi_{x_tip} exactly (missing
    tips contribute 0).  n = 600 drives the unscaled product below fp64's
    range, so the unscaled oracle returns -inf and the scaled one is exact."""
    w = make_workload(tree_kind="random", n=600, p=5, model="gtr", c=1, seed=3,
                      missing_frac=0.1)
    tree = with_blen(w.tree, 50.0 / 1.0)
    res = _run(w, tree=tree)
    pi = w.model.pi
    for i in range(w.p):
        col = w.tips[:, i]
        exp = sum(math.log(pi[x]) for x in col if x < 4)
        assert abs(res.site_lnl[i] - exp) < 1e-9 * abs(exp)
    un = _run(w, tree=tree, scale=False)
    assert np.all(np.isneginf(un.site_lnl))


def test_all_missing_and_zero_length():
    w = make_workload(tree_kind="yule", n=25, p=6, model="gtr", c=4, seed=4)
    w.tips[:, 0] = 4                          # all missing -> lnL = 0
    for x in range(4):
        w.tips[:, 1 + x] = x                  # constant patterns
    res0 = _run(w)
    assert abs(res0.site_lnl[0]) < 1e-13
    tree = with_blen(w.tree, 0.0)             # t = 0: lnL = ln pi_x for constants
    res = _run(w, tree=tree)
    for x in range(4):
        assert abs(res.site_lnl[1 + x] - math.log(w.model.pi[x])) < 1e-13


def test_scaled_equals_unscaled_small_tree():
    w = make_workload(tree_kind="random", n=30, p=50, model="gtr", c=4, seed=8)
    a = _run(w, scale=True).site_lnl
    b = _run(w, scale=False).site_lnl
    np.testing.assert_allclose(a, b, rtol=1e-13)


def test_weights_and_permutation():
    w = make_workload(tree_kind="random", n=12, p=20, model="gtr", c=4, seed=6)
    Q = om.rate_matrix(w.model)
    args = (Q, w.model.pi, w.rates, w.cat_weights)
    base = pruning.prune(w.tree, *args, w.tips, w.pattern_weights)
    perm = np.random.default_rng(0).permutation(20)
    pr = pruning.prune(w.tree, *args, w.tips[:, perm], w.pattern_weights)
    np.testing.assert_allclose(pr.site_lnl, base.site_lnl[perm], rtol=0, atol=0)
    wt = w.pattern_weights.copy()
    wt[3] = 2.0
    dup = np.concatenate([w.tips, w.tips[:, 3:4]], axis=1)
    a = pruning.prune(w.tree, *args, w.tips, wt).lnl
    b = pruning.prune(w.tree, *args, dup, np.ones(21)).lnl
    assert abs(a - b) < 1e-12 * abs(a)


def test_edge_lnl_pulley_equals_root():
    """Edge log-likelihood across the root's two child subtrees with branch
    t_a + t_b (pulley principle, reversibility) equals the root likelihood."""
    w = make_workload(tree_kind="balanced", n=16, p=30, model="gtr", c=4, seed=12)
    Q = om.rate_matrix(w.model)
    res = _run(w, keep_partials=True)
    ch = pruning.children_of(w.tree.parent)
    a, b = ch[w.tree.root]
    T = w.tree.blen[a] + w.tree.blen[b]
    Ps = [pruning.transition_matrix(Q, r * T) for r in w.rates]
    site = pruning.edge_site_lnl(res.partials[a], res.cum_exponent[a], res.partials[b],
                                 res.cum_exponent[b], Ps, w.model.pi, w.cat_weights)
    np.testing.assert_allclose(site, res.site_lnl, rtol=1e-12)


def test_per_node_exponents_sum():
    w = make_workload(tree_kind="pectinate", n=40, p=10, model="gtr", c=4, seed=1)
    res = _run(w, keep_partials=True)
    tot = sum(res.exponent.values())
    np.testing.assert_array_equal(tot, res.cum_exponent[w.tree.root])
    for v, L in res.partials.items():
        m = L.max(axis=(0, 2))
        assert np.all((m >= 0.5) & (m < 1.0))
