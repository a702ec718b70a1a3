"""Input-generator pins (CPU): tree generators of PAPER.md:148, Gamma rates."""
import json
import math
import os
from collections import Counter

import numpy as np
import pytest

from workloads import config_workload, discrete_gamma_rates, make_tree, make_workload

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _children(parent):
    ch = [[] for _ in range(len(parent))]
    for v, u in enumerate(parent):
        if u >= 0:
            ch[u].append(v)
    return ch


def _is_binary_tree(t):
    n = t.n
    assert t.parent.shape == (2 * n - 1,)
    roots = np.flatnonzero(t.parent < 0)
    assert len(roots) == 1 and roots[0] >= n or n == 1
    ch = _children(t.parent.tolist())
    for v in range(n):
        assert ch[v] == []
    for v in range(n, 2 * n - 1):
        assert len(ch[v]) == 2
    # connected: every node reaches the root
    for v in range(2 * n - 1):
        x, steps = v, 0
        while t.parent[x] >= 0:
            x = t.parent[x]
            steps += 1
            assert steps < 2 * n
        assert x == roots[0]
    return True


@pytest.mark.parametrize("kind", ["pectinate", "random", "yule", "balanced"])
@pytest.mark.parametrize("n", [2, 3, 5, 8, 64, 257])
def test_generators_make_binary_trees(kind, n):
    t = make_tree(kind, n, seed=7)
    assert _is_binary_tree(t)
    nonroot = t.parent >= 0
    assert np.all((t.blen[nonroot] >= 0.01) & (t.blen[nonroot] <= 0.3))
    assert t.blen[t.root] == 0.0


def test_pectinate_is_caterpillar():
    # sibling is always the current root -> every internal node
    # has at least one tip child, and the depth of tip i is n - i (tip 0, 1 deepest).
    n = 40
    t = make_tree("pectinate", n, seed=1)
    ch = _children(t.parent.tolist())
    for v in range(n, 2 * n - 1):
        assert any(c < n for c in ch[v])


def _shape_counts(kind, n, seeds):
    cnt = Counter()
    for s in seeds:
        t = make_tree(kind, n, seed=s)
        ch = _children(t.parent.tolist())
        # canonical unlabeled-shape-with-labels signature: set of clades
        def clade(v):
            if v < n:
                return frozenset([v])
            return frozenset().union(*[clade(c) for c in ch[v]])
        clades = frozenset(clade(v) for v in range(n, 2 * n - 1))
        cnt[clades] += 1
    return cnt


def test_paper_random_is_uniform_on_rooted_topologies():
    # Attaching each new tip to a uniform random node gives the
    # uniform (PDA) distribution on rooted labelled topologies: n=4 has
    # (2n-3)!! = 15 rooted topologies, each with probability 1/15.
    N = 3000
    cnt = _shape_counts("random", 4, range(N))
    assert len(cnt) == 15
    exp = N / 15
    chi2 = sum((v - exp) ** 2 / exp for v in cnt.values())
    assert chi2 < 36.1  # chi2(14) 0.999 quantile


def test_yule_balanced_shape_frequency():
    # Yule with n=4: P(balanced shape) = 1/3; PDA gives 1/5 -- distinguishes them.
    N = 3000
    for kind, p_bal in (("yule", 1 / 3), ("random", 1 / 5)):
        bal = 0
        for s in range(N):
            t = make_tree(kind, 4, seed=s)
            ch = _children(t.parent.tolist())
            if all(c >= 4 for c in ch[t.root]):
                bal += 1
        sd = math.sqrt(N * p_bal * (1 - p_bal))
        assert abs(bal - N * p_bal) < 4 * sd, (kind, bal)


def test_gamma_rates_yang1994_table():
    g = json.load(open(os.path.join(GOLDEN, "yang1994_gamma.json")))
    r = discrete_gamma_rates(g["alpha"], g["categories"])
    np.testing.assert_allclose(r, g["rates"], atol=g["abs_tol"])


@pytest.mark.parametrize("c", [2, 4, 8])
def test_gamma_rates_exponential_closed_form(c):
    # alpha = 1 is the exponential distribution: category k between the
    # quantiles a = -ln(1-(k-1)/c), b = -ln(1-k/c) has mean
    # c * [(a+1) e^-a - (b+1) e^-b].
    r = discrete_gamma_rates(1.0, c)
    exp = []
    for k in range(1, c + 1):
        a = -math.log(1 - (k - 1) / c)
        b = math.inf if k == c else -math.log(1 - k / c)
        tb = 0.0 if k == c else (b + 1) * math.exp(-b)
        exp.append(c * ((a + 1) * math.exp(-a) - tb))
    np.testing.assert_allclose(r, exp, rtol=1e-10)
    assert abs(r.mean() - 1) < 1e-12


def test_workload_is_seeded_and_deterministic():
    a = config_workload("c1", seed=3, p=100)
    b = config_workload("c1", seed=3, p=100)
    c = config_workload("c1", seed=4, p=100)
    assert np.array_equal(a.tips, b.tips) and np.array_equal(a.tree.blen, b.tree.blen)
    assert not np.array_equal(a.tips, c.tips)
    assert a.tips.dtype == np.uint8 and a.tips.max() < 4
    assert abs(a.rates.mean() - 1) < 1e-12


def test_missing_fraction():
    w = make_workload(tree_kind="yule", n=10, p=2000, model="gtr", c=4, seed=1,
                      missing_frac=0.25)
    frac = (w.tips == 4).mean()
    assert 0.2 < frac < 0.3
