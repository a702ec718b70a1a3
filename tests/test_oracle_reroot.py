"""Pins for oracle/reroot.py (CPU): the paper's printed set counts and bounds.

tests/golden/paper_set_counts.json holds the values PAPER.md prints
(Fig. 2, Fig. 3, §V-A, §V-B, Table III), each with its citation.
"""
import json
import math
import os

import numpy as np
import pytest

from oracle import reroot as rr
from oracle.pruning import children_of
from workloads import make_tree

G = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_set_counts.json")))


def test_fig2_balanced_8():
    g = G["fig2_balanced_8"]
    t = make_tree("balanced", g["n"], seed=1)
    ops, offs = rr.schedule_sequential(t)
    assert len(offs) - 1 == g["sequential_sets"] == len(ops)
    ops, offs = rr.schedule_level(t)
    assert len(offs) - 1 == g["level_sets"]
    assert rr.count_sets_greedy(t) == g["level_sets"]


def test_fig3_pectinate_8():
    g = G["fig3_pectinate_8"]
    t = make_tree("pectinate", g["n"], seed=1)
    assert rr.count_sets_height(t) == g["original_sets"] == rr.count_sets_greedy(t)
    key, sets = rr.best_rooting(t)
    assert sets == g["rerooted_sets"]
    rt = rr.reroot_at(t, key)
    _, offs = rr.schedule_level(rt)
    assert len(offs) - 1 == g["rerooted_sets"]
    # widths 2,2,2,1 (survey §8(d) C0)
    assert np.diff(offs).tolist() == [2, 2, 2, 1]


@pytest.mark.parametrize("n", list(range(2, 41)) + [64, 127, 128])
def test_pectinate_formula(n):
    """PAPER.md:96 §V-A: n-1 sets, ceil(n/2) after optimal rerooting."""
    t = make_tree("pectinate", n, seed=n)
    assert rr.count_sets_height(t) == n - 1
    _, sets = rr.best_rooting(t)
    assert sets == math.ceil(n / 2)


def test_table3_theoretical_64():
    g = G["table3_theoretical_64"]
    n = g["n"]
    bal = make_tree("balanced", n, seed=1)
    pec = make_tree("pectinate", n, seed=1)
    assert round((n - 1) / rr.count_sets_height(bal), 2) == g["balanced"]
    assert round((n - 1) / rr.count_sets_height(pec), 2) == g["pectinate"]
    _, s = rr.best_rooting(pec)
    assert round((n - 1) / s, 2) == g["pectinate_rerooted"]


@pytest.mark.parametrize("kind", ["random", "yule"])
def test_bounds_and_closed_form_on_random_trees(kind):
    """PAPER.md:102 §V-B interval [ceil(log2 n), ceil(n/2)]; the survey's
    identity min sets = ceil((D+1)/2) with D the unrooted leaf-leaf diameter;
    greedy == height (asserted inside best_rooting); and
    rerooting at most halves the count (D >= original height)."""
    for seed in range(1, 16):
        for n in (5, 17, 40, 64):
            t = make_tree(kind, n, seed=seed)
            h0 = rr.count_sets_height(t)
            assert rr.count_sets_greedy(t) == h0
            key, s = rr.best_rooting(t)
            assert math.ceil(math.log2(n)) <= s <= math.ceil(n / 2)
            assert s <= h0 < 2 * s
            D = rr.unrooted_diameter(t)
            assert s == math.ceil((D + 1) / 2)


def test_reroot_at_preserves_tree():
    t = make_tree("random", 30, seed=4)
    total = t.blen.sum()
    for key, *_ in rr.unrooted_edges(t):
        rt = rr.reroot_at(t, key)
        assert rt.root == t.root                      # reading A11
        ch = children_of(rt.parent)
        assert all(len(ch[v]) == 0 for v in range(30))
        assert all(len(ch[v]) == 2 for v in range(30, 59))
        assert abs(rt.blen.sum() - total) < 1e-12
        # the unrooted tree (edge set + lengths) is unchanged
        e0 = {(k, round(l, 12)) for k, _, _, l in rr.unrooted_edges(t)}
        e1 = sorted(tuple(sorted((u, v))) + (round(l, 12),) for _, u, v, l in rr.unrooted_edges(rt))
        e0 = sorted(tuple(sorted((u, v))) + (round(l, 12),) for _, u, v, l in rr.unrooted_edges(t))
        assert e0 == e1


def test_tie_break_keeps_current_root_when_optimal():
    # balanced trees are already optimal: rerooting is a no-op
    t = make_tree("balanced", 32, seed=1)
    key, s = rr.best_rooting(t)
    assert key == min(children_of(t.parent)[t.root])
    rt = rr.reroot_at(t, key)
    assert np.array_equal(rt.parent, t.parent) and np.array_equal(rt.blen, t.blen)


def test_tie_break_balance_then_key():
    # pectinate n = 7 has 3 optimal edges (survey App. A); the choice is the
    # most tip-balanced, then smallest key.
    t = make_tree("pectinate", 7, seed=1)
    key, s, table = rr.best_rooting(t, with_table=True)
    opt = [r for r in table if r[0] == s]
    assert len(opt) == 3
    assert key == min(opt)[3]


def _valid_schedule(tree, ops, offs):
    n = tree.n
    done = set(range(n))
    seen = []
    for k in range(len(offs) - 1):
        batch = ops[offs[k]:offs[k + 1]]
        assert batch, "empty set"
        dests = [o[0] for o in batch]
        assert dests == sorted(dests)
        for d, sw, sr, c1, m1, c2, m2 in batch:
            assert c1 in done and c2 in done and c1 < c2
            assert m1 == c1 and m2 == c2 and sw == d - n and sr == -1
            assert {c1, c2} == set(children_of(tree.parent)[d])
        done.update(dests)
        seen += dests
    assert sorted(seen) == list(range(n, 2 * n - 1))


@pytest.mark.parametrize("mode", ["sequential", "level", "reroot"])
@pytest.mark.parametrize("kind", ["pectinate", "random", "yule", "balanced"])
def test_schedules_are_valid(mode, kind):
    t = make_tree(kind, 50, seed=3)
    rt, ops, offs, key = rr.reroot_and_schedule(t, mode)
    _valid_schedule(rt, ops, offs)
    if mode == "sequential":
        assert len(offs) - 1 == 49
    else:
        assert len(offs) - 1 == rr.count_sets_height(rt)


def test_fig4_qualitative_rerooting_never_hurts():
    """PAPER.md:205 §VII-A: rerooting reduces the set count 'by as much as
    half'; some trees are already optimal.  (Paper-random generator, smaller
    n than the paper's 256 to keep the exhaustive oracle fast.)"""
    ratios = []
    for seed in range(1, 31):
        t = make_tree("random", 64, seed=seed)
        h0 = rr.count_sets_height(t)
        _, s = rr.best_rooting(t)
        assert s <= h0
        ratios.append(h0 / s)
    assert max(ratios) <= 2.0 and max(ratios) > 1.5
    assert min(ratios) >= 1.0
