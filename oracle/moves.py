"""ORACLE (test infrastructure only) -- topology moves and partial-update schedules.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  Shares no code with the product's
C++ (csrc/schedule.cpp: O(n) validity pass and an all-edges DP).

SURVEY.md §8(f) NEXT-2.  PAPER.md:258 §VII-D: "phylogenetic inference
programs are optimized such that only a subtree representing the modified
portion of the overall tree is recomputed for each topology change.  These
subtrees are often less symmetrical than the full tree"; PAPER.md:268 and
:282-286 §VIII-A (partial recomputation on topology changes, rerooting the
starting tree and "further balanced rerootings, later in the search").
The paper defines neither the moves nor which stored partials survive them;
the readings are:

A26 SPR(x, r) (subtree prune and regraft): x is any non-root node whose
    parent p is not the root; r is any node outside x's subtree other than p
    and the root.  Prune: p's other child s takes p's place under g =
    parent(p), with branch length t_s + t_p.  Regraft: p is inserted on the
    branch above r (parent q = parent(r), after the prune): p's parent is q,
    r and x are p's children, t_p = t_r' = t_r / 2 (t_r as it stands after
    the prune); x keeps t_x.  Node ids and the root are kept.  r = s gives
    the original unrooted topology back.
A27 NNI(v, which) (nearest-neighbour interchange) on the unrooted internal
    edge keyed like A9 (the edge above v; the root's merged edge is keyed by
    min(a, b)).  Non-root-child v with parent u and sibling w: v's child
    number `which` (0 = smaller id) and w exchange places.  Merged root edge
    (v = min(a, b), both internal): v's child `which` and the other root
    child's smaller child exchange places.  Moved subtrees keep their branch
    lengths.
A28 A stored partial of node v is the likelihood of v's rooted subtree as it
    was when it was computed.  It is reused iff v's rooted subtree -- its two
    children, their branch lengths, and recursively their subtrees -- is the
    same in the tree being computed as when stored, and, when the update is
    rerooted, also the same as in the new tree as given (the library does not
    look for stored partials that a rerooting happens to recreate).  Every
    other internal node is recomputed; those operations are level-batched
    among themselves: level(v) = 1 + max level of v's recomputed children.
    The rerooted update picks, over all 2n-3 edges, the fewest sets, then the
    fewest operations, then the current root edge, then the smallest key.
"""
from __future__ import annotations

import math

import numpy as np

from .pruning import LN2, PruningResult, children_of, postorder, tip_partials, transition_matrix
from .reroot import NONE, RTree, reroot_at, unrooted_edges


# ----------------------------------------------------------------------------
# Moves (A26, A27)
# ----------------------------------------------------------------------------

def _subtree_nodes(tree, x: int) -> set[int]:
    ch = children_of(tree.parent)
    out, stack = set(), [x]
    while stack:
        v = stack.pop()
        out.add(v)
        stack.extend(ch[v])
    return out


def spr(tree, x: int, r: int) -> RTree:
    """Reading A26."""
    parent = np.asarray(tree.parent).copy()
    blen = np.asarray(tree.blen, dtype=np.float64).copy()
    root = int(np.flatnonzero(parent < 0)[0])
    if x == root or not 0 <= x < parent.shape[0]:
        raise ValueError("x must be a non-root node")
    p = int(parent[x])
    if p == root:
        raise ValueError("x's parent must not be the root")
    if r in _subtree_nodes(tree, x) or r == p or r == root:
        raise ValueError("bad regraft node")
    g = int(parent[p])
    s = [c for c in children_of(parent)[p] if c != x][0]
    # prune: s replaces p under g
    parent[s] = g
    blen[s] = blen[s] + blen[p]
    # regraft p on the branch above r
    q = int(parent[r])
    half = blen[r] / 2.0
    parent[p] = q
    blen[p] = half
    parent[r] = p
    blen[r] = half
    return RTree(tree.n, parent, blen)


def nni(tree, v: int, which: int) -> RTree:
    """Reading A27."""
    parent = np.asarray(tree.parent).copy()
    blen = np.asarray(tree.blen, dtype=np.float64).copy()
    root = int(np.flatnonzero(parent < 0)[0])
    ch = children_of(parent)
    if v < tree.n or v == root or which not in (0, 1):
        raise ValueError("v must be an internal non-root node, which in {0, 1}")
    u = int(parent[v])
    mine = ch[v][which]
    if u == root:
        a, b = ch[root]
        if v != min(a, b):
            raise ValueError("the root's merged edge is keyed by its smaller child")
        other = max(a, b)
        if other < tree.n:
            raise ValueError("merged root edge is not internal")
        theirs = ch[other][0]
        parent[mine], parent[theirs] = other, v
    else:
        w = [c for c in ch[u] if c != v][0]
        parent[mine], parent[w] = u, v
    return RTree(tree.n, parent, blen)


def unrooted_splits(tree) -> frozenset:
    """Non-trivial bipartitions of the tips, each as the side without tip 0."""
    n = tree.n
    below: dict[int, frozenset] = {t: frozenset([t]) for t in range(n)}
    ch = children_of(tree.parent)
    for v in postorder(tree.parent):
        below[v] = below[ch[v][0]] | below[ch[v][1]]
    allt = frozenset(range(n))
    out = set()
    for v, s in below.items():
        if 1 < len(s) < n - 1:
            out.add(s if 0 not in s else allt - s)
    return frozenset(out)


# ----------------------------------------------------------------------------
# Which stored partials survive (A28)
# ----------------------------------------------------------------------------

class SubtreeIds:
    """Hash-consing of rooted subtrees: equal ids <=> equal (node, children,
    children's branch lengths, recursively).  Exact (dict on tuples), and
    shared across trees so ids are comparable."""

    def __init__(self):
        self.table: dict[tuple, int] = {}

    def ids(self, tree) -> dict[int, int]:
        ch = children_of(tree.parent)
        out = {t: self.table.setdefault((t,), len(self.table)) for t in range(tree.n)}
        for v in postorder(tree.parent):
            a, b = ch[v]
            key = (v, a, float(tree.blen[a]), out[a], b, float(tree.blen[b]), out[b])
            out[v] = self.table.setdefault(key, len(self.table))
        return out


def level_batch(tree, nodes) -> tuple[list[tuple[int, ...]], list[int]]:
    """Level sets over exactly `nodes` (children outside it are stored)."""
    nodes = set(int(v) for v in nodes)
    ch = children_of(tree.parent)
    level: dict[int, int] = {}
    for v in postorder(tree.parent):
        if v in nodes:
            level[v] = 1 + max([level[c] for c in ch[v] if c in nodes] or [0])
    H = max(level.values()) if level else 0
    ops, offs = [], [0]
    for k in range(1, H + 1):
        for v in sorted(x for x in nodes if level[x] == k):
            a, b = ch[v]
            ops.append((v, v - tree.n, NONE, a, a, b, b))
        offs.append(len(ops))
    return ops, offs


def recompute_set(stored, tree, given=None, ids: SubtreeIds | None = None) -> set[int]:
    """Internal nodes of `tree` whose stored partial cannot be reused (A28).
    `given`: the new tree as given when `tree` is a rerooting of it."""
    ids = ids or SubtreeIds()
    s_ids, t_ids = ids.ids(stored), ids.ids(tree)
    g_ids = ids.ids(given) if given is not None else t_ids
    return {v for v in range(tree.n, 2 * tree.n - 1) if t_ids[v] != s_ids[v] or t_ids[v] != g_ids[v]}


def schedule_update(stored, new, reroot: bool = False):
    """Operations that bring partials stored for `stored` up to date for
    `new` (A28).  Returns (tree, ops, offsets, key, table): `tree` is `new` or
    the chosen rerooting of it; `table` = [(sets, ops, not_current, key)]."""
    ch = children_of(new.parent)
    cur = min(ch[int(np.flatnonzero(np.asarray(new.parent) < 0)[0])])
    ids = SubtreeIds()
    keys = [e[0] for e in unrooted_edges(new)] if reroot else [cur]
    table, trees = [], {}
    for key in keys:
        rt = reroot_at(new, key)
        dirty = recompute_set(stored, rt, new, ids)
        ops, offs = level_batch(rt, dirty)
        table.append((len(offs) - 1, len(ops), 0 if key == cur else 1, key))
        trees[key] = (rt, ops, offs)
    best = min(table)
    rt, ops, offs = trees[best[3]]
    return rt, ops, offs, best[3], table


# ----------------------------------------------------------------------------
# Executing an operation list on top of stored partials (Eq. (1))
# ----------------------------------------------------------------------------

def apply_ops(tree, ops, stored: PruningResult, Q, pi, rates, cat_w, tips, pattern_weights) -> PruningResult:
    """Run `ops` (in order) on `tree`, reading every child that no op writes
    from `stored` (a keep_partials prune): Eq. (1), power-of-two rescaling
    and root integration exactly as oracle.pruning.prune does them."""
    n, s, c, p = tree.n, Q.shape[0], rates.shape[0], tips.shape[1]
    L = {v: stored.partials[v] for v in stored.partials}
    E = {v: stored.cum_exponent[v] for v in stored.cum_exponent}
    for v in range(n):
        L[v] = np.broadcast_to(tip_partials(tips[v], s), (c, p, s))
        E[v] = np.zeros(p, dtype=np.int64)
    res = PruningResult()
    for (v, _, _, a, ma, b, mb) in ops:
        out = np.empty((c, p, s))
        for k in range(c):
            Pa = transition_matrix(Q, rates[k] * tree.blen[ma])
            Pb = transition_matrix(Q, rates[k] * tree.blen[mb])
            out[k] = (L[a][k] @ Pa.T) * (L[b][k] @ Pb.T)
        m = out.max(axis=(0, 2))
        e = np.frexp(m)[1].astype(np.int64)
        L[v] = np.ldexp(out, -e[None, :, None])
        E[v] = E[a] + E[b] + e
        res.partials[v] = L[v]
        res.exponent[v] = e
        res.cum_exponent[v] = E[v]
    root = int(np.flatnonzero(np.asarray(tree.parent) < 0)[0])
    site = np.einsum("c,cpz,z->p", cat_w, L[root], pi)
    with np.errstate(divide="ignore"):
        res.site_lnl = np.log(site) + E[root] * LN2
    res.lnl = math.fsum((pattern_weights * res.site_lnl).tolist())
    return res
