"""ORACLE (test infrastructure only) -- Felsenstein pruning in fp64.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  Shares no code with the CUDA path.

What it computes, in the paper's order:

1. Transition matrices.  Pr(x | z, t) of Eq. (1) (§II-A) for a
   branch of length t in rate category c is P = expm(Q * r_c * t) (scipy's
   library matrix exponential -- deliberately NOT the eigen route the GPU uses),
   rows = parent state z, columns = child state x (reading A2).
2. Partial likelihoods, Eq. (1):
       L_k(z) = (sum_x Pr(x|z,t_l) L_l(x)) * (sum_y Pr(y|z,t_m) L_m(y))
   for every pattern i, parent state z, category c (reading A3) and internal
   node k, children visited before parents (post-order, Fig. 2).
   A tip's partials are the one-hot vector of its state, all-ones if missing
   (reading A23).
3. Rescaling ("application-managed"; reading A5): after
   each node, per pattern m = max over (c, z); e = frexp(m) exponent; the
   node's partials are multiplied by 2^-e (exact) and e is added to the
   pattern's cumulative exponent E_i.
4. Root integration (Felsenstein [7]; reading A4):
       lnL_i = ln( sum_c w_c sum_z pi_z L_root(i, c, z) ) + E_i ln 2,
       lnL   = math.fsum_i( wt_i lnL_i ).
5. Edge log-likelihood at a branch (parent u, child v, matrix P_v):
       lnL_i = ln( sum_c w_c sum_z pi_z L_u(z) sum_x P_v(z,x) L_v(x) )
               + (E_u + E_v) ln 2.

Pins: tests/test_oracle_pruning.py (JC 2- and 3-taxon closed forms, brute
force over ancestral states, reroot invariance, t -> infinity limit,
all-missing patterns, scaled == unscaled).
"""
from __future__ import annotations

import math

import numpy as np
from scipy.linalg import expm

LN2 = math.log(2.0)


def transition_matrix(Q: np.ndarray, t: float) -> np.ndarray:
    """Pr(x | z, t) = expm(Q t)[z, x] (reading A2)."""
    return expm(Q * t)


def tip_partials(states: np.ndarray, s: int) -> np.ndarray:
    """[p, s] one-hot rows; code s (missing) -> all ones (reading A23)."""
    p = states.shape[0]
    L = np.zeros((p, s))
    ok = states < s
    L[np.flatnonzero(ok), states[ok].astype(np.int64)] = 1.0
    L[~ok, :] = 1.0
    return L


def children_of(parent: np.ndarray) -> list[list[int]]:
    ch: list[list[int]] = [[] for _ in range(parent.shape[0])]
    for v, u in enumerate(parent.tolist()):
        if u >= 0:
            ch[u].append(v)
    for c in ch:
        c.sort()
    return ch


def postorder(parent: np.ndarray) -> list[int]:
    """Internal nodes, children before parents (child1 = smaller id first)."""
    ch = children_of(parent)
    root = int(np.flatnonzero(parent < 0)[0])
    out: list[int] = []
    stack = [(root, False)]
    while stack:
        v, done = stack.pop()
        if not ch[v]:
            continue
        if done:
            out.append(v)
        else:
            stack.append((v, True))
            for c in reversed(ch[v]):
                stack.append((c, False))
    return out


class PruningResult:
    def __init__(self):
        self.site_lnl: np.ndarray | None = None   # [p]
        self.lnl: float = float("nan")
        self.partials: dict[int, np.ndarray] = {}   # node -> [c, p, s] (scaled)
        self.exponent: dict[int, np.ndarray] = {}   # node -> own exponent e [p] (int64)
        self.cum_exponent: dict[int, np.ndarray] = {}  # node -> subtree sum [p]


def prune(tree, Q: np.ndarray, pi: np.ndarray, rates: np.ndarray, cat_w: np.ndarray,
          tips: np.ndarray, pattern_weights: np.ndarray, *, scale: bool = True,
          keep_partials: bool = False, tip_partial_override: dict | None = None
          ) -> PruningResult:
    """Post-order Felsenstein pruning on ``tree`` as rooted (steps 1-4 above)."""
    n = tree.n
    s = Q.shape[0]
    c = rates.shape[0]
    p = tips.shape[1]
    parent = np.asarray(tree.parent)
    ch = children_of(parent)
    res = PruningResult()

    def leaf(v: int) -> np.ndarray:  # [c, p, s]
        if tip_partial_override is not None and v in tip_partial_override:
            base = np.asarray(tip_partial_override[v], dtype=np.float64)
        else:
            base = tip_partials(tips[v], s)
        return np.broadcast_to(base, (c, p, s))

    L: dict[int, np.ndarray] = {}
    E: dict[int, np.ndarray] = {}
    for v in range(n):
        L[v] = leaf(v)
        E[v] = np.zeros(p, dtype=np.int64)
    for v in postorder(parent):
        a, b = ch[v]
        out = np.empty((c, p, s))
        for k in range(c):
            Pa = transition_matrix(Q, rates[k] * tree.blen[a])
            Pb = transition_matrix(Q, rates[k] * tree.blen[b])
            out[k] = (L[a][k] @ Pa.T) * (L[b][k] @ Pb.T)          # Eq. (1)
        e = np.zeros(p, dtype=np.int64)
        if scale:
            m = out.max(axis=(0, 2))
            e = np.frexp(m)[1].astype(np.int64)
            out = np.ldexp(out, -e[None, :, None])
        L[v] = out
        E[v] = E[a] + E[b] + e
        if keep_partials:
            res.partials[v] = out
            res.exponent[v] = e
            res.cum_exponent[v] = E[v]
        # free children no longer needed
        if a >= n:
            del L[a]
        if b >= n:
            del L[b]
    root = tree.root
    site = np.einsum("c,cpz,z->p", cat_w, L[root], pi)
    with np.errstate(divide="ignore"):
        res.site_lnl = np.log(site) + E[root] * LN2
    res.lnl = math.fsum((pattern_weights * res.site_lnl).tolist())
    return res


def loglik(tree, Q, pi, rates, cat_w, tips, pattern_weights, scale=True) -> float:
    return prune(tree, Q, pi, rates, cat_w, tips, pattern_weights, scale=scale).lnl


def edge_site_lnl(Lu: np.ndarray, Eu: np.ndarray, Lv: np.ndarray, Ev: np.ndarray,
                  P_by_cat: list[np.ndarray], pi: np.ndarray, cat_w: np.ndarray) -> np.ndarray:
    """Step 5: per-pattern edge log-likelihood.  L* are [c, p, s]."""
    acc = np.zeros(Lu.shape[1])
    for k in range(Lu.shape[0]):
        acc += cat_w[k] * np.einsum("pz,z,pz->p", Lu[k], pi, Lv[k] @ P_by_cat[k].T)
    return np.log(acc) + (Eu + Ev) * LN2
