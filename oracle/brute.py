"""ORACLE (test infrastructure only) -- brute-force likelihood for tiny trees.

Only tests/ may use this module.  It is the textbook definition the pruning
recursion of Eq. (1) (§II-A) factorises (Felsenstein [7],
PAPER.md:310): for each pattern i

    L_i = sum_c w_c  sum_{states of all internal nodes}
              pi(x_root) * prod_{branches (u -> v)} P_c(x_u -> x_v; t_v)

with tip states fixed by the data (a missing tip sums over its s states).
Cost s^(n-1) per pattern: use only for n <= 6 (s = 4) or n <= 3 (s = 61).
"""
from __future__ import annotations

import itertools
import math

import numpy as np
from scipy.linalg import expm


def site_likelihoods(tree, Q, pi, rates, cat_w, tips) -> np.ndarray:
    n = tree.n
    s = Q.shape[0]
    p = tips.shape[1]
    N = tree.parent.shape[0]
    internal = list(range(n, N))
    root = tree.root
    out = np.zeros(p)
    for k, r in enumerate(rates):
        P = {v: expm(Q * r * tree.blen[v]) for v in range(N) if tree.parent[v] >= 0}
        for i in range(p):
            tip_choices = [range(s) if tips[v, i] >= s else [int(tips[v, i])] for v in range(n)]
            total = 0.0
            for xs_int in itertools.product(range(s), repeat=len(internal)):
                x = {}
                for v, xv in zip(internal, xs_int):
                    x[v] = xv
                for xs_tip in itertools.product(*tip_choices):
                    for v in range(n):
                        x[v] = xs_tip[v]
                    term = pi[x[root]]
                    for v in range(N):
                        u = int(tree.parent[v])
                        if u >= 0:
                            term *= P[v][x[u], x[v]]
                    total += term
            out[i] += cat_w[k] * total
    return out


def loglik(tree, Q, pi, rates, cat_w, tips, pattern_weights) -> float:
    L = site_likelihoods(tree, Q, pi, rates, cat_w, tips)
    return math.fsum((pattern_weights * np.log(L)).tolist())
