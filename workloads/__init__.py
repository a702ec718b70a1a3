"""Seeded synthetic inputs shared by the oracle tests, GPU parity tests and bench.

Inputs only: trees, raw model parameters, Gamma rate categories and
alignments.  Nothing here computes Q, P, partial likelihoods, reroots or
schedules (that is the method: ``oracle/`` on the reference side and the
C-ABI library on the product side).  Recipe: DESIGN.md "Input recipe".
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .params import (ModelParams, discrete_gamma_rates, hky_fixed,  # noqa: F401
                     random_alignment, random_model)
from .trees import Tree, make_tree, with_blen  # noqa: F401


@dataclass
class Workload:
    """One seeded problem instance."""

    tree: Tree
    model: ModelParams
    rates: np.ndarray           # float64 [c]  (category rates, mean 1)
    cat_weights: np.ndarray     # float64 [c]  (1/c each)
    tips: np.ndarray            # uint8 [n, p] (code s = missing)
    pattern_weights: np.ndarray  # float64 [p]
    alpha: float

    @property
    def n(self) -> int:
        return self.tree.n

    @property
    def p(self) -> int:
        return self.tips.shape[1]

    @property
    def s(self) -> int:
        return self.model.states

    @property
    def c(self) -> int:
        return self.rates.shape[0]


def make_workload(*, tree_kind: str, n: int, p: int, model: str, c: int,
                  seed: int, missing_frac: float = 0.0,
                  model_params: ModelParams | None = None,
                  alpha: float | None = None) -> Workload:
    """Seeded workload.  Streams: SeedSequence(seed).spawn(4) ->
    [topology, branch lengths, model parameters, alignment]."""
    ss = np.random.SeedSequence(seed)
    t_ss, b_ss, m_ss, d_ss = ss.spawn(4)
    tree = make_tree(tree_kind, n, seed, topo_rng=np.random.default_rng(t_ss),
                     blen_rng=np.random.default_rng(b_ss))
    mrng = np.random.default_rng(m_ss)
    mp = model_params if model_params is not None else random_model(model, mrng)
    a = float(mrng.uniform(0.2, 2.0)) if alpha is None else float(alpha)
    rates = discrete_gamma_rates(a, c)
    tips = random_alignment(n, p, mp.states, np.random.default_rng(d_ss), missing_frac)
    return Workload(tree=tree, model=mp, rates=rates, cat_weights=np.full(c, 1.0 / c),
                    tips=tips, pattern_weights=np.ones(p), alpha=a)


# BASELINE.json configs, as concrete seeded recipes.
CONFIGS = {
    "c0_jc": dict(tree_kind="pectinate", n=8, p=1000, model="jc69", c=1),
    "c0_hky": dict(tree_kind="pectinate", n=8, p=1000, model="hky", c=1,
                   model_params=hky_fixed()),
    "c1": dict(tree_kind="pectinate", n=128, p=10_000, model="gtr", c=4),
    "c2": dict(tree_kind="yule", n=1024, p=100_000, model="gtr", c=4),
    "c2_paper": dict(tree_kind="random", n=1024, p=100_000, model="gtr", c=4),
    "c3": dict(tree_kind="random", n=256, p=10_000, model="gy94", c=4),
    "c4": dict(tree_kind="pectinate", n=4096, p=1 << 22, model="gtr", c=4),
}


def config_workload(name: str, seed: int = 1, **over) -> Workload:
    kw = dict(CONFIGS[name])
    kw.update(over)
    return make_workload(seed=seed, **kw)
