"""Seeded model-parameter, rate-category and alignment generators (inputs only).

The paper draws "arbitrary datasets, evolutionary models" per ``--seed``
(§VI-F) without stating distributions.  DESIGN.md reading
A13 fixes them:

  * GTR exchangeabilities r_ij ~ U(0.5, 2) in the order AC, AG, AT, CG, CT, GT;
  * nucleotide frequencies pi proportional to U(0.5, 1.5);
  * Gamma shape alpha ~ U(0.2, 2);
  * GY94: kappa ~ U(1.5, 3), omega ~ U(0.1, 1), codon pi proportional to U(0.5, 1.5);
  * tip states i.i.d. uniform over the s states; pattern weights 1.

Only *raw parameters* are produced here.  Building Q, its eigensystem or the
transition matrices is the method's arithmetic and lives separately in
``oracle/`` (fp64 reference) and in the product's C++ host code.

The discrete-Gamma rate categories (Yang 1994, mean of each category) are an
input to both sides, like branch lengths: the library receives them through
``rrl_set_category_rates`` (the paper's Eq. (1) has no category axis,
DESIGN.md reading A3).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np
from scipy import special, stats


NUC_MODELS = ("jc69", "hky", "gtr")
CODON_MODELS = ("gy94",)


@dataclass
class ModelParams:
    """Raw substitution-model parameters (no derived matrices)."""

    name: str                 # jc69 | hky | gtr | gy94
    states: int               # 4 or 61
    pi: np.ndarray            # float64 [s], sums to 1
    kappa: float = 1.0        # hky, gy94
    omega: float = 1.0        # gy94
    exch: np.ndarray | None = None  # gtr: float64 [6] (AC, AG, AT, CG, CT, GT)
    extra: dict = field(default_factory=dict)


def discrete_gamma_rates(alpha: float, c: int) -> np.ndarray:
    """Yang (1994) mean-of-category discrete Gamma rates with mean 1.

    Cut points x_k = F^{-1}(k/c) of Gamma(shape=alpha, rate=alpha); the rate of
    category k is c * [P(alpha+1, alpha x_k) - P(alpha+1, alpha x_{k-1})],
    where P is the regularised lower incomplete gamma function.
    """
    if c == 1:
        return np.ones(1)
    cuts = stats.gamma.ppf(np.arange(1, c) / c, a=alpha, scale=1.0 / alpha)
    upper = np.concatenate([special.gammainc(alpha + 1.0, cuts * alpha), [1.0]])
    lower = np.concatenate([[0.0], upper[:-1]])
    return c * (upper - lower)


def _norm(v: np.ndarray) -> np.ndarray:
    return v / v.sum()


def random_model(name: str, rng: np.random.Generator) -> ModelParams:
    if name == "jc69":
        return ModelParams("jc69", 4, np.full(4, 0.25))
    if name == "hky":
        return ModelParams("hky", 4, _norm(rng.uniform(0.5, 1.5, 4)),
                           kappa=float(rng.uniform(1.5, 3.0)))
    if name == "gtr":
        pi = _norm(rng.uniform(0.5, 1.5, 4))
        return ModelParams("gtr", 4, pi, exch=rng.uniform(0.5, 2.0, 6))
    if name == "gy94":
        kappa = float(rng.uniform(1.5, 3.0))
        omega = float(rng.uniform(0.1, 1.0))
        return ModelParams("gy94", 61, _norm(rng.uniform(0.5, 1.5, 61)),
                           kappa=kappa, omega=omega)
    raise ValueError(name)


def hky_fixed() -> ModelParams:
    """BASELINE.json configs[0]: HKY with kappa = 2, pi = (0.1, 0.2, 0.3, 0.4)."""
    return ModelParams("hky", 4, np.array([0.1, 0.2, 0.3, 0.4]), kappa=2.0)


def random_alignment(n: int, p: int, s: int, rng: np.random.Generator,
                     missing_frac: float = 0.0) -> np.ndarray:
    """uint8 [n, p] tip states, i.i.d. uniform; code s means missing/gap."""
    a = rng.integers(0, s, size=(n, p), dtype=np.uint8)
    if missing_frac > 0:
        m = rng.random((n, p)) < missing_frac
        a[m] = s
    return a
