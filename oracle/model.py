"""ORACLE (test infrastructure only) -- substitution-model rate matrices, fp64.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  It shares no code with the product
(paper_conf_ipps_ayresc18_b200/), which builds its own Q in C++.

The paper evaluates "time-reversible evolutionary models" (§V-A)
with transition probabilities Pr(x | z, t) (Eq. (1), §II-A) but does
not list the models; readings A2/A13 fix them.  Here:

  Q_ij (i != j) as defined per model, Q_ii = -sum_{j != i} Q_ij, then Q is
  scaled so that the expected rate -sum_i pi_i Q_ii equals 1.

  JC69: Q_ij equal for all i != j (pi uniform).
  HKY : Q_ij = kappa * pi_j for transitions (A<->G, C<->T), pi_j otherwise.
  GTR : Q_ij = r_ij * pi_j with symmetric exchangeabilities r (AC,AG,AT,CG,CT,GT).
  GY94: codons = the 61 sense codons of the standard genetic code in ACGT
        lexicographic order (stops TAA, TAG, TGA removed).  Q_ij = 0 if codons
        i and j differ at more than one position, else
        pi_j * (kappa if the change is a transition) * (omega if it changes
        the amino acid).

Parity: pinned by tests/test_oracle_model.py (row sums, detailed balance,
normalisation, JC closed form, codon count and synonymous-pair counts).
"""
from __future__ import annotations

import itertools

import numpy as np

NUC = "ACGT"
# Standard genetic code written in the conventional TCAG x TCAG x TCAG order.
_TCAG = "TCAG"
_AA_TCAG = "FFLLSSSSYY**CC*WLLLLPPPPHHQQRRRRIIIMTTTTNNKKSSRRVVVVAAAADDEEGGGG"


def _standard_code() -> dict[str, str]:
    code = {}
    k = 0
    for a in _TCAG:
        for b in _TCAG:
            for c in _TCAG:
                code[a + b + c] = _AA_TCAG[k]
                k += 1
    return code


def sense_codons() -> list[str]:
    """The 61 sense codons in ACGT-lexicographic order."""
    code = _standard_code()
    return ["".join(t) for t in itertools.product(NUC, repeat=3) if code["".join(t)] != "*"]


def _is_transition(x: str, y: str) -> bool:
    return {x, y} in ({"A", "G"}, {"C", "T"})


def _normalise(Q: np.ndarray, pi: np.ndarray) -> np.ndarray:
    Q = Q.copy()
    np.fill_diagonal(Q, 0.0)
    np.fill_diagonal(Q, -Q.sum(axis=1))
    rate = -np.dot(pi, np.diag(Q))
    return Q / rate


def rate_matrix(model) -> np.ndarray:
    """Normalised Q (fp64) from a ``workloads.ModelParams``."""
    pi = np.asarray(model.pi, dtype=np.float64)
    s = model.states
    Q = np.zeros((s, s))
    if model.name == "jc69":
        Q[:] = 1.0
    elif model.name == "hky":
        for i in range(4):
            for j in range(4):
                if i != j:
                    Q[i, j] = pi[j] * (model.kappa if _is_transition(NUC[i], NUC[j]) else 1.0)
    elif model.name == "gtr":
        pairs = [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)]
        r = np.zeros((4, 4))
        for (i, j), v in zip(pairs, model.exch):
            r[i, j] = r[j, i] = v
        for i in range(4):
            for j in range(4):
                if i != j:
                    Q[i, j] = r[i, j] * pi[j]
    elif model.name == "gy94":
        code = _standard_code()
        cod = sense_codons()
        assert len(cod) == 61 == s
        for i, ci in enumerate(cod):
            for j, cj in enumerate(cod):
                if i == j:
                    continue
                diff = [k for k in range(3) if ci[k] != cj[k]]
                if len(diff) != 1:
                    continue
                k = diff[0]
                q = pi[j]
                if _is_transition(ci[k], cj[k]):
                    q *= model.kappa
                if code[ci] != code[cj]:
                    q *= model.omega
                Q[i, j] = q
    else:
        raise ValueError(model.name)
    return _normalise(Q, pi)
