"""Pins for oracle/model.py and the oracle's transition matrices (CPU)."""
import math

import numpy as np
import pytest
from scipy.linalg import expm

from oracle import model as om
from oracle.pruning import transition_matrix
from workloads import hky_fixed, random_model

MODELS = ["jc69", "hky", "gtr", "gy94"]


def _mp(name, seed=0):
    return random_model(name, np.random.default_rng(seed))


@pytest.mark.parametrize("name", MODELS)
def test_q_generator_properties(name):
    mp = _mp(name)
    Q = om.rate_matrix(mp)
    pi = mp.pi
    s = mp.states
    assert Q.shape == (s, s)
    np.testing.assert_allclose(Q.sum(axis=1), 0, atol=1e-13)
    assert abs(-np.dot(pi, np.diag(Q)) - 1) < 1e-13          # normalised rate
    D = pi[:, None] * Q
    np.testing.assert_allclose(D, D.T, atol=1e-14)           # reversibility
    off = Q[~np.eye(s, dtype=bool)]
    assert np.all(off >= 0)
    np.testing.assert_allclose(pi @ Q, 0, atol=1e-13)        # stationarity


def test_jc_transition_closed_form():
    Q = om.rate_matrix(_mp("jc69"))
    for t in [0.0, 0.01, 0.3, 1.7, 50.0]:
        P = transition_matrix(Q, t)
        e = math.exp(-4 * t / 3)
        same, diff = 0.25 + 0.75 * e, 0.25 - 0.25 * e
        exp = np.full((4, 4), diff)
        np.fill_diagonal(exp, same)
        np.testing.assert_allclose(P, exp, atol=1e-15)


def test_hky_transition_closed_form():
    # HKY85 closed form (Hasegawa et al. 1985): with purines R = piA+piG,
    # pyrimidines Y = piC+piT, beta = 1/(2 R Y + 2 kappa (piA piG + piC piT)),
    # for a transition j within the same class (Pj = R or Y):
    #   P_ij = pi_j (1 + (1/Pj - 1) e^{-beta t}) / 1 ... written below as the
    #   standard three-exponential form; check against the rate-matrix expm.
    mp = hky_fixed()
    Q = om.rate_matrix(mp)
    piA, piC, piG, piT = mp.pi
    k = mp.kappa
    R, Y = piA + piG, piC + piT
    beta = 1.0 / (2 * R * Y + 2 * k * (piA * piG + piC * piT))
    grp = [R, Y, R, Y]
    purine = [True, False, True, False]
    for t in [0.05, 0.4, 2.0]:
        P = transition_matrix(Q, t)
        for i in range(4):
            for j in range(4):
                Pj = grp[j]
                A = 1 + Pj * (k - 1)
                e1 = math.exp(-beta * t)
                eA = math.exp(-beta * A * t)
                pj = mp.pi[j]
                if i == j:
                    val = pj + pj * (1 / Pj - 1) * e1 + ((Pj - pj) / Pj) * eA
                elif purine[i] == purine[j]:
                    val = pj + pj * (1 / Pj - 1) * e1 - (pj / Pj) * eA
                else:
                    val = pj * (1 - e1)
                assert abs(P[i, j] - val) < 1e-14, (t, i, j)


@pytest.mark.parametrize("name", MODELS)
def test_transition_matrix_properties(name):
    mp = _mp(name, 3)
    Q = om.rate_matrix(mp)
    s = mp.states
    np.testing.assert_allclose(transition_matrix(Q, 0.0), np.eye(s), atol=1e-15)
    t1, t2 = 0.13, 0.29
    P1, P2, P12 = (transition_matrix(Q, t) for t in (t1, t2, t1 + t2))
    np.testing.assert_allclose(P1 @ P2, P12, atol=1e-13)     # Chapman-Kolmogorov
    np.testing.assert_allclose(P12.sum(axis=1), 1, atol=1e-13)
    D = mp.pi[:, None] * P12
    np.testing.assert_allclose(D, D.T, atol=1e-14)           # detailed balance
    Pinf = transition_matrix(Q, 200.0)
    np.testing.assert_allclose(Pinf, np.tile(mp.pi, (s, 1)), atol=1e-12)


def test_gy94_structure():
    cod = om.sense_codons()
    assert len(cod) == 61 and cod[0] == "AAA" and cod[-1] == "TTT"
    assert "TAA" not in cod and "TAG" not in cod and "TGA" not in cod
    mp = _mp("gy94")
    Q = om.rate_matrix(mp)
    # Sense codons with one-nucleotide neighbours: 61*9 ordered pairs minus the
    # 23 sense->stop pairs (TAA has 7 sense neighbours, TAG and TGA 8 each).
    nz = np.count_nonzero(Q[~np.eye(61, dtype=bool)])
    assert nz == 61 * 9 - 23
    # omega scales exactly the non-synonymous entries: ATG (Met) -> ATA (Ile)
    # is a transition and non-synonymous; CTT -> CTC (Leu) is synonymous.
    i, j = cod.index("ATG"), cod.index("ATA")
    a, b = cod.index("CTT"), cod.index("CTC")
    r1 = Q[i, j] / mp.pi[j]
    r2 = Q[a, b] / mp.pi[b]
    assert abs(r1 / r2 - mp.omega) < 1e-12
    # transversion synonymous: CTT -> CTA (Leu); ratio to transition synonymous = 1/kappa
    c_ = cod.index("CTA")
    r3 = Q[a, c_] / mp.pi[c_]
    assert abs(r2 / r3 - mp.kappa) < 1e-12


def test_expm_is_not_eigen_route():
    # The oracle's P comes from scipy's Pade expm, not an eigendecomposition:
    # sanity-check it against an independent Taylor series at small t.
    mp = _mp("gtr", 5)
    Q = om.rate_matrix(mp)
    t = 0.05
    T = np.eye(4)
    term = np.eye(4)
    for k in range(1, 30):
        term = term @ (Q * t) / k
        T = T + term
    np.testing.assert_allclose(transition_matrix(Q, t), T, atol=1e-15)
    np.testing.assert_allclose(expm(Q * t), T, atol=1e-15)
