"""The dt filter of KB1 (pointwise.cuh, point_eval3<FILTER=true>) skips the exact sigma_min(J) solve at
points whose inverse dt provably stays below an exact value already found.  Its soundness rests on one
inequality, checked here on the host (no GPU): for a symmetric 3x3 M with q = tr(M)/3 and B = M - qI,

    lambda_min(M) >= q - sqrt(2/3) |B|_F

(B is traceless: with mu_1 the most negative eigenvalue of B, |B|_F^2 >= mu_1^2 + (mu_2 + mu_3)^2 / 2
= 3/2 mu_1^2), tight when the two larger eigenvalues tie.  And the resulting inverse-dt bound
k / sqrt(l) * (c_s + 2.5 k (mu/rho) / sqrt(l)) decreases in l, so a lower bound of lambda_min gives an
upper bound of the inverse dt (reading R10)."""
import numpy as np


def bound(M):
    q = np.trace(M) / 3.0
    B = M - q * np.eye(3)
    return q - np.sqrt(2.0 / 3.0) * np.linalg.norm(B)


def test_lower_bound_of_smallest_eigenvalue_random_jacobians():
    rng = np.random.default_rng(7)
    worst = np.inf
    for _ in range(20000):
        J = np.eye(3) * rng.uniform(0.5, 2.0) + rng.normal(scale=rng.uniform(0.0, 0.6), size=(3, 3))
        M = J.T @ J
        lam = np.linalg.eigvalsh(M)[0]
        b = bound(M)
        assert b <= lam * (1 + 1e-13) + 1e-15
        worst = min(worst, lam - b)
    assert worst >= -1e-14


def test_bound_is_tight_when_the_larger_two_tie():
    # eigenvalues (l, L, L): the bound is exact
    for l, L in ((1.0, 1.44), (0.3, 2.0), (1.0, 1.0)):
        Q, _ = np.linalg.qr(np.random.default_rng(1).normal(size=(3, 3)))
        M = Q @ np.diag([l, L, L]) @ Q.T
        assert abs(bound(M) - l) <= 1e-13 * L


def test_bound_on_the_triple_point_zone_shape():
    # C5 zones are 7/48 x 1/8 x 1/8: J^T J = diag(h_x^2, h^2, h^2), smallest two tied -> bound 15 % low
    hx, h = 7.0 / 48.0, 0.125
    M = np.diag([hx * hx, h * h, h * h])
    lam = h * h
    b = bound(M)
    assert b <= lam and b > 0.8 * lam


def test_inverse_dt_is_monotone_in_lambda():
    k, cs, mor = 4.0, 1.3, 0.2
    inv = lambda l: k / np.sqrt(l) * (cs + 2.5 * k * mor / np.sqrt(l))
    ls = np.linspace(0.01, 2.0, 200)
    v = inv(ls)
    assert np.all(np.diff(v) < 0)
