"""Pins of the oracle's 1-D tables and small linear algebra (not gpu).

Each check uses something other than the oracle: exactness of Gauss-Legendre on monomials (closed
form 1/(m+1)), numpy's Legendre roots for GLL, Lagrange/Bernstein identities, LAPACK (numpy.linalg)
for the symmetric eigen-solver and the smallest singular value.
Readings: DESIGN.md R3 (GL, n = 2k per dim), R4 (GLL Lagrange kinematic basis), R5 (Bernstein thermo).
"""
import json
import os

import numpy as np
import pytest

from tests._closed import gll01

K_ALL = list(range(1, 9))


@pytest.mark.parametrize("k", K_ALL)
def test_gauss_legendre_exactness(orc, k):
    t = orc.tables_1d(k)
    n = 2 * k
    assert t["qpt"].shape == (n,)
    assert abs(t["qwt"].sum() - 1.0) < 4e-16
    # exact for degree <= 2n-1 = 4k-1 (the integrands of eq (4) have degree <= 3k-1)
    for m in range(0, 4 * k):
        assert abs((t["qwt"] * t["qpt"] ** m).sum() - 1.0 / (m + 1)) < 2e-15, m
    # at degree 2n the error is the closed-form Gauss remainder (n!)^4 / ((2n+1) ((2n)!)^2) on [0,1]
    from math import factorial
    rem = factorial(n) ** 4 / ((2 * n + 1) * factorial(2 * n) ** 2)
    err = 1.0 / (4 * k + 1) - (t["qwt"] * t["qpt"] ** (4 * k)).sum()
    assert abs(err - rem) <= 2e-3 * rem + 1e-16, (err, rem)


@pytest.mark.parametrize("k", K_ALL)
def test_gll_nodes_match_numpy(orc, k):
    t = orc.tables_1d(k)
    x, _ = gll01(k)
    assert np.abs(t["gll"] - x).max() < 2e-15


@pytest.mark.parametrize("k", K_ALL)
def test_lagrange_identities(orc, k):
    t = orc.tables_1d(k)
    B, G, q, g = t["B"], t["G"], t["qpt"], t["gll"]
    # partition of unity and its derivative
    assert np.abs(B.sum(1) - 1.0).max() < 5e-15
    assert np.abs(G.sum(1)).max() < 5e-13
    # interpolation exactness for polynomials of degree <= k: sum_a f(x_a) W_a(q) = f(q)
    for m in range(k + 1):
        assert np.abs(B @ g ** m - q ** m).max() < 1e-13
        assert np.abs(G @ g ** m - (m * q ** (m - 1) if m else 0 * q)).max() < 1e-11


@pytest.mark.parametrize("k", K_ALL)
def test_bernstein_identities(orc, k):
    t = orc.tables_1d(k)
    Phi, w, q = t["Phi"], t["qwt"], t["qpt"]
    assert np.abs(Phi.sum(1) - 1.0).max() < 4e-15          # B^T 1 = 1 (partition of unity)
    assert (Phi >= 0).all()
    # each Bernstein polynomial of degree k-1 integrates to 1/k
    assert np.abs(w @ Phi - 1.0 / k).max() < 4e-16
    # linear precision: sum_j (j/(k-1)) phi_j(x) = x
    if k > 1:
        assert np.abs(Phi @ (np.arange(k) / (k - 1)) - q).max() < 4e-15


def test_paper_printed_shapes(orc):
    """3D Q2-Q1: 81 x 64 basis-gradient table; F_z 81 x 8.  3D Q4-Q3: 375 x 512."""
    import synth
    gold = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_values.json")))
    for name, k in (("Q2-Q1", 2), ("Q4-Q3", 4)):
        m = synth.box_mesh(3, k, (1, 1, 1))
        s = synth.sedov_s0(m)
        assert 3 * m.nk == gold["basis_sizes_3d"][name]["kinematic_dofs"]
        assert m.nq == gold["basis_sizes_3d"][name]["quad_points"]
        if k == 2:
            r = orc.evaluate(m, s, definition=True)
            assert r.Fz.shape[1:] == (gold["Fz_shape_3d_Q2Q1"]["rows"], gold["Fz_shape_3d_Q2Q1"]["cols"])


@pytest.mark.parametrize("d", [2, 3])
def test_sym_eig_vs_lapack(orc, d):
    rng = np.random.default_rng(11 + d)
    worst_val = worst_vec = 0.0
    for _ in range(3000):
        A = rng.standard_normal((d, d)) * 10 ** rng.uniform(-3, 3)
        A = 0.5 * (A + A.T)
        lam, V = orc.sym_eig(A)
        ref = np.linalg.eigvalsh(A)
        nrm = np.abs(ref).max()
        worst_val = max(worst_val, np.abs(lam - ref).max() / nrm)
        # eigenvector residual and orthonormality
        worst_vec = max(worst_vec, np.abs(A @ V - V * lam).max() / nrm, np.abs(V.T @ V - np.eye(d)).max())
    assert worst_val < 1e-14
    assert worst_vec < 1e-14


def test_sym_eig_ties(orc):
    """Reading R9: a scalar (or zero) matrix yields s = e_1; ties keep the lower coordinate first."""
    for d in (2, 3):
        for c in (0.0, -1.5):
            lam, V = orc.sym_eig(c * np.eye(d))
            assert np.all(lam == c)
            assert np.array_equal(V, np.eye(d))


@pytest.mark.parametrize("d", [2, 3])
def test_sigma_min_vs_lapack(orc, d):
    rng = np.random.default_rng(7 + d)
    worst = 0.0
    for _ in range(3000):
        J = np.eye(d) + 0.4 * rng.standard_normal((d, d))
        s = orc.sigma_min(J)
        ref = np.linalg.svd(J, compute_uv=False)
        # sigma_min via eig(J^T J): relative error ~ eps * cond(J)^2
        worst = max(worst, abs(s - ref[-1]) / ref[0] / (ref[0] / ref[-1]))
    assert worst < 1e-14
