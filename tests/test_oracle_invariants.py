"""Invariants and exact brute force pinning the oracle on general (curved, moving) states (not gpu).

* momentum conservation: sum_a (F_z 1)_{c,a} = 0 for ANY state because sum_a grad W_a = 0
* discrete energy identity v^T (F.1) = 1^T (F^T v) (basis of Table 6's energy conservation)
* Galilean invariance (v -> v + U) and frame indifference (rigid rotation Q of x, x0, v)
* definition mode (F_z = A_z B^T formed, kernels 7/8/10) == associativity mode
* exact-rational brute force of F_z on a single sheared Q1-Q0 and Q2-Q1 zone (viscosity off), 2D and 3D
"""
from fractions import Fraction

import numpy as np
import pytest

import synth
from tests._closed import exact_Fz_affine_novisc

CASES = [("C1", None, None), ("C2", (6, 5), None), ("C3", (3, 3, 2), None), ("C4", (2, 2, 2), None),
         ("C5", (3, 2, 2), 3)]


def _case(name, N, k, which="S1"):
    return synth.config(name, which, N=N, k=k)


@pytest.mark.parametrize("name,N,k", CASES)
def test_momentum_and_energy(orc, name, N, k):
    m, s = _case(name, N, k)
    r = orc.evaluate(m, s)
    assert r.diag["n_bad"] == 0
    scale = np.abs(r.Fz1).sum()
    assert np.abs(r.F1.sum(1)).max() < 1e-14 * scale
    assert np.abs(r.Fz1.sum(2)).max() < 1e-14 * np.abs(r.Fz1).max() * m.nk
    ev = (s.v * r.F1).sum()
    assert abs(ev - r.FTv.sum()) < 1e-13 * (np.abs(s.v).max() * scale)


@pytest.mark.parametrize("name,N,k", CASES[:4])
def test_galilean_invariance(orc, name, N, k):
    m, s = _case(name, N, k)
    r = orc.evaluate(m, s)
    U = np.array([0.7, -1.1, 0.4])[:m.dim, None]
    s2 = synth.State(s.x, np.ascontiguousarray(s.v + U), s.e, s.rho0detJ0)
    r2 = orc.evaluate(m, s2)
    assert np.abs(r2.F1 - r.F1).max() < 1e-13 * np.abs(r.F1).max()
    assert np.abs(r2.FTv - r.FTv).max() < 1e-12 * np.abs(r.FTv).max()
    assert abs(r2.dt_min - r.dt_min) < 1e-13 * r.dt_min


def _rot(dim):
    if dim == 2:
        t = 0.61
        return np.array([[np.cos(t), -np.sin(t)], [np.sin(t), np.cos(t)]])
    a, b = 0.61, -0.37
    Rz = np.array([[np.cos(a), -np.sin(a), 0], [np.sin(a), np.cos(a), 0], [0, 0, 1]])
    Rx = np.array([[1, 0, 0], [0, np.cos(b), -np.sin(b)], [0, np.sin(b), np.cos(b)]])
    return Rz @ Rx


@pytest.mark.parametrize("name,N,k", CASES[:4])
def test_frame_indifference(orc, name, N, k):
    """Rotating x, x0 and v by Q rotates F.1 by Q and leaves F^T v and dt unchanged."""
    m, s = _case(name, N, k)
    r = orc.evaluate(m, s)
    Q = _rot(m.dim)
    m2 = synth.Mesh(m.dim, m.order, m.N, m.L, np.ascontiguousarray(Q @ m.x0), m.zone_nodes, m.zone_mat,
                    m.mat_gamma)
    s2 = synth.State(np.ascontiguousarray(Q @ s.x), np.ascontiguousarray(Q @ s.v), s.e, s.rho0detJ0)
    r2 = orc.evaluate(m2, s2)
    assert np.abs(r2.F1 - Q @ r.F1).max() < 1e-12 * np.abs(r.F1).max()
    assert np.abs(r2.FTv - r.FTv).max() < 1e-12 * np.abs(r.FTv).max()
    assert abs(r2.dt_min - r.dt_min) < 1e-12 * r.dt_min


@pytest.mark.parametrize("name,N,k", [("C1", None, None), ("C3", (2, 2, 2), None), ("C2", (2, 2), 3)])
def test_definition_mode_matches(orc, name, N, k):
    """F_z formed explicitly (eq 5-6, kernel 7) then F.1 / F^T v (kernels 8, 10) == associativity mode."""
    m, s = _case(name, N, k)
    a = orc.evaluate(m, s)
    b = orc.evaluate(m, s, definition=True)
    assert np.abs(a.F1 - b.F1).max() < 1e-14 * np.abs(a.F1).max()
    assert np.abs(a.FTv - b.FTv).max() < 1e-14 * np.abs(a.FTv).max()
    assert a.dt_min == b.dt_min
    # F_z 1 and F_z^T V recomputed from the formed matrices with numpy
    Vz = s.v[:, m.zone_nodes].transpose(1, 0, 2).reshape(m.num_zones, -1)
    assert np.abs(b.Fz.sum(2).reshape(b.Fz1.shape) - b.Fz1).max() < 1e-15 * np.abs(b.Fz1).max()
    assert np.abs(np.einsum("zij,zi->zj", b.Fz, Vz) - b.FTv).max() < 1e-14 * np.abs(b.FTv).max()


@pytest.mark.parametrize("dim", [2, 3])
@pytest.mark.parametrize("k", [1, 2])
def test_exact_rational_single_zone(orc, dim, k):
    """Sheared affine zone, viscosity off, non-uniform positive e: every integrand of eq (4) is a
    polynomial of degree <= 3k-2, so F_z is computed exactly in rationals and compared."""
    A = [[1.5, 0.375, 0.125], [-0.25, 1.25, 0.0625], [0.1875, -0.125, 0.875]]
    A = [row[:dim] for row in A[:dim]]
    b = [0.25, -0.5, 0.75][:dim]
    m = synth.box_mesh(dim, k, (1,) * dim)
    Am = np.array(A)
    x = np.ascontiguousarray(Am @ m.x0 + np.array(b)[:, None])
    rng = np.random.default_rng(3)
    v = np.ascontiguousarray(rng.standard_normal(x.shape))
    E = np.round(rng.uniform(0.2, 1.0, size=(1, m.nt)) * 64) / 64
    R = np.full((1, m.nq), 1.375)
    s = synth.State(x, v, np.ascontiguousarray(E), R)
    r = orc.evaluate(m, s, params=orc.Params(use_viscosity=0), definition=True)
    gam = Fraction(1.4)
    ex = exact_Fz_affine_novisc(dim, k, [[Fraction(a) for a in row] for row in A], Fraction(1.375), gam,
                                [Fraction(e) for e in E[0]])
    exf = np.array([[float(c) for c in row] for row in ex])
    assert np.abs(r.Fz[0] - exf).max() < 2e-15 * np.abs(exf).max()
    # and F^T v from the exact F_z
    ftv = exf.T @ v[:, m.zone_nodes[0]].reshape(-1)
    assert np.abs(r.FTv[0] - ftv).max() < 1e-14 * np.abs(ftv).max()
