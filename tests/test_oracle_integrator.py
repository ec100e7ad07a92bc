"""Pins of the integrator oracle (oracle/integrator.py) against closed forms and the
structure of the scheme — not gpu.

* mass matrices: 1-D Lagrange-on-GLL and Bernstein mass matrices in closed form (textbook values),
  tensor structure, total mass, internal-energy weights int rho b_j = rho vol / t^dim (Bernstein
  integrals are all 1/(deg+1));
* CG: residual bound and agreement with a direct sparse solve;
* RK2-average: exact total-energy conservation (Table 6: the triple point keeps
  E = 10.05), a quiescent uniform box stays at rest, x<->y mirror symmetry of the 2D Sedov blast.
"""
from fractions import Fraction as Fr

import numpy as np
import pytest
import scipy.sparse.linalg as spla

import synth
from oracle import integrator as it


def test_q1_q2_lagrange_mass_closed_form(orc):
    # single unit zone, rho = 1 -> M_V = tensor product of 1-D Lagrange mass matrices
    for k, M1 in [(1, np.array([[Fr(1, 3), Fr(1, 6)], [Fr(1, 6), Fr(1, 3)]])),
                  (2, np.array([[Fr(4, 30), Fr(2, 30), Fr(-1, 30)], [Fr(2, 30), Fr(16, 30), Fr(2, 30)],
                                [Fr(-1, 30), Fr(2, 30), Fr(4, 30)]]))]:
        M1 = M1.astype(float)
        for dim in (2, 3):
            m = synth.box_mesh(dim, k, (1,) * dim, L=(1.0,) * dim)
            R = np.ones((1, m.nq))
            M = it.mass_matrices(m, R)
            ref = M1
            for _ in range(dim - 1):
                ref = np.kron(M1, ref)   # node a = a0 + p (a1 + p a2): a0 fastest
            A = M.MV.toarray()
            zn = m.zone_nodes[0]
            assert np.abs(A[np.ix_(zn, zn)] - ref).max() < 1e-15


def test_bernstein_mass_closed_form(orc):
    # degree 1: [[1/3,1/6],[1/6,1/3]];  degree 2: C(2,i)C(2,j) / (C(4,i+j) 5)
    from math import comb
    for k in (2, 3, 4):
        deg = k - 1
        M1 = np.array([[comb(deg, i) * comb(deg, j) / (comb(2 * deg, i + j) * (2 * deg + 1)) for j in range(k)]
                       for i in range(k)])
        for dim in (2, 3):
            m = synth.box_mesh(dim, k, (1,) * dim, L=(1.0,) * dim)
            M = it.mass_matrices(m, np.full((1, m.nq), 2.5))
            ref = M1
            for _ in range(dim - 1):
                ref = np.kron(M1, ref)
            assert np.abs(M.ME[0] - 2.5 * ref).max() < 2e-15
            assert np.abs(M.me1[0] - 2.5 / k ** dim).max() < 1e-15


@pytest.mark.parametrize("kind,dim,k,N", [("sedov", 2, 3, (5, 4)), ("triple", 2, 3, (14, 6)),
                                           ("sedov", 3, 2, (3, 3, 2)), ("triple", 3, 2, (7, 3, 3))])
def test_total_mass_and_ie_weights(orc, kind, dim, k, N):
    m = synth.make_mesh(kind, dim, k, N)
    s = synth.make_state(m, kind, "S0", 1)
    M = it.mass_matrices(m, s.rho0detJ0)
    one = np.ones(m.num_nodes)
    rho = s.rho0detJ0[:, 0] / np.prod(m.h)
    mass = (rho * np.prod(m.h)).sum()
    assert abs(one @ (M.MV @ one) - mass) < 1e-14 * mass
    assert abs(M.me1.sum() - mass) < 1e-14 * mass
    assert np.abs(M.me1 - (rho * np.prod(m.h))[:, None] / m.nt).max() < 1e-15 * mass
    A = M.MV
    assert abs(A - A.T).max() < 1e-17 * mass
    assert np.abs(np.einsum("zij,zjk->zik", M.ME, M.ME_inv) - np.eye(m.nt)).max() < 1e-10


def test_pcg_matches_direct_solve(orc):
    m = synth.box_mesh(3, 3, (3, 2, 2))
    s = synth.sedov_s0(m)
    M = it.mass_matrices(m, s.rho0detJ0)
    fixed = it.wall_mask(m)
    b = np.random.default_rng(3).standard_normal(m.num_nodes)
    free = ~fixed[1]
    x, n = it.pcg(M.MV, b, free, 1e-15)
    A = M.MV.tocsr()[free][:, free]
    xd = spla.spsolve(A.tocsc(), b[free])
    assert np.all(x[~free] == 0.0)
    assert np.abs(x[free] - xd).max() < 1e-12 * np.abs(xd).max()
    r = b[free] - A @ x[free]
    assert np.linalg.norm(r) <= 1e-15 * np.linalg.norm(b[free]) * 1.0001
    assert 0 < n < 200


def test_wall_mask_counts(orc):
    m = synth.box_mesh(2, 3, (4, 3))
    f = it.wall_mask(m)
    nx, ny = 4 * 3 + 1, 3 * 3 + 1
    assert f[0].sum() == 2 * ny and f[1].sum() == 2 * nx


def _run(rk, x, v, e, steps, dt_scale=0.5):
    dt = None
    for _ in range(steps):
        if dt is None:
            dt = dt_scale * rk.forces(x, v, e).dt_min
        x, v, e, dte = rk.step(x, v, e, dt)
        dt = min(dt * 1.02, dte)
    return x, v, e


@pytest.mark.parametrize("kind,dim,k,N,steps", [("triple", 2, 3, (14, 6), 4), ("sedov", 2, 2, (6, 6), 4),
                                                 ("sedov", 3, 2, (3, 3, 3), 2)])
def test_rk2avg_conserves_total_energy(orc, kind, dim, k, N, steps):
    m = synth.make_mesh(kind, dim, k, N)
    s = synth.make_state(m, kind, "S0", 1)
    rk = it.RK2Avg(m, s.rho0detJ0)
    E0 = sum(it.energies(rk.masses, s.v, s.e))
    if kind == "triple" and dim == 2:
        assert abs(E0 - 10.05) < 1e-13   # Table 6
    if kind == "sedov":
        assert abs(E0 - synth.E_BLAST) < 1e-15
    x, v, e = _run(rk, s.x, s.v, s.e, steps)
    ke, ie = it.energies(rk.masses, v, e)
    assert ke > 0.0                                  # something moved
    assert abs(ke + ie - E0) < 1e-13 * E0


def test_quiescent_box_stays_at_rest(orc):
    m = synth.box_mesh(2, 3, (4, 3))
    R = np.ones((m.num_zones, m.nq)) * np.prod(m.h)
    e = np.full((m.num_zones, m.nt), 2.0)
    rk = it.RK2Avg(m, R)
    x, v, e1 = _run(rk, m.x0.copy(), np.zeros_like(m.x0), e, 2)
    assert np.abs(v).max() < 1e-13 and np.abs(x - m.x0).max() < 1e-14 and np.abs(e1 - 2.0).max() < 1e-13


def test_sedov_mirror_symmetry(orc):
    m = synth.box_mesh(2, 2, (5, 5))
    s = synth.sedov_s0(m)
    rk = it.RK2Avg(m, s.rho0detJ0)
    x, v, e = _run(rk, s.x, s.v, s.e, 3)
    # mirror x <-> y: node (i, j) <-> (j, i) on the (5k+1)^2 lattice, thermo dofs likewise
    n1 = 5 * 2 + 1
    perm = np.arange(n1 * n1).reshape(n1, n1).T.reshape(-1)
    assert np.abs(v[0] - v[1][perm]).max() < 1e-13 * np.abs(v).max()
    assert np.abs(x[0] - x[1][perm]).max() < 1e-14
    zp = np.arange(25).reshape(5, 5).T.reshape(-1)
    tp = np.arange(m.nt).reshape(m.order, m.order).T.reshape(-1)
    assert np.abs(e - e[zp][:, tp]).max() < 1e-12 * np.abs(e).max()


def test_advance_step_control_sequence(orc):
    """RK2Avg.advance's step control (reading R24), pinned on a scripted dt-estimate sequence worked out by
    hand: reject (retry with 0.85 dt) when the estimate is below the dt used, grow by 2 % when it is at
    least 1.25 dt, clip the last step to t_final.  step() is replaced by a stub that records the dt it was
    given and returns the next scripted estimate, so only the control logic runs (t_final = 0.3):
        dt 0.1      est 1.0  accept  t 0.1      next 0.102      (1.0 >= 0.125: grow)
        dt 0.102    est 0.05 reject           next 0.0867     (0.85 dt)
        dt 0.0867   est 0.1  accept  t 0.1867   next 0.0867     (0.1 < 0.108375: keep)
        dt 0.0867   est 0.2  accept  t 0.2734   next 0.088434   (grow)
        dt 0.0266   est 0.02 reject           next 0.02261    (clipped to t_final - t, then 0.85 dt)
        dt 0.02261  est 1.0  accept  t 0.29601  next 0.0230622
        dt 0.00399  est 1.0  accept  t 0.3      next 0.0040698  (clipped, then grown from the clipped dt)"""
    m = synth.box_mesh(2, 1, (1, 1))
    rk = it.RK2Avg(m, np.ones((1, m.nq)))
    script = iter([1.0, 0.05, 0.1, 0.2, 0.02, 1.0, 1.0])
    used = []

    def stub(x, v, e, dt):
        used.append(dt)
        return x + dt, v, e, next(script)

    rk.step = stub
    x0 = np.zeros((2, m.num_nodes))
    x, v, e, t, dt, steps, rejected = rk.advance(x0, x0.copy(), np.zeros((1, 1)), 0.3, 0.1, 10)
    expect = [0.1, 0.102, 0.0867, 0.0867, 0.0266, 0.02261, 0.00399]
    assert np.allclose(used, expect, rtol=0, atol=1e-14), used
    assert (steps, rejected) == (5, 2)
    assert abs(t - 0.3) < 1e-14
    assert np.allclose(x, 0.3, atol=1e-14)   # rejected steps are not applied: x advanced by the accepted dts
    assert abs(dt - 1.02 * 0.00399) < 1e-14
