"""Closed-form pins of the oracle (not gpu).

Every expected value below is derived by hand from eq (4)-(6) and the
stress/time-step readings of DESIGN.md §3 (R1, R2, R6, R8, R10, R11), evaluated with numpy — never
with the oracle's code.  Each case is chosen so that a plausible mistake fails it:
  * Nanson on a *sheared* zone             -> transpose of adj(J) (R6), sign of F.1 (R12)
  * uniform pressure on a closed mesh      -> assembly, interior cancellation, face totals
  * Sedov S0 / dt at rest                  -> EOS, linear viscosity term, psi0 = 1 at rest, sigma_min(J), cfl
  * uniform expansion                      -> quadratic viscosity term, F^T v projection, integral of phi_j
  * stretched mesh + 1-D compression       -> compression eigenvector, l = h0 |J J0^-1 s|, rho = rho0|J0|/|J|
  * shear / rigid rotation                 -> psi0 = |div v|/|grad v|, smallest eigenvalue, F^T v = 0 for div-free
  * lambda inside the switch window        -> smoothstep polynomial
"""
import numpy as np
import pytest

import synth
from tests._closed import gll01, nanson_F1

GAM = 1.4


def uniform_case(dim, k, N, A=None, vfun=None, E=0.7, rho0=1.0, gamma=GAM):
    """Unit-box initial mesh x0; current x = A x0; v = vfun(x); e = E; rho0|J0| = rho0 h^d."""
    m = synth.box_mesh(dim, k, N)
    m.mat_gamma = np.array([gamma])
    A = np.eye(dim) if A is None else np.asarray(A, dtype=float)
    x = np.ascontiguousarray(A @ m.x0)
    v = np.zeros_like(x) if vfun is None else np.ascontiguousarray(vfun(x))
    e = np.full((m.num_zones, m.nt), E)
    R = np.full((m.num_zones, m.nq), rho0 * np.prod(m.h))
    return m, synth.State(x, v, e, R)


def assemble_uniform(m, zone_vec):
    """numpy assembly of the same zone vector [dim][nk] into every zone's nodes."""
    out = np.zeros((m.dim, m.num_nodes))
    for c in range(m.dim):
        np.add.at(out[c], m.zone_nodes.ravel(), np.tile(zone_vec[c], m.num_zones))
    return out


def zone_F1_uniform_stress(dim, k, J, sigma):
    """(F_z 1)_{c,a} = sum_d (sigma adj(J)^T)_{cd} int dW_a/dxi_d for constant J and sigma."""
    # nanson_F1 gives -p * sum_d adj_{dc} (...): linear in the matrix M = sigma adj(J)^T with sigma = -p I.
    # For a general constant sigma use the unit-pressure version per column.
    adjJ = np.linalg.det(J) * np.linalg.inv(J)
    M = sigma @ adjJ.T
    _, w = gll01(k)
    nk = (k + 1) ** dim
    out = np.zeros((dim, nk))
    for a in range(nk):
        ai = [(a // (k + 1) ** t) % (k + 1) for t in range(dim)]
        for d in range(dim):
            jump = (1.0 if ai[d] == k else 0.0) - (1.0 if ai[d] == 0 else 0.0)
            if jump == 0.0:
                continue
            wt = np.prod([w[ai[t]] for t in range(dim) if t != d])
            out[:, a] += M[:, d] * jump * wt
    return out


def rel(a, b):
    return np.abs(a - b).max() / max(np.abs(b).max(), 1e-300)


# ------------------------------------------------------------------------------------------------
@pytest.mark.parametrize("dim", [2, 3])
@pytest.mark.parametrize("k", [1, 2, 3, 4])
def test_affine_volume(orc, dim, k):
    """sum_q alpha_q det J = |zone| on an affine (sheared) zone (det J is the local volume)."""
    A = np.array([[1.5, 0.4, 0.1], [-0.3, 1.2, 0.2], [0.05, -0.1, 0.9]])[:dim, :dim]
    m = synth.box_mesh(dim, k, (1,) * dim)
    x = A @ m.x0 + 0.3
    assert abs(orc.volume(dim, k, m.zone_nodes, x) - np.linalg.det(A)) < 1e-14 * np.linalg.det(A)


@pytest.mark.parametrize("name,N", [("C1", None), ("C3", (4, 4, 4)), ("C5", (6, 3, 3))])
def test_curved_mesh_total_volume(orc, name, N):
    """Fixed-boundary curved S1 meshes keep the domain volume exactly (det J has degree <= 3k-1 <= 4k-1)."""
    m, s = synth.config(name, "S1", N=N, k=2 if name == "C5" else None)
    vol = float(np.prod(m.L))
    assert abs(orc.volume(m.dim, m.order, m.zone_nodes, s.x) - vol) < 1e-14 * vol


@pytest.mark.parametrize("dim", [2, 3])
@pytest.mark.parametrize("k", [1, 2, 3, 4, 5])
def test_nanson_sheared_zone(orc, dim, k):
    """Uniform pressure on one sheared zone, v = 0: F_z.1 = -p sum_faces adj(J)^T N ∫_face W_a (R6, R12)."""
    A = np.array([[1.5, 0.4, 0.2], [-0.3, 1.2, 0.1], [0.1, 0.25, 0.8]])[:dim, :dim]
    m, s = uniform_case(dim, k, (1,) * dim, A=A, E=0.7, rho0=1.3)
    r = orc.evaluate(m, s)
    detJ = np.linalg.det(A)              # J = A h with h = 1
    p = (GAM - 1.0) * 1.3 / detJ * 0.7
    expect = nanson_F1(dim, k, A, p)
    assert rel(r.Fz1[0], expect) < 1e-14
    assert np.abs(r.FTv).max() == 0.0     # v = 0 => F^T v = 0 exactly
    # the test discriminates the transpose: with adj(J) (not adj(J)^T) the answer is far off
    wrong = nanson_F1(dim, k, A.T, p * detJ / np.linalg.det(A.T))
    assert rel(wrong, expect) > 1e-2


@pytest.mark.parametrize("dim,k,N", [(2, 2, (3, 4)), (2, 3, (2, 2)), (3, 2, (2, 2, 2)), (3, 3, (2, 1, 2))])
def test_uniform_pressure_closed_mesh(orc, dim, k, N):
    """Undeformed mesh, uniform p, v = 0: interior F.1 = 0, boundary face totals = p * face area, sum F.1 = 0."""
    m, s = uniform_case(dim, k, N, E=0.9)
    r = orc.evaluate(m, s)
    p = (GAM - 1.0) * 1.0 * 0.9
    F1 = r.F1
    X = m.x0
    onb = np.zeros(m.num_nodes, bool)
    for t in range(dim):
        onb |= (np.abs(X[t]) < 1e-14) | (np.abs(X[t] - 1.0) < 1e-14)
    assert np.abs(F1[:, ~onb]).max() < 1e-15
    assert np.abs(F1.sum(1)).max() < 1e-15
    for t in range(dim):
        lo = np.abs(X[t]) < 1e-14
        hi = np.abs(X[t] - 1.0) < 1e-14
        # (F.1)_t summed over the x_t = 0 face = +p * area (area of the unit face = 1); x_t = 1 face: -p
        assert abs(F1[t, lo].sum() - p) < 1e-14
        assert abs(F1[t, hi].sum() + p) < 1e-14
    # node-by-node: assembled closed form of every zone
    J = np.diag(m.h)
    expect = assemble_uniform(m, zone_F1_uniform_stress(dim, k, J, -p * np.eye(dim)))
    assert np.abs(F1 - expect).max() < 1e-15


@pytest.mark.parametrize("name,N,expect_dt", [
    ("C1", None, 0.018559808466140585),
    ("C2", None, 3.624962591043083e-05),
    ("C3", None, 5.1264712593482434e-05),
    ("C4", None, 2.5632356296741217e-05),
])
def test_sedov_s0_closed_form(orc, name, N, expect_dt):
    """Sedov IC: only the origin zone has e > 0, so dt_min, F^T v = 0 and F.1 follow in closed form.
    dt_min = cfl h / (2.25 k c_s), c_s = sqrt(gamma(gamma-1) E_b/(rho0 h^d)) (R8, R10)."""
    m, s = synth.config(name, "S0", N=N)
    dim, k, h = m.dim, m.order, m.h[0]
    e0 = 0.25 / h ** dim
    cs = np.sqrt(GAM * (GAM - 1.0) * e0)
    dt = 0.5 * h / (2.25 * k * cs)
    assert abs(dt - expect_dt) < 4e-16 * expect_dt
    # the origin zone and its neighbours (enough for every node of zone 0): cheap subset evaluation,
    # h0 given in closed form h/k for the uniform mesh
    params = orc.Params(h0=h / k)
    zones = sorted({ix + m.N[0] * (iy + m.N[1] * iz) for ix in (0, 1) for iy in (0, 1)
                    for iz in ((0, 1) if dim == 3 else (0,))})
    r = orc.evaluate(m, s, params=params, zones=zones)
    assert abs(r.dt_min - dt) < 2e-14 * dt
    assert np.abs(r.FTv).max() == 0.0
    p = (GAM - 1.0) * e0
    expect = zone_F1_uniform_stress(dim, k, np.diag(m.h), -p * np.eye(dim))
    assert rel(r.Fz1[0], expect) < 1e-14
    assert np.abs(r.Fz1[1:]).max() == 0.0


@pytest.mark.parametrize("dim,k", [(2, 1), (2, 2), (2, 4), (3, 2), (3, 3)])
def test_dt_at_rest(orc, dim, k):
    """Undeformed, v = 0, uniform e: dt = cfl h / (2.25 k c_s); the 2.25 = 1 + 2.5 * 1/2 (linear term,
    psi0 = 1 at rest, switch on at lambda = 0)."""
    m, s = uniform_case(dim, k, (2,) * dim, E=0.3)
    r = orc.evaluate(m, s)
    h = m.h[0]
    cs = np.sqrt(GAM * (GAM - 1) * 0.3)
    assert abs(r.dt_min - 0.5 * h / (2.25 * k * cs)) < 2e-14 * r.dt_min
    assert abs(orc.h0_of(m) - h / k) < 1e-15


@pytest.mark.parametrize("dim,k", [(2, 2), (2, 3), (3, 2)])
@pytest.mark.parametrize("beta", [0.37, 2e-12])
def test_uniform_expansion(orc, dim, k, beta):
    """v = beta x on the undeformed mesh: sigma = (-p + mu beta) I with
    mu = 2 rho h0^2 beta + 1/2 rho h0 c_s sqrt(d) (1 - smoothstep(beta - 2 eps, eps));
    (F^T v)_j = tr(sigma) beta |zone| / k^d;  dt = cfl / (c_s k/h + 2.5 mu / (rho h0^2))."""
    E = 0.45
    m, s = uniform_case(dim, k, (2,) * dim, vfun=lambda x: beta * x, E=E)
    r = orc.evaluate(m, s)
    h = m.h[0]
    h0 = h / k
    rho = 1.0
    cs = np.sqrt(GAM * (GAM - 1) * E)
    p = (GAM - 1) * rho * E
    eps = 1e-12
    y = (beta - 2 * eps + eps) / (2 * eps)
    sm = 0.0 if y < 0 else 1.0 if y > 1 else (3 - 2 * y) * y * y
    mu = 2 * rho * h0 ** 2 * abs(beta) + 0.5 * rho * h0 * cs * np.sqrt(dim) * (1 - sm)
    sig = -p + mu * beta
    zone_vol = h ** dim
    ftv = dim * sig * beta * zone_vol / k ** dim
    assert np.abs(r.FTv - ftv).max() < 1e-13 * abs(ftv) + 1e-30
    dt = 0.5 / (cs / h0 + 2.5 * mu / (rho * h0 ** 2))
    assert abs(r.dt_min - dt) < 1e-14 * dt
    expect = assemble_uniform(m, zone_F1_uniform_stress(dim, k, np.diag(m.h), sig * np.eye(dim)))
    assert np.abs(r.F1 - expect).max() < 1e-14 * np.abs(expect).max()


@pytest.mark.parametrize("dim,k", [(2, 2), (2, 3), (3, 2)])
def test_stretched_mesh_compression(orc, dim, k):
    """x = A x0 with A = diag(a), v = (-beta x_1, 0, ...): lambda_min = -beta with s = e_1, psi0 = 1,
    l = h0 |A e_1| = h0 a_1 (J J0^-1 = A), rho = rho0 / det A, h_min = h min(a) / k."""
    a = np.array([1.6, 0.7, 1.2])[:dim]
    beta = 0.8
    E = 0.6

    def vf(x):
        v = np.zeros_like(x)
        v[0] = -beta * x[0]
        return v

    m, s = uniform_case(dim, k, (2,) * dim, A=np.diag(a), vfun=vf, E=E)
    r = orc.evaluate(m, s)
    h = m.h[0]
    h0 = h / k
    rho = 1.0 / np.prod(a)
    cs = np.sqrt(GAM * (GAM - 1) * E)
    p = (GAM - 1) * rho * E
    ell = h0 * a[0]
    mu = 2 * rho * ell ** 2 * beta + 0.5 * rho * ell * cs
    sigma = -p * np.eye(dim)
    sigma[0, 0] += mu * (-beta)
    ftv = (p * beta + mu * beta ** 2) * h ** dim * np.prod(a) / k ** dim
    assert np.abs(r.FTv - ftv).max() < 1e-13 * abs(ftv)
    hmin = h * a.min() / k
    dt = 0.5 / (cs / hmin + 2.5 * mu / rho / hmin ** 2)
    assert abs(r.dt_min - dt) < 1e-14 * dt
    expect = assemble_uniform(m, zone_F1_uniform_stress(dim, k, np.diag(a * h), sigma))
    assert np.abs(r.F1 - expect).max() < 1e-14 * np.abs(expect).max()
    assert r.diag["min_gap"] > 0.5


@pytest.mark.parametrize("dim,k", [(2, 2), (3, 2)])
def test_shear_flow(orc, dim, k):
    """v = (g y, 0, ...): div v = 0 => psi0 = 0; lambda_min = -g/2; mu = rho h0^2 g;
    (F^T v)_j = mu g^2/2 |zone| / k^d; dt = cfl / (c_s k/h + 2.5 g)."""
    g = 0.9
    E = 0.5

    def vf(x):
        v = np.zeros_like(x)
        v[0] = g * x[1]
        return v

    m, s = uniform_case(dim, k, (2,) * dim, vfun=vf, E=E)
    r = orc.evaluate(m, s)
    h = m.h[0]
    h0 = h / k
    cs = np.sqrt(GAM * (GAM - 1) * E)
    mu = 1.0 * h0 ** 2 * g
    ftv = mu * g * g / 2 * h ** dim / k ** dim
    assert np.abs(r.FTv - ftv).max() < 1e-12 * abs(ftv)
    dt = 0.5 / (cs * k / h + 2.5 * g)
    assert abs(r.dt_min - dt) < 1e-13 * dt


def test_rigid_rotation(orc):
    """v = w(-y, x): eps = 0 and div v = 0 => mu = 0, F^T v = 0, dt = cfl h / (k c_s)."""
    w = 1.3
    E = 0.5
    m, s = uniform_case(2, 3, (3, 3), vfun=lambda x: np.stack([-w * x[1], w * x[0]]), E=E)
    r = orc.evaluate(m, s)
    p = (GAM - 1) * E
    scale = p * w * m.h[0] ** 2
    assert np.abs(r.FTv).max() < 1e-14 * scale
    cs = np.sqrt(GAM * (GAM - 1) * E)
    dt = 0.5 * m.h[0] / (3 * cs)
    assert abs(r.dt_min - dt) < 1e-12 * dt


@pytest.mark.parametrize("dim,k", [(2, 2), (2, 3), (3, 2)])
def test_length_scale_orientation(orc, dim, k):
    """l = h0 |J J0^-1 s| (reading R8) with a SHEARED initial zone and a differently sheared current zone.

    Initial nodes X = A0 xi (A0 non-diagonal), current x = A1 xi, so J0 = A0 h, J = A1 h and the
    deformation gradient J J0^-1 = A1 A0^-1 =: Fd.  v = B x with B symmetric (distinct eigenvalues):
    grad v = B exactly (isoparametric affine field), eps = B, (lambda, s) = its smallest eigenpair
    (numpy eigh).  e = 0 => p = 0, c_s = 0, so mu = q_quad rho l^2 |lambda| alone and
        dt = cfl h_min^2 / (2.5 q_quad l^2 |lambda|),  h_min = sigma_min(J) / k   (numpy svd),
        (F^T v)_j = mu (B : B) det J / k^d,  F_z.1 = Nanson with sigma = mu B.
    The transposed / reversed products (J0^-1 J, (J J0^-1)^T, J^T J0^-T) give |. s| values that differ by
    more than 1e-3 here (asserted), so a wrong orientation fails."""
    A0 = np.array([[1.1, 0.35, -0.2], [0.15, 0.9, 0.25], [-0.1, 0.3, 1.2]])[:dim, :dim]
    A1 = np.array([[1.4, -0.45, 0.3], [0.5, 0.8, -0.15], [0.2, 0.1, 0.7]])[:dim, :dim]
    th = 0.7
    Q = np.eye(dim)
    Q[:2, :2] = [[np.cos(th), -np.sin(th)], [np.sin(th), np.cos(th)]]
    if dim == 3:
        R2 = np.array([[1, 0, 0], [0, np.cos(0.4), -np.sin(0.4)], [0, np.sin(0.4), np.cos(0.4)]])
        Q = R2 @ Q
    B = Q @ np.diag([-0.9, 0.2, 0.6][:dim]) @ Q.T
    m = synth.box_mesh(dim, k, (1,) * dim)
    box = m.x0.copy()
    m.x0 = np.ascontiguousarray(A0 @ box)
    x = np.ascontiguousarray(A1 @ box + 0.2)
    v = np.ascontiguousarray(B @ x)
    e = np.zeros((1, m.nt))
    R = np.full((1, m.nq), np.linalg.det(A0))       # rho0 = 1
    h0 = 0.13
    r = orc.evaluate(m, synth.State(x, v, e, R), params=orc.Params(h0=h0))
    lam, V = np.linalg.eigh(B)
    s = V[:, 0]
    Fd = A1 @ np.linalg.inv(A0)
    ell = h0 * np.linalg.norm(Fd @ s)
    for wrong in (np.linalg.inv(A0) @ A1, Fd.T, A1.T @ np.linalg.inv(A0).T):
        assert abs(h0 * np.linalg.norm(wrong @ s) - ell) > 1e-3 * ell
    rho = np.linalg.det(A0) / np.linalg.det(A1)
    mu = 2.0 * rho * ell ** 2 * abs(lam[0])
    hmin = np.linalg.svd(A1, compute_uv=False).min() / k
    dt = 0.5 * hmin ** 2 / (2.5 * 2.0 * ell ** 2 * abs(lam[0]))
    assert abs(r.dt_min - dt) < 1e-13 * dt, (r.dt_min, dt)
    ftv = mu * (B * B).sum() * np.linalg.det(A1) / k ** dim
    assert np.abs(r.FTv - ftv).max() < 1e-13 * abs(ftv)
    expect = zone_F1_uniform_stress(dim, k, A1, mu * B)[:, :]
    assert np.abs(r.Fz1[0] - expect).max() < 1e-13 * np.abs(expect).max()
