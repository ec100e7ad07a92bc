"""GPU parity of the time integrator (blast_cf_rk2_* in include/blast_cf.h) against
oracle/integrator.py on the same seeded inputs.

Tolerances:
* M_V u, energies, M_E^{-1} F^T Vbar: no solver involved -> 1e-13 (M_V u) / 1e-12 (F^T path, the
  corner-force bar);
* dv/dt = -M_V^{-1} F.1 and full steps: both sides run CG to ||r|| <= 1e-15 ||b||, so each is within
  cond(M_V) * 1e-15 of the exact solve; cond(M_V) <= 4e3 for k <= 8 (Jacobi-preconditioned far less)
  -> 1e-11;
* conservation: |E_n - E_0| <= 1e-12 E_0 over 20 steps (Table 6; E_0 = 10.05 for
  the triple point).
"""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


def _torch():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def _setup(mesh, st, R=None, **opts):
    torch = _torch()
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    h = cf.from_synth(mesh)
    R = st.rho0detJ0 if R is None else R
    opts.setdefault("cg_rel_tol", 1e-15)
    rk = cf.RK2(h, R, **opts)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    return rk, t


def rel(a, b):
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-300))


CASES = [("sedov", 2, 1, (7, 5)), ("sedov", 2, 3, (6, 5)), ("triple", 2, 4, (7, 3)), ("sedov", 2, 8, (2, 2)),
         ("sedov", 3, 1, (4, 3, 3)), ("sedov", 3, 2, (3, 3, 2)), ("triple", 3, 3, (4, 2, 2)), ("sedov", 3, 4, (2, 2, 2))]


@pytest.mark.parametrize("kind,dim,k,N", CASES)
def test_mass_apply_and_energy(orc, kind, dim, k, N):
    from oracle import integrator as it
    m = synth.make_mesh(kind, dim, k, N)
    s = synth.make_state(m, kind, "S1", 7)
    rk, t = _setup(m, s)
    M = it.mass_matrices(m, s.rho0detJ0)
    u = np.random.default_rng(11).standard_normal((dim, m.num_nodes))
    got = rk.mass_apply(t(u)).cpu().numpy()
    ref = np.stack([M.MV @ u[c] for c in range(dim)])
    assert rel(got, ref) < 1e-13
    ke, ie = rk.energy(t(s.v), t(s.e))
    ke0, ie0 = it.energies(M, s.v, s.e)
    assert abs(ke - ke0) < 1e-13 * ke0 and abs(ie - ie0) < 1e-13 * ie0


@pytest.mark.parametrize("kind,dim,k,N", CASES)
def test_rates_parity(orc, kind, dim, k, N):
    from oracle import integrator as it
    m = synth.make_mesh(kind, dim, k, N)
    s = synth.make_state(m, kind, "S1", 5)
    rk, t = _setup(m, s)
    vbar = s.v + 0.1 * np.random.default_rng(2).standard_normal(s.v.shape)
    dv, de, dt, iters = rk.rates(t(s.x), t(s.v), t(s.e), t(vbar))
    o = it.RK2Avg(m, s.rho0detJ0)
    r = o.forces(s.x, s.v, s.e)
    dv0, _ = o.accel(r.F1)
    de0 = o.de_dt(r, vbar)
    assert rel(dv.cpu().numpy(), dv0) < 1e-11
    _check_de(o, r, vbar, de.cpu().numpy(), de0)
    assert abs(dt - r.dt_min) <= 1e-12 * r.dt_min
    assert 0 < iters < 500


def _check_de(o, r, vbar, de, de0):
    """de = M_E^{-1} F^T Vbar.  Backward error (residual of the block solve) at the corner-force bar;
    forward error bounded by cond(M_E) * eps (the Bernstein mass matrix of degree k-1 in dim d has
    cond ~ 1e2 (2D k=3) .. 4e7 (2D k=8): DESIGN.md §8)."""
    Z = de.shape[0]
    Vz = vbar[:, o.mesh.zone_nodes].transpose(1, 0, 2).reshape(Z, -1)
    FTV = np.einsum("zij,zi->zj", r.Fz, Vz)
    res = np.einsum("zij,zj->zi", o.masses.ME, de) - FTV
    cond = max(np.linalg.cond(o.masses.ME[z]) for z in range(min(Z, 4)))
    # An explicit inverse is not backward stable: fl(M^-1) b has residual up to ~cond(M) eps |b|, so the
    # residual bar is 1e-12 only while cond(M_E) eps stays below it (zone-constant rho0|J0|: the tensor
    # path; the per-point rho0|J0| of the S1 states takes the dense per-zone inverse, cond up to 4e7 at
    # 2D k = 8).
    assert np.abs(res).max() < max(1e-12, 20 * cond * 2.2e-16) * np.abs(FTV).max(), cond
    assert rel(de, de0) < max(1e-12, 20 * cond * 2.2e-16), (rel(de, de0), cond)


def test_rates_dense_minv_nonuniform_density(orc):
    """rho0|J0| varying inside the zones: M_E^{-1} takes the dense per-zone path."""
    from oracle import integrator as it
    m = synth.box_mesh(2, 3, (5, 4))
    s = synth.sedov_s1(m, 3)
    R = s.rho0detJ0 * (1.0 + 0.2 * np.sin(np.arange(m.nq) * 0.7))[None, :] * (1.0 + 0.1 * np.arange(m.num_zones))[:, None]
    R = np.ascontiguousarray(R)
    rk, t = _setup(m, s, R=R)
    dv, de, dt, _ = rk.rates(t(s.x), t(s.v), t(s.e))
    o = it.RK2Avg(m, R)
    r = o.forces(s.x, s.v, s.e)
    dv0, _ = o.accel(r.F1)
    assert rel(dv.cpu().numpy(), dv0) < 1e-11
    _check_de(o, r, s.v, de.cpu().numpy(), o.de_dt(r, s.v))


@pytest.mark.parametrize("kind,dim,k,N,which", [("triple", 2, 3, (14, 6), "S0"), ("sedov", 2, 4, (5, 5), "S1"),
                                                 ("sedov", 3, 2, (3, 3, 3), "S0"), ("triple", 3, 2, (6, 3, 3), "S1")])
def test_step_parity(orc, kind, dim, k, N, which):
    from oracle import integrator as it
    m = synth.make_mesh(kind, dim, k, N)
    s = synth.make_state(m, kind, which, 9)
    rk, t = _setup(m, s)
    o = it.RK2Avg(m, s.rho0detJ0)
    x, v, e = t(s.x), t(s.v), t(s.e)
    ox, ov, oe = s.x, s.v, s.e
    dt = 0.5 * o.forces(ox, ov, oe).dt_min
    for _ in range(2):
        dte, _ = rk.step(x, v, e, dt)
        ox, ov, oe, odte = o.step(ox, ov, oe, dt)
        assert abs(dte - odte) <= 1e-11 * odte
    assert rel(x.cpu().numpy() - s.x, ox - s.x) < 1e-11
    assert rel(v.cpu().numpy(), ov) < 1e-11
    assert rel(e.cpu().numpy(), oe) < 1e-11


@pytest.mark.parametrize("kind,dim,k,N", [("triple", 2, 3, (14, 6)), ("sedov", 3, 2, (4, 4, 4)),
                                           ("sedov", 3, 4, (3, 3, 3))])
def test_energy_conservation(orc, kind, dim, k, N):
    m = synth.make_mesh(kind, dim, k, N)
    s = synth.make_state(m, kind, "S0", 1)
    rk, t = _setup(m, s, cg_rel_tol=1e-14)
    x, v, e = t(s.x), t(s.v), t(s.e)
    ke0, ie0 = rk.energy(v, e)
    E0 = ke0 + ie0
    if kind == "triple":
        assert abs(E0 - 10.05) < 1e-12          # Table 6 initial total energy
    else:
        assert abs(E0 - synth.E_BLAST) < 1e-14
    _, _, dt0 = rk.cf.eval(x, v, e, t(s.rho0detJ0))
    tr, dt, steps, rej = rk.advance(x, v, e, 1.0, 0.5 * float(dt0.cpu()[0]), 20)
    assert steps == 20
    ke, ie = rk.energy(v, e)
    assert ke > 1e-3 * E0
    assert abs(ke + ie - E0) <= 1e-12 * E0, (ke, ie, E0)


def test_step_is_deterministic(orc):
    m = synth.box_mesh(3, 2, (4, 3, 3))
    s = synth.sedov_s1(m, 4)
    outs = []
    for _ in range(2):
        rk, t = _setup(m, s)
        x, v, e = t(s.x), t(s.v), t(s.e)
        for _ in range(3):
            rk.step(x, v, e, 1e-3)
        outs.append((x.cpu().numpy(), v.cpu().numpy(), e.cpu().numpy()))
    for a, b in zip(*outs):
        assert np.array_equal(a, b)


def test_quiescent_box_gpu(orc):
    m = synth.box_mesh(3, 3, (2, 2, 3))
    R = np.ascontiguousarray(np.ones((m.num_zones, m.nq)) * np.prod(m.h))
    e0 = np.full((m.num_zones, m.nt), 2.0)
    st = synth.State(m.x0.copy(), np.zeros_like(m.x0), e0, R)
    rk, t = _setup(m, st)
    x, v, e = t(st.x), t(st.v), t(st.e)
    for _ in range(3):
        rk.step(x, v, e, 1e-2)
    assert float(v.abs().max()) < 1e-13 and float((e - 2.0).abs().max()) < 1e-13


def test_loopback_integrator_needs_global_box(orc):
    """A loopback rank cannot find the global walls by itself (no collective at create): EINVAL."""
    torch = _torch()
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    import oracle
    m = synth.box_mesh(2, 2, (4, 2))
    parts = synth.partition(m, 2)
    p = cf.default_params()
    p.h0 = oracle.h0_of(m)
    h = cf.from_synth(m, p, part=parts[0])
    s = synth.sedov_s0(m)
    with pytest.raises(cf.BlastCFError):
        cf.RK2(h, np.ascontiguousarray(s.rho0detJ0[parts[0].zones]))


@pytest.mark.parametrize("kind,dim,k,N", [("sedov", 2, 3, (5, 5)), ("sedov", 3, 4, (2, 2, 2))])
def test_advance_parity(orc, kind, dim, k, N):
    """Same accept / reject decisions and trajectory as the oracle's controller (reading R24)."""
    from oracle import integrator as it
    m = synth.make_mesh(kind, dim, k, N)
    s = synth.make_state(m, kind, "S0", 1)
    rk, t = _setup(m, s)
    o = it.RK2Avg(m, s.rho0detJ0)
    dt0 = 0.5 * o.forces(s.x, s.v, s.e).dt_min
    x, v, e = t(s.x), t(s.v), t(s.e)
    tr, dt, steps, rej = rk.advance(x, v, e, 1.0, dt0, 8)
    ox, ov, oe, otr, odt, osteps, orej = o.advance(s.x, s.v, s.e, 1.0, dt0, 8)
    assert (steps, rej) == (osteps, orej)
    assert abs(tr - otr) <= 1e-11 * otr
    assert rel(v.cpu().numpy(), ov) < 1e-10
    assert rel(e.cpu().numpy(), oe) < 1e-10
