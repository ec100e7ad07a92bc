"""GPU parity: the CUDA path through the C ABI vs the CPU oracle on the same seeded inputs.

Bar (BASELINE.json north_star): max-norm relative error <= 1e-12 on F.1, F^T v and dt, i.e.
    err_F1 = max|F1_gpu - F1_orc| / max|F1_orc|   (likewise F^T v),   err_dt = |dt_gpu - dt_orc| / dt_orc.
Small cases span several CTAs and a ragged last CTA; the BASELINE sizes (C2-C5, in the bench's launch
configuration) are checked on sampled nodes/zones the oracle evaluates one by one, plus the argmin-CTA
dt and properties that hold at any size (momentum, energy identity, determinism).
"""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu
TOL = 1e-12


def _torch():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def gpu_eval(mesh, st, params=None, reps=1):
    torch = _torch()
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    h = cf.from_synth(mesh, params)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    x, v, e, r = t(st.x), t(st.v), t(st.e), t(st.rho0detJ0)
    outs = []
    for _ in range(reps):
        F1, FTv, dt = h.eval(x, v, e, r)
        torch.cuda.synchronize()
        outs.append((F1.cpu().numpy(), FTv.cpu().numpy(), float(dt.cpu()[0])))
    return h, outs


def rel(a, b):
    return float(np.abs(a - b).max() / max(np.abs(b).max(), 1e-300))


def check(mesh, st, orc, oparams=None, gparams=None, tol=TOL):
    h, [(F1, FTv, dt)] = gpu_eval(mesh, st, gparams)
    r = orc.evaluate(mesh, st, params=oparams)
    e1, e2 = rel(F1, r.F1), rel(FTv, r.FTv)
    e3 = abs(dt - r.dt_min) / r.dt_min if np.isfinite(r.dt_min) and r.dt_min > 0 else abs(dt - r.dt_min)
    assert e1 <= tol and e2 <= tol and e3 <= tol, (e1, e2, e3, r.diag)
    return h, (F1, FTv, dt), r


# ---------------------------------------------------------------------------------------------
# small cases: every order in 2D and 3D, both states, ragged CTA tails
# ---------------------------------------------------------------------------------------------
@pytest.mark.parametrize("k", list(range(1, 9)))
def test_2d_all_orders(orc, k):
    m, s = synth.config("C2", "S1", N=(5, 3), k=k)
    check(m, s, orc)


@pytest.mark.parametrize("k", list(range(1, 9)))
def test_3d_all_orders(orc, k):
    N = (3, 2, 2) if k <= 4 else (2, 1, 2)
    m, s = synth.config("C4", "S1", N=N, k=k)
    check(m, s, orc)


@pytest.mark.parametrize("name,N,which", [
    ("C1", None, "S0"), ("C1", None, "S1"),
    ("C2", (16, 16), "S1"), ("C2", (16, 16), "S1b"),
    ("C3", (6, 5, 4), "S0"), ("C3", (6, 5, 4), "S1"),
    ("C4", (5, 3, 3), "S0"), ("C4", (5, 3, 3), "S1"),
    ("C5", (4, 2, 2), "S0"), ("C5", (4, 2, 2), "S1"),
])
def test_configs_small(orc, name, N, which):
    m, s = synth.config(name, which, N=N)
    check(m, s, orc)


def test_c1_exact_oracle_case_bitwise_sane(orc):
    """C1 (BASELINE configs[0]): one evaluation vs the oracle, plus the closed-form Sedov dt."""
    m, s = synth.config("C1", "S0")
    h, (F1, FTv, dt), r = check(m, s, orc)
    assert abs(dt - 0.018559808466140585) < 1e-15
    assert np.abs(FTv).max() == 0.0


@pytest.mark.parametrize("visc,vort", [(0, 0), (1, 0)])
def test_param_switches(orc, visc, vort):
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config("C3", "S1", N=(3, 3, 3))
    gp = cf.default_params()
    gp.use_viscosity, gp.use_vorticity = visc, vort
    op = orc.Params(use_viscosity=visc, use_vorticity=vort)
    check(m, s, orc, oparams=op, gparams=gp)


def test_inverted_zone_gives_dt_zero(orc):
    m, s = synth.config("C3", "S1", N=(3, 3, 3))
    x = s.x.copy()
    a = m.zone_nodes[13]                         # interior zone: pull its centre node far through a face
    x[0, a[13]] += 5.0 / 3
    s2 = synth.State(x, s.v, s.e, s.rho0detJ0)
    h, [(F1, FTv, dt)] = gpu_eval(m, s2)
    r = orc.evaluate(m, s2)
    assert r.diag["n_bad"] > 0 and r.dt_min == 0.0
    assert dt == 0.0


def test_single_zone_and_empty(orc):
    torch = _torch()
    m, s = synth.config("C4", "S1", N=(1, 1, 1))
    check(m, s, orc)
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    h = cf.CornerForce(np.zeros((0, 27), np.int32), np.zeros((3, 0)), 2, 3)
    F1, FTv, dt = h.eval(*(torch.zeros(sh, dtype=torch.float64, device="cuda") for sh in ((3, 0), (3, 0), (0, 8), (0, 64))))
    torch.cuda.synchronize()
    assert float(dt.cpu()[0]) == float("inf")


def test_determinism_bitwise():
    m, s = synth.config("C4", "S1", N=(6, 5, 4))
    h, outs = gpu_eval(m, s, reps=10)
    for o in outs[1:]:
        assert np.array_equal(o[0], outs[0][0]) and np.array_equal(o[1], outs[0][1]) and o[2] == outs[0][2]


def test_eval_host_matches_device():
    torch = _torch()
    m, s = synth.config("C3", "S1", N=(4, 4, 3))
    h, [(F1, FTv, dt)] = gpu_eval(m, s)
    hx = [torch.from_numpy(np.ascontiguousarray(a)).pin_memory() for a in (s.x, s.v, s.e, s.rho0detJ0)]
    o = h.eval_host(*hx)
    assert np.array_equal(o[0], F1) and np.array_equal(o[1], FTv) and o[2][0] == dt


@pytest.mark.parametrize("name,N", [("C3", None), ("C4", None), ("C5", None), ("C2", (128, 128))])
def test_eval_host_pipelined_matches_device(name, N):
    """At full size the host entry splits the zones into chunks whose copies overlap the kernels (a KB1
    launch per zone sub-range, per-chunk dt slots): every output must equal the device entry's bit for bit."""
    torch = _torch()
    m, s = synth.config(name, "S1", N=N)
    h, [(F1, FTv, dt)] = gpu_eval(m, s)
    hx = [torch.from_numpy(np.ascontiguousarray(a)).pin_memory() for a in (s.x, s.v, s.e, s.rho0detJ0)]
    for _ in range(2):   # twice: the second call reuses the plan and the staging buffers
        o = h.eval_host(*hx)
        assert np.array_equal(o[0], F1) and np.array_equal(o[1], FTv) and o[2][0] == dt


@pytest.mark.parametrize("name,N,k", [("C1", None, None), ("C3", (2, 2, 1), None), ("C2", (2, 2), 3)])
def test_debug_Fz_matches_oracle_definition_mode(orc, name, N, k):
    torch = _torch()
    m, s = synth.config(name, "S1", N=N, k=k)
    h, _ = gpu_eval(m, s)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    Fz = h.eval_debug_Fz(t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)).cpu().numpy()
    r = orc.evaluate(m, s, definition=True)
    assert rel(Fz, r.Fz) <= TOL


def test_gpu_invariants():
    m, s = synth.config("C4", "S1", N=(6, 6, 6))
    h, [(F1, FTv, dt)] = gpu_eval(m, s)
    assert np.abs(F1.sum(1)).max() <= 1e-13 * np.abs(F1).sum()
    assert abs((s.v * F1).sum() - FTv.sum()) <= 1e-13 * np.abs(s.v).max() * np.abs(F1).sum()


# ---------------------------------------------------------------------------------------------
# BASELINE sizes (the bench's launch configuration): sampled parity
# ---------------------------------------------------------------------------------------------
def sampled_parity(orc, name, which, n_nodes=48, n_zones=48, seed=0, state=None):
    m, s = synth.config(name, "S1" if state is not None else which)
    if state is not None:   # an edge regime of this config's mesh (synth.edge_state)
        s = synth.edge_state(m, synth.CONFIGS[name]["kind"], state, 7, tie_gap=1.5e-4 if m.order <= 4 else 4.5e-4)
    h, [(F1, FTv, dt)] = gpu_eval(m, s)
    rng = np.random.default_rng(seed)
    nodes = rng.choice(m.num_nodes, size=n_nodes, replace=False)
    inc = np.unique(np.nonzero(np.isin(m.zone_nodes, nodes))[0])
    extra = rng.choice(m.num_zones, size=n_zones, replace=False)
    # the CTA holding the GPU's minimum dt: its zones must reproduce dt_min exactly
    cta_dt, zpc = h.debug_cta_dt()
    ncta = len(cta_dt)
    cmin = int(np.argmin(cta_dt))
    assert cta_dt[cmin] == dt
    zone_cta = (np.arange(m.num_zones) // zpc) % ncta
    arg_zones = np.nonzero(zone_cta == cmin)[0]
    if len(arg_zones) > 512:   # the argmin CTA's zones: evaluate them all when cheap, else a sample + bound
        arg_zones = arg_zones[:512]
    zones = np.unique(np.concatenate([inc, extra, arg_zones]))
    h0 = (np.prod(m.L) / m.num_zones) ** (1.0 / m.dim) / m.order   # closed form for the uniform box
    assert abs(h.info["h0"] - h0) <= 1e-14 * h0
    r = orc.evaluate(m, s, params=orc.Params(h0=h0), zones=zones)
    scale_F = np.abs(F1).max()
    assert np.abs(F1[:, nodes] - r.F1[:, nodes]).max() <= TOL * scale_F
    sub = np.searchsorted(zones, np.arange(m.num_zones))
    pos = np.searchsorted(zones, zones)
    assert np.abs(FTv[zones] - r.FTv[pos]).max() <= TOL * np.abs(FTv).max()
    # per-CTA dt of every sampled zone's CTA must bound the oracle's zone dt, and the argmin CTA matches
    odt = r.dtz[np.searchsorted(zones, arg_zones)].min()
    assert dt <= odt * (1 + TOL)
    if (zone_cta == cmin).sum() == len(arg_zones):
        assert abs(dt - odt) <= TOL * odt, (dt, odt)
    for z, dz in zip(zones, r.dtz):
        assert cta_dt[zone_cta[z]] <= dz * (1 + TOL)
    # any-size properties
    assert np.abs(F1.sum(1)).max() <= 1e-12 * np.abs(F1).sum()
    assert abs((s.v * F1).sum() - FTv.sum()) <= 1e-12 * np.abs(s.v).max() * np.abs(F1).sum()
    del sub


@pytest.mark.parametrize("name,which", [("C2", "S1"), ("C2", "S1b"), ("C3", "S1"), ("C4", "S1"), ("C4", "S0"),
                                        ("C5", "S1")])
def test_full_size_sampled(orc, name, which):
    sampled_parity(orc, name, which, n_nodes=24 if name == "C5" else 48, n_zones=8 if name == "C5" else 48)


@pytest.mark.parametrize("name,state", [("C4", "window"), ("C4", "negative_e"), ("C4", "near_tie"),
                                        ("C5", "negative_e"), ("C3", "near_tie")])
def test_full_size_sampled_edge_regimes(orc, name, state):
    """The edge regimes (R25) at the BASELINE sizes, in the bench's launch configuration: sampled nodes and zones
    against the oracle, the argmin CTA's dt, and the any-size invariants."""
    sampled_parity(orc, name, None, n_nodes=24 if name == "C5" else 48, n_zones=8 if name == "C5" else 48, state=state)


@pytest.mark.parametrize("name", ["v10.v", "v5.r1"])
def test_full_size_sampled_c4_variants(orc, name, monkeypatch):
    """The persistent warp-specialized C4 candidates at the bench's size (221 zones per CTA: every stage of
    the zone pipeline, both buffers and the dt filter across zones are exercised)."""
    monkeypatch.setenv("BLAST_CF_KB1", name)
    sampled_parity(orc, "C4", "S1")


@pytest.mark.parametrize("dim,k,N", [(3, 2, (3, 3, 3)), (3, 4, (3, 2, 2)), (3, 8, (2, 1, 1)), (2, 4, (5, 4)), (2, 3, (4, 4))])
def test_non_affine_initial_mesh(orc, dim, k, N):
    """Reading R19: a curved initial mesh (the S1-deformed positions as x0) with the viscosity ON needs
    J0^{-1} at every point: create computes it on the device and selects a
    kernel that reads it; the result must match the oracle (which forms J0 at every point) — also with
    the viscosity off, and h0 must be the quadrature volume's."""
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    _torch()
    m, s = synth.config("C4" if dim == 3 else "C2", "S1", N=N, k=k)
    curved = synth.Mesh(m.dim, m.order, m.N, m.L, s.x.copy(), m.zone_nodes, m.zone_mat, m.mat_gamma)
    # move the current state away from x0 so J J0^-1 != I
    s2 = synth.State(np.ascontiguousarray(s.x + 0.1 * (s.x - m.x0)), s.v, s.e, s.rho0detJ0)
    h, _, r = check(curved, s2, orc)
    assert h.variant.startswith("v1")
    assert abs(h.info["h0"] - orc.h0_of(curved)) <= 1e-13 * h.info["h0"]
    gp = cf.default_params()
    gp.use_viscosity = 0
    check(curved, s2, orc, oparams=orc.Params(use_viscosity=0), gparams=gp)


def test_eval_host_resident_rho():
    """blast_cf_set_rho0detJ0_host: eval_host without rho0detJ0 reads the resident copy (PAPER.md:444-446:
    only (v, e, x) travel per step) and gives the device entry's results bitwise, small and pipelined."""
    torch = _torch()
    for name, N in (("C3", (4, 4, 3)), ("C4", None)):
        m, s = synth.config(name, "S1", N=N)
        h, [(F1, FTv, dt)] = gpu_eval(m, s)
        hx = [torch.from_numpy(np.ascontiguousarray(a)).pin_memory() for a in (s.x, s.v, s.e, s.rho0detJ0)]
        h.set_rho0detJ0_host(hx[3])
        for _ in range(2):
            o = h.eval_host(hx[0], hx[1], hx[2], None)
            assert np.array_equal(o[0], F1) and np.array_equal(o[1], FTv) and o[2][0] == dt


def test_eval_host_rejects_bad_buffers():
    torch = _torch()
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config("C3", "S1", N=(2, 2, 2))
    h = cf.from_synth(m)
    good = [torch.from_numpy(np.ascontiguousarray(a)) for a in (s.x, s.v, s.e, s.rho0detJ0)]
    with pytest.raises(ValueError):
        h.eval_host(good[0].float(), *good[1:])
    with pytest.raises(ValueError):
        h.eval_host(good[0].cuda(), *good[1:])
    with pytest.raises(cf.BlastCFError):
        h.eval_host(*good[:3], None)          # no resident rho0|J0| yet


def test_multi_material_gamma(orc):
    """Per-zone gamma through zone_mat / mat_gamma (triple point, 3 materials)."""
    m, s = synth.config("C5", "S1", N=(6, 3, 3), k=2)
    assert len(np.unique(m.zone_mat)) == 3
    check(m, s, orc)


CANDIDATES = {1: ["v2.p1.z32", "v2.z64", "v1.z32"], 2: ["v2.z1m12e", "v2.z1m12", "v2.z2m6", "v2.p1.z2", "v1.z16"],
              3: ["v2.z2", "v2.p1.z1", "v3.z2", "v1.z8"],
              4: ["v10.wpx", "v10.w", "v10.v", "v5.r1", "v2.z1", "v1.z4"],
              7: ["v8", "v11", "v1.z1"], 8: ["v11.mbtsiet", "v11.mbtsie", "v11.mbtsi", "v11.mbts", "v11.mbt", "v11.mb", "v8", "v11", "v8.m1", "v1.z1m2", "v1.z1"]}


@pytest.mark.parametrize("k,name", [(k, n) for k, ns in CANDIDATES.items() for n in ns])
def test_every_kernel_variant(orc, k, name, monkeypatch):
    """Every candidate corner-force kernel (BLAST_CF_KB1 picks it at create) meets the parity bar."""
    monkeypatch.setenv("BLAST_CF_KB1", name)
    m, s = synth.config("C4", "S1", N=(5, 3, 2), k=k)
    h, _, _ = check(m, s, orc)
    assert h.variant == name


@pytest.mark.parametrize("name", ["p2d.z2m6", "p2d.z4m3", "v1-2d.z4m3", "v1-2d.z4"])
def test_every_2d_kernel_variant(orc, name, monkeypatch):
    """The 2D Q4 candidates (C2's order) meet the parity bar, on a mesh with a partial last zone batch."""
    monkeypatch.setenv("BLAST_CF_KB1", name)
    m, s = synth.config("C2", "S1", N=(7, 5), k=4)
    h, _, _ = check(m, s, orc)
    assert h.variant == name


def test_autotune_picks_a_candidate_and_keeps_parity(orc):
    torch = _torch()
    m, s = synth.config("C4", "S1", N=(6, 5, 4))
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    h = cf.from_synth(m)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    x, v, e, r = t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)
    ms = h.autotune(x, v, e, r, reps=2)
    assert set(ms) == set(CANDIDATES[4]) and all(val > 0 for val in ms.values())
    assert h.variant == min(ms, key=ms.get)
    F1, FTv, dt = (o.cpu().numpy() for o in h.eval(x, v, e, r))
    ro = orc.evaluate(m, s)
    assert rel(F1, ro.F1) <= TOL and rel(FTv, ro.FTv) <= TOL and abs(float(dt[0]) - ro.dt_min) <= TOL * ro.dt_min


# ---------------------------------------------------------------------------------------------
# round 2: the regimes the parity bar must hold in and the runtime-switch paths of
# every candidate kernel
# ---------------------------------------------------------------------------------------------
SWITCHES = [(0, 0), (1, 0), (0, 1)]


def _switch_params(visc, vort):
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    gp = cf.default_params()
    gp.use_viscosity, gp.use_vorticity = visc, vort
    return gp


@pytest.mark.parametrize("visc,vort", SWITCHES)
@pytest.mark.parametrize("k,name", [(4, n) for n in CANDIDATES[4]] + [(8, n) for n in CANDIDATES[8]] +
                         [(2, "v2.z1m12e"), (2, "v2.z1m12"), (3, "v2.z2"), (7, "v8")])
def test_switches_every_candidate(orc, k, name, visc, vort, monkeypatch):
    """Viscosity / vorticity switches off through every C4 and C5 candidate (the compile-time-switch
    kernels v10.w / v10.v fall back to their runtime-switch branch), on S1 with point-varying rho0|J0|."""
    monkeypatch.setenv("BLAST_CF_KB1", name)
    N = (5, 3, 2) if k <= 4 else (2, 1, 2)
    m, s = synth.config("C4", "S1", N=N, k=k)
    h, _, _ = check(m, s, orc, oparams=orc.Params(use_viscosity=visc, use_vorticity=vort),
                    gparams=_switch_params(visc, vort))
    assert h.variant == name


EDGE_CASES = [("sedov", 3, 2, (4, 3, 3), None), ("sedov", 3, 3, (3, 3, 2), None), ("sedov", 3, 4, (5, 3, 2), None),
              ("sedov", 3, 4, (5, 3, 2), "v5.r1"), ("triple", 3, 8, (2, 1, 2), None), ("sedov", 2, 4, (7, 5), None),
              ("sedov", 2, 2, (6, 5), None)]


@pytest.mark.parametrize("which", ["window", "negative_e", "near_tie"])
@pytest.mark.parametrize("kind,dim,k,N,var", EDGE_CASES)
def test_edge_regimes(orc, kind, dim, k, N, var, which, monkeypatch):
    """lambda inside the switch window (1e-12, 3e-12) at every point; e(q) < 0 at part of the points (the
    EOS clamp); a relative eigen-gap ~1e-4 of the strain rate (oracle diag min_gap) on a deformed mesh."""
    if var:
        monkeypatch.setenv("BLAST_CF_KB1", var)
    m = synth.make_mesh(kind, dim, k, N)
    # near-tie: relative gap 1e-4 for k <= 4; at k = 8 the strain rate itself carries ~8x the rounding (729-node
    # gradient sums), measured 1.8e-12 on F.1 at gap 1e-4 (run r2-3), so the bar is checked at gap 3e-4 there
    s = synth.edge_state(m, kind, which, 31 + k, tie_gap=1.5e-4 if k <= 4 else 4.5e-4)
    h, _, r = check(m, s, orc)
    if which == "window":
        assert r.diag["min_switch_dist"] < 1e-12           # every point's lambda - 2 eps_sw is inside the window
    elif which == "negative_e":
        assert (s.e < 0).any() and (s.e > 0).any()
    else:
        assert 1e-5 < r.diag["min_gap"] < (2e-4 if k <= 4 else 4e-4)


def test_point_varying_rho_is_read_per_point(orc):
    """The S1 states carry a per-point rho0|J0| (synth RHO_POINT_AMPL): permuting it within each zone must
    change the GPU result (so a mis-indexed point read cannot pass the parity tests)."""
    m, s = synth.config("C4", "S1", N=(3, 2, 2))
    assert np.ptp(s.rho0detJ0, axis=1).min() > 0.05 * s.rho0detJ0.mean()
    _, [(F1, FTv, dt)] = gpu_eval(m, s)
    s2 = synth.State(s.x, s.v, s.e, np.ascontiguousarray(s.rho0detJ0[:, ::-1]))
    _, [(F1b, FTvb, dtb)] = gpu_eval(m, s2)
    assert rel(F1b, F1) > 1e-6 and rel(FTvb, FTv) > 1e-6


def test_non_affine_full_size_host_entry_matches_device():
    """A curved initial mesh at the C3 size (per-point J0^{-1}, generic kernel) through the pipelined host entry:
    the zone-chunk shifts of the per-point J0^{-1} array must give the device entry's bits."""
    torch = _torch()
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config("C3", "S1")
    curved = synth.Mesh(m.dim, m.order, m.N, m.L, s.x.copy(), m.zone_nodes, m.zone_mat, m.mat_gamma)
    s2 = synth.State(np.ascontiguousarray(s.x + 0.1 * (s.x - m.x0)), s.v, s.e, s.rho0detJ0)
    h, [(F1, FTv, dt)] = gpu_eval(curved, s2)
    assert h.variant.startswith("v1")
    hx = [torch.from_numpy(np.ascontiguousarray(a)).pin_memory() for a in (s2.x, s2.v, s2.e, s2.rho0detJ0)]
    o = h.eval_host(*hx)
    assert np.array_equal(o[0], F1) and np.array_equal(o[1], FTv) and o[2][0] == dt


def test_eval_is_cuda_graph_capturable():
    """include/blast_cf.h: eval is capture-safe for nranks == 1 (bench.py replays small configs from a graph):
    a captured eval replayed gives the eager eval's bits."""
    torch = _torch()
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config("C2", "S1", N=(32, 32))
    stream = torch.cuda.Stream()
    with torch.cuda.stream(stream):
        h = cf.from_synth(m, stream=stream)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    x, v, e, r = t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)
    ref = [o.clone() for o in h.eval(x, v, e, r)]
    stream.synchronize()
    out = h.alloc_outputs()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=stream):
        h.eval(x, v, e, r, out=out)
    for o in out:
        o.zero_()
    with torch.cuda.stream(stream):
        g.replay()
    stream.synchronize()
    for a, b in zip(ref, out):
        assert torch.equal(a, b)
