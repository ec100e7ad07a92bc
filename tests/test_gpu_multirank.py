"""Domain decomposition on ONE GPU (loopback exchange): the library's pack kernel, ascending-rank plan
and combine kernel — the same code the NCCL path runs between the NCCL calls — checked against the
single-domain GPU evaluation and the oracle (SURVEY §4 T4 "loopback exchanger")."""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("overlap", ["1", "0"])
@pytest.mark.parametrize("name,N,k,P", [("C3", (4, 4, 4), None, 2), ("C3", (4, 4, 4), None, 8),
                                        ("C4", (4, 3, 2), None, 4), ("C2", (8, 6), 3, 8), ("C1", None, None, 4),
                                        ("C5", (4, 2, 2), None, 8), ("C3", (8, 6, 6), None, 8), ("C2", (12, 10), 4, 4)])
def test_loopback_exchange(orc, name, N, k, P, overlap, monkeypatch):
    """Both exchange schedules (overlap: boundary zones, exchange on the comm stream while the interior
    zones compute; single round) give the single-domain result on every node."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    monkeypatch.setenv("BLAST_CF_OVERLAP", overlap)
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config(name, "S1", N=N, k=k)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    h1 = cf.from_synth(m)
    F1, FTv, dt = (o.cpu().numpy() for o in h1.eval(t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)))
    par = cf.default_params()
    par.h0 = h1.info["h0"]
    parts = synth.partition(m, P)
    hs = [cf.from_synth(m, params=par, part=p, nccl_uid=None) for p in parts]
    for h, p in zip(hs, parts):
        mode, nb = h.exchange_schedule()
        interior = len(p.zones) - nb
        assert mode == (2 if overlap == "1" and nb > 0 and interior > 0 else 1), (mode, nb, len(p.zones))
    ls = [p.local_state(s) for p in parts]
    outs = cf.eval_loopback(hs, [t(l.x) for l in ls], [t(l.v) for l in ls], [t(l.e) for l in ls],
                            [t(l.rho0detJ0) for l in ls])
    torch.cuda.synchronize()
    scale = np.abs(F1).max()
    shared = {}
    for p, (f1, ftv, d) in zip(parts, outs):
        f1, ftv, d = f1.cpu().numpy(), ftv.cpu().numpy(), float(d.cpu()[0])
        assert np.abs(f1 - F1[:, p.nodes]).max() <= 1e-14 * scale
        assert np.array_equal(ftv, FTv[p.zones])
        assert d == float(dt[0])
        for g, val in zip(p.nodes, f1.T):
            if g in shared:
                assert np.array_equal(shared[g], val)   # every sharer holds the same bits
            else:
                shared[g] = val
    r = orc.evaluate(m, s)
    glob = np.zeros_like(F1)
    for p, (f1, _, _) in zip(parts, outs):
        glob[:, p.nodes] = f1.cpu().numpy()
    assert np.abs(glob - r.F1).max() <= 1e-12 * np.abs(r.F1).max()


@pytest.mark.parametrize("name,N,k,P", [("C3", (4, 4, 4), None, 2), ("C3", (4, 4, 4), None, 8),
                                        ("C2", (8, 6), 3, 4), ("C5", (4, 2, 2), 2, 8)])
def test_loopback_integrator(name, N, k, P):
    """Multi-GPU CG for M_V on one GPU: every rank of a loopback group runs the group
    CG (shared-node sum of A p each iteration, owner-weighted dot products summed over the ranks) inside
    blast_cf_rk2_rates_loopback; dv/dt, de/dt, dt and the energies must match the single-domain
    integrator, and every sharer of a node must hold the same bits."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import ctypes
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config(name, "S1", N=N, k=k)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    h1 = cf.from_synth(m)
    r1 = cf.RK2(h1, s.rho0detJ0, cg_rel_tol=1e-15)
    x, v, e = t(s.x), t(s.v), t(s.e)
    dv1, de1, dt1, it1 = (a.cpu().numpy() if hasattr(a, "cpu") else a for a in r1.rates(x, v, e))
    ke1, ie1 = r1.energy(v, e)
    par = cf.default_params()
    par.h0 = h1.info["h0"]
    parts = synth.partition(m, P)
    box = dict(box_lo=(ctypes.c_double * 3)(*([0.0] * 3)),
               box_hi=(ctypes.c_double * 3)(*(list(m.L) + [0.0] * (3 - m.dim))))
    hs = [cf.from_synth(m, params=par, part=p, nccl_uid=None) for p in parts]
    ls = [p.local_state(s) for p in parts]
    rk = [cf.RK2(h, l.rho0detJ0, cg_rel_tol=1e-15, **box) for h, l in zip(hs, ls)]
    cf.rk2_setup_loopback(rk)
    xs, vs, es = [t(l.x) for l in ls], [t(l.v) for l in ls], [t(l.e) for l in ls]
    dvs, des, dt, it = cf.rk2_rates_loopback(rk, xs, vs, es)
    ke, ie = cf.rk2_energy_loopback(rk, vs, es)
    assert dt == dt1
    assert abs(it - it1) <= 3, (it, it1)
    sdv, sde = np.abs(dv1).max(), np.abs(de1).max()
    shared = {}
    for p, dv, de in zip(parts, dvs, des):
        dv, de = dv.cpu().numpy(), de.cpu().numpy()
        assert np.abs(dv - dv1[:, p.nodes]).max() <= 1e-11 * sdv
        assert np.abs(de - de1[p.zones]).max() <= 1e-12 * sde
        for g, val in zip(p.nodes, dv.T):
            if g in shared:
                assert np.array_equal(shared[g], val)   # every sharer holds the same iterate bits
            else:
                shared[g] = val
    assert abs(ke - ke1) <= 1e-13 * max(abs(ke1), 1e-300) and abs(ie - ie1) <= 1e-13 * abs(ie1)


def test_loopback_schedules_bitwise_equal_and_overlap_visible(monkeypatch):
    """C4-like mesh split over 2 ranks: the overlap schedule and the single-round schedule give the same
    bits (same per-node summation orders), and with timing on the shared-row exchange ends before the
    interior zones' corner force does (the exchange is hidden behind the interior)."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config("C4", "S1", N=(16, 16, 16))
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    par = cf.default_params()
    par.h0 = (1.0 / m.num_zones) ** (1 / 3) / m.order
    parts = synth.partition(m, 2)
    ls = [p.local_state(s) for p in parts]
    args = ([t(l.x) for l in ls], [t(l.v) for l in ls], [t(l.e) for l in ls], [t(l.rho0detJ0) for l in ls])
    res = {}
    for ov in ("1", "0"):
        monkeypatch.setenv("BLAST_CF_OVERLAP", ov)
        hs = [cf.from_synth(m, params=par, part=p, nccl_uid=None) for p in parts]
        assert all(h.exchange_schedule()[0] == (2 if ov == "1" else 1) for h in hs)
        for h in hs:
            h.set_timing(True)
        for _ in range(3):
            outs = cf.eval_loopback(hs, *args)
        torch.cuda.synchronize()
        res[ov] = [[o.cpu().numpy() for o in out] for out in outs]
        if ov == "1":
            for h in hs:
                sent, interior_end, end = h.debug_exchange_times()
                assert sent < interior_end <= end, (sent, interior_end, end)
        for h in hs:
            h.close()
    for a, b in zip(res["1"], res["0"]):
        for x, y in zip(a, b):
            assert np.array_equal(x, y)


def _nccl_worker(rank, world, uid, overlap, q, transport="nccl", port=0):
    import os
    os.environ["BLAST_CF_OVERLAP"] = overlap
    import torch
    torch.cuda.set_device(rank)
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config("C3", "S1", N=(8, 6, 6))
    part = synth.partition(m, world)[rank]
    h = cf.from_synth(m, part=part, nccl_uid=uid)
    if transport == "p2p":   # NCCL for create, peer memory for every eval (bootstrap all-gather over gloo)
        import torch.distributed as dist
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=world)
        h.p2p_connect()
        assert h.exchange_transport() == "p2p"
    ls = part.local_state(s)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    outs = None
    for _ in range(3):
        outs = h.eval(t(ls.x), t(ls.v), t(ls.e), t(ls.rho0detJ0))
    torch.cuda.synchronize()
    q.put((rank, h.exchange_schedule()[0], h.info["h0"], *(o.cpu().numpy() for o in outs)))
    h.close()


@pytest.mark.parametrize("transport", ["nccl", "p2p"])
@pytest.mark.parametrize("overlap", ["1", "0"])
def test_nccl_multiprocess(orc, overlap, transport):
    """The real NCCL path: P = min(#GPUs, 8) processes, one per GPU, both schedules, the exchange by NCCL or
    through peer memory (NCCL then only at create); every rank's F.1 matches the single-domain oracle,
    sharers hold the same bits, dt is the global min.  Needs >= 2 GPUs (NCCL refuses two ranks on one
    device; the peer-memory transport alone is tested on one GPU in test_gpu_p2p.py)."""
    import torch
    if not torch.cuda.is_available() or torch.cuda.device_count() < 2:
        pytest.skip("needs >= 2 GPUs")
    import torch.multiprocessing as mp
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    P = min(torch.cuda.device_count(), 8)
    uid = cf.nccl_unique_id()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    procs = [ctx.Process(target=_nccl_worker, args=(r, P, uid, overlap, q, transport, port)) for r in range(P)]
    for p in procs:
        p.start()
    got = sorted(q.get(timeout=300) for _ in range(P))
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    m, s = synth.config("C3", "S1", N=(8, 6, 6))
    r = orc.evaluate(m, s, params=orc.Params(h0=got[0][2]))
    parts = synth.partition(m, P)
    shared = {}
    for (rank, mode, h0, F1, FTv, dt), p in zip(got, parts):
        assert mode == (2 if overlap == "1" else 1)
        assert np.abs(F1 - r.F1[:, p.nodes]).max() <= 1e-12 * np.abs(r.F1).max()
        assert np.abs(FTv - r.FTv[p.zones]).max() <= 1e-12 * np.abs(r.FTv).max()
        assert abs(float(dt[0]) - r.dt_min) <= 1e-12 * r.dt_min
        for g, val in zip(p.nodes, F1.T):
            if g in shared:
                assert np.array_equal(shared[g], val)
            else:
                shared[g] = val
