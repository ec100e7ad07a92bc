"""Peer-memory transport of the shared-DOF exchange (include/blast_cf.h blast_cf_p2p_*) in
real multi-process runs on ONE GPU: every rank is its own process (gloo process group for the bootstrap
all-gather only), maps the other ranks' mailboxes through CUDA IPC, and exchanges its shared rows and dt
by peer stores + system-scope flags — the code path an 8-GPU run takes, minus NVLink (the contexts of the
processes time-slice the device, so every wait in the protocol is really exercised).

Each rank evaluates the states S1, S1b, S1, S1b, S1 in turn: a receiver that read the rows of the wrong
eval (epoch parity, stale buffers) would mix the two states.  Checked against the single-domain
evaluation (itself checked against the oracle in test_gpu_parity.py): F.1 on every local node to 1e-14
of max|F.1| (only the summation order of shared nodes differs), F^T v and dt bitwise, and every sharer
of a node holding the same bits."""
import os
import socket
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, name, N, k, overlap, outdir):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), BLAST_CF_OVERLAP=overlap)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    import synth
    m, sa = synth.config(name, "S1", N=N, k=k)
    sb = synth.config(name, "S1b", N=N, k=k)[1]
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    h1 = cf.from_synth(m)
    ref = [tuple(o.cpu().numpy() for o in h1.eval(t(s_.x), t(s_.v), t(s_.e), t(s_.rho0detJ0))) for s_ in (sa, sb)]
    par = cf.default_params()
    par.h0 = h1.info["h0"]
    h1.close()
    p = synth.partition(m, world)[rank]
    h = cf.from_synth(m, params=par, part=p, nccl_uid=None)
    h.p2p_connect()
    transport, (mode, nb) = h.exchange_transport(), h.exchange_schedule()
    ins = [tuple(t(a) for a in (ls.x, ls.v, ls.e, ls.rho0detJ0)) for ls in (p.local_state(sa), p.local_state(sb))]
    got = []
    for it in range(5):
        f1, ftv, dt = h.eval(*ins[it % 2])
        torch.cuda.synchronize()
        got.append((f1.cpu().numpy(), ftv.cpu().numpy(), float(dt.cpu()[0])))
    h.close()
    np.savez(os.path.join(outdir, f"r{rank}.npz"), nodes=p.nodes, zones=p.zones, mode=mode, nb=nb,
             transport=transport, f1=np.stack([g[0] for g in got]), ftv=np.stack([g[1] for g in got]),
             dt=np.array([g[2] for g in got]), ref_f1=np.stack([r[0] for r in ref]),
             ref_ftv=np.stack([r[1] for r in ref]), ref_dt=np.array([float(r[2][0]) for r in ref]))
    dist.destroy_process_group()


@pytest.mark.timeout(600)
@pytest.mark.parametrize("overlap", ["1", "0"])
@pytest.mark.parametrize("name,N,k,P", [("C3", (4, 4, 4), None, 2), ("C4", (4, 3, 2), None, 4), ("C2", (8, 6), 3, 3)])
def test_p2p_multiprocess(tmp_path, name, N, k, P, overlap):
    import torch
    import torch.multiprocessing as mp
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    mp.spawn(_worker, args=(P, _free_port(), name, N, k, overlap, str(tmp_path)), nprocs=P, join=True)
    ds = [np.load(tmp_path / f"r{r}.npz") for r in range(P)]
    # the schedule is agreed at connect: overlap only if every rank has boundary AND interior zones
    can = overlap == "1" and all(0 < int(d["nb"]) < len(d["zones"]) for d in ds)
    shared = {}
    for r, d in enumerate(ds):
        assert str(d["transport"]) == "p2p"
        assert int(d["mode"]) == (2 if can else 1)
        nodes, zones = d["nodes"], d["zones"]
        for it in range(5):
            st = it % 2
            rf1 = d["ref_f1"][st]
            scale = np.abs(rf1).max()
            assert np.abs(d["f1"][it] - rf1[:, nodes]).max() <= 1e-14 * scale, (r, it)
            assert np.array_equal(d["ftv"][it], d["ref_ftv"][st][zones]), (r, it)
            assert d["dt"][it] == d["ref_dt"][st], (r, it)
            for g, val in zip(nodes, d["f1"][it].T):
                key = (it, int(g))
                if key in shared:
                    assert np.array_equal(shared[key], val), (r, it, g)   # every sharer holds the same bits
                else:
                    shared[key] = val


def test_p2p_connect_errors():
    """blast_cf_p2p_*: the error paths (include/blast_cf.h) — single-rank handle, enable before connect,
    a record of the wrong size or not from this group, a fall-back without an NCCL communicator."""
    import ctypes
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    import synth
    L = cf.lib()
    m, _ = synth.config("C3", "S1", N=(4, 4, 4))
    h1 = cf.from_synth(m)
    n = ctypes.c_int64(0)
    assert L.blast_cf_p2p_export(h1._h, None, ctypes.byref(n)) == 1          # single rank: EINVAL
    par = cf.default_params()
    par.h0 = h1.info["h0"]
    parts = synth.partition(m, 2)
    h = cf.from_synth(m, params=par, part=parts[0], nccl_uid=None)
    assert L.blast_cf_p2p_enable(h._h, 1) == 1                              # not connected
    assert L.blast_cf_p2p_export(h._h, None, ctypes.byref(n)) == 0 and n.value > 0
    small = ctypes.c_int64(n.value - 1)
    buf = ctypes.create_string_buffer(n.value)
    assert L.blast_cf_p2p_export(h._h, buf, ctypes.byref(small)) == 1        # buffer too small
    assert L.blast_cf_p2p_export(h._h, buf, ctypes.byref(n)) == 0
    assert L.blast_cf_p2p_connect(h._h, buf.raw * 2, n.value - 8) == 1       # wrong record size
    assert L.blast_cf_p2p_connect(h._h, buf.raw * 2, n.value) == 1           # record 1 is not rank 1's
    assert L.blast_cf_p2p_connect(h._h, b"\0" * (2 * n.value), n.value) == 1  # not records at all
    assert L.blast_cf_p2p_enable(h._h, 0) == 1                              # no NCCL communicator
    assert h.exchange_transport() == "loopback"
    h.close()
    h1.close()
