"""Domain decomposition on ONE GPU (loopback exchange): the library's pack kernel, ascending-rank plan
and combine kernel — the same code the NCCL path runs between the NCCL calls — checked against the
single-domain GPU evaluation and the oracle (SURVEY §4 T4 "loopback exchanger")."""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("name,N,k,P", [("C3", (4, 4, 4), None, 2), ("C3", (4, 4, 4), None, 8),
                                        ("C4", (4, 3, 2), None, 4), ("C2", (8, 6), 3, 8), ("C1", None, None, 4),
                                        ("C5", (4, 2, 2), None, 8)])
def test_loopback_exchange(orc, name, N, k, P):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ipps_dongdkrtd14_b200 as cf
    m, s = synth.config(name, "S1", N=N, k=k)
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    h1 = cf.from_synth(m)
    F1, FTv, dt = (o.cpu().numpy() for o in h1.eval(t(s.x), t(s.v), t(s.e), t(s.rho0detJ0)))
    par = cf.default_params()
    par.h0 = h1.info["h0"]
    parts = synth.partition(m, P)
    hs = [cf.from_synth(m, params=par, part=p, nccl_uid=None) for p in parts]
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
