"""N > 1 path on CPU (world_size 2 and 4, gloo): domain decomposition + shared-DOF exchange.

Each rank evaluates its sub-domain with the oracle (test infrastructure), then runs exactly the
exchange the library performs on the GPU — pack rows per neighbour, grouped send/recv, sum every
shared node's partials in the order of the library's own plan (blast_cf_exchange_plan: ascending
rank), global min dt — over torch.distributed gloo.  Checks:
  * the assembled F.1 equals the single-domain oracle on every local node (<= 1e-14 relative),
  * every sharing rank holds bitwise identical values on shared nodes,
  * F^T v per zone and the global dt equal the single-domain values,
  * owner-rule invariants: sum over owned nodes of F.1 = 0 and v.F1 = sum F^T v globally.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, name, N, k, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import paper_conf_ipps_dongdkrtd14_b200 as cf
        import synth
        mesh, st = synth.config(name, "S1", N=N, k=k)
        h0 = oracle.h0_of(mesh)
        par = oracle.Params(h0=h0)
        part = synth.partition(mesh, world)[rank]
        lm, ls = part.local_mesh(mesh), part.local_state(st)
        r = oracle.evaluate(lm, ls, params=par)
        F1 = r.F1.copy()
        dim = mesh.dim
        # --- the library's exchange, on CPU ---
        rows = part.nbr_nodes
        send = np.ascontiguousarray(F1[:, rows].T)             # [nrows][dim]
        recv = np.zeros_like(send)
        reqs = []
        for i, q_rank in enumerate(part.nbr_rank):
            o0, o1 = part.nbr_offset[i], part.nbr_offset[i + 1]
            sb = torch.from_numpy(send[o0:o1].copy())
            rb = torch.zeros_like(sb)
            reqs.append((dist.isend(sb, int(q_rank)), dist.irecv(rb, int(q_rank)), rb, o0, o1))
        for s_req, r_req, rb, o0, o1 in reqs:
            s_req.wait()
            r_req.wait()
            recv[o0:o1] = rb.numpy()
        uniq, sptr, src = cf.exchange_plan(rank, part.nbr_rank, part.nbr_offset, part.nbr_nodes)
        for u, node in enumerate(uniq):
            acc = np.zeros(dim)
            for code in src[sptr[u]:sptr[u + 1]]:
                acc += send[code] if code >= 0 else recv[-code - 1]
            F1[:, node] = acc
        # global min dt, as the library's single-round schedule does it: every rank's dt travels with its F.1
        # rows to every neighbour (in these block partitions every rank neighbours every other, which the
        # library checks before it drops the allreduce)
        assert len(part.nbr_rank) == world - 1
        mine = torch.tensor([r.dt_min], dtype=torch.float64)
        got = []
        for q_rank in part.nbr_rank:
            t_in = torch.zeros(1, dtype=torch.float64)
            a_ = dist.isend(mine.clone(), int(q_rank))
            b_ = dist.irecv(t_in, int(q_rank))
            a_.wait()
            b_.wait()
            got.append(float(t_in[0]))
        dt = torch.tensor([min([r.dt_min] + got)], dtype=torch.float64)
        ref_dt = torch.tensor([r.dt_min], dtype=torch.float64)
        dist.all_reduce(ref_dt, op=dist.ReduceOp.MIN)   # the overlap schedule's allreduce gives the same value
        assert float(ref_dt[0]) == float(dt[0])
        # --- checks against the single-domain oracle ---
        g = oracle.evaluate(mesh, st, params=par)
        ref = g.F1[:, part.nodes]
        err = np.abs(F1 - ref).max() / np.abs(g.F1).max()
        assert err <= 1e-14, err
        assert np.array_equal(r.FTv, g.FTv[part.zones])
        assert float(dt[0]) == g.dt_min
        # bitwise agreement of all sharers: compare with every neighbour's values on shared rows
        vals = torch.from_numpy(np.ascontiguousarray(F1[:, rows].T))
        for i, q_rank in enumerate(part.nbr_rank):
            o0, o1 = part.nbr_offset[i], part.nbr_offset[i + 1]
            mine = vals[o0:o1].clone()
            theirs = torch.zeros_like(mine)
            a = dist.isend(mine, int(q_rank))
            b = dist.irecv(theirs, int(q_rank))
            a.wait()
            b.wait()
            assert torch.equal(mine, theirs)
        # owner-rule global invariants
        loc = torch.tensor(np.concatenate([F1[:, part.owned].sum(1), [(ls.v[:, part.owned] * F1[:, part.owned]).sum(),
                                                                      r.FTv.sum(), np.abs(F1).sum()]]))
        dist.all_reduce(loc)
        tot = loc.numpy()
        assert np.abs(tot[:dim]).max() <= 1e-13 * tot[-1]
        assert abs(tot[dim] - tot[dim + 1]) <= 1e-13 * np.abs(st.v).max() * tot[-1]
        q.put((rank, "ok"))
    except BaseException as e:  # report to the parent
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,name,N,k", [(2, "C3", (4, 3, 2), None), (4, "C3", (4, 4, 2), None),
                                            (2, "C2", (6, 4), 3), (4, "C2", (4, 6), 2), (8, "C4", (2, 2, 2), 2)])
def test_exchange_matches_single_domain(world, name, N, k):
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    mp.start_processes(_worker, args=(world, _free_port(), name, N, k, q), nprocs=world, join=True,
                       start_method="spawn")
    res = sorted(q.get() for _ in range(world))
    assert all(r[1] == "ok" for r in res), res
