"""N > 1 path of the integrator's M_V solve on CPU (world_size 2, 4 and 8, gloo).

Each rank assembles the kinematic mass matrix of ITS zones only (oracle/integrator.py, test
infrastructure) and runs exactly the multi-rank Jacobi PCG the library runs on the GPU (integrator.cu
cg_group): the Jacobi diagonal and every A p get their shared-node sum in the order of the library's own
plan (blast_cf_exchange_plan: ascending rank), every dot product is the owner-weighted local sum
(blast_cf_owner_mask) summed over the ranks, and the walls are those of the global box.  Checks:
  * the library's owner weights are the partition's ownership (each node counted once in the group),
  * the solution equals the single-domain oracle solve on every local node (<= 1e-11 relative; both
    sides stop at ||r|| <= 1e-15 ||b||),
  * every sharing rank holds bitwise identical iterates, and all ranks take the same iteration count.
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


def _exchange_sum(vec, part, plan, rank):
    """Shared-node sum of a [dim][nodes] vector: pack rows, send/recv per neighbour, ascending-rank sum."""
    rows = part.nbr_nodes
    send = np.ascontiguousarray(vec[:, rows].T)
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
    uniq, sptr, src = plan
    out = vec.copy()
    for u, node in enumerate(uniq):
        acc = np.zeros(vec.shape[0])
        for code in src[sptr[u]:sptr[u + 1]]:
            acc += send[code] if code >= 0 else recv[-code - 1]
        out[:, node] = acc
    return out


def _allreduce(a):
    t = torch.from_numpy(np.ascontiguousarray(a, dtype=np.float64))
    dist.all_reduce(t)
    return t.numpy()


def _worker(rank, world, port, name, N, k, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import integrator as oi
        import paper_conf_ipps_dongdkrtd14_b200 as cf
        import synth
        mesh, st = synth.config(name, "S1", N=N, k=k)
        part = synth.partition(mesh, world)[rank]
        lm, ls = part.local_mesh(mesh), part.local_state(st)
        dim, nn = mesh.dim, lm.num_nodes
        plan = cf.exchange_plan(rank, part.nbr_rank, part.nbr_offset, part.nbr_nodes)
        own = cf.owner_mask(rank, part.nbr_rank, part.nbr_offset, part.nbr_nodes, nn)
        owned = np.zeros(nn, bool)
        owned[part.owned] = True
        assert np.array_equal(own == 1.0, owned)
        cnt = _allreduce(np.array([own.sum()]))[0]
        assert cnt == mesh.num_nodes                           # each node counted once in the group
        # --- the library's multi-rank PCG (integrator.cu cg_group), on CPU ---
        MV = oi.mass_matrices(lm, ls.rho0detJ0).MV               # this rank's zones only
        fixed = oi.wall_mask(mesh)[:, part.nodes]                # walls of the GLOBAL box
        rng = np.random.default_rng(7)
        bg = rng.standard_normal((dim, mesh.num_nodes))          # a fully summed right-hand side
        b = bg[:, part.nodes]
        diag = _exchange_sum(np.tile(MV.diagonal(), (dim, 1)), part, plan, rank)
        invd = np.where(fixed, 0.0, 1.0 / diag)
        x = np.zeros((dim, nn))
        r = np.where(fixed, 0.0, b)
        z = r * invd
        p = np.zeros((dim, nn))
        red = _allreduce(np.concatenate([(own * r * z).sum(1), (own * r * r).sum(1)]))
        rz, bb = red[:dim], red[dim:]
        beta = np.zeros(dim)
        done = bool(np.all(bb == 0.0))
        it = 0
        tol2 = 1e-30
        while not done and it < 2000:
            p = z + beta[:, None] * p
            Ap = _exchange_sum(np.stack([MV @ p[c] for c in range(dim)]), part, plan, rank)
            Ap = np.where(fixed, 0.0, Ap)
            pap = _allreduce((own * p * Ap).sum(1))
            alpha = np.where(pap > 0.0, rz / np.where(pap > 0.0, pap, 1.0), 0.0)
            x += alpha[:, None] * p
            r -= alpha[:, None] * Ap
            z = r * invd
            red = _allreduce(np.concatenate([(own * r * z).sum(1), (own * r * r).sum(1)]))
            beta = np.where(rz > 0.0, red[:dim] / np.where(rz > 0.0, rz, 1.0), 0.0)
            rz, rr = red[:dim], red[dim:]
            it += 1
            done = bool(np.all(rr <= tol2 * bb))
        assert done, it
        # --- against the single-domain oracle solve ---
        MVg = oi.mass_matrices(mesh, st.rho0detJ0).MV
        fg = oi.wall_mask(mesh)
        ref = np.stack([oi.pcg(MVg, bg[c], ~fg[c], 1e-15)[0] for c in range(dim)])
        err = np.abs(x - ref[:, part.nodes]).max() / np.abs(ref).max()
        assert err <= 1e-11, err
        # every sharer holds the same bits; every rank took the same number of iterations
        vals = torch.from_numpy(np.ascontiguousarray(x[:, part.nbr_nodes].T))
        for i, q_rank in enumerate(part.nbr_rank):
            o0, o1 = part.nbr_offset[i], part.nbr_offset[i + 1]
            mine = vals[o0:o1].clone()
            theirs = torch.zeros_like(mine)
            a = dist.isend(mine, int(q_rank))
            bq = dist.irecv(theirs, int(q_rank))
            a.wait()
            bq.wait()
            assert torch.equal(mine, theirs)
        its = torch.tensor([float(it)], dtype=torch.float64)
        dist.all_reduce(its, op=dist.ReduceOp.MAX)
        assert float(its[0]) == it
        q.put((rank, "ok"))
    except BaseException as e:  # report to the parent
        q.put((rank, repr(e)))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,name,N,k", [(2, "C3", (4, 3, 2), None), (4, "C2", (6, 4), 3), (8, "C4", (2, 2, 2), 2)])
def test_multirank_cg_matches_single_domain(world, name, N, k):
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    mp.start_processes(_worker, args=(world, _free_port(), name, N, k, q), nprocs=world, join=True,
                       start_method="spawn")
    res = sorted(q.get() for _ in range(world))
    assert all(r[1] == "ok" for r in res), res
