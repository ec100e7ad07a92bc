"""CPU oracle of the time step around the corner force.  TEST INFRASTRUCTURE ONLY.

BLAST's semi-discrete system (§2, eqs (1)-(3)):
    M_V dv/dt = -F.1          (kinematic mass matrix: global, symmetric, sparse; PCG each step,
                               PAPER.md:193-198; kernel 9 "CUDA-PCG")
    M_E de/dt = F^T v         (thermodynamic mass matrix: block diagonal, inverse precomputed once,
                               PAPER.md:198-205; kernel 11 "SpMV")
    dx/dt = v
with (M_V)_ab = int rho W_a W_b and (M_E)_ij = int rho phi_i phi_j over the current configuration.
Since rho |J| = rho0 |J0| (reading R2) both are time-independent:
    (M_V)_ab = sum_z sum_q alpha_q rho0|J0|(z,q) W_a(q) W_b(q),  (M_E)_z,ij = sum_q alpha_q rho0|J0| phi_i phi_j.
The paper does not name its time integrator; the reading (R22) is the RK2-average scheme of
the BLAST line of work (Dobrev, Kolev, Rieben 2012; as in the public Laghos proxy), which conserves the
discrete total energy  E = 1/2 v^T M_V v + sum_z 1^T M_E e_z  exactly up to the solver tolerance —
the property the paper validates in Table 6.  Boundary condition (reading R23):
reflecting walls of the box domain, v . n = 0 (the normal velocity component of wall nodes is fixed).

Plain and slow: dense per-zone tables (W, phi, alpha at every point), scipy sparse assembly of M_V,
Jacobi-preconditioned CG written out, F_z formed explicitly by the corner-force oracle (definition
mode) and applied as F_z^T Vbar.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Optional

import numpy as np
import scipy.sparse as sp

import oracle


def dense_tables(dim: int, k: int):
    """W[q][a], phi[q][j], alpha[q] on the reference element from the oracle's 1-D tables."""
    t = oracle.tables_1d(k)
    n, p = 2 * k, k + 1
    B, Phi, w = t["B"], t["Phi"], t["qwt"]
    if dim == 2:
        W = np.einsum("ya,xb->yxab", B, B).reshape(n * n, p * p)        # q = qx + n qy, a = ax + p ay
        ph = np.einsum("yi,xj->yxij", Phi, Phi).reshape(n * n, k * k)
        al = np.einsum("y,x->yx", w, w).reshape(-1)
    else:
        W = np.einsum("za,yb,xc->zyxabc", B, B, B).reshape(n ** 3, p ** 3)
        ph = np.einsum("zi,yj,xl->zyxijl", Phi, Phi, Phi).reshape(n ** 3, k ** 3)
        al = np.einsum("z,y,x->zyx", w, w, w).reshape(-1)
    return W, ph, al


@dataclass
class Masses:
    MV: sp.csr_matrix        # [nnodes][nnodes] scalar kinematic mass (one copy per component)
    ME: np.ndarray           # [Z][nt][nt]
    ME_inv: np.ndarray       # [Z][nt][nt]
    me1: np.ndarray          # [Z][nt] = M_E 1 (internal-energy weights)


def mass_matrices(mesh, rho0detJ0: np.ndarray) -> Masses:
    W, ph, al = dense_tables(mesh.dim, mesh.order)
    wq = al[None, :] * rho0detJ0                              # [Z][nq]
    ME = np.einsum("zq,qi,qj->zij", wq, ph, ph)
    Mz = np.einsum("zq,qa,qb->zab", wq, W, W)                 # per-zone kinematic blocks
    nk = W.shape[1]
    rows = np.repeat(mesh.zone_nodes, nk, axis=1).ravel()
    cols = np.tile(mesh.zone_nodes, (1, nk)).ravel()
    MV = sp.coo_matrix((Mz.ravel(), (rows, cols)), shape=(mesh.num_nodes, mesh.num_nodes)).tocsr()
    MV.sum_duplicates()
    return Masses(MV, ME, np.linalg.inv(ME), ME.sum(2))


def wall_mask(mesh) -> np.ndarray:
    """[dim][nnodes] True where the velocity component is fixed (node on a wall normal to it)."""
    X = mesh.x0
    m = np.zeros_like(X, dtype=bool)
    for t in range(mesh.dim):
        lo, hi = X[t].min(), X[t].max()
        tol = 1e-12 * (hi - lo)
        m[t] = (np.abs(X[t] - lo) <= tol) | (np.abs(X[t] - hi) <= tol)
    return m


def pcg(A: sp.csr_matrix, b: np.ndarray, free: np.ndarray, tol: float = 1e-15, maxit: int = 5000):
    """Jacobi-preconditioned CG on the free DOFs (fixed DOFs held at 0).  Plain loop."""
    d = A.diagonal()
    x = np.zeros_like(b)
    r = np.where(free, b, 0.0)
    z = np.where(free, r / d, 0.0)
    pdir = z.copy()
    rz = r @ z
    bnorm = np.sqrt(np.where(free, b, 0.0) @ np.where(free, b, 0.0))
    it = 0
    if bnorm == 0.0:
        return x, 0
    while it < maxit:
        Ap = np.where(free, A @ pdir, 0.0)
        alpha = rz / (pdir @ Ap)
        x += alpha * pdir
        r -= alpha * Ap
        it += 1
        if np.sqrt(r @ r) <= tol * bnorm:
            break
        z = np.where(free, r / d, 0.0)
        rz_new = r @ z
        pdir = z + (rz_new / rz) * pdir
        rz = rz_new
    return x, it


def energies(masses: Masses, v: np.ndarray, e: np.ndarray):
    ke = 0.5 * sum(v[c] @ (masses.MV @ v[c]) for c in range(v.shape[0]))
    ie = float((masses.me1 * e).sum())
    return ke, ie


class RK2Avg:
    """One RK2-average step (reading R22) on (x, v, e) with the corner force from oracle.evaluate."""

    def __init__(self, mesh, rho0detJ0, params: Optional[oracle.Params] = None, cg_tol: float = 1e-15):
        import synth
        self.mesh = mesh
        self.R = np.ascontiguousarray(rho0detJ0)
        self.params = params or oracle.Params(h0=oracle.h0_of(mesh))
        self.masses = mass_matrices(mesh, self.R)
        self.fixed = wall_mask(mesh)
        self.cg_tol = cg_tol
        self._State = synth.State

    def forces(self, x, v, e):
        st = self._State(x, v, e, self.R)
        return oracle.evaluate(self.mesh, st, params=self.params, definition=True)

    def accel(self, F1):
        a = np.zeros_like(F1)
        its = 0
        for c in range(F1.shape[0]):
            a[c], it = pcg(self.masses.MV, -F1[c], ~self.fixed[c], self.cg_tol)
            its += it
        return a, its

    def de_dt(self, r, Vbar):
        Vz = Vbar[:, self.mesh.zone_nodes].transpose(1, 0, 2).reshape(self.mesh.num_zones, -1)
        FTV = np.einsum("zij,zi->zj", r.Fz, Vz)
        return np.einsum("zij,zj->zi", self.masses.ME_inv, FTV)

    def step(self, x, v, e, dt):
        r0 = self.forces(x, v, e)
        dv, _ = self.accel(r0.F1)
        Vb = v + 0.5 * dt * dv
        de = self.de_dt(r0, Vb)
        xh, vh, eh = x + 0.5 * dt * Vb, Vb, e + 0.5 * dt * de
        r1 = self.forces(xh, vh, eh)
        dv, _ = self.accel(r1.F1)
        Vb = v + 0.5 * dt * dv
        de = self.de_dt(r1, Vb)
        return x + dt * Vb, v + dt * dv, e + dt * de, min(r0.dt_min, r1.dt_min)

    def advance(self, x, v, e, t_final, dt, max_steps):
        """Step to t_final with the step-size control of reading R24 (Laghos's rule): a step whose
        dt estimate (min over its two force evaluations) falls below the dt it used is rejected and
        retried with 0.85 dt; an accepted step with estimate >= 1.25 dt grows dt by 2 %."""
        t, steps, rejected = 0.0, 0, 0
        while t < t_final and steps < max_steps:
            dt_use = min(dt, t_final - t)
            x1, v1, e1, dte = self.step(x, v, e, dt_use)
            if dte < dt_use:
                dt = 0.85 * dt_use
                rejected += 1
                continue
            x, v, e = x1, v1, e1
            t += dt_use
            steps += 1
            dt = 1.02 * dt_use if dte >= 1.25 * dt_use else dt_use
        return x, v, e, t, dt, steps, rejected
