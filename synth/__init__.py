"""Seeded synthetic meshes, states and partitions for the corner-force path.

This module is the ONE piece shared by the oracle side (tests/, oracle/) and the
CUDA side (bench.py, the GPU tests): it only builds inputs.  It holds none of the
method's arithmetic — no quadrature, no basis evaluation at quadrature points, no
Jacobians, no stress.  The only geometric helper is the placement of mesh nodes at
the Gauss–Lobatto–Legendre (GLL) lattice of each zone, which is how a Q_k mesh
*is* described (its node positions are the kinematic DOFs, §2).

Workload recipe (DESIGN.md §"Input recipe"):

* C1  2D Sedov Q2-Q1 4x4            [0,1]^2          seed 1
* C2  2D Sedov Q4-Q3 64x64          [0,1]^2          seed 2  (RK2 step = states S1, S1b)
* C3  3D Sedov Q2-Q1 32^3           [0,1]^3          seed 3
* C4  3D Sedov Q4-Q3 32^3           [0,1]^3          seed 4  (headline)
* C5  3D triple-point Q8-Q7 48x24x24 [0,7]x[0,3]x[0,3] seed 5

Layouts follow include/blast_cf.h: x, v are [dim][num_nodes] (SoA), e is
[Z][k^dim] (Bernstein coefficients, x fastest), rho0detJ0 is [Z][(2k)^dim].
Zone id = ex + Nx(ey + Ny ez); node id = ix + Mx(iy + My iz), M_t = k N_t + 1;
local node a = l0 + (k+1)(l1 + (k+1) l2).
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import List, Optional, Sequence, Tuple

import numpy as np

GAMMA_SEDOV = 1.4
E_BLAST = 0.25


def gll_nodes01(k: int) -> np.ndarray:
    """GLL node positions on [0,1] (k+1 points) used to *place* mesh nodes.

    Endpoints plus the roots of P'_k, from numpy's Legendre class, polished by
    Newton steps in float64.  Geometry only; the oracle and the CUDA library
    compute their own tables independently.
    """
    if k < 1:
        raise ValueError("k >= 1")
    if k == 1:
        return np.array([0.0, 1.0])
    leg = np.polynomial.legendre.Legendre.basis(k)
    d1 = leg.deriv()
    d2 = d1.deriv()
    r = np.sort(np.real(d1.roots()))
    for _ in range(3):
        r = r - d1(r) / d2(r)
    r = 0.5 * (r - r[::-1])  # exact symmetry
    pts = np.concatenate([[-1.0], r, [1.0]])
    return 0.5 * (pts + 1.0)


@dataclass
class Mesh:
    dim: int
    order: int
    N: Tuple[int, ...]            # zones per axis
    L: Tuple[float, ...]          # domain extents (origin at 0)
    x0: np.ndarray                # [dim][num_nodes] float64
    zone_nodes: np.ndarray        # [Z][(k+1)^dim] int32
    zone_mat: np.ndarray          # [Z] int32
    mat_gamma: np.ndarray         # [num_mats] float64
    name: str = ""

    @property
    def num_zones(self) -> int:
        return int(self.zone_nodes.shape[0])

    @property
    def num_nodes(self) -> int:
        return int(self.x0.shape[1])

    @property
    def h(self) -> Tuple[float, ...]:
        return tuple(self.L[t] / self.N[t] for t in range(self.dim))

    @property
    def nk(self) -> int:
        return (self.order + 1) ** self.dim

    @property
    def nt(self) -> int:
        return self.order ** self.dim

    @property
    def nq(self) -> int:
        return (2 * self.order) ** self.dim

    def zone_gamma(self) -> np.ndarray:
        return self.mat_gamma[self.zone_mat].astype(np.float64)

    def zone_index(self, z: int) -> Tuple[int, ...]:
        out = []
        for t in range(self.dim):
            out.append(z % self.N[t])
            z //= self.N[t]
        return tuple(out)


@dataclass
class State:
    x: np.ndarray          # [dim][num_nodes]
    v: np.ndarray          # [dim][num_nodes]
    e: np.ndarray          # [Z][k^dim]
    rho0detJ0: np.ndarray  # [Z][(2k)^dim]
    name: str = ""


def box_mesh(dim: int, k: int, N: Sequence[int], L: Optional[Sequence[float]] = None, name: str = "") -> Mesh:
    """Structured Q_k box mesh with nodes on each zone's GLL lattice."""
    N = tuple(int(n) for n in N)
    L = tuple(float(l) for l in (L if L is not None else [1.0] * dim))
    assert len(N) == dim and len(L) == dim
    g = gll_nodes01(k)
    M = [k * N[t] + 1 for t in range(dim)]
    coords = []
    for t in range(dim):
        h = L[t] / N[t]
        i = np.arange(M[t])
        ez = np.minimum(i // k, N[t] - 1)
        l = i - ez * k
        coords.append(h * (ez + g[l]))
        coords[-1][-1] = L[t]
    grids = np.meshgrid(*coords, indexing="ij")  # index order (ix, iy[, iz])
    # node id = ix + Mx(iy + My iz): x fastest => transpose to (iz, iy, ix) then ravel
    x0 = np.stack([gr.transpose(tuple(range(dim))[::-1]).ravel() for gr in grids])
    # zone -> node map
    Z = int(np.prod(N))
    ez = np.indices(N[::-1]).reshape(dim, -1)[::-1]  # ez[t][z], z = ex + Nx(ey + ...)
    loc = np.indices([k + 1] * dim).reshape(dim, -1)[::-1]  # loc[t][a], a = l0 + (k+1)(l1 + ...)
    nid = np.zeros((Z, (k + 1) ** dim), dtype=np.int64)
    stride = 1
    for t in range(dim):
        it = ez[t][:, None] * k + loc[t][None, :]
        nid += it * stride
        stride *= M[t]
    return Mesh(dim, k, N, L, np.ascontiguousarray(x0, dtype=np.float64),
                np.ascontiguousarray(nid.astype(np.int32)), np.zeros(Z, dtype=np.int32),
                np.array([GAMMA_SEDOV]), name=name)


# ---------------------------------------------------------------------------
# helpers for fields
# ---------------------------------------------------------------------------

def _bump(r: np.ndarray) -> np.ndarray:
    return np.exp(-(((r - 0.5) / 0.1) ** 2))


def sine_field(rng: np.random.Generator, X: np.ndarray, L: Sequence[float], modes: int = 3) -> np.ndarray:
    """dim-vector random field sum_m a_m prod_t sin(pi kappa_mt X_t / L_t); vanishes on the box boundary."""
    dim = X.shape[0]
    out = np.zeros_like(X)
    for c in range(dim):
        for _ in range(modes):
            a = rng.uniform(-1.0, 1.0)
            kap = rng.integers(1, 4, size=dim)
            term = np.full(X.shape[1], a)
            for t in range(dim):
                term = term * np.sin(np.pi * kap[t] * X[t] / L[t])
            out[c] += term
    return out


def thermo_control_points(mesh: Mesh) -> np.ndarray:
    """Physical positions (in x0) of the Bernstein control points of every zone: [dim][Z][k^dim]."""
    k, dim = mesh.order, mesh.dim
    xi = np.array([0.5]) if k == 1 else np.arange(k) / (k - 1)
    loc = np.indices([k] * dim).reshape(dim, -1)[::-1]
    h = mesh.h
    out = np.zeros((dim, mesh.num_zones, k ** dim))
    zidx = np.indices(mesh.N[::-1]).reshape(dim, -1)[::-1]
    for t in range(dim):
        out[t] = h[t] * (zidx[t][:, None] + xi[loc[t]][None, :])
    return out


def _rho0detJ0_const(mesh: Mesh, rho_zone: np.ndarray) -> np.ndarray:
    vol = float(np.prod(mesh.h))
    return np.ascontiguousarray(np.repeat((rho_zone * vol)[:, None], mesh.nq, axis=1))


RHO_POINT_AMPL = 0.25


def _rho0detJ0_varying(mesh: Mesh, rho_zone: np.ndarray) -> np.ndarray:
    """rho0|J0| of the S1 states: the zone value times a seeded per-point factor 1 + 0.25 (U(0,1) - 1/2).

    A varying initial density inside a zone is allowed by the method (rho0|J0| is an input at every
    quadrature point, reading R2), and it makes the parity tests see a mis-indexed point read of this
    array.  It is a property of the initial mesh (time-invariant): its generator is seeded from the mesh
    shape only, so the two RK2 stage states S1 / S1b of a config share it, and the x, v, e draws of S1 are
    unchanged."""
    rng = np.random.default_rng([7919, mesh.dim, mesh.order, *mesh.N])
    f = 1.0 + RHO_POINT_AMPL * (rng.uniform(0.0, 1.0, size=(mesh.num_zones, mesh.nq)) - 0.5)
    return np.ascontiguousarray(_rho0detJ0_const(mesh, rho_zone) * f)


# ---------------------------------------------------------------------------
# Sedov (reading SURVEY §8c #16)
# ---------------------------------------------------------------------------

def sedov_s0(mesh: Mesh) -> State:
    """Sedov initial condition: rho0 = 1, v = 0, all blast energy E_b in the origin zone."""
    Z = mesh.num_zones
    vol = float(np.prod(mesh.h))
    e = np.zeros((Z, mesh.nt))
    e[0, :] = E_BLAST / (1.0 * vol)
    return State(mesh.x0.copy(), np.zeros_like(mesh.x0), e, _rho0detJ0_const(mesh, np.ones(Z)), name="S0")


def sedov_s1(mesh: Mesh, seed: int) -> State:
    """Synthetic mid-blast state: radially displaced curved mesh, radial shell velocity, random parts."""
    rng = np.random.default_rng(seed)
    X0 = mesh.x0
    dim = mesh.dim
    h = min(mesh.h)
    r0 = np.sqrt((X0 ** 2).sum(0))
    rhat = X0 / np.maximum(r0, 1e-300)
    b = _bump(r0)
    prod_sin = np.ones(X0.shape[1])
    for t in range(dim):
        prod_sin = prod_sin * np.sin(np.pi * X0[t] / mesh.L[t])
    x = X0 + 0.3 * h * b * rhat * prod_sin + 0.05 * h * sine_field(rng, X0, mesh.L)
    v = b * rhat + 0.05 * sine_field(rng, X0, mesh.L)
    cp = thermo_control_points(mesh)
    rc = np.sqrt((cp ** 2).sum(0))
    e = _bump(rc) + 0.1 + 0.1 * rng.uniform(0.0, 1.0, size=rc.shape)
    return State(np.ascontiguousarray(x), np.ascontiguousarray(v), np.ascontiguousarray(e),
                 _rho0detJ0_varying(mesh, np.ones(mesh.num_zones)), name=f"S1(seed={seed})")


# ---------------------------------------------------------------------------
# Triple point (reading SURVEY §8c #15, #17)
# ---------------------------------------------------------------------------

TP_REGIONS = {  # name: (rho, p, material)
    "left": (1.0, 1.0, 0),
    "top_right": (0.125, 0.1, 1),
    "bottom_right": (1.0, 0.1, 2),
}
TP_GAMMA = np.array([1.5, 1.5, 1.4])


def triple_point_mesh(dim: int, k: int, N: Sequence[int], name: str = "") -> Mesh:
    L = (7.0, 3.0, 3.0)[:dim]
    m = box_mesh(dim, k, N, L, name=name)
    Z = m.num_zones
    zidx = np.indices(m.N[::-1]).reshape(dim, -1)[::-1]
    xc = (zidx[0] + 0.5) * m.h[0]
    yc = (zidx[1] + 0.5) * m.h[1]
    mat = np.where(xc < 1.0, 0, np.where(yc >= 1.5, 1, 2)).astype(np.int32)
    m.zone_mat = np.ascontiguousarray(mat)
    m.mat_gamma = TP_GAMMA.copy()
    assert mat.shape == (Z,)
    return m


def _tp_rho_p(mesh: Mesh):
    rho = np.array([1.0, 0.125, 1.0])[mesh.zone_mat]
    p = np.array([1.0, 0.1, 0.1])[mesh.zone_mat]
    return rho, p


def triple_point_s0(mesh: Mesh) -> State:
    rho, p = _tp_rho_p(mesh)
    gam = mesh.zone_gamma()
    ez = p / ((gam - 1.0) * rho)
    e = np.repeat(ez[:, None], mesh.nt, axis=1)
    return State(mesh.x0.copy(), np.zeros_like(mesh.x0), np.ascontiguousarray(e),
                 _rho0detJ0_const(mesh, rho), name="S0")


def triple_point_s1(mesh: Mesh, seed: int) -> State:
    rng = np.random.default_rng(seed)
    X0 = mesh.x0
    hmin = min(mesh.h)
    x = X0 + 0.2 * hmin * sine_field(rng, X0, mesh.L)
    v = 0.05 * sine_field(rng, X0, mesh.L)
    v[0] += 0.5 * np.exp(-(((X0[0] - 1.5) / 0.3) ** 2))
    s0 = triple_point_s0(mesh)
    e = s0.e * (1.0 + 0.05 * rng.uniform(-1.0, 1.0, size=s0.e.shape))
    rho, _ = _tp_rho_p(mesh)
    return State(np.ascontiguousarray(x), np.ascontiguousarray(v), np.ascontiguousarray(e),
                 _rho0detJ0_varying(mesh, rho), name=f"S1(seed={seed})")


# ---------------------------------------------------------------------------
# BASELINE.json configs
# ---------------------------------------------------------------------------

CONFIGS = {
    "C1": dict(kind="sedov", dim=2, k=2, N=(4, 4), seed=1,
               desc="2D Sedov blast Q2-Q1, 4x4 zones, one corner-force evaluation vs CPU oracle"),
    "C2": dict(kind="sedov", dim=2, k=4, N=(64, 64), seed=2,
               desc="2D Sedov blast Q4-Q3, 64x64 zones, full RK2 step RHS"),
    "C3": dict(kind="sedov", dim=3, k=2, N=(32, 32, 32), seed=3,
               desc="3D Sedov blast Q2-Q1, 32^3 zones"),
    "C4": dict(kind="sedov", dim=3, k=4, N=(32, 32, 32), seed=4,
               desc="3D Sedov blast Q4-Q3, 32^3 zones (headline)"),
    "C5": dict(kind="triple", dim=3, k=8, N=(48, 24, 24), seed=5,
               desc="3D triple-point Q8-Q7 multi-material, 48x24x24 zones"),
}


def make_mesh(kind: str, dim: int, k: int, N: Sequence[int], name: str = "") -> Mesh:
    if kind == "sedov":
        return box_mesh(dim, k, N, name=name)
    if kind == "triple":
        return triple_point_mesh(dim, k, N, name=name)
    raise ValueError(kind)


def make_state(mesh: Mesh, kind: str, which: str, seed: int) -> State:
    if kind == "sedov":
        return sedov_s0(mesh) if which == "S0" else sedov_s1(mesh, seed)
    return triple_point_s0(mesh) if which == "S0" else triple_point_s1(mesh, seed)


def config(name: str, which: str = "S1", N: Optional[Sequence[int]] = None, k: Optional[int] = None):
    """(mesh, state) for a BASELINE config; N/k override gives a scaled-down case of the same recipe."""
    c = CONFIGS[name]
    kk = c["k"] if k is None else k
    NN = c["N"] if N is None else tuple(N)
    mesh = make_mesh(c["kind"], c["dim"], kk, NN, name=name)
    seed = c["seed"] + (100 if which == "S1b" else 0)
    st = make_state(mesh, c["kind"], "S0" if which == "S0" else "S1", seed)
    return mesh, st


# ---------------------------------------------------------------------------
# Domain decomposition (§3.4)
# ---------------------------------------------------------------------------

def block_dims(dim: int, P: int) -> Tuple[int, ...]:
    """Split P ranks over the zone grid: 3D 2->2x1x1, 4->2x2x1, 8->2x2x2; 2D 2->2x1, 4->2x2, 8->4x2."""
    dims = [1] * dim
    p = P
    t = 0
    while p > 1:
        f = 2 if p % 2 == 0 else p
        dims[t % dim] *= f
        p //= f
        t += 1
    assert int(np.prod(dims)) == P
    return tuple(dims)


@dataclass
class RankPart:
    rank: int
    nranks: int
    zones: np.ndarray        # [Zl] global zone ids: boundary zones first, then interior (each ascending)
    nodes: np.ndarray        # [Nl] global node ids (ascending)
    zone_nodes: np.ndarray   # [Zl][Nk] local node ids (int32)
    nbr_rank: np.ndarray     # [num_nbr] int32 ascending
    nbr_offset: np.ndarray   # [num_nbr+1] int64
    nbr_nodes: np.ndarray    # [nbr_offset[-1]] int32 local node ids, sorted by global id per neighbour
    owned: np.ndarray        # [Nl] bool: this rank is the lowest sharing rank (owner rule, MFEM group master)

    def local_mesh(self, mesh: Mesh) -> Mesh:
        return Mesh(mesh.dim, mesh.order, mesh.N, mesh.L, np.ascontiguousarray(mesh.x0[:, self.nodes]),
                    np.ascontiguousarray(self.zone_nodes), np.ascontiguousarray(mesh.zone_mat[self.zones]),
                    mesh.mat_gamma, name=f"{mesh.name}[r{self.rank}/{self.nranks}]")

    def local_state(self, st: State) -> State:
        return State(np.ascontiguousarray(st.x[:, self.nodes]), np.ascontiguousarray(st.v[:, self.nodes]),
                     np.ascontiguousarray(st.e[self.zones]), np.ascontiguousarray(st.rho0detJ0[self.zones]),
                     name=st.name)


def partition(mesh: Mesh, P: int) -> List[RankPart]:
    dim = mesh.dim
    pd = block_dims(dim, P)
    zidx = np.indices(mesh.N[::-1]).reshape(dim, -1)[::-1]
    owner = np.zeros(mesh.num_zones, dtype=np.int64)
    stride = 1
    for t in range(dim):
        # balanced contiguous blocks along axis t
        b = (zidx[t] * pd[t]) // mesh.N[t]
        owner += b * stride
        stride *= pd[t]
    parts_nodes = []
    parts = []
    for r in range(P):
        zones = np.nonzero(owner == r)[0]
        nodes = np.unique(mesh.zone_nodes[zones].ravel())
        parts_nodes.append(nodes)
    node_ranks = np.zeros(mesh.num_nodes, dtype=np.int64)   # how many ranks touch each node
    for r in range(P):
        node_ranks[parts_nodes[r]] += 1
    for r in range(P):
        zones = np.nonzero(owner == r)[0]
        # boundary zones (touching a node shared with another rank) first, each group in ascending global
        # id: the library then overlaps the shared-DOF exchange with the interior zones
        bnd = (node_ranks[mesh.zone_nodes[zones]] > 1).any(axis=1)
        zones = np.concatenate([zones[bnd], zones[~bnd]])
        nodes = parts_nodes[r]
        g2l = {int(g): i for i, g in enumerate(nodes)}
        zn = np.searchsorted(nodes, mesh.zone_nodes[zones]).astype(np.int32)
        nbr, offs, lst = [], [0], []
        owned = np.ones(len(nodes), dtype=bool)
        for q in range(P):
            if q == r:
                continue
            shared = np.intersect1d(nodes, parts_nodes[q], assume_unique=True)
            if len(shared) == 0:
                continue
            nbr.append(q)
            loc = np.searchsorted(nodes, shared)
            lst.append(loc)
            offs.append(offs[-1] + len(loc))
            if q < r:
                owned[loc] = False
        del g2l
        parts.append(RankPart(r, P, zones, nodes, np.ascontiguousarray(zn), np.array(nbr, dtype=np.int32),
                              np.array(offs, dtype=np.int64),
                              np.ascontiguousarray(np.concatenate(lst).astype(np.int32)) if lst else np.zeros(0, np.int32),
                              owned))
    return parts


# ---------------------------------------------------------------------------
# Edge-case states for the parity tests (inputs only: an affine velocity field v = B x on the current
# nodes, shifted or scaled thermodynamic coefficients).  SURVEY §8(c) c5 names the risky regimes.
# ---------------------------------------------------------------------------

def _rotation(dim: int, rng: np.random.Generator) -> np.ndarray:
    Q, Rr = np.linalg.qr(rng.standard_normal((dim, dim)))
    return Q * np.sign(np.diag(Rr))


def edge_state(mesh: Mesh, kind: str, which: str, seed: int, tie_gap: float = 1.5e-4) -> State:
    """S1 of `kind` ("sedov" | "triple") modified into one of the regimes the parity tests must cover:

    * "window":   v = B x with B = Q diag(1.5, 4, 6) 1e-12 Q^T: the smallest eigenvalue of the strain rate
                  is 1.5e-12, inside the viscosity switch window (eps_sw, 3 eps_sw) = (1e-12, 3e-12) at every
                  point; e scaled to ~1e-6 so the linear viscosity term is visible next to the pressure.
    * "negative_e": S1 with every thermodynamic coefficient lowered by 0.15 (Sedov: the background
                  e in [0.1, 0.2] straddles 0) / (triple point: by the mean coefficient): e(q) < 0 at part of the points, where the EOS clamps it to 0.
    * "near_tie": v = B x with B = Q diag(-1, -1 + tie_gap, 0.5) Q^T (tie_gap 1.5e-4: relative eigen-gap
                  1e-4 of the strain rate, gap / |B|_F) at every point, on a mesh deformed by 0.2 x the S1 displacement (J J0^-1
                  mildly anisotropic there: the eigenvector error eps/gap enters l = h0 |J J0^-1 s| scaled
                  by that anisotropy; gap >= 1e-4, and reduce the anisotropy rather than
                  loosen the tolerance).
    """
    base = make_state(mesh, kind, "S1", seed)
    rng = np.random.default_rng(seed + 4242)
    dim = mesh.dim
    Q = _rotation(dim, rng)
    if which == "window":
        B = Q @ np.diag([1.5e-12, 4e-12, 6e-12][:dim]) @ Q.T
        v = np.ascontiguousarray(B @ base.x)
        e = np.ascontiguousarray(1e-6 * (0.5 + base.e / base.e.max()))
        return State(base.x, v, e, base.rho0detJ0, name=f"window(seed={seed})")
    if which == "negative_e":
        shift = 0.15 if kind == "sedov" else float(base.e.mean())
        return State(base.x, base.v, np.ascontiguousarray(base.e - shift), base.rho0detJ0,
                     name=f"negative_e(seed={seed})")
    if which == "near_tie":
        B = Q @ np.diag([-1.0, -1.0 + tie_gap, 0.5][:dim]) @ Q.T
        x = np.ascontiguousarray(mesh.x0 + 0.2 * (base.x - mesh.x0))
        return State(x, np.ascontiguousarray(B @ x), base.e, base.rho0detJ0, name=f"near_tie(seed={seed})")
    raise ValueError(which)
