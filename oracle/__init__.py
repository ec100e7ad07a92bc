"""ctypes wrapper of the CPU oracle (oracle/blast_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs.  The product package never imports this module and this
module never imports the product package.  See blast_oracle.c's header for what it computes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "blast_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain C11, no FMA contraction, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        dp = ctypes.POINTER(ctypes.c_double)
        ip = ctypes.POINTER(ctypes.c_int32)
        lp = ctypes.POINTER(ctypes.c_int64)
        L.oracle_eval.restype = ctypes.c_int
        L.oracle_eval.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int64, ctypes.c_int64, ip, dp, dp, dp, dp, dp,
                                  dp, dp, lp, ctypes.c_int64, dp, dp, dp, dp, dp, dp, dp, ctypes.c_int]
        L.oracle_volume.restype = ctypes.c_double
        L.oracle_volume.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int64, ip, ctypes.c_int64, dp]
        L.oracle_tables_1d.restype = None
        L.oracle_tables_1d.argtypes = [ctypes.c_int, dp, dp, dp, dp, dp, dp]
        L.oracle_sym_eig.restype = None
        L.oracle_sym_eig.argtypes = [ctypes.c_int, dp, dp, dp]
        L.oracle_sigma_min.restype = ctypes.c_double
        L.oracle_sigma_min.argtypes = [ctypes.c_int, dp]
        L.oracle_max_threads.restype = ctypes.c_int
        L.oracle_gauss_legendre01.restype = None
        L.oracle_gauss_legendre01.argtypes = [ctypes.c_int, dp, dp]
        _lib = L
    return _lib


def _dp(a: Optional[np.ndarray]):
    if a is None:
        return None
    assert a.dtype == np.float64 and a.flags.c_contiguous
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _ip(a):
    assert a.dtype == np.int32 and a.flags.c_contiguous
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int32))


def _lp(a):
    if a is None:
        return None
    assert a.dtype == np.int64 and a.flags.c_contiguous
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


@dataclass
class Params:
    """Reading DESIGN.md R8/R10/R11: cfl 0.5, q_quad 2, q_lin 1/2, eps_switch 1e-12, h0 computed."""
    cfl: float = 0.5
    q_quad: float = 2.0
    q_lin: float = 0.5
    eps_switch: float = 1e-12
    h0: float = 0.0
    use_viscosity: int = 1
    use_vorticity: int = 1

    def array(self) -> np.ndarray:
        return np.array([self.cfl, self.q_quad, self.q_lin, self.eps_switch, self.h0, self.use_viscosity,
                         self.use_vorticity], dtype=np.float64)


@dataclass
class Result:
    F1: Optional[np.ndarray]      # [dim][nnodes]
    Fz1: np.ndarray               # [nsub][dim][nk]
    FTv: np.ndarray               # [nsub][nt]
    dtz: np.ndarray               # [nsub]
    dt_min: float
    Fz: Optional[np.ndarray]      # [nsub][dim*nk][nt]
    diag: dict


def tables_1d(k: int):
    n, p = 2 * k, k + 1
    qpt, qwt, gll = np.zeros(n), np.zeros(n), np.zeros(p)
    B, G, Phi = np.zeros((n, p)), np.zeros((n, p)), np.zeros((n, k))
    lib().oracle_tables_1d(k, _dp(qpt), _dp(qwt), _dp(gll), _dp(B), _dp(G), _dp(Phi))
    return dict(qpt=qpt, qwt=qwt, gll=gll, B=B, G=G, Phi=Phi)


def sym_eig(A: np.ndarray):
    d = A.shape[0]
    A = np.ascontiguousarray(A, dtype=np.float64)
    lam, V = np.zeros(d), np.zeros((d, d))
    lib().oracle_sym_eig(d, _dp(A), _dp(lam), _dp(V))
    return lam, V


def sigma_min(J: np.ndarray) -> float:
    J = np.ascontiguousarray(J, dtype=np.float64)
    return lib().oracle_sigma_min(J.shape[0], _dp(J))


def volume(dim, k, zone_nodes, x0) -> float:
    zn = np.ascontiguousarray(zone_nodes, dtype=np.int32)
    x0 = np.ascontiguousarray(x0, dtype=np.float64)
    return lib().oracle_volume(dim, k, zn.shape[0], _ip(zn), x0.shape[1], _dp(x0))


def h0_of(mesh) -> float:
    """h0 = (V/Z)^(1/d) / k over the whole mesh (reading R11)."""
    V = volume(mesh.dim, mesh.order, mesh.zone_nodes, mesh.x0)
    return (V / mesh.num_zones) ** (1.0 / mesh.dim) / mesh.order


def evaluate(mesh, state, params: Optional[Params] = None, zones: Optional[Sequence[int]] = None,
             definition: bool = False, assemble: bool = True, nthreads: int = 0) -> Result:
    """Run the oracle on `mesh` (synth.Mesh) and `state` (synth.State)."""
    params = params or Params()
    dim, k = mesh.dim, mesh.order
    nk, nt = (k + 1) ** dim, k ** dim
    Z, nn = mesh.num_zones, mesh.num_nodes
    zl = None if zones is None else np.ascontiguousarray(np.asarray(zones, dtype=np.int64))
    if zl is not None:
        assert np.all(np.diff(zl) > 0), "zone subset must be ascending"
    nsub = Z if zl is None else len(zl)
    F1 = np.zeros((dim, nn)) if assemble else None
    Fz1 = np.zeros((nsub, dim, nk))
    FTv = np.zeros((nsub, nt))
    dtz = np.zeros(nsub)
    dtm = np.zeros(1)
    Fz = np.zeros((nsub, dim * nk, nt)) if definition else None
    diag = np.zeros(5)
    zn = np.ascontiguousarray(mesh.zone_nodes, dtype=np.int32)
    c = lambda a: np.ascontiguousarray(a, dtype=np.float64)
    x, v, e, r, x0 = c(state.x), c(state.v), c(state.e), c(state.rho0detJ0), c(mesh.x0)
    gam = c(mesh.zone_gamma())
    pa = params.array()
    rc = lib().oracle_eval(dim, k, Z, nn, _ip(zn), _dp(x), _dp(v), _dp(e), _dp(r), _dp(x0), _dp(gam), _dp(pa),
                           _lp(zl), nsub, _dp(F1), _dp(Fz1), _dp(FTv), _dp(dtz), _dp(dtm), _dp(Fz), _dp(diag),
                           int(nthreads))
    if rc != 0:
        raise RuntimeError(f"oracle_eval failed ({rc})")
    dg = dict(min_detJ=diag[0], min_gap=diag[1], min_switch_dist=diag[2], n_noinv=int(diag[3]), n_bad=int(diag[4]))
    return Result(F1, Fz1, FTv, dtz, float(dtm[0]), Fz, dg)


def max_threads() -> int:
    return lib().oracle_max_threads()
