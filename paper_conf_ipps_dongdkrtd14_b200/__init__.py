"""B200-native BLAST corner force (Dong et al., IPDPS 2014) — thin Python binding of libblastcf.so.

Argument marshalling only: every step of the corner-force path runs in the CUDA kernels of
csrc/ behind the C ABI in include/blast_cf.h.  PyTorch is used for device memory, streams and
torch.distributed (the ncclUniqueId broadcast); there is no CPU fallback — if the extension is
missing the import of the library raises.

    cf = CornerForce(mesh_arrays..., order=k, dim=d)
    F1, FTv, dt = cf.eval(x, v, e, rho0detJ0)          # torch.cuda float64 tensors
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libblastcf.so")
_lib = None

OK, EINVAL, EUNSUPPORTED, ENOMEM, ECUDA, ENCCL = range(6)


class BlastCFError(RuntimeError):
    def __init__(self, code: int, where: str):
        L = _lib
        name = L.blast_cf_error_string(code).decode() if L else str(code)
        msg = L.blast_cf_last_error().decode() if L else ""
        super().__init__(f"{where}: {name}: {msg}")
        self.code = code


class _Mesh(ctypes.Structure):
    _fields_ = [("dim", ctypes.c_int32), ("order", ctypes.c_int32), ("num_zones", ctypes.c_int64),
                ("num_nodes", ctypes.c_int64), ("zone_nodes", ctypes.c_void_p), ("x0", ctypes.c_void_p),
                ("zone_mat", ctypes.c_void_p), ("mat_gamma", ctypes.c_void_p), ("num_mats", ctypes.c_int32),
                ("rank", ctypes.c_int32), ("nranks", ctypes.c_int32), ("num_neighbors", ctypes.c_int32),
                ("nbr_rank", ctypes.c_void_p), ("nbr_offset", ctypes.c_void_p), ("nbr_nodes", ctypes.c_void_p)]


class Params(ctypes.Structure):
    """blast_cf_params (DESIGN.md §3 readings R8, R10, R11)."""
    _fields_ = [("cfl", ctypes.c_double), ("q_quad", ctypes.c_double), ("q_lin", ctypes.c_double),
                ("eps_switch", ctypes.c_double), ("h0", ctypes.c_double), ("use_viscosity", ctypes.c_int32),
                ("use_vorticity", ctypes.c_int32)]


class RK2Opts(ctypes.Structure):
    _fields_ = [("cg_rel_tol", ctypes.c_double), ("cg_max_iter", ctypes.c_int32), ("cg_check_every", ctypes.c_int32),
                ("wall_bc", ctypes.c_int32), ("box_lo", ctypes.c_double * 3), ("box_hi", ctypes.c_double * 3)]


class Info(ctypes.Structure):
    _fields_ = [("dim", ctypes.c_int32), ("order", ctypes.c_int32), ("nq", ctypes.c_int32), ("nk", ctypes.c_int32),
                ("nt", ctypes.c_int32), ("num_zones", ctypes.c_int64), ("num_nodes", ctypes.c_int64),
                ("h0", ctypes.c_double), ("zones_per_cta", ctypes.c_int32), ("threads_per_cta", ctypes.c_int32),
                ("num_ctas", ctypes.c_int32), ("smem_bytes", ctypes.c_int32), ("regs_per_thread", ctypes.c_int32),
                ("local_bytes", ctypes.c_int32), ("flops_per_zone", ctypes.c_double), ("alg_bytes", ctypes.c_double),
                ("kernels_per_eval", ctypes.c_int32), ("flops_per_zone_alg", ctypes.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


def lib():
    """Load libblastcf.so (in-tree).  Raises if it has not been built — there is no fallback."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_ipps_dongdkrtd14_b200.build` "
                          "(or __graft_entry__.build()); the corner force has no CPU fallback")
    if "BLAST_CF_NCCL_LIB" not in os.environ:
        try:
            from .build import nccl_lib
            os.environ["BLAST_CF_NCCL_LIB"] = nccl_lib()
        except Exception:
            pass
    L = ctypes.CDLL(LIB_PATH)
    vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    L.blast_cf_error_string.restype = ctypes.c_char_p
    L.blast_cf_error_string.argtypes = [ctypes.c_int]
    L.blast_cf_last_error.restype = ctypes.c_char_p
    L.blast_cf_default_params.argtypes = [ctypes.POINTER(Params)]
    L.blast_cf_create.argtypes = [ctypes.POINTER(_Mesh), ctypes.c_int, ctypes.c_int, ctypes.POINTER(Params), vp, vp,
                                  ctypes.POINTER(vp)]
    L.blast_cf_eval.argtypes = [vp] * 8
    L.blast_cf_eval_host.argtypes = [vp] * 8
    L.blast_cf_set_rho0detJ0_host.argtypes = [vp, vp]
    L.blast_cf_exchange_schedule.argtypes = [vp, ctypes.POINTER(i32), ctypes.POINTER(i64)]
    L.blast_cf_debug_exchange_times.argtypes = [vp, ctypes.POINTER(ctypes.c_float)]
    L.blast_cf_eval_debug_Fz.argtypes = [vp] * 6
    L.blast_cf_get_info.argtypes = [vp, ctypes.POINTER(Info)]
    L.blast_cf_set_timing.argtypes = [vp, ctypes.c_int]
    L.blast_cf_kernel_times.argtypes = [vp, ctypes.POINTER(ctypes.c_float)]
    L.blast_cf_destroy.argtypes = [vp]
    L.blast_cf_nccl_unique_id_size.argtypes = []
    L.blast_cf_nccl_get_unique_id.argtypes = [vp]
    L.blast_cf_exchange_plan.argtypes = [i32, i32, vp, vp, vp, i64, ctypes.POINTER(i64), vp, vp, vp]
    L.blast_cf_owner_mask.argtypes = [i32, i32, vp, vp, vp, i64, vp]
    L.blast_cf_debug_cta_dt.argtypes = [vp, vp, i64, ctypes.POINTER(i32), ctypes.POINTER(i32)]
    L.blast_cf_debug_stage_clocks.argtypes = [vp, vp, i64]
    L.blast_cf_eval_loopback.argtypes = [vp, ctypes.c_int, vp, vp, vp, vp, vp, vp, vp]
    L.blast_cf_p2p_export.argtypes = [vp, vp, ctypes.POINTER(i64)]
    L.blast_cf_p2p_connect.argtypes = [vp, vp, i64]
    L.blast_cf_exchange_transport.argtypes = [vp, ctypes.POINTER(i32)]
    L.blast_cf_p2p_enable.argtypes = [vp, ctypes.c_int]
    L.blast_cf_autotune.argtypes = [vp] * 8 + [ctypes.c_int, vp, ctypes.c_int, ctypes.POINTER(ctypes.c_int)]
    L.blast_cf_variant_name.argtypes = [vp, ctypes.c_int]
    L.blast_cf_variant_name.restype = ctypes.c_char_p
    L.blast_cf_rk2_default_opts.argtypes = [ctypes.POINTER(RK2Opts)]
    L.blast_cf_rk2_create.argtypes = [vp, ctypes.POINTER(_Mesh), vp, ctypes.POINTER(RK2Opts), vp]
    L.blast_cf_rk2_step.argtypes = [vp, vp, vp, vp, ctypes.c_double, ctypes.POINTER(ctypes.c_double),
                                    ctypes.POINTER(i32)]
    L.blast_cf_rk2_rates.argtypes = [vp] * 7 + [ctypes.POINTER(ctypes.c_double), ctypes.POINTER(i32)]
    L.blast_cf_rk2_mass_apply.argtypes = [vp, vp, vp]
    L.blast_cf_rk2_advance.argtypes = [vp, vp, vp, vp, ctypes.c_double, i32, ctypes.POINTER(ctypes.c_double),
                                       ctypes.POINTER(ctypes.c_double), ctypes.POINTER(i32), ctypes.POINTER(i32)]
    L.blast_cf_rk2_energy.argtypes = [vp, vp, vp, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]
    L.blast_cf_rk2_destroy.argtypes = [vp]
    L.blast_cf_rk2_setup_loopback.argtypes = [vp, ctypes.c_int]
    L.blast_cf_rk2_rates_loopback.argtypes = [vp, ctypes.c_int] + [vp] * 6 + [ctypes.POINTER(ctypes.c_double),
                                                                             ctypes.POINTER(i32)]
    L.blast_cf_rk2_energy_loopback.argtypes = [vp, ctypes.c_int, vp, vp, ctypes.POINTER(ctypes.c_double),
                                               ctypes.POINTER(ctypes.c_double)]
    for f in ("blast_cf_rk2_create", "blast_cf_rk2_step", "blast_cf_rk2_rates", "blast_cf_rk2_mass_apply",
              "blast_cf_rk2_energy", "blast_cf_rk2_destroy", "blast_cf_rk2_advance", "blast_cf_rk2_setup_loopback",
              "blast_cf_rk2_rates_loopback", "blast_cf_rk2_energy_loopback",
              "blast_cf_create", "blast_cf_eval", "blast_cf_eval_host", "blast_cf_set_rho0detJ0_host",
              "blast_cf_exchange_schedule", "blast_cf_debug_exchange_times", "blast_cf_eval_debug_Fz", "blast_cf_get_info",
              "blast_cf_set_timing", "blast_cf_kernel_times", "blast_cf_destroy", "blast_cf_nccl_unique_id_size",
              "blast_cf_nccl_get_unique_id", "blast_cf_exchange_plan", "blast_cf_owner_mask", "blast_cf_debug_cta_dt",
              "blast_cf_debug_stage_clocks", "blast_cf_eval_loopback", "blast_cf_autotune", "blast_cf_p2p_export",
              "blast_cf_p2p_connect", "blast_cf_exchange_transport", "blast_cf_p2p_enable"):
        getattr(L, f).restype = ctypes.c_int
    _lib = L
    return L


def _check(rc: int, where: str):
    if rc != OK:
        raise BlastCFError(rc, where)


def default_params() -> Params:
    p = Params()
    lib().blast_cf_default_params(ctypes.byref(p))
    return p


def _ptr(a: Optional[np.ndarray], dtype) -> Optional[int]:
    if a is None:
        return None
    assert a.dtype == dtype and a.flags.c_contiguous, (a.dtype, dtype)
    return a.ctypes.data


def exchange_plan(rank: int, nbr_rank: np.ndarray, nbr_offset: np.ndarray, nbr_nodes: np.ndarray):
    """The library's shared-node summation plan (host only; see blast_cf_exchange_plan)."""
    nbr_rank = np.ascontiguousarray(nbr_rank, dtype=np.int32)
    nbr_offset = np.ascontiguousarray(nbr_offset, dtype=np.int64)
    nbr_nodes = np.ascontiguousarray(nbr_nodes, dtype=np.int32)
    cap = int(2 * len(nbr_nodes) + 2)
    uniq = np.zeros(cap, np.int32)
    sptr = np.zeros(cap + 1, np.int64)
    src = np.zeros(cap, np.int64)
    nu = ctypes.c_int64(0)
    _check(lib().blast_cf_exchange_plan(rank, len(nbr_rank), _ptr(nbr_rank, np.int32), _ptr(nbr_offset, np.int64),
                                        _ptr(nbr_nodes, np.int32), cap, ctypes.byref(nu), uniq.ctypes.data,
                                        sptr.ctypes.data, src.ctypes.data), "blast_cf_exchange_plan")
    n = nu.value
    return uniq[:n].copy(), sptr[:n + 1].copy(), src[:sptr[n]].copy()


def owner_mask(rank: int, nbr_rank: np.ndarray, nbr_offset: np.ndarray, nbr_nodes: np.ndarray, num_nodes: int):
    """The library's owner weights of a rank's local nodes (host only; see blast_cf_owner_mask)."""
    nbr_rank = np.ascontiguousarray(nbr_rank, dtype=np.int32)
    nbr_offset = np.ascontiguousarray(nbr_offset, dtype=np.int64)
    nbr_nodes = np.ascontiguousarray(nbr_nodes, dtype=np.int32)
    out = np.zeros(max(int(num_nodes), 1))
    _check(lib().blast_cf_owner_mask(rank, len(nbr_rank), _ptr(nbr_rank, np.int32), _ptr(nbr_offset, np.int64),
                                     _ptr(nbr_nodes, np.int32), int(num_nodes), out.ctypes.data), "blast_cf_owner_mask")
    return out[:int(num_nodes)]


class CornerForce:
    """Handle around blast_cf_create / blast_cf_eval.

    Mesh arrays are host numpy arrays (copied at create).  eval() takes torch.cuda float64 tensors
    in the layouts of include/blast_cf.h and returns (F1 [dim][nodes], FTv [Z][Nt], dt [1]) tensors.
    """

    def __init__(self, zone_nodes: np.ndarray, x0: np.ndarray, order: int, dim: int,
                 zone_mat: Optional[np.ndarray] = None, mat_gamma=(1.4,), params: Optional[Params] = None,
                 stream=None, rank: int = 0, nranks: int = 1, nbr_rank=None, nbr_offset=None, nbr_nodes=None,
                 nccl_unique_id: Optional[bytes] = None, device=None):
        import torch
        L = lib()
        self.dim, self.order = int(dim), int(order)
        self._zone_nodes = np.ascontiguousarray(zone_nodes, dtype=np.int32)
        self._x0 = np.ascontiguousarray(x0, dtype=np.float64)
        self._zone_mat = None if zone_mat is None else np.ascontiguousarray(zone_mat, dtype=np.int32)
        self._gamma = np.ascontiguousarray(np.asarray(mat_gamma, dtype=np.float64).reshape(-1))
        self.num_zones = int(self._zone_nodes.shape[0])
        self.num_nodes = int(self._x0.shape[1])
        self.device = torch.device("cuda", torch.cuda.current_device()) if device is None else torch.device(device)
        self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
        m = _Mesh()
        m.dim, m.order, m.num_zones, m.num_nodes = self.dim, self.order, self.num_zones, self.num_nodes
        m.zone_nodes = _ptr(self._zone_nodes, np.int32)
        m.x0 = _ptr(self._x0, np.float64)
        m.zone_mat = _ptr(self._zone_mat, np.int32)
        m.mat_gamma = _ptr(self._gamma, np.float64)
        m.num_mats = len(self._gamma)
        m.rank, m.nranks = int(rank), int(nranks)
        self._nbr = None
        uid = None
        if nranks > 1:
            self._nbr = (np.ascontiguousarray(nbr_rank, dtype=np.int32), np.ascontiguousarray(nbr_offset, dtype=np.int64),
                         np.ascontiguousarray(nbr_nodes, dtype=np.int32))
            m.num_neighbors = len(self._nbr[0])
            m.nbr_rank, m.nbr_offset, m.nbr_nodes = (_ptr(self._nbr[0], np.int32), _ptr(self._nbr[1], np.int64),
                                                     _ptr(self._nbr[2], np.int32))
            if nccl_unique_id is not None:   # None: loopback handle (eval_loopback, single GPU tests)
                assert len(nccl_unique_id) == L.blast_cf_nccl_unique_id_size()
                uid = ctypes.create_string_buffer(bytes(nccl_unique_id), len(nccl_unique_id))
        self.params = params if params is not None else default_params()
        h = ctypes.c_void_p()
        with torch.cuda.device(self.device):
            _check(L.blast_cf_create(ctypes.byref(m), self.order, self.dim, ctypes.byref(self.params),
                                     ctypes.c_void_p(self.stream.cuda_stream), uid, ctypes.byref(h)), "blast_cf_create")
        self._h = h
        self._mesh_struct = m   # the arrays it points to live in self (the integrator re-reads x0)
        self.info = self.get_info()

    # ------------------------------------------------------------------
    def get_info(self) -> dict:
        inf = Info()
        _check(lib().blast_cf_get_info(self._h, ctypes.byref(inf)), "blast_cf_get_info")
        return inf.as_dict()

    @property
    def nq(self):
        return (2 * self.order) ** self.dim

    @property
    def nt(self):
        return self.order ** self.dim

    def alloc_outputs(self):
        import torch
        F1 = torch.empty((self.dim, self.num_nodes), dtype=torch.float64, device=self.device)
        FTv = torch.empty((self.num_zones, self.nt), dtype=torch.float64, device=self.device)
        dt = torch.empty(1, dtype=torch.float64, device=self.device)
        return F1, FTv, dt

    @staticmethod
    def _dev(t, shape):
        import torch
        assert isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == torch.float64, "float64 CUDA tensor required"
        assert t.is_contiguous() and tuple(t.shape) == tuple(shape), (tuple(t.shape), shape)
        return ctypes.c_void_p(t.data_ptr())

    def eval(self, x, v, e, rho0detJ0, out=None):
        """Enqueue one corner-force evaluation on the handle's stream (no synchronization)."""
        F1, FTv, dt = out if out is not None else self.alloc_outputs()
        d, nn, Z = self.dim, self.num_nodes, self.num_zones
        _check(lib().blast_cf_eval(self._h, self._dev(x, (d, nn)), self._dev(v, (d, nn)), self._dev(e, (Z, self.nt)),
                                   self._dev(rho0detJ0, (Z, self.nq)), self._dev(F1, (d, nn)),
                                   self._dev(FTv, (Z, self.nt)), self._dev(dt, (1,))), "blast_cf_eval")
        return F1, FTv, dt

    def eval_host(self, x, v, e, rho0detJ0, out=None):
        """Host-buffer evaluation (numpy arrays or pinned CPU tensors); synchronous.  rho0detJ0=None: use the
        copy made resident by set_rho0detJ0_host (no upload per call)."""
        d, nn, Z = self.dim, self.num_nodes, self.num_zones
        if out is None:
            out = (np.empty((d, nn)), np.empty((Z, self.nt)), np.empty(1))

        def hp(a, shape):
            # the C side reads / writes 8 bytes per element of HOST memory: float64, CPU, contiguous
            if hasattr(a, "data_ptr"):
                import torch
                if not (a.dtype == torch.float64 and a.device.type == "cpu" and a.is_contiguous()
                        and tuple(a.shape) == tuple(shape)):
                    raise ValueError(f"eval_host needs contiguous float64 CPU tensors of shape {tuple(shape)}, got "
                                     f"{a.dtype} on {a.device} with shape {tuple(a.shape)}")
                return ctypes.c_void_p(a.data_ptr())
            if not (isinstance(a, np.ndarray) and a.dtype == np.float64 and a.flags.c_contiguous
                    and a.shape == tuple(shape)):
                raise ValueError(f"eval_host needs C-contiguous float64 arrays of shape {tuple(shape)}")
            return ctypes.c_void_p(a.ctypes.data)

        _check(lib().blast_cf_eval_host(self._h, hp(x, (d, nn)), hp(v, (d, nn)), hp(e, (Z, self.nt)),
                                        None if rho0detJ0 is None else hp(rho0detJ0, (Z, self.nq)),
                                        hp(out[0], (d, nn)), hp(out[1], (Z, self.nt)), hp(out[2], (1,))),
               "blast_cf_eval_host")
        return out

    def set_rho0detJ0_host(self, rho0detJ0):
        """Make the time-invariant rho0|J0| (host array) resident for eval_host(..., rho0detJ0=None, ...)."""
        a = rho0detJ0
        shape = (self.num_zones, self.nq)
        if hasattr(a, "data_ptr"):
            import torch
            if not (a.dtype == torch.float64 and a.device.type == "cpu" and a.is_contiguous() and tuple(a.shape) == shape):
                raise ValueError(f"set_rho0detJ0_host needs a contiguous float64 CPU tensor of shape {shape}")
            p = a.data_ptr()
        else:
            if not (isinstance(a, np.ndarray) and a.dtype == np.float64 and a.flags.c_contiguous and a.shape == shape):
                raise ValueError(f"set_rho0detJ0_host needs a C-contiguous float64 array of shape {shape}")
            p = a.ctypes.data
        _check(lib().blast_cf_set_rho0detJ0_host(self._h, ctypes.c_void_p(p)), "blast_cf_set_rho0detJ0_host")

    def eval_debug_Fz(self, x, v, e, rho0detJ0):
        import torch
        nk = (self.order + 1) ** self.dim
        Fz = torch.empty((self.num_zones, self.dim * nk, self.nt), dtype=torch.float64, device=self.device)
        d, nn, Z = self.dim, self.num_nodes, self.num_zones
        _check(lib().blast_cf_eval_debug_Fz(self._h, self._dev(x, (d, nn)), self._dev(v, (d, nn)),
                                            self._dev(e, (Z, self.nt)), self._dev(rho0detJ0, (Z, self.nq)),
                                            self._dev(Fz, Fz.shape)), "blast_cf_eval_debug_Fz")
        return Fz

    def autotune(self, x, v, e, rho0detJ0, reps: int = 3):
        """Time every candidate corner-force kernel on these inputs and keep the fastest
        (blast_cf_autotune).  Returns {variant name: ms} and sets self.variant."""
        F1, FTv, dt = self.alloc_outputs()
        ms = (ctypes.c_double * 16)()
        n = ctypes.c_int(0)
        d, nn, Z = self.dim, self.num_nodes, self.num_zones
        _check(lib().blast_cf_autotune(self._h, self._dev(x, (d, nn)), self._dev(v, (d, nn)), self._dev(e, (Z, self.nt)),
                                       self._dev(rho0detJ0, (Z, self.nq)), self._dev(F1, (d, nn)),
                                       self._dev(FTv, (Z, self.nt)), self._dev(dt, (1,)), int(reps), ms, 16,
                                       ctypes.byref(n)), "blast_cf_autotune")
        self.info = self.get_info()
        return {lib().blast_cf_variant_name(self._h, i).decode(): ms[i] for i in range(n.value)}

    @property
    def variant(self) -> str:
        return lib().blast_cf_variant_name(self._h, -1).decode()

    def debug_cta_dt(self):
        """(per-CTA min dt of the last eval, zones per CTA) — tests only."""
        n, z = ctypes.c_int32(0), ctypes.c_int32(0)
        L = lib()
        _check(L.blast_cf_debug_cta_dt(self._h, None, 0, ctypes.byref(n), ctypes.byref(z)), "blast_cf_debug_cta_dt")
        out = np.zeros(max(n.value, 1))
        _check(L.blast_cf_debug_cta_dt(self._h, out.ctypes.data, len(out), ctypes.byref(n), ctypes.byref(z)),
               "blast_cf_debug_cta_dt")
        return out[:n.value], z.value

    def debug_stage_clocks(self):
        """[num_ctas][16] clock64 stamps at KB1's stage barriers (needs BLAST_CF_PROFILE=1 at create)."""
        n = self.info["num_ctas"]
        out = np.zeros((n, 16), dtype=np.int64)
        _check(lib().blast_cf_debug_stage_clocks(self._h, out.ctypes.data, out.size), "blast_cf_debug_stage_clocks")
        return out

    def exchange_schedule(self):
        """(0 single rank | 1 single round | 2 overlap, number of boundary zones) — blast_cf_exchange_schedule."""
        nb, mode = ctypes.c_int64(0), ctypes.c_int32(0)
        _check(lib().blast_cf_exchange_schedule(self._h, ctypes.byref(mode), ctypes.byref(nb)), "blast_cf_exchange_schedule")
        return mode.value, nb.value

    TRANSPORTS = {0: "single rank", 1: "nccl", 2: "loopback", 3: "p2p"}

    def exchange_transport(self) -> str:
        """How eval moves the shared rows and dt: blast_cf_exchange_transport."""
        t = ctypes.c_int32(0)
        _check(lib().blast_cf_exchange_transport(self._h, ctypes.byref(t)), "blast_cf_exchange_transport")
        return self.TRANSPORTS[t.value]

    def p2p_connect(self, group=None, required=True):
        """Switch the exchange to the peer-memory transport (blast_cf_p2p_export / _connect): a collective over
        the torch process group `group` (any backend; its rank r must be mesh rank r).  The records are
        all-gathered as opaque bytes; the library maps the peers' mailboxes itself.  All ranks agree on the
        outcome: if the mapping failed on any rank, every rank stays on NCCL (needs the NCCL communicator of
        create) and, with required=True, raises.  Returns whether the peer-memory transport is in use."""
        import torch.distributed as dist
        L = lib()
        n = ctypes.c_int64(0)
        _check(L.blast_cf_p2p_export(self._h, None, ctypes.byref(n)), "blast_cf_p2p_export")
        buf = ctypes.create_string_buffer(n.value)
        _check(L.blast_cf_p2p_export(self._h, buf, ctypes.byref(n)), "blast_cf_p2p_export")
        recs = [None] * dist.get_world_size(group)
        dist.all_gather_object(recs, buf.raw, group=group)
        rc = L.blast_cf_p2p_connect(self._h, b"".join(recs), n.value)
        err = None if rc == 0 else f"blast_cf_p2p_connect: {L.blast_cf_last_error().decode()}"
        errs = [None] * len(recs)
        dist.all_gather_object(errs, err, group=group)
        failed = [e for e in errs if e is not None]
        self._p2p_group = group if group is not None else dist.group.WORLD   # the mailbox exists either way
        if failed:
            if rc == 0:
                _check(L.blast_cf_p2p_enable(self._h, 0), "blast_cf_p2p_enable")
            if required:
                raise RuntimeError(f"peer-memory transport unavailable: {failed[0]}")
            self.p2p_error = failed[0]
            return False
        self.info = self.get_info()   # kernels_per_eval of the new transport
        return True

    def debug_exchange_times(self):
        ms = (ctypes.c_float * 3)()
        _check(lib().blast_cf_debug_exchange_times(self._h, ms), "blast_cf_debug_exchange_times")
        return list(ms)

    def set_timing(self, enable: bool):
        _check(lib().blast_cf_set_timing(self._h, int(enable)), "blast_cf_set_timing")

    def kernel_times(self):
        ms = (ctypes.c_float * 3)()
        _check(lib().blast_cf_kernel_times(self._h, ms), "blast_cf_kernel_times")
        return list(ms)

    def close(self):
        """Destroy the handle.  A peer-memory connected handle first synchronizes its device and waits for the
        whole process group (a peer may still be writing into this rank's mailbox), so every rank must call
        close() explicitly; without that (garbage collection) its mailbox is left allocated."""
        if getattr(self, "_h", None):
            if getattr(self, "_p2p_group", None) is not None:
                import torch
                import torch.distributed as dist
                torch.cuda.synchronize(self.device)
                dist.barrier(group=self._p2p_group)
                self._p2p_group = None
            lib().blast_cf_destroy(self._h)
            self._h = None

    def _abandon(self):   # garbage collection of a connected handle: never free a mailbox a peer may write
        self._h = None

    def __del__(self):
        try:
            if getattr(self, "_p2p_group", None) is not None:
                self._abandon()
            else:
                self.close()
        except Exception:
            pass


def rk2_default_opts() -> RK2Opts:
    o = RK2Opts()
    lib().blast_cf_rk2_default_opts(ctypes.byref(o))
    return o


class RK2:
    """The time integrator around a CornerForce handle (blast_cf_rk2_*).

    State arrays are torch.cuda float64 tensors x, v [dim][nodes], e [Z][Nt], advanced in place.
    """

    def __init__(self, cf: CornerForce, rho0detJ0: np.ndarray, opts: Optional[RK2Opts] = None, **kw):
        self.cf = cf
        self._R = np.ascontiguousarray(rho0detJ0, dtype=np.float64)
        assert self._R.shape == (cf.num_zones, cf.nq)
        self.opts = opts if opts is not None else rk2_default_opts()
        for k_, v_ in kw.items():
            setattr(self.opts, k_, v_)
        h = ctypes.c_void_p()
        _check(lib().blast_cf_rk2_create(cf._h, ctypes.byref(cf._mesh_struct), self._R.ctypes.data,
                                         ctypes.byref(self.opts), ctypes.byref(h)), "blast_cf_rk2_create")
        self._h = h

    def _shapes(self):
        c = self.cf
        return (c.dim, c.num_nodes), (c.num_zones, c.nt)

    def step(self, x, v, e, dt: float):
        """One RK2-average step in place; returns (dt estimate, CG iterations)."""
        sx, se = self._shapes()
        d = ctypes.c_double(0.0)
        it = ctypes.c_int32(0)
        _check(lib().blast_cf_rk2_step(self._h, self.cf._dev(x, sx), self.cf._dev(v, sx), self.cf._dev(e, se),
                                       float(dt), ctypes.byref(d), ctypes.byref(it)), "blast_cf_rk2_step")
        return d.value, it.value

    def advance(self, x, v, e, t_final: float, dt: float, max_steps: int):
        """March in place to t_final (<= max_steps accepted steps) with the R24 step control.
        Returns (t reached, next dt, steps, rejected)."""
        sx, se = self._shapes()
        d, tr = ctypes.c_double(dt), ctypes.c_double(0.0)
        ns, nr = ctypes.c_int32(0), ctypes.c_int32(0)
        _check(lib().blast_cf_rk2_advance(self._h, self.cf._dev(x, sx), self.cf._dev(v, sx), self.cf._dev(e, se),
                                          float(t_final), int(max_steps), ctypes.byref(d), ctypes.byref(tr),
                                          ctypes.byref(ns), ctypes.byref(nr)), "blast_cf_rk2_advance")
        return tr.value, d.value, ns.value, nr.value

    def rates(self, x, v, e, vbar=None):
        """(dv/dt, de/dt, dt estimate, CG iterations) at state (x, v, e); de/dt uses vbar (default v)."""
        import torch
        sx, se = self._shapes()
        dv = torch.empty(sx, dtype=torch.float64, device=self.cf.device)
        de = torch.empty(se, dtype=torch.float64, device=self.cf.device)
        d = ctypes.c_double(0.0)
        it = ctypes.c_int32(0)
        _check(lib().blast_cf_rk2_rates(self._h, self.cf._dev(x, sx), self.cf._dev(v, sx), self.cf._dev(e, se),
                                        None if vbar is None else self.cf._dev(vbar, sx), self.cf._dev(dv, sx),
                                        self.cf._dev(de, se), ctypes.byref(d), ctypes.byref(it)), "blast_cf_rk2_rates")
        return dv, de, d.value, it.value

    def mass_apply(self, u):
        import torch
        sx, _ = self._shapes()
        out = torch.empty(sx, dtype=torch.float64, device=self.cf.device)
        _check(lib().blast_cf_rk2_mass_apply(self._h, self.cf._dev(u, sx), self.cf._dev(out, sx)),
               "blast_cf_rk2_mass_apply")
        return out

    def energy(self, v, e):
        """(kinetic, internal) discrete energies."""
        sx, se = self._shapes()
        ke, ie = ctypes.c_double(0.0), ctypes.c_double(0.0)
        _check(lib().blast_cf_rk2_energy(self._h, self.cf._dev(v, sx), self.cf._dev(e, se), ctypes.byref(ke),
                                         ctypes.byref(ie)), "blast_cf_rk2_energy")
        return ke.value, ie.value

    def close(self):
        if getattr(self, "_h", None):
            lib().blast_cf_rk2_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def eval_loopback(handles, xs, vs, es, rs):
    """Evaluate the ranks of a loopback group on one GPU (see blast_cf_eval_loopback); returns per-rank
    (F1, FTv, dt) tensors."""
    n = len(handles)
    outs = [h.alloc_outputs() for h in handles]
    P = ctypes.c_void_p * n
    hs = P(*[h._h for h in handles])
    arr = lambda ts: P(*[ctypes.c_void_p(t.data_ptr()) for t in ts])
    _check(lib().blast_cf_eval_loopback(hs, n, arr(xs), arr(vs), arr(es), arr(rs), arr([o[0] for o in outs]),
                                        arr([o[1] for o in outs]), arr([o[2] for o in outs])), "blast_cf_eval_loopback")
    return outs


def rk2_setup_loopback(rk2s):
    """Complete the creation of a loopback group's integrators (blast_cf_rk2_setup_loopback)."""
    P = ctypes.c_void_p * len(rk2s)
    _check(lib().blast_cf_rk2_setup_loopback(P(*[r._h for r in rk2s]), len(rk2s)), "blast_cf_rk2_setup_loopback")


def rk2_rates_loopback(rk2s, xs, vs, es, vbars=None):
    """RK2.rates of a whole loopback group (one GPU): per-rank (dv/dt, de/dt) tensors, group dt, CG iterations."""
    import torch
    n = len(rk2s)
    P = ctypes.c_void_p * n
    arr = lambda ts: P(*[None if t is None else ctypes.c_void_p(t.data_ptr()) for t in ts])
    dvs = [torch.empty((r.cf.dim, r.cf.num_nodes), dtype=torch.float64, device=r.cf.device) for r in rk2s]
    des = [torch.empty((r.cf.num_zones, r.cf.nt), dtype=torch.float64, device=r.cf.device) for r in rk2s]
    d, it = ctypes.c_double(0.0), ctypes.c_int32(0)
    _check(lib().blast_cf_rk2_rates_loopback(P(*[r._h for r in rk2s]), n, arr(xs), arr(vs), arr(es),
                                             arr(vbars if vbars is not None else [None] * n), arr(dvs), arr(des),
                                             ctypes.byref(d), ctypes.byref(it)), "blast_cf_rk2_rates_loopback")
    return dvs, des, d.value, it.value


def rk2_energy_loopback(rk2s, vs, es):
    """(kinetic, internal) energies of a whole loopback group."""
    n = len(rk2s)
    P = ctypes.c_void_p * n
    arr = lambda ts: P(*[ctypes.c_void_p(t.data_ptr()) for t in ts])
    ke, ie = ctypes.c_double(0.0), ctypes.c_double(0.0)
    _check(lib().blast_cf_rk2_energy_loopback(P(*[r._h for r in rk2s]), n, arr(vs), arr(es), ctypes.byref(ke),
                                              ctypes.byref(ie)), "blast_cf_rk2_energy_loopback")
    return ke.value, ie.value


def nccl_unique_id() -> bytes:
    L = lib()
    n = L.blast_cf_nccl_unique_id_size()
    buf = ctypes.create_string_buffer(n)
    _check(L.blast_cf_nccl_get_unique_id(buf), "blast_cf_nccl_get_unique_id")
    return buf.raw


def from_synth(mesh, params: Optional[Params] = None, part=None, nccl_uid: Optional[bytes] = None, **kw) -> CornerForce:
    """Create a CornerForce from a synth.Mesh (and, for nranks > 1, a synth.RankPart)."""
    if part is None or part.nranks == 1:
        return CornerForce(mesh.zone_nodes, mesh.x0, mesh.order, mesh.dim, mesh.zone_mat, mesh.mat_gamma, params, **kw)
    lm = part.local_mesh(mesh)
    return CornerForce(lm.zone_nodes, lm.x0, lm.order, lm.dim, lm.zone_mat, lm.mat_gamma, params, rank=part.rank,
                       nranks=part.nranks, nbr_rank=part.nbr_rank, nbr_offset=part.nbr_offset,
                       nbr_nodes=part.nbr_nodes, nccl_unique_id=nccl_uid, **kw)
