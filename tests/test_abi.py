"""The C-ABI library loads on a CPU-only host and exports every function include/blast_cf.h declares
(no compute calls here: there is no GPU).  Also the host-only exchange plan."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_dongdkrtd14_b200 as cf
from paper_conf_ipps_dongdkrtd14_b200 import build as cfbuild

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    cfbuild.build()
    return cf.lib()


def declared_functions():
    src = open(os.path.join(ROOT, "include", "blast_cf.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(blast_cf_\w+)\s*\(", src, flags=re.M)))


def test_exports_every_declared_symbol(L):
    names = declared_functions()
    assert len(names) >= 14, names
    for n in names:
        assert hasattr(L, n), n
    # and nothing is linked against the oracle
    out = os.popen(f"nm -D --defined-only {cf.LIB_PATH}").read()
    assert "oracle_" not in out


def test_no_nccl_link_dependency(L):
    """NCCL is dlopen'ed only for nranks > 1; single-GPU users do not need it."""
    out = os.popen(f"readelf -d {cf.LIB_PATH}").read()
    assert "libnccl" not in out


def test_error_strings_and_defaults(L):
    for code in range(6):
        assert L.blast_cf_error_string(code).startswith(b"BLAST_CF_")
    p = cf.default_params()
    assert (p.cfl, p.q_quad, p.q_lin, p.eps_switch, p.h0, p.use_viscosity, p.use_vorticity) == \
        (0.5, 2.0, 0.5, 1e-12, 0.0, 1, 1)
    assert L.blast_cf_nccl_unique_id_size() == 128


def test_create_rejects_bad_arguments_without_gpu(L):
    out = ctypes.c_void_p()
    m = cf._Mesh()
    m.dim, m.order = 3, 9
    rc = L.blast_cf_create(ctypes.byref(m), 9, 3, None, None, None, ctypes.byref(out))
    assert rc == cf.EUNSUPPORTED
    rc = L.blast_cf_create(None, 2, 3, None, None, None, ctypes.byref(out))
    assert rc == cf.EINVAL
    m.order = 2
    rc = L.blast_cf_create(ctypes.byref(m), 2, 2, None, None, None, ctypes.byref(out))   # dim mismatch
    assert rc == cf.EINVAL
    assert L.blast_cf_eval(None, None, None, None, None, None, None, None) == cf.EINVAL


def test_exchange_plan_orders_by_rank(L):
    # rank 1 shares node 5 with ranks 0 and 2, node 7 with rank 2 only, node 3 with rank 0 only
    nbr_rank = np.array([0, 2], np.int32)
    nbr_offset = np.array([0, 2, 4], np.int64)
    nbr_nodes = np.array([3, 5, 5, 7], np.int32)
    uniq, sptr, src = cf.exchange_plan(1, nbr_rank, nbr_offset, nbr_nodes)
    assert uniq.tolist() == [3, 5, 7]
    groups = [src[sptr[i]:sptr[i + 1]].tolist() for i in range(3)]
    # node 3: recv(row 0 from rank 0), own ; node 5: recv(row 1, rank 0), own, recv(row 2, rank 2) ;
    # node 7: own, recv(row 3, rank 2).  own partials come from a send row of the same node.
    assert groups[0] == [-1, 0]
    assert groups[1] == [-2, 1, -3]
    assert groups[2] == [3, -4]
