"""ctypes declarations of libcagmres.so (include/cagmres.h).  Argument marshalling only.

The library is the product: there is no Python or CPU fallback.  If libcagmres.so is
missing this module raises; build it with ``python -m paper_conf_ipps_yamazakiathd14_b200.build``
(or ``__graft_entry__.build()``).
"""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libcagmres.so")

OK, NOT_CONVERGED = 0, 1
EINVAL, ECUDA, ENCCL, EBREAKDOWN, ENOMEM, EGHOST, ENOTSUP = -1, -2, -3, -4, -5, -6, -7
MONOMIAL, NEWTON, GMRES = 0, 1, 2
CHOLQR, SVQR, CGS, MGS, CAQR = 0, 1, 2, 3, 4
REORTH, BORTH_MGS, ONEPASS, SVQR_RETRY = 0x100, 0x200, 0x400, 0x800
OPT_MPK_WAVE, OPT_WAVE_CHUNK, OPT_WAVE_CTAS, OPT_WAVE_LAG, OPT_FUSE, OPT_SPMV = 1, 3, 4, 5, 6, 7


class CSRStruct(C.Structure):
    _fields_ = [("n", C.c_int64), ("nnz", C.c_int64),
                ("rowptr", C.c_void_p), ("colind", C.c_void_p), ("val", C.c_void_p),
                ("row_begin", C.c_int64), ("row_end", C.c_int64),
                ("own_begin", C.c_int64), ("own_end", C.c_int64)]


class StatsStruct(C.Structure):
    _fields_ = [("cycles", C.c_int), ("iters", C.c_int), ("hist_cap", C.c_int),
                ("hist_len", C.c_int), ("rel_resid_hist", C.POINTER(C.c_double)),
                ("collect_timing", C.c_int),
                ("ms_mpk", C.c_double), ("ms_borth", C.c_double), ("ms_tsqr", C.c_double),
                ("ms_other", C.c_double), ("ms_total", C.c_double),
                ("bytes_mpk", C.c_double), ("bytes_borth", C.c_double),
                ("bytes_tsqr", C.c_double), ("bytes_other", C.c_double),
                ("spmv_launches", C.c_int), ("ms_spmv", C.c_double), ("bytes_spmv", C.c_double),
                ("collect_diag", C.c_int), ("max_orth_err", C.c_double), ("max_gram_cond", C.c_double),
                ("ms_setup", C.c_double), ("retried_panels", C.c_int)]


class CagmresError(RuntimeError):
    def __init__(self, status, what=""):
        self.status = status
        msg = _lib.cagmres_strerror(status).decode() if _lib is not None else str(status)
        super().__init__(f"{what}: {msg} (status {status})")


_lib = None

_P = C.c_void_p
_I64 = C.c_int64
_PI64 = C.POINTER(C.c_int64)
_PI32 = C.POINTER(C.c_int32)
_PD = C.POINTER(C.c_double)

SIGNATURES = {
    "cagmres_strerror": ([C.c_int], C.c_char_p),
    "cagmres_create": ([C.POINTER(_P), C.POINTER(CSRStruct), C.c_int, C.c_int, C.c_int, C.c_int], C.c_int),
    "cagmres_create_dist": ([C.POINTER(_P), C.POINTER(CSRStruct), _PI64, C.c_int, C.c_int, C.c_int,
                             C.c_int, _P, C.c_int, C.c_int, C.c_int], C.c_int),
    "cagmres_destroy": ([_P], C.c_int),
    "cagmres_group_create": ([C.POINTER(_P), C.c_int, C.POINTER(C.c_int)], C.c_int),
    "cagmres_group_destroy": ([_P], C.c_int),
    "cagmres_create_group": ([C.POINTER(_P), C.POINTER(CSRStruct), _PI64, C.c_int, C.c_int, C.c_int,
                              C.c_int, _P, C.c_int], C.c_int),
    "cagmres_set_stream": ([_P, _P], C.c_int),
    "cagmres_set_option": ([_P, C.c_int, C.c_int64], C.c_int),
    "cagmres_get_option": ([_P, C.c_int, C.POINTER(C.c_int64)], C.c_int),
    "cagmres_sizes": ([_P, _PI64, _PI64, _PI64], C.c_int),
    "cagmres_set_shifts": ([_P, _PD, _PD, C.c_int], C.c_int),
    "cagmres_get_shifts": ([_P, _PD, _PD, C.c_int, C.POINTER(C.c_int)], C.c_int),
    "cagmres_mpk": ([_P, _P, _P, _I64, C.c_int], C.c_int),
    "cagmres_borth": ([_P, _P, _I64, C.c_int, _P, _I64, C.c_int, _P], C.c_int),
    "cagmres_tsqr": ([_P, _P, _I64, C.c_int, _P, C.c_int], C.c_int),
    "cagmres_solve": ([_P, _P, _P, C.c_double, C.c_int, C.POINTER(StatsStruct)], C.c_int),
    "cagmres_kernel_launches": ([], C.c_int64),
    "cagmres_plan_create": ([C.POINTER(_P), C.POINTER(CSRStruct), _PI64, C.c_int, C.c_int, C.c_int], C.c_int),
    "cagmres_plan_destroy": ([_P], C.c_int),
    "cagmres_plan_info": ([_P, _PI64, _PI64, _PI64, _PI64, _PI64], C.c_int),
    "cagmres_plan_ext_rows": ([_P, _PI64], C.c_int),
    "cagmres_plan_ext_csr": ([_P, _PI64, _PI32, _PD], C.c_int),
    "cagmres_plan_requests": ([_P, _PI64, _PI64, _PI32], C.c_int),
    "cagmres_plan_recv_index": ([_P, _PI64], C.c_int),
    "cagmres_plan_set_sends": ([_P, _PI64, _PI64, _PI32], C.c_int),
    "cagmres_plan_send_index": ([_P, _PI64], C.c_int),
    "cagmres_plan_sell": ([_P, _PI64, _PI64, _PI64, _PI64, _PI64, _PI32, _PD], C.c_int),
    "cagmres_host_sym_eigvals": ([_PD, C.c_int, C.c_int, _PD], C.c_int),
    "cagmres_host_eigvals": ([_PD, C.c_int, C.c_int, _PD, _PD], C.c_int),
    "cagmres_host_rcm": ([_I64, _PI64, _PI32, _PI64], C.c_int),
    "cagmres_host_partition": ([_I64, _PI64, _PI32, C.c_int, C.c_double, _PI32, _PI64], C.c_int),
    "cagmres_host_partition_order": ([_I64, _PI32, C.c_int, _PI64, _PI64], C.c_int),
    "cagmres_host_permute": ([_I64, _PI64, _PI32, _PD, _PI64, _PI64, _PI32, _PD], C.c_int),
    "cagmres_host_leja": ([_PD, _PD, C.c_int, C.c_int, _PD, _PD, C.c_int, C.POINTER(C.c_int)], C.c_int),
    "cagmres_host_change_of_basis": ([_PD, _PD, C.c_int, _PD], C.c_int),
    "cagmres_host_hessenberg_update": ([_PD, C.c_int, C.c_int, C.c_int, _PD, C.c_int, _PD], C.c_int),
    "cagmres_host_givens_ls": ([_PD, C.c_int, C.c_int, C.c_double, _PD, _PD], C.c_int),
}


def load():
    """Load libcagmres.so (raises if it has not been built — no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build it with "
                           "`python -m paper_conf_ipps_yamazakiathd14_b200.build`")
    lib = C.CDLL(LIB_PATH)
    for name, (args, res) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = res
    _lib = lib
    return lib


def check(status, what):
    if status < 0:
        raise CagmresError(status, what)
    return status


def dptr(a):
    """ctypes double* of a C-contiguous float64 numpy array."""
    return a.ctypes.data_as(_PD)


def i64ptr(a):
    return a.ctypes.data_as(_PI64)


def i32ptr(a):
    return a.ctypes.data_as(_PI32)
