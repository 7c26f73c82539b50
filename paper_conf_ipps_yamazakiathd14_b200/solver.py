"""Thin Python binding of the CA-GMRES C ABI (include/cagmres.h): argument marshalling only.

Every step of the hot path runs in libcagmres.so (hand-written sm_100a kernels + NCCL);
PyTorch only provides device memory, the stream and (multi-GPU) the process group used to
broadcast the NCCL unique id.
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass, field

import numpy as np

from . import _lib as L

_BASIS = {"monomial": L.MONOMIAL, "newton": L.NEWTON, "gmres": L.GMRES}
_TSQR = {"cholqr": L.CHOLQR, "svqr": L.SVQR, "cgs": L.CGS, "mgs": L.MGS, "caqr": L.CAQR}


def orth_flags(tsqr="cholqr", reorth=False, borth="cgs", onepass=False):
    f = _TSQR[tsqr]
    if reorth:
        f |= L.REORTH
    if onepass:
        f |= L.ONEPASS
    if borth == "mgs":
        f |= L.BORTH_MGS
    return f


def _csr_struct(A, own_begin=None, own_end=None):
    rowptr = np.ascontiguousarray(A.rowptr, dtype=np.int64)
    colind = np.ascontiguousarray(A.colind, dtype=np.int32)
    val = np.ascontiguousarray(A.val, dtype=np.float64)
    rb = int(getattr(A, "row_begin", 0))
    re = rb + len(rowptr) - 1
    s = L.CSRStruct(int(A.n), int(rowptr[-1]), rowptr.ctypes.data, colind.ctypes.data,
                    val.ctypes.data, rb, re,
                    rb if own_begin is None else int(own_begin), re if own_end is None else int(own_end))
    return s, (rowptr, colind, val)


class Group:
    """In-process group of `nranks` ranks (cagmres_group_create): each rank's Solver is built
    and driven from its own Python thread (ctypes releases the GIL inside the library), on
    devices[rank] (default: all on the current device).  Runs the whole multi-rank device
    path — halo exchange, cross-rank sums — inside one process, e.g. on one GPU."""

    def __init__(self, nranks, devices=None):
        self._lib = L.load()
        self.nranks = int(nranks)
        self._g = C.c_void_p()
        if devices is None:
            import torch
            devices = [torch.cuda.current_device()] * self.nranks
        self.devices = [int(d) for d in devices]
        arr = (C.c_int * self.nranks)(*self.devices)
        L.check(self._lib.cagmres_group_create(C.byref(self._g), self.nranks, arr), "group_create")

    def close(self):
        if self._g:
            L.check(self._lib.cagmres_group_destroy(self._g), "group_destroy")
            self._g = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


@dataclass
class SolveStats:
    status: int
    cycles: int
    iters: int
    hist: np.ndarray
    ms: dict = field(default_factory=dict)
    bytes: dict = field(default_factory=dict)
    spmv_launches: int = 0
    max_orth_err: float = 0.0
    max_gram_cond: float = 0.0
    ms_setup: float = 0.0
    retried_panels: int = 0


class Solver:
    """CA-GMRES(s, m) handle on the current CUDA device (or one rank of a process group).

    A: host CSR with attributes n, rowptr (int64), colind (int32, global ids), val (float64)
       and row_begin (first global row described; 0 for the full matrix).
    group: a torch.distributed process group for the multi-GPU path (one process per GPU,
       NCCL), or a `Group` (in-process ranks, one thread each; pass `rank`); the caller
       passes this rank's owned rows plus >= (s-1)-hop ghost rows and row_starts.
    """

    def __init__(self, A, s, m, basis="newton", tsqr="cholqr", reorth=False, borth="cgs",
                 group=None, row_starts=None, device=None, onepass=False, rank=None, svqr_retry=False):
        import torch
        self._lib = L.load()
        self.s, self.m = int(s), int(m)
        self.basis = basis
        self.orth = orth_flags(tsqr, reorth, borth, onepass) | (L.SVQR_RETRY if svqr_retry else 0)
        self._h = C.c_void_p()
        if isinstance(group, Group):
            device = group.devices[rank]
        if device is None:
            device = torch.cuda.current_device()
        self.device = torch.device("cuda", device)
        torch.cuda.set_device(self.device)
        if isinstance(group, Group):
            rs = np.ascontiguousarray(row_starts, dtype=np.int64)
            st, keep = _csr_struct(A, rs[rank], rs[rank + 1])
            self._group = group                          # keeps the group alive
            L.check(self._lib.cagmres_create_group(C.byref(self._h), C.byref(st), L.i64ptr(rs), self.s, self.m,
                                                   _BASIS[basis], self.orth, group._g, int(rank)),
                    "cagmres_create_group")
        elif group is None:
            st, keep = _csr_struct(A)
            L.check(self._lib.cagmres_create(C.byref(self._h), C.byref(st), self.s, self.m,
                                             _BASIS[basis], self.orth), "cagmres_create")
        else:
            import torch.distributed as dist
            rank, nranks = dist.get_rank(group), dist.get_world_size(group)
            rs = np.ascontiguousarray(row_starts, dtype=np.int64)
            st, keep = _csr_struct(A, rs[rank], rs[rank + 1])
            uid = self._nccl_unique_id(group, rank)
            L.check(self._lib.cagmres_create_dist(
                C.byref(self._h), C.byref(st), L.i64ptr(rs), self.s, self.m, _BASIS[basis],
                self.orth, uid, rank, nranks, self.device.index), "cagmres_create_dist")
        del keep
        n_loc, n_ext, ldv = C.c_int64(), C.c_int64(), C.c_int64()
        self._lib.cagmres_sizes(self._h, C.byref(n_loc), C.byref(n_ext), C.byref(ldv))
        self.n_loc, self.n_ext, self.ldv = n_loc.value, n_ext.value, ldv.value
        self.use_torch_stream()

    @staticmethod
    def _nccl_unique_id(group, rank):
        """ncclUniqueId made by rank 0 (via the library's NCCL) and broadcast over `group`."""
        import torch
        import torch.distributed as dist
        buf = torch.zeros(128, dtype=torch.uint8)
        if rank == 0:
            lib = C.CDLL("libnccl.so.2")
            raw = (C.c_char * 128)()
            if lib.ncclGetUniqueId(raw) != 0:
                raise RuntimeError("ncclGetUniqueId failed")
            buf[:] = torch.frombuffer(bytearray(raw.raw), dtype=torch.uint8)
        if dist.get_backend(group) == "nccl":
            b = buf.cuda()
            dist.broadcast(b, src=dist.get_global_rank(group, 0), group=group)
            buf = b.cpu()
        else:
            dist.broadcast(buf, src=dist.get_global_rank(group, 0), group=group)
        return C.c_char_p(bytes(buf.numpy()))

    # ------------------------------------------------------------------------------------
    CUDA_STREAM_LEGACY = 1                       # cudaStreamLegacy: torch's default stream

    def use_torch_stream(self):
        """Enqueue on torch's current stream, so the library's work is ordered after whatever the
        caller queued on it (e.g. an asynchronous copy of b) — called before every device call.
        torch reports its default (legacy) stream as handle 0, which the C ABI reads as "the
        handle's own stream": pass cudaStreamLegacy for it instead.  In-process group ranks
        never share the legacy stream (their collectives wait on each other's events): a rank
        thread on the default stream keeps the handle's own stream."""
        import torch
        s = torch.cuda.current_stream(self.device).cuda_stream
        if not s:
            if getattr(self, "_group", None) is not None:
                return
            s = self.CUDA_STREAM_LEGACY
        if s != getattr(self, "_bound_stream", None):
            L.check(self._lib.cagmres_set_stream(self._h, C.c_void_p(s)), "set_stream")
            self._bound_stream = s

    OPTIONS = {"mpk_wave": 1, "wave_chunk": 3, "wave_ctas": 4, "wave_lag": 5, "fuse": 6, "spmv": 7, "gram": 8,
               "arnoldi": 9, "panel_tw": 10, "trsm": 11, "pdl": 12, "panel_pf": 13, "peer": 14, "graph": 15, "fold": 16, "serp": 17}

    def set_option(self, opt, value):
        """opt: "mpk_wave", "wave_chunk", "wave_ctas", "wave_lag", "fuse", "spmv", "gram", "arnoldi" (CAGMRES_OPT_*)."""
        L.check(self._lib.cagmres_set_option(self._h, self.OPTIONS[opt], int(value)), "set_option")

    def get_option(self, opt):
        v = C.c_int64(0)
        L.check(self._lib.cagmres_get_option(self._h, self.OPTIONS[opt], C.byref(v)), "get_option")
        return int(v.value)

    def close(self):
        if self._h:
            self._lib.cagmres_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_shifts(self, re, im=None):
        re = np.ascontiguousarray(re, dtype=np.float64)
        im = np.zeros_like(re) if im is None else np.ascontiguousarray(im, dtype=np.float64)
        L.check(self._lib.cagmres_set_shifts(self._h, L.dptr(re), L.dptr(im), len(re)), "set_shifts")

    def clear_shifts(self):
        """Forget the Newton shifts: the next solve runs its own first GMRES cycle."""
        L.check(self._lib.cagmres_set_shifts(self._h, None, None, 0), "set_shifts")

    def get_shifts(self):
        cap = 4 * self.m + 8
        re, im = np.zeros(cap), np.zeros(cap)
        cnt = C.c_int()
        L.check(self._lib.cagmres_get_shifts(self._h, L.dptr(re), L.dptr(im), cap, C.byref(cnt)), "get_shifts")
        return re[:cnt.value], im[:cnt.value]

    # ---- hot-path entry points (device tensors, owned rows) -------------------------------
    @staticmethod
    def _col_major(t, rows):
        """(ptr, ld) of a column-major view: a torch tensor of shape (cols, ld) row-major or
        (rows, cols) with stride(0) == 1."""
        assert t.dtype.is_floating_point and t.element_size() == 8 and t.is_cuda
        if t.dim() == 1:
            return t.data_ptr(), max(rows, 1)
        assert t.stride(0) == 1, "expect column-major (stride(0) == 1)"
        # torch reports stride 1 for a size-1 dimension: a single column has ld = its rows
        return t.data_ptr(), (t.stride(1) if t.size(1) > 1 else max(t.size(0), rows))

    def mpk(self, q, sb, out=None):
        import torch
        self.use_torch_stream()
        if out is None:
            out = torch.empty((sb + 1, self.n_loc), dtype=torch.float64, device=self.device).t()
        W, ldw = self._col_major(out, self.n_loc)
        L.check(self._lib.cagmres_mpk(self._h, C.c_void_p(q.data_ptr()), C.c_void_p(W), ldw, int(sb)), "mpk")
        return out

    def borth(self, Q, j, P, w):
        import torch
        self.use_torch_stream()
        Cm = torch.zeros((w, max(j, 1)), dtype=torch.float64, device=self.device)  # j x w col-major
        qp, ldq = self._col_major(Q, self.n_loc)
        pp, ldp = self._col_major(P, self.n_loc)
        L.check(self._lib.cagmres_borth(self._h, C.c_void_p(qp), ldq, int(j), C.c_void_p(pp), ldp,
                                        int(w), C.c_void_p(Cm.data_ptr())), "borth")
        return Cm.t()[:j]

    def tsqr(self, P, w, tsqr="cholqr", reorth=False, svqr_retry=False):
        import torch
        self.use_torch_stream()
        R = torch.zeros((w, w), dtype=torch.float64, device=self.device)
        pp, ldp = self._col_major(P, self.n_loc)
        st = self._lib.cagmres_tsqr(self._h, C.c_void_p(pp), ldp, int(w), C.c_void_p(R.data_ptr()),
                                    orth_flags(tsqr, reorth) | (L.SVQR_RETRY if svqr_retry else 0))
        L.check(st, "tsqr")
        return R.t()

    def solve(self, b, x=None, tol=1e-8, maxit=200, timing=False, diag=False):
        """Solve on device tensors b, x (owned rows, float64); x updated in place."""
        import torch
        self.use_torch_stream()
        if x is None:
            x = torch.zeros_like(b)
        hist = np.zeros(maxit + 1)
        st = L.StatsStruct()
        st.hist_cap = len(hist)
        st.rel_resid_hist = L.dptr(hist)
        st.collect_timing = int(timing) if timing else 0       # True/1: all phases, 2: MPK kernel only
        st.collect_diag = int(bool(diag))
        status = self._lib.cagmres_solve(self._h, C.c_void_p(b.data_ptr()), C.c_void_p(x.data_ptr()),
                                         float(tol), int(maxit), C.byref(st))
        L.check(status, "solve")
        stats = SolveStats(status=status, cycles=st.cycles, iters=st.iters, hist=hist[:st.hist_len].copy(),
                           ms=dict(mpk=st.ms_mpk, borth=st.ms_borth, tsqr=st.ms_tsqr, other=st.ms_other,
                                   total=st.ms_total, spmv=st.ms_spmv),
                           bytes=dict(mpk=st.bytes_mpk, borth=st.bytes_borth, tsqr=st.bytes_tsqr,
                                      other=st.bytes_other, spmv=st.bytes_spmv),
                           spmv_launches=st.spmv_launches, max_orth_err=st.max_orth_err,
                           max_gram_cond=st.max_gram_cond, ms_setup=st.ms_setup,
                           retried_panels=st.retried_panels)
        return x, stats
