"""Wrappers of the host-only parts of libcagmres.so (no GPU needed): the multi-GPU setup plan
(boundary sets P:60-64, extended numbering, halo lists) and the small dense host algorithms
(Ritz values, Leja order, change of basis, Hessenberg update, Givens LS)."""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _lib as L
from .solver import _csr_struct


class Plan:
    def __init__(self, A, row_starts, rank, s):
        self._lib = L.load()
        rs = np.ascontiguousarray(row_starts, dtype=np.int64)
        self.nranks = len(rs) - 1
        st, keep = _csr_struct(A, rs[rank], rs[rank + 1])
        self._p = C.c_void_p()
        L.check(self._lib.cagmres_plan_create(C.byref(self._p), C.byref(st), L.i64ptr(rs),
                                              self.nranks, int(rank), int(s)), "plan_create")
        del keep
        self.s = int(s)
        a = [C.c_int64() for _ in range(4)]
        ll = np.zeros(self.s + 1, dtype=np.int64)
        self._lib.cagmres_plan_info(self._p, *[C.byref(x) for x in a], L.i64ptr(ll))
        self.n_loc, self.n_ext, self.n_mat, self.nnz_mat = (x.value for x in a)
        self.level_len = ll

    def __del__(self):
        try:
            if self._p:
                self._lib.cagmres_plan_destroy(self._p)
        except Exception:
            pass

    def ext_rows(self):
        g = np.zeros(self.n_ext, dtype=np.int64)
        L.check(self._lib.cagmres_plan_ext_rows(self._p, L.i64ptr(g)), "ext_rows")
        return g

    def ext_csr(self):
        rp = np.zeros(self.n_mat + 1, dtype=np.int64)
        ci = np.zeros(max(self.nnz_mat, 1), dtype=np.int32)
        va = np.zeros(max(self.nnz_mat, 1), dtype=np.float64)
        L.check(self._lib.cagmres_plan_ext_csr(self._p, L.i64ptr(rp), L.i32ptr(ci), L.dptr(va)), "ext_csr")
        return rp, ci[:self.nnz_mat], va[:self.nnz_mat]

    def requests(self):
        cnt = np.zeros(self.nranks, dtype=np.int64)
        self._lib.cagmres_plan_requests(self._p, L.i64ptr(cnt), None, None)
        tot = int(cnt.sum())
        g = np.zeros(max(tot, 1), dtype=np.int64)
        lv = np.zeros(max(tot, 1), dtype=np.int32)
        L.check(self._lib.cagmres_plan_requests(self._p, L.i64ptr(cnt), L.i64ptr(g), L.i32ptr(lv)), "requests")
        ext = np.zeros(max(tot, 1), dtype=np.int64)
        L.check(self._lib.cagmres_plan_recv_index(self._p, L.i64ptr(ext)), "recv_index")
        return cnt, g[:tot], lv[:tot], ext[:tot]

    def set_sends(self, counts, gids, levels):
        counts = np.ascontiguousarray(counts, dtype=np.int64)
        gids = np.ascontiguousarray(gids if len(gids) else np.zeros(1), dtype=np.int64)
        levels = np.ascontiguousarray(levels if len(levels) else np.zeros(1), dtype=np.int32)
        L.check(self._lib.cagmres_plan_set_sends(self._p, L.i64ptr(counts), L.i64ptr(gids),
                                                 L.i32ptr(levels)), "set_sends")
        self._send_total = int(counts.sum())

    def sell(self):
        """The SELL-32 layout create() uploads (cagmres_plan_sell): dict of numpy arrays."""
        ns, nd, nv = C.c_int64(), C.c_int64(), C.c_int64()
        L.check(self._lib.cagmres_plan_sell(self._p, C.byref(ns), C.byref(nd), C.byref(nv), None, None, None,
                                            None), "plan_sell")
        sptr = np.zeros(ns.value + 1, dtype=np.int64)
        sinfo = np.zeros(max(ns.value, 1), dtype=np.int64)
        dcol = np.zeros(max(nd.value, 1), dtype=np.int32)
        val = np.zeros(max(nv.value, 1), dtype=np.float64)
        L.check(self._lib.cagmres_plan_sell(self._p, None, None, None, L.i64ptr(sptr), L.i64ptr(sinfo),
                                            L.i32ptr(dcol), L.dptr(val)), "plan_sell")
        return dict(sptr=sptr, sinfo=sinfo[:ns.value], dcol=dcol[:nd.value], val=val[:nv.value])

    def send_index(self):
        idx = np.zeros(max(self._send_total, 1), dtype=np.int64)
        L.check(self._lib.cagmres_plan_send_index(self._p, L.i64ptr(idx)), "send_index")
        return idx[:self._send_total]


def sym_eigvals(A):
    """Eigenvalues (ascending) of a symmetric matrix by the library's host Jacobi routine."""
    lib = L.load()
    Af = np.asfortranarray(A, dtype=np.float64)
    n = Af.shape[0]
    ev = np.zeros(n)
    L.check(lib.cagmres_host_sym_eigvals(Af.ctypes.data_as(L._PD), n, n, L.dptr(ev)), "sym_eigvals")
    return ev


def eigvals(H, m):
    lib = L.load()
    Hf = np.asfortranarray(H, dtype=np.float64)
    wr, wi = np.zeros(m), np.zeros(m)
    L.check(lib.cagmres_host_eigvals(Hf.ctypes.data_as(L._PD), Hf.shape[0], m, L.dptr(wr), L.dptr(wi)), "eigvals")
    return wr + 1j * wi


def leja(theta, s):
    lib = L.load()
    theta = np.asarray(theta, dtype=np.complex128)
    wr = np.ascontiguousarray(theta.real)
    wi = np.ascontiguousarray(theta.imag)
    cap = 2 * len(theta) + 2
    ore, oim = np.zeros(cap), np.zeros(cap)
    nout = C.c_int()
    L.check(lib.cagmres_host_leja(L.dptr(wr), L.dptr(wi), len(theta), int(s), L.dptr(ore), L.dptr(oim),
                                  cap, C.byref(nout)), "leja")
    k = min(nout.value, cap)
    return ore[:k], oim[:k]


def change_of_basis(re, im, sb):
    lib = L.load()
    re = np.ascontiguousarray(np.r_[re, np.zeros(sb)][:sb], dtype=np.float64)
    im = np.ascontiguousarray(np.r_[im, np.zeros(sb)][:sb], dtype=np.float64)
    B = np.zeros((sb + 1, sb), order="F")
    L.check(lib.cagmres_host_change_of_basis(L.dptr(re), L.dptr(im), sb, B.ctypes.data_as(L._PD)), "cob")
    return B


def hessenberg_update(H, j, sb, Rt, B):
    lib = L.load()
    Hf = np.asfortranarray(H, dtype=np.float64).copy(order="F")
    Rf = np.asfortranarray(Rt, dtype=np.float64)
    Bf = np.asfortranarray(B, dtype=np.float64)
    L.check(lib.cagmres_host_hessenberg_update(Hf.ctypes.data_as(L._PD), Hf.shape[0], j, sb,
                                               Rf.ctypes.data_as(L._PD), Rf.shape[0],
                                               Bf.ctypes.data_as(L._PD)), "hessenberg_update")
    return Hf


def givens_ls(H, beta):
    lib = L.load()
    Hf = np.asfortranarray(H, dtype=np.float64)
    k = Hf.shape[1]
    y, res = np.zeros(k), np.zeros(k)
    L.check(lib.cagmres_host_givens_ls(Hf.ctypes.data_as(L._PD), Hf.shape[0], k, float(beta),
                                       L.dptr(y), L.dptr(res)), "givens_ls")
    return y, res


def rcm(A):
    """Reverse Cuthill-McKee permutation (perm[new] = old) of the symmetrised pattern of the
    n x n host CSR A (cagmres_host_rcm; NEXT-4 reordering for the MPK row partition)."""
    lib = L.load()
    rp = np.ascontiguousarray(A.rowptr, dtype=np.int64)
    ci = np.ascontiguousarray(A.colind, dtype=np.int32)
    perm = np.zeros(A.n, dtype=np.int64)
    L.check(lib.cagmres_host_rcm(int(A.n), L.i64ptr(rp), ci.ctypes.data_as(L._PI32), L.i64ptr(perm)), "rcm")
    return perm


def permute(A, perm):
    """B = P A P^T (cagmres_host_permute); returns a CSR of the same type as A."""
    import dataclasses
    lib = L.load()
    rp = np.ascontiguousarray(A.rowptr, dtype=np.int64)
    ci = np.ascontiguousarray(A.colind, dtype=np.int32)
    va = np.ascontiguousarray(A.val, dtype=np.float64)
    pm = np.ascontiguousarray(perm, dtype=np.int64)
    orp = np.zeros(A.n + 1, dtype=np.int64)
    oci = np.zeros(len(ci), dtype=np.int32)
    ova = np.zeros(len(va), dtype=np.float64)
    L.check(lib.cagmres_host_permute(int(A.n), L.i64ptr(rp), ci.ctypes.data_as(L._PI32), L.dptr(va),
                                     L.i64ptr(pm), L.i64ptr(orp), oci.ctypes.data_as(L._PI32), L.dptr(ova)),
            "permute")
    return dataclasses.replace(A, rowptr=orp, colind=oci, val=ova)


def partition(A, nparts, imbalance=0.03):
    """k-way partition of the symmetrised graph of the n x n host CSR A (cagmres_host_partition;
    NEXT-4): returns (part ids int32[n], edge cut)."""
    lib = L.load()
    rp = np.ascontiguousarray(A.rowptr, dtype=np.int64)
    ci = np.ascontiguousarray(A.colind, dtype=np.int32)
    part = np.zeros(A.n, dtype=np.int32)
    cut = C.c_int64()
    L.check(lib.cagmres_host_partition(int(A.n), L.i64ptr(rp), ci.ctypes.data_as(L._PI32), int(nparts),
                                       float(imbalance), part.ctypes.data_as(L._PI32), C.byref(cut)), "partition")
    return part, int(cut.value)


def partition_order(part, nparts):
    """(perm, row_starts): perm[new] = old groups every part into a contiguous block of rows."""
    lib = L.load()
    pt = np.ascontiguousarray(part, dtype=np.int32)
    perm = np.zeros(len(pt), dtype=np.int64)
    rs = np.zeros(nparts + 1, dtype=np.int64)
    L.check(lib.cagmres_host_partition_order(len(pt), pt.ctypes.data_as(L._PI32), int(nparts), L.i64ptr(perm),
                                             L.i64ptr(rs)), "partition_order")
    return perm, rs


def distribute(A, nranks, order="natural", imbalance=0.03):
    """Row distribution for the block-row create_dist under an ordering (NEXT-4,
    P:98-118): "natural" (A as given), "rcm" (reverse Cuthill-McKee, then equal blocks) or
    "kway" (partition(), parts made contiguous).  Returns (B = P A P^T, perm, row_starts);
    solve B y = P b, then x[perm] = y."""
    n = A.n
    if order == "natural":
        return A, np.arange(n, dtype=np.int64), np.array([(p * n) // nranks for p in range(nranks + 1)], dtype=np.int64)
    if order == "rcm":
        perm = rcm(A)
        return permute(A, perm), perm, np.array([(p * n) // nranks for p in range(nranks + 1)], dtype=np.int64)
    if order == "kway":
        part, _ = partition(A, nranks, imbalance)
        perm, rs = partition_order(part, nranks)
        return permute(A, perm), perm, rs
    raise ValueError(order)
