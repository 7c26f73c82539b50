"""Seeded synthetic inputs shared by the oracle tests, the CUDA-path tests and bench.py.

This module holds NO arithmetic of the CA-GMRES method (no SpMV, no orthogonalisation,
no Krylov step).  It only builds CSR matrices and right-hand sides, deterministically,
from the recipes in DESIGN.md "Input recipe" (which restates SURVEY.md §8(d)).

Every random draw is u(seed, idx) = splitmix64(seed XOR idx) mapped to [-1, 1), so any
row range of a matrix can be generated independently and any partition of the rows sees
identical data (needed for the multi-GPU row-block distribution).

Matrices are returned as host CSR with int64 row pointers, int32 column indices
(global ids) and float64 values, columns sorted ascending inside each row, duplicates
summed.  ``rows=(r0, r1)`` generates only rows [r0, r1) (rowptr then starts at 0).
"""
from __future__ import annotations

from dataclasses import dataclass
import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x):
    """splitmix64 finaliser of (x + golden gamma); x is a uint64 array (wrapping)."""
    z = np.asarray(x, dtype=np.uint64) + _GOLDEN
    z = (z ^ (z >> np.uint64(30))) * _M1
    z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def u(seed: int, idx) -> np.ndarray:
    """Counter-based uniform draw in [-1, 1): 2*(splitmix64(seed ^ idx) >> 11)*2^-53 - 1."""
    with np.errstate(over="ignore"):
        x = np.uint64(seed) ^ np.asarray(idx, dtype=np.uint64)
        z = splitmix64(x)
    return (z >> np.uint64(11)).astype(np.float64) * (2.0 ** -52) - 1.0


@dataclass
class CSR:
    n: int                # global dimension
    row_begin: int        # first global row described
    rowptr: np.ndarray    # int64, len = nrows + 1, rowptr[0] == 0
    colind: np.ndarray    # int32 global column ids
    val: np.ndarray       # float64

    @property
    def nrows(self) -> int:
        return len(self.rowptr) - 1

    @property
    def row_end(self) -> int:
        return self.row_begin + self.nrows

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])

    def to_scipy(self):
        import scipy.sparse as sp
        return sp.csr_matrix((self.val, self.colind.astype(np.int64), self.rowptr),
                             shape=(self.nrows, self.n))


def _rows(n, rows):
    r0, r1 = (0, n) if rows is None else (int(rows[0]), int(rows[1]))
    if not (0 <= r0 <= r1 <= n):
        raise ValueError("bad row range")
    return r0, r1


def _assemble(n, r0, r1, ri, ci, vv) -> CSR:
    """COO (global row ids in [r0,r1)) -> CSR sorted by (row, col), duplicates summed."""
    ri = np.asarray(ri, dtype=np.int64)
    ci = np.asarray(ci, dtype=np.int64)
    vv = np.asarray(vv, dtype=np.float64)
    key = (ri - r0) * np.int64(n) + ci
    order = np.argsort(key, kind="stable")
    key, vv = key[order], vv[order]
    uniq, start = np.unique(key, return_index=True)
    vals = np.add.reduceat(vv, start) if len(vv) else vv
    rows = uniq // n
    cols = uniq % n
    counts = np.bincount(rows, minlength=r1 - r0)
    rowptr = np.zeros(r1 - r0 + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    return CSR(n=n, row_begin=r0, rowptr=rowptr, colind=cols.astype(np.int32), val=vals)


def convection_diffusion(N: int, dim: int, points: int, gamma: float = 0.1, rows=None) -> CSR:
    """A = L_h + gamma*S_h on an N^dim grid, natural lexicographic order (x fastest),
    Dirichlet (out-of-grid neighbours dropped), no h^2 scaling.

    5-pt (dim=2) / 7-pt (dim=3): diagonal 2*dim; neighbour +e_i -> -1+gamma, -e_i -> -1-gamma.
    27-pt (dim=3): diagonal 26; neighbour (dx,dy,dz) -> -1 + gamma*(dx+dy+dz)/3.
    (DESIGN.md input recipe; SURVEY.md §8(d) "Convection-diffusion matrices".)
    """
    n = N ** dim
    r0, r1 = _rows(n, rows)
    g = np.arange(r0, r1, dtype=np.int64)
    coords = []
    t = g.copy()
    for _ in range(dim):
        coords.append(t % N)
        t //= N
    strides = [N ** k for k in range(dim)]
    if points == 2 * dim + 1:
        offs = []
        for k in range(dim):
            for sgn in (-1, 1):
                d = [0] * dim
                d[k] = sgn
                offs.append((tuple(d), -1.0 + sgn * gamma))
        diag = 2.0 * dim
    elif points == 27 and dim == 3:
        offs = []
        for dz in (-1, 0, 1):
            for dy in (-1, 0, 1):
                for dx in (-1, 0, 1):
                    if dx == dy == dz == 0:
                        continue
                    offs.append(((dx, dy, dz), -1.0 + gamma * (dx + dy + dz) / 3.0))
        diag = 26.0
    else:
        raise ValueError("unsupported stencil")
    RI, CI, VV = [g], [g], [np.full(len(g), diag)]
    for d, v in offs:
        ok = np.ones(len(g), dtype=bool)
        col = g.copy()
        for k in range(dim):
            c = coords[k] + d[k]
            ok &= (c >= 0) & (c < N)
            col += d[k] * strides[k]
        RI.append(g[ok]); CI.append(col[ok]); VV.append(np.full(int(ok.sum()), v))
    return _assemble(n, r0, r1, np.concatenate(RI), np.concatenate(CI), np.concatenate(VV))


def convection_diffusion_stream(N: int, dim: int, points: int, gamma: float = 0.1, rows=None,
                                chunk: int = 1 << 21) -> CSR:
    """The same matrix as ``convection_diffusion`` (identical CSR, bit for bit), built without
    the COO sort so the C5 size (400^3, 1.72e9 nnz) fits in seconds and one copy of memory.

    In natural order the column of neighbour (dx, dy[, dz]) is row + dx + N dy (+ N^2 dz); with
    the offsets enumerated z-major, then y, then x the columns come out ascending inside a row
    and there are no duplicates, so each row chunk is a masked (rows x points) table.
    """
    n = N ** dim
    r0, r1 = _rows(n, rows)
    strides = [N ** k for k in range(dim)]
    if points == 2 * dim + 1:
        offs = [tuple(0 for _ in range(dim))]
        for k in range(dim):
            for sgn in (-1, 1):
                d = [0] * dim
                d[k] = sgn
                offs.append(tuple(d))
        vals = {d: (2.0 * dim if not any(d) else -1.0 + sum(d) * gamma) for d in offs}
    elif points == 27 and dim == 3:
        offs = [(dx, dy, dz) for dz in (-1, 0, 1) for dy in (-1, 0, 1) for dx in (-1, 0, 1)]
        vals = {d: (26.0 if not any(d) else -1.0 + gamma * (d[0] + d[1] + d[2]) / 3.0) for d in offs}
    else:
        raise ValueError("unsupported stencil")
    coloff = np.array([sum(d[k] * strides[k] for k in range(dim)) for d in offs], dtype=np.int64)
    order = np.argsort(coloff, kind="stable")
    offs = [offs[i] for i in order]
    coloff = coloff[order]
    vtab = np.array([vals[d] for d in offs])
    dtab = np.array(offs, dtype=np.int64).reshape(len(offs), dim)
    nr = r1 - r0
    counts = np.empty(nr, dtype=np.int64)
    for c0 in range(r0, r1, chunk):          # pass 1: row lengths (in-grid neighbours per axis)
        t = np.arange(c0, min(r1, c0 + chunk), dtype=np.int64)
        cnt = np.ones(len(t), dtype=np.int64)
        for _ in range(dim):
            c = t % N
            per = 2 - (c == 0).astype(np.int64) - (c == N - 1).astype(np.int64)   # of the offsets -1, +1
            cnt = cnt * (per + 1) if points == 27 else cnt + per
            t //= N
        counts[c0 - r0:c0 - r0 + len(cnt)] = cnt
    rowptr = np.zeros(nr + 1, dtype=np.int64)
    np.cumsum(counts, out=rowptr[1:])
    colind = np.empty(int(rowptr[-1]), dtype=np.int32)
    val = np.empty(int(rowptr[-1]), dtype=np.float64)
    for c0 in range(r0, r1, chunk):          # pass 2: entries
        g = np.arange(c0, min(r1, c0 + chunk), dtype=np.int64)
        ok = _stencil_mask(g, N, dim, dtab)
        a, b = int(rowptr[c0 - r0]), int(rowptr[c0 - r0 + len(g)])
        colind[a:b] = (g[:, None] + coloff[None, :])[ok]
        val[a:b] = np.broadcast_to(vtab[None, :], ok.shape)[ok]
    return CSR(n=n, row_begin=r0, rowptr=rowptr, colind=colind, val=val)


def _stencil_mask(g, N, dim, dtab):
    ok = np.ones((len(g), len(dtab)), dtype=bool)
    t = g.copy()
    for k in range(dim):
        c = (t % N)[:, None] + dtab[None, :, k]
        ok &= (c >= 0) & (c < N)
        t //= N
    return ok


def g3_shaped(n: int = 1585478, width: int = 1260, p_keep: float = 0.9575,
              leak: float = 1e-3, rows=None) -> CSR:
    """G3_circuit-shaped nonsymmetric matrix (Fig. 12).

    Grid of `width` columns, row-major, last row partial.  Undirected grid edge
    (i, dir) with dir E=0 (i,i+1 if same grid row) or S=1 (i,i+width) is kept iff
    u(2014, 2i+dir) < 2*p_keep-1.  Node i gets one long-range edge iff u(2015,i) < -0.999
    to t = floor(n*(u(2016,i)+1)/2) (dropped if t == i).  Conductance
    g = 0.55 + 0.45*u(2017, key), key = 2i+dir (grid) or 2n+i (long range).
    a_ij = -g*(1 + 0.1*sign(j-i)); a_ii = sum_j |a_ij| + leak.
    """
    r0, r1 = _rows(n, rows)
    thr = 2.0 * p_keep - 1.0
    # Undirected edges touching rows [r0, r1): grid edges are local (|j-i| <= width), long
    # range edges can come from anywhere, so scan all nodes for long-range (cheap: 1 draw/node).
    lo = max(0, r0 - width)
    hi = min(n, r1 + width)
    i = np.arange(lo, hi, dtype=np.int64)
    E_ok = ((i % width) + 1 < width) & (i + 1 < n) & (u(2014, 2 * i) < thr)
    S_ok = (i + width < n) & (u(2014, 2 * i + 1) < thr)
    ea = [i[E_ok], i[S_ok]]
    eb = [i[E_ok] + 1, i[S_ok] + width]
    eg = [0.55 + 0.45 * u(2017, 2 * i[E_ok]), 0.55 + 0.45 * u(2017, 2 * i[S_ok] + 1)]
    # long-range edges (chunked over all nodes to bound memory)
    la, lb, lg = [], [], []
    CH = 1 << 22
    for c0 in range(0, n, CH):
        ii = np.arange(c0, min(n, c0 + CH), dtype=np.int64)
        sel = u(2015, ii) < -0.999
        ii = ii[sel]
        t = np.floor(n * (u(2016, ii) + 1.0) / 2.0).astype(np.int64)
        t = np.minimum(t, n - 1)
        ok = t != ii
        ii, t = ii[ok], t[ok]
        touch = ((ii >= r0) & (ii < r1)) | ((t >= r0) & (t < r1))
        ii, t = ii[touch], t[touch]
        la.append(ii); lb.append(t); lg.append(0.55 + 0.45 * u(2017, 2 * n + ii))
    A = np.concatenate(ea + la); B = np.concatenate(eb + lb); G = np.concatenate(eg + lg)
    # both directions
    RI = np.concatenate([A, B]); CI = np.concatenate([B, A]); GG = np.concatenate([G, G])
    keep = (RI >= r0) & (RI < r1)
    RI, CI, GG = RI[keep], CI[keep], GG[keep]
    VV = -GG * (1.0 + 0.1 * np.sign(CI - RI))
    off = _assemble(n, r0, r1, RI, CI, VV)
    # diagonal = row sum of |off-diagonals| + leak
    cnt = np.diff(off.rowptr)
    rr = np.repeat(np.arange(r0, r1, dtype=np.int64), cnt)
    absrow = np.bincount(rr - r0, weights=np.abs(off.val), minlength=r1 - r0)
    g = np.arange(r0, r1, dtype=np.int64)
    return _assemble(n, r0, r1, np.concatenate([rr, g]),
                     np.concatenate([off.colind.astype(np.int64), g]),
                     np.concatenate([off.val, absrow + leak]))


def banded(n: int = 4194304, half_bw: int = 13, skew: float = 0.3, tau: float = 1e-5,
           rows=None) -> CSR:
    """Ill-conditioned banded nonsymmetric matrix.

    Offsets -13..13, w_k = 1/k^2, a_{i,i+k} = -w_k(1-skew), a_{i,i-k} = -w_k(1+skew),
    a_ii = 2*sum_k w_k + tau*(1 + u(2014, i))/2.
    """
    r0, r1 = _rows(n, rows)
    g = np.arange(r0, r1, dtype=np.int64)
    wk = 1.0 / np.arange(1, half_bw + 1, dtype=np.float64) ** 2
    RI, CI, VV = [g], [g], [2.0 * wk.sum() + tau * (1.0 + u(2014, g)) / 2.0]
    for k in range(1, half_bw + 1):
        for sgn in (1, -1):
            col = g + sgn * k
            ok = (col >= 0) & (col < n)
            RI.append(g[ok]); CI.append(col[ok])
            VV.append(np.full(int(ok.sum()), -wk[k - 1] * (1.0 - sgn * skew)))
    return _assemble(n, r0, r1, np.concatenate(RI), np.concatenate(CI), np.concatenate(VV))


def rhs(n: int, rows=None, seed: int = 1) -> np.ndarray:
    """b_i = u(seed, i) for global row i."""
    r0, r1 = _rows(n, rows)
    return u(seed, np.arange(r0, r1, dtype=np.int64))


def random_panel(nrows: int, ncols: int, seed: int, row0: int = 0) -> np.ndarray:
    """Dense column-major (Fortran-order) test panel, entries u(seed, col*2^40 + row)."""
    r = np.arange(row0, row0 + nrows, dtype=np.int64)
    out = np.empty((nrows, ncols), order="F")
    for c in range(ncols):
        out[:, c] = u(seed, (np.int64(c) << np.int64(40)) + r)
    return out


# Named workloads of BASELINE.json "configs" (index -> builder, solver settings).
CONFIGS = {
    "C1": dict(desc="2D convection-diffusion 5-point 32x32 (n=1024), s=5, m=30",
               build=lambda rows=None: convection_diffusion(32, 2, 5, rows=rows),
               n=1024, s=5, m=30),
    "C2": dict(desc="3D convection-diffusion 7-point 128^3 (n=2,097,152), s=10, m=30, Newton, CholQR",
               build=lambda rows=None: convection_diffusion(128, 3, 7, rows=rows),
               n=128 ** 3, s=10, m=30),
    "C3": dict(desc="G3_circuit-shaped (n=1,585,478, ~4.83 nnz/row), s=5, m=60",
               build=lambda rows=None: g3_shaped(rows=rows), n=1585478, s=5, m=60),
    "C4": dict(desc="ill-conditioned banded-27 (n=4,194,304), s=10, m=30",
               build=lambda rows=None: banded(rows=rows), n=4194304, s=10, m=30),
    "C5": dict(desc="3D convection-diffusion 27-point 400^3 (n=64M), s=10, m=30",
               build=lambda rows=None: convection_diffusion_stream(400, 3, 27, rows=rows),
               n=400 ** 3, s=10, m=30),
}
