"""Pins for synth/generators.py (seeded inputs shared by both sides)."""
import os

import numpy as np
import pytest

from synth import generators as G
from _golden_io import read_golden


def test_splitmix64_reference_stream(golden_dir):
    rows = read_golden(os.path.join(golden_dir, "splitmix64_seed0.txt"))
    x = np.array([int(r[0], 16) for r in rows], dtype=np.uint64)
    y = G.splitmix64(x)
    assert [int(v) for v in y] == [int(r[1], 16) for r in rows]


def test_uniform_range_and_determinism():
    v = G.u(7, np.arange(100000))
    assert v.min() >= -1.0 and v.max() < 1.0
    assert abs(v.mean()) < 0.01
    assert np.array_equal(v[10:20], G.u(7, np.arange(10, 20)))


@pytest.mark.parametrize("N,dim,pts", [(32, 2, 5), (16, 3, 7), (9, 3, 27)])
def test_stencil_nnz_closed_form(N, dim, pts):
    A = G.convection_diffusion(N, dim, pts)
    if pts == 2 * dim + 1:
        expect = (2 * dim + 1) * N ** dim - 2 * dim * N ** (dim - 1)
    else:
        expect = (3 * N - 2) ** 3
    assert A.nnz == expect
    S = A.to_scipy()
    assert (abs(S - S.T) > 1e-14).nnz > 0          # nonsymmetric values
    P = (S != 0).astype(int)
    assert (P - P.T).nnz == 0                      # symmetric pattern


def test_stencil_golden_rows(golden_dir):
    A = G.convection_diffusion(3, 2, 5).to_scipy().toarray()
    for c, v in read_golden(os.path.join(golden_dir, "cd5pt_N3_row4.txt")):
        assert A[4, int(c)] == pytest.approx(float(v), abs=1e-15)
    assert np.count_nonzero(A[4]) == 5
    A = G.convection_diffusion(3, 3, 27).to_scipy().toarray()
    for c, v in read_golden(os.path.join(golden_dir, "cd27pt_N3_row13.txt")):
        assert A[13, int(c)] == pytest.approx(float(v), abs=1e-15)
    assert np.count_nonzero(A[13]) == 27


def test_row_ranges_are_partition_independent():
    full = G.convection_diffusion(12, 3, 7)
    part = G.convection_diffusion(12, 3, 7, rows=(300, 901))
    lo, hi = full.rowptr[300], full.rowptr[901]
    assert np.array_equal(part.colind, full.colind[lo:hi])
    assert np.array_equal(part.val, full.val[lo:hi])
    g = G.g3_shaped(n=20000, width=150)
    gp = G.g3_shaped(n=20000, width=150, rows=(7000, 13000))
    lo, hi = g.rowptr[7000], g.rowptr[13000]
    assert np.array_equal(gp.colind, g.colind[lo:hi]) and np.array_equal(gp.val, g.val[lo:hi])
    b = G.banded(n=5000)
    bp = G.banded(n=5000, rows=(100, 200))
    assert np.array_equal(bp.val, b.val[b.rowptr[100]:b.rowptr[200]])


def test_g3_shaped_structure():
    A = G.g3_shaped(n=200000, width=400).to_scipy()
    nnz_row = A.nnz / A.shape[0]
    assert 4.6 < nnz_row < 5.0                     # ~4.83 at the C3 parameters
    d = A.diagonal()
    off = abs(A).sum(axis=1).A1 - abs(d)
    assert np.allclose(d - off, 1e-3)              # leak = 1e-3 diagonal excess
    P = (A != 0).astype(int)
    assert (P - P.T).nnz == 0


def test_banded_structure():
    A = G.banded(n=1000).to_scipy()
    assert A.nnz == 27 * 1000 - 2 * sum(range(1, 14))
    wk = 1.0 / np.arange(1, 14) ** 2
    assert A[500, 501] == pytest.approx(-wk[0] * 0.7)
    assert A[500, 499] == pytest.approx(-wk[0] * 1.3)
    assert 2 * wk.sum() <= A[500, 500] <= 2 * wk.sum() + 1e-5


@pytest.mark.parametrize("N,dim,pts,rows", [(12, 3, 27, None), (9, 3, 7, None), (11, 2, 5, None),
                                            (13, 3, 27, (100, 1500)), (10, 3, 7, (7, 777)),
                                            (2, 3, 27, None), (1, 2, 5, None), (2, 3, 7, (3, 7))])
def test_stream_stencil_generator_is_identical(N, dim, pts, rows):
    """The sort-free generator used for C5 builds the same CSR bit for bit (small chunks so
    several chunk boundaries are crossed)."""
    A = G.convection_diffusion(N, dim, pts, rows=rows)
    B = G.convection_diffusion_stream(N, dim, pts, rows=rows, chunk=97)
    assert A.row_begin == B.row_begin and A.n == B.n
    assert np.array_equal(A.rowptr, B.rowptr) and np.array_equal(A.colind, B.colind)
    assert A.val.tobytes() == B.val.tobytes()
