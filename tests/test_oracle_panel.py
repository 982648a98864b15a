"""Pins of the panel-sliced BCCOO+ oracle (oracle/panel.py, DESIGN.md §2.1 readings P1-P6):
a hand-derived example on the paper's matrix A (tests/golden/panel_eq1_A.txt), the
degenerate case that must reproduce the paper's plain BCCOO arrays bit for bit (one panel,
one slice: P:83-119 through oracle/encode.py), brute force y = A x with exact integer
arithmetic, and the format's invariants.  CPU only."""
import numpy as np
import pytest

import synth
from golden_io import load_golden
from oracle import decode, encode as E, panel as PN


def _csr_of(A):
    m, n = A.shape
    r, c = np.nonzero(A)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=m), out=rp[1:])
    return m, n, rp, c.astype(np.int32), A[r, c]


def _bits(enc):
    return np.unpackbits(enc.flags, bitorder="little")[: enc.nband_pad]


def test_hand_example_eq1_A():
    g = load_golden("panel_eq1_A.txt")
    A = np.array(load_golden("eq1_A.txt")["A"], dtype=np.float64).reshape(4, 8)
    pp = PN.PanelParams(R=g["R"], W=g["W"], B=g["B"], T=g["T"], C=g["C_threads"],
                        far=E.Params(1, 1, 1, 4, 64, E.COL_I32, E.EMPTY_FILLER))
    enc = PN.encode_panel(*_csr_of(A), pp)
    assert enc.KS == g["KS"]
    assert _bits(enc).tolist() == g["flags"]
    assert enc.col16.tolist() == g["col16"]
    assert enc.val.tolist() == g["val"]
    assert enc.panel_blk0.tolist() == g["panel_blk0"]
    assert enc.slice_ptr.ravel().tolist() == g["slice_ptr"]
    assert enc.stop_ptr.ravel().tolist() == g["stop_ptr"]
    assert enc.first_row.ravel().tolist() == g["first_row"] and enc.nfill == 0
    assert enc.tile_rank.tolist() == g["tile_rank"]
    assert enc.far_csr[2].tolist() == g["far_val"]
    x = np.arange(1, 9, dtype=np.float64)
    assert decode.spmv(enc.far, x).tolist() == g["y_far"]
    assert PN.spmv(enc, x).tolist() == g["y"]
    assert np.array_equal(PN.to_dense(enc), A)


def test_hand_example_eq1_A_far_in_panel():
    """Reading P7 on the paper's matrix A: far entries as slice 0 of every panel."""
    g = load_golden("panel_eq1_A_fip.txt")
    A = np.array(load_golden("eq1_A.txt")["A"], dtype=np.float64).reshape(4, 8)
    pp = PN.PanelParams(R=g["R"], W=g["W"], B=g["B"], T=g["T"], C=g["C_threads"], far_in_panel=True)
    enc = PN.encode_panel(*_csr_of(A), pp)
    assert enc.KS == g["KS"] and enc.NS == g["KS"] + 1 and enc.far is None
    assert _bits(enc).tolist() == g["flags"]
    assert enc.val.tolist() == g["val"]
    assert enc.col16.tolist() == g["col16"]
    assert enc.far_col.tolist() == g["far_col"]
    assert enc.far_blk0.tolist() == g["far_blk0"]
    assert enc.panel_blk0.tolist() == g["panel_blk0"]
    assert enc.slice_ptr.ravel().tolist() == g["slice_ptr"]
    assert enc.stop_ptr.ravel().tolist() == g["stop_ptr"]
    assert enc.first_row.ravel().tolist() == g["first_row"] and enc.nfill == 0
    assert enc.tile_rank.tolist() == g["tile_rank"]
    x = np.arange(1, 9, dtype=np.float64)
    assert PN.spmv(enc, x).tolist() == g["y"]
    assert np.array_equal(PN.to_dense(enc), A)
    # the far slices alone: A without its band entries (P2)
    m, n, rp, c, v = _csr_of(A)
    rows, p, k, band = PN.split(m, n, rp, c, v, pp)
    Af = A.copy()
    Af[rows[band], c[band]] = 0
    assert (Af @ x).tolist() == g["y_far"]


@pytest.mark.parametrize("seed", range(12))
def test_one_panel_all_far_is_plain_bccoo(seed):
    """P7 degenerate case: one panel, band placed outside the matrix (diag0 beyond n), so
    every entry is in the far slice, which must be the paper's BCCOO arrays bit for bit
    (1x1 blocks, S = 1, int32 columns, FILLER blocks R1 with column NB = n, Q3) for the rows
    from the first to the last non-empty one — including the pad columns (Q3) and the
    per-tile first-result entries (tile_rank = cta_seg0)."""
    a = synth.random_tiny(seed)
    R = 32 * (-(-a.m // 32))
    pp = PN.PanelParams(R=R, W=4, B=0, T=4, C=2, diag0=a.n + 8, far_in_panel=True)
    enc = PN.encode_panel(a.m, a.n, a.row_ptr, a.col, a.val, pp)
    lens = np.diff(a.row_ptr)
    nz = np.flatnonzero(lens > 0)
    assert enc.nband == 0 and enc.col16.size == 0
    if nz.size == 0:
        assert enc.nband_pad == 0
        return
    r0, r1 = nz[0], nz[-1] + 1
    sub = synth.CSR(r1 - r0, a.n, a.row_ptr[r0:r1 + 1] - a.row_ptr[r0], a.col[a.row_ptr[r0]:a.row_ptr[r1]],
                    a.val[a.row_ptr[r0]:a.row_ptr[r1]])
    plain = E.encode(sub.m, sub.n, sub.row_ptr, sub.col, sub.val, E.Params(1, 1, 1, 4, 2, E.COL_I32, E.EMPTY_FILLER))
    assert enc.first_row[0, 0] == r0 and enc.nfill == plain.n_filler
    assert enc.nband_pad == plain.nnzb_pad and enc.far_blk0.tolist() == [0, plain.nnzb_pad]
    assert np.array_equal(enc.flags, plain.flags)
    assert np.array_equal(enc.val, plain.val[0])
    assert np.array_equal(enc.far_col.astype(np.int64), plain.col.astype(np.int64))   # fillers: NB = n
    assert np.array_equal(enc.tile_rank, plain.cta_seg0)


@pytest.mark.parametrize("seed", range(12))
def test_one_panel_one_slice_is_plain_bccoo(seed):
    """R >= m, B = 0, W >= R: every entry is a band entry of the single slice, and the
    band arrays are exactly the paper's BCCOO arrays (1x1 blocks, S = 1) with the seg_row
    reading (Q1/R2): same flags, columns (u16), values;
    and FILLER blocks exactly where the paper's reading R1 puts them."""
    a = synth.random_tiny(seed)
    R = 32 * (-(-a.m // 32))
    pp = PN.PanelParams(R=R, W=max(R, 4 * (-(-a.n // 4))), B=0, T=4, C=2)
    enc = PN.encode_panel(a.m, a.n, a.row_ptr, a.col, a.val, pp)
    # the paper's arrays for the rows [first non-empty, last non-empty] with FILLER blocks
    # (R1) for the empty rows in between; a filler's column is the zero slot W (Q3)
    lens = np.diff(a.row_ptr)
    nz = np.flatnonzero(lens > 0)
    if nz.size == 0:
        assert enc.nband_pad == 0
        return
    r0, r1 = nz[0], nz[-1] + 1
    sub = synth.CSR(r1 - r0, a.n, a.row_ptr[r0:r1 + 1] - a.row_ptr[r0], a.col[a.row_ptr[r0]:a.row_ptr[r1]],
                    a.val[a.row_ptr[r0]:a.row_ptr[r1]])
    plain = E.encode(sub.m, sub.n, sub.row_ptr, sub.col, sub.val, E.Params(1, 1, 1, 4, 2, E.COL_U16, E.EMPTY_FILLER))
    assert enc.KS == 1 and enc.far.nnzb == 0 and enc.nband == a.nnz
    assert enc.first_row[0, 0] == r0 and enc.nfill == plain.n_filler
    assert enc.nband_pad == plain.nnzb_pad
    assert np.array_equal(enc.flags, plain.flags)
    assert np.array_equal(enc.val, plain.val[0])
    assert np.array_equal(enc.tile_rank, plain.cta_seg0)      # first-result entries
    fill = enc.col16 == pp.W
    pcol = plain.col.astype(np.int64)
    assert np.array_equal(enc.col16[~fill], pcol[~fill].astype(np.uint16))
    assert np.all(pcol[fill] == plain.NB)                     # both name the zero column (Q3)


def _banded(seed, m, n, band, extra=0.1):
    g = np.random.default_rng(seed)
    A = np.zeros((m, n))
    for i in range(m):
        k = g.integers(0, 6)
        cols = np.clip(i + g.integers(-band, band + 1, size=k), 0, n - 1)
        A[i, cols] = g.integers(-3, 4, size=k)
        if g.random() < extra:
            A[i, g.integers(0, n)] = g.integers(1, 4)
    A[g.integers(0, m, size=max(1, m // 7))] = 0          # empty rows
    return A


@pytest.mark.parametrize("fip", [False, True])
@pytest.mark.parametrize("seed", range(16))
def test_brute_force_integer_exact(seed, fip):
    g = np.random.default_rng(100 + seed)
    m, n = int(g.integers(1, 90)), int(g.integers(1, 90))
    A = _banded(seed, m, n, int(g.integers(0, 12)))
    pp = PN.PanelParams(R=int(g.integers(1, 20)), W=int(g.integers(1, 9)), B=int(g.integers(0, 10)),
                        T=int(g.choice([1, 2, 4])), C=int(g.choice([1, 2, 3])),
                        diag0=int(g.integers(-3, 4)),
                        far=E.Params(1, 1, 1, 4, 2, 0, int(g.choice([E.EMPTY_FILLER, E.EMPTY_MAP]))),
                        far_in_panel=fip)
    enc = PN.encode_panel(*_csr_of(A), pp)
    x = g.integers(-4, 5, size=n).astype(np.float64)
    assert np.array_equal(PN.spmv(enc, x), A @ x)
    assert np.array_equal(PN.to_dense(enc), A)


@pytest.mark.parametrize("fip", [False, True])
@pytest.mark.parametrize("seed", range(8))
def test_invariants(seed, fip):
    a = synth.circuit_like_rows(0, 3000, kind="integer", n=3000, band=300, n_net=2, net_log2=(9, 10))
    pp = PN.PanelParams(R=256, W=64, B=300, T=4, C=8, far=E.Params(1, 1, 1, 4, 8, 0, 0), far_in_panel=fip)
    if seed % 2:
        pp.diag0 = 17
    enc = PN.encode_panel(a.m, a.n, a.row_ptr, a.col, a.val, pp)
    bits = _bits(enc)
    rows, p, k, band = PN.split(a.m, a.n, a.row_ptr, a.col, a.val, pp)
    # every entry once: band + far = nnz; far entries lie outside their panel's band
    assert enc.nband == int(band.sum()) and enc.far_csr[1].size == a.nnz - enc.nband
    # stops = set bits of the occupancy bitmaps, slice by slice
    TC = pp.T * pp.C
    for q in range(enc.npanels):
        b0 = enc.panel_blk0[q]
        assert enc.panel_blk0[q + 1] - b0 == enc.slice_ptr[q, -1]
        for kk in range(enc.NS):
            g0, g1 = b0 + enc.slice_ptr[q, kk], b0 + enc.slice_ptr[q, kk + 1]
            assert g0 % TC == 0 and g1 % TC == 0               # no tile holds two slices (P4)
            seg = bits[g0:g1]
            # one stop per row from the slice's first to its last non-empty row (P6, P7)
            in_k = (~band & (p == q)) if kk < enc.fip else (band & (p == q) & (k == kk - enc.fip))
            rows_k = np.unique(rows[in_k] - q * pp.R)
            pops = int(rows_k[-1] - rows_k[0] + 1) if rows_k.size else 0
            assert int((seg == 0).sum()) == pops == enc.stop_ptr[q, kk + 1] - enc.stop_ptr[q, kk]
            if rows_k.size:
                assert enc.first_row[q, kk] == rows_k[0]
            if pops:
                last = g0 + np.flatnonzero(seg == 0)[-1]
                assert g1 - last - 1 < TC and np.all(bits[last + 1:g1] == 1)   # pad bits
                assert np.all(enc.val[last + 1:g1] == 0)
            for tt in range(g0 // TC, g1 // TC):               # first-result entry per tile
                assert enc.tile_rank[tt] == int((bits[g0:tt * TC] == 0).sum())
    assert np.all(enc.col16.astype(np.int64) <= pp.W)            # W: a FILLER block's zero slot
    if fip:   # P7: far columns in [0, n], n = a far-slice FILLER; col16 / far_col partition the stream
        assert enc.col16.size + enc.far_col.size == enc.nband_pad and enc.far_blk0[-1] == enc.far_col.size
        assert np.all((enc.far_col >= 0) & (enc.far_col <= a.n))
        assert enc.nfill == int((enc.col16 == pp.W).sum() + (enc.far_col == a.n).sum()) > 0
    else:
        assert enc.nfill == int(((enc.col16 == pp.W) & (enc.val == 0)).sum()) > 0
    x = synth.make_x(a.n, np.float64, "int", seed)
    A = a.to_dense()
    assert np.array_equal(PN.spmv(enc, x), A @ x)
