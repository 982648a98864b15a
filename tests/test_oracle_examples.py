"""Pins of the oracle (O2 encoder, O3 decode, O4 simulator) to the paper's worked
examples (tests/golden/*, each citing its PAPER.md passage).  CPU only."""
import numpy as np
import pytest

from oracle import decode, encode as E, simulate
from golden_io import load_golden


def _dense(vals, m, n):
    return np.array(vals, dtype=np.float64).reshape(m, n)


def _csr(A):
    m, n = A.shape
    r, c = np.nonzero(A)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=m), out=rp[1:])
    return m, n, rp, c.astype(np.int32), A[r, c]


def test_coo_of_A_fig1():
    g = load_golden("eq1_A.txt")
    A = _dense(g["A"], g["rows"], g["cols"])
    m, n, rp, c, v = _csr(A)
    assert list(E.csr_to_coo_rows(m, rp)) == g["coo_row"]
    assert list(c) == g["coo_col"]
    assert list(v) == list(range(1, 17))          # a..p in order (Fig. 1)


def _encode_A(h, w, S, T=4, C=64):
    g = load_golden("eq1_A.txt")
    A = _dense(g["A"], g["rows"], g["cols"])
    return E.encode(*_csr(A), E.Params(h=h, w=w, S=S, T=T, C=C, col_mode=E.COL_I32)), A


def test_bccoo_fig3():
    g = load_golden("fig3_bccoo_2x2.txt")
    enc, _ = _encode_A(g["h"], g["w"], g["S"])
    nb = enc.nnzb
    assert nb == 5
    assert list(E.unpack_flags(enc)[:nb]) == g["flags"]
    assert list(enc.col[:nb]) == g["col"]
    assert list(enc.val[0][: nb * 2]) == g["val0"]
    assert list(enc.val[1][: nb * 2]) == g["val1"]
    # the difference-function view: flags == 1 - (row[b+1] - row[b]), last = 0
    row = np.array(g["bcoo_row"])
    diff = np.append(np.diff(row), 1)
    assert list(1 - diff) == g["flags"]


def test_bccoo_plus_fig4():
    g = load_golden("fig4_bccoo_plus_2x2_s2.txt")
    enc, A = _encode_A(g["h"], g["w"], g["S"])
    nb = enc.nnzb
    assert list(E.unpack_flags(enc)[:nb]) == g["flags"]
    assert list(enc.col[:nb]) == g["col"]
    assert list(enc.val[0][: nb * 2]) == g["val0"]
    assert list(enc.val[1][: nb * 2]) == g["val1"]
    # Fig. 4a: the stacked matrix B = vstack(A[:, 0:4], A[:, 4:8])
    B = np.array(g["B"], dtype=np.float64).reshape(8, 4)
    assert np.array_equal(B, np.vstack([A[:, 0:4], A[:, 4:8]]))


def test_slice_sum_fig5():
    g = load_golden("fig5_slice_sum.txt")
    ga = load_golden("eq1_A.txt")
    A = _dense(ga["A"], 4, 8)
    x = np.array(g["x"], dtype=np.float64)
    assert list(A[:, :4] @ x[:4]) == g["slice0"]
    assert list(A[:, 4:] @ x[4:]) == g["slice1"]
    for S in (1, 2):
        enc, _ = _encode_A(2, 2, S)
        assert list(decode.spmv(enc, x)) == g["y"]


def test_matrix_C_fig6():
    g = load_golden("fig6_matrix_C.txt")
    Cm = _dense(g["C"], g["rows"], g["cols"])
    enc = E.encode(*_csr(Cm), E.Params(h=1, w=1, S=1, T=g["T"], C=g["C_threads"], col_mode=E.COL_I32))
    assert enc.nnzb == 16 and enc.nnzb_pad == 16
    assert list(E.unpack_flags(enc)) == g["flags"]
    assert list(enc.col) == g["col"]
    assert list(enc.val[0]) == list(range(1, 17))
    assert list(enc.fre) == g["fre"]
    assert list(enc.cta_seg0) == [0]


def test_segmented_scan_fig7():
    g = load_golden("fig7_segscan.txt")
    vals, bits = g["input"], g["flags"]
    # start flags are derived from the bit flags: a block starts a segment when it is the
    # first block or follows a row stop
    start = [1] + [1 if bits[i - 1] == 0 else 0 for i in range(1, 16)]
    assert start == g["start"]
    # inclusive segmented scan
    res, s = [], 0
    for v, st in zip(vals, start):
        s = v if st else s + v
        res.append(s)
    assert res == g["result"]
    assert [res[i] for i in range(16) if bits[i] == 0] == g["segment_sums"]
    # the same sums as SpMV: matrix C with block values = input, x = 1 (Fig. 7 / Fig. 6)
    gc = load_golden("fig6_matrix_C.txt")
    Cm = _dense(gc["C"], 4, 8)
    Cm[Cm != 0] = np.array(vals, dtype=np.float64)
    enc = E.encode(*_csr(Cm), E.Params(h=1, w=1, T=4, C=4, col_mode=E.COL_I32))
    assert list(decode.spmv(enc, np.ones(8))) == g["segment_sums"]


def test_walkthrough_fig9_fig10():
    g = load_golden("fig9_walkthrough.txt")
    g7 = load_golden("fig7_segscan.txt")
    sums, trace = simulate.simulate(g7["input"], g7["flags"], g["T"], g["C_threads"])
    assert sums == g7["segment_sums"]
    tr = trace[0]
    assert tr["last_partial_sums"] == g["last_partial_sums"]
    assert tr["start_flags"] == g["start_flags"]
    assert int(tr["skip_scan"]) == g["skip_scan"]
    # first stop of threads 1, 2, 3 close segments 0, 2, 3 (fre = [0, 0, 2, 3], Fig. 6b)
    assert [sums[0], sums[2], sums[3]] == g["first_stop_results"]


@pytest.mark.parametrize("T,C", [(1, 1), (2, 2), (4, 1), (2, 4), (1, 16), (8, 2)])
def test_simulator_across_workgroups(T, C):
    """Adjacent synchronization: the Fig. 7 data split over several
    workgroups (segments spanning workgroups) gives the same segment sums."""
    g7 = load_golden("fig7_segscan.txt")
    vals, bits = list(g7["input"]), list(g7["flags"])
    pad = (-len(vals)) % (T * C)
    sums, _ = simulate.simulate(vals + [0] * pad, bits + [1] * pad, T, C)
    assert sums == g7["segment_sums"]


def test_table3_dense_footprint():
    g = load_golden("table3_dense.txt")
    n = g["n"]
    nnz = n * n
    assert round(12 * nnz / 1e6) == g["coo_mb"]
    # the 4x4 shape (cheapest of the 12 Table-1 shapes for Dense): 250,000 blocks
    best = min(E.footprint_bytes(-(-n // h) * -(-n // w), h, w, 4, 2)
               for h in (1, 2, 3, 4) for w in (1, 2, 4))
    assert round(best / 1e6) == g["bccoo_mb"]
    assert E.footprint_bytes(250_000, 4, 4, 4, 2) == best


def test_strategy2_result_cache_fig10():
    """O4 strategy 2 reproduces the Fig. 10 result-cache walk-through
    on matrix C with R_i = 2^i, and its segment sums equal strategy 1's."""
    g = load_golden("fig10_result_cache.txt")
    gc = load_golden("fig6_matrix_C.txt")
    bits = list(gc["flags"])
    vals = [2 ** i for i in range(16)]
    sums, trace = simulate.simulate_s2(vals, bits, 4, 4, 4)
    tr = trace[0]
    assert tr["fre"] == g["fre"]
    assert tr["cache_walk"] == g["cache_walk"]
    assert tr["cache"] == g["cache"]
    assert sums == simulate.simulate(vals, bits, 4, 4)[0]


@pytest.mark.parametrize("T,C,RC", [(4, 4, 1), (4, 4, 2), (2, 2, 2), (1, 16, 3), (8, 2, 1), (2, 4, 8)])
def test_strategy2_equals_strategy1_across_workgroups(T, C, RC):
    """Fig. 7 data over several workgroups with caches smaller than the stop count (the
    global-result overflow of P:278) and larger: identical segment sums to strategy 1."""
    g7 = load_golden("fig7_segscan.txt")
    vals, bits = list(g7["input"]), list(g7["flags"])
    pad = (-len(vals)) % (T * C)
    s2, _ = simulate.simulate_s2(vals + [0] * pad, bits + [1] * pad, T, C, RC)
    assert s2 == g7["segment_sums"]


def test_delta_reset_per_thread_tile_p121():
    """P:121 segmented difference resets at every THREAD tile (T blocks), not every
    workgroup tile (T*C) and not every block: hand-derived fixture with T = 2, C = 2 over
    two workgroup tiles (tests/golden/p121_delta_reset.txt)."""
    g = load_golden("p121_delta_reset.txt")
    m = g["rows"]
    rp = np.arange(m + 1, dtype=np.int64)
    col = np.array(g["col"], dtype=np.int32)
    e = E.encode(m, g["ncols"], rp, col, np.ones(m), E.Params(1, 1, 1, g["T"], g["C_threads"], E.COL_DELTA, 1))
    assert e.ntiles == 2 and e.nnzb_pad == m
    assert e.col_delta.tolist() == g["delta"]
    assert e.col.tolist() == g["col"]                    # int32 array kept for escapes (Q7)
    assert E.block_columns(e).tolist() == g["col"]
