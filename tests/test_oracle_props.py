"""Brute-force and invariant pins of the oracle encoder/decoder (O2/O3/O4) on random tiny
matrices: decode(encode(A)) = A, the decoded product equals dense A@x EXACTLY on integer
data, and the structural invariants of PAPER.md §2 hold.  CPU only."""
import itertools

import numpy as np
import pytest

import synth
from oracle import decode, encode as E, simulate


def _grid(seed):
    rng = np.random.default_rng(1000 + seed)
    hs, ws, Ts, Cs = [1, 2, 3, 4], [1, 2, 4], [1, 2, 4, 8], [1, 2, 4, 8]
    combos = list(itertools.product(hs, ws, Ts, Cs))
    pick = rng.choice(len(combos), size=12, replace=False)
    return [combos[i] for i in pick]


@pytest.mark.parametrize("seed", range(40))
def test_roundtrip_and_exact_product(seed):
    a = synth.random_tiny(seed)
    A = a.to_dense()
    x = synth.make_x(a.n, np.float64, "int", seed)
    y_dense = A @ x
    for (h, w, T, C) in _grid(seed):
        NB = -(-a.n // w)
        for S in sorted({1, 2, min(3, NB), NB}):
            if S > NB:
                continue
            for empty_mode in (E.EMPTY_FILLER, E.EMPTY_MAP):
                for col_mode in (E.COL_I32, E.COL_DELTA):
                    p = E.Params(h, w, S, T, C, col_mode, empty_mode)
                    enc = E.encode(a.m, a.n, a.row_ptr, a.col, a.val, p)
                    _check_invariants(a, enc)
                    assert np.array_equal(decode.to_dense(enc), A)
                    assert np.array_equal(decode.spmv(enc, x), y_dense)


def _check_invariants(a, enc):
    p = enc.p
    TC = p.T * p.C
    bits = E.unpack_flags(enc)
    assert enc.nnzb_pad % TC == 0 and enc.nnzb_pad >= enc.nnzb
    assert np.all(bits[enc.nnzb:] == 1)                       # pad with 1s
    # stops == non-empty stacked block rows (R2) / all stacked block rows (R1)
    MB, SW = enc.MB, enc.SW
    rows = np.repeat(np.arange(a.m), np.diff(a.row_ptr))
    sr = (a.col // p.w // SW) * MB + rows // p.h
    n_nonempty = np.unique(sr).size
    if p.empty_mode == E.EMPTY_FILLER:
        assert enc.n_stops == p.S * MB
        assert enc.n_filler == p.S * MB - n_nonempty
    else:
        assert enc.n_stops == n_nonempty
        assert enc.zero_rows.size == p.S * MB - n_nonempty
    assert (bits == 0).sum() == enc.n_stops
    # blocks hold every structural entry exactly once (nnz preserved)
    R, Cc, V = decode.decode_blocks(enc)
    keyset = set(zip(rows.tolist(), a.col.tolist()))
    assert keyset <= set(zip(R.tolist(), Cc.tolist()))
    assert len(keyset) == a.nnz
    # aux: cta_seg0 non-decreasing, <= stops, equal to fre at tile starts
    assert np.all(np.diff(enc.cta_seg0) >= 0)
    assert enc.cta_seg0.size == 0 or enc.cta_seg0[-1] <= enc.n_stops
    assert np.array_equal(enc.cta_seg0, enc.fre[:: p.C][: enc.ntiles])
    # delta decode reproduces the block columns
    if p.col_mode == E.COL_DELTA:
        assert np.array_equal(E.block_columns(enc), enc.col.astype(np.int64))


def _brute_bccoo_plus(A, struct, h, w, S):
    """Fig. 4 construction by brute force: cut the (zero-padded) matrix into S vertical
    slices of SW block columns, stack them top-down, scan block rows of the
    stacked matrix left to right keeping blocks that hold a structural entry
    with their ORIGINAL block column; the row index array becomes bit flags by
    the inverted difference function."""
    m, n = A.shape
    MB, NB = -(-m // h), -(-n // w)
    SW = -(-NB // S)
    Ap = np.zeros((MB * h, NB * w)); Ap[:m, :n] = A
    Sp = np.zeros((MB * h, NB * w), bool); Sp[:m, :n] = struct
    row_index, col, v = [], [], [[] for _ in range(h)]
    for s in range(S):
        for br in range(MB):
            for bc in range(s * SW, min((s + 1) * SW, NB)):
                if Sp[br * h:(br + 1) * h, bc * w:(bc + 1) * w].any():
                    row_index.append(s * MB + br)
                    col.append(bc)
                    for r in range(h):
                        v[r].extend(Ap[br * h + r, bc * w:(bc + 1) * w].tolist())
    flags = [1 - (row_index[i + 1] - row_index[i]) for i in range(len(row_index) - 1)] + [0]
    return flags, col, v


@pytest.mark.parametrize("seed", range(16))
def test_encoder_matches_brute_force_construction(seed):
    a = synth.random_tiny(seed, force_empty=False, density=0.5)
    A = a.to_dense()
    struct = np.zeros(A.shape, bool)
    rows = np.repeat(np.arange(a.m), np.diff(a.row_ptr))
    struct[rows, a.col] = True
    for h, w in ((1, 1), (2, 2), (3, 1), (4, 2), (1, 4)):
        NB = -(-a.n // w)
        for S in sorted({1, min(2, NB), NB}):
            enc = E.encode(a.m, a.n, a.row_ptr, a.col, a.val, E.Params(h, w, S, 2, 2, E.COL_I32, 2))
            flags, col, v = _brute_bccoo_plus(A, struct, h, w, S)
            nb = enc.nnzb
            assert nb == len(col)
            if enc.zero_rows.size == 0:      # no empty stacked row: flags are 0/1 differences
                assert list(E.unpack_flags(enc)[:nb]) == flags
            assert list(enc.col[:nb]) == col
            for r in range(h):
                assert list(enc.val[r][: nb * w]) == v[r]


@pytest.mark.parametrize("seed", range(12))
def test_simulator_equals_decode(seed):
    """O4 (tiled simulator with adjacent sync) == O3 on random tiny inputs."""
    a = synth.random_tiny(seed, integer=True)
    x = synth.make_x(a.n, np.float64, "int", seed)
    for T, C in ((1, 1), (2, 2), (4, 2), (2, 8)):
        enc = E.encode(a.m, a.n, a.row_ptr, a.col, a.val, E.Params(1, 1, 1, T, C, E.COL_I32, 1))
        prods = decode.block_products(enc, x)[:, 0]
        sums, _ = simulate.simulate([int(v) for v in prods], list(E.unpack_flags(enc)), T, C)
        assert np.array_equal(np.array(sums, dtype=np.float64), decode.spmv(enc, x))


@pytest.mark.parametrize("seed", range(6))
def test_normalize_sums_duplicates(seed):
    m, n = 9, 7
    r, c, v = synth.random_coo(seed, m, n, 60)
    rp, col, val = E.normalize(m, n, r, c, v)
    D = np.zeros((m, n)); np.add.at(D, (r, c), v)
    got = np.zeros((m, n))
    rows = np.repeat(np.arange(m), np.diff(rp))
    got[rows, col] = val
    assert np.array_equal(got, D)
    # sorted, unique (row, col) and structural zeros kept (sum may be 0)
    key = rows * n + col
    assert np.all(np.diff(key) > 0)
    assert col.size == len(set(zip(r.tolist(), c.tolist())))


def test_empty_and_degenerate():
    # nnz = 0: R2 encodes nothing (every row zero-filled); R1 puts a filler per row
    rp = np.zeros(6, dtype=np.int64)
    e = E.encode(5, 4, rp, np.zeros(0, np.int32), np.zeros(0), E.Params(1, 1, 1, 4, 2, 0, 2))
    assert e.nnzb == 0 and e.ntiles == 0 and e.zero_rows.size == 5
    assert np.array_equal(decode.spmv(e, np.ones(4)), np.zeros(5))
    e = E.encode(5, 4, rp, np.zeros(0, np.int32), np.zeros(0), E.Params(1, 1, 1, 4, 2, 0, 1))
    assert e.nnzb == 5 and e.n_stops == 5
    assert np.array_equal(decode.spmv(e, np.ones(4)), np.zeros(5))
    # 1x1
    e = E.encode(1, 1, np.array([0, 1]), np.array([0], np.int32), np.array([3.0]), E.Params())
    assert decode.spmv(e, np.array([2.0]))[0] == 6.0
    # u16 / i32 switch at NB = 65535 (Q6)
    assert E.resolve_col_mode(65534, 0) == E.COL_U16
    assert E.resolve_col_mode(65535, 0) == E.COL_I32
    with pytest.raises(ValueError):
        E.resolve_col_mode(65535, E.COL_U16)


def test_delta_escape_rule():
    # one row with columns chosen to hit deltas 0, 32767, 32768 (escape), -1 (escape)
    cols = np.array([5, 5 + 32767, 5 + 32767 + 32768, 70000], dtype=np.int32)
    # put them in separate rows so that they may be in any order within a thread tile
    m = 4
    rp = np.arange(m + 1, dtype=np.int64)
    order_cols = np.array([10, 10 + 32767, 10 + 32767 + 32768, 10 + 32767 + 32768 - 1], dtype=np.int32)
    e = E.encode(m, 70000, rp, order_cols, np.ones(m), E.Params(1, 1, 1, 4, 1, E.COL_DELTA, 1))
    d = e.col_delta[:4].tolist()
    assert d == [10, 32767, -1, -1]     # 32768 out of int16 range; -1 is the escape value
    assert np.array_equal(E.block_columns(e), e.col.astype(np.int64))
    del cols


@pytest.mark.parametrize("seed", range(20))
def test_inf_x_reaches_rows_through_stored_blocks_only(seed):
    """DESIGN Q19, pinned by brute force: with one x_j = +Inf, the decoded 1x1 product is
    non-finite exactly in the rows with a structural entry in column j — with the seg_row
    map (R2) and with FILLER blocks (R1), whose column NB reads x as 0 (Q3) — and every
    empty row is exactly 0.  tests/test_nonfinite_gpu.py compares the GPU with this decode."""
    a = synth.random_tiny(seed)
    mask = a.to_dense() != 0
    rows = np.repeat(np.arange(a.m), np.diff(a.row_ptr))
    mask[rows, a.col] = True                       # structural zeros read x too
    for j in range(a.n):
        x = synth.make_x(a.n, np.float64, "int", seed)
        x[j] = np.inf
        reads = mask[:, j]
        with np.errstate(invalid="ignore"):
            e2 = E.encode(a.m, a.n, a.row_ptr, a.col, a.val, E.Params(1, 1, 1, 4, 2, 0, E.EMPTY_MAP))
            assert np.array_equal(~np.isfinite(decode.spmv(e2, x)), reads)
            e1 = E.encode(a.m, a.n, a.row_ptr, a.col, a.val, E.Params(1, 1, 1, 4, 2, 0, E.EMPTY_FILLER))
            y1 = decode.spmv(e1, x)
        stop_pos = np.flatnonzero(E.unpack_flags(e1) == 0)
        empty = np.diff(a.row_ptr) == 0
        if e1.n_filler:
            assert np.all(E.block_columns(e1)[stop_pos[empty]] == e1.NB)   # Q3: column NB
        assert np.array_equal(~np.isfinite(y1), reads)
        assert np.all(y1[empty] == 0)
