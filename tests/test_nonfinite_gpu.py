"""Non-finite values stay inside their own row segment (include/yaspmv.h semantics: NaN/Inf
propagate per IEEE rules).

The matrix-based segmented sum combines partial sums with the operator
(f1,v1) (+) (f2,v2) = (f1|f2, f2 ? v2 : v1+v2) and passes carries between
workgroups by adjacent synchronization / look-back.  A kernel that resets a
segment by arithmetic (v*(1-f)), or that derives a segment sum as a difference of prefix
sums, leaks a NaN or an Inf into every later row of the tile chain; a select does not.
These tests poison a few rows and check that (a) the poisoned rows come out NaN / +Inf and
(b) every other row is finite and within the BASELINE.json tolerance of the oracle run on
the clean matrix.

x = +Inf: every stored block multiplies x, including the zero padding of an h x w block
(P:83-105), so 0 * Inf = NaN can reach a row of a stored h x w block that has no
structural entry in the Inf column.  The expected NaN / +Inf pattern is therefore the one
the oracle's decode of the canonical arrays (oracle/decode.py, IEEE arithmetic over every
stored block) produces.  A FILLER block of an empty stacked row sits in block column NB,
where x reads 0 (Q3/Q19), so with 1x1 blocks the pattern is exactly the CSR one
(y = A.x, O1) for both empty-row encodings, and every row of an empty block row is 0.
"""
import numpy as np
import pytest

import synth
from oracle import decode, encode as E, ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

PARAMS = [
    dict(T=16, C=256),
    dict(T=8, C=128, S=2),
    dict(T=4, C=64, tpc=2),
    dict(T=16, C=128, rc=2),
    dict(T=16, C=128, col_mode=E.COL_DELTA, empty_mode=E.EMPTY_MAP),
    dict(h=2, w=2, T=8, C=256),
]


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanlzz14_b200  # noqa: F401  (fails loudly if the .so is missing)


@pytest.fixture(scope="module")
def web():
    return synth.webbase_like(m=200_000)


def _run(csr, val, x, **params):
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, val, device=0, **params)
    try:
        y = A.spmv(torch.from_numpy(np.ascontiguousarray(x)).cuda())
        torch.cuda.synchronize()
        return y.cpu().numpy()
    finally:
        A.free()


def _check_clean_rows(csr, y, x, bad_rows):
    y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    keep = np.ones(csr.m, dtype=bool)
    keep[bad_rows] = False
    assert np.all(np.isfinite(y[keep])), np.flatnonzero(~np.isfinite(y) & keep)[:10]
    ok, worst = ref.check_tolerance(y[keep], y_ref[keep], bound[keep], csr.val.dtype)
    assert ok, worst


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
@pytest.mark.parametrize("pi", range(len(PARAMS)))
def test_nan_value_stays_in_its_row(web, pi, dtype):
    csr = web if dtype == np.float32 else synth.CSR(web.m, web.n, web.row_ptr, web.col, web.val.astype(dtype))
    lens = np.diff(csr.row_ptr)
    rng = np.random.default_rng(11)
    # poison short rows, the longest rows (they span many tiles) and the last non-empty row
    cand = np.flatnonzero(lens > 0)
    bad = np.unique(np.concatenate([rng.choice(cand, 24, replace=False), np.argsort(lens)[-4:], cand[-1:]]))
    val = csr.val.copy()
    for r in bad:
        val[csr.row_ptr[r] + rng.integers(lens[r])] = np.nan
    x = synth.make_x(csr.n, dtype, "uniform", 3)
    y = _run(csr, val, x, **PARAMS[pi])
    assert np.all(np.isnan(y[bad]))
    _check_clean_rows(csr, y, x, bad)


def _oracle_params(p):
    return E.Params(p.get("h", 1), p.get("w", 1), p.get("S", 1), p["T"], p["C"],
                    p.get("col_mode", 0), p.get("empty_mode", 0))


@pytest.mark.parametrize("pi", range(len(PARAMS)))
def test_inf_x_reaches_exactly_the_rows_that_read_it(web, pi):
    csr = web
    p = PARAMS[pi]
    x = synth.make_x(csr.n, np.float32, "uniform", 4)
    rng = np.random.default_rng(12)
    cols = rng.choice(csr.n, 6, replace=False)
    x[cols] = np.inf
    hit = np.isin(csr.col, cols)
    rows = np.repeat(np.arange(csr.m), np.diff(csr.row_ptr))
    reads = np.unique(rows[hit])             # rows with a structural entry in an Inf column
    assert reads.size > 0
    assert np.all(csr.val[hit] > 0)          # webbase values are 1/L_i > 0
    y = _run(csr, csr.val, x, **p)
    enc = E.encode(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, _oracle_params(p))
    with np.errstate(invalid="ignore"):
        y_dec = decode.spmv(enc, x)
    assert np.array_equal(np.isnan(y), np.isnan(y_dec))
    assert np.array_equal(np.isposinf(y), np.isposinf(y_dec))
    assert not np.any(np.isneginf(y))
    assert np.all(~np.isfinite(y[reads]))
    if enc.p.h == enc.p.w == 1:              # exactly O1's pattern, FILLER or MAP
        assert np.array_equal(np.flatnonzero(~np.isfinite(y)), reads)
    # "empty rows give y = 0" (include/yaspmv.h): every row of an empty block row, any x
    h = enc.p.h
    blk_nnz = np.add.reduceat(np.diff(csr.row_ptr), np.arange(0, csr.m, h)) if csr.m else np.zeros(0)
    empty_rows = np.flatnonzero(np.repeat(blk_nnz == 0, h)[: csr.m])
    assert empty_rows.size > 0
    assert np.all(y[empty_rows] == 0)
    x_clean = x.copy()
    x_clean[cols] = 0
    _check_clean_rows(csr, y, x_clean, np.flatnonzero(~np.isfinite(y_dec)))
