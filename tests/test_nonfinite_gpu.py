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

x = +Inf is only tested with 1x1 blocks: with h x w > 1 the zero padding of a block
multiplies x too (0 * Inf = NaN in a neighbouring row), which the blocked format
implies and the ABI leaves unspecified.
"""
import numpy as np
import pytest

import synth
from oracle import encode as E, ref

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


@pytest.mark.parametrize("pi", [0, 1, 2, 3, 4])
def test_inf_x_reaches_exactly_the_rows_that_read_it(web, pi):
    csr = web
    x = synth.make_x(csr.n, np.float32, "uniform", 4)
    rng = np.random.default_rng(12)
    cols = rng.choice(csr.n, 6, replace=False)
    x[cols] = np.inf
    hit = np.isin(csr.col, cols)
    rows = np.repeat(np.arange(csr.m), np.diff(csr.row_ptr))
    bad = np.unique(rows[hit])
    assert bad.size > 0
    assert np.all(csr.val[hit] > 0)          # webbase values are 1/L_i > 0, so those rows are +Inf
    y = _run(csr, csr.val, x, **PARAMS[pi])
    assert np.all(y[bad] == np.inf), y[bad][y[bad] != np.inf][:10]
    x_clean = x.copy()
    x_clean[cols] = 0
    _check_clean_rows(csr, y, x_clean, bad)
