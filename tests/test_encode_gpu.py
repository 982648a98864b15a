"""GPU-accelerated translation to BCCOO/BCCOO+ (PAPER.md P:321): every array the GPU
encoder writes (read back from the device and un-permuted) is bit-identical to the
oracle encoder's canonical array, for a grid of shapes / slices / column modes / empty-row
modes, and the SpMV over it is exact on integer data."""
import itertools

import numpy as np
import pytest

import synth
from oracle import encode as E, ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
GPU_ENCODE = 4


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _check(csr, h, w, S, T, C, cm, em):
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, YaspmvError
    try:
        A = Matrix.from_synth(csr, device=0, h=h, w=w, S=S, T=T, C=C, col_mode=cm, empty_mode=em,
                              flags=GPU_ENCODE)
    except YaspmvError as e:
        assert e.status == 4  # no kernel compiled for this combination
        return
    info = A.info()
    q = info["params"]
    enc = E.encode(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, E.Params(h, w, S, T, C, cm, em))
    assert (q["col_mode"], q["empty_mode"]) == (enc.p.col_mode, enc.p.empty_mode)
    assert (info["nnzb"], info["nnzb_pad"], info["ntiles"], info["n_stops"], info["n_filler"], info["n_zero_rows"]) == \
        (enc.nnzb, enc.nnzb_pad, enc.ntiles, enc.n_stops, enc.n_filler, enc.zero_rows.size)
    assert np.array_equal(A.export("flags", device=True), enc.flags)
    assert np.array_equal(A.export("col", device=True), enc.col)
    if enc.p.col_mode == E.COL_DELTA:
        assert np.array_equal(A.export("col_delta", device=True), enc.col_delta)
    for r in range(h):
        assert np.array_equal(A.export(f"val{r}", device=True).view(np.uint8), enc.val[r].view(np.uint8))
    assert np.array_equal(A.export("cta_seg0", device=True), enc.cta_seg0)
    assert np.array_equal(A.export("fre", device=True), enc.fre)
    if enc.seg_row.size:
        assert np.array_equal(A.export("seg_row", device=True), enc.seg_row)
        assert np.array_equal(A.export("zero_rows", device=True), enc.zero_rows)
    x = synth.make_x(csr.n, csr.val.dtype, "int2", 3)
    y = A.spmv(torch.from_numpy(x).cuda()).cpu().numpy()
    ye, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    assert np.array_equal(y.astype(np.float64), ye)
    A.free()


@pytest.mark.parametrize("seed", range(12))
def test_gpu_encoder_grid(seed):
    rng = np.random.default_rng(seed)
    dt = np.float32 if seed % 2 == 0 else np.float64
    m, n = int(rng.integers(1, 2500)), int(rng.integers(1, 2500))
    a = synth.random_tiny(seed, m=m, n=n, density=float(rng.uniform(0.001, 0.05)), dtype=dt, integer=True)
    combos = list(itertools.product([1, 2, 3, 4], [1, 2, 4, 8], [4, 8, 16, 32], [64, 128, 256],
                                    [0, E.COL_I32, E.COL_DELTA], [E.EMPTY_FILLER, E.EMPTY_MAP]))
    for i in rng.choice(len(combos), size=6, replace=False):
        h, w, T, C, cm, em = combos[i]
        NB = -(-a.n // w)
        for S in sorted({1, min(3, NB)}):
            _check(a, h, w, S, T, C, cm, em)


@pytest.mark.parametrize("name,p", [("c4", (1, 1, 1, 16, 128, 0, 0)), ("c4", (1, 1, 4, 8, 128, E.COL_DELTA, E.EMPTY_MAP)),
                                    ("c3-ship", (2, 2, 1, 32, 128, 0, 0)), ("c2-f64", (4, 2, 1, 4, 128, 0, 0))])
def test_gpu_encoder_configs(name, p):
    _check(synth.config_matrix(name, integer=True), *p)
