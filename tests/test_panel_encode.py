"""The C++ panel-sliced BCCOO+ encoder (csrc/panel.cpp, host-only handles, no GPU) against
the independent oracle (oracle/panel.py): every band array and every far-part array
bit-identical (readings P1-P6 of DESIGN.md §2.1; the far part follows E1-E9).  CPU only."""
import numpy as np
import pytest

import synth
from oracle import encode as E, panel as PN
from paper_conf_ppopp_yanlzz14_b200 import Matrix
from paper_conf_ppopp_yanlzz14_b200._lib import FAR_IN_PANEL, FAR_SEPARATE, PANEL_BC, PANEL_BT, YaspmvError


def _compare(csr, R, W, B, col0=0, far=(16, 256, 0, 0), fip=False):
    T, C, cm, em = far
    pp = PN.PanelParams(R=R, W=W, B=B, T=PANEL_BT, C=PANEL_BC, diag0=col0, far=E.Params(1, 1, 1, T, C, cm, em),
                        far_in_panel=fip)
    enc = PN.encode_panel(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, pp)
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=-1, T=T, C=C, col_mode=cm,
                        empty_mode=em, B=B, R=R, W=W, col0=col0, far=FAR_IN_PANEL if fip else FAR_SEPARATE)
    try:
        info = A.info()
        assert info["nnz"] == csr.nnz
        assert (info["band_blocks"], info["band_blocks_pad"], info["band_panels"], info["band_slices"]) == \
            (enc.nband, enc.nband_pad, enc.npanels, enc.KS)
        assert info["band_stops"] == int(enc.stop_ptr[:, -1].sum())
        assert np.array_equal(A.export("band_flags"), enc.flags)
        assert np.array_equal(A.export("band_col16"), enc.col16)
        assert np.array_equal(A.export("band_val").view(np.uint8), enc.val.view(np.uint8))
        assert np.array_equal(A.export("band_panel_blk0"), enc.panel_blk0)
        assert np.array_equal(A.export("band_slice_ptr"), enc.slice_ptr.ravel())
        assert np.array_equal(A.export("band_stop_ptr"), enc.stop_ptr.ravel())
        assert np.array_equal(A.export("band_first_row"), enc.first_row.ravel())
        assert np.array_equal(A.export("band_tile_rank"), enc.tile_rank)
        assert info["params"]["band_far"] == (FAR_IN_PANEL if fip else FAR_SEPARATE)
        if fip:   # P7: far slices in the band stream, no plain part
            assert info["band_far_blocks_pad"] == enc.far_blk0[-1]
            assert np.array_equal(A.export("band_far_col"), enc.far_col)
            assert np.array_equal(A.export("band_far_blk0"), enc.far_blk0)
            assert (info["nnzb"], info["ntiles"]) == (0, 0)
            return enc
        with pytest.raises(YaspmvError):
            A.export("band_far_col")
        f = enc.far
        assert (info["nnzb"], info["nnzb_pad"], info["ntiles"], info["n_stops"]) == \
            (f.nnzb, f.nnzb_pad, f.ntiles, f.n_stops)
        assert np.array_equal(A.export("flags"), f.flags)
        assert np.array_equal(A.export("col"), f.col)
        assert np.array_equal(A.export("val0").view(np.uint8), f.val[0].view(np.uint8))
        assert np.array_equal(A.export("seg_row"), f.seg_row)
        assert np.array_equal(A.export("zero_rows"), f.zero_rows)
        assert np.array_equal(A.export("cta_seg0"), f.cta_seg0)
    finally:
        A.free()
    return enc


@pytest.mark.parametrize("fip", [False, True])
def test_scaled_c5(fip):
    csr = synth.circuit_like_rows(0, 300_000, n=300_000, band=4096, n_net=3, net_log2=(12, 14))
    enc = _compare(csr, R=2048, W=1024, B=4096, fip=fip)
    assert enc.nband > 0.8 * csr.nnz and (enc.far_blk0[-1] if fip else enc.far.nnzb) > 0


@pytest.mark.parametrize("fip", [False, True])
@pytest.mark.parametrize("col0", [0, 1000, -700])
def test_scaled_c5_col0(col0, fip):
    csr = synth.circuit_like_rows(0, 40_000, n=50_000, band=2000, n_net=1, net_log2=(10, 11))
    _compare(csr, R=512, W=256, B=2000, col0=col0, far=(8, 128, E.COL_I32, E.EMPTY_MAP), fip=fip)


@pytest.mark.parametrize("fip", [False, True])
def test_webbase_like(fip):
    csr = synth.webbase_like(m=200_000)
    _compare(csr, R=4096, W=512, B=1024, fip=fip)


@pytest.mark.parametrize("fip", [False, True])
@pytest.mark.parametrize("seed", range(8))
def test_tiny(seed, fip):
    a = synth.random_tiny(seed, dtype=np.float32)
    _compare(a, R=256, W=8 * (1 + seed % 3), B=seed + 1, fip=fip)   # band = 0 means "plain format" in the ABI


def test_default_is_far_separate():
    a = synth.random_tiny(1, dtype=np.float32)
    A = Matrix.from_csr(a.m, a.n, a.row_ptr, a.col, a.val, device=-1, B=4, R=256, W=8)
    try:
        assert A.info()["params"]["band_far"] == FAR_SEPARATE
    finally:
        A.free()


def test_rejects_bad_band_params():
    a = synth.random_tiny(0, dtype=np.float32)
    for kw in (dict(B=8, R=100), dict(B=8, R=256, W=6), dict(B=8, R=256, W=8, h=2), dict(B=100000, R=256, W=8),
               dict(B=8, R=256, W=4), dict(B=8, R=256, W=8, far=3)):
        with pytest.raises(YaspmvError):
            Matrix.from_csr(a.m, a.n, a.row_ptr, a.col, a.val, device=-1, **kw)
    b = a.astype(np.float64)
    with pytest.raises(YaspmvError):
        Matrix.from_csr(b.m, b.n, b.row_ptr, b.col, b.val, device=-1, B=8, R=256, W=8)
