"""Panel-sliced BCCOO+ on the GPU (K4 panel_kernel, with the far entries as a separate far
part run by K1 first (the default) or as every panel's slice 0 (reading P7); DESIGN.md §2.1,
§6.6) against the oracle: y = A x within the BASELINE.json tolerance per row (O1), bitwise
exact with integer data, run-to-run deterministic; the uploaded band arrays read back from
the device equal oracle/panel.py; the power-iteration epilogue; shapes that exercise the
kernel's edges (panels past m, windows clipped at 0 and n, a tile spanning more slices than
are resident, unaligned x, empty band, negative / positive band_col0)."""
import numpy as np
import pytest

import synth
from oracle import encode as E, panel as PN, ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanlzz14_b200  # noqa: F401


def _build(csr, **kw):
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    return Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, **kw)


def _run(A, x_np, offset=0):
    xb = torch.zeros(x_np.size + offset, dtype=torch.float32, device="cuda")
    xb[offset:] = torch.from_numpy(x_np).cuda()
    y = A.spmv(xb[offset:])
    torch.cuda.synchronize()
    return y.cpu().numpy()


def _check(csr, y, x):
    y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    ok, worst = ref.check_tolerance(y, y_ref, bound, np.float32)
    assert ok, worst


CASES = {
    # name: (matrix factory, params)
    "c5-scaled": (lambda: synth.circuit_like_rows(0, 400_000, n=400_000, band=8192, n_net=4, net_log2=(12, 16)),
                  dict(B=8192, R=4096, W=1024, T=32, C=128, col_mode=E.COL_I32)),
    "c5-scaled-default-RW": (lambda: synth.circuit_like_rows(0, 300_000, n=300_000, band=65536, n_net=2,
                                                             net_log2=(14, 15)),
                             dict(B=65536, T=32, C=128, col_mode=E.COL_I32)),
    "webbase": (lambda: synth.webbase_like(m=200_000), dict(B=1024, R=4096, W=512)),
    "small-many-slices": (lambda: synth.circuit_like_rows(0, 20_000, n=20_000, band=3000, n_net=1, net_log2=(9, 10)),
                          dict(B=3000, R=256, W=128)),
    "col0-neg": (lambda: synth.circuit_like_rows(0, 30_000, n=40_000, band=2000, n_net=1, net_log2=(9, 10)),
                 dict(B=2000, R=512, W=256, col0=-1500)),
    "col0-pos": (lambda: synth.circuit_like_rows(0, 30_000, n=40_000, band=2000, n_net=1, net_log2=(9, 10)),
                 dict(B=2000, R=512, W=256, col0=9000, empty_mode=E.EMPTY_MAP)),
    "empty-band": (lambda: synth.circuit_like_rows(0, 5_000, n=5_000, band=100, n_net=0),
                   dict(B=4, R=256, W=8, col0=100000)),
    "all-band": (lambda: synth.circuit_like_rows(0, 9_000, n=9_000, band=500, n_net=0, p_local=1.0),
                 dict(B=20000, R=8192, W=4096)),
    "tiny-m": (lambda: synth.random_tiny(3, dtype=np.float32, m=17, n=23), dict(B=8, R=256, W=8)),
    # far part as BCCOO+ (S = 2): its slice results are combined by the band kernel
    "c5-scaled-far-S2": (lambda: synth.circuit_like_rows(0, 400_000, n=400_000, band=8192, n_net=4,
                                                         net_log2=(12, 16)),
                         dict(B=8192, R=4096, W=1024, S=2, T=32, C=128, col_mode=E.COL_I32, far=1)),
    "webbase-far-S3": (lambda: synth.webbase_like(m=200_000), dict(B=1024, R=4096, W=512, S=3, far=1)),
    # P7: one far row of 2^17-2^18 entries per panel region (its far slice spans 256-512
    # tiles: the look-back runs through tiles without a row stop) and panels whose far
    # slices hold FILLER rows
    "fip-long-rows": (lambda: synth.circuit_like_rows(0, 300_000, n=300_000, band=2000, n_net=3, net_log2=(16, 18),
                                                      p_local=0.5),
                      dict(B=2000, R=2048, W=1024, far=2)),
}
FARS = {"sep": 1, "fip": 2}


def _params(name, far):
    mk, params = CASES[name]
    return mk, dict(params, far=params.get("far", FARS[far]))


@pytest.mark.parametrize("far", sorted(FARS))
@pytest.mark.parametrize("name", sorted(CASES))
def test_tolerance_and_determinism(name, far):
    if "far" in CASES[name][1] and CASES[name][1]["far"] != FARS[far]:
        pytest.skip("the case fixes its far mode")
    mk, params = _params(name, far)
    csr = mk()
    x = synth.make_x(csr.n, np.float32, "uniform", 1)
    A = _build(csr, **params)
    try:
        y1 = _run(A, x)
        y2 = _run(A, x, offset=1)          # unaligned x: windows still agree mod 16 B
        _check(csr, y1, x)
        assert np.array_equal(y1.view(np.int32), _run(A, x).view(np.int32))   # deterministic
        _check(csr, y2, x)
        info = A.info()
        assert info["nnz"] == csr.nnz and info["band_panels"] == -(-csr.m // params.get("R", 16384))
    finally:
        A.free()


@pytest.mark.parametrize("far", sorted(FARS))
@pytest.mark.parametrize("name", ["c5-scaled", "small-many-slices", "col0-neg", "tiny-m", "fip-long-rows"])
def test_integer_exact(name, far):
    mk, params = _params(name, far)
    csr0 = mk()
    csr = synth.CSR(csr0.m, csr0.n, csr0.row_ptr, csr0.col,
                    np.random.default_rng(3).integers(-3, 4, csr0.nnz).astype(np.float32))
    x = synth.make_x(csr.n, np.float32, "int2", 2)
    A = _build(csr, **params)
    try:
        y = _run(A, x)
        ye, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
        assert np.array_equal(y.astype(np.float64), ye)
    finally:
        A.free()


@pytest.mark.parametrize("far", sorted(FARS))
@pytest.mark.parametrize("name", ["c5-scaled", "col0-pos", "small-many-slices", "fip-long-rows"])
def test_device_arrays_equal_oracle(name, far):
    mk, params = _params(name, far)
    csr = mk()
    from paper_conf_ppopp_yanlzz14_b200._lib import PANEL_BC, PANEL_BT
    farp = E.Params(1, 1, 1, params.get("T", 16), params.get("C", 256), params.get("col_mode", 0),
                    params.get("empty_mode", 0))
    fip = params["far"] == 2
    pp = PN.PanelParams(R=params.get("R", 16384), W=params.get("W", 16384), B=params["B"], T=PANEL_BT, C=PANEL_BC,
                        diag0=params.get("col0", 0), far=farp, far_in_panel=fip)
    enc = PN.encode_panel(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, pp)
    A = _build(csr, **params)
    try:
        assert np.array_equal(A.export("band_flags", device=True), enc.flags)
        assert np.array_equal(A.export("band_col16", device=True), enc.col16)
        assert np.array_equal(A.export("band_val", device=True).view(np.uint32), enc.val.view(np.uint32))
        assert np.array_equal(A.export("band_first_row", device=True), enc.first_row.ravel())
        assert np.array_equal(A.export("band_tile_rank", device=True), enc.tile_rank)
        assert np.array_equal(A.export("band_slice_ptr", device=True), enc.slice_ptr.ravel())
        assert np.array_equal(A.export("band_stop_ptr", device=True), enc.stop_ptr.ravel())
        if fip:
            assert np.array_equal(A.export("band_far_col", device=True), enc.far_col)
            assert np.array_equal(A.export("band_far_blk0", device=True), enc.far_blk0)
        else:
            assert np.array_equal(A.export("flags", device=True), enc.far.flags)
            assert np.array_equal(A.export("col", device=True), enc.far.col)
    finally:
        A.free()


def test_gpu_encoded_far_part():
    """flags 2|4 (drop the CSR, GPU translation of the far part) as bench.py builds C5."""
    mk, params = CASES["c5-scaled"]
    csr = mk()
    x = synth.make_x(csr.n, np.float32, "uniform", 5)
    A = _build(csr, flags=2 | 4, **params)
    try:
        _check(csr, _run(A, x), x)
    finally:
        A.free()


@pytest.mark.parametrize("name,far", [("c5-scaled", "sep"), ("c5-scaled", "fip"), ("webbase", "fip"),
                                      ("webbase-far-S3", "sep")])
def test_power_step(name, far):
    mk, params = _params(name, far)
    csr0 = mk()
    csr = synth.CSR(csr0.m, csr0.n, csr0.row_ptr, csr0.col,
                    np.random.default_rng(4).integers(-2, 3, csr0.nnz).astype(np.float32))
    A = _build(csr, **params)
    try:
        xn = synth.make_x(csr.n, np.float32, "int2", 1)
        x = torch.from_numpy(xn).cuda()
        y = torch.empty(csr.m, dtype=torch.float32, device="cuda")
        out = torch.zeros(1, dtype=torch.float64, device="cuda")
        inn = torch.tensor([4.0], dtype=torch.float64, device="cuda")   # scale 1/2: exact
        ye, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, xn)
        A.spmv_power(x, y, inn, out)
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy().astype(np.float64), ye / 2)
        assert out.item() == float(np.sum((ye / 2) ** 2))
        assert A.launches_per_spmv() == (1 if params["far"] == 2 else 2)
    finally:
        A.free()


def test_host_buffers():
    mk, params = CASES["webbase"]
    csr = mk()
    x = synth.make_x(csr.n, np.float32, "uniform", 6)
    A = _build(csr, **params)
    try:
        _check(csr, A.spmv_host(x), x)
    finally:
        A.free()


def test_tune_and_reencode_keep_the_band():
    """yaspmv_tune on a panel-sliced handle times the far entries inside the panels (P7)
    against a separate far part tuned over Table 1 (1x1 blocks) and keeps the band stream;
    yaspmv_reencode(band = -1) returns to the plain format."""
    mk, params = CASES["webbase"]
    csr = mk()
    x = synth.make_x(csr.n, np.float32, "uniform", 7)
    A = _build(csr, **params)
    try:
        chosen = A.tune()
        info = A.info()
        assert info["band_blocks"] > 0 and chosen["block_h"] == chosen["block_w"] == 1
        assert info["params"]["band"] == params["B"] and chosen["band_far"] in (1, 2)
        assert info["params"]["band_far"] == chosen["band_far"]
        _check(csr, _run(A, x), x)
        A.reencode(B=-1)
        assert A.info()["band_blocks"] == 0
        _check(csr, _run(A, x), x)
    finally:
        A.free()


_CTA_SCRIPT = r"""
import sys, json, numpy as np, torch
sys.path.insert(0, %r)
import synth
from oracle import ref
from paper_conf_ppopp_yanlzz14_b200 import Matrix
out = []
for far, S in ((1, 3), (2, 1)):
    csr = synth.circuit_like_rows(0, 300_000, n=300_000, band=8192, n_net=3, net_log2=(12, 16))
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, B=8192, R=4096, W=2048,
                        S=S, T=8, C=128, far=far)
    x = synth.make_x(csr.n, np.float32, "uniform", 3)
    y1 = A.spmv(torch.from_numpy(x).cuda()).cpu().numpy()
    y2 = A.spmv(torch.from_numpy(x).cuda()).cpu().numpy()
    y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    ok, worst = ref.check_tolerance(y1, y_ref, bound, np.float32)
    out.append(dict(ok=bool(ok), worst=float(worst), det=bool(np.array_equal(y1.view(np.uint32), y2.view(np.uint32))),
                    regs=A.info()["band_regs"] if "band_regs" in A.info() else None))
    A.free()
print("CTA-RESULT " + json.dumps(out))
"""


@pytest.mark.parametrize("cta", [512, 640, 704, 768, 896, 1024])
def test_band_kernel_every_cta_size(cta):
    """The band kernel's CTA size (YASPMV_PANEL_CTA, read once per process): every compiled
    size — 19 / 21 / 23 / 27 / 31 compute warps + the window producer — against the oracle
    (separate far part with S = 3, and the far entries as slice 0, P7), run-to-run bitwise."""
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, YASPMV_PANEL_CTA=str(cta))
    r = subprocess.run([sys.executable, "-c", _CTA_SCRIPT % root], env=env, capture_output=True, text=True,
                       timeout=600)
    line = [l for l in r.stdout.splitlines() if l.startswith("CTA-RESULT ")]
    assert line, r.stdout[-2000:] + r.stderr[-2000:]
    for res in json.loads(line[0][len("CTA-RESULT "):]):
        assert res["ok"], res
        assert res["det"], res
