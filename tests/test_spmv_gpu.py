"""GPU parity of the CUDA path (through the C ABI) against the CPU oracle.

  * integer-valued A and x: y BITWISE equal to the oracle for every parameter set;
  * realistic values: per-row tolerance of BASELINE.json (fp64 1e-12, fp32 1e-5 x sum|a||x|);
  * run-to-run bitwise determinism; device arrays equal the oracle's canonical arrays;
  * edge cases: empty, 1x1, one long row over many CTAs, ragged h/w, NB around 65535,
    delta escapes, empty rows in both empty-row modes.
"""
import itertools

import numpy as np
import pytest

import synth
from oracle import decode, encode as E, ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_ppopp_yanlzz14_b200  # noqa: F401  (fails loudly if the .so is missing)


def _mat():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    return Matrix


def _run(csr, x, **params):
    Matrix = _mat()
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, **params)
    try:
        xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
        y = A.spmv(xd)
        torch.cuda.synchronize()
        return y.cpu().numpy(), A.info()
    finally:
        A.free()


def _dense_exact(csr, x):
    return csr.to_dense().astype(np.float64) @ x.astype(np.float64)


# ----------------------------------------------------------------------------- paper example
@pytest.mark.parametrize("S", [1, 2])
@pytest.mark.parametrize("T,C", [(4, 64), (16, 256), (32, 256), (8, 512)])
def test_paper_example_A(S, T, C):
    A = np.array([[0, 0, 1, 0, 0, 0, 2, 3], [0, 0, 4, 5, 0, 0, 6, 0],
                  [0, 0, 0, 0, 7, 8, 9, 10], [11, 12, 0, 0, 13, 14, 15, 16]], dtype=np.float32)
    r, c = np.nonzero(A)
    rp = np.zeros(5, dtype=np.int64); np.cumsum(np.bincount(r, minlength=4), out=rp[1:])
    csr = synth.CSR(4, 8, rp, c.astype(np.int32), A[r, c])
    y, _ = _run(csr, np.arange(1, 9, dtype=np.float32), h=2, w=2, S=S, T=T, C=C)
    assert y.tolist() == [41, 74, 226, 417]          # Fig. 5


def test_launch_bound_is_reported():
    """2x2 fp32 blocks with T=32 hold 512 B of values per thread: compiled for C <= 256
    only; C = 512 is refused with EUNSUPPORTED instead of failing at launch."""
    from paper_conf_ppopp_yanlzz14_b200 import YaspmvError
    csr = synth.random_tiny(1, m=8, n=8, density=0.5, dtype=np.float32)
    with pytest.raises(YaspmvError) as e:
        _run(csr, np.ones(8, np.float32), h=2, w=2, T=32, C=512)
    assert e.value.status == 4


# ----------------------------------------------------------------------------- brute force grid
GRID = list(itertools.product([1, 2, 3, 4], [1, 2, 4, 8], [4, 8, 16, 32], [64, 128, 256, 512],
                              [0, E.COL_I32, E.COL_DELTA], [E.EMPTY_FILLER, E.EMPTY_MAP]))


@pytest.mark.parametrize("seed", range(30))
def test_integer_exact_random_grid(seed):
    rng = np.random.default_rng(seed)
    dt = np.float32 if seed % 2 == 0 else np.float64
    # several tiles: a few hundred rows, sometimes long rows
    m = int(rng.integers(1, 3000)); n = int(rng.integers(1, 3000))
    dens = float(rng.uniform(0.0005, 0.05))
    a = synth.random_tiny(seed, m=m, n=n, density=dens, dtype=dt, integer=True)
    x = synth.make_x(n, dt, "int", seed)
    y_exact = _dense_exact(a, x)
    for i in rng.choice(len(GRID), size=6, replace=False):
        h, w, T, C, cm, em = GRID[i]
        NB = -(-n // w)
        for S in sorted({1, min(3, NB)}):
            try:
                y, info = _run(a, x, h=h, w=w, S=S, T=T, C=C, col_mode=cm, empty_mode=em)
            except Exception as e:  # combinations without a compiled kernel are reported, not run
                assert "no compiled kernel" in str(e) or "launch bound" in str(e), e
                continue
            assert np.array_equal(y.astype(np.float64), y_exact), (h, w, T, C, S, cm, em, info)


@pytest.mark.parametrize("flags", [0, 8, 32])
def test_long_row_spanning_many_ctas(flags):
    """One row of 600k entries crosses hundreds of workgroup tiles: carries travel through
    the look-back chain (adjacent synchronization)."""
    n = 700_000
    rng = np.random.default_rng(7)
    cols = np.sort(rng.choice(n, size=600_000, replace=False)).astype(np.int32)
    rows = [np.array([0], np.int32), cols, np.array([3, 9], np.int32)]
    rp = np.array([0, 1, 1 + cols.size, 3 + cols.size], dtype=np.int64)
    col = np.concatenate(rows)
    val = rng.integers(-2, 3, size=col.size).astype(np.float32)
    csr = synth.CSR(3, n, rp, col, val)
    x = synth.make_x(n, np.float32, "int2", 1)
    ref_y = _dense_exact_rows(csr, x)
    for T, C in ((4, 64), (16, 256), (32, 512)):
        y, info = _run(csr, x, T=T, C=C, col_mode=E.COL_I32, flags=flags)
        assert info["ntiles"] > 30
        assert np.array_equal(y.astype(np.float64), ref_y)


def _dense_exact_rows(csr, x):
    y, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    return y


# ----------------------------------------------------------------------------- configs
CONFIG_PARAMS = {
    "c1": [dict(T=4, C=64), dict(T=16, C=256)],
    "c2-f32": [dict(h=4, w=4, T=4, C=128), dict(h=2, w=4, T=8, C=256)],
    "c2-f64": [dict(h=4, w=4, T=4, C=128), dict(h=4, w=2, T=4, C=256)],
    "c3-spheres": [dict(h=4, w=4, T=4, C=256), dict(h=2, w=2, T=8, C=128)],
    "c3-cantilever": [dict(h=4, w=4, T=4, C=128)],
    "c3-ship": [dict(h=2, w=2, T=8, C=256), dict(h=4, w=4, T=4, C=256)],
    "c3-ship-f64": [dict(h=2, w=2, T=8, C=128)],
    "c4": [dict(T=16, C=256), dict(T=8, C=128, S=4), dict(T=16, C=128, col_mode=E.COL_DELTA, empty_mode=E.EMPTY_MAP)],
}


@pytest.mark.parametrize("name", list(CONFIG_PARAMS))
def test_configs_tolerance(name):
    _configs_tolerance(name, 0)


@pytest.mark.parametrize("name", ["c1", "c3-ship", "c4"])
def test_configs_tolerance_ticket_ids(name):
    """YASPMV_TICKET_IDS: logical tile ids from the atomic ticket."""
    _configs_tolerance(name, 8)


def _configs_tolerance(name, flags):
    csr = synth.config_matrix(name)
    dt = csr.val.dtype
    x = synth.make_x(csr.n, dt, "unit" if name == "c4" else "uniform", 3)
    y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    for p in CONFIG_PARAMS[name]:
        y, info = _run(csr, x, flags=flags, **p)
        ok, worst = ref.check_tolerance(y, y_ref, bound, dt)
        assert ok, (name, p, worst)


@pytest.mark.parametrize("name", ["c1", "c3-ship", "c4"])
def test_configs_tolerance_forced_handoff(name):
    """YASPMV_FORCE_HANDOFF: every carried first segment goes through the non-blocking
    hand-off (tile k leaves its partial, whichever of tiles k-1 / k arrives second finishes
    it); both finishing sides occur, and y equals the default path bit for bit."""
    _configs_tolerance(name, 32)
    csr = synth.config_matrix(name)
    x = synth.make_x(csr.n, csr.val.dtype, "unit" if name == "c4" else "uniform", 3)
    for p in CONFIG_PARAMS[name]:
        y0, _ = _run(csr, x, flags=0, **p)
        y1, _ = _run(csr, x, flags=32, **p)
        assert np.array_equal(y0, y1), (name, p)


@pytest.mark.parametrize("name", ["c2-f32", "c3-ship", "c4"])
def test_configs_integer_exact(name):
    csr = synth.config_matrix(name, integer=True)
    x = synth.make_x(csr.n, csr.val.dtype, "int2", 4)
    y_ref, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    for p in CONFIG_PARAMS[name][:2]:
        y, _ = _run(csr, x, **p)
        assert np.array_equal(y.astype(np.float64), y_ref), p


def test_deterministic_and_device_arrays_match_oracle():
    Matrix = _mat()
    csr = synth.config_matrix("c4")
    x = torch.from_numpy(synth.make_x(csr.n, np.float32, "unit", 5)).cuda()
    for p in (dict(T=16, C=256), dict(T=8, C=128, S=2, col_mode=E.COL_DELTA), dict(T=32, C=512, empty_mode=2)):
        A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, flags=1, **p)
        ys = [A.spmv(x).cpu().numpy() for _ in range(5)]
        for y in ys[1:]:
            assert np.array_equal(y.view(np.uint32), ys[0].view(np.uint32))
        info = A.info()
        q = info["params"]
        enc = E.encode(csr.m, csr.n, csr.row_ptr, csr.col, csr.val,
                       E.Params(q["block_h"], q["block_w"], q["slices"], q["thread_tile"], q["cta_size"],
                                q["col_mode"], q["empty_mode"]))
        assert np.array_equal(A.export("flags", device=True), enc.flags)
        assert np.array_equal(A.export("col", device=True), enc.col)
        assert np.array_equal(A.export("val0", device=True), enc.val[0])
        assert np.array_equal(A.export("cta_seg0", device=True), enc.cta_seg0)
        assert np.array_equal(A.export("fre", device=True), enc.fre)
        if enc.p.col_mode == E.COL_DELTA:
            assert np.array_equal(A.export("col_delta", device=True), enc.col_delta)
        if enc.seg_row.size:
            assert np.array_equal(A.export("seg_row", device=True), enc.seg_row)
            assert np.array_equal(A.export("zero_rows", device=True), enc.zero_rows)
        A.free()


# ----------------------------------------------------------------------------- edge cases
def test_edge_empty_and_tiny():
    Matrix = _mat()
    # nnz = 0 in both empty-row modes -> y = 0
    for em in (1, 2):
        csr = synth.CSR(5, 4, np.zeros(6, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32))
        y, _ = _run(csr, np.ones(4, np.float32), empty_mode=em)
        assert np.array_equal(y, np.zeros(5, np.float32))
    # 1 x 1
    csr = synth.CSR(1, 1, np.array([0, 1]), np.array([0], np.int32), np.array([3.0]))
    y, _ = _run(csr, np.array([2.0]))
    assert y.tolist() == [6.0]
    # single column, all rows non-empty
    m = 10000
    csr = synth.CSR(m, 1, np.arange(m + 1, dtype=np.int64), np.zeros(m, np.int32), np.arange(m, dtype=np.float64))
    y, _ = _run(csr, np.array([2.0]), T=4, C=64)
    assert np.array_equal(y, 2.0 * np.arange(m))
    # all rows empty but one, y stays 0 for the empty rows in both modes
    rp = np.zeros(2001, np.int64); rp[1001:] = 3
    csr = synth.CSR(2000, 50, rp, np.array([1, 7, 49], np.int32), np.array([1.0, 2.0, 3.0], np.float32))
    x = np.arange(50, dtype=np.float32)
    for em in (1, 2):
        for S in (1, 3):
            y, _ = _run(csr, x, empty_mode=em, S=S)
            exp = np.zeros(2000, np.float32); exp[1000] = 1 + 14 + 147
            assert np.array_equal(y, exp)
    # zero-sized matrices
    Matrix.from_csr(0, 0, np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0, np.float32), device=0).free()


@pytest.mark.parametrize("n", [65534 * 1, 65535, 65536])
def test_edge_column_type_switch(n):
    a = synth.random_tiny(11, m=300, n=n, density=0.0005, dtype=np.float32, integer=True)
    x = synth.make_x(n, np.float32, "int", 2)
    ye = _dense_exact_rows(a, x)
    y, info = _run(a, x)
    assert info["params"]["col_mode"] == (1 if n < 65535 else 2)
    assert np.array_equal(y.astype(np.float64), ye)
    y, info = _run(a, x, col_mode=E.COL_DELTA, T=8, C=64)
    assert np.array_equal(y.astype(np.float64), ye)


def test_edge_ragged_blocks_and_delta_escapes():
    # M, N not multiples of h, w; deltas at +-32767, 32768, -1
    m, n = 1003, 200_001
    rows, cols = [], []
    for i in range(m):
        base = (i * 37) % (n - 70_000)
        for c in (base, base + 32767, base + 32767 + 32768, base + 32767 + 32768 - 1, n - 1):
            rows.append(i); cols.append(c)
    rows = np.array(rows); cols = np.array(cols)
    key = np.unique(rows * n + cols)
    r = key // n; c = (key % n).astype(np.int32)
    rp = np.zeros(m + 1, np.int64); np.cumsum(np.bincount(r, minlength=m), out=rp[1:])
    val = (np.arange(c.size) % 5 - 2).astype(np.float32)
    csr = synth.CSR(m, n, rp, c, val)
    x = synth.make_x(n, np.float32, "int", 9)
    ye = _dense_exact_rows(csr, x)
    for h, w in ((1, 1), (3, 1), (4, 4), (3, 2)):
        for cm in (E.COL_I32, E.COL_DELTA):
            T = 4 if h * w > 8 else 8
            y, _ = _run(csr, x, h=h, w=w, T=T, C=64, col_mode=cm)
            assert np.array_equal(y.astype(np.float64), ye), (h, w, cm)


def test_spmv_host_and_power_helpers():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, nrm2sq, nrm2sq_scratch_bytes, scale
    csr = synth.config_matrix("c3-cantilever")
    x = synth.make_x(csr.n, np.float32, "uniform", 6)
    A = Matrix.from_synth(csr, device=0, h=4, w=4, T=4, C=128)
    yd = A.spmv(torch.from_numpy(x).cuda()).cpu().numpy()
    yh = A.spmv_host(x)
    assert np.array_equal(yd, yh)
    v = torch.from_numpy(yh).cuda()
    out = torch.zeros(1, dtype=torch.float64, device="cuda")
    scratch = torch.zeros(nrm2sq_scratch_bytes(v.numel()) // 8 + 1, dtype=torch.float64, device="cuda")
    nrm2sq(v, out, scratch)
    exp = float(np.sum(yh.astype(np.float64) ** 2))
    assert abs(out.item() - exp) <= 1e-12 * exp
    dst = torch.empty_like(v)
    scale(v, dst, out)
    assert np.allclose(dst.cpu().numpy(), yh / np.sqrt(exp), rtol=1e-6, atol=0)
    A.free()


@pytest.mark.parametrize("flags", [0, 4])
def test_tune_keeps_results(flags):
    """yaspmv_tune (§4): host encode + derived (T, C) variants, or GPU translation."""
    Matrix = _mat()
    csr = synth.config_matrix("c3-cantilever")
    x = synth.make_x(csr.n, np.float32, "uniform", 8)
    y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    A = Matrix.from_synth(csr, device=0, flags=flags)
    chosen = A.tune()
    info = A.info()
    assert info["tune_seconds"] > 0 and chosen["block_h"] in (1, 2, 3, 4) and info["tune_candidates"] > 8
    y = A.spmv(torch.from_numpy(x).cuda()).cpu().numpy()
    assert ref.check_tolerance(y, y_ref, bound, np.float32)[0]
    A.free()


def test_oracle_decode_matches_gpu_on_bccoo_plus():
    """O3 (decode of the canonical arrays) and the GPU agree exactly on integer data with
    several slices (Fig. 5 combine)."""
    csr = synth.webbase_like(m=50_000, integer=True)
    x = synth.make_x(csr.n, np.float32, "int2", 12)
    for S in (2, 5):
        enc = E.encode(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, E.Params(1, 1, S, 8, 128, 0, 0))
        y, _ = _run(csr, x, S=S, T=8, C=128)
        assert np.array_equal(y.astype(np.float64), decode.spmv(enc, x))


# ------------------------------------------------------------- warp-staged y stores (wstage)
@pytest.mark.parametrize("params", [dict(T=8, C=256), dict(T=8, C=256, S=3), dict(T=16, C=128, tpc=2),
                                    dict(T=4, C=64, S=2), dict(T=32, C=256)])
def test_warp_staged_stores_bitwise(params, monkeypatch):
    """KArgs::wstage (each warp's finished rows staged in shared memory and written as one
    contiguous run, plain or streaming stores) writes exactly the values of the direct
    per-row stores: y bitwise equal for wstage 0 / 1 / 2, and equal to the oracle's exact
    integer result (integer-valued A, x), on a power-law matrix with empty rows, a long row
    over many tiles (the carried segment's slot is skipped by the staged write-out) and
    BCCOO+ slices."""
    csr = synth.webbase_like(m=60000, integer=True)
    x = np.random.default_rng(2).integers(-2, 3, csr.n).astype(np.float32)
    exact = ref.spmv(csr.row_ptr, csr.col, csr.val, x)[0]
    ys = []
    for ws in ("0", "1", "2"):
        monkeypatch.setenv("YASPMV_WSTAGE", ws)
        y, _ = _run(csr, x, **params)
        ys.append(y)
    for y in ys[1:]:
        assert np.array_equal(ys[0].view(np.uint32), y.view(np.uint32))
    assert np.array_equal(ys[0].astype(np.float64), exact)


def test_warp_staged_stores_power_step(monkeypatch):
    """The staged stores under the power-iteration epilogue (EPI 1: y scaled by 1/sqrt(in),
    sum y^2 partials): y and ||y||^2 bitwise equal for wstage 0 and 2 (the per-thread y^2
    accumulation order is unchanged by the staging)."""
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = synth.webbase_like(m=60000)
    x = torch.from_numpy(synth.make_x(csr.n, np.float32, "uniform", 4)).cuda()
    outs = []
    for ws in ("0", "2"):
        monkeypatch.setenv("YASPMV_WSTAGE", ws)
        A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, T=8, C=128, tpc=2)
        n_in = torch.full((1,), 4.0, dtype=torch.float64, device="cuda")
        n_out = torch.zeros(1, dtype=torch.float64, device="cuda")
        y = torch.empty(csr.m, dtype=torch.float32, device="cuda")
        A.spmv_power(x, y, n_in, n_out)
        torch.cuda.synchronize()
        outs.append((y.cpu().numpy(), float(n_out.item())))
        A.free()
    assert np.array_equal(outs[0][0].view(np.uint32), outs[1][0].view(np.uint32))
    assert outs[0][1] == outs[1][1]
    y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x.cpu().numpy())
    ok, worst = ref.check_tolerance(outs[0][0], y_ref / 2.0, bound / 2.0, np.float32)
    assert ok, worst
