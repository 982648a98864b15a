"""C5 at its full size (50M x 50M, ~1.0B non-zeros) in the launch configuration bench.py
times (bench.DEFAULT_PARAMS["c5"]): outputs the oracle can compute row
by row are checked — a uniform sample of rows plus every long 'net' row (2^16-2^21 entries,
spanning up to ~500 workgroup tiles, so their carries cross hundreds of CTAs) — for both
the plain SpMV and the fused power-iteration step, plus run-to-run bitwise determinism."""
import numpy as np
import pytest

from oracle import ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def c5():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from synth import matrices as sm
    import bench
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = sm.circuit_like_rows(0, 50_000_000)
    params = dict(bench.DEFAULT_PARAMS["c5"])
    A = Matrix.from_synth(csr, device=0, flags=2 | 4, **params)
    yield csr, A
    A.free()


def _sample_rows(csr):
    from synth import matrices as sm
    net, _ = sm.c5_net_rows()
    rng = np.random.default_rng(5)
    rows = np.unique(np.concatenate([rng.integers(0, csr.m, 200_000), net, [0, csr.m - 1]]))
    return rows, net


def test_c5_spmv_sampled_rows(c5):
    csr, A = c5
    x_np = np.random.default_rng(7).uniform(-1, 1, csr.n).astype(np.float32)
    x = torch.from_numpy(x_np).cuda()
    y1 = A.spmv(x)
    y2 = A.spmv(x)
    torch.cuda.synchronize()
    assert torch.equal(y1.view(torch.int32), y2.view(torch.int32))   # bitwise deterministic
    rows, net = _sample_rows(csr)
    yr, bound = ref.spmv_rows(rows, csr.row_ptr, csr.col, csr.val, x_np)
    got = y1.cpu().numpy()[rows]
    ok, worst = ref.check_tolerance(got, yr, bound, np.float32)
    assert ok, worst
    assert A.info()["nnz"] == csr.nnz and (np.diff(csr.row_ptr)[net] > 60_000).all()


def test_c5_power_step_sampled_rows(c5):
    csr, A = c5
    x_np = np.full(csr.n, 1.0 / np.sqrt(csr.n), dtype=np.float32)
    x = torch.from_numpy(x_np).cuda()
    y = torch.empty(csr.m, dtype=torch.float32, device="cuda")
    inn = torch.tensor([9.0], dtype=torch.float64, device="cuda")
    out = torch.zeros(1, dtype=torch.float64, device="cuda")
    A.spmv_power(x, y, inn, out)
    torch.cuda.synchronize()
    rows, _ = _sample_rows(csr)
    yr, bound = ref.spmv_rows(rows, csr.row_ptr, csr.col, csr.val, x_np)
    ok, worst = ref.check_tolerance(y.cpu().numpy()[rows] * 3.0, yr, bound, np.float32)
    assert ok, worst
    yy = y.cpu().numpy().astype(np.float64)
    assert abs(out.item() - float(np.dot(yy, yy))) <= 1e-6 * out.item()


def _panel_windows(csr, R):
    """Panel windows to check: the first two panels, the panel of the longest net row,
    the last two panels."""
    from synth import matrices as sm
    net, ln = sm.c5_net_rows()
    npan = -(-csr.m // R)
    pn = int(net[np.argmax(ln)]) // R
    return sorted({(0, 2), (pn, pn + 1), (npan - 2, npan)})


def test_c5_encoding_windows_bit_exact(c5):
    """north_star "Encoded arrays and row-segment boundaries must match bit-exactly" at C5
    scale: windows of the device arrays of the bench's handle (host panel encoder for the
    band stream, GPU translation, for the BCCOO+ far part) against oracle/encode.py
    and oracle/panel.py run on the same rows (
    readings P1-P6)."""
    from oracle import encode as E, panel as PN
    csr, A = c5
    info = A.info()
    prm = info["params"]
    R, W, B = prm["panel_rows"], prm["slice_width"], prm["band"]
    S, T, C = prm["slices"], prm["thread_tile"], prm["cta_size"]
    assert B > 0 and info["band_panels"] == -(-csr.m // R)
    fip = prm["band_far"] == 2
    blk0 = A.export("band_panel_blk0", device=True)
    fblk0 = A.export("band_far_blk0", device=True) if fip else np.zeros_like(blk0)
    sptr = A.export("band_slice_ptr", device=True).reshape(info["band_panels"], -1)
    frow = A.export("band_first_row", device=True).reshape(info["band_panels"], -1)
    if not fip:
        far_flags = np.unpackbits(A.export("flags", device=True), bitorder="little")
        far_stop = np.flatnonzero(far_flags[: info["nnzb"]] == 0)      # FILLER: stop k ends stacked row k
        assert prm["empty_mode"] == E.EMPTY_FILLER and far_stop.size == S * csr.m
    TCf = T * C
    for p0, p1 in _panel_windows(csr, R):
        r0, r1 = p0 * R, min(csr.m, p1 * R)
        sub = csr.row_slice(r0, r1)
        pp = PN.PanelParams(R=R, W=W, B=B, T=16, C=32, diag0=r0,
                            far=E.Params(1, 1, S, T, C, prm["col_mode"], E.EMPTY_FILLER), far_in_panel=fip)
        # the window's slices use the full matrix' slice width of the far part
        enc = PN.encode_panel(sub.m, csr.n, sub.row_ptr, sub.col, sub.val, pp)
        # band stream: panels are independent, so the window's arrays are a slice of the whole
        assert np.array_equal(sptr[p0:p1], enc.slice_ptr) and np.array_equal(frow[p0:p1], enc.first_row)
        t0, nt = int(blk0[p0]) // 512, (int(blk0[p1]) - int(blk0[p0])) // 512
        assert nt == enc.nband_pad // 512
        assert np.array_equal(A.export_range("band_flags", t0, nt), enc.flags)
        assert np.array_equal(A.export_range("band_val", t0, nt).view(np.uint32), enc.val.view(np.uint32))
        assert np.array_equal(A.export_range("band_tile_rank", t0, nt), enc.tile_rank)
        # col16 counts band blocks only, far_col far-slice blocks only (P7)
        f0, f1 = int(fblk0[p0]) // 512, int(fblk0[p1]) // 512
        assert np.array_equal(A.export_range("band_col16", t0 - f0, nt - (f1 - f0)), enc.col16)
        if fip:
            assert np.array_equal(A.export_range("band_far_col", f0, f1 - f0), enc.far_col)
            assert np.array_equal(fblk0[p0:p1 + 1] - fblk0[p0], enc.far_blk0)
            continue
        # far part (BCCOO+, S slices stacked top-down): stacked rows s*m + [r0, r1)
        ef = enc.far
        ebits = np.unpackbits(ef.flags, bitorder="little")[: ef.nnzb]
        estop = np.flatnonzero(ebits == 0)
        ecol = ef.col.astype(np.int64)
        for s in range(S):
            gb0 = 0 if s * csr.m + r0 == 0 else int(far_stop[s * csr.m + r0 - 1]) + 1
            gb1 = int(far_stop[s * csr.m + r1 - 1]) + 1
            wb0 = 0 if s * sub.m == 0 else int(estop[s * sub.m - 1]) + 1
            wb1 = int(estop[s * sub.m + sub.m - 1]) + 1
            assert gb1 - gb0 == wb1 - wb0
            k0, k1 = gb0 // TCf, -(-gb1 // TCf)
            off = gb0 - k0 * TCf
            fl = np.unpackbits(A.export_range("flags", k0, k1 - k0), bitorder="little")
            assert np.array_equal(fl[off: off + gb1 - gb0], ebits[wb0:wb1])
            col = A.export_range("col", k0, k1 - k0).astype(np.int64)
            assert np.array_equal(col[off: off + gb1 - gb0], ecol[wb0:wb1])
            v = A.export_range("val0", k0, k1 - k0).view(np.uint32)
            assert np.array_equal(v[off: off + gb1 - gb0], ef.val[0].view(np.uint32)[wb0:wb1])
