"""C5 at its full size (50M x 50M, ~1.0B non-zeros) in the launch configuration bench.py
times (1x1, T=32, C=128, i32 columns, GPU translation): outputs the oracle can compute row
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
