"""Runtime properties of the CUDA path: CUDA-graph replay (the per-launch epoch and ticket
live on the device, so replays stay correct), the pipelined host API, and a
compute-sanitizer memcheck / synccheck run of the kernels."""
import os
import subprocess
import sys

import numpy as np
import pytest

import synth
from oracle import ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def _gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def test_cuda_graph_replay():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = synth.webbase_like(m=200_000, integer=True)
    A = Matrix.from_synth(csr, device=0, T=8, C=128, S=2)
    xs = [synth.make_x(csr.n, np.float32, "int2", s) for s in range(3)]
    x = torch.from_numpy(xs[0]).cuda()
    y = torch.empty(csr.m, dtype=torch.float32, device="cuda")
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        A.spmv(x, y)  # warm-up outside capture
    torch.cuda.current_stream().wait_stream(s)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        A.spmv(x, y)
        A.spmv(x, y)
    for k in range(3):
        x.copy_(torch.from_numpy(xs[k]))
        g.replay()
        torch.cuda.synchronize()
        ye, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, xs[k])
        assert np.array_equal(y.cpu().numpy().astype(np.float64), ye)
    A.free()


@pytest.mark.parametrize("flags", [0, 16, 8, 8 | 16])
@pytest.mark.parametrize("S,empty", [(1, 2), (2, 1)])
def test_back_to_back_chain(flags, S, empty):
    """Dependent SpMVs queued without a host sync (x_{k+1} = A x_k, ping-pong buffers):
    with programmatic dependent launch (default) the next launch streams its matrix tiles
    while the previous drains, but x, y, the zero-fill and the carries wait for it.
    Exact on an integer f64 matrix (|A x| stays far below 2^53)."""
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = synth.webbase_like(m=300_000, dtype=np.float64, integer=True)
    A = Matrix.from_synth(csr, device=0, T=8, C=128, S=S, empty_mode=empty, flags=flags)
    x0 = synth.make_x(csr.n, np.float64, "int2", 5)
    buf = [torch.from_numpy(x0).cuda(), torch.empty(csr.m, dtype=torch.float64, device="cuda")]
    for k in range(4):
        A.spmv(buf[k % 2], buf[(k + 1) % 2])
    torch.cuda.synchronize()
    ye = x0
    for k in range(4):
        ye, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, ye)
    assert np.array_equal(buf[0].cpu().numpy(), ye)
    A.free()


def test_host_async_pipeline():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = synth.fem_like("cantilever", integer=True)
    A = Matrix.from_synth(csr, device=0, h=4, w=4, T=4, C=128)
    xs = [torch.from_numpy(synth.make_x(csr.n, np.float32, "int2", s)).pin_memory() for s in range(4)]
    ys = [torch.empty(csr.m, dtype=torch.float32).pin_memory() for _ in range(4)]
    for k in range(4):
        A.spmv_host_async(xs[k].numpy(), ys[k].numpy())
    A.host_sync()
    for k in range(4):
        ye, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, xs[k].numpy())
        assert np.array_equal(ys[k].numpy().astype(np.float64), ye)
    A.free()


SANITIZE = r"""
import numpy as np, torch, sys
sys.path.insert(0, %r)
import synth
from paper_conf_ppopp_yanlzz14_b200 import Matrix
csr = synth.webbase_like(m=20000)
x = torch.from_numpy(synth.make_x(csr.n, np.float32, "unit", 0)).cuda()
PLAIN = (dict(T=4, C=64), dict(T=16, C=256, S=3, empty_mode=2), dict(T=8, C=128, col_mode=3),
         dict(T=4, C=64, tpc=2), dict(T=16, C=128, rc=2), dict(T=8, C=64, rc=2, tpc=2))
for p in PLAIN + (() if "--plain-only" in sys.argv else (dict(B=1024, R=4096, W=512), dict(B=1024, R=4096, W=512, S=2))):
    A = Matrix.from_synth(csr, device=0, **p)
    A.spmv(x); torch.cuda.synchronize(); A.free()
c = synth.fem_like("cantilever")
A = Matrix.from_synth(c, device=0, h=4, w=4, T=4, C=128)
A.spmv(torch.from_numpy(synth.make_x(c.n, np.float32, "uniform", 0)).cuda()); torch.cuda.synchronize()
print("SANITIZE-DONE")
""" % ROOT


@pytest.mark.parametrize("tool", ["memcheck", "synccheck", "initcheck", "racecheck"])
def test_compute_sanitizer(tool, tmp_path):
    """memcheck / synccheck / initcheck over the plain kernels (incl. tiles_per_cta = 2 and
    the strategy-2 result cache) and the panel-sliced band kernel; racecheck over the plain
    kernels (the band kernel's look-back flags are volatile shared-memory polls, which
    racecheck cannot order)."""
    exe = "/usr/local/cuda/bin/compute-sanitizer"
    if not os.path.exists(exe):
        pytest.skip("compute-sanitizer not available")
    script = tmp_path / "san.py"
    script.write_text(SANITIZE)
    extra = ["--plain-only"] if tool == "racecheck" else []
    args = [exe, "--tool", tool, "--error-exitcode", "9", "--kernel-name", "kns=yaspmv"]
    r = subprocess.run(args + [sys.executable, str(script)] + extra, capture_output=True, text=True, timeout=1800)
    if "closed on this pool" in r.stdout + r.stderr:  # the GPU pool's own wrapper refuses it
        pytest.skip("compute-sanitizer is closed on this GPU pool (its wrapper refuses to run)")
    assert "SANITIZE-DONE" in r.stdout, r.stdout[-2000:] + r.stderr[-2000:]
    assert r.returncode == 0, r.stdout[-3000:]
    assert ("RACECHECK SUMMARY: 0 hazards" if tool == "racecheck" else "ERROR SUMMARY: 0 errors") in r.stdout, \
        r.stdout[-3000:]


@pytest.mark.parametrize("S", [1, 3])
def test_fused_power_step(S):
    """yaspmv_spmv_power: y = (A x)/sqrt(in), out = sum y^2 (fused epilogue / combine)."""
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = synth.webbase_like(m=300_000, integer=True)
    A = Matrix.from_synth(csr, device=0, T=16, C=128, S=S)
    xn = synth.make_x(csr.n, np.float32, "int2", 1)
    x = torch.from_numpy(xn).cuda()
    y = torch.empty(csr.m, dtype=torch.float32, device="cuda")
    out = torch.zeros(1, dtype=torch.float64, device="cuda")
    inn = torch.tensor([4.0], dtype=torch.float64, device="cuda")      # scale by 1/2: exact
    ye, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, xn)
    A.spmv_power(x, y, None, out)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().astype(np.float64), ye)
    assert out.item() == float(np.sum(ye ** 2))                         # integers: exact
    A.spmv_power(x, y, inn, out)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().astype(np.float64), ye / 2)
    assert out.item() == float(np.sum((ye / 2) ** 2))
    # deterministic run to run
    vals = set()
    for _ in range(3):
        A.spmv_power(x, y, inn, out)
        torch.cuda.synchronize()
        vals.add(out.item())
    assert len(vals) == 1
    A.free()


def test_power_iteration_gpu_matches_fp64():
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, dist as D
    from synth import matrices as sm
    n = 1 << 16
    a = sm.circuit_like_rows(0, n, n=n, n_net=2, net_log2=(10, 12), band=4096)
    A = Matrix.from_synth(a, device=0, T=16, C=128)
    L = D.Layout(0, 1, np.array([0, n], dtype=np.int64), n)
    pit = D.PowerIteration(L, D.GpuOps(A, n, torch.device("cuda")), torch.float32, torch.device("cuda"))
    x = np.full(n, 1.0 / np.sqrt(n))
    for _ in range(6):
        pit.step()
        y, _ = ref.spmv(a.row_ptr, a.col, a.val.astype(np.float64), x, with_bound=False)
        x = y / np.linalg.norm(y)
    torch.cuda.synchronize()
    assert np.allclose(pit.current_x().cpu().numpy(), x, rtol=1e-4, atol=1e-7)
    A.free()


def test_ablation_variants_match():
    """The Fig. 14 ablation steps (tools/ablation.py) compute the same y."""
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, _lib
    from paper_conf_ppopp_yanlzz14_b200._lib import check, lib
    csr = synth.webbase_like(m=200_000, integer=True)
    xn = synth.make_x(csr.n, np.float32, "int2", 2)
    ye, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, xn)
    x = torch.from_numpy(xn).cuda()
    st = torch.cuda.current_stream().cuda_stream
    outs = []
    # COO + tree
    y = torch.zeros(csr.m, dtype=torch.float32, device="cuda")
    rows = torch.from_numpy(np.repeat(np.arange(csr.m, dtype=np.int32), np.diff(csr.row_ptr))).cuda()
    col = torch.from_numpy(csr.col).cuda(); val = torch.from_numpy(csr.val).cuda()
    sb = int(lib.yaspmv_ablation_tree_scratch_bytes(csr.nnz)); scr = torch.empty(sb, dtype=torch.uint8, device="cuda")
    check(lib.yaspmv_ablation_tree(rows.data_ptr(), None, None, col.data_ptr(), val.data_ptr(), csr.nnz,
                                   x.data_ptr(), y.data_ptr(), csr.m, _lib.F32, scr.data_ptr(), sb, st))
    outs.append(y.cpu().numpy())
    # BCCOO + tree
    A = Matrix.from_synth(csr, device=0, T=4, C=256, col_mode=2, flags=1)
    fl = torch.from_numpy(A.export("flags")).cuda(); cb = torch.from_numpy(A.export("col")).cuda()
    vb = torch.from_numpy(A.export("val0")).cuda(); cs = torch.from_numpy(A.export("cta_seg0")).cuda()
    nb = A.info()["nnzb_pad"]
    sb = int(lib.yaspmv_ablation_tree_scratch_bytes(nb)); scr = torch.empty(sb, dtype=torch.uint8, device="cuda")
    y = torch.zeros(csr.m, dtype=torch.float32, device="cuda")
    check(lib.yaspmv_ablation_tree(None, fl.data_ptr(), cs.data_ptr(), cb.data_ptr(), vb.data_ptr(), nb,
                                   x.data_ptr(), y.data_ptr(), csr.m, _lib.F32, scr.data_ptr(), sb, st))
    outs.append(y.cpu().numpy())
    A.free()
    for T, C in ((16, 128), (4, 64)):
        A = Matrix.from_synth(csr, device=0, T=T, C=C, col_mode=2)
        for v in (1, 2, 3):
            y = torch.zeros(csr.m, dtype=torch.float32, device="cuda")
            check(lib.yaspmv_ablation_spmv(A._h, v, x.data_ptr(), y.data_ptr(), st))
            outs.append(y.cpu().numpy())
        A.free()
    torch.cuda.synchronize()
    for o in outs:
        assert np.array_equal(o.astype(np.float64), ye)


SPIN = r"""
import ctypes, numpy as np, torch, sys
sys.path.insert(0, %r)
from paper_conf_ppopp_yanlzz14_b200 import Matrix
from paper_conf_ppopp_yanlzz14_b200._lib import lib
# row 0 holds 600 blocks (tiles of 4 x 64 = 256 blocks: it ends in tile 2), then short rows
m, n = 2000, 4096
lens = np.ones(m, dtype=np.int64); lens[0] = 600
rp = np.zeros(m + 1, dtype=np.int64); np.cumsum(lens, out=rp[1:])
col = np.concatenate([np.arange(600), np.arange(1, m) %% n]).astype(np.int32)
A = Matrix.from_csr(m, n, rp, col, np.ones(rp[-1], np.float32), device=0, T=4, C=64, col_mode=2)
x = torch.ones(n, device="cuda"); y = torch.empty(m, device="cuda")
st = lib.yaspmv_ablation_spmv(A._h, 12, x.data_ptr(), y.data_ptr(), torch.cuda.current_stream().cuda_stream)
try:
    torch.cuda.synchronize()
    print("NO-TRAP")
except Exception as e:
    print("TRAPPED", type(e).__name__)
print("SPIN-TILE", int(lib.yaspmv_debug_spin_tile()))
""" % ROOT


def test_debug_spin_bound_traps_with_tile_id(tmp_path):
    """with YASPMV_SPIN_LIMIT set, a look-back whose predecessor never publishes
    (ablation variant 12: tile 0 skips its publish) traps instead of hanging the GPU, and the
    waiting tile's id is readable afterwards (tile 2: the stop of the 600-block row)."""
    script = tmp_path / "spin.py"
    script.write_text(SPIN)
    env = dict(os.environ, YASPMV_SPIN_LIMIT="20000")
    r = subprocess.run([sys.executable, str(script)], capture_output=True, text=True, timeout=300, env=env)
    assert "TRAPPED" in r.stdout, r.stdout + r.stderr[-2000:]
    assert "SPIN-TILE 2" in r.stdout, r.stdout


def test_l2_persist_set_aside():
    """yaspmv_l2_persist: the set-aside is applied (clamped to the device maximum), SpMV
    results are bitwise unchanged by it (only cache residency changes), and 0 restores it."""
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, l2_persist
    csr = synth.webbase_like(m=50000)
    x = torch.from_numpy(synth.make_x(csr.n, np.float32, "uniform", 1)).cuda()
    A = Matrix.from_synth(csr, device=0, T=8, C=128, S=2)
    y0 = A.spmv(x).cpu().numpy()
    got = l2_persist(0, 60 << 20)
    assert got > 0
    y1 = A.spmv(x).cpu().numpy()
    assert np.array_equal(y0.view(np.uint32), y1.view(np.uint32))
    assert l2_persist(0, 0) == 0
    A.free()
