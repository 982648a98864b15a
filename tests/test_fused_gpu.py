"""The fused multi-rank power step (yaspmv_power_step_fused) on the
one GPU of this run.

Each rank's SpMV stores its rows of z_k straight into every rank's copy of the next x (peer
stores), and the one-warp publish/wait kernels replace the all-reduce + all-gather.  Here P
ranks run as P handles of ONE process on cuda:0, each on its own stream, their comms
connected with ``Comm.connect_local`` (the peers' "remote" buffers are other allocations of
the same device — the same stores, flags and fences as over NVLink), and as 2 processes
mapping each other through CUDA IPC.

Bars: bitwise equality with the unfused protocol (yaspmv_spmv_power per rank on the
gathered x, norms summed in rank order in fp64: the fused path must reproduce exactly that
arithmetic), and the first product against the fp64 oracle within the north-star tolerance.
"""
import os
import socket
import tempfile

import numpy as np
import pytest

import synth
from oracle import ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

KW = dict(n=1 << 16, n_net=3, net_log2=(11, 13), band=4096)


def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _rank_matrices(csr_full, P, params):
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, dist as D
    Ls, As = [], []
    for r in range(P):
        L = D.make_layout(csr_full.row_ptr, r, P)
        sub = csr_full.row_slice(L.r0, L.r1)
        col = D.remap_columns(sub.col, L.bounds, L.m_max)
        As.append(Matrix.from_csr(sub.m, L.n_padded, sub.row_ptr, col, sub.val, device=0, **params))
        Ls.append(L)
    return Ls, As


def _unfused_reference(Ls, As, tdt, iters):
    """yaspmv_spmv_power per rank on the gathered x; norms summed in rank order (fp64)."""
    L0 = Ls[0]
    P = L0.world
    dev = torch.device("cuda", 0)
    x = torch.zeros(L0.n_padded, dtype=tdt, device=dev)
    n_true = int(L0.bounds[-1])
    for r in range(P):
        x[r * L0.m_max: r * L0.m_max + Ls[r].m_local] = 1.0 / np.sqrt(n_true)
    tot = None
    norms = [torch.zeros(1, dtype=torch.float64, device=dev) for _ in range(P)]
    for _ in range(iters):
        xn = torch.zeros_like(x)
        for r in range(P):
            y = torch.empty(max(Ls[r].m_local, 1), dtype=tdt, device=dev)
            As[r].spmv_power(x, y[: Ls[r].m_local], tot, norms[r])
            xn[r * L0.m_max: r * L0.m_max + Ls[r].m_local] = y[: Ls[r].m_local]
        t = torch.zeros(1, dtype=torch.float64, device=dev)
        for r in range(P):
            t = t + norms[r]
        tot = t
        x = xn
    torch.cuda.synchronize()
    return x, tot


def _fused_local(Ls, As, tdt, iters):
    from paper_conf_ppopp_yanlzz14_b200 import Comm, dist as D
    P = Ls[0].world
    npdt = np.float32 if tdt == torch.float32 else np.float64
    comms = [Comm(0, r, P, Ls[0].m_max, npdt, timeout_ms=20000) for r in range(P)]
    for c in comms:
        c.connect_local(comms)
    pits = [D.FusedPowerIteration(Ls[r], As[r], tdt, "cuda:0", comm=comms[r]) for r in range(P)]
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream() for _ in range(P)]
    for _ in range(iters):
        for r in range(P):  # rank r's step only waits (on the device) for the peers' previous step
            pits[r].step(stream=streams[r])
    for r in range(P):
        comms[r].wait(stream=streams[r])
    torch.cuda.synchronize()
    for c in comms:
        c.check()
    out = [(c.x(0).clone(), c.norm2().clone()) for c in comms]
    return out, comms


BAND = dict(B=4096, R=4096, W=4096, S=2, T=16, C=128)  # panel-sliced BCCOO+ (DESIGN §2.1), far part S = 2


@pytest.mark.parametrize("P", [1, 2, 3])
@pytest.mark.parametrize("case", ["circuit-f32", "circuit-f32-S2", "laplace-f64", "circuit-band"])
def test_fused_step_bitwise_equals_unfused(P, case):
    _need_gpu()
    from synth import matrices as sm
    if case.startswith("circuit"):
        csr = sm.circuit_like_rows(0, KW["n"], **KW)
        tdt = torch.float32
        params = (dict(T=16, C=128, S=2) if case.endswith("S2") else BAND if case.endswith("band")
                  else dict(T=16, C=128))
    else:
        csr = synth.laplacian_2d(64)
        tdt = torch.float64
        params = dict(T=8, C=64)
    iters = 4
    Ls, As = _rank_matrices(csr, P, params)
    x_ref, tot_ref = _unfused_reference(Ls, As, tdt, iters)
    outs, comms = _fused_local(Ls, As, tdt, iters)
    for r, (x, tot) in enumerate(outs):
        assert torch.equal(x, x_ref), f"rank {r}: fused x differs from the unfused protocol"
        assert torch.equal(tot, tot_ref), f"rank {r}: ||z||^2 differs"
        assert comms[r].seq == iters
    for A in As:
        A.free()


def test_fused_first_step_matches_oracle():
    """z_1 = A x_0 assembled from 3 ranks' peer stores, against the fp64 oracle."""
    _need_gpu()
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import dist as D
    csr = sm.circuit_like_rows(0, KW["n"], **KW)
    Ls, As = _rank_matrices(csr, 3, dict(T=32, C=128))
    outs, _ = _fused_local(Ls, As, torch.float32, 1)
    z = D.unpad(outs[1][0].cpu().numpy(), Ls[0].bounds, Ls[0].m_max)
    x0 = np.full(csr.n, np.float32(1.0 / np.sqrt(csr.n)), dtype=np.float32)
    y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x0)
    ok, worst = ref.check_tolerance(z, y_ref, bound, np.float32)
    assert ok, worst
    n2 = float(outs[1][1].item())
    assert abs(n2 - float(np.sum(z.astype(np.float64) ** 2))) <= 1e-9 * n2


def test_fused_restart_and_rank_with_no_rows():
    """begin() restarts from x_0 (same result twice); a rank whose block is empty still
    publishes (its chunk stays zero) so the others never wait forever."""
    _need_gpu()
    from paper_conf_ppopp_yanlzz14_b200 import Comm, Matrix, dist as D
    csr = synth.laplacian_2d(16)  # 256 rows
    P = 2
    # force rank 1 empty: bounds [0, 256, 256]
    b = np.array([0, csr.m, csr.m], dtype=np.int64)
    m_max = csr.m
    Ls = [D.Layout(r, P, b, m_max) for r in range(P)]
    As = []
    for r in range(P):
        sub = csr.row_slice(int(b[r]), int(b[r + 1]))
        As.append(Matrix.from_csr(sub.m, P * m_max, sub.row_ptr, D.remap_columns(sub.col, b, m_max), sub.val,
                                  device=0, T=4, C=64))
    comms = [Comm(0, r, P, m_max, np.float64, timeout_ms=20000) for r in range(P)]
    for c in comms:
        c.connect_local(comms)
    pits = [D.FusedPowerIteration(Ls[r], As[r], torch.float64, "cuda:0", comm=comms[r]) for r in range(P)]
    res = []
    for _ in range(2):
        for _ in range(3):
            for r in range(P):
                pits[r].step()
        x = pits[0].current_x()
        torch.cuda.synchronize()
        res.append(x.clone())
        for p in pits:
            p.restart()
    assert torch.equal(res[0], res[1])
    xr = np.full(csr.n, 1.0 / np.sqrt(csr.n))
    for _ in range(3):
        y, _ = ref.spmv(csr.row_ptr, csr.col, csr.val, xr, with_bound=False)
        xr = y / np.linalg.norm(y)
    assert np.allclose(res[0].cpu().numpy()[: csr.m], xr, rtol=1e-12, atol=1e-14)
    for c in comms:
        c.check()


def test_fused_wait_times_out_instead_of_hanging():
    """A peer that never steps: the device wait gives up after the timeout, reports ECUDA."""
    _need_gpu()
    from paper_conf_ppopp_yanlzz14_b200 import Comm, Matrix, YaspmvError, dist as D
    csr = synth.laplacian_2d(8)
    P = 2
    b = D.nnz_balanced_bounds(csr.row_ptr, P)
    m_max = int(np.diff(b).max())
    sub = csr.row_slice(int(b[0]), int(b[1]))
    A0 = Matrix.from_csr(sub.m, P * m_max, sub.row_ptr, D.remap_columns(sub.col, b, m_max), sub.val, device=0,
                         T=4, C=64)
    comms = [Comm(0, r, P, m_max, np.float64, timeout_ms=300) for r in range(P)]
    for c in comms:
        c.connect_local(comms)
    comms[0].begin()
    A0.power_step_fused(comms[0])
    A0.power_step_fused(comms[0])  # waits for rank 1's step 0, which never comes
    torch.cuda.synchronize()
    with pytest.raises(YaspmvError):
        comms[0].check()
    comms[0].check()  # cleared


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, port, path, iters, per_rank_device=False, multicast=False):
    import torch.distributed as dist
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, dist as D
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    dev = rank if per_rank_device else 0
    torch.cuda.set_device(dev)
    csr = sm.circuit_like_rows(0, KW["n"], **KW)
    L = D.make_layout(csr.row_ptr, rank, world)
    sub = csr.row_slice(L.r0, L.r1)
    A = Matrix.from_csr(sub.m, L.n_padded, sub.row_ptr, D.remap_columns(sub.col, L.bounds, L.m_max), sub.val,
                        device=dev, T=16, C=128)
    pit = D.FusedPowerIteration(L, A, torch.float32, f"cuda:{dev}", timeout_ms=60000,  # IPC handle exchange
                                multicast=multicast)
    assert pit.multicast == bool(multicast)
    for _ in range(iters):
        pit.step()
    pit.comm.wait()
    torch.cuda.synchronize()
    pit.comm.check()
    np.save(path + f".{rank}.npy", pit.z().cpu().numpy())
    np.save(path + f".{rank}.n2.npy", pit.comm.norm2().cpu().numpy())
    dist.barrier()  # no rank unmaps while a peer may still store into it
    A.free()
    pit.comm.free()
    dist.destroy_process_group()


@pytest.mark.parametrize("two_devices", [False, True])
def test_fused_two_processes_ipc(two_devices):
    """Two processes mapping each other's comm through CUDA IPC; the result equals the
    single-process unfused protocol bitwise.  two_devices = False: both map cuda:0 (always
    runs); True: rank r on cuda:r, so the peer stores, the system-scope fences and the
    acquire/release flags cross NVLink (runs only where two GPUs are visible)."""
    _need_gpu()
    if two_devices and torch.cuda.device_count() < 2:
        pytest.skip("needs two visible GPUs")
    import torch.multiprocessing as mp
    from synth import matrices as sm
    iters = 3
    with tempfile.TemporaryDirectory() as td:
        path = os.path.join(td, "z")
        mp.spawn(_ipc_worker, args=(2, _free_port(), path, iters, two_devices), nprocs=2, join=True)
        zs = [np.load(path + f".{r}.npy") for r in range(2)]
        n2 = [np.load(path + f".{r}.n2.npy") for r in range(2)]
    csr = sm.circuit_like_rows(0, KW["n"], **KW)
    Ls, As = _rank_matrices(csr, 2, dict(T=16, C=128))
    x_ref, tot_ref = _unfused_reference(Ls, As, torch.float32, iters)
    for r in range(2):
        assert np.array_equal(zs[r], x_ref.cpu().numpy())
        assert np.array_equal(n2[r], tot_ref.cpu().numpy())


def _mc_supported():
    from paper_conf_ppopp_yanlzz14_b200 import Comm
    return Comm.mc_supported(0)


@pytest.mark.parametrize("case", ["circuit-f32", "circuit-f32-S2", "laplace-f64", "circuit-band"])
def test_fused_multicast_one_rank(case):
    """NVSwitch multicast exchange (yaspmv_comm_mc_*): the multicast object of one device,
    the x buffers bound to it, every z row stored once through the multicast mapping by the
    SpMV epilogue (S = 1) or the BCCOO+ combine (S = 2) — bitwise equal to the unfused
    protocol.  The object, the binding and the multimem.st path are the ones a multi-GPU
    node uses (there the switch replicates each store into every rank's buffer)."""
    _need_gpu()
    if not _mc_supported():
        pytest.skip("the device reports no switch multicast")
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import dist as D
    if case.startswith("circuit"):
        csr = sm.circuit_like_rows(0, KW["n"], **KW)
        tdt = torch.float32
        params = (dict(T=16, C=128, S=2) if case.endswith("S2") else BAND if case.endswith("band")
                  else dict(T=16, C=128))
    else:
        csr = synth.laplacian_2d(64)
        tdt = torch.float64
        params = dict(T=8, C=64)
    iters = 4
    Ls, As = _rank_matrices(csr, 1, params)
    x_ref, tot_ref = _unfused_reference(Ls, As, tdt, iters)
    try:
        pit = D.FusedPowerIteration(Ls[0], As[0], tdt, "cuda:0", timeout_ms=20000, multicast=True)
    except RuntimeError as e:  # e.g. a container without the switch's fabric channels
        if "create the multicast object" in str(e):
            pytest.skip(f"the driver refuses multicast objects here: {e}")
        raise
    assert pit.multicast and pit.comm.mc_active
    for _ in range(iters):
        pit.step()
    pit.comm.wait()
    torch.cuda.synchronize()
    pit.comm.check()
    assert torch.equal(pit.comm.x(0), x_ref)
    assert torch.equal(pit.comm.norm2(), tot_ref)
    pit.comm.free()
    for A in As:
        A.free()


def test_fused_two_processes_multicast():
    """Two processes on two GPUs, the multicast object created by rank 0 and imported by
    rank 1 through pidfd_getfd: every z row crosses the switch once.  Runs only where two
    GPUs with switch multicast are visible."""
    _need_gpu()
    if torch.cuda.device_count() < 2 or not _mc_supported():
        pytest.skip("needs two visible GPUs with switch multicast")
    import torch.multiprocessing as mp
    from synth import matrices as sm
    iters = 3
    with tempfile.TemporaryDirectory() as td:
        path = os.path.join(td, "z")
        mp.spawn(_ipc_worker, args=(2, _free_port(), path, iters, True, True), nprocs=2, join=True)
        zs = [np.load(path + f".{r}.npy") for r in range(2)]
        n2 = [np.load(path + f".{r}.n2.npy") for r in range(2)]
    csr = sm.circuit_like_rows(0, KW["n"], **KW)
    Ls, As = _rank_matrices(csr, 2, dict(T=16, C=128))
    x_ref, tot_ref = _unfused_reference(Ls, As, torch.float32, iters)
    for r in range(2):
        assert np.array_equal(zs[r], x_ref.cpu().numpy())
        assert np.array_equal(n2[r], tot_ref.cpu().numpy())
