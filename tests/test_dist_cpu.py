"""Multi-GPU exchange logic on CPU: nnz-balanced row partition, column remap into the
padded all-gather space, and the power-iteration loop over a world-size-2 gloo process
group (the local products run in the oracle here — only the exchange is under test; on
GPUs the same loop runs the CUDA kernels, tests/test_dist_gpu.py / bench.py)."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch

import synth
from oracle import ref
from paper_conf_ppopp_yanlzz14_b200 import dist as D


def test_partition_balanced_and_aligned():
    a = synth.webbase_like(m=50_000)
    for P in (1, 2, 3, 4, 8):
        for h in (1, 2, 4):
            b = D.nnz_balanced_bounds(a.row_ptr, P, h)
            assert b[0] == 0 and b[-1] == a.m and np.all(np.diff(b) >= 0)
            assert np.all(b[1:-1] % h == 0)
            part = a.row_ptr[b[1:]] - a.row_ptr[b[:-1]]
            maxrow = int(np.diff(a.row_ptr).max())
            assert part.max() - a.nnz / P <= h * maxrow + 1   # balanced up to one block row


def test_remap_is_a_bijection_into_padded_space():
    rp = np.arange(0, 1001, dtype=np.int64) * 3
    b = D.nnz_balanced_bounds(rp, 3)
    m_max = int(np.diff(b).max())
    cols = np.arange(1000)
    r = D.remap_columns(cols, b, m_max)
    assert len(set(r.tolist())) == 1000 and r.max() < 3 * m_max
    x = np.arange(1000, dtype=np.float64)
    xp = np.zeros(3 * m_max)
    xp[r] = x
    assert np.array_equal(D.unpad(xp, b, m_max), x)


class _CpuOps:
    """Local steps on the CPU for the exchange test (oracle product, fp64 norm); the
    unfused protocol (spmv / nrm2sq / scale)."""

    def __init__(self, csr):
        self.csr = csr

    def spmv(self, x, y):
        yy, _ = ref.spmv(self.csr.row_ptr, self.csr.col, self.csr.val, x.numpy(), with_bound=False)
        y.copy_(torch.from_numpy(yy.astype(np.float32)))

    def nrm2sq(self, y, out):
        out[0] = float(np.sum(y.numpy().astype(np.float64) ** 2))

    def scale(self, src, dst, norm2):
        dst.copy_(src / float(np.sqrt(norm2[0].item())))


def _worker(rank, world, port, path, n, iters, fused=False):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    kw = dict(n=n, n_net=2, net_log2=(8, 10), band=512)
    from synth import matrices as sm
    full_counts = np.diff(sm.circuit_like_rows(0, n, **kw).row_ptr)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(full_counts, out=rp[1:])
    L = D.make_layout(rp, rank, world)
    csr = sm.circuit_like_rows(L.r0, L.r1, **kw)        # only this rank's rows
    csr.col = D.remap_columns(csr.col, L.bounds, L.m_max)
    ops = _CpuFusedOps(csr) if fused else _CpuOps(csr)
    pit = D.PowerIteration(L, ops, torch.float32, torch.device("cpu"))
    for _ in range(iters):
        pit.step()
    if rank == 0:
        np.save(path, D.unpad(pit.current_x().numpy(), L.bounds, L.m_max))
    dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class _CpuFusedOps:
    """The fused protocol (power_step: z = (A v)/sqrt(in_norm2), out_norm2 = ||z||^2)."""

    def __init__(self, csr):
        self.csr = csr

    def power_step(self, v, z, in_norm2, out_norm2):
        yy, _ = ref.spmv(self.csr.row_ptr, self.csr.col, self.csr.val, v.numpy(), with_bound=False)
        if in_norm2 is not None:
            yy = yy / np.sqrt(in_norm2[0].item())
        z.copy_(torch.from_numpy(yy.astype(np.float32)))
        out_norm2[0] = float(np.sum(z.numpy().astype(np.float64) ** 2))


@pytest.mark.parametrize("world,fused", [(2, False), (2, True), (1, True)])
def test_power_iteration_world2_matches_single_process(world, fused):
    import torch.multiprocessing as mp
    n, iters = 1 << 13, 4
    with tempfile.TemporaryDirectory() as td:
        path = os.path.join(td, "x.npy")
        mp.spawn(_worker, args=(world, _free_port(), path, n, iters, fused), nprocs=world, join=True)
        x_dist = np.load(path)
    # single-process fp64 power iteration on the same matrix
    from synth import matrices as sm
    a = sm.circuit_like_rows(0, n, n=n, n_net=2, net_log2=(8, 10), band=512)
    x = np.full(n, 1.0 / np.sqrt(n))
    for _ in range(iters):
        y, _ = ref.spmv(a.row_ptr, a.col, a.val.astype(np.float64), x, with_bound=False)
        x = y / np.linalg.norm(y)
    assert np.allclose(x_dist, x, rtol=1e-4, atol=1e-6)
