"""The multi-rank power iteration with the real CUDA kernels: 2 ranks sharing the one GPU of
this run, exchanging over gloo (NCCL refuses two ranks on one device).  Checks the whole
N > 1 path of dist.py on hardware — nnz-balanced row blocks, remapped columns, the fused
SpMV step per rank, the scalar all-reduce and the padded all-gather — against the fp64
oracle power iteration.  (Performance across GPUs is bench.py's business.)"""
import os
import socket
import tempfile

import numpy as np
import pytest

import synth  # noqa: F401
from oracle import ref

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
KW = dict(n=1 << 17, n_net=3, net_log2=(12, 14), band=8192)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, path, iters):
    import torch.distributed as dist
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, dist as D
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n = KW["n"]
    counts = np.diff(sm.circuit_like_rows(0, n, **KW).row_ptr)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    L = D.make_layout(rp, rank, world)
    csr = sm.circuit_like_rows(L.r0, L.r1, **KW)
    csr.col = D.remap_columns(csr.col, L.bounds, L.m_max)
    A = Matrix.from_csr(csr.m, L.n_padded, csr.row_ptr, csr.col, csr.val, device=0, T=16, C=128)
    dev = torch.device("cuda", 0)
    pit = D.PowerIteration(L, D.GpuOps(A, L.m_local, dev), torch.float32, dev)
    for _ in range(iters):
        pit.step()
        torch.cuda.synchronize()
    if rank == 0:
        np.save(path, D.unpad(pit.current_x().cpu().numpy(), L.bounds, L.m_max))
    A.free()
    dist.destroy_process_group()


def test_power_iteration_two_ranks_one_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    iters = 5
    with tempfile.TemporaryDirectory() as td:
        path = os.path.join(td, "x.npy")
        mp.spawn(_worker, args=(2, _free_port(), path, iters), nprocs=2, join=True)
        x_dist = np.load(path)
    from synth import matrices as sm
    a = sm.circuit_like_rows(0, KW["n"], **KW)
    x = np.full(KW["n"], 1.0 / np.sqrt(KW["n"]))
    for _ in range(iters):
        y, _ = ref.spmv(a.row_ptr, a.col, a.val.astype(np.float64), x, with_bound=False)
        x = y / np.linalg.norm(y)
    assert np.allclose(x_dist, x, rtol=1e-4, atol=1e-7)
