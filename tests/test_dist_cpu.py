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


# ---------------------------------------------------------------- fused exchange (host side)
class _ShmComm:
    """CPU model of yaspmv_comm for the host logic of dist.FusedPowerIteration on gloo:
    the "device allocation" is a shared file ([x0 | x1 | flags | norms[2][P]], fp64 here),
    the "IPC handle" its path; the protocol (parity, epochs, rank-order norm sum) mirrors
    csrc/comm.cu."""

    def __init__(self, device, rank, world, chunk, dtype, timeout_ms, root=None):
        self.rank, self.world, self.chunk = rank, world, chunk
        self.n = world * chunk
        self.path = os.path.join(root or os.environ["SHM_ROOT"], f"comm{rank}")
        self.size = 2 * self.n + 3 * world
        self.buf = torch.from_file(self.path, shared=True, size=self.size, dtype=torch.float64)
        self.buf.zero_()
        self.peers = None
        self.seq, self.fresh = 0, True
        self.total = torch.zeros(1, dtype=torch.float64)

    def _x(self, b, k):
        return b[(k % 2) * self.n: (k % 2 + 1) * self.n]

    def _flags(self, b):
        return b[2 * self.n: 2 * self.n + self.world]

    def _norms(self, b, parity):
        o = 2 * self.n + self.world + parity * self.world
        return b[o: o + self.world]

    def ipc_handle(self):
        return self.path.encode()

    def open_ipc(self, handles):
        assert len(handles) == self.world and handles[self.rank] == self.path.encode()
        self.peers = [torch.from_file(h.decode(), shared=True, size=self.size, dtype=torch.float64)
                      for h in handles]

    def x(self, which=0):
        return self._x(self.buf, self.seq + which)

    def norm2(self):
        return self.total

    def begin(self):
        self.fresh = True

    def wait(self, stream=None):
        import time
        t0 = time.time()
        while float(self._flags(self.buf).min()) < self.seq:
            assert time.time() - t0 < 60, "peer never published"
            time.sleep(0.001)
        self.total[0] = float(sum(float(v) for v in self._norms(self.buf, (self.seq - 1) % 2)))

    def check(self):
        pass


class _ShmFusedMatrix:
    """The rank's rows on the CPU (oracle product) behind the fused-step interface."""

    def __init__(self, csr, m_local):
        self.csr, self.m = csr, m_local

    def power_step_fused(self, c, stream=None):
        if not c.fresh:
            c.wait()
        x = c._x(c.buf, c.seq).numpy()
        z, _ = ref.spmv(self.csr.row_ptr, self.csr.col, self.csr.val, x, with_bound=False)
        if not c.fresh:
            z = z / np.sqrt(float(c.total[0]))
        n2 = float(np.sum(z ** 2))
        for p in c.peers:  # peer stores, then norm + flag (the publish kernel)
            c._x(p, c.seq + 1)[c.rank * c.chunk: c.rank * c.chunk + self.m] = torch.from_numpy(z)
            c._norms(p, c.seq % 2)[c.rank] = n2
            c._flags(p)[c.rank] = c.seq + 1
        c.seq += 1
        c.fresh = False

    def launches_per_fused_step(self):
        return 0


def _fused_worker(rank, world, port, root, n, iters, restart_after=0):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ["SHM_ROOT"] = root
    dist.init_process_group("gloo", rank=rank, world_size=world)
    kw = dict(n=n, n_net=2, net_log2=(8, 10), band=512)
    from synth import matrices as sm
    full = sm.circuit_like_rows(0, n, **kw)
    L = D.make_layout(full.row_ptr, rank, world)
    sub = full.row_slice(L.r0, L.r1)
    sub.col = D.remap_columns(sub.col, L.bounds, L.m_max)
    sub.val = sub.val.astype(np.float64)
    pit = D.FusedPowerIteration(L, _ShmFusedMatrix(sub, L.m_local), torch.float64, "cpu",
                                comm_factory=_ShmComm)
    if restart_after:  # a few steps, then restart: the peers' last stores must land first
        for _ in range(restart_after):
            pit.step()
        pit.restart()
    for _ in range(iters):
        pit.step()
    x = pit.current_x()
    np.save(os.path.join(root, f"x{rank}.npy"), D.unpad(x.numpy(), L.bounds, L.m_max))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("restart_after", [0, 3])
def test_fused_power_iteration_host_protocol_world2(restart_after):
    """dist.FusedPowerIteration over gloo world 2: IPC-handle exchange in rank order, x_0
    layout, restart barrier, and the parity/epoch protocol of comm.cu (modelled on shared
    files) give every rank the single-process power iteration — also after a restart in the
    middle (the restart waits for every peer's last step before re-initialising x_0)."""
    import torch.multiprocessing as mp
    n, iters, world = 1 << 12, 4, 2
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_fused_worker, args=(world, _free_port(), td, n, iters, restart_after), nprocs=world, join=True)
        xs = [np.load(os.path.join(td, f"x{r}.npy")) for r in range(world)]
    from synth import matrices as sm
    a = sm.circuit_like_rows(0, n, n=n, n_net=2, net_log2=(8, 10), band=512)
    x = np.full(n, 1.0 / np.sqrt(n))
    for _ in range(iters):
        y, _ = ref.spmv(a.row_ptr, a.col, a.val.astype(np.float64), x, with_bound=False)
        x = y / np.linalg.norm(y)
    for xr in xs:
        assert np.allclose(xr, x, rtol=1e-12, atol=1e-15)


class _FailingOpenComm(_ShmComm):
    """Rank 1 cannot map its peers (e.g. no P2P between the GPUs)."""

    def open_ipc(self, handles):
        if self.rank == 1:
            raise OSError("peer mapping refused")
        super().open_ipc(handles)


class _FailingHandleComm(_ShmComm):
    """Rank 1 cannot export an IPC handle for its buffer."""

    def ipc_handle(self):
        if self.rank == 1:
            raise OSError("cudaIpcGetMemHandle failed")
        return super().ipc_handle()


def _fused_fail_worker(rank, world, port, root, fail_create, fail_handle=False):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ["SHM_ROOT"] = root
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n = 1 << 10
    from synth import matrices as sm
    full = sm.circuit_like_rows(0, n, n=n, n_net=1, net_log2=(6, 7), band=64)
    L = D.make_layout(full.row_ptr, rank, world)

    def factory(*a):
        if fail_create and rank == 0:
            raise MemoryError("no device memory for the exchange buffers")
        return _FailingHandleComm(*a) if fail_handle else _FailingOpenComm(*a)

    try:
        D.FusedPowerIteration(L, None, torch.float64, "cpu", comm_factory=factory)
        outcome = "ok"
    except RuntimeError as e:
        outcome = str(e)
    with open(os.path.join(root, f"r{rank}.txt"), "w") as f:
        f.write(outcome)
    dist.barrier()          # every rank got here: nobody is left waiting for a peer
    dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["create", "open", "handle"])
def test_fused_setup_failure_is_agreed_by_every_rank(mode):
    """If one rank cannot create, export or map the exchange buffers, every rank raises (so
    bench.py falls back to the NCCL protocol everywhere) instead of the others blocking in a
    collective or a barrier."""
    import torch.multiprocessing as mp
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_fused_fail_worker, args=(2, _free_port(), td, mode == "create", mode == "handle"), nprocs=2,
                 join=True)
        outs = [open(os.path.join(td, f"r{r}.txt")).read() for r in range(2)]
    want = {"create": "create the exchange buffers on rank(s) [0]", "open": "map the peers' buffers on rank(s) [1]",
            "handle": "export the IPC handles on rank(s) [1]"}[mode]
    assert all(want in o for o in outs), outs


# ---------------------------------------------------------------- multicast setup (host side)
class _McShmComm(_ShmComm):
    """The multicast setup calls of yaspmv_comm_mc_* on the shared-file comm: each call is
    logged; ``fail`` names a stage that raises on rank 1.  A bound comm keeps the peer-store
    protocol of _ShmComm underneath (the exchange itself is modelled by the parent)."""

    fail = None

    def __init__(self, *a, **kw):
        super().__init__(*a, **kw)
        self.log, self.mc_active = [], False

    def _maybe_fail(self, stage):
        self.log.append(stage)
        if self.rank == 1 and self.fail == stage:
            raise OSError(f"{stage} refused on rank 1")

    def mc_supported(self, device):
        self._maybe_fail("probe")
        return True

    def mc_create(self):
        assert self.rank == 0
        self._maybe_fail("create")
        return 17

    def mc_import(self, pid, fd):
        assert fd == 17 and pid > 0 and pid != os.getpid()  # the creator's descriptor
        self._maybe_fail("import")

    def mc_add_device(self):
        self._maybe_fail("add")

    def mc_bind(self):
        self._maybe_fail("bind")
        self.mc_active = True

    def mc_release(self):
        self.log.append("release")
        self.mc_active = False


def _mc_worker(rank, world, port, root, fail, multicast):
    import json
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    os.environ["SHM_ROOT"] = root
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n = 1 << 10
    from synth import matrices as sm
    full = sm.circuit_like_rows(0, n, n=n, n_net=1, net_log2=(6, 7), band=64)
    L = D.make_layout(full.row_ptr, rank, world)

    class F(_McShmComm):
        pass
    F.fail = fail
    out = {}
    try:
        pit = D.FusedPowerIteration(L, None, torch.float64, "cpu", comm_factory=F, multicast=multicast)
        out = {"ok": True, "multicast": pit.multicast, "log": pit.comm.log}
    except RuntimeError as e:
        out = {"ok": False, "err": str(e)}
    with open(os.path.join(root, f"mc{rank}.json"), "w") as f:
        json.dump(out, f)
    dist.barrier()  # every rank got here: no rank waits on a peer's setup
    dist.destroy_process_group()


@pytest.mark.parametrize("fail,multicast", [(None, True), ("bind", "auto"), ("import", "auto"),
                                            ("probe", "auto"), ("add", True)])
def test_multicast_setup_is_agreed_by_every_rank(fail, multicast):
    """dist.FusedPowerIteration(multicast=...) over gloo world 2: rank 0 creates the object,
    rank 1 imports rank 0's (pid, fd), both add their device, then bind — every stage agreed
    on, so a failure anywhere leaves EVERY rank on peer stores (multicast="auto": a rank whose
    own bind succeeded releases it) or makes every rank raise (multicast=True); no rank hangs."""
    import json
    import torch.multiprocessing as mp
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_mc_worker, args=(2, _free_port(), td, fail, multicast), nprocs=2, join=True)
        res = [json.load(open(os.path.join(td, f"mc{r}.json"))) for r in range(2)]
    if fail is None:
        assert all(r["ok"] and r["multicast"] for r in res)
        assert res[0]["log"] == ["probe", "create", "add", "bind"]
        assert res[1]["log"] == ["probe", "import", "add", "bind"]
    elif multicast is True:
        assert all(not r["ok"] and "rank(s) [1]" in r["err"] for r in res)
    else:
        assert all(r["ok"] and not r["multicast"] for r in res)
        if fail == "bind":  # rank 0 had bound: it went back to peer stores
            assert res[0]["log"][-1] == "release"
