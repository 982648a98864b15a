"""Multi-GPU iterated SpMV (power iteration) — one process per GPU, torch.distributed/NCCL.

Not in the paper (single GPU); BASELINE.json north_star asks for it:
  * rows are partitioned nnz-balanced into contiguous blocks, one per rank
    (``nnz_balanced_bounds``); each rank encodes only its own row block (all N columns);
  * x is replicated: every iteration all-gathers the ranks' y blocks into x over
    NVLink/NVSwitch (NCCL ``all_gather_into_tensor``).  To use NCCL's equal-size path,
    each rank's chunk is padded to m_max rows and column indices are remapped at build
    time into that padded space (``remap_columns``); pad entries of x are never read;
  * the normalisation needs one scalar all-reduce (sum of ||y_r||^2).

The exchange logic is independent of where the local product runs: ``PowerIteration``
takes an ``ops`` object (GPU kernels in the product; the CPU tests inject others to
exercise the gloo path on world_size 2).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


def nnz_balanced_bounds(row_ptr: np.ndarray, P: int, h: int = 1) -> np.ndarray:
    """b_r = lower_bound(row_ptr, r*nnz/P), rounded down to a multiple of h (block rows
    never straddle ranks); b_0 = 0, b_P = m.  Ties go to the lower row."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    m = row_ptr.size - 1
    nnz = int(row_ptr[-1])
    b = np.zeros(P + 1, dtype=np.int64)
    for r in range(1, P):
        target = (r * nnz) // P
        i = int(np.searchsorted(row_ptr, target, side="left"))
        i = min(max(i, 0), m)
        b[r] = (i // h) * h
    b[P] = m
    b = np.maximum.accumulate(b)
    return b


def remap_columns(col: np.ndarray, bounds: np.ndarray, m_max: int) -> np.ndarray:
    """Column j (owned by rank r = the block with bounds[r] <= j < bounds[r+1]) moves to
    r*m_max + (j - bounds[r]) in the padded, all-gathered x."""
    col = np.asarray(col, dtype=np.int64)
    r = np.searchsorted(bounds, col, side="right") - 1
    return (r * m_max + (col - bounds[r])).astype(np.int32)


def unpad(x_padded: np.ndarray, bounds: np.ndarray, m_max: int) -> np.ndarray:
    P = bounds.size - 1
    return np.concatenate([x_padded[r * m_max: r * m_max + (bounds[r + 1] - bounds[r])] for r in range(P)])


@dataclass
class Layout:
    rank: int
    world: int
    bounds: np.ndarray
    m_max: int

    @property
    def r0(self) -> int:
        return int(self.bounds[self.rank])

    @property
    def r1(self) -> int:
        return int(self.bounds[self.rank + 1])

    @property
    def m_local(self) -> int:
        return self.r1 - self.r0

    @property
    def n_padded(self) -> int:
        return self.world * self.m_max


def make_layout(row_ptr: np.ndarray, rank: int, world: int, h: int = 1) -> Layout:
    b = nnz_balanced_bounds(row_ptr, world, h)
    m_max = int(np.max(np.diff(b))) if world > 0 else 0
    return Layout(rank, world, b, max(m_max, 1))


class GpuOps:
    """Local steps on the GPU (libyaspmv): the fused power step — the BCCOO SpMV kernel
    with its epilogue scaling y by 1/||z_prev|| and producing the partials of ||y||^2 —
    plus the plain SpMV / norm / scale kernels for the unfused path."""

    def __init__(self, A, n_local_rows: int, device):
        import torch

        from .matrix import nrm2sq_scratch_bytes
        self.A = A
        self.scratch = torch.zeros(nrm2sq_scratch_bytes(max(n_local_rows, 1)) // 8 + 1, dtype=torch.float64,
                                   device=device)

    def power_step(self, v, z, in_norm2, out_norm2):
        self.A.spmv_power(v, z, in_norm2, out_norm2)

    def spmv(self, x, y):
        self.A.spmv(x, y)

    def nrm2sq(self, y, out):
        from .matrix import nrm2sq
        nrm2sq(y, out, self.scratch)

    def scale(self, src, dst, norm2):
        from .matrix import scale
        scale(src, dst, norm2)

    def launches_per_step(self) -> int:
        return self.A.launches_per_power_step()


class PowerIteration:
    """x_{k+1} = A x_k / ||A x_k|| with A row-partitioned over the process group.

    Fused form (ops with ``power_step``): the iterate is kept unnormalised, z_k = A x_k,
    and x_k = z_{k-1} / ||z_{k-1}|| is never materialised — each step is one SpMV launch
    whose epilogue applies 1/||z_{k-1}|| and produces ||z_k||^2 partials, then one scalar
    all-reduce and the all-gather of z_k's row blocks (N > 1).  Unfused form (ops with
    spmv / nrm2sq / scale): normalise explicitly after every SpMV."""

    def __init__(self, layout: Layout, ops, dtype, device, group=None):
        import torch
        self.L = layout
        self.ops = ops
        self.group = group
        self.fused = hasattr(ops, "power_step")
        self.x = torch.zeros(layout.n_padded, dtype=dtype, device=device)      # replicated vector
        self.y = torch.zeros(layout.m_max, dtype=dtype, device=device)         # padded local block
        self.norm2 = torch.zeros(1, dtype=torch.float64, device=device)
        self.norm_prev = torch.ones(1, dtype=torch.float64, device=device)     # ||z_{k-1}||^2 (1: x_0)
        self.first = True
        n_true = int(layout.bounds[-1])
        for r in range(layout.world):  # x_0 = 1/sqrt(N) on the real entries
            a = r * layout.m_max
            self.x[a: a + int(layout.bounds[r + 1] - layout.bounds[r])] = 1.0 / np.sqrt(max(n_true, 1))

    def step(self):
        import torch.distributed as dist
        L = self.L
        y_loc = self.y[: L.m_local]
        if self.fused:
            # z_k = (A z_{k-1}) / ||z_{k-1}||  and  ||z_k||^2  (one SpMV launch + 2 tiny sums)
            self.ops.power_step(self.x, y_loc, None if self.first else self.norm_prev, self.norm2)
            self.first = False
            if L.world > 1:
                dist.all_reduce(self.norm2, group=self.group)                  # 1 fp64 over NVLink
                dist.all_gather_into_tensor(self.x, self.y, group=self.group)  # replicate z_k
            else:
                self.x, self.y = self.y, self.x                                  # z_k is the next input
            self.norm_prev, self.norm2 = self.norm2, self.norm_prev
            return self.x
        self.ops.spmv(self.x, y_loc)                    # y_r = A_r x
        self.ops.nrm2sq(y_loc, self.norm2)              # ||y_r||^2
        if L.world > 1:
            dist.all_reduce(self.norm2, group=self.group)
            self.ops.scale(y_loc, y_loc, self.norm2)
            dist.all_gather_into_tensor(self.x, self.y, group=self.group)
        else:
            self.ops.scale(y_loc, self.x[: L.m_local], self.norm2)
        return self.x

    def current_x(self):
        """The normalised iterate x_k (materialised; for checks)."""
        if self.fused and not self.first:
            return self.x / self.norm_prev.sqrt().to(self.x.dtype)
        return self.x


class FusedPowerIteration:
    """The power iteration with the exchange fused into the SpMV (yaspmv_power_step_fused,
    SURVEY.md §8(f) NEXT #1): each rank's SpMV stores its rows of z_k directly into every
    rank's copy of the next x over peer memory (NVLink P2P through CUDA IPC), and a one-warp
    publish / wait kernel pair replaces the NCCL all-reduce + all-gather.  One call of
    ``step`` = wait for the peers' previous step + SpMV (+ BCCOO+ combine) + ||z||^2 + publish,
    all on the device; the host never blocks.

    ``comm``: an already connected ``Comm`` (tests: several ranks as several handles of one
    process, ``Comm.connect_local``); otherwise one is created on ``device`` and, for
    world > 1, the ranks exchange IPC handles over ``group`` (torch.distributed
    all_gather_object) and map each other's buffers.  ``comm_factory`` replaces the Comm
    class (CPU tests of the exchange logic)."""

    def __init__(self, layout: Layout, A, dtype, device, group=None, comm=None, timeout_ms: int = 0,
                 comm_factory=None, multicast=False):
        import torch
        self.L = layout
        self.A = A
        self.group = group
        self.device = torch.device(device)
        self.own_comm = comm is None
        self.multicast = False
        if comm is None:
            if comm_factory is None:
                from .matrix import Comm as comm_factory
            npdt = np.float32 if dtype == torch.float32 else np.float64
            err = None
            try:
                comm = comm_factory(self.device.index or 0, layout.rank, layout.world, layout.m_max, npdt, timeout_ms)
            except Exception as e:  # agreed on below, so that no rank is left waiting for a peer
                comm, err = None, e
            if layout.world > 1:
                import torch.distributed as dist
                self._agree(err, group, "create the exchange buffers")
                # the IPC handle too is agreed on: a rank that cannot export its buffer
                # gathers None instead of raising before the collective (no rank hangs)
                try:
                    mine = comm.ipc_handle()
                except Exception as e:
                    mine, err = None, e
                handles = [None] * layout.world
                dist.all_gather_object(handles, mine, group=group)
                try:
                    self._agree(err, group, "export the IPC handles")
                except RuntimeError:
                    if hasattr(comm, "free"):
                        comm.free()
                    raise
                try:
                    comm.open_ipc(handles)
                except Exception as e:
                    err = e
                try:
                    self._agree(err, group, "map the peers' buffers")
                except RuntimeError:
                    if hasattr(comm, "free"):
                        comm.free()
                    raise
            elif err is not None:
                raise err
            if multicast:
                self._setup_multicast(comm, layout, group, required=multicast is True)
        self.comm = comm
        self.restart()

    def _setup_multicast(self, comm, layout, group, required):
        """NVSwitch multicast (yaspmv_comm_mc_*): rank 0 creates the multicast object and
        exports it as a POSIX fd, the others duplicate it (pidfd_getfd), every rank adds its
        device, then every rank binds its x buffers; from then on each step stores z once
        through the multicast mapping instead of once per rank.  Every stage is agreed on;
        ``required`` False (multicast="auto") keeps the peer stores if any rank fails."""
        import os
        world = layout.world
        def stage(fn, what):
            err = None
            try:
                out = fn()
            except Exception as e:
                out, err = None, e
            if world > 1:
                self._agree(err, group, what)
            elif err is not None:
                raise RuntimeError(f"fused exchange: could not {what}: {err}")
            return out
        def probe():
            if not comm.mc_supported(self.device.index or 0):
                raise RuntimeError("the device reports no switch multicast")
        try:
            stage(probe, "use switch multicast")
            mine = stage(lambda: (os.getpid(), comm.mc_create()) if layout.rank == 0 else None,
                         "create the multicast object")
            if world > 1:
                import torch.distributed as dist
                infos = [None] * world
                dist.all_gather_object(infos, mine, group=group)
                pid, fd = infos[0]
            else:
                pid, fd = mine
            stage(lambda: None if layout.rank == 0 else comm.mc_import(pid, fd), "import the multicast object")
            stage(comm.mc_add_device, "add the devices to the multicast object")
            stage(comm.mc_bind, "bind the x buffers to the multicast object")
        except RuntimeError:
            # every rank learned of the failure (the stages are agreed on): a rank whose own
            # bind succeeded goes back to peer stores too, so all ranks use one protocol
            if getattr(comm, "mc_active", False):
                comm.mc_release()
            if required:
                raise
        self.multicast = bool(getattr(comm, "mc_active", False))

    @staticmethod
    def _agree(err, group, what):
        """Every rank learns whether every rank succeeded; all raise together (the caller
        then falls back to the NCCL protocol on every rank, never on some)."""
        import torch.distributed as dist
        oks = [None] * dist.get_world_size(group)
        dist.all_gather_object(oks, None if err is None else f"{type(err).__name__}: {err}", group=group)
        bad = {r: m for r, m in enumerate(oks) if m is not None}
        if bad:
            raise RuntimeError(f"fused exchange: could not {what} on rank(s) {sorted(bad)}: {next(iter(bad.values()))}")

    def restart(self):
        """x_0 = 1/sqrt(N) on the real entries of this rank's copy, then (world > 1, own comm)
        a barrier so that no peer writes into a buffer before every rank is ready.  Before
        x_0 is written, every peer's last step must be over: its SpMV stores z rows into this
        rank's buffers over peer memory (wait for the peers on the device, synchronize,
        barrier)."""
        import torch
        L = self.L
        if self.own_comm and L.world > 1 and getattr(self, "first", None) is False:
            import torch.distributed as dist
            self.comm.wait(None)
            if self.device.type == "cuda":
                torch.cuda.synchronize(self.device)
            dist.barrier(group=self.group)
        x = self.comm.x(0)
        x.zero_()
        n_true = int(L.bounds[-1])
        for r in range(L.world):
            a = r * L.m_max
            x[a: a + int(L.bounds[r + 1] - L.bounds[r])] = 1.0 / np.sqrt(max(n_true, 1))
        self.comm.begin()
        if self.own_comm and L.world > 1:
            import torch.distributed as dist
            if self.device.type == "cuda":
                torch.cuda.synchronize(self.device)
            dist.barrier(group=self.group)
        self.first = True

    def step(self, stream=None):
        self.A.power_step_fused(self.comm, stream)
        self.first = False

    def launches_per_step(self) -> int:
        return self.A.launches_per_fused_step()

    def z(self):
        """The latest unnormalised iterate z_k (this rank's replicated copy, padded layout)."""
        return self.comm.x(0)

    def current_x(self, stream=None):
        """x_k = z_k / ||z_k|| (materialised; waits on the device for every peer's step)."""
        if self.first:
            return self.comm.x(0).clone()
        self.comm.wait(stream)
        return self.comm.x(0) / self.comm.norm2().sqrt().to(self.comm.x(0).dtype)
