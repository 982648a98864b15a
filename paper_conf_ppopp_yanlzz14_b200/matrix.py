"""Python binding of the C ABI (include/yaspmv.h): argument marshalling only.

Every step of the SpMV runs in libyaspmv.so (host encoder in C++, kernels in CUDA for
sm_100a).  torch is used for device memory and streams only; numpy for host arrays.
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _lib
from ._lib import check, lib

_DT = {np.dtype(np.float32): _lib.F32, np.dtype(np.float64): _lib.F64}


def _ptr(a) -> int | None:
    if a is None:
        return None
    if isinstance(a, int):
        return a
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()  # torch.Tensor


def _stream(stream) -> int | None:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def make_params(**kw) -> _lib.Params:
    p = _lib.Params()
    names = {"h": "block_h", "w": "block_w", "S": "slices", "T": "thread_tile", "C": "cta_size",
             "rc": "result_cache", "tpc": "tiles_per_cta", "B": "band", "R": "panel_rows", "W": "slice_width",
             "col0": "band_col0", "far": "band_far"}
    for k, v in kw.items():
        setattr(p, names.get(k, k), int(v))
    return p


class Matrix:
    """A BCCOO / BCCOO+ encoded sparse matrix resident on one GPU (or host-only with
    device=-1, for inspecting the encoder)."""

    def __init__(self, handle: ctypes.c_void_p, dtype):
        self._h = handle
        self.dtype = np.dtype(dtype)

    # ---------------------------------------------------------------- builders
    @classmethod
    def from_csr(cls, m: int, n: int, row_ptr, col, val, device: int = 0, **params) -> "Matrix":
        row_ptr = np.ascontiguousarray(row_ptr, dtype=np.int64)
        col = np.ascontiguousarray(col, dtype=np.int32)
        val = np.ascontiguousarray(val)
        if val.dtype not in _DT:
            raise TypeError("values must be float32 or float64")
        h = ctypes.c_void_p()
        p = make_params(**params)
        check(lib.yaspmv_build_csr(m, n, row_ptr.ctypes.data, col.ctypes.data, val.ctypes.data, _DT[val.dtype],
                                   ctypes.byref(p), device, ctypes.byref(h)))
        return cls(h, val.dtype)

    @classmethod
    def from_coo(cls, m: int, n: int, rows, cols, vals, device: int = 0, **params) -> "Matrix":
        rows = np.ascontiguousarray(rows, dtype=np.int32)
        cols = np.ascontiguousarray(cols, dtype=np.int32)
        vals = np.ascontiguousarray(vals)
        h = ctypes.c_void_p()
        p = make_params(**params)
        check(lib.yaspmv_build_coo(m, n, rows.size, rows.ctypes.data, cols.ctypes.data, vals.ctypes.data,
                                   _DT[vals.dtype], ctypes.byref(p), device, ctypes.byref(h)))
        return cls(h, vals.dtype)

    @classmethod
    def from_synth(cls, csr, device: int = 0, **params) -> "Matrix":
        return cls.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=device, **params)

    # ---------------------------------------------------------------- lifetime
    def free(self) -> None:
        if self._h is not None and self._h.value:
            lib.yaspmv_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()

    # ---------------------------------------------------------------- compute
    def spmv(self, x, y=None, stream=None):
        """y := A·x for device tensors (torch) or raw device pointers; returns y."""
        if y is None:
            import torch
            y = torch.empty(self.info()["m"], dtype=x.dtype, device=x.device)
        check(lib.yaspmv_spmv(self._h, _ptr(x), _ptr(y), _stream(stream)))
        return y

    def spmv_power(self, x, y, in_norm2=None, out_norm2=None, stream=None):
        """y := (A·x)/sqrt(in_norm2[0]) and out_norm2[0] := sum y^2 (device tensors; either
        norm may be None) — one fused power-iteration step."""
        check(lib.yaspmv_spmv_power(self._h, _ptr(x), _ptr(y), _ptr(in_norm2), _ptr(out_norm2), _stream(stream)))
        return y

    def launches_per_power_step(self) -> int:
        return int(lib.yaspmv_launches_per_power_step(self._h))

    def power_step_fused(self, comm: "Comm", stream=None) -> None:
        """One fused power step over `comm` (yaspmv_power_step_fused): z_k of this rank's
        rows goes straight into every rank's copy of the next x."""
        check(lib.yaspmv_power_step_fused(self._h, comm._h, _stream(stream)))

    def launches_per_fused_step(self) -> int:
        return int(lib.yaspmv_launches_per_fused_step(self._h))

    def spmv_host(self, x: np.ndarray, y: np.ndarray | None = None, stream=None) -> np.ndarray:
        """y := A·x with host arrays (copies in and out inside the call)."""
        x = np.ascontiguousarray(x, dtype=self.dtype)
        if y is None:
            y = np.empty(self.info()["m"], dtype=self.dtype)
        check(lib.yaspmv_spmv_host(self._h, _ptr(x), _ptr(y), _stream(stream) if stream != 0 else 0))
        return y

    def spmv_host_async(self, x: np.ndarray, y: np.ndarray, stream=None) -> None:
        """Queue y := A·x with host arrays (pinned for overlap); call host_sync() before
        reading y or reusing x."""
        check(lib.yaspmv_spmv_host_async(self._h, _ptr(x), _ptr(y), _stream(stream) if stream != 0 else 0))

    def host_sync(self) -> None:
        check(lib.yaspmv_host_sync(self._h))

    def tune(self, stream=None, exhaustive: bool = False) -> dict:
        p = _lib.Params()
        check(lib.yaspmv_tune_ex(self._h, _stream(stream), ctypes.byref(p), 1 if exhaustive else 0))
        return p.as_dict()

    def reencode(self, **params) -> None:
        p = make_params(**params)
        check(lib.yaspmv_reencode(self._h, ctypes.byref(p)))

    # ---------------------------------------------------------------- introspection
    def info(self) -> dict:
        inf = _lib.Info()
        check(lib.yaspmv_get_info(self._h, ctypes.byref(inf)))
        return inf.as_dict()

    def launches_per_spmv(self) -> int:
        return int(lib.yaspmv_launches_per_spmv(self._h))

    def profile_begin(self) -> None:
        """Record CUDA events around every kernel group of the following SpMVs."""
        check(lib.yaspmv_profile_begin(self._h))

    def profile_end(self) -> dict:
        """Summed device milliseconds per stage since profile_begin(): plain/far part,
        band kernel, band y^2 sum; and the number of calls."""
        ms = (ctypes.c_double * 3)()
        calls = ctypes.c_int64()
        check(lib.yaspmv_profile_end(self._h, ms, 3, ctypes.byref(calls)))
        return {"plain_ms": ms[0], "band_ms": ms[1], "band_sum_ms": ms[2], "calls": calls.value}

    _ARR_DT = {"flags": np.uint8, "col_delta": np.int16, "seg_row": np.int32, "zero_rows": np.int32,
               "cta_seg0": np.int32, "fre": np.int32, "band_flags": np.uint8, "band_col16": np.uint16,
               "band_panel_blk0": np.int64, "band_slice_ptr": np.int32, "band_stop_ptr": np.int32,
               "band_first_row": np.int32, "band_tile_rank": np.int32, "band_far_col": np.int32,
               "band_far_blk0": np.int64}

    def _arr_dtype(self, name: str):
        if name.startswith("val") or name == "band_val":
            return self.dtype
        if name == "col":
            return np.uint16 if self.info()["params"]["col_mode"] == _lib.COL_U16 else np.int32
        return self._ARR_DT[name]

    def export(self, name: str, device: bool = False) -> np.ndarray:
        """Canonical encoded array; device=True reads the uploaded
        device copy and un-permutes it."""
        fn = lib.yaspmv_export_device if device else lib.yaspmv_export
        nb = ctypes.c_int64()
        check(fn(self._h, _lib.ARR[name], None, 0, ctypes.byref(nb)))
        out = np.empty(nb.value, dtype=np.uint8)
        check(fn(self._h, _lib.ARR[name], out.ctypes.data if nb.value else None, nb.value, ctypes.byref(nb)))
        return out.view(self._arr_dtype(name))

    def export_range(self, name: str, first_tile: int, ntiles: int) -> np.ndarray:
        """Canonical array `name` for workgroup tiles [first_tile, first_tile + ntiles),
        read back from the device (yaspmv_export_device_range)."""
        nb = ctypes.c_int64()
        check(lib.yaspmv_export_device_range(self._h, _lib.ARR[name], first_tile, ntiles, None, 0, ctypes.byref(nb)))
        out = np.empty(nb.value, dtype=np.uint8)
        check(lib.yaspmv_export_device_range(self._h, _lib.ARR[name], first_tile, ntiles,
                                              out.ctypes.data if nb.value else None, nb.value, ctypes.byref(nb)))
        return out.view(self._arr_dtype(name))


class Comm:
    """The replicated x of a row-partitioned power iteration (yaspmv_comm, include/yaspmv.h
    "fused multi-GPU power step"): two x buffers + a signal pad in one device allocation,
    mapped by every peer."""

    def __init__(self, device: int, rank: int, world: int, chunk: int, dtype, timeout_ms: int = 0):
        self.dtype = np.dtype(dtype)
        self.device, self.rank, self.world, self.chunk = device, rank, world, chunk
        h = ctypes.c_void_p()
        check(lib.yaspmv_comm_create(device, rank, world, chunk, _DT[self.dtype], timeout_ms, ctypes.byref(h)))
        self._h = h

    def ipc_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(_lib.IPC_HANDLE_BYTES)
        check(lib.yaspmv_comm_ipc_handle(self._h, buf, _lib.IPC_HANDLE_BYTES))
        return buf.raw

    def open_ipc(self, handles: list[bytes]) -> None:
        blob = b"".join(h if h is not None else bytes(_lib.IPC_HANDLE_BYTES) for h in handles)
        check(lib.yaspmv_comm_open_ipc(self._h, blob, len(blob)))

    def connect_local(self, peers: list["Comm"]) -> None:
        arr = (ctypes.c_void_p * len(peers))(*[p._h.value for p in peers])
        check(lib.yaspmv_comm_connect_local(self._h, arr, len(peers)))

    # ---- NVSwitch multicast (include/yaspmv.h "yaspmv_comm_mc_*")
    @staticmethod
    def mc_supported(device: int) -> bool:
        return bool(lib.yaspmv_comm_mc_supported(device))

    def mc_create(self) -> int:
        """Creator rank: the multicast object for `world` devices; returns its POSIX fd."""
        fd = ctypes.c_int64()
        check(lib.yaspmv_comm_mc_create(self._h, ctypes.byref(fd)))
        return fd.value

    def mc_import(self, pid: int, fd: int) -> None:
        check(lib.yaspmv_comm_mc_import(self._h, pid, fd))

    def mc_add_device(self) -> None:
        check(lib.yaspmv_comm_mc_add_device(self._h))

    def mc_bind(self) -> None:
        check(lib.yaspmv_comm_mc_bind(self._h))

    @property
    def mc_active(self) -> bool:
        return bool(lib.yaspmv_comm_mc_active(self._h))

    def mc_release(self) -> None:
        check(lib.yaspmv_comm_mc_release(self._h))

    def x(self, which: int = 0):
        """torch view of x buffer (seq + which) % 2 (which = 0: the next step's input /
        the latest z; 1: the buffer the next step writes), world * chunk elements."""
        import torch
        ptr = lib.yaspmv_comm_x(self._h, which)
        n = self.world * self.chunk
        tdt = torch.float32 if self.dtype == np.float32 else torch.float64
        return _device_view(ptr, n, tdt, self.device)

    def norm2(self):
        """torch view of the device double written by wait(): total ||z||^2."""
        import torch
        return _device_view(lib.yaspmv_comm_norm2_device(self._h), 1, torch.float64, self.device)

    def begin(self) -> None:
        check(lib.yaspmv_comm_begin(self._h))

    def wait(self, stream=None) -> None:
        check(lib.yaspmv_comm_wait(self._h, _stream(stream)))

    def check(self) -> None:
        check(lib.yaspmv_comm_check(self._h))

    @property
    def seq(self) -> int:
        return int(lib.yaspmv_comm_seq(self._h))

    def free(self) -> None:
        if self._h is not None and self._h.value:
            lib.yaspmv_comm_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def _device_view(ptr: int, n: int, tdt, device: int):
    """A torch tensor over n elements of raw device memory owned by libyaspmv (no copy)."""
    import torch
    itemsize = torch.empty(0, dtype=tdt).element_size()

    class _Arr:  # __cuda_array_interface__ shim
        __cuda_array_interface__ = {"shape": (n,), "typestr": ("<f%d" % itemsize), "data": (ptr, False),
                                    "version": 3, "strides": None}
    with torch.cuda.device(device):
        return torch.as_tensor(_Arr(), device=f"cuda:{device}")


def nrm2sq(v, out, scratch, stream=None) -> None:
    """out[0] := sum v^2 (device, fp64, deterministic)."""
    import torch
    dt = _lib.F32 if v.dtype == torch.float32 else _lib.F64
    check(lib.yaspmv_nrm2sq(v.data_ptr(), v.numel(), dt, out.data_ptr(), scratch.data_ptr(), _stream(stream)))


def nrm2sq_scratch_bytes(n: int) -> int:
    return int(lib.yaspmv_nrm2sq_scratch_bytes(n))


def scale(src, dst, norm2, stream=None) -> None:
    """dst := src / sqrt(norm2[0]) (device)."""
    import torch
    dt = _lib.F32 if src.dtype == torch.float32 else _lib.F64
    check(lib.yaspmv_scale(src.data_ptr(), dst.data_ptr(), src.numel(), dt, norm2.data_ptr(), _stream(stream)))


def version() -> str:
    return lib.yaspmv_version().decode()


def l2_persist(device: int, nbytes: int) -> int:
    """cudaLimitPersistingL2CacheSize for `device` (yaspmv_l2_persist): the L2 set-aside the
    kernels' evict_last x gathers use; returns the bytes now in effect."""
    out = ctypes.c_int64()
    check(lib.yaspmv_l2_persist(device, nbytes, ctypes.byref(out)))
    return out.value
