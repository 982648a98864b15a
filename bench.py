#!/usr/bin/env python
"""bench.py — iterated SpMV (power iteration) over BCCOO/BCCOO+ on B200, one JSON line.

Workload (BASELINE.json configs[4], the config the metric "SpMV GFLOPS and achieved HBM
GB/s at 1/2/4/8 B200" is quoted on; it fits one GPU): C5, a circuit/LP-like 50M x 50M
matrix with ~1.0B non-zeros, fp32 (synth/c5gen.c).  A step is one power iteration:
y_r = A_r x (fused BCCOO SpMV kernel, §3 of the paper), ||y||^2, scale, and for N > 1 the
NCCL all-reduce of one scalar + all-gather of x.  The matrix is fixed as N grows
(strong scaling); each rank builds only its nnz-balanced row block.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl yaspmv|reference]
                  [--config c5|c4|c3-spheres|...] [--params '{"T":16,"C":256}']

--impl reference times the CPU oracle (oracle/ref_csr.c, compensated CSR matvec with
OpenMP) on a bounded row sample of the same workload — the slow baseline of this tier.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# tuned defaults per config (yaspmv_tune on B200)
DEFAULT_PARAMS = {
    # C5: band kernel on panels of 16128 rows (3,101 panels = 20.95 waves of 148 SMs; 9 slices of
    # 16384 columns); far part BCCOO+ S = 3, T = 8, C = 128, 4 tiles per CTA (profiles/r05_*)
    "c5": dict(h=1, w=1, S=3, T=8, C=128, tpc=4, col_mode=2, B=65536, R=16128, W=16384),
    "c4": dict(h=1, w=1, S=1, T=16, C=256),
    "c3-spheres": dict(h=4, w=4, T=4, C=128),
    "c3-cantilever": dict(h=4, w=4, T=4, C=128),
    "c3-ship": dict(h=2, w=2, T=8, C=256),
    "c2-f32": dict(h=4, w=4, T=4, C=128),
    "c2-f64": dict(h=4, w=4, T=4, C=128),
    "c1": dict(T=4, C=64),
}


# cudaLimitPersistingL2CacheSize per config (MB; yaspmv_l2_persist), --l2-persist-mb overrides
L2_PERSIST_MB = {"c5": 60}


def _env_int(k, d):
    try:
        return int(os.environ.get(k, d))
    except ValueError:
        return d


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""
    FIELDS = ["clocks.sm", "clocks.max.sm", "clocks_event_reasons.sw_power_cap",
              "clocks_event_reasons.hw_slowdown", "clocks_event_reasons.hw_thermal_slowdown",
              "clocks_event_reasons.sw_thermal_slowdown"]

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), "--query-gpu=" + ",".join(self.FIELDS),
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
            return
        self.t = threading.Thread(target=self._read, daemon=True)
        self.t.start()
        t0 = time.time()
        while not self.rows and time.time() - t0 < 5:
            time.sleep(0.02)

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) == len(self.FIELDS):
                self.rows.append(parts)

    def stop(self) -> dict:
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.1)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        rows = self.rows
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        reasons = set()
        for r in rows:
            for name, v in zip(["sw_power_cap", "hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown"], r[2:]):
                if v.lower().startswith("active"):
                    reasons.add(name)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(rows)}


def bind_numa_local(gpu: int) -> dict:
    """Run on the CPUs of the GPU's NUMA node, so that pinned host buffers (first touch)
    are NUMA-local to the GPU for the e2e copies."""
    try:
        import torch
        p = torch.cuda.get_device_properties(gpu)
        bus = f"{p.pci_domain_id:04x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0"
        with open(f"/sys/bus/pci/devices/{bus}/numa_node") as f:
            node = int(f.read().strip())
        if node < 0:
            return {"numa_node": None, "note": "no NUMA affinity reported"}
        with open(f"/sys/devices/system/node/node{node}/cpulist") as f:
            cpus = set()
            for part in f.read().strip().split(","):
                a, _, b = part.partition("-")
                cpus.update(range(int(a), int(b or a) + 1))
        os.sched_setaffinity(0, cpus)
        return {"numa_node": node, "cpus": len(cpus), "pci": bus}
    except Exception as e:
        return {"numa_node": None, "note": f"{type(e).__name__}: {e}"[:120]}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def load_matrix(config: str, rank: int, world: int, dtype, rows: int = 0):
    """Returns (local CSR, layout) — the rank's nnz-balanced row block, columns remapped to
    the padded all-gather space when world > 1."""
    import synth
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import dist as D
    if config == "c5":
        kw = dict(n=rows) if rows else {}
        if world == 1:
            csr = sm.circuit_like_rows(0, rows or 50_000_000, dtype=dtype, **kw)
            L = D.Layout(0, 1, np.array([0, csr.m], dtype=np.int64), csr.m)
            return csr, L
        # global row lengths (cheap pass) -> partition -> generate only this rank's rows
        import ctypes
        P = sm.c5_params(**kw)
        counts = np.empty(P.n, dtype=np.int64)
        sm._lib().c5_count(ctypes.byref(P), ctypes.c_int64(0), ctypes.c_int64(P.n),
                            counts.ctypes.data_as(ctypes.c_void_p))
        rp = np.zeros(P.n + 1, dtype=np.int64)
        np.cumsum(counts, out=rp[1:])
        del counts
        L = D.make_layout(rp, rank, world)
        csr = sm.circuit_like_rows(L.r0, L.r1, dtype=dtype, **kw)
    else:
        full = synth.config_matrix(config)
        if world == 1:
            return full, D.Layout(0, 1, np.array([0, full.m], dtype=np.int64), full.m)
        L = D.make_layout(full.row_ptr, rank, world)
        csr = full.row_slice(L.r0, L.r1)
    csr.col = D.remap_columns(csr.col, L.bounds, L.m_max)
    csr.n = L.n_padded
    return csr, L


def run_reference(args, rank, world):
    """The oracle (oracle/ref_csr.c) on a bounded row sample of the workload."""
    if rank != 0:
        return
    from oracle import ref
    import synth
    from synth import matrices as sm
    if args.config == "c5":
        rows = 1 << 21  # 2M rows x ~20 nnz: ~0.3 s per oracle call on 16 cores
        csr = sm.circuit_like_rows(0, rows, dtype=np.float32)
        x = np.full(50_000_000, 1.0 / np.sqrt(5e7), dtype=np.float32)
        sample = f"rows [0, {rows}) of C5 ({csr.nnz} nnz), all 50M columns"
    else:
        csr = synth.config_matrix(args.config)
        x = synth.make_x(csr.n, csr.val.dtype, "uniform", 0)
        sample = f"full {args.config} ({csr.nnz} nnz)"
    for _ in range(args.warmup):
        ref.spmv(csr.row_ptr, csr.col, csr.val, x, with_bound=False)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        ref.spmv(csr.row_ptr, csr.col, csr.val, x, with_bound=False)
    dt = (time.perf_counter() - t0) / max(args.steps, 1)
    gflops = 2.0 * csr.nnz / dt / 1e9
    cores = ref.num_threads()
    line = {"impl": "reference", "metric": "SpMV GFLOPS and achieved HBM GB/s (% of 8 TB/s)", "value": gflops, "unit": "GFLOPS",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32" if csr.val.dtype == np.float32 else "f64",
            "data": "synthetic", "config": {"workload": args.config, "sample": sample},
            "cpu_baseline": {"value": gflops, "unit": "GFLOPS", "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": gflops, "unit": "GFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


_ONE_THREAD = r"""
import sys, time, numpy as np
sys.path.insert(0, %r)
from oracle import ref
d = np.load(%r)
x = np.load(%r)
ref.spmv(d["rp"], d["col"], d["val"], x, with_bound=False)
ts = []
for _ in range(3):
    t0 = time.perf_counter(); ref.spmv(d["rp"], d["col"], d["val"], x, with_bound=False); ts.append(time.perf_counter() - t0)
print(min(ts), ref.num_threads())
"""


def cpu_baseline(csr_full, x_np, budget_s=12.0):
    """The oracle as it stands on the box's host cores, on a bounded row sample (SURVEY
    §8(d) "Oracle timing": all cores, one thread, and scipy's csr @ x for reference)."""
    from oracle import ref
    m = csr_full.m
    rows = min(m, 1 << 20)
    while True:
        sub = csr_full.row_slice(0, rows)
        t0 = time.perf_counter()
        ref.spmv(sub.row_ptr, sub.col, sub.val, x_np, with_bound=False)
        dt = time.perf_counter() - t0
        if dt > 0.5 or rows >= m:
            break
        rows = min(m, rows * 4)
    reps = max(1, min(5, int(budget_s / max(dt, 1e-3))))
    ts = []
    for _ in range(reps):
        t0 = time.perf_counter()
        ref.spmv(sub.row_ptr, sub.col, sub.val, x_np, with_bound=False)
        ts.append(time.perf_counter() - t0)
    t = float(np.median(ts))
    out = {"value": 2.0 * sub.nnz / t / 1e9, "unit": "GFLOPS", "cores": ref.num_threads(), "kind": "oracle",
           "sample": f"rows [0, {rows}) ({sub.nnz} nnz) of the workload, median of {reps}",
           "cpu_model": cpu_model(), "logical_cpus": os.cpu_count()}
    # one thread (a subprocess with OMP_NUM_THREADS=1) on a quarter of the sample
    try:
        import tempfile
        r1 = max(1, rows // 4)
        s1 = csr_full.row_slice(0, r1)
        with tempfile.TemporaryDirectory() as td:
            fa, fx = os.path.join(td, "a.npz"), os.path.join(td, "x.npy")
            np.savez(fa, rp=s1.row_ptr, col=s1.col, val=s1.val)
            np.save(fx, x_np)
            env = dict(os.environ, OMP_NUM_THREADS="1")
            r = subprocess.run([sys.executable, "-c", _ONE_THREAD % (ROOT, fa, fx)], env=env, capture_output=True,
                               text=True, timeout=300)
            t1, nt = r.stdout.split()
            out["single_thread"] = {"value": 2.0 * s1.nnz / float(t1) / 1e9, "unit": "GFLOPS", "threads": int(nt),
                                    "sample": f"rows [0, {r1}) ({s1.nnz} nnz), best of 3"}
    except Exception as e:  # report, never fail the bench line
        out["single_thread"] = {"error": str(e)[:200]}
    try:  # scipy's CSR matvec (single-threaded), same sample as the all-core number
        import scipy.sparse as sp
        A = sp.csr_matrix((sub.val, sub.col, sub.row_ptr), shape=(sub.m, x_np.size))
        A @ x_np
        t2 = min(_timed(lambda: A @ x_np) for _ in range(3))
        out["scipy_csr_matvec"] = {"value": 2.0 * sub.nnz / t2 / 1e9, "unit": "GFLOPS", "threads": 1,
                                   "sample": out["sample"]}
    except Exception as e:
        out["scipy_csr_matvec"] = {"error": str(e)[:200]}
    return out


def _timed(f) -> float:
    t0 = time.perf_counter()
    f()
    return time.perf_counter() - t0


def roofline_of(kern, dom, step_gbs, info, peak, peak_kind, traffic, traffic_src):
    """The bench line's roofline object for the dominant kernel (longest per-step device
    time, from the events recorded between the kernel groups during the timed region)."""
    if not dom:  # fused multi-GPU step: the whole step
        return {"bound": "hbm", "achieved": step_gbs, "peak": peak, "unit": "GB/s", "frac": step_gbs / peak,
                "traffic": None, "peak_kind": peak_kind, "kernel": "whole fused step",
                "alg_bytes_per_launch": info["alg_bytes"]}
    ms, alg = kern[dom]
    ach = alg / (ms * 1e-3) / 1e9
    r = {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak, "traffic": traffic,
         "peak_kind": peak_kind, "kernel": dom, "alg_bytes_per_launch": alg, "ms_per_launch": ms,
         "share_of_step": None}
    tot = sum(v[0] for v in kern.values())
    if tot > 0:
        r["share_of_step"] = ms / tot
    if traffic:
        r["dram_frac"] = traffic / (ms * 1e-3) / 1e9 / peak
        r["traffic_over_alg"] = traffic / alg
        r["traffic_source"] = traffic_src
    return r


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=400)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="yaspmv", choices=["yaspmv", "reference"])
    ap.add_argument("--config", default="c5")
    ap.add_argument("--params", default=None, help="JSON dict of build parameters")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=30)
    ap.add_argument("--backend", default="nccl", help="process-group backend for N > 1 (gloo: exchange-path "
                    "check with several ranks on one GPU; never a performance number)")
    ap.add_argument("--rows", type=int, default=0, help="C5 only: use the first ROWS rows/cols (checks)")
    ap.add_argument("--l2-persist-mb", type=int, default=-1,
                    help="L2 set-aside for persisting (evict_last) accesses in MB; -1: the config's default")
    ap.add_argument("--exchange", default="auto", choices=["auto", "fused", "nccl"],
                    help="x replication for N > 1: nccl = all_reduce + all_gather_into_tensor (the default "
                         "until the fused path has run across devices); fused = SpMV write-back into every "
                         "rank's x over peer memory (yaspmv_power_step_fused, CUDA IPC, plain BCCOO/BCCOO+ "
                         "only). auto: nccl for N > 1 (the fused step is timed as extra keys when it can run)")
    args = ap.parse_args()

    world = _env_int("WORLD_SIZE", 1)
    rank = _env_int("RANK", 0)
    local_rank = _env_int("LOCAL_RANK", 0)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    from paper_conf_ppopp_yanlzz14_b200 import dist as D

    ngpu = max(1, torch.cuda.device_count())
    torch.cuda.set_device(local_rank % ngpu)
    dev = torch.device("cuda", local_rank % ngpu)
    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(args.backend)
    dtype_np = np.float64 if args.config in ("c1", "c2-f64", "c3-ship-f64") else np.float32
    tdt = torch.float64 if dtype_np == np.float64 else torch.float32

    t_build0 = time.perf_counter()
    csr, L = load_matrix(args.config, rank, world, dtype_np, args.rows)
    t_gen = time.perf_counter() - t_build0
    params = dict(DEFAULT_PARAMS.get(args.config, {}))
    if args.params:
        params.update(json.loads(args.params))
    if params.get("B", 0) and world > 1:
        params["col0"] = L.rank * L.m_max  # the rank's diagonal in the padded column space
    big = csr.nnz > 50_000_000
    # DROP_CSR (no host copy kept) + GPU translation to BCCOO for the 1B-nnz matrix
    params.setdefault("flags", (2 | 4) if big else 0)
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=local_rank % ngpu, **params)
    # L2 set-aside for the evict_last x gathers (yaspmv_l2_persist): C5's far part gathers from
    # 67 MB BCCOO+ slices of x; 60 MB measured best (far part 1.05 -> 0.99 ms)
    l2_persist_mb = L2_PERSIST_MB.get(args.config, 0) if args.l2_persist_mb < 0 else args.l2_persist_mb
    l2_persist_set = None
    if l2_persist_mb > 0:
        from paper_conf_ppopp_yanlzz14_b200 import l2_persist
        l2_persist_set = l2_persist(local_rank % ngpu, l2_persist_mb << 20)
    info = A.info()
    t_build = time.perf_counter() - t_build0

    ops = D.GpuOps(A, L.m_local, dev)
    if args.config != "c5" and csr.m != csr.n and world == 1:
        raise SystemExit("power iteration needs a square matrix")
    stream = torch.cuda.current_stream()
    exchange = args.exchange
    if exchange == "auto":
        exchange = "nccl" if world > 1 else "none"
    fpit = None
    if exchange == "fused":
        try:
            fpit = D.FusedPowerIteration(L, A, tdt, dev, timeout_ms=120000)
        except Exception as e:  # e.g. no P2P/IPC between the GPUs: the NCCL protocol instead
            if args.exchange == "fused":
                raise
            print(f"[bench] fused exchange unavailable ({e}); using NCCL", file=sys.stderr)
            exchange = "nccl"
    if exchange == "none" and world > 1:
        exchange = "nccl"
    pit = D.PowerIteration(L, ops, tdt, dev) if fpit is None else None

    def one_step():
        if fpit is not None:
            fpit.step(stream)
        else:
            pit.step()

    for _ in range(max(args.warmup, 3)):
        one_step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()

    # ---- timed region: K steps, CUDA events on the launching stream ----------------
    sampler = ClockSampler(local_rank % ngpu)
    sampler.start()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    if fpit is None:
        A.profile_begin()  # events between the kernel groups of every timed step (per-kernel roofline)
    e0.record(stream)
    L_ = L
    for k in range(args.steps):
        if fpit is not None:
            # fused exchange: wait for the peers' previous step + SpMV storing z_k into every
            # rank's x + ||z_k||^2 + publish; the events bracket the whole step
            ev[k][0].record(stream)
            fpit.step(stream)
            ev[k][1].record(stream)
            continue
        # the fused step: SpMV kernel with the 1/||z_{k-1}|| scaling and ||z_k||^2 partials in
        # its epilogue (+ 2 tiny reduction kernels); events bracket it on the launching stream
        ev[k][0].record(stream)
        ops.power_step(pit.x, pit.y[: L_.m_local], None if pit.first else pit.norm_prev, pit.norm2)
        ev[k][1].record(stream)
        pit.first = False
        if world > 1:
            dist.all_reduce(pit.norm2)
            dist.all_gather_into_tensor(pit.x, pit.y)
        else:
            pit.x, pit.y = pit.y, pit.x
        pit.norm_prev, pit.norm2 = pit.norm2, pit.norm_prev
    if fpit is not None:
        fpit.comm.wait(stream)  # every peer's last step is complete
    e1.record(stream)
    torch.cuda.synchronize()
    prof = A.profile_end() if fpit is None else None
    if fpit is not None:
        fpit.comm.check()
    if world > 1:
        dist.barrier()
    clocks = sampler.stop()
    ms_total = e0.elapsed_time(e1)
    spmv_ms = float(np.mean([a.elapsed_time(b) for a, b in ev]))
    t = torch.tensor([ms_total, spmv_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_total, spmv_ms_max = float(t[0]), float(t[1])
    ms_step = ms_total / args.steps

    nnz_local = torch.tensor([float(info["nnz"])], dtype=torch.float64, device=dev)
    alg_local = torch.tensor([float(info["alg_bytes"])], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(nnz_local)
        dist.all_reduce(alg_local)
    nnz_total = float(nnz_local.item())
    gflops = 2.0 * nnz_total / (ms_step * 1e-3) / 1e9

    # ---- e2e through the public API with HOST buffers (pinned) -----------------------
    # every step copies x host->device and y device->host; yaspmv_spmv_host_async overlaps
    # the copies of consecutive steps with the SpMV (three buffer slots, two copy streams)
    numa = bind_numa_local(local_rank % ngpu)  # pinned buffers on the GPU's NUMA node
    xh = torch.empty(L.n_padded, dtype=tdt).pin_memory()
    x_cur = fpit.current_x(stream) if fpit is not None else pit.current_x()
    xh.copy_(x_cur.cpu())
    yh = torch.empty(L.m_local, dtype=tdt).pin_memory()
    # the copy engines alone: one H2D of x and one D2H of y, CUDA events
    xd = torch.empty_like(xh, device=dev)
    yd = torch.empty_like(yh, device=dev)
    c0, c1, c2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    xd.copy_(xh, non_blocking=True)  # warm both directions once (first touch of the mappings)
    yh.copy_(yd, non_blocking=True)
    c0.record(stream)
    xd.copy_(xh, non_blocking=True)
    c1.record(stream)
    yh.copy_(yd, non_blocking=True)
    c2.record(stream)
    torch.cuda.synchronize()
    h2d_gbs = xh.numel() * xh.element_size() / (c0.elapsed_time(c1) * 1e-3) / 1e9
    d2h_gbs = yh.numel() * yh.element_size() / (c1.elapsed_time(c2) * 1e-3) / 1e9
    del xd, yd
    A.spmv_host_async(xh.numpy(), yh.numpy(), stream=stream.cuda_stream)
    A.host_sync()
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(args.e2e_steps):
        A.spmv_host_async(xh.numpy(), yh.numpy(), stream=stream.cuda_stream)
    A.host_sync()
    te = torch.tensor([(time.perf_counter() - t0) / args.e2e_steps], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_s = float(te.item())
    e2e = {"value": 2.0 * nnz_total / e2e_s / 1e9, "unit": "GFLOPS",
           "h2d_bytes_per_step": int(L.n_padded * np.dtype(dtype_np).itemsize * world),
           "d2h_bytes_per_step": int(int(L.bounds[-1]) * np.dtype(dtype_np).itemsize),
           "api": "yaspmv_spmv_host_async + yaspmv_host_sync (pinned x in, y out every step, per rank)",
           "steps": args.e2e_steps, "h2d_gbs": h2d_gbs, "d2h_gbs": d2h_gbs, "pinned_numa": numa,
           # the pipeline overlaps copy-in, SpMV and copy-out of consecutive steps: a step
           # costs at least the slowest of the three
           "h2d_ms": L.n_padded * np.dtype(dtype_np).itemsize / h2d_gbs / 1e6,
           "d2h_ms": L.m_local * np.dtype(dtype_np).itemsize / d2h_gbs / 1e6}

    # ---- N > 1: the fused exchange (peer stores from the SpMV epilogue) as extra keys ---
    fused_info = None
    if world > 1 and fpit is None and args.exchange == "auto":
        # the fused exchange (SpMV epilogue stores z into every rank's x; no NCCL), with peer
        # stores and, where the GPUs report switch multicast, with one multimem.st per element
        fused_info = {}

        def agreed_check(comm):
            # every rank learns whether any rank's device waits timed out, and all raise
            # together (no rank is left in a collective the others skipped)
            ok = 1
            try:
                comm.check()
            except Exception:
                ok = 0
            t = torch.tensor([ok], dtype=torch.int32, device=dev)
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
            if int(t.item()) == 0:
                raise RuntimeError("a fused step's device wait timed out on some rank")

        for mode, mc in (("p2p", False), ("multicast", "auto")):
            try:
                # a short device-wait timeout: a peer signal that never arrives costs seconds,
                # not minutes, and the warm-up check below skips the timed loop
                fp = D.FusedPowerIteration(L, A, tdt, dev, timeout_ms=5000, multicast=mc)
                if mc and not fp.multicast:
                    fused_info[mode] = {"unavailable": "no switch multicast on every rank"}
                    dist.barrier()
                    fp.comm.free()
                    continue
                for _ in range(3):
                    fp.step(stream)
                fp.comm.wait(stream)
                torch.cuda.synchronize()
                agreed_check(fp.comm)  # a warm-up step timed out on any rank: all skip the timed loop
                dist.barrier()
                f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                f0.record(stream)
                for _ in range(20):
                    fp.step(stream)
                fp.comm.wait(stream)
                f1.record(stream)
                torch.cuda.synchronize()
                agreed_check(fp.comm)
                tf = torch.tensor([f0.elapsed_time(f1) / 20], dtype=torch.float64, device=dev)
                dist.all_reduce(tf, op=dist.ReduceOp.MAX)
                fused_info[mode] = {"ms_per_step": float(tf.item()), "steps": 20,
                                    "gflops": 2.0 * nnz_total / (float(tf.item()) * 1e-3) / 1e9}
                dist.barrier()
                fp.comm.free()
            except Exception as e:  # never fail the bench line on the optional path
                fused_info[mode] = {"error": f"{type(e).__name__}: {e}"[:300]}

    if rank == 0:
        peak, peak_kind = measured_peaks()
        achieved = info["alg_bytes"] / (spmv_ms * 1e-3) / 1e9
        sv = np.dtype(dtype_np).itemsize
        band = info["band_blocks_pad"] > 0
        # per-kernel algorithmic bytes (DESIGN §6.1/§6.6): the band kernel K4
        # reads its stream + aux, x once, the far part's y, and writes y; the plain / far K1
        # reads its format + x and writes y
        kern = {}
        if prof and prof["calls"]:
            S = info["params"]["slices"]
            if band and info["params"]["band_far"] == 2:  # P7: one kernel, far entries in every panel's slice 0
                kern["panel_kernel (band + far slices)"] = (prof["band_ms"] / prof["calls"], info["alg_bytes"])
            elif band:  # far K1 writes its S slice results, the band kernel K4 reads and combines them
                far_bytes = info["format_bytes"] - info["band_format_bytes"] + info["n"] * sv + S * info["m"] * sv
                kern["spmv_bccoo_kernel (far part)"] = (prof["plain_ms"] / prof["calls"], far_bytes)
                kern["panel_kernel (band)"] = (prof["band_ms"] / prof["calls"],
                                               info["band_format_bytes"] + info["n"] * sv + (S + 1) * info["m"] * sv)
            else:
                kern["spmv_bccoo_kernel" + (" + combine" if S > 1 else "")] = (prof["plain_ms"] / prof["calls"],
                                                                               info["alg_bytes"])
        dom = max(kern, key=lambda k: kern[k][0]) if kern else None
        traffic, traffic_src = None, None
        tp = os.path.join(ROOT, "profiles", f"ncu_traffic_{args.config}.json")
        if os.path.exists(tp) and world == 1 and dom:
            with open(tp) as f:
                tr = json.load(f)
            strip = lambda p: {k: v for k, v in p.items() if k != "flags"}
            ent = tr.get("kernels", {}).get(dom.split(" ")[0])
            if ent and strip(ent.get("params", {})) == strip(info["params"]):
                traffic = ent.get("dram_bytes_per_launch")
                traffic_src = {"file": os.path.relpath(tp, ROOT), "commit": tr.get("commit"),
                               "captured": tr.get("captured")}
        line = {
            "metric": "SpMV GFLOPS and achieved HBM GB/s (% of 8 TB/s)", "value": gflops, "unit": "GFLOPS",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "f32" if dtype_np == np.float32 else "f64", "data": "synthetic",
            "config": {"workload": args.config, "m": int(L.bounds[-1]), "nnz": int(nnz_total),
                       "params": info["params"],
                       "parallelism": f"row-partition x{world}" + (
                           ", x replicated by peer stores from the SpMV epilogue (CUDA IPC over NVLink)"
                           if fpit is not None else ", NCCL all-gather of x" if world > 1 else ""),
                       "l2": "inputs larger than L2 (matrix 8.5 GB vs 126 MB L2), no flush" if args.config == "c5"
                       else "L2-resident workload; back-to-back steps (warm L2)",
                       "l2_persist_bytes": l2_persist_set,
                       "step": "z_k = A z_{k-1}/||z_{k-1}|| and ||z_k||^2 in one fused BCCOO SpMV launch (+2 tiny sums)"
                               + (" + NCCL allreduce(1 fp64) + allgather(z)" if world > 1 and fpit is None else "")
                               + (" storing z_k into every rank's x (peer memory) + publish/wait kernels"
                                  if fpit is not None else "")},
            "spmv_ms": spmv_ms, "spmv_ms_max_over_ranks": spmv_ms_max,
            "spmv_gflops": 2.0 * info["nnz"] / (spmv_ms * 1e-3) / 1e9,
            "hbm_gbs_alg": achieved, "pct_of_8TBs": achieved / 8000.0 * 100.0,
            "roofline": roofline_of(kern, dom, achieved, info, peak, peak_kind, traffic, traffic_src),
            "step_roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                              "frac": achieved / peak, "alg_bytes_per_step": info["alg_bytes"],
                              "kernels": {k: {"ms": v[0], "alg_bytes": v[1], "gbs": v[1] / (v[0] * 1e-3) / 1e9}
                                          for k, v in kern.items()}},
            "gpu_launches": (fpit.launches_per_step() if fpit is not None else A.launches_per_power_step())
                            * args.steps,
            "clocks": clocks, "e2e": e2e, "fused_exchange": fused_info,
            "build": {"generate_s": t_gen, "build_s": t_build, "encode_upload_s": info["build_seconds"]},
        }
        if world == 1 and not args.no_cpu_baseline:
            x_np = x_cur[: L.m_local].cpu().numpy().astype(dtype_np)
            if args.config == "c5":
                line["cpu_baseline"] = cpu_baseline(csr, x_np)
            else:
                line["cpu_baseline"] = cpu_baseline(csr, x_np)
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()  # no rank frees its comm while a peer may still map it
    if fpit is not None:
        fpit.comm.free()
    A.free()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
