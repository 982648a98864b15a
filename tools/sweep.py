"""Time the SpMV over a list of parameter sets on one config (CUDA events, warm-up 3,
median of K).  Exploration tool; bench.py is the measurement of record."""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--sets", required=True, help="JSON list of param dicts")
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--flush", action="store_true", help="write 2x L2 between launches")
    ap.add_argument("--persist", type=int, default=-1, help="cudaLimitPersistingL2CacheSize in MB (-1: leave)")
    ap.add_argument("--power", action="store_true", help="time yaspmv_spmv_power (fused epilogue)")
    ap.add_argument("--l2fetch", type=int, default=0, help="cudaLimitMaxL2FetchGranularity (32/64/128), 0 = leave")
    args = ap.parse_args()
    import torch

    import synth
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    if args.persist >= 0:
        import ctypes
        torch.cuda.init(); torch.zeros(1, device="cuda")
        rt = ctypes.CDLL(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                      "libcudart.so.12"))
        mx = ctypes.c_int()
        rt.cudaDeviceGetAttribute(ctypes.byref(mx), 108, 0)  # cudaDevAttrMaxPersistingL2CacheSize
        want = min(mx.value, args.persist << 20)
        rc = rt.cudaDeviceSetLimit(0x06, ctypes.c_size_t(want))
        got = ctypes.c_size_t()
        rt.cudaDeviceGetLimit(ctypes.byref(got), 0x06)
        print(f"# persisting L2: max {mx.value >> 20} MB, set {want >> 20} MB rc={rc} now {got.value >> 20} MB", flush=True)
    if args.l2fetch:
        import ctypes
        torch.zeros(1, device="cuda")
        rt = ctypes.CDLL(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                      "libcudart.so.12"))
        cur = ctypes.c_size_t()
        rt.cudaDeviceGetLimit(ctypes.byref(cur), 0x05)
        rc = rt.cudaDeviceSetLimit(0x05, ctypes.c_size_t(args.l2fetch))
        now = ctypes.c_size_t()
        rt.cudaDeviceGetLimit(ctypes.byref(now), 0x05)
        print(f"# L2 fetch granularity: was {cur.value}, set {args.l2fetch} rc={rc}, now {now.value}", flush=True)
    t0 = time.time()
    csr = sm.circuit_like_rows(0, 50_000_000) if args.config == "c5" else synth.config_matrix(args.config)
    print(f"# generated {args.config} nnz={csr.nnz} in {time.time()-t0:.1f}s", flush=True)
    x = torch.from_numpy(synth.make_x(csr.n, csr.val.dtype, "unit", 0)).cuda()
    y = torch.empty(csr.m, dtype=x.dtype, device="cuda")
    scratch = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for p in json.loads(args.sets):
        p = dict(p)
        p.setdefault("flags", 2)
        try:
            t1 = time.time()
            A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, **p)
            tb = time.time() - t1
        except Exception as e:
            print(json.dumps({"params": p, "error": str(e)}), flush=True)
            continue
        n2a = torch.ones(1, dtype=torch.float64, device="cuda")
        n2b = torch.zeros(1, dtype=torch.float64, device="cuda")
        call = (lambda: A.spmv_power(x, y, n2a, n2b)) if args.power else (lambda: A.spmv(x, y))
        for _ in range(3):
            call()
        ts = []
        A.profile_begin()
        for _ in range(args.iters):
            if args.flush:
                scratch.zero_()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); call(); b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        prof = A.profile_end()
        info = A.info()
        ms = float(np.median(ts))
        kern = {k: v / max(prof.get("calls", 1), 1) for k, v in prof.items() if k.endswith("_ms")}
        print(json.dumps({"params": {k: v for k, v in info["params"].items() if k != "flags"}, "ms": ms,
                          "min_ms": float(np.min(ts)), "alg_GBs": info["alg_bytes"] / ms / 1e6,
                          "gflops": 2 * info["nnz"] / ms / 1e6, "regs": info["regs_per_thread"],
                          "alg_bytes": info["alg_bytes"], "build_s": tb, "kern_ms": kern}), flush=True)
        A.free()


if __name__ == "__main__":
    main()
