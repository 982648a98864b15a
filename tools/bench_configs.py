"""Per-config SpMV measurements (BASELINE.json configs C1-C4; C5 is bench.py's workload):
auto-tuned parameters (yaspmv_tune, §4), SpMV time warm (L2-resident, back-to-back) and
cold (a 2x-L2 scratch write between launches), GFLOPS, algorithmic GB/s and fraction of
the measured HBM peak, parity against the oracle, and the oracle's own CPU time.
One JSON line per config; --md writes a markdown table.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CONFIGS = ["c1", "c2-f32", "c2-f64", "c3-spheres", "c3-cantilever", "c3-ship", "c3-ship-f64", "c4"]


def timed(fn, iters, flush=None):
    import torch
    ts = []
    for _ in range(iters):
        if flush is not None:
            flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return float(np.median(ts))


def timed_b2b(fn, n=100):
    """Steady-state time per launch of n back-to-back launches (one event pair)."""
    import torch
    for _ in range(5):
        fn()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default=",".join(CONFIGS))
    ap.add_argument("--iters", type=int, default=50)
    ap.add_argument("--md", default=None)
    ap.add_argument("--exhaustive", action="store_true", help="also run the exhaustive search (P:322)")
    ap.add_argument("--from-jsonl", default=None, help="only rewrite --md from a previous run's JSON lines")
    args = ap.parse_args()
    if args.from_jsonl:
        write_md([json.loads(l) for l in open(args.from_jsonl) if l.startswith("{")], args.md)
        return
    import torch

    import synth
    from oracle import ref
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    flush = torch.empty(2 * l2, dtype=torch.uint8, device="cuda")
    rows = []
    for name in args.configs.split(","):
        csr = synth.config_matrix(name)
        dt = csr.val.dtype
        x_np = synth.make_x(csr.n, dt, "unit" if name == "c4" else "uniform", 3)
        x = torch.from_numpy(x_np).cuda()
        y = torch.empty(csr.m, dtype=x.dtype, device="cuda")
        y_ref, bound = ref.spmv(csr.row_ptr, csr.col, csr.val, x_np)
        t0 = time.perf_counter()
        ref.spmv(csr.row_ptr, csr.col, csr.val, x_np, with_bound=False)
        t_cpu = time.perf_counter() - t0
        A = Matrix.from_synth(csr, device=0)
        ex = None
        if args.exhaustive:  # the paper's tuned-vs-exhaustive comparison
            A.tune(exhaustive=True)
            for _ in range(5):
                A.spmv(x, y)
            ex = {"params": A.info()["params"], "ms_warm": timed(lambda: A.spmv(x, y), args.iters),
                  "tune_s": A.info()["tune_seconds"]}
        chosen = A.tune()
        info = A.info()
        for _ in range(5):
            A.spmv(x, y)
        warm = timed(lambda: A.spmv(x, y), args.iters)
        cold = timed(lambda: A.spmv(x, y), max(10, args.iters // 5), flush)
        b2b = timed_b2b(lambda: A.spmv(x, y))
        ok, worst = ref.check_tolerance(y.cpu().numpy(), y_ref, bound, dt)
        # the same tuned parameters launched without programmatic dependent launch
        q = {k: v for k, v in chosen.items()}
        B = Matrix.from_synth(csr, device=0, h=q["block_h"], w=q["block_w"], S=q["slices"], T=q["thread_tile"],
                              C=q["cta_size"], col_mode=q["col_mode"], empty_mode=q["empty_mode"],
                              rc=q.get("result_cache", 0), flags=16)
        b2b_nopdl = timed_b2b(lambda: B.spmv(x, y))
        B.free()
        r = {"config": name, "m": csr.m, "nnz": csr.nnz, "dtype": str(dt), "params": chosen,
             "tune_s": info["tune_seconds"], "tune_candidates": info["tune_candidates"],
             "ms_warm": warm, "ms_cold": cold, "ms_b2b": b2b, "ms_b2b_no_pdl": b2b_nopdl,
             "gflops_warm": 2 * csr.nnz / warm / 1e6, "gflops_cold": 2 * csr.nnz / cold / 1e6,
             "alg_bytes": info["alg_bytes"], "alg_GBs_cold": info["alg_bytes"] / cold / 1e6,
             "frac_of_measured_hbm_cold": info["alg_bytes"] / cold / 1e6 / peak,
             "footprint_MB": info["footprint_bytes"] / 1e6, "parity_ok": ok, "worst_err_over_tol": worst,
             "oracle_cpu_ms": t_cpu * 1e3, "oracle_threads": ref.num_threads(), "exhaustive": ex}
        print(json.dumps(r), flush=True)
        rows.append(r)
        A.free()
    if args.md:
        write_md(rows, args.md)



def write_md(rows, path):
    with open(path, "w") as f:
        f.write("| config | nnz | dtype | tuned (h,w,T,C,S,col,rc) | tune s | warm ms | cold ms | back-to-back ms (no PDL) | GFLOPS (cold) | alg GB/s (cold) | frac of measured HBM | parity (worst err/tol) | oracle CPU ms |\n")
        f.write("|---|---|---|---|---|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            p = r["params"]
            f.write(f"| {r['config']} | {r['nnz']:,} | {r['dtype']} | {p['block_h']}x{p['block_w']}, T={p['thread_tile']}, "
                    f"C={p['cta_size']}, S={p['slices']}, col={p['col_mode']}, rc={p.get('result_cache', 0)} | {r['tune_s']:.1f} | {r['ms_warm']:.4f} | "
                    f"{r['ms_cold']:.4f} | {r['ms_b2b']:.4f} ({r['ms_b2b_no_pdl']:.4f}) | {r['gflops_cold']:.1f} | {r['alg_GBs_cold']:.0f} | {r['frac_of_measured_hbm_cold']:.3f} | "
                    f"{'ok' if r['parity_ok'] else 'FAIL'} ({r['worst_err_over_tol']:.2g}) | {r['oracle_cpu_ms']:.2f} |\n")
        if any(r["exhaustive"] for r in rows):
            f.write("\n### tuned (4 smallest-footprint shapes, P:321) vs exhaustive over all compiled shapes (P:322)\n\n")
            f.write("| config | tuned params | tuned warm ms | exhaustive params | exhaustive warm ms | exhaustive tune s | tuned/exhaustive time |\n|---|---|---|---|---|---|---|\n")
            for r in rows:
                e = r["exhaustive"]
                if not e:
                    continue
                p, q = r["params"], e["params"]
                f.write(f"| {r['config']} | {p['block_h']}x{p['block_w']} T={p['thread_tile']} C={p['cta_size']} | {r['ms_warm']:.4f} | "
                        f"{q['block_h']}x{q['block_w']} T={q['thread_tile']} C={q['cta_size']} | {e['ms_warm']:.4f} | {e['tune_s']:.1f} | {r['ms_warm'] / e['ms_warm']:.3f} |\n")


if __name__ == "__main__":
    main()
