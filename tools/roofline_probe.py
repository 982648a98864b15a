"""Roofline probes for the SpMV kernel K1: how much of K1's time any kernel
that reads this format and gathers x must spend.

For one configuration, on the same encoded matrix and the same launch configuration:
  full          yaspmv_spmv (K1: loads, gathers, segmented sum, scan, carries, stores)
  stream+gather ablation variant 4: K1's loads and x gathers only
  stream+L2-gather ablation variant 6: gathers confined to an L2-resident 4 MB window of x
  stream        ablation variant 5: K1's loads only (gathers redirected to L1-resident x[0..15])
CUDA-event medians over back-to-back launches; C5 (8.5 GB) is far larger than L2, so
every launch streams the matrix from HBM.  One JSON line per probe (+ --md table).
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--iters", type=int, default=30)
    ap.add_argument("--params", default=None)
    ap.add_argument("--md", default=None)
    ap.add_argument("--sweep", nargs="*", default=None, help="JSON param overrides, one re-encode each")
    ap.add_argument("--ncu", action="store_true", help="launch every probe exactly twice, untimed (run under ncu; "
                    "launch order = probe order)")
    args = ap.parse_args()
    import torch

    import synth
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    from paper_conf_ppopp_yanlzz14_b200._lib import check, lib
    sys.path.insert(0, ROOT)
    from bench import DEFAULT_PARAMS, measured_peaks

    csr = sm.circuit_like_rows(0, 50_000_000) if args.config == "c5" else synth.config_matrix(args.config)
    params = dict(DEFAULT_PARAMS.get(args.config, {}))
    if args.params:
        params.update(json.loads(args.params))
    sweep = [json.loads(p) for p in args.sweep] if args.sweep else [{}]
    if csr.nnz > 50_000_000:
        params.setdefault("flags", 4 if len(sweep) > 1 else 2 | 4)
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, **params)
    nnz = csr.nnz
    del csr
    for sw in sweep:
        if sw:
            A.reencode(**sw)
        _probe(A, nnz, args)
    A.free()


def _probe(A, nnz, args):
    import torch
    from paper_conf_ppopp_yanlzz14_b200._lib import check, lib
    from bench import measured_peaks
    info = A.info()
    x = torch.full((info["n"],), 1.0 / np.sqrt(info["n"]), dtype=torch.float32 if A.dtype == np.float32
                   else torch.float64, device="cuda")
    y = torch.zeros(info["m"], dtype=x.dtype, device="cuda")
    st = torch.cuda.current_stream().cuda_stream
    peak, kind = measured_peaks()

    def run(variant):
        if variant == 0:
            A.spmv(x, y)
        else:
            check(lib.yaspmv_ablation_spmv(A._h, variant, x.data_ptr(), y.data_ptr(), st))

    out = []
    probes = [("full", 0), ("no carries (7)", 7), ("7 - y stores (9)", 9),
              ("up to the scan (8)", 8), ("8 + status store (10)", 10), ("8 + C stores (11)", 11),
              ("stream+gather", 4),
              ("stream+L2-gather", 6), ("stream", 5), ("full (again)", 0)]
    for name, v in probes:
        if v == 6 and info["n"] < (1 << 20) * info["params"]["block_w"]:
            continue
        if args.ncu:
            for _ in range(2):
                run(v)
            torch.cuda.synchronize()
            print(json.dumps({"probe": name, "variant": v, "launches": 2}), flush=True)
            continue
        for _ in range(3):
            run(v)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.iters)]
        for a, b in ev:
            a.record()
            run(v)
            b.record()
        torch.cuda.synchronize()
        ms = float(np.median([a.elapsed_time(b) for a, b in ev]))
        fmt_bytes = info["format_bytes"] + info["m"] * x.element_size()
        line = {"config": args.config, "probe": name, "ms": ms, "gflops_equiv": 2.0 * nnz / (ms * 1e-3) / 1e9,
                "alg_gbs": info["alg_bytes"] / (ms * 1e-3) / 1e9, "alg_frac": info["alg_bytes"] / (ms * 1e-3) / 1e9 / peak,
                "format_gbs": fmt_bytes / (ms * 1e-3) / 1e9, "peak_gbs": peak, "peak_kind": kind,
                "params": info["params"]}
        out.append(line)
        print(json.dumps(line), flush=True)
    if args.md:
        with open(args.md, "a") as f:
            f.write(f"# K1 roofline probes — {args.config} ({nnz:,} nnz), params {info['params']}\n\n")
            f.write("| probe | ms | GFLOPS-equiv | algorithmic GB/s | frac of measured HBM |\n|---|---|---|---|---|\n")
            for r in out:
                f.write(f"| {r['probe']} | {r['ms']:.3f} | {r['gflops_equiv']:.0f} | {r['alg_gbs']:.0f} | "
                        f"{r['alg_frac']:.3f} |\n")
            f.write("\n")


if __name__ == "__main__":
    main()
