"""Fig. 14 of the paper on B200: the contribution of each optimisation.

  COO          COO format (12 B/nnz) + tree-based segmented sum + carry kernel
  BCCOO        BCCOO bit flags + the same tree-based segmented sum + carry kernel
  seg-sum      BCCOO + matrix-based segmented sum (our kernel), carries by a 2nd kernel
  adj-sync     + adjacent synchronization (look-back) instead of the 2nd kernel
  fine-grain   + short column indices (u16 when NB < 65535) and the skipped workgroup scan
               (= the production yaspmv_spmv)

All on 1x1 blocks (the tree baselines are scalar), same T/C for the last three steps.
Each step is checked against the CPU oracle (per-row tolerance); times are CUDA-event
medians.  Writes one JSON line per (config, step) and, with --md, a table.
"""
import argparse
import ctypes
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def timed(fn, iters):
    import torch
    ts = []
    for _ in range(3):
        fn()
    for _ in range(iters):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return float(np.median(ts))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="c4,c3-ship,c2-f32,c5")
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--md", default=None)
    args = ap.parse_args()
    import torch

    import synth
    from oracle import ref
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import Matrix, _lib
    from paper_conf_ppopp_yanlzz14_b200._lib import check, lib
    rows_out = []
    for name in args.configs.split(","):
        csr = sm.circuit_like_rows(0, 50_000_000) if name == "c5" else synth.config_matrix(name)
        dt = csr.val.dtype
        dtc = _lib.F32 if dt == np.float32 else _lib.F64
        x_np = synth.make_x(csr.n, dt, "unit" if name in ("c4", "c5") else "uniform", 3)
        x = torch.from_numpy(x_np).cuda()
        y = torch.zeros(csr.m, dtype=x.dtype, device="cuda")
        sample = np.unique(np.linspace(0, csr.m - 1, 200_000).astype(np.int64))
        y_ref, bound = ref.spmv_rows(sample, csr.row_ptr, csr.col, csr.val, x_np)

        def ok():
            torch.cuda.synchronize()
            return ref.check_tolerance(y.cpu().numpy()[sample], y_ref, bound, dt)

        T, C = (32, 128) if name in ("c5", "c4") else (16, 256)
        res = {}
        # --- COO + tree
        rows_d = torch.from_numpy(np.repeat(np.arange(csr.m, dtype=np.int32), np.diff(csr.row_ptr))).cuda()
        col_d = torch.from_numpy(csr.col).cuda()
        val_d = torch.from_numpy(csr.val).cuda()
        sb = int(lib.yaspmv_ablation_tree_scratch_bytes(csr.nnz))
        scratch = torch.empty(sb, dtype=torch.uint8, device="cuda")
        st = torch.cuda.current_stream().cuda_stream
        coo = lambda: check(lib.yaspmv_ablation_tree(rows_d.data_ptr(), None, None, col_d.data_ptr(), val_d.data_ptr(),
                                                      csr.nnz, x.data_ptr(), y.data_ptr(), csr.m, dtc,
                                                      scratch.data_ptr(), sb, st))
        ms = timed(coo, args.iters)
        res["COO"] = (ms, ok(), 12 * csr.nnz + (4 + 4) * csr.m)
        del rows_d, col_d, val_d
        # --- BCCOO + tree (canonical arrays of a 1024-block tile encoding)
        A = Matrix.from_synth(csr, device=0, T=4, C=256, col_mode=2, flags=1)
        fl = torch.from_numpy(A.export("flags")).cuda()
        cb = torch.from_numpy(A.export("col")).cuda()
        vb = torch.from_numpy(A.export("val0")).cuda()
        cs = torch.from_numpy(A.export("cta_seg0")).cuda()
        nb = A.info()["nnzb_pad"]
        A.free()
        sb = int(lib.yaspmv_ablation_tree_scratch_bytes(nb))
        scratch = torch.empty(sb, dtype=torch.uint8, device="cuda")
        y.zero_()
        bt = lambda: check(lib.yaspmv_ablation_tree(None, fl.data_ptr(), cs.data_ptr(), cb.data_ptr(), vb.data_ptr(), nb,
                                                     x.data_ptr(), y.data_ptr(), csr.m, dtc, scratch.data_ptr(), sb, st))
        ms = timed(bt, args.iters)
        res["BCCOO"] = (ms, ok(), None)
        del fl, cb, vb, cs
        # --- our kernel: 2nd-kernel carries, look-back without skip, production
        A = Matrix.from_synth(csr, device=0, T=T, C=C, col_mode=2, flags=2 | 4)
        for v, key in ((1, "seg-sum"), (2, "adj-sync")):
            y.zero_()
            f = lambda v=v: check(lib.yaspmv_ablation_spmv(A._h, v, x.data_ptr(), y.data_ptr(), st))
            res[key] = (timed(f, args.iters), ok(), A.info()["alg_bytes"])
        A.free()
        A = Matrix.from_synth(csr, device=0, T=T, C=C, flags=2 | 4)
        y.zero_()
        res["fine-grain"] = (timed(lambda: A.spmv(x, y), args.iters), ok(), A.info()["alg_bytes"])
        colmode = A.info()["params"]["col_mode"]
        A.free()
        for k, (ms, (good, worst), ab) in res.items():
            r = {"config": name, "step": k, "ms": ms, "gflops": 2 * csr.nnz / ms / 1e6, "parity_ok": good,
                 "worst_err_over_tol": worst, "T": T, "C": C, "fine_col_mode": colmode, "nnz": csr.nnz}
            print(json.dumps(r), flush=True)
            rows_out.append(r)
        del csr
    if args.md:
        cfgs = list(dict.fromkeys(r["config"] for r in rows_out))
        steps = ["COO", "BCCOO", "seg-sum", "adj-sync", "fine-grain"]
        with open(args.md, "w") as f:
            f.write("| config | " + " | ".join(steps) + " | speedup fine-grain / COO |\n")
            f.write("|---|" + "---|" * (len(steps) + 1) + "\n")
            for c in cfgs:
                rr = {r["step"]: r for r in rows_out if r["config"] == c}
                cells = [f"{rr[s]['gflops']:.0f} GF ({rr[s]['ms']:.3f} ms){'' if rr[s]['parity_ok'] else ' FAIL'}" for s in steps]
                f.write(f"| {c} | " + " | ".join(cells) + f" | {rr['COO']['ms'] / rr['fine-grain']['ms']:.2f}x |\n")


if __name__ == "__main__":
    main()
