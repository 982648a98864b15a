"""Experiment: consecutive tiles per workgroup (params tiles_per_cta) on one encoding.
Not a benchmark of record: CUDA-event medians of back-to-back SpMVs per setting."""
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
    ap.add_argument("--params", default='{"T":32,"C":128,"col_mode":2}')
    ap.add_argument("--tpc", default="1,2,4,8,1")
    ap.add_argument("--rc", default="0")
    ap.add_argument("--iters", type=int, default=20)
    args = ap.parse_args()
    import torch

    import synth
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    csr = sm.circuit_like_rows(0, 50_000_000) if args.config == "c5" else synth.config_matrix(args.config)
    p = json.loads(args.params)
    p.setdefault("flags", 0)
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, **p)
    x = torch.from_numpy(synth.make_x(csr.n, csr.val.dtype, "uniform", 0)).cuda()
    y = torch.empty(csr.m, dtype=x.dtype, device="cuda")
    ref_y = None
    for rc in [int(v) for v in args.rc.split(",")]:
        for k in [int(v) for v in args.tpc.split(",")]:
            A.reencode(rc=rc if rc > 0 else -1, tpc=k)   # launch-time: no re-encode
            for _ in range(3):
                A.spmv(x, y)
            ts = []
            for _ in range(args.iters):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(); A.spmv(x, y); b.record()
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            yy = y.cpu().numpy()
            same = None
            if ref_y is None:
                ref_y = yy
            else:
                same = bool(np.array_equal(yy.view(np.uint32 if yy.dtype == np.float32 else np.uint64),
                                           ref_y.view(np.uint32 if yy.dtype == np.float32 else np.uint64)))
            print(json.dumps({"config": args.config, "tpc": k, "rc": rc, "ms": float(np.median(ts)),
                              "min_ms": float(np.min(ts)), "gflops": 2 * csr.nnz / float(np.median(ts)) / 1e6,
                              "bitwise_equal_to_first": same}), flush=True)
    A.free()


if __name__ == "__main__":
    main()
