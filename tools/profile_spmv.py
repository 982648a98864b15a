"""Launch the SpMV of one config a few times (for ncu).  Not a benchmark: numbers printed
under a profiler are never bench values.

  python tools/profile_spmv.py --config c5 --params '{"T":16,"C":256}' --iters 3
"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--params", default="{}")
    ap.add_argument("--iters", type=int, default=3)
    ap.add_argument("--rows", type=int, default=0, help="C5: only the first ROWS rows")
    args = ap.parse_args()
    import torch

    import synth
    from synth import matrices as sm
    from paper_conf_ppopp_yanlzz14_b200 import Matrix
    if args.config == "c5":
        rows = args.rows or 50_000_000
        csr = sm.circuit_like_rows(0, rows)
        csr.n = 50_000_000
    else:
        csr = synth.config_matrix(args.config)
    p = json.loads(args.params)
    p.setdefault("flags", 2)
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=0, **p)
    x = torch.from_numpy(synth.make_x(csr.n, csr.val.dtype, "unit", 0)).cuda()
    y = torch.empty(csr.m, dtype=x.dtype, device="cuda")
    for _ in range(args.iters):
        A.spmv(x, y)
    torch.cuda.synchronize()
    info = A.info()
    print(json.dumps({"config": args.config, "params": info["params"], "alg_bytes": info["alg_bytes"],
                      "format_bytes": info["format_bytes"], "ntiles": info["ntiles"], "nnz": info["nnz"],
                      "regs": info["regs_per_thread"]}))


if __name__ == "__main__":
    main()
