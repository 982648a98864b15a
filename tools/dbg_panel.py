"""Debug: panel-sliced BCCOO+ GPU results vs O1 on several shapes; prints where rows go wrong."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
from oracle import ref
from paper_conf_ppopp_yanlzz14_b200 import Matrix

def run(name, csr, **kw):
    x = synth.make_x(csr.n, np.float32, "uniform", 1)
    A = Matrix.from_synth(csr, device=0, **kw)
    y = A.spmv(torch.from_numpy(x).cuda()); torch.cuda.synchronize(); y = y.cpu().numpy()
    info = A.info(); A.free()
    yr, b = ref.spmv(csr.row_ptr, csr.col, csr.val, x)
    err = np.abs(y - yr) / np.maximum(b, 1e-30)
    bad = np.flatnonzero(err > 1e-5)
    R = kw.get("R", 16384)
    print(f"{name}: params={kw} KS={info['band_slices']} band={info['band_blocks']} far={info['nnzb']} bad={bad.size}/{csr.m}")
    if bad.size:
        print("   first bad rows", bad[:10], "panels", np.unique(bad // R)[:10], "local", (bad % R)[:10])
        print("   y", y[bad[:5]], "ref", yr[bad[:5]])
    sys.stdout.flush()

c = synth.circuit_like_rows(0, 400_000, n=400_000, band=8192, n_net=4, net_log2=(12, 16))
run("c5s R4096 W1024", c, B=8192, R=4096, W=1024, T=32, C=128, col_mode=2)
run("c5s R4096 W4096", c, B=8192, R=4096, W=4096, T=32, C=128, col_mode=2)
run("c5s R4096 W16384", c, B=8192, R=4096, W=16384, T=32, C=128, col_mode=2)
run("c5s R16384 W8192", c, B=8192, R=16384, W=8192, T=32, C=128, col_mode=2)
c2 = synth.circuit_like_rows(0, 400_000, n=400_000, band=8192, n_net=0, p_local=1.0)
run("c5s-nofar R4096 W1024", c2, B=8192, R=4096, W=1024)
run("c5s-nofar R4096 W4096", c2, B=8192, R=4096, W=4096)
c3 = synth.circuit_like_rows(0, 9_000, n=9_000, band=500, n_net=0, p_local=1.0)
run("allband", c3, B=20000, R=8192, W=4096)
run("allband W512", c3, B=2000, R=8192, W=512)
