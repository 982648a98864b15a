import itertools, sys, os
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth
from oracle import encode as E
from paper_conf_ppopp_yanlzz14_b200 import Matrix
seed = 0
rng = np.random.default_rng(seed)
dt = np.float32
m, n = int(rng.integers(1, 2500)), int(rng.integers(1, 2500))
a = synth.random_tiny(seed, m=m, n=n, density=float(rng.uniform(0.001, 0.05)), dtype=dt, integer=True)
combos = list(itertools.product([1, 2, 3, 4], [1, 2, 4], [4, 8, 16, 32], [64, 128, 256],
                                [0, E.COL_I32, E.COL_DELTA], [E.EMPTY_FILLER, E.EMPTY_MAP]))
for i in rng.choice(len(combos), size=6, replace=False):
    h, w, T, C, cm, em = combos[i]
    NB = -(-a.n // w)
    for S in sorted({1, min(3, NB)}):
        try:
            A = Matrix.from_synth(a, device=0, h=h, w=w, S=S, T=T, C=C, col_mode=cm, empty_mode=em, flags=4)
        except Exception as ex:
            print("skip", h, w, T, C, S, ex); continue
        enc = E.encode(a.m, a.n, a.row_ptr, a.col, a.val, E.Params(h, w, S, T, C, cm, em))
        for r in range(h):
            g = A.export(f"val{r}", device=True); o = enc.val[r]
            bad = np.flatnonzero(g != o)
            print(f"m={a.m} n={a.n} h={h} w={w} T={T} C={C} S={S} cm={cm} em={em} r={r} bad={bad.size}", bad[:8], g[bad[:8]], o[bad[:8]])
        A.free()
