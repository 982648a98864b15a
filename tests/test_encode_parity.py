"""The C++ encoder of libyaspmv (host-only handles, no GPU needed) against the independent
oracle encoder: every canonical array bit-identical.  CPU only."""
import itertools

import numpy as np
import pytest

import synth
from oracle import encode as E
from paper_conf_ppopp_yanlzz14_b200 import Matrix


def _compare(csr, h, w, S, T, C, cm, em):
    enc = E.encode(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, E.Params(h, w, S, T, C, cm, em))
    A = Matrix.from_csr(csr.m, csr.n, csr.row_ptr, csr.col, csr.val, device=-1,
                        h=h, w=w, S=S, T=T, C=C, col_mode=cm, empty_mode=em)
    try:
        info = A.info()
        p = info["params"]
        assert (p["col_mode"], p["empty_mode"]) == (enc.p.col_mode, enc.p.empty_mode)
        assert (info["nnzb"], info["nnzb_pad"], info["ntiles"], info["n_stops"], info["n_filler"]) == \
            (enc.nnzb, enc.nnzb_pad, enc.ntiles, enc.n_stops, enc.n_filler)
        assert (info["MB"], info["NB"], info["SW"]) == (enc.MB, enc.NB, enc.SW)
        assert np.array_equal(A.export("flags"), enc.flags)
        assert np.array_equal(A.export("col"), enc.col)
        if enc.p.col_mode == E.COL_DELTA:
            assert np.array_equal(A.export("col_delta"), enc.col_delta)
        for r in range(h):
            assert np.array_equal(A.export(f"val{r}").view(np.uint8), enc.val[r].view(np.uint8))
        assert np.array_equal(A.export("seg_row"), enc.seg_row)
        assert np.array_equal(A.export("zero_rows"), enc.zero_rows)
        assert np.array_equal(A.export("cta_seg0"), enc.cta_seg0)
        assert np.array_equal(A.export("fre"), enc.fre)
    finally:
        A.free()


@pytest.mark.parametrize("seed", range(24))
def test_tiny_random_grid(seed):
    a = synth.random_tiny(seed, dtype=np.float64 if seed % 2 else np.float32, integer=seed % 3 != 0)
    rng = np.random.default_rng(seed)
    combos = list(itertools.product([1, 2, 3, 4], [1, 2, 4, 8], [4, 8, 16, 32], [64, 128],
                                    [0, E.COL_I32, E.COL_DELTA], [E.EMPTY_FILLER, E.EMPTY_MAP, 0]))
    for i in rng.choice(len(combos), size=20, replace=False):
        h, w, T, C, cm, em = combos[i]
        NB = -(-a.n // w)
        for S in sorted({1, min(2, NB), NB}):
            _compare(a, h, w, S, T, C, cm, em)


def test_paper_example_A():
    A = np.array([[0, 0, 1, 0, 0, 0, 2, 3], [0, 0, 4, 5, 0, 0, 6, 0],
                  [0, 0, 0, 0, 7, 8, 9, 10], [11, 12, 0, 0, 13, 14, 15, 16]], dtype=np.float32)
    r, c = np.nonzero(A)
    rp = np.zeros(5, dtype=np.int64); np.cumsum(np.bincount(r, minlength=4), out=rp[1:])
    csr = synth.CSR(4, 8, rp, c.astype(np.int32), A[r, c])
    for S in (1, 2):
        _compare(csr, 2, 2, S, 4, 64, E.COL_I32, 0)


@pytest.mark.parametrize("name", ["c1", "c3-ship", "c4"])
def test_configs_full_size(name):
    csr = synth.config_matrix(name)
    params = {"c1": [(1, 1, 1, 16, 256, 0, 0), (1, 1, 1, 4, 64, 0, 0)],
              "c3-ship": [(2, 2, 1, 8, 128, 0, 0), (4, 4, 1, 4, 128, 0, 0)],
              "c4": [(1, 1, 1, 16, 256, 0, 0), (1, 1, 4, 8, 128, E.COL_DELTA, 0), (1, 1, 2, 16, 128, 0, E.EMPTY_MAP)]}[name]
    for p in params:
        _compare(csr, *p)


def test_coo_normalisation_matches_oracle():
    m, n = 40, 33
    r, c, v = synth.random_coo(5, m, n, 500)
    rp, col, val = E.normalize(m, n, r, c, v)
    enc = E.encode(m, n, rp, col, val, E.Params(2, 2, 2, 4, 64, E.COL_I32, 0))
    A = Matrix.from_coo(m, n, r, c, v, device=-1, h=2, w=2, S=2, T=4, C=64, col_mode=E.COL_I32)
    assert A.info()["nnz"] == col.size
    for r_ in range(2):
        assert np.array_equal(A.export(f"val{r_}"), enc.val[r_])
    assert np.array_equal(A.export("flags"), enc.flags)
    # unsorted CSR with duplicates goes through the same normalisation
    order = np.random.default_rng(1).permutation(r.size)
    rows = r[order]; cols = c[order]; vals = v[order]
    srt = np.argsort(rows, kind="stable")
    rp2 = np.zeros(m + 1, dtype=np.int64); np.cumsum(np.bincount(rows, minlength=m), out=rp2[1:])
    B = Matrix.from_csr(m, n, rp2, cols[srt], vals[srt], device=-1, h=2, w=2, S=2, T=4, C=64, col_mode=E.COL_I32)
    rpo, colo, valo = E.normalize(m, n, rows[srt], cols[srt], vals[srt])
    enc2 = E.encode(m, n, rpo, colo, valo, E.Params(2, 2, 2, 4, 64, E.COL_I32, 0))
    assert np.array_equal(B.export("val0"), enc2.val[0])



def test_delta_reset_per_thread_tile_cpp_encoder():
    """The C++ encoder resets the P:121 difference at every thread tile of T blocks (the
    rule pinned by tests/golden/p121_delta_reset.txt on the oracle): 512 rows of one block
    each, col = 100 + b, T = 4, C = 64 -> stored 100 + b at b % 4 == 0, else 1."""
    m = 512
    rp = np.arange(m + 1, dtype=np.int64)
    col = (100 + np.arange(m)).astype(np.int32)
    A = Matrix.from_csr(m, 1000, rp, col, np.ones(m, np.float32), device=-1, T=4, C=64,
                        col_mode=E.COL_DELTA, empty_mode=E.EMPTY_FILLER)
    try:
        want = np.where(np.arange(m) % 4 == 0, col, 1)
        assert np.array_equal(A.export("col_delta").astype(np.int64), want)
    finally:
        A.free()
