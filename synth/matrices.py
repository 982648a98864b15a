"""Seeded synthetic sparse matrices and vectors (input generation only; see __init__).

Every generator returns a ``CSR`` with sorted, distinct column indices per row
(explicit zeros allowed) and int64 row pointers / int32 column indices, which is the
layout both the oracle and the C-ABI build call accept.

Shapes follow BASELINE.json ``configs`` and the paper's Table 2:
  C1  2-D 5-point Laplacian 64x64 (4,096 rows, 20,224 nnz)            fp64
  C2  Dense 2,000 x 2,000, every entry stored                   fp32 / fp64
  C3  FEM node-block matrices shaped like Spheres / Cantilever / Ship    fp32 (+fp64)
      
  C4  power-law webbase-like 1M x 1M, ~3.1M nnz, 2% empty rows  fp32
  C5  circuit/LP-like 50M x 50M, ~1.0B nnz (Circuit5M scaled)     fp32
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

SEED = 20140215
_HERE = os.path.dirname(os.path.abspath(__file__))


@dataclass
class CSR:
    m: int
    n: int
    row_ptr: np.ndarray  # int64, m+1
    col: np.ndarray      # int32, nnz
    val: np.ndarray      # float32 / float64, nnz

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    @property
    def dtype(self):
        return self.val.dtype

    def astype(self, dtype) -> "CSR":
        return CSR(self.m, self.n, self.row_ptr, self.col, self.val.astype(dtype))

    def to_dense(self) -> np.ndarray:
        d = np.zeros((self.m, self.n), dtype=self.val.dtype)
        rows = np.repeat(np.arange(self.m), np.diff(self.row_ptr))
        d[rows, self.col] = self.val
        return d

    def row_slice(self, r0: int, r1: int) -> "CSR":
        a, b = int(self.row_ptr[r0]), int(self.row_ptr[r1])
        return CSR(r1 - r0, self.n, self.row_ptr[r0:r1 + 1] - a, self.col[a:b], self.val[a:b])


def _rng(config_id: int, block: int = 0) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(np.random.SeedSequence([SEED, config_id, block])))


def _from_keys(m: int, n: int, rows: np.ndarray, cols: np.ndarray) -> tuple[np.ndarray, np.ndarray]:
    """Unique (row, col) pairs in row-major order -> (row_ptr, col)."""
    key = np.unique(rows.astype(np.int64) * n + cols.astype(np.int64))
    r = key // n
    c = (key % n).astype(np.int32)
    row_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=m), out=row_ptr[1:])
    return row_ptr, c


# --------------------------------------------------------------------------- C1
def laplacian_2d(g: int = 64, dtype=np.float64) -> CSR:
    """2-D 5-point Laplacian on a g x g grid, Dirichlet boundary, natural row-major
    ordering: diag 4, neighbours -1.  g=64 -> 4,096 rows, 20,224 nnz."""
    m = g * g
    i = np.arange(m)
    r, c = i // g, i % g
    rows, cols = [], []
    for dr, dc in ((-1, 0), (0, -1), (0, 0), (0, 1), (1, 0)):
        ok = (r + dr >= 0) & (r + dr < g) & (c + dc >= 0) & (c + dc < g)
        rows.append(i[ok])
        cols.append((i + dr * g + dc)[ok])
    rp, cl = _from_keys(m, m, np.concatenate(rows), np.concatenate(cols))
    rr = np.repeat(np.arange(m), np.diff(rp))
    val = np.where(rr == cl, 4.0, -1.0).astype(dtype)
    return CSR(m, m, rp, cl, val)


# --------------------------------------------------------------------------- C2
def dense(n: int = 2000, dtype=np.float32, integer: bool = False) -> CSR:
    """n x n with every entry stored (Table 2 'Dense').  Values U[-1,1), or
    integers in {-2..2} (zeros kept as structural entries)."""
    g = _rng(2)
    if integer:
        v = g.integers(-2, 3, size=n * n).astype(dtype)
    else:
        v = g.uniform(-1.0, 1.0, size=n * n).astype(dtype)
    rp = np.arange(0, n * n + 1, n, dtype=np.int64)
    cl = np.tile(np.arange(n, dtype=np.int32), n)
    return CSR(n, n, rp, cl, v)


# --------------------------------------------------------------------------- C3
FEM_SHAPES = {
    # name: (rows, node block b, node blocks per node row k)   -> nnz/row = b*k
    "spheres": (83336, 4, 18),      # P:330  6,010,480 nnz, 72/row
    "cantilever": (62452, 4, 16),   # P:331  4,007,383 nnz, ~64/row
    "ship": (141000, 2, 28),        # P:335  7,813,404 nnz, ~56/row (Q16)
}


def fem_like(kind: str = "spheres", dtype=np.float32, integer: bool = False) -> CSR:
    """FEM-like node-block matrix: n_nodes = rows/b node rows; node row u couples to
    itself and k-1 distinct neighbour nodes u+off, off uniform in +-ceil(n_nodes^(2/3))
    (resampled at the edges); each coupling is a dense b x b block.  Values U[-1,1)
    with the diagonal made dominant (1 + sum |off-diagonal|), or small integers."""
    m, b, k = FEM_SHAPES[kind]
    cid = {"spheres": 31, "cantilever": 32, "ship": 33}[kind]
    g = _rng(cid)
    nn = m // b
    d = int(np.ceil(nn ** (2.0 / 3.0)))
    nbr = np.empty((nn, k), dtype=np.int64)
    nbr[:, 0] = np.arange(nn)
    cand = g.integers(-d, d + 1, size=(nn, 4 * k))
    for u in range(nn):
        v = u + cand[u]
        v = v[(v >= 0) & (v < nn) & (v != u)]
        _, first = np.unique(v, return_index=True)
        v = v[np.sort(first)][: k - 1]
        while v.size < k - 1:  # rare: resample
            extra = u + g.integers(-d, d + 1, size=4 * k)
            v = np.concatenate([v, extra[(extra >= 0) & (extra < nn) & (extra != u)]])
            _, first = np.unique(v, return_index=True)
            v = v[np.sort(first)][: k - 1]
        nbr[u, 1:] = v
    nbr.sort(axis=1)
    # expand node couplings into scalar entries
    rows = (np.arange(nn)[:, None, None, None] * b + np.arange(b)[None, None, :, None])
    cols = (nbr[:, :, None, None] * b + np.arange(b)[None, None, None, :])
    rows = np.broadcast_to(rows, (nn, k, b, b)).transpose(0, 2, 1, 3).reshape(-1)
    cols = np.broadcast_to(cols, (nn, k, b, b)).transpose(0, 2, 1, 3).reshape(-1)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(rows, minlength=m), out=rp[1:])
    cl = cols.astype(np.int32)
    if integer:
        val = g.integers(-2, 3, size=cl.size).astype(dtype)
    else:
        v = g.uniform(-1.0, 1.0, size=cl.size)
        rr = rows
        diag = rr == cols
        off = np.where(diag, 0.0, np.abs(v))
        rs = np.bincount(rr, weights=off, minlength=m)
        v[diag] = 1.0 + rs[rr[diag]]
        val = v.astype(dtype)
    return CSR(m, m, rp, cl, val)


# --------------------------------------------------------------------------- C4
def webbase_like(m: int = 1_000_000, dtype=np.float32, alpha: float = 2.1, lmax: int = 5000,
                 empty_frac: float = 0.02, integer: bool = False) -> CSR:
    """Power-law web-graph-like matrix (Webbase: 1M^2, 3.1M nnz, 3/row).
    Row lengths P(L=k) ~ k^-alpha on [1, lmax] with empty_frac of rows empty; columns
    60% local (i +- geometric offset, |off| <= 1024), 40% 'popular' (Zipf 1.2 over a
    fixed random column permutation); duplicates merged.  Values 1/L_i (row-stochastic)
    or small integers."""
    g = _rng(4)
    ks = np.arange(1, lmax + 1, dtype=np.float64)
    p = ks ** (-alpha)
    p /= p.sum()
    L = g.choice(np.arange(1, lmax + 1), size=m, p=p)
    L[g.random(m) < empty_frac] = 0
    rows = np.repeat(np.arange(m, dtype=np.int64), L)
    t = rows.size
    local = g.random(t) < 0.6
    off = np.minimum(g.geometric(1.0 / 32.0, size=t), 1024) * np.where(g.random(t) < 0.5, -1, 1)
    c_loc = rows + off
    c_loc = np.where(c_loc < 0, -c_loc, c_loc)
    c_loc = np.where(c_loc >= m, 2 * (m - 1) - c_loc, c_loc)
    perm = g.permutation(m)
    z = g.zipf(1.2, size=t)
    c_pop = perm[(z - 1) % m]
    cols = np.where(local, c_loc, c_pop)
    rp, cl = _from_keys(m, m, rows, cols)
    lens = np.diff(rp)
    rr = np.repeat(np.arange(m), lens)
    if integer:
        val = g.integers(-2, 3, size=cl.size).astype(dtype)
    else:
        val = (1.0 / lens[rr]).astype(dtype)
    return CSR(m, m, rp, cl, val)


# --------------------------------------------------------------------------- C5
class _C5Params(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("lam", ctypes.c_double), ("p_local", ctypes.c_double),
                ("band", ctypes.c_int64), ("n_net", ctypes.c_int32), ("net_lo_log2", ctypes.c_int32),
                ("net_hi_log2", ctypes.c_int32), ("seed", ctypes.c_uint64)]


_LIB = None


def _lib():
    global _LIB
    if _LIB is None:
        so = os.path.join(_HERE, "libsynth.so")
        src = os.path.join(_HERE, "c5gen.c")
        if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
            subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fopenmp", "-fPIC", "-shared",
                                   "-o", so, src, "-lm"])
        _LIB = ctypes.CDLL(so)
        for f in (_LIB.c5_count, _LIB.c5_fill, _LIB.c5_net_rows):
            f.restype = ctypes.c_int
    return _LIB


def c5_params(n: int = 50_000_000, n_net: int = 32, net_log2=(16, 21), lam: float = 18.6,
              p_local: float = 0.85, band: int = 65536) -> _C5Params:
    return _C5Params(n, lam, p_local, band, n_net, net_log2[0], net_log2[1],
                     (SEED * 1000003 + 5) & 0xFFFFFFFFFFFFFFFF)


def circuit_like_rows(r0: int, r1: int, dtype=np.float32, kind: str = "positive", **kw) -> CSR:
    """Rows [r0, r1) of the C5 matrix (all N columns).  The structure of each row is a
    function of (seed, row) only, so any row block is the same for every rank count."""
    P = c5_params(**kw)
    lib = _lib()
    m = r1 - r0
    counts = np.empty(m, dtype=np.int64)
    rc = lib.c5_count(ctypes.byref(P), ctypes.c_int64(r0), ctypes.c_int64(r1),
                      counts.ctypes.data_as(ctypes.c_void_p))
    if rc != 0:
        raise RuntimeError(f"c5_count failed ({rc})")
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    nnz = int(rp[-1])
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=dtype)
    kid = {"positive": 0, "signed": 1, "integer": 2}[kind]
    rc = lib.c5_fill(ctypes.byref(P), ctypes.c_int64(r0), ctypes.c_int64(r1),
                     rp.ctypes.data_as(ctypes.c_void_p), col.ctypes.data_as(ctypes.c_void_p),
                     val.ctypes.data_as(ctypes.c_void_p), 0 if np.dtype(dtype) == np.float32 else 1, kid)
    if rc != 0:
        raise RuntimeError(f"c5_fill failed ({rc})")
    return CSR(m, P.n, rp, col, val)


def circuit_like(dtype=np.float32, kind: str = "positive", **kw) -> CSR:
    n = kw.get("n", 50_000_000)
    return circuit_like_rows(0, n, dtype=dtype, kind=kind, **kw)


def c5_net_rows(**kw):
    P = c5_params(**kw)
    pos = np.zeros(64, dtype=np.int64)
    ln = np.zeros(64, dtype=np.int64)
    _lib().c5_net_rows(ctypes.byref(P), pos.ctypes.data_as(ctypes.c_void_p), ln.ctypes.data_as(ctypes.c_void_p))
    return pos[:P.n_net].copy(), ln[:P.n_net].copy()


# --------------------------------------------------------------------------- tiny / COO
def random_tiny(seed: int, m: int | None = None, n: int | None = None, density: float | None = None,
                dtype=np.float64, integer: bool = True, force_empty: bool = True) -> CSR:
    """Small random matrix (m, n <= 24) for brute-force property tests; some rows and
    columns forced empty; integer values in {-3..3} (zeros kept structural)."""
    g = _rng(900, seed)
    m = int(g.integers(1, 25)) if m is None else m
    n = int(g.integers(1, 25)) if n is None else n
    density = float(g.uniform(0.0, 0.7)) if density is None else density
    mask = g.random((m, n)) < density
    if force_empty and m > 1:
        mask[g.integers(0, m, size=max(1, m // 5))] = False
    if force_empty and n > 1:
        mask[:, g.integers(0, n, size=max(1, n // 5))] = False
    rows, cols = np.nonzero(mask)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(rows, minlength=m), out=rp[1:])
    if integer:
        val = g.integers(-3, 4, size=rows.size).astype(dtype)
    else:
        val = g.uniform(-1, 1, size=rows.size).astype(dtype)
    return CSR(m, n, rp, cols.astype(np.int32), val)


def random_coo(seed: int, m: int, n: int, nnz: int, dtype=np.float64):
    """Unsorted COO triples WITH duplicates (for the input-normalisation step)."""
    g = _rng(901, seed)
    r = g.integers(0, m, size=nnz).astype(np.int32)
    c = g.integers(0, n, size=nnz).astype(np.int32)
    v = g.integers(-3, 4, size=nnz).astype(dtype)
    return r, c, v


# --------------------------------------------------------------------------- vectors
def make_x(n: int, dtype=np.float32, kind: str = "uniform", seed: int = 0) -> np.ndarray:
    g = _rng(700, seed)
    if kind == "uniform":
        return g.uniform(-1.0, 1.0, size=n).astype(dtype)
    if kind == "unit":
        return g.random(n).astype(dtype)
    if kind == "int":
        return g.integers(-4, 5, size=n).astype(dtype)
    if kind == "int2":
        return g.integers(-2, 3, size=n).astype(dtype)
    if kind == "const":
        return np.full(n, 1.0 / np.sqrt(n), dtype=dtype)
    raise ValueError(kind)


# --------------------------------------------------------------------------- configs
CONFIGS = {
    # name: (BASELINE.json configs index, description)
    "c1": (0, "2D 5-point Laplacian 64x64, fp64"),
    "c2-f32": (1, "Dense 2000x2000, fp32"),
    "c2-f64": (1, "Dense 2000x2000, fp64"),
    "c3-spheres": (2, "FEM Spheres-like 83,336 rows, fp32"),
    "c3-cantilever": (2, "FEM Cantilever-like 62,452 rows, fp32"),
    "c3-ship": (2, "FEM Ship-like 141,000 rows, fp32"),
    "c3-ship-f64": (2, "FEM Ship-like 141,000 rows, fp64"),
    "c4": (3, "power-law webbase-like 1M rows, fp32"),
    "c5": (4, "circuit/LP-like 50M rows ~1.0B nnz, fp32"),
}


def config_matrix(name: str, integer: bool = False) -> CSR:
    if name == "c1":
        return laplacian_2d(64, np.float64)
    if name == "c2-f32":
        return dense(2000, np.float32, integer)
    if name == "c2-f64":
        return dense(2000, np.float64, integer)
    if name.startswith("c3-"):
        kind = name.split("-")[1]
        dt = np.float64 if name.endswith("f64") else np.float32
        return fem_like(kind, dt, integer)
    if name == "c4":
        return webbase_like(dtype=np.float32, integer=integer)
    if name == "c5":
        return circuit_like(np.float32, "integer" if integer else "positive")
    raise ValueError(name)
