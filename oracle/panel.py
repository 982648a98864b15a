"""O2-P / O3-P — the panel-sliced BCCOO+ encoding and its decode-and-multiply
(TEST INFRASTRUCTURE ONLY, see oracle/__init__).

BCCOO+ (§2.3) cuts the matrix into vertical slices and stacks them
top-down so that every row of a slice uses the same part of the multiplied vector
("Different rows in the same vertical slice ... will all use y[0] ~ y[3]"); its cost
is the temporary buffer of per-slice results and the combine kernel.  The panel
variant applies that stacking to each horizontal panel of R rows separately, with slices
of W columns placed relative to the panel (readings P1-P6):

  P1  panel p = rows [p*R, (p+1)*R);  column base cb(p) = p*R + diag0 - B
  P2  slice k (0 <= k < KS, KS = ceil((R + 2B) / W)) of panel p = columns
      [cb(p) + k*W, cb(p) + (k+1)*W); entry (i, j) of panel p is a BAND entry iff
      0 <= j - cb(p) < KS*W, else a FAR entry
  P3  band entries ordered by (p, k, i, j): the slices of a panel stacked top-down (the
      BCCOO+ rearrangement of P:150 inside the panel), every slice in BCCOO order (Fig. 2)
  P4  bit flag 0 = last entry of row i inside slice (p, k); each slice (p, k) padded
      with '1' bits to a multiple of the workgroup tile T*C (pad entries: value 0
      and the stored column of the slice's last entry, as Q3 reads P:119 for plain BCCOO),
      so that no workgroup tile holds two slices; empty slices hold no blocks
  P5  column stored as the unsigned short offset j - cb(p) - k*W  (< W < 65535; the short
      column type of P:121/P:302 with a per-slice base, the original column = base +
      offset as P:150 requires)
  P6  inside slice (p, k), every row between the slice's first and last non-empty rows
      holds at least one block: an empty row there gets one FILLER block (value 0, column
      offset W, where the window of x reads 0) — the paper's "multiple 1s" for a row
      difference larger than 1 (reading Q1/R1) — so the s-th row stop of the
      slice is row first_row(p, k) + s; aux: first_row per slice, stops per slice and,
      per workgroup tile, the stops before it inside its slice (the first-result entry
      of P:188-189, like cta_seg0)
  far entries: a plain BCCOO matrix of the same shape (encode.encode, E1-E9)

  y = A_far x  (O3 decode of the far part), then for every panel, slices in ascending k
      (the BCCOO+ combine order, P:184 / Q11): y[i] += segment sum of row i in slice k.

Everything here is plain numpy; the input must be normalised CSR (E1).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import decode, encode as E


@dataclass
class PanelParams:
    R: int = 16384        # panel rows (<= 32768; the product requires a multiple of 32)
    W: int = 8192         # slice width in columns (multiple of 4, <= 65536)
    B: int = 65536        # band half-width in columns
    T: int = 16           # band stream: blocks per thread
    C: int = 32           # band stream: threads per workgroup tile (one warp)
    diag0: int = 0        # column of local row 0 (row-partitioned ranks: the rank's first row)
    far: E.Params = field(default_factory=E.Params)   # parameters of the far BCCOO part


@dataclass
class PanelEncoded:
    m: int
    n: int
    pp: PanelParams
    KS: int
    npanels: int
    nband: int              # band entries (real blocks)
    nfill: int              # FILLER blocks (P6)
    nband_pad: int          # blocks after per-slice padding
    flags: np.ndarray       # uint8 LSB-first bit stream [nband_pad / 8]
    col16: np.ndarray       # uint16 [nband_pad]
    val: np.ndarray         # [nband_pad], dtype of A
    panel_blk0: np.ndarray  # int64 [npanels + 1]: first block of each panel
    slice_ptr: np.ndarray   # int32 [npanels, KS + 1]: block offset of slice k inside its panel (padded)
    stop_ptr: np.ndarray    # int32 [npanels, KS + 1]: row stops before slice k inside its panel
    first_row: np.ndarray   # int32 [npanels, KS]: first non-empty row of the slice (panel-relative; 0 if empty)
    tile_rank: np.ndarray   # int32 [nband_pad / (T*C)]: stops before each tile inside its slice
    far: E.Encoded          # the far part (plain BCCOO)
    far_csr: tuple          # (row_ptr, col, val) of the far part


def slices_per_panel(pp: PanelParams) -> int:
    return -(-(pp.R + 2 * pp.B) // pp.W)


def split(m: int, n: int, row_ptr, col, val, pp: PanelParams):
    """P1/P2: panel, slice and band membership of every entry (CSR order)."""
    rows = E.csr_to_coo_rows(m, np.asarray(row_ptr, dtype=np.int64))
    col = np.asarray(col, dtype=np.int64)
    KS = slices_per_panel(pp)
    p = rows // pp.R
    rel = col - (p * pp.R + pp.diag0 - pp.B)
    band = (rel >= 0) & (rel < KS * pp.W)
    k = np.where(band, rel // pp.W, -1)
    return rows, p, k, band


def encode_panel(m: int, n: int, row_ptr, col, val, pp: PanelParams) -> PanelEncoded:
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    col = np.asarray(col, dtype=np.int64)
    val = np.asarray(val)
    if not 0 < pp.R <= 32768 or not 0 < pp.W < 65535 or pp.B < 0:
        raise ValueError("need 0 < R <= 32768, 0 < W < 65535, B >= 0")
    KS = slices_per_panel(pp)
    TC = pp.T * pp.C
    npanels = -(-m // pp.R)
    rows, p, k, band = split(m, n, row_ptr, col, val, pp)

    # far part: every entry outside its panel's band, as a plain BCCOO matrix
    fr = rows[~band]
    frp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(fr, minlength=m), out=frp[1:])
    fcol = col[~band].astype(np.int32)
    fval = val[~band]
    far = E.encode(m, n, frp, fcol, fval, pp.far)

    # band entries with their panel-relative row and in-slice column offset
    bi = np.flatnonzero(band)
    bp, bk = p[bi], k[bi]
    blr = rows[bi] - bp * pp.R                        # row inside the panel
    boff = col[bi] - (bp * pp.R + pp.diag0 - pp.B) - bk * pp.W   # P5
    bv = val[bi]
    nband = bi.size
    # P6: first / last non-empty row of every slice; FILLER blocks for the empty rows between
    first_row = np.zeros((npanels, KS), dtype=np.int64)
    last_row = np.full((npanels, KS), -1, dtype=np.int64)
    if nband:
        g = bp * KS + bk
        lo = np.full(npanels * KS, np.iinfo(np.int64).max)
        hi = np.full(npanels * KS, -1)
        np.minimum.at(lo, g, blr)
        np.maximum.at(hi, g, blr)
        nonempty = hi >= 0
        first_row.ravel()[nonempty] = lo[nonempty]
        last_row.ravel()[:] = hi
    occupied = np.zeros((npanels, KS, pp.R), dtype=bool)
    occupied[bp, bk, blr] = True
    fp, fk, flr = [], [], []
    for q in range(npanels):
        for kk in range(KS):
            if last_row[q, kk] >= 0:
                r = np.arange(first_row[q, kk], last_row[q, kk] + 1)
                e = r[~occupied[q, kk, r]]
                fp.append(np.full(e.size, q)); fk.append(np.full(e.size, kk)); flr.append(e)
    fp = np.concatenate(fp) if fp else np.zeros(0, np.int64)
    fk = np.concatenate(fk) if fk else np.zeros(0, np.int64)
    flr = np.concatenate(flr) if flr else np.zeros(0, np.int64)
    nfill = fp.size
    # P3: blocks (entries + fillers) in (panel, slice, row, column) order; a filler sits in W
    ap = np.concatenate([bp, fp]); ak = np.concatenate([bk, fk]); alr = np.concatenate([blr, flr])
    aoff = np.concatenate([boff, np.full(nfill, pp.W, np.int64)])
    av = np.concatenate([bv, np.zeros(nfill, dtype=val.dtype)])
    order = np.lexsort((aoff, alr, ak, ap))
    ap, ak, alr, aoff, av = ap[order], ak[order], alr[order], aoff[order], av[order]
    nblk = ap.size

    # P4: every slice (p, k) padded to the workgroup tile; slices laid out in order
    gcnt = np.zeros((npanels, KS), dtype=np.int64)
    np.add.at(gcnt, (ap, ak), 1)
    gpad = -(-gcnt // TC) * TC
    slice_ptr = np.zeros((npanels, KS + 1), dtype=np.int64)
    slice_ptr[:, 1:] = np.cumsum(gpad, axis=1)
    panel_blk0 = np.zeros(npanels + 1, dtype=np.int64)
    np.cumsum(slice_ptr[:, -1], out=panel_blk0[1:])
    nband_pad = int(panel_blk0[-1])
    gstart = (np.cumsum(gcnt.ravel()) - gcnt.ravel()).reshape(npanels, KS)
    pos = panel_blk0[ap] + slice_ptr[ap, ak] + (np.arange(nblk) - gstart[ap, ak])

    # flags, 0 = last block of its row inside its slice
    bits = np.ones(nband_pad, dtype=np.uint8)
    if nblk:
        last = np.ones(nblk, dtype=bool)
        last[:-1] = ~((ap[1:] == ap[:-1]) & (ak[1:] == ak[:-1]) & (alr[1:] == alr[:-1]))
        bits[pos[last]] = 0
    flags = np.packbits(bits, bitorder="little")

    # P5 columns and values; pad entries repeat the slice's last stored column (Q3)
    col16 = np.zeros(nband_pad, dtype=np.uint16)
    col16[pos] = aoff.astype(np.uint16)
    vals = np.zeros(nband_pad, dtype=val.dtype)
    vals[pos] = av
    for q in range(npanels):
        for kk in range(KS):
            if gcnt[q, kk]:
                last_pos = panel_blk0[q] + slice_ptr[q, kk] + gcnt[q, kk] - 1
                col16[last_pos + 1: panel_blk0[q] + slice_ptr[q, kk + 1]] = col16[last_pos]

    # aux: stops per slice, stops before each tile inside its slice
    nst = np.where(last_row >= 0, last_row - first_row + 1, 0)
    stop_ptr = np.zeros((npanels, KS + 1), dtype=np.int32)
    stop_ptr[:, 1:] = np.cumsum(nst, axis=1)
    tile_rank = np.zeros(nband_pad // TC, dtype=np.int32)
    stops_cum = np.zeros(nband_pad + 1, dtype=np.int64)
    np.cumsum(1 - bits.astype(np.int64), out=stops_cum[1:])
    for q in range(npanels):
        for kk in range(KS):
            g0 = panel_blk0[q] + slice_ptr[q, kk]
            for tt in range(int(g0 // TC), int((panel_blk0[q] + slice_ptr[q, kk + 1]) // TC)):
                tile_rank[tt] = stops_cum[tt * TC] - stops_cum[g0]
    return PanelEncoded(m, n, pp, KS, npanels, nband, nfill, nband_pad, flags, col16, vals, panel_blk0,
                        slice_ptr.astype(np.int32), stop_ptr, first_row.astype(np.int32), tile_rank, far,
                        (frp, fcol, fval))


def spmv(enc: PanelEncoded, x: np.ndarray, acc=np.float64) -> np.ndarray:
    """O3-P: y = A_far x (plain BCCOO decode), then per panel the slices in ascending
    order, each walked in stream order with segments ending at '0' bits; the s-th segment
    of slice k belongs to row first_row + s (P6).  Column offset W reads 0 (FILLER)."""
    pp = enc.pp
    y = decode.spmv(enc.far, x, acc).astype(acc)
    bits = np.unpackbits(enc.flags, bitorder="little")[: enc.nband_pad]
    for q in range(enc.npanels):
        b0 = int(enc.panel_blk0[q])
        cb = q * pp.R + pp.diag0 - pp.B
        for k in range(enc.KS):
            base = cb + k * pp.W
            nst = int(enc.stop_ptr[q, k + 1] - enc.stop_ptr[q, k])
            run = acc(0)
            s = 0
            for b in range(b0 + int(enc.slice_ptr[q, k]), b0 + int(enc.slice_ptr[q, k + 1])):
                if s == nst:                     # padding after the slice's last stop
                    break
                c = int(enc.col16[b])
                xv = acc(0) if c == pp.W else acc(x[base + c])
                run = run + acc(enc.val[b]) * xv
                if bits[b] == 0:
                    i = q * pp.R + int(enc.first_row[q, k]) + s
                    y[i] = y[i] + run
                    run = acc(0)
                    s += 1
    return y


def to_dense(enc: PanelEncoded) -> np.ndarray:
    """Every stored band entry (fillers excluded) and every far entry back at (row, col)."""
    pp = enc.pp
    d = decode.to_dense(enc.far)
    bits = np.unpackbits(enc.flags, bitorder="little")[: enc.nband_pad]
    for q in range(enc.npanels):
        b0 = int(enc.panel_blk0[q])
        cb = q * pp.R + pp.diag0 - pp.B
        for k in range(enc.KS):
            s = 0
            nst = int(enc.stop_ptr[q, k + 1] - enc.stop_ptr[q, k])
            for b in range(b0 + int(enc.slice_ptr[q, k]), b0 + int(enc.slice_ptr[q, k + 1])):
                if s == nst:
                    break
                c = int(enc.col16[b])
                if c != pp.W:
                    i = q * pp.R + int(enc.first_row[q, k]) + s
                    d[i, cb + k * pp.W + c] += float(enc.val[b])
                s += bits[b] == 0
    return d
