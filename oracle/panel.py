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
  P5  column stored as the unsigned short offset j - cb(p) - k*W  (< W <= 65536; the short
      column type of P:121/P:302 with a per-slice base, the original column = base +
      offset as P:150 requires)
  P6  rows of a slice without an entry hold no block; the slice's row-occupancy bitmap
      (R bits) maps the s-th row stop of the slice to the s-th set bit (the seg_row map of
      reading Q1/R2, as a bitmap); per-word prefix counts, per-slice stop offsets and,
      per workgroup tile, the stops before it inside its slice (the first-result entry
      of P:188-189, like cta_seg0) are aux arrays
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
    nband_pad: int          # after per-panel padding
    flags: np.ndarray       # uint8 LSB-first bit stream [nband_pad / 8]
    col16: np.ndarray       # uint16 [nband_pad]
    val: np.ndarray         # [nband_pad], dtype of A
    panel_blk0: np.ndarray  # int64 [npanels + 1]: first block of each panel
    slice_ptr: np.ndarray   # int32 [npanels, KS + 1]: block offset of slice k inside its panel (padded)
    stop_ptr: np.ndarray    # int32 [npanels, KS + 1]: row stops before slice k inside its panel
    occ: np.ndarray         # uint32 [npanels, KS, ceil(R / 32)]: row-occupancy bitmaps (LSB = lower row)
    pre: np.ndarray         # uint16 [npanels, KS, ceil(R / 32)]: set bits before each word
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
    if not 0 < pp.R <= 32768 or not 0 < pp.W <= 65536 or pp.B < 0:
        raise ValueError("need 0 < R <= 32768, 0 < W <= 65536, B >= 0")
    KS = slices_per_panel(pp)
    nw = -(-pp.R // 32)                     # bitmap words per slice
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

    # P3: band entries in (panel, slice, row, col) order (stable: CSR order is (row, col))
    bi = np.flatnonzero(band)
    order = bi[np.lexsort((col[bi], rows[bi], k[bi], p[bi]))]
    bp, bk, br, bc, bv = p[order], k[order], rows[order], col[order], val[order]
    nband = order.size

    # P4: every slice (p, k) padded to the workgroup tile; slices laid out in order
    gcnt = np.zeros((npanels, KS), dtype=np.int64)
    np.add.at(gcnt, (bp, bk), 1)
    gpad = -(-gcnt // TC) * TC
    slice_ptr = np.zeros((npanels, KS + 1), dtype=np.int64)
    slice_ptr[:, 1:] = np.cumsum(gpad, axis=1)
    panel_blk0 = np.zeros(npanels + 1, dtype=np.int64)
    np.cumsum(slice_ptr[:, -1], out=panel_blk0[1:])
    nband_pad = int(panel_blk0[-1])
    gstart = np.zeros((npanels, KS), dtype=np.int64)       # first entry of each group in `order`
    flat = np.cumsum(gcnt.ravel()) - gcnt.ravel()
    gstart[:, :] = flat.reshape(npanels, KS)
    pos = panel_blk0[bp] + slice_ptr[bp, bk] + (np.arange(nband) - gstart[bp, bk])

    # flags, 0 = last entry of its row inside its slice
    bits = np.ones(nband_pad, dtype=np.uint8)
    if nband:
        last = np.ones(nband, dtype=bool)
        same = (bp[1:] == bp[:-1]) & (bk[1:] == bk[:-1]) & (br[1:] == br[:-1])
        last[:-1] = ~same
        bits[pos[last]] = 0
    flags = np.packbits(bits, bitorder="little")

    # P5: unsigned short column offset inside the slice; pad entries repeat the slice's
    # last stored column (Q3)
    cb = bp * pp.R + pp.diag0 - pp.B
    col16 = np.zeros(nband_pad, dtype=np.uint16)
    col16[pos] = (bc - cb - bk * pp.W).astype(np.uint16)
    for q in range(npanels):
        for kk in range(KS):
            if gcnt[q, kk]:
                last_pos = panel_blk0[q] + slice_ptr[q, kk] + gcnt[q, kk] - 1
                col16[last_pos + 1: panel_blk0[q] + slice_ptr[q, kk + 1]] = col16[last_pos]
    vals = np.zeros(nband_pad, dtype=val.dtype)
    vals[pos] = bv

    # P6: row-occupancy bitmaps, prefix counts, stop offsets, stops before each tile
    occ_bits = np.zeros((npanels, KS, nw * 32), dtype=np.uint8)
    occ_bits[bp, bk, br - bp * pp.R] = 1
    occ = np.packbits(occ_bits.reshape(npanels, KS, nw, 32), axis=-1, bitorder="little")
    occ = occ.reshape(npanels, KS, nw, 4).copy().view("<u4").reshape(npanels, KS, nw).astype(np.uint32)
    wc = occ_bits.reshape(npanels, KS, nw, 32).sum(axis=-1)
    pre = np.zeros((npanels, KS, nw), dtype=np.uint16)
    pre[:, :, 1:] = np.cumsum(wc, axis=-1)[:, :, :-1]
    stop_ptr = np.zeros((npanels, KS + 1), dtype=np.int32)
    stop_ptr[:, 1:] = np.cumsum(wc.sum(axis=-1), axis=-1)
    ntile = nband_pad // TC
    tile_rank = np.zeros(ntile, dtype=np.int32)
    stops_cum = np.zeros(nband_pad + 1, dtype=np.int64)
    np.cumsum(1 - bits.astype(np.int64), out=stops_cum[1:])
    for q in range(npanels):
        for kk in range(KS):
            g0 = panel_blk0[q] + slice_ptr[q, kk]
            for tt in range(int(g0 // TC), int((panel_blk0[q] + slice_ptr[q, kk + 1]) // TC)):
                tile_rank[tt] = stops_cum[tt * TC] - stops_cum[g0]
    return PanelEncoded(m, n, pp, KS, npanels, nband, nband_pad, flags, col16, vals, panel_blk0,
                        slice_ptr.astype(np.int32), stop_ptr, occ, pre, tile_rank, far, (frp, fcol, fval))


def select_row(enc: PanelEncoded, q: int, k: int, s: int) -> int:
    """P6: the row (inside panel q) of the s-th stop of slice k = the s-th set bit of the
    slice's occupancy bitmap, found through the per-word prefix counts."""
    pre = enc.pre[q, k].astype(np.int64)
    w = int(np.searchsorted(pre, s, side="right")) - 1
    word = int(enc.occ[q, k, w])
    r = s - int(pre[w])
    for b in range(32):
        if (word >> b) & 1:
            if r == 0:
                return w * 32 + b
            r -= 1
    raise AssertionError("stop beyond the slice's bitmap")


def spmv(enc: PanelEncoded, x: np.ndarray, acc=np.float64) -> np.ndarray:
    """O3-P: y = A_far x (plain BCCOO decode), then per panel the slices in ascending
    order, each walked in stream order with segments ending at '0' bits."""
    pp = enc.pp
    y = decode.spmv(enc.far, x, acc).astype(acc)
    bits = np.unpackbits(enc.flags, bitorder="little")[: enc.nband_pad]
    for q in range(enc.npanels):
        b0 = int(enc.panel_blk0[q])
        cb = q * pp.R + pp.diag0 - pp.B
        for k in range(enc.KS):
            base = cb + k * pp.W
            run = acc(0)
            s = 0
            for b in range(b0 + int(enc.slice_ptr[q, k]), b0 + int(enc.slice_ptr[q, k + 1])):
                j = base + int(enc.col16[b])
                run = run + acc(enc.val[b]) * acc(x[j])
                if bits[b] == 0:
                    i = q * pp.R + select_row(enc, q, k, s)
                    y[i] = y[i] + run
                    run = acc(0)
                    s += 1
    return y


def to_dense(enc: PanelEncoded) -> np.ndarray:
    """Every stored band entry and every far entry back at (row, col)."""
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
                if s == nst:            # padding after the slice's last stop
                    break
                i = q * pp.R + select_row(enc, q, k, s)
                d[i, cb + k * pp.W + int(enc.col16[b])] += float(enc.val[b])
                s += bits[b] == 0
    return d
