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
  far entries: a plain BCCOO matrix of the same shape (encode.encode, E1-E9), or with
  far_in_panel:
  P7  the far entries of panel p are the panel's slice 0 (the band slices are 1..KS): one
      BCCOO slice over all n columns (P:83-119 with the row rules P4/P6), its columns
      stored as int32 in a separate array (the int column type of P:121); a FILLER block
      there has column n (reads 0, as column NB of plain BCCOO, Q3).  The stream of panel p
      is [far slice | band slices 1..KS], each padded to T*C; flags, values and tile_rank
      run over that stream, col16 over the band blocks only, far_col over the far blocks
      only (far_blk0[p] = far blocks before panel p).

  y = A_far x  (O3 decode of the far part), then for every panel, slices in ascending k
      (the BCCOO+ combine order, P:184 / Q11): y[i] += segment sum of row i in slice k.
      With P7, y = 0 and the far slice is slice 0 of every panel (the same order).

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
    far_in_panel: bool = False                         # P7: far entries as slice 0 of each panel


@dataclass
class PanelEncoded:
    m: int
    n: int
    pp: PanelParams
    KS: int                 # band slices per panel (the panel holds KS + fip slices)
    npanels: int
    nband: int              # band entries (real blocks)
    nfill: int              # FILLER blocks (P6)
    nband_pad: int          # blocks after per-slice padding
    flags: np.ndarray       # uint8 LSB-first bit stream [nband_pad / 8]
    col16: np.ndarray       # uint16 [nband_pad - far_blk0[-1]]: band blocks only
    val: np.ndarray         # [nband_pad], dtype of A
    panel_blk0: np.ndarray  # int64 [npanels + 1]: first block of each panel
    slice_ptr: np.ndarray   # int32 [npanels, NS + 1]: block offset of slice k inside its panel (padded)
    stop_ptr: np.ndarray    # int32 [npanels, NS + 1]: row stops before slice k inside its panel
    first_row: np.ndarray   # int32 [npanels, NS]: first non-empty row of the slice (panel-relative; 0 if empty)
    tile_rank: np.ndarray   # int32 [nband_pad / (T*C)]: stops before each tile inside its slice
    far: E.Encoded | None   # the far part (plain BCCOO); None with P7
    far_csr: tuple          # (row_ptr, col, val) of the far entries
    fip: int = 0            # 1 with P7 (NS = KS + fip slices per panel, slice 0 = far slice)
    far_col: np.ndarray = None   # P7: int32 [far_blk0[-1]], column of every far-slice block (n: FILLER)
    far_blk0: np.ndarray = None  # P7: int64 [npanels + 1], far-slice blocks before each panel

    @property
    def NS(self) -> int:
        return self.KS + self.fip


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

    fip = 1 if pp.far_in_panel else 0
    NS = KS + fip
    # far entries: every entry outside its panel's band
    fr = rows[~band]
    frp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(fr, minlength=m), out=frp[1:])
    fcol = col[~band].astype(np.int32)
    fval = val[~band]
    far = None if fip else E.encode(m, n, frp, fcol, fval, pp.far)

    # the blocks of every slice with their panel-relative row and stored column: band
    # entries (slice k + fip, column offset P5), with P7 the far entries (slice 0, column)
    bi = np.flatnonzero(band if not fip else np.ones(rows.size, dtype=bool))
    bp = p[bi]
    bk = np.where(band[bi], k[bi] + fip, 0)
    blr = rows[bi] - bp * pp.R                        # row inside the panel
    boff = np.where(band[bi], col[bi] - (bp * pp.R + pp.diag0 - pp.B) - k[bi] * pp.W, col[bi])   # P5 / P7
    bv = val[bi]
    nband = int(band.sum())
    # P6: first / last non-empty row of every slice; FILLER blocks for the empty rows between
    first_row = np.zeros((npanels, NS), dtype=np.int64)
    last_row = np.full((npanels, NS), -1, dtype=np.int64)
    if bi.size:
        g = bp * NS + bk
        lo = np.full(npanels * NS, np.iinfo(np.int64).max)
        hi = np.full(npanels * NS, -1)
        np.minimum.at(lo, g, blr)
        np.maximum.at(hi, g, blr)
        nonempty = hi >= 0
        first_row.ravel()[nonempty] = lo[nonempty]
        last_row.ravel()[:] = hi
    occupied = np.zeros((npanels, NS, pp.R), dtype=bool)
    occupied[bp, bk, blr] = True
    fp, fk, flr = [], [], []
    for q in range(npanels):
        for kk in range(NS):
            if last_row[q, kk] >= 0:
                r = np.arange(first_row[q, kk], last_row[q, kk] + 1)
                e = r[~occupied[q, kk, r]]
                fp.append(np.full(e.size, q)); fk.append(np.full(e.size, kk)); flr.append(e)
    fp = np.concatenate(fp) if fp else np.zeros(0, np.int64)
    fk = np.concatenate(fk) if fk else np.zeros(0, np.int64)
    flr = np.concatenate(flr) if flr else np.zeros(0, np.int64)
    nfill = fp.size
    # P3: blocks (entries + fillers) in (panel, slice, row, column) order; a filler sits in
    # column W of a band slice (the window's zero slot) or column n of the far slice (P7)
    ap = np.concatenate([bp, fp]); ak = np.concatenate([bk, fk]); alr = np.concatenate([blr, flr])
    aoff = np.concatenate([boff, np.where(fk < fip, n, pp.W)])
    av = np.concatenate([bv, np.zeros(nfill, dtype=val.dtype)])
    order = np.lexsort((aoff, alr, ak, ap))
    ap, ak, alr, aoff, av = ap[order], ak[order], alr[order], aoff[order], av[order]
    nblk = ap.size

    # P4: every slice (p, k) padded to the workgroup tile; slices laid out in order
    gcnt = np.zeros((npanels, NS), dtype=np.int64)
    np.add.at(gcnt, (ap, ak), 1)
    gpad = -(-gcnt // TC) * TC
    slice_ptr = np.zeros((npanels, NS + 1), dtype=np.int64)
    slice_ptr[:, 1:] = np.cumsum(gpad, axis=1)
    panel_blk0 = np.zeros(npanels + 1, dtype=np.int64)
    np.cumsum(slice_ptr[:, -1], out=panel_blk0[1:])
    nband_pad = int(panel_blk0[-1])
    gstart = (np.cumsum(gcnt.ravel()) - gcnt.ravel()).reshape(npanels, NS)
    pos = panel_blk0[ap] + slice_ptr[ap, ak] + (np.arange(nblk) - gstart[ap, ak])

    # flags, 0 = last block of its row inside its slice
    bits = np.ones(nband_pad, dtype=np.uint8)
    if nblk:
        last = np.ones(nblk, dtype=bool)
        last[:-1] = ~((ap[1:] == ap[:-1]) & (ak[1:] == ak[:-1]) & (alr[1:] == alr[:-1]))
        bits[pos[last]] = 0
    flags = np.packbits(bits, bitorder="little")

    # stored columns and values; pad entries repeat the slice's last stored column (Q3)
    colall = np.zeros(nband_pad, dtype=np.int64)
    colall[pos] = aoff
    vals = np.zeros(nband_pad, dtype=val.dtype)
    vals[pos] = av
    for q in range(npanels):
        for kk in range(NS):
            if gcnt[q, kk]:
                last_pos = panel_blk0[q] + slice_ptr[q, kk] + gcnt[q, kk] - 1
                colall[last_pos + 1: panel_blk0[q] + slice_ptr[q, kk + 1]] = colall[last_pos]
    # P5 / P7: u16 offsets of the band blocks, int32 columns of the far-slice blocks
    is_far = np.zeros(nband_pad, dtype=bool)
    far_blk0 = None
    if fip:
        far_blk0 = np.zeros(npanels + 1, dtype=np.int64)
        np.cumsum(slice_ptr[:, 1], out=far_blk0[1:])
        for q in range(npanels):
            is_far[panel_blk0[q]: panel_blk0[q] + slice_ptr[q, 1]] = True
    col16 = colall[~is_far].astype(np.uint16)
    far_col = colall[is_far].astype(np.int32) if fip else None

    # aux: stops per slice, stops before each tile inside its slice
    nst = np.where(last_row >= 0, last_row - first_row + 1, 0)
    stop_ptr = np.zeros((npanels, NS + 1), dtype=np.int32)
    stop_ptr[:, 1:] = np.cumsum(nst, axis=1)
    tile_rank = np.zeros(nband_pad // TC, dtype=np.int32)
    stops_cum = np.zeros(nband_pad + 1, dtype=np.int64)
    np.cumsum(1 - bits.astype(np.int64), out=stops_cum[1:])
    for q in range(npanels):
        for kk in range(NS):
            g0 = panel_blk0[q] + slice_ptr[q, kk]
            for tt in range(int(g0 // TC), int((panel_blk0[q] + slice_ptr[q, kk + 1]) // TC)):
                tile_rank[tt] = stops_cum[tt * TC] - stops_cum[g0]
    return PanelEncoded(m, n, pp, KS, npanels, nband, nfill, nband_pad, flags, col16, vals, panel_blk0,
                        slice_ptr.astype(np.int32), stop_ptr, first_row.astype(np.int32), tile_rank, far,
                        (frp, fcol, fval), fip, far_col, far_blk0)


def _slice_columns(enc: PanelEncoded, q: int, kk: int):
    """Original column of every block of slice (q, kk) (None for a FILLER block): the far
    slice's stored column (P7; n = FILLER), or base + offset of a band slice (P5; W = FILLER)."""
    pp = enc.pp
    b0 = int(enc.panel_blk0[q])
    lo, hi = b0 + int(enc.slice_ptr[q, kk]), b0 + int(enc.slice_ptr[q, kk + 1])
    if kk < enc.fip:
        f0 = int(enc.far_blk0[q]) + int(enc.slice_ptr[q, kk]) - int(enc.slice_ptr[q, 0])
        c = enc.far_col[f0: f0 + hi - lo].astype(np.int64)
        return lo, hi, [None if v == enc.n else int(v) for v in c]
    base = q * pp.R + pp.diag0 - pp.B + (kk - enc.fip) * pp.W
    # band blocks of panels < q and the far slice of panels <= q precede these in col16
    c0 = lo - (int(enc.far_blk0[q + 1]) if enc.fip else 0)
    c = enc.col16[c0: c0 + hi - lo].astype(np.int64)
    return lo, hi, [None if v == pp.W else base + int(v) for v in c]


def spmv(enc: PanelEncoded, x: np.ndarray, acc=np.float64) -> np.ndarray:
    """O3-P: y = A_far x (plain BCCOO decode; 0 with P7), then per panel the slices in
    ascending order (P7: the far slice first), each walked in stream order with segments
    ending at '0' bits; the s-th segment of slice k belongs to row first_row + s (P6).  A
    FILLER block reads 0."""
    pp = enc.pp
    y = decode.spmv(enc.far, x, acc).astype(acc) if enc.far is not None else np.zeros(enc.m, dtype=acc)
    bits = np.unpackbits(enc.flags, bitorder="little")[: enc.nband_pad]
    for q in range(enc.npanels):
        for k in range(enc.NS):
            lo, hi, cols = _slice_columns(enc, q, k)
            nst = int(enc.stop_ptr[q, k + 1] - enc.stop_ptr[q, k])
            run = acc(0)
            s = 0
            for b in range(lo, hi):
                if s == nst:                     # padding after the slice's last stop
                    break
                c = cols[b - lo]
                xv = acc(0) if c is None else acc(x[c])
                run = run + acc(enc.val[b]) * xv
                if bits[b] == 0:
                    i = q * pp.R + int(enc.first_row[q, k]) + s
                    y[i] = y[i] + run
                    run = acc(0)
                    s += 1
    return y


def to_dense(enc: PanelEncoded) -> np.ndarray:
    """Every stored entry (fillers excluded) back at (row, col)."""
    pp = enc.pp
    d = decode.to_dense(enc.far) if enc.far is not None else np.zeros((enc.m, enc.n))
    bits = np.unpackbits(enc.flags, bitorder="little")[: enc.nband_pad]
    for q in range(enc.npanels):
        for k in range(enc.NS):
            lo, hi, cols = _slice_columns(enc, q, k)
            s = 0
            nst = int(enc.stop_ptr[q, k + 1] - enc.stop_ptr[q, k])
            for b in range(lo, hi):
                if s == nst:
                    break
                if cols[b - lo] is not None:
                    i = q * pp.R + int(enc.first_row[q, k]) + s
                    d[i, cols[b - lo]] += float(enc.val[b])
                s += bits[b] == 0
    return d
