"""O2 — independent BCCOO / BCCOO+ encoder (TEST INFRASTRUCTURE ONLY, see oracle/__init__).

Follows PAPER.md §2 step by step; every step cites the passage it implements.  Readings
where the paper is silent or garbled are SURVEY §8(c) Q1-Q16 and are listed in DESIGN.md.

  E1  normalise input: sort by (row, col), sum duplicates in input order, explicit zeros
      stay structural (COO; Q14)
  E2  h x w blocking; BCCOO+ vertical slices stacked top-down: stacked block row
      sr = (bc div SW)*MB + br (Q5)
  E3  blocks ordered by (sr, bc)                                          (Fig. 2, Fig. 4)
  E4  h value arrays, w values per block, zeros inside a block stored
  E5  col = ORIGINAL block column, also for BCCOO+ 
  E6  bit flag 0 = row stop (last block of its stacked row), 1 = continue
      empty stacked rows: R1 a zero filler block (paper's "multiple 1s") whose
                          column is NB, past the last block column (Q3)
                          R2 a seg_row map + zero list                    (Q1)
  E7  pad with '1' bits to a multiple of the workgroup tile T*C; pad blocks
      hold zero values and repeat the last column of the stream (Q3)
  E8  flags packed LSB-first in bytes (Q2)
  E9  col storage: unsigned short if NB < 65535 (Q6) else int32; or the
      segmented int16 difference with -1 escape (Q7)
  aux cta_seg0 / first-result entry = exclusive scan of inverted flags
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

COL_U16, COL_I32, COL_DELTA = 1, 2, 3
EMPTY_FILLER, EMPTY_MAP = 1, 2


@dataclass
class Params:
    h: int = 1            # block height, Table 1 {1,2,3,4}
    w: int = 1            # block width,  Table 1 {1,2,4}
    S: int = 1            # vertical slices; 1 = BCCOO, >1 = BCCOO+ 
    T: int = 16           # non-zero blocks per thread (thread-level tile)
    C: int = 256          # threads per workgroup
    col_mode: int = 0     # 0 auto, 1 u16, 2 i32, 3 int16 delta + int32 escape
    empty_mode: int = 0   # 0 auto, 1 filler blocks (R1), 2 seg_row map (R2)


@dataclass
class Encoded:
    m: int
    n: int
    p: Params
    MB: int
    NB: int
    SW: int
    nnzb: int            # stored blocks including R1 fillers, excluding padding
    nnzb_pad: int
    ntiles: int
    n_stops: int
    n_filler: int
    flags: np.ndarray    # uint8[nnzb_pad/8]
    col: np.ndarray      # uint16 or int32 [nnzb_pad] (int32 in delta mode)
    col_delta: np.ndarray  # int16[nnzb_pad] (delta mode) else empty
    val: list            # h arrays [nnzb_pad*w]
    seg_row: np.ndarray  # int32[n_stops] (R2 with empty rows) else empty
    zero_rows: np.ndarray  # int32 stacked rows with no block (R2) else empty
    cta_seg0: np.ndarray   # int32[ntiles]
    fre: np.ndarray        # int32[ntiles*C]
    extra: dict = field(default_factory=dict)


# ----------------------------------------------------------------------------- E1
def normalize(m: int, n: int, rows, cols, vals):
    """E1 (Q14): stable sort of COO triples by (row, col); duplicates are summed
    in input order; explicit zeros stay structural.  Returns CSR (row_ptr, col, val)."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    vals = np.asarray(vals)
    if rows.size and (rows.min() < 0 or rows.max() >= m or cols.min() < 0 or cols.max() >= n):
        raise ValueError("index out of range")
    order = np.lexsort((cols, rows))           # stable: equal keys keep input order
    r, c, v = rows[order], cols[order], vals[order]
    if r.size:
        new = np.ones(r.size, dtype=bool)
        new[1:] = (r[1:] != r[:-1]) | (c[1:] != c[:-1])
        if not new.all():
            starts = np.flatnonzero(new)
            out = v[starts].copy()
            # sum duplicates one by one in input order (left fold)
            dup = np.flatnonzero(~new)
            grp = np.cumsum(new) - 1
            for k in dup:
                out[grp[k]] = out[grp[k]] + v[k]
            r, c, v = r[starts], c[starts], out
    row_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=m), out=row_ptr[1:])
    return row_ptr, c.astype(np.int32), v


def csr_to_coo_rows(m: int, row_ptr: np.ndarray) -> np.ndarray:
    return np.repeat(np.arange(m, dtype=np.int64), np.diff(row_ptr))


# ----------------------------------------------------------------------------- helpers
def resolve_col_mode(NB: int, col_mode: int) -> int:
    """E9 / Q6: 'unsigned short ... if the width of a sparse matrix is less than 65535'
    (P:302), read on BLOCK columns."""
    if col_mode == 0:
        return COL_U16 if NB < 65535 else COL_I32
    if col_mode == COL_U16 and NB >= 65535:
        raise ValueError("u16 col requires NB < 65535")
    return col_mode


def col_bytes(mode: int) -> int:
    return {COL_U16: 2, COL_I32: 4, COL_DELTA: 2}[mode]


def footprint_bytes(nnzb: int, h: int, w: int, s_v: int, s_c: int) -> int:
    """Memory footprint of the format = sum of array sizes: values, col_index and
    the bit-flag array (one bit per block)."""
    return nnzb * (h * w * s_v + s_c) + (nnzb + 7) // 8


# ----------------------------------------------------------------------------- encode
def encode(m: int, n: int, row_ptr, col, val, p: Params) -> Encoded:
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    col = np.asarray(col, dtype=np.int64)
    val = np.asarray(val)
    h, w, S, T, C = p.h, p.w, p.S, p.T, p.C
    s_v = val.dtype.itemsize
    TC = T * C

    # E2: blocking and vertical slicing
    MB = -(-m // h)
    NB = -(-n // w)
    if S < 1 or (NB > 0 and S > NB):
        raise ValueError("slices must satisfy 1 <= S <= NB")
    SW = -(-NB // S) if NB > 0 else 1
    rows = csr_to_coo_rows(m, row_ptr)
    br = rows // h
    bc = col // w
    sr = (bc // SW) * MB + br                   # stacked block row (top-down slices)

    # E3: unique blocks ordered by (stacked row, block column)
    key = sr * max(NB, 1) + bc
    ukey, inv = np.unique(key, return_inverse=True)
    blk_sr = ukey // max(NB, 1)
    blk_bc = ukey % max(NB, 1)
    n_real = ukey.size

    # E6 / Q1: stacked rows that hold no block
    n_srows = S * MB
    has = np.zeros(n_srows, dtype=bool)
    has[blk_sr] = True
    empty = np.flatnonzero(~has)
    col_mode = resolve_col_mode(NB, p.col_mode)
    s_c = col_bytes(col_mode)
    empty_mode = p.empty_mode
    if empty_mode == 0:
        # auto: the cheaper of filler blocks (R1) and a seg_row map (R2), by footprint
        r1 = empty.size * (h * w * s_v + s_c)
        r2 = 4 * int(has.sum()) + 4 * empty.size
        empty_mode = EMPTY_FILLER if (empty.size == 0 or r1 <= r2) else EMPTY_MAP

    # R1: insert one zero filler block per empty stacked row (bit flag '0' for it)
    if empty_mode == EMPTY_FILLER and empty.size:
        all_sr = np.concatenate([blk_sr, empty])
        is_fill = np.concatenate([np.zeros(n_real, bool), np.ones(empty.size, bool)])
        # real blocks are already in (sr, bc) order and a filler owns its row alone,
        # so a stable sort on the stacked row places every filler in its row's slot
        order = np.argsort(all_sr, kind="stable")
        rank = np.empty(order.size, dtype=np.int64)
        rank[order] = np.arange(order.size)
        pos_of_real = rank[:n_real]
        stream_sr = all_sr[order]
        stream_fill = is_fill[order]
        stream_bc = np.concatenate([blk_bc, np.zeros(empty.size, np.int64)])[order]
        # filler column = NB, one past the last block column: x reads 0 there (Q4), so an
        # empty row is exactly 0 for every x, also x = +-Inf (Q3, round 2)
        stream_bc = np.where(stream_fill, NB, stream_bc)
        n_filler = int(empty.size)
    else:
        pos_of_real = np.arange(n_real, dtype=np.int64)
        stream_sr = blk_sr
        stream_bc = blk_bc
        n_filler = 0
    nnzb = n_real + n_filler

    # E7: pad to a multiple of the workgroup tile
    nnzb_pad = -(-nnzb // TC) * TC
    ntiles = nnzb_pad // TC

    # E6: bit flags, 0 = last block of its stacked row; pad bits 1
    bits = np.ones(nnzb_pad, dtype=np.uint8)
    if nnzb:
        stop = np.ones(nnzb, dtype=bool)
        stop[:-1] = stream_sr[1:] != stream_sr[:-1]
        bits[:nnzb][stop] = 0
    n_stops = int(nnzb_pad - bits.sum())
    # E8: pack LSB-first (Q2)
    flags = np.packbits(bits, bitorder="little")

    # E5: original block column per block; pad blocks repeat the last column (Q3)
    colb = np.zeros(nnzb_pad, dtype=np.int64)
    colb[:nnzb] = stream_bc
    if nnzb_pad > nnzb:
        colb[nnzb:] = stream_bc[-1] if nnzb else 0

    # E4: h value arrays with w values per block
    vals = [np.zeros(nnzb_pad * w, dtype=val.dtype) for _ in range(h)]
    b_of_entry = pos_of_real[inv]
    r_in = rows % h
    c_in = col % w
    for r in range(h):
        sel = r_in == r
        vals[r][b_of_entry[sel] * w + c_in[sel]] = val[sel]

    # E9: column storage
    col_delta = np.zeros(0, dtype=np.int16)
    if col_mode == COL_U16:
        colarr = colb.astype(np.uint16)
    else:
        colarr = colb.astype(np.int32)
        if col_mode == COL_DELTA:
            prev = np.zeros(nnzb_pad, dtype=np.int64)
            prev[1:] = colb[:-1]
            prev[np.arange(nnzb_pad) % T == 0] = 0      # segmented difference per thread tile
            d = colb - prev
            esc = (d < -32768) | (d > 32767) | (d == -1)
            col_delta = np.where(esc, -1, d).astype(np.int16)

    # Q1 R2: stop -> stacked row map, and the stacked rows without any block
    seg_row = np.zeros(0, dtype=np.int32)
    zero_rows = np.zeros(0, dtype=np.int32)
    if empty_mode == EMPTY_MAP and empty.size:
        seg_row = stream_sr[:nnzb][bits[:nnzb] == 0].astype(np.int32)
        zero_rows = empty.astype(np.int32)

    # aux: number of stops before each thread tile / workgroup tile
    stops_cum = np.zeros(nnzb_pad + 1, dtype=np.int64)
    np.cumsum(1 - bits.astype(np.int64), out=stops_cum[1:])
    fre = stops_cum[np.arange(ntiles * C) * T].astype(np.int32)
    cta_seg0 = stops_cum[np.arange(ntiles) * TC].astype(np.int32)

    p_res = Params(h, w, S, T, C, col_mode, empty_mode)
    return Encoded(m, n, p_res, MB, NB, SW, nnzb, nnzb_pad, ntiles, n_stops, n_filler, flags,
                   colarr, col_delta, vals, seg_row, zero_rows, cta_seg0, fre)


def unpack_flags(enc: Encoded) -> np.ndarray:
    return np.unpackbits(enc.flags, bitorder="little")[: enc.nnzb_pad]


def block_columns(enc: Encoded) -> np.ndarray:
    """Block columns per block, reconstructed from the stored column array(s)."""
    if enc.p.col_mode != COL_DELTA:
        return enc.col.astype(np.int64)
    T = enc.p.T
    d = enc.col_delta.astype(np.int64)
    out = np.zeros(enc.nnzb_pad, dtype=np.int64)
    for b in range(enc.nnzb_pad):
        base = 0 if b % T == 0 else out[b - 1]
        out[b] = enc.col[b] if d[b] == -1 else base + d[b]
    return out
