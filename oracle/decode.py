"""O3 — decode-and-multiply over the canonical BCCOO/BCCOO+ arrays
(TEST INFRASTRUCTURE ONLY, see oracle/__init__).

Walks the bit-flag stream in order (Fig. 7 semantics: a segmented sum whose
segments end at '0' bits), multiplies each h x w block with x indexed by its
ORIGINAL block column, writes the segment sum of stacked row k to the
per-slice partial result, then combines the slices in ascending order (Fig. 5,
P:156-184; Q11).  With integer data every step is exact, so y equals A·x exactly.
"""
from __future__ import annotations

import numpy as np

from .encode import EMPTY_MAP, Encoded, block_columns, unpack_flags


def block_products(enc: Encoded, x: np.ndarray, acc=np.float64) -> np.ndarray:
    """p[b, r] = sum_c val[r][b*w + c] * x[col_b*w + c]   (step 1 of P:226); x entries at
    index >= N read as 0 (Q4)."""
    h, w = enc.p.h, enc.p.w
    cols = block_columns(enc)
    xp = np.zeros(enc.NB * w + w, dtype=acc)
    xp[: enc.n] = x
    P = np.zeros((enc.nnzb_pad, h), dtype=acc)
    for r in range(h):
        v = enc.val[r].astype(acc).reshape(enc.nnzb_pad, w)
        for c in range(w):
            P[:, r] += v[:, c] * xp[cols * w + c]
    return P


def stacked_row_of_segments(enc: Encoded) -> np.ndarray:
    """Stacked block row of each segment: the seg_row map (R2), else the segment index
    itself (R1: every stacked row holds >= 1 block, P:114 'multiple 1s')."""
    if enc.p.empty_mode == EMPTY_MAP and enc.seg_row.size:
        return enc.seg_row.astype(np.int64)
    return np.arange(enc.n_stops, dtype=np.int64)


def spmv(enc: Encoded, x: np.ndarray, acc=np.float64) -> np.ndarray:
    """y = A·x from the encoded arrays (segmented sum, then slice combine)."""
    h = enc.p.h
    bits = unpack_flags(enc)
    P = block_products(enc, x, acc)
    stop = bits == 0
    seg = np.cumsum(stop) - stop            # segment index of every block
    valid = seg < enc.n_stops                # pad blocks after the last stop are dropped
    part = np.zeros((enc.n_stops, h), dtype=acc)
    np.add.at(part, seg[valid], P[valid])
    # per-slice partial results tmp[s][br*h + r] (Fig. 5); empty stacked rows stay 0
    tmp = np.zeros((enc.p.S * enc.MB, h), dtype=acc)
    tmp[stacked_row_of_segments(enc)] = part
    tmp = tmp.reshape(enc.p.S, enc.MB * h)
    y = tmp[0].copy()
    for s in range(1, enc.p.S):              # ascending slice order (Q11)
        y = y + tmp[s]
    return y[: enc.m]


def decode_blocks(enc: Encoded):
    """Reconstruct the structural entries (row, col, value) from the encoding, keeping
    every stored value (including zeros inside blocks)."""
    h, w = enc.p.h, enc.p.w
    bits = unpack_flags(enc)
    stop = bits == 0
    seg = np.cumsum(stop) - stop
    nb = enc.nnzb
    srow = stacked_row_of_segments(enc)[seg[:nb]]
    br = srow % enc.MB
    cols = block_columns(enc)[:nb]
    out = []
    for r in range(h):
        v = enc.val[r].reshape(enc.nnzb_pad, w)[:nb]
        for c in range(w):
            out.append((br * h + r, cols * w + c, v[:, c]))
    R = np.concatenate([o[0] for o in out])
    Cc = np.concatenate([o[1] for o in out])
    V = np.concatenate([o[2] for o in out])
    keep = (R < enc.m) & (Cc < enc.n)
    return R[keep], Cc[keep], V[keep]


def to_dense(enc: Encoded) -> np.ndarray:
    R, Cc, V = decode_blocks(enc)
    d = np.zeros((enc.m, enc.n), dtype=np.float64)
    np.add.at(d, (R, Cc), V.astype(np.float64))
    return d
