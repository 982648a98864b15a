"""CPU oracle for the yaSpMV hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import, call, link or execute anything under ``oracle/``.
The product (``paper_conf_ppopp_yanlzz14_b200``) never imports it, and this package
never imports the product: the two share no code (inputs come from ``synth/``).

Parts:
  O1 ``ref``      — the plain definition y = A·x, compensated fp64
                    (Ogita-Rump-Oishi Dot2) per row, plus bound[i] = sum_j |a_ij||x_j|.
                    Plain C (``ref_csr.c``) with OpenMP; also the CPU baseline.
  O2 ``encode``   — an independent BCCOO / BCCOO+ encoder following PAPER.md §2
                     step by step (E1-E9 in DESIGN.md).
  O3 ``decode``   — decode-and-multiply over the canonical arrays (Fig. 7 semantics,
                    P:230, Fig. 5 slice combine P:156-184).
  O4 ``simulate`` — tiled simulator of the matrix-based segmented sum with
                    last_partial_sums and the adjacent-synchronization chain
                    (P:259-298), for tiny inputs.

Parity status: O1, O2 (flags, col, values, seg_row, zero_rows, cta_seg0, fre), O3, O4 are
pinned by tests/test_oracle_*.py (paper examples in tests/golden/, exact rational brute
force, closed forms, invariants).  The int16 column-delta array is pinned only by
round-trip invariants and its stated rule — the paper prints no example: "parity
unpinned" by the paper for that one array ("Readings").
"""
