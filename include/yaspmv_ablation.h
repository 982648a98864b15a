/* yaspmv_ablation.h — measurement-only entry points reproducing the ablation of the paper's
 * Fig. 14 (§6) on B200: the contribution of (1) the BCCOO format over
 * COO, (2) the matrix-based segmented sum over the tree-based one, (3) adjacent
 * synchronization over a second kernel for the cross-workgroup carries, (4) the fine-grain
 * optimizations (short column indices, skipping the workgroup scan).  Same
 * conventions as yaspmv.h; none of these is on the production path.
 */
#ifndef YASPMV_ABLATION_H
#define YASPMV_ABLATION_H

#include "yaspmv.h"

#ifdef __cplusplus
extern "C" {
#endif

/* y := A·x with one ablation step of our kernel (A built with h = w = S = 1):
 *   variant 1 "Efficient segmented sum/scan": matrix-based segmented sum, carries across
 *             workgroups by a second kernel after the first completes;
 *   variant 2 "Adjacent synchronization": carries by look-back, workgroup scan never skipped;
 *   variant 3 "Fine-grain optimizations": = yaspmv_spmv;
 *   variant 4 roofline probe "stream + gather": K1's tile loads and x gathers exactly as
 *             issued by yaspmv_spmv, then nothing but a per-thread sum (no segmented sum,
 *             scan, carries or y stores; y's contents are unspecified) — the time any kernel that
 *             reads this format and gathers x must spend;
 *   variant 5 roofline probe "stream only": as 4 with every gather redirected to
 *             x[col & 15] (L1 hits): the format stream alone;
 *   variant 6 roofline probe "stream + L2 gather": as 4 with every gather redirected to
 *             x[col & (2^20 - 1)] (an L2-resident 4-8 MB window: L1 misses, L2 hits) —
 *             separates the cost of the gather requests from that of x's DRAM misses.
 *             Needs n >= 2^20;
 *   variant 7 roofline probe "no carries": variant 1 without its carry kernel — every
 *             segment that spans a workgroup boundary is left without its carry-in (y wrong
 *             there): the cost of adjacent synchronization is the difference to variant 3;
 *   variant 8 roofline probe "up to the scan": returns after the workgroup segmented scan
 *             (no carry publish, no y stores, no look-back);
 *   variant 9 roofline probe: variant 7 without the y stores of the write-back;
 *   variant 10 roofline probe: variant 8 + thread C-1's 16-byte status store (publish);
 *   variant 11 roofline probe: variant 8 + one coalesced 4-byte store per thread;
 *   variant 12 test of the debug spin bound: variant 3 whose tile 0 never publishes its
 *             carry-out, so the look-back of a later tile of a row spanning >= 3 tiles
 *             polls forever (traps under YASPMV_SPIN_LIMIT, yaspmv.h).
 * Variants 4 and 5 do not compute y; they exist to measure.
 * x, y: device; the column storage is whatever A was built with (the caller builds A with
 * col_mode I32 for steps 1-2 and the auto/short mode for step 3). */
yaspmv_status yaspmv_ablation_spmv(yaspmv_matrix A, int32_t variant, const void* x, void* y, void* stream);

/* Tree-based segmented sum (Blelloch-style levels with a barrier each) over
 * 1024-element tiles + a carry kernel; all pointers are DEVICE memory, canonical layout:
 *   COO   ("COO" step): rows = int32 row index per element, flags = tile_seg0 = NULL;
 *   BCCOO ("BCCOO" step, 1x1 blocks): rows = NULL, flags = the BCCOO bit-flag stream,
 *          tile_seg0 = row stops before each 1024-element tile;
 *   col = int32 columns, val = values (dtype), n_elem elements; y (m entries) must hold zeros
 *   in rows without entries.  scratch: >= yaspmv_ablation_tree_scratch_bytes(n_elem). */
yaspmv_status yaspmv_ablation_tree(const int32_t* rows, const uint8_t* flags, const int32_t* tile_seg0,
                                   const int32_t* col, const void* val, int64_t n_elem, const void* x, void* y,
                                   int64_t m, yaspmv_dtype dtype, void* scratch, int64_t scratch_bytes, void* stream);
int64_t yaspmv_ablation_tree_scratch_bytes(int64_t n_elem);

#ifdef __cplusplus
}
#endif
#endif /* YASPMV_ABLATION_H */
