/* yaspmv.h — C ABI of the B200-native yaSpMV hot path: y = A·x over BCCOO / BCCOO+.
 *
 * The operation is the paper's problem statement, "sparse matrix vector multiplication"
 * y = A·x (§1; §2.3), computed over the BCCOO format (§2.2,
 * P:81-121) or its vertically sliced variant BCCOO+ (§2.3) by the
 * matrix-based segmented sum of §3, with parameters chosen by the
 * auto-tuner of §4 (Table 1).  The entry points are SURVEY.md §8(b).
 *
 * Conventions for every call
 *   - extern "C", fixed-width integer types, plain host or device pointers; no C++ or
 *     torch types cross this boundary.
 *   - Return value is a yaspmv_status; on failure a message is available from
 *     yaspmv_last_error() (thread-local, valid until the next call on that thread).
 *   - "host" pointers are ordinary CPU memory (pageable or pinned); "device" pointers are
 *     CUDA global memory of the handle's device (e.g. torch tensor .data_ptr()).
 *   - Streams are cudaStream_t passed as void* (NULL = the legacy default stream).
 *   - Matrix data types: YASPMV_F32 (float values, float x/y) or YASPMV_F64 (double).
 *     Indices are int32 column indices and int64 row pointers.
 *   - There is no CPU fallback: spmv-family calls on a host-only handle, or without a
 *     CUDA device, fail with YASPMV_EINVAL / YASPMV_ECUDA.
 */
#ifndef YASPMV_H
#define YASPMV_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct yaspmv_matrix_s* yaspmv_matrix; /* opaque; owns every encoded array */

typedef enum {
  YASPMV_OK = 0,
  YASPMV_EINVAL = 1,       /* bad argument / index out of range / host-only handle     */
  YASPMV_ENOMEM = 2,       /* host or device allocation failed                         */
  YASPMV_ECUDA = 3,        /* CUDA runtime or launch error (message has the CUDA text) */
  YASPMV_EUNSUPPORTED = 4  /* parameter combination with no compiled kernel            */
} yaspmv_status;

typedef enum { YASPMV_F32 = 0, YASPMV_F64 = 1 } yaspmv_dtype;

/* Column-index storage (Table 1 "Col_index compress"). */
enum { YASPMV_COL_AUTO = 0, YASPMV_COL_U16 = 1, YASPMV_COL_I32 = 2, YASPMV_COL_DELTA16 = 3 };
/* Empty (stacked) block rows (reading Q1):
 *   FILLER = one zero block per empty row (the paper's "multiple 1s"),
 *   MAP    = seg_row map from row stops to rows + a zero-fill list. */
enum { YASPMV_EMPTY_AUTO = 0, YASPMV_EMPTY_FILLER = 1, YASPMV_EMPTY_MAP = 2 };
/* yaspmv_params.flags */
enum {
  YASPMV_KEEP_HOST = 1, /* keep the canonical host arrays for yaspmv_export              */
  YASPMV_DROP_CSR = 2,  /* free the normalised host CSR after upload (no tune/reencode)  */
  YASPMV_GPU_ENCODE = 4, /* translate to BCCOO/BCCOO+ on the GPU; no host arrays  */
  YASPMV_TICKET_IDS = 8, /* take logical tile ids from an atomic ticket (for GPUs
                            that dispatch workgroups out of order).  Default: tile =
                            workgroup id, relying on in-order dispatch as the paper does
                            ("Current GPUs dispatch workgroups in-order"); the
                            ticket then only yields the launch epoch                       */
  YASPMV_NO_PDL = 16,    /* launch without programmatic dependent launch (by default each
                            SpMV may start streaming its matrix tiles while the previous
                            kernel on the stream drains; x, y and carries wait for it)     */
  YASPMV_FORCE_HANDOFF = 32 /* testing: a tile always hands its carried first segment to the
                            predecessor hand-off protocol, even when the predecessor's
                            carry is already published (results are identical)            */
};

/* Tunable parameters, Table 1.  0 in any field = auto/default. */
typedef struct {
  int32_t block_h;     /* h in {1,2,3,4}     (Table 1 "Block height")            */
  int32_t block_w;     /* w in {1,2,4} (Table 1 "Block width"); 8 = extension */
  int32_t slices;      /* S >= 1; 1 = BCCOO, > 1 = BCCOO+ (P:307); S <= ceil(n/w) */
  int32_t thread_tile; /* T in {4,8,16,32}: non-zero blocks per thread       */
  int32_t cta_size;    /* C in {64,128,256,512}: threads per workgroup           */
  int32_t col_mode;    /* YASPMV_COL_*; U16 requires ceil(n/w) < 65535           */
  int32_t empty_mode;  /* YASPMV_EMPTY_*                                                  */
  int32_t flags;       /* YASPMV_KEEP_HOST | YASPMV_DROP_CSR | YASPMV_GPU_ENCODE         */
  int32_t result_cache; /* segmented-sum strategy (Table 1; §3.2.2-3.2.3):
                           0 = strategy 1 (intermediate sums in registers);
                           k in {1,2,4} = strategy 2 with a per-workgroup result cache of
                           k*C entries in shared memory, written back coalesced (P:274-278,
                           P:293).  Results agree within rounding (the first stop's sum is
                           associated differently).  yaspmv_reencode: 0 = keep current,
                           -1 = strategy 1.  A launch-time choice: no re-encode needed. */
  int32_t tiles_per_cta; /* consecutive workgroup-level tiles one CTA processes (B200
                           scheduling, not in Table 1): 0 = auto (2 when the matrix has
                           >= 32 waves of tiles, else 1), k in 1..64.  A warp that finishes
                           a tile issues the next tile's loads at once while the tile's
                           stores drain.  Results are bitwise identical for every k.
                           Launch-time (no re-encode); forced to 1 with YASPMV_TICKET_IDS. */
  /* Panel-sliced BCCOO+ (BCCOO+'s vertical slices, stacked
     inside each panel of R rows, slices of W columns placed relative to the panel): the
     entries of panel p with a column in [p*R + band_col0 - band, ... + KS*W), KS =
     ceil((R + 2*band)/W), go to the band stream, whose every gather is served from a
     W-value window of x in shared memory; the rest is a plain BCCOO/BCCOO+ matrix encoded
     with the fields above.  fp32, 1x1 blocks; not with the fused multi-GPU step. */
  int32_t band;        /* band half-width B in columns; 0 = off (plain format);
                          yaspmv_reencode: 0 = keep the handle's band fields, -1 = off      */
  int32_t panel_rows;  /* R: multiple of 256, <= 32768; 0 = 16384                        */
  int32_t slice_width; /* W: multiple of 4, <= 65532, KS <= 64; 0 = 16384                */
  int32_t band_col0;   /* column of row 0 (a row-partitioned rank: its first global row) */
  int32_t band_far;    /* where the entries outside the band go (reading P7):
                          YASPMV_FAR_SEPARATE = a plain BCCOO/BCCOO+ matrix run before the
                          band kernel (its S slices combined in the band kernel's prologue);
                          YASPMV_FAR_IN_PANEL = slice 0 of every panel: one BCCOO slice over
                          all n columns with int32 columns, gathered from global memory by
                          the band kernel itself (one launch per SpMV, no partial vectors;
                          on C5 its random gathers over all of x miss L2 far more often
                          than BCCOO+'s column slices: 10.0 vs 3.3 ms).
                          0 = YASPMV_FAR_SEPARATE; yaspmv_tune times both;
                          yaspmv_reencode: 0 = keep                                        */
} yaspmv_params;

enum { YASPMV_FAR_SEPARATE = 1, YASPMV_FAR_IN_PANEL = 2 };

typedef struct {
  int64_t m, n, nnz;         /* matrix shape and structural non-zeros after normalisation */
  int64_t MB, NB, SW;        /* block rows, block columns, block columns per slice        */
  int64_t nnzb;              /* stored blocks (incl. filler blocks), before padding       */
  int64_t nnzb_pad;          /* padded to a multiple of T*C                       */
  int64_t ntiles;            /* workgroup-level tiles = CTAs per SpMV launch              */
  int64_t n_stops;           /* row stops ('0' bits)                               */
  int64_t n_filler;          /* filler blocks (empty_mode FILLER)                         */
  int64_t n_zero_rows;       /* zero-filled stacked rows (empty_mode MAP)                 */
  int64_t format_bytes;      /* device bytes of the format read by one SpMV               */
  int64_t alg_bytes;         /* algorithmic bytes per SpMV: format + x + y (+ 2*S*M tmp)  */
  int64_t footprint_bytes;   /* Table-3 footprint: values + col + flag bits       */
  yaspmv_params params;      /* resolved parameters (no zeros)                            */
  int32_t dtype;             /* yaspmv_dtype                                               */
  int32_t device;            /* CUDA device ordinal, -1 for a host-only handle            */
  int32_t has_seg_row;       /* 1 if a seg_row map is stored                              */
  int32_t regs_per_thread;   /* registers of the selected SpMV kernel (0 if host-only)    */
  double build_seconds;      /* wall time of the last (re-)encode + upload                */
  double tune_seconds;       /* wall time of the last yaspmv_tune                         */
  int32_t tune_candidates;   /* candidates timed by the last yaspmv_tune                   */
  int32_t reserved;
  /* panel-sliced BCCOO+ (params.band > 0): the fields above describe the far part        */
  int64_t band_blocks;       /* band entries (1x1 blocks; FILLER blocks not included)     */
  int64_t band_blocks_pad;   /* after padding every panel to the band tile                */
  int64_t band_panels;       /* panels = CTAs of the band kernel                          */
  int64_t band_slices;       /* KS, slices per panel                                      */
  int64_t band_stops;        /* row stops of the band stream                              */
  int64_t band_format_bytes; /* device bytes of the band stream + its aux read by one SpMV
                                (included in format_bytes; the far part is the rest)       */
  int64_t band_far_blocks_pad; /* YASPMV_FAR_IN_PANEL: blocks of the panels' far slices
                                (incl. FILLER blocks and padding; part of band_blocks_pad);
                                its entries are nnz - band_blocks                          */
} yaspmv_info;

/* ---------------------------------------------------------------- build / free
 * yaspmv_build_csr: encode A (m x n, CSR) into BCCOO/BCCOO+ and upload it to `device`.
 *   row_ptr: host, int64[m+1], row_ptr[0] = 0, non-decreasing (borrowed for the call).
 *   col_idx: host, int32[nnz] in [0, n); rows may be unsorted and hold duplicates —
 *            entries are stably sorted by column and duplicates summed in input order
 *            (COO semantics); explicit zeros stay structural.
 *   vals:    host, float or double [nnz] per `dtype`.
 *   params:  NULL = defaults (h = w = S = 1, T = 16, C = 256, auto col / empty modes).
 *   device:  CUDA device ordinal, or -1 for a HOST-ONLY handle (encode only: usable by
 *            yaspmv_get_info / yaspmv_export, not by spmv).
 *   out:     receives the new handle; the caller frees it with yaspmv_free.
 * Errors: EINVAL (m, n < 0; NULL arrays with nnz > 0; index out of range; row_ptr not
 * monotone; parameter outside Table 1's ranges; U16 with NB >= 65535; S > NB),
 * ENOMEM, ECUDA, EUNSUPPORTED (no kernel compiled for (dtype, h, w, T, C)). */
yaspmv_status yaspmv_build_csr(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                               const void* vals, yaspmv_dtype dtype, const yaspmv_params* params,
                               int32_t device, yaspmv_matrix* out);

/* yaspmv_build_coo: as build_csr from COO triples (row_idx, col_idx, vals)[nnz], any order,
 * duplicates summed in input order (Q14). */
yaspmv_status yaspmv_build_coo(int64_t m, int64_t n, int64_t nnz, const int32_t* row_idx,
                               const int32_t* col_idx, const void* vals, yaspmv_dtype dtype,
                               const yaspmv_params* params, int32_t device, yaspmv_matrix* out);

/* yaspmv_free: releases every host and device array of A.  NULL-safe.  Must not be called
 * while work using A is still pending on a stream (synchronize first). */
void yaspmv_free(yaspmv_matrix A);

/* ---------------------------------------------------------------- SpMV
 * yaspmv_spmv: y := A·x  (overwrite; no alpha/beta).  Stream-ordered and asynchronous.
 *   x: device, n elements of A's dtype, aligned to w * sizeof(value) bytes.
 *   y: device, m elements; must not overlap x.
 * Deterministic: the same handle and x give a bitwise identical y.  One handle must not
 * run on two streams concurrently (it owns per-call scratch: ticket counter, carry
 * status words, BCCOO+ partial-result buffer).  Empty rows give y = 0 for every x (a FILLER
 * block names block column NB, where x reads 0: DESIGN.md Q3); a row inside a stored h x w
 * block reads the block's zero padding, 0 * x_j, so a non-finite x_j can reach
 * it when h > 1.
 * Kernels: the fused SpMV (multiply, per-thread segmented sum, CTA segmented scan,
 * decoupled look-back carries, write-back; §3) and, when S > 1, the slice
 * combine. */
yaspmv_status yaspmv_spmv(yaspmv_matrix A, const void* x, void* y, void* stream);

/* yaspmv_spmv_power: one step of the power iteration fused into the SpMV (not in the
 * paper; BASELINE.json's iterated SpMV):  y := (A·x) / sqrt(in_norm2[0])  (no scaling if
 * in_norm2 is NULL) and, if out_norm2 is not NULL, out_norm2[0] := sum_i y[i]^2 (fp64,
 * deterministic fixed-tree reduction).  in_norm2 / out_norm2 are DEVICE doubles.  With
 * z_k = A x_k, calling it on (z_{k-1}, ||z_{k-1}||^2) yields z_k and ||z_k||^2 without a
 * separate normalisation pass.  Launches: the SpMV (+ the BCCOO+ combine, which then does
 * the scaling and the partial sums) + two small reduction kernels. */
yaspmv_status yaspmv_spmv_power(yaspmv_matrix A, const void* x, void* y, const double* in_norm2, double* out_norm2,
                                void* stream);
int32_t yaspmv_launches_per_power_step(yaspmv_matrix A);

/* yaspmv_spmv_host: y := A·x with HOST x / y: copies x host->device into handle-owned
 * scratch, runs yaspmv_spmv, copies y device->host, and synchronizes `stream` before
 * returning.  Pinned host memory gives full PCIe/NVLink-C2C bandwidth. */
yaspmv_status yaspmv_spmv_host(yaspmv_matrix A, const void* x_host, void* y_host, void* stream);

/* yaspmv_spmv_host_async: y := A·x with HOST x / y, returning before completion.  Calls on
 * one handle overlap the host->device copy of call k+1, the SpMV of call k and the
 * device->host copy of call k-1 (three handle-owned device buffer pairs — with two, the
 * copy-in of call k would wait for the copy-out of call k-2 — two internal copy
 * streams, events chaining them to `stream`).  x_host must stay unchanged and y_host valid
 * until yaspmv_host_sync(A); pinned host memory is needed for the copies to overlap.
 * yaspmv_host_sync: waits for every outstanding yaspmv_spmv_host_async of the handle. */
yaspmv_status yaspmv_spmv_host_async(yaspmv_matrix A, const void* x_host, void* y_host, void* stream);
yaspmv_status yaspmv_host_sync(yaspmv_matrix A);

/* ---------------------------------------------------------------- tuning (§4)
 * yaspmv_tune: auto-tuner of PAPER.md §4: for the 4 block shapes with the
 * smallest footprint it times the SpMV over thread tile T, CTA size C, slice count
 * S and column mode with strategy 1, then strategy 2 with result cache sizes 1 and 2 (the
 * paper's pinned values) for every (T, C), then tiles_per_cta in {1, 2, 4} for the
 * winner, on the device (scratch x/y owned by the tuner), then re-encodes A with
 * the fastest parameters (ties within 1%: smaller footprint, then lexicographic).
 * Re-encoding needs the normalised CSR the handle keeps unless built with
 * YASPMV_DROP_CSR (then EINVAL).  On failure A keeps its previous parameters.
 * `chosen` (nullable, host) receives the selected parameters. */
yaspmv_status yaspmv_tune(yaspmv_matrix A, void* stream, yaspmv_params* chosen);
/* yaspmv_tune_ex: mode 0 = yaspmv_tune (the paper's pruned search); mode 1 = exhaustive
 * over every compiled block shape (the "exhaustive search" the paper compares its tuner
 * against). */
yaspmv_status yaspmv_tune_ex(yaspmv_matrix A, void* stream, yaspmv_params* chosen, int32_t mode);

/* yaspmv_reencode: re-encode A with new parameters (0 fields — flags included — keep the
 * current value; see
 * result_cache for its -1).  A change of result_cache / tiles_per_cta alone only
 * re-selects the launch (no re-encode). */
yaspmv_status yaspmv_reencode(yaspmv_matrix A, const yaspmv_params* params);

/* ---------------------------------------------------------------- introspection
 * yaspmv_get_info: fills *out (host). */
yaspmv_status yaspmv_get_info(yaspmv_matrix A, yaspmv_info* out);

/* Canonical (un-permuted) encoded arrays, SURVEY §8(c) E1-E9:
 *  FLAGS      uint8 [nnzb_pad/8]  bit flags, 0 = row stop, LSB-first, pad bits 1
 *  COL        uint16 [nnzb_pad] (COL_U16) or int32 [nnzb_pad] (I32 / DELTA16 escape array)
 *  COL_DELTA  int16 [nnzb_pad]    segmented difference per thread tile, -1 = escape
 *  VAL0..3    value array r [nnzb_pad*w] of A's dtype
 *  SEG_ROW    int32 [n_stops]     stacked block row of each row stop (empty_mode MAP)
 *  ZERO_ROWS  int32 [n_zero_rows] stacked block rows without blocks (empty_mode MAP)
 *  CTA_SEG0   int32 [ntiles]      row stops before each workgroup tile
 *  FRE        int32 [ntiles*C]    first-result entry of each thread (Fig. 6b) */
enum {
  YASPMV_ARR_FLAGS = 0, YASPMV_ARR_COL = 1, YASPMV_ARR_COL_DELTA = 2,
  YASPMV_ARR_VAL0 = 3, YASPMV_ARR_VAL1 = 4, YASPMV_ARR_VAL2 = 5, YASPMV_ARR_VAL3 = 6,
  YASPMV_ARR_SEG_ROW = 7, YASPMV_ARR_ZERO_ROWS = 8, YASPMV_ARR_CTA_SEG0 = 9, YASPMV_ARR_FRE = 10,
  /* panel-sliced BCCOO+ band stream (params.band > 0; readings P1-P7 of DESIGN.md §2.1).
   * A panel holds NS = KS slices, or NS = KS + 1 with YASPMV_FAR_IN_PANEL, whose slice 0 is
   * the far slice (reading P7) and whose band slices are 1..KS; F = band_far_blocks_pad:
   *  BAND_FLAGS      uint8 [band_blocks_pad/8]  0 = last block of its row in its slice
   *  BAND_COL16      uint16 [band_blocks_pad - F] band blocks only: column - (p*R + col0 - B)
   *                  - k*W; W = FILLER block (value 0) of an empty row inside the slice's rows
   *  BAND_VAL        value [band_blocks_pad]
   *  BAND_PANEL_BLK0 int64 [panels + 1]         first block of each panel
   *  BAND_SLICE_PTR  int32 [panels * (NS+1)]    block offset of slice k inside its panel (padded)
   *  BAND_STOP_PTR   int32 [panels * (NS+1)]    row stops before slice k inside its panel
   *  BAND_FIRST_ROW  int32 [panels * NS]        first non-empty row of each slice (the s-th
   *                                              row stop of the slice is row first_row + s)
   *  BAND_TILE_RANK  int32 [band_blocks_pad/512] stops before each 512-block tile in its slice
   *  BAND_FAR_COL    int32 [F]                  far-slice blocks only: column; n = FILLER
   *  BAND_FAR_BLK0   int64 [panels + 1]         far-slice blocks before each panel
   *  (every slice is padded to a multiple of 512 blocks = 16 blocks x 32 threads; block b of
   *  panel p is the (b - far_blk0[p+1])-th BAND_COL16 entry if it belongs to a band slice, the
   *  (b - band blocks before p)-th BAND_FAR_COL entry if to the far slice) */
  YASPMV_ARR_BAND_FLAGS = 11, YASPMV_ARR_BAND_COL16 = 12, YASPMV_ARR_BAND_VAL = 13,
  YASPMV_ARR_BAND_PANEL_BLK0 = 14, YASPMV_ARR_BAND_SLICE_PTR = 15, YASPMV_ARR_BAND_STOP_PTR = 16,
  YASPMV_ARR_BAND_FIRST_ROW = 17, YASPMV_ARR_BAND_TILE_RANK = 18, YASPMV_ARR_BAND_FAR_COL = 19,
  YASPMV_ARR_BAND_FAR_BLK0 = 20
};

/* yaspmv_export: copy canonical array `which` into host_dst (capacity `bytes`).  Returns
 * the array's byte size in *nbytes (nullable).  host_dst may be NULL to query the size.
 * Needs YASPMV_KEEP_HOST (or a host-only handle) except for CTA_SEG0 / FRE.
 * yaspmv_export_device: the same array read back FROM THE DEVICE copy and un-permuted
 * from the device layout (checks the uploaded arrays; device handles only). */
yaspmv_status yaspmv_export(yaspmv_matrix A, int32_t which, void* host_dst, int64_t bytes, int64_t* nbytes);
yaspmv_status yaspmv_export_device(yaspmv_matrix A, int32_t which, void* host_dst, int64_t bytes,
                                   int64_t* nbytes);
/* yaspmv_export_device_range: as yaspmv_export_device for the workgroup tiles
 * [first_tile, first_tile + ntiles) only (per-block arrays: the tiles' T*C blocks — 512 for the
 * band stream; CTA_SEG0 / BAND_TILE_RANK: those tiles' entries), for checking windows of
 * matrices whose full arrays are too large to copy.  BAND_COL16 / BAND_FAR_COL count tiles
 * of their own arrays (band-slice tiles / far-slice tiles). */
yaspmv_status yaspmv_export_device_range(yaspmv_matrix A, int32_t which, int64_t first_tile, int64_t ntiles,
                                         void* host_dst, int64_t bytes, int64_t* nbytes);

/* ---------------------------------------------------------------- power-iteration helpers
 * yaspmv_nrm2sq: out_dev[0] (device double) := sum_i v[i]^2 over device v[n] of `dtype`,
 *   accumulated in fp64, deterministic (fixed reduction tree).  scratch_dev: device,
 *   >= yaspmv_nrm2sq_scratch_bytes(n) bytes, zero-initialised once by the caller.
 * yaspmv_scale: dst[i] := src[i] / sqrt(norm2_dev[0]) (device; dst may equal src). */
yaspmv_status yaspmv_nrm2sq(const void* v, int64_t n, yaspmv_dtype dtype, double* out_dev, void* scratch_dev,
                            void* stream);
int64_t yaspmv_nrm2sq_scratch_bytes(int64_t n);
yaspmv_status yaspmv_scale(const void* src, void* dst, int64_t n, yaspmv_dtype dtype, const double* norm2_dev,
                           void* stream);

/* ---------------------------------------------------------------- fused multi-GPU power step
 * Iterated SpMV with A row-partitioned over P ranks (one process or one handle per GPU)
 * and x replicated (BASELINE.json north_star; not in the
 * paper, whose method is single-GPU).  Instead of "SpMV, then an all-gather of y"
 * the SpMV's write-back stores every finished row of z_k straight into ALL ranks' copies of
 * the next x over peer memory (NVLink P2P stores through CUDA IPC mappings), tile by tile,
 * so the exchange overlaps the SpMV; a one-warp publish kernel then posts the rank's
 * ||z_k||^2 partial and an epoch flag into every peer's signal pad (system-scope release),
 * and the next step's one-warp wait kernel acquires all P flags before x is read.
 *
 * A yaspmv_comm owns ONE device allocation on its rank's device (so one IPC handle maps it):
 *   xbuf[2][n_padded] of dtype   the replicated x, double-buffered by step parity
 *   signal pad                    per source rank: epoch flag (u64), ||z||^2 partials (f64)[2]
 * Rank r's rows are the padded chunk [r*chunk, r*chunk + m_r) of x (dist.remap_columns
 * maps the matrix columns into that padded space; pad entries are zero and never read).
 *
 * Protocol (all ranks call the same sequence; seq = steps issued on this comm so far):
 *   yaspmv_comm_create          on every rank;
 *   yaspmv_comm_ipc_handle      -> exchange the 64-byte handles (e.g. torch all_gather_object)
 *   yaspmv_comm_open_ipc        maps every peer (cudaIpcMemLazyEnablePeerAccess), or
 *   yaspmv_comm_connect_local   same-process peers (tests: P ranks as P handles on 1 GPU);
 *   write x_0 (replicated) into yaspmv_comm_x(c, 0) on every rank, yaspmv_comm_begin(c),
 *   then a host barrier across ranks (every rank's x_0 and peers' buffers ready);
 *   yaspmv_power_step_fused     repeatedly: step k reads xbuf[k%2] (z_{k-1}, or x_0 right
 *                               after begin) and computes z_k = A_r x / ||z_{k-1}|| (no
 *                               scaling right after begin) into every rank's xbuf[(k+1)%2];
 *                               for k after begin it first waits (on the device) for every
 *                               peer's step k-1;
 *   yaspmv_comm_wait            waits for every peer's latest step and writes the total
 *                               ||z||^2 (fp64, summed in rank order: identical on all ranks)
 *                               into the device double yaspmv_comm_norm2_device(c).
 * Deterministic: bitwise identical to running yaspmv_spmv_power per rank on the gathered x
 * with the norms summed in rank order.  The device waits time out after `timeout_ms`
 * (yaspmv_comm_create; 0 = 60 s): the wait kernel then gives up, and the next
 * yaspmv_comm_check reports YASPMV_ECUDA instead of hanging the GPU.
 * A comm and the matrices stepped with it must live on the same device; A's column count
 * must equal n_padded, A's row count must be <= chunk.  world <= YASPMV_MAX_RANKS. */
#define YASPMV_MAX_RANKS 8
typedef struct yaspmv_comm_s* yaspmv_comm;
yaspmv_status yaspmv_comm_create(int32_t device, int32_t rank, int32_t world, int64_t chunk, yaspmv_dtype dtype,
                                 int32_t timeout_ms, yaspmv_comm* out);
/* out: host buffer of >= 64 bytes (a cudaIpcMemHandle_t of the comm's allocation). */
yaspmv_status yaspmv_comm_ipc_handle(yaspmv_comm c, void* out, int64_t bytes);
/* handles: host, world * 64 bytes, rank order (this rank's own entry is ignored). */
yaspmv_status yaspmv_comm_open_ipc(yaspmv_comm c, const void* handles, int64_t bytes);
/* peers: host array of `world` comms of this process on the same device, rank order. */
yaspmv_status yaspmv_comm_connect_local(yaspmv_comm c, const yaspmv_comm* peers, int32_t world);
/* device pointer of x buffer (seq + which) % 2: which = 0 is the next step's input (after a
 * completed step: the latest z), 1 the buffer the next step writes. */
void* yaspmv_comm_x(yaspmv_comm c, int32_t which);
/* the next step reads x_0 unscaled and does not wait for peers (see the protocol). */
yaspmv_status yaspmv_comm_begin(yaspmv_comm c);
yaspmv_status yaspmv_power_step_fused(yaspmv_matrix A, yaspmv_comm c, void* stream);
yaspmv_status yaspmv_comm_wait(yaspmv_comm c, void* stream);
double* yaspmv_comm_norm2_device(yaspmv_comm c);
int64_t yaspmv_comm_seq(yaspmv_comm c);
/* reports (and clears) a device-side wait timeout of an earlier step; synchronizes nothing. */
yaspmv_status yaspmv_comm_check(yaspmv_comm c);
int32_t yaspmv_launches_per_fused_step(yaspmv_matrix A);
/* NVSwitch multicast for the fused step (not in the paper): instead of P
 * stores of every finished row (one per rank's copy of x), ONE multimem.st through a
 * multicast object to which every rank's x buffers are bound — the switch replicates it.
 * Optional, after open_ipc / connect_local (the signal pads stay peer-mapped):
 *   yaspmv_comm_mc_supported(device)  1 if the device reports switch multicast;
 *   one rank: yaspmv_comm_mc_create(c, &fd)  multicast object for `world` devices, exported
 *             as a POSIX file descriptor of the calling process (*fd_out);
 *   the others: yaspmv_comm_mc_import(c, pid, fd)  the creator's pid and fd (duplicated with
 *             pidfd_getfd, Linux >= 5.6; pid <= 0 or this process: dup(fd));
 *   every rank: yaspmv_comm_mc_add_device(c); host barrier; yaspmv_comm_mc_bind(c) (allocates
 *             2 x buffers of physical memory, binds them, maps them locally and through the
 *             multicast object, copies the current x buffers in); host barrier.
 * After bind, yaspmv_comm_x returns the bound buffers and every fused step stores through
 * the multicast mapping.  Errors: YASPMV_EUNSUPPORTED without switch multicast or driver
 * entry points, YASPMV_ECUDA with the CUresult of a failing driver call; a failed sequence
 * leaves the comm on peer stores (mc_active = 0); if another rank failed, every rank that
 * did bind calls yaspmv_comm_mc_release (dist.FusedPowerIteration does). */
int32_t yaspmv_comm_mc_supported(int32_t device);
yaspmv_status yaspmv_comm_mc_create(yaspmv_comm c, int64_t* fd_out);
yaspmv_status yaspmv_comm_mc_import(yaspmv_comm c, int64_t pid, int64_t fd);
yaspmv_status yaspmv_comm_mc_add_device(yaspmv_comm c);
yaspmv_status yaspmv_comm_mc_bind(yaspmv_comm c);
int32_t yaspmv_comm_mc_active(yaspmv_comm c);
/* back to peer stores after a bind (e.g. another rank's bind failed): the x buffers' contents
 * return to the peer-mapped allocation; the multicast mappings stay until yaspmv_comm_free. */
yaspmv_status yaspmv_comm_mc_release(yaspmv_comm c);
/* NULL-safe; unmaps the peers and frees the allocation (synchronize first; peers must not
 * write into this comm any more). */
void yaspmv_comm_free(yaspmv_comm c);

/* ---------------------------------------------------------------- misc */
const char* yaspmv_last_error(void);
const char* yaspmv_version(void);
/* L2 set-aside for persisting accesses on `device` (cudaLimitPersistingL2CacheSize; a
 * device-wide setting of the calling process — the library never changes it on its own).
 * The kernels' x gathers are evict_last accesses (the paper's cached x): on C5 the far
 * part's BCCOO+ slices of x (67 MB at S = 3) keep more of themselves in L2 with a 60 MB
 * set-aside.  bytes is clamped to the device maximum; *set_bytes (nullable)
 * receives the value now in effect.  Errors: YASPMV_EINVAL (bad device, bytes < 0),
 * YASPMV_ECUDA. */
yaspmv_status yaspmv_l2_persist(int32_t device, int64_t bytes, int64_t* set_bytes);
/* Per-kernel device timing (measurement only; bench.py's roofline).  yaspmv_profile_begin
 * makes every later SpMV on A record CUDA events on its stream around its kernel groups:
 * stage 0 = the plain BCCOO/BCCOO+ part (K1, + combine, + its y^2 sum), stage 1 = the band
 * kernel of a panel-sliced handle (K4), stage 2 = K4's y^2 sum.  yaspmv_profile_end
 * synchronizes those events, writes the summed milliseconds of stage s to ms[s] (s < n,
 * n <= 3) and the number of profiled calls to *calls (nullable), and stops profiling. */
yaspmv_status yaspmv_profile_begin(yaspmv_matrix A);
yaspmv_status yaspmv_profile_end(yaspmv_matrix A, double* ms, int32_t n, int64_t* calls);
/* Kernel launches issued by the last yaspmv_spmv on this handle (1, or 2 with S > 1). */
int32_t yaspmv_launches_per_spmv(yaspmv_matrix A);
/* Debug spin bound: with the environment variable YASPMV_SPIN_LIMIT=N (> 0, read
 * once per process) a carry look-back that polls its predecessors' status words
 * more than N times traps the kernel instead of hanging (the stream reports
 * cudaErrorLaunchFailure, sticky for the process) after writing the waiting tile id to
 * mapped host memory.  Returns that tile id, or -1 if no bound was hit (or none is set). */
int64_t yaspmv_debug_spin_tile(void);

#ifdef __cplusplus
}
#endif
#endif /* YASPMV_H */
