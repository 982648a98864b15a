// panel.hpp — the panel-sliced BCCOO+ part of an encoding (readings P1-P6).
//
// BCCOO+ (§2.3) stacks vertical slices of the matrix top-down so that
// the rows of one slice share one part of x.  The panel variant does that inside
// every horizontal panel of R rows, with slices of W columns placed relative to the panel
// (column base cb(p) = p*R + col0 - B), so that one slice's part of x — W values — fits in
// a CTA's shared memory and every gather of the slice is served from there instead of one
// 32-byte L2 request per non-zero (profiles/r02_gather_microbench.md).  Entries outside
// their panel's band [cb(p), cb(p) + KS*W) form an ordinary BCCOO matrix (the "far part",
// encoded and run by the existing path).  y = A_far x, then each panel's slices in
// ascending order add their segment sums (the BCCOO+ combine order, Q11) — in
// shared memory, so BCCOO+'s temporary buffer never reaches HBM.
#pragma once

#include <cstdint>
#include <vector>

#include "../../include/yaspmv.h"

namespace yaspmv {

// band stream: workgroup-level tiles of BT blocks x WT threads (one warp), every slice
// padded to a whole number of tiles (reading P4); the kernel runs CTA threads per panel
constexpr int PANEL_BT = 16;
constexpr int PANEL_WT = 32;
constexpr int PANEL_TC = PANEL_BT * PANEL_WT;
constexpr int PANEL_CTA = 640;       // 20 warps, <= 96 registers; C5 band kernel after the round-2
                                      // changes, 640 / 704 / 768 / 896 / 1024 threads -> 1.875 (R =
                                      // 16128) / 1.99 / 1.91 / 1.94 / 2.28 ms (YASPMV_PANEL_CTA)
constexpr int PANEL_MAX_KS = 64;      // slices per panel
constexpr int PANEL_NBUF = 2;         // x windows resident per CTA (current + next slice)


struct PanelGeom {
  int64_t R = 0, W = 0, B = 0, col0 = 0;  // panel rows, slice width, band half-width, column of row 0
  int64_t KS = 0;                         // band slices per panel = ceil((R + 2B) / W)
  int64_t npanels = 0;
  int fip = 0;                            // 1: far entries as slice 0 of every panel (reading P7)
  int64_t NS() const { return KS + fip; } // slices per panel
};

// host arrays (canonical layout, like Canonical for the plain format)
struct PanelCanonical {
  PanelGeom g;
  int64_t nband = 0, nfill = 0, nband_pad = 0, n_stops = 0;
  int64_t nfar_pad = 0;             // P7: blocks of the far slices (incl. fillers and padding)
  std::vector<uint8_t> flags;       // nband_pad / 8, LSB-first, 0 = last entry of its row in its slice
  std::vector<uint16_t> col16;      // nband_pad - nfar_pad band blocks: column - cb(p) - k*W (W: FILLER)
  std::vector<int32_t> far_col;     // P7: nfar_pad far-slice blocks: column (n: FILLER block)
  std::vector<int64_t> far_blk0;    // P7: npanels + 1, far-slice blocks before each panel
  std::vector<uint8_t> val;         // nband_pad values (raw bytes)
  std::vector<int64_t> panel_blk0;  // npanels + 1
  std::vector<int32_t> slice_ptr;   // npanels * (NS + 1)
  std::vector<int32_t> stop_ptr;    // npanels * (NS + 1)
  std::vector<int32_t> first_row;   // npanels * NS: first non-empty row of each slice (panel-relative)
  std::vector<int32_t> tile_rank;   // nband_pad / TC: stops before each tile inside its slice
  void release_arrays() {
    std::vector<uint8_t>().swap(flags);
    std::vector<uint16_t>().swap(col16);
    std::vector<int32_t>().swap(far_col);
    std::vector<int64_t>().swap(far_blk0);
    std::vector<uint8_t>().swap(val);
    std::vector<int64_t>().swap(panel_blk0);
    std::vector<int32_t>().swap(slice_ptr);
    std::vector<int32_t>().swap(stop_ptr);
    std::vector<int32_t>().swap(first_row);
    std::vector<int32_t>().swap(tile_rank);
  }
};

struct PanelDev {
  void* col16 = nullptr;        // device layout (tile transpose)
  void* val = nullptr;          // device layout
  uint8_t* flags = nullptr;     // canonical bit stream
  int64_t* panel_blk0 = nullptr;
  int32_t* slice_ptr = nullptr;
  int32_t* stop_ptr = nullptr;
  int32_t* first_row = nullptr;
  int32_t* tile_rank = nullptr;
  void* far_col = nullptr;      // P7: device layout (tile transpose), int32
  int64_t* far_blk0 = nullptr;  // P7
  double* part = nullptr;       // per panel: sum of y^2 (power-iteration epilogue)
  double* scratch = nullptr;
  void free_all();
};

struct CSR;
// split the normalised CSR A into the far part (owned CSR, all of A's rows) and the band
// part (panel-sliced canonical arrays); R, W, B, col0 validated by the caller
yaspmv_status encode_panel(const CSR& A, const PanelGeom& g, CSR& far, PanelCanonical& out);

struct PanelArgs {
  const void* col16;
  const void* val;
  const uint8_t* flags;
  const int64_t* panel_blk0;
  const int32_t* slice_ptr;
  const int32_t* stop_ptr;
  const int32_t* first_row;
  const int32_t* tile_rank;
  const void* far_col;       // P7 (fip): int32 columns of the far-slice blocks, device layout
  const int64_t* far_blk0;   // P7 (fip): far-slice blocks before each panel
  int fip;                   // 1: slice 0 of every panel is its far slice (KS counts it)
  const void* x;
  void* y;            // out: y = A x (scaled by the epilogue)
  // the far part's result: ninit partial vectors init + s * init_stride (s < ninit), summed in
  // ascending s in fp64 — the BCCOO+ slice combine (Q11) folded into the band kernel
  const void* init;
  int ninit;
  int64_t init_stride;
  int64_t m, n;
  int64_t R, W, B, col0, KS, npanels;
  int epi;            // bit 0: scale by 1/sqrt(*in_norm2); bit 1: part[p] = sum over the panel of y^2
  int pdl;            // launched as a programmatic dependent of the far kernel (see launch_panel)
  const double* in_norm2;
  double* part;
  // fused exchange (yaspmv_power_step_fused): npeer > 0 writes y to peer_out[q] for q < npeer
  // (every rank's copy of the next x) instead of y; peer_mc: peer_out[0] is a multicast
  // address (one multimem.st per element)
  int npeer = 0;
  int peer_mc = 0;
  void* peer_out[YASPMV_MAX_RANKS] = {};
};
// panel_kernel.cu
int launch_panel(const PanelArgs& a, int dtype, void* stream);  // returns cudaError_t
size_t panel_smem_bytes(int64_t R, int64_t W);
int panel_attr(int64_t R, int64_t W, int* regs);                // cudaError_t; regs of the kernel

}  // namespace yaspmv
