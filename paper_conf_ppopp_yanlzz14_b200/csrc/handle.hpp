// handle.hpp — the opaque yaspmv_matrix handle (internal; not part of the ABI).
#pragma once

#include <cuda_runtime.h>

#include <array>
#include <vector>

#include "common.hpp"
#include "panel.hpp"

using yaspmv::CSR;
using yaspmv::Canonical;
using yaspmv::KernelEntry;

struct DevArrays {
  void* val[4] = {nullptr, nullptr, nullptr, nullptr};
  void* col = nullptr;
  int32_t* col32 = nullptr;
  uint8_t* flags = nullptr;
  int32_t* cta_seg0 = nullptr;
  int32_t* seg_row = nullptr;
  int32_t* zero_rows = nullptr;
  unsigned long long* ticket = nullptr;
  unsigned long long* status = nullptr;
  double* carry = nullptr;
  unsigned long long* bnd = nullptr;  // per tile boundary: hand-off word of the carried segment
  double* pend_val = nullptr;         // per tile: the waiting first segment's partial (h fp64)
  long long* pend_row = nullptr;      // per tile: its output row
  void* tmp = nullptr;
  void free_all() {
    void* ps[] = {val[0], val[1], val[2], val[3], col, col32, flags, cta_seg0, seg_row, zero_rows,
                  ticket, status, carry, bnd, pend_val, pend_row, tmp};
    for (void* p : ps)
      if (p) cudaFree(p);
    *this = DevArrays();
  }
};

struct yaspmv_matrix_s {
  int device = -1;
  int dtype = 0;
  int vsize = 4;
  CSR csr;
  bool have_csr = false;
  Canonical can;
  bool have_host_arrays = false;
  DevArrays d;
  const KernelEntry* kern = nullptr;
  int regs = 0;
  int64_t grid = 1;  // CTAs per launch
  int tpc = 1;       // resolved tiles per CTA (params.tiles_per_cta; block-id mode only)
  void* xs = nullptr;  // scratch for spmv_host
  void* ys = nullptr;
  // spmv_host_async: three buffer slots (H2D of call k+1, SpMV of call k and D2H of call k-1
  // in flight with no slot reuse stalling the pipeline), two copy streams, chaining events
  struct HostSlot {
    void* x = nullptr;
    void* y = nullptr;
    cudaEvent_t in = nullptr, comp = nullptr, done = nullptr;
  } hslot[3];
  cudaStream_t s_in = nullptr, s_out = nullptr;
  int next_slot = 0;
  double* d_part = nullptr;     // power-iteration epilogue: partials of sum y^2
  double* d_scratch = nullptr;  // two-level reduction scratch
  int64_t npart = 0;
  int64_t* d_dep_row = nullptr;  // ablation: carried segment row per tile
  int64_t abl_ntiles = 0;
  int64_t n_escapes = 0;
  double build_s = 0, tune_s = 0;
  int tune_candidates = 0;
  int64_t nnz_total = 0;          // structural non-zeros of A (far + band)
  // panel-sliced BCCOO+ band part (params.band > 0); can/d then hold the far part
  bool band_on = false;
  yaspmv::PanelCanonical pan;     // host arrays (kept with YASPMV_KEEP_HOST / host-only)
  yaspmv::PanelDev pd;
  bool have_pan_host = false;
  int pan_regs = 0;
  // yaspmv_profile_*: events around the kernel groups of every SpMV while profiling
  bool prof_on = false;
  std::vector<std::array<cudaEvent_t, 4>> prof_ev;
  ~yaspmv_matrix_s() {
    if (device >= 0) {
      int cur = 0;
      cudaGetDevice(&cur);
      cudaSetDevice(device);
      d.free_all();
      if (xs) cudaFree(xs);
      if (ys) cudaFree(ys);
      if (s_out) cudaStreamSynchronize(s_out);
      for (auto& s : hslot) {
        if (s.x) cudaFree(s.x);
        if (s.y) cudaFree(s.y);
        if (s.in) cudaEventDestroy(s.in);
        if (s.comp) cudaEventDestroy(s.comp);
        if (s.done) cudaEventDestroy(s.done);
      }
      if (s_in) cudaStreamDestroy(s_in);
      if (d_part) cudaFree(d_part);
      if (d_dep_row) cudaFree(d_dep_row);
      if (d_scratch) cudaFree(d_scratch);
      pd.free_all();
      for (auto& ev : prof_ev)
        for (cudaEvent_t e : ev)
          if (e) cudaEventDestroy(e);
      if (s_out) cudaStreamDestroy(s_out);
      cudaSetDevice(cur);
    }
  }
};

// capi.cpp: make an already encoded Canonical the handle's encoding (kernel + upload)
yaspmv_status install_canonical(yaspmv_matrix A, Canonical&& c, int flags);
// capi.cpp: one power-iteration SpMV whose output goes to peers.p[q] (q < peers.n) instead
// of a local y (the fused exchange of comm.cu); out_norm2 receives sum y^2 (nullable)
yaspmv_status run_spmv_peers(yaspmv_matrix A, const void* x, const double* in_norm2, double* out_norm2,
                             const yaspmv::PeerOut& peers, void* stream);
// capi.cpp: switch the launch-time parameters (result_cache, tiles_per_cta; 0 = auto) of an
// encoded handle
yaspmv_status set_launch(yaspmv_matrix A, int rc, int tpc);
