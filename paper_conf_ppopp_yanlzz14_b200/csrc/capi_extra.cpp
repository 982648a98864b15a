// capi_extra.cpp — export / introspection of the encoded arrays, the auto-tuner of
// PAPER.md §4, and the power-iteration helpers.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <string>
#include <tuple>
#include <vector>

#include "handle.hpp"
#include "trace.hpp"

using namespace yaspmv;

#define CUDA_TRY(expr)                                                                       \
  do {                                                                                       \
    cudaError_t _e = (expr);                                                                 \
    if (_e != cudaSuccess)                                                                   \
      return fail(_e == cudaErrorMemoryAllocation ? YASPMV_ENOMEM : YASPMV_ECUDA,            \
                  std::string(#expr) + ": " + cudaGetErrorString(_e));                       \
  } while (0)

namespace {

// first-result entry of every thread (Fig. 6b): stops before its thread tile
void compute_fre(const Canonical& c, const uint8_t* flags, const int32_t* cta_seg0, std::vector<int32_t>& fre) {
  const int T = c.p.T, C = c.p.C;
  fre.assign((size_t)c.ntiles * C, 0);
  for (int64_t k = 0; k < c.ntiles; ++k) {
    int64_t acc = cta_seg0[k];
    for (int t = 0; t < C; ++t) {
      fre[(size_t)k * C + t] = (int32_t)acc;
      const int64_t b0 = (k * C + t) * (int64_t)T;
      for (int b = 0; b < T; ++b) acc += !((flags[(b0 + b) >> 3] >> ((b0 + b) & 7)) & 1);
    }
  }
}

struct ArrDesc {
  int64_t bytes = 0;
  int ptb = 0;            // >0: stored permuted on the device with this per-thread byte run
  const void* host = nullptr;
  const void* dev = nullptr;
  int64_t ntiles = -1;    // device layout tiles / threads (-1: the plain format's)
  int C = 0;
  bool band = false;      // a band-stream array (host copy: A->pan)
};

yaspmv_status describe(yaspmv_matrix A, int which, ArrDesc& d) {
  const Canonical& c = A->can;
  const Params& p = c.p;
  d = ArrDesc();
  switch (which) {
    case YASPMV_ARR_FLAGS:
      d.bytes = c.nnzb_pad / 8;
      d.host = c.flags.data();
      d.dev = A->d.flags;
      break;
    case YASPMV_ARR_COL:
      if (p.col_mode == COL_U16) {
        d.bytes = c.nnzb_pad * 2;
        d.host = c.col16.data();
        d.dev = A->d.col;
        d.ptb = 2 * p.T;
      } else {
        d.bytes = c.nnzb_pad * 4;
        d.host = c.col32.data();
        d.dev = p.col_mode == COL_I32 ? A->d.col : (const void*)A->d.col32;
        d.ptb = p.col_mode == COL_I32 ? 4 * p.T : 0;
      }
      break;
    case YASPMV_ARR_COL_DELTA:
      if (p.col_mode != COL_DELTA) return fail(YASPMV_EINVAL, "no delta array: col_mode is not DELTA16");
      d.bytes = c.nnzb_pad * 2;
      d.host = c.delta.data();
      d.dev = A->d.col;
      d.ptb = 2 * p.T;
      break;
    case YASPMV_ARR_VAL0:
    case YASPMV_ARR_VAL1:
    case YASPMV_ARR_VAL2:
    case YASPMV_ARR_VAL3: {
      const int r = which - YASPMV_ARR_VAL0;
      if (r >= p.h) return fail(YASPMV_EINVAL, "value array index >= block height");
      d.bytes = c.nnzb_pad * p.w * A->vsize;
      d.host = c.val[r].data();
      d.dev = A->d.val[r];
      d.ptb = p.T * p.w * A->vsize;
      break;
    }
    case YASPMV_ARR_SEG_ROW:
      d.bytes = c.has_seg_row ? c.n_stops * 4 : 0;
      d.host = c.seg_row.data();
      d.dev = A->d.seg_row;
      break;
    case YASPMV_ARR_ZERO_ROWS:
      d.bytes = c.n_zero * 4;
      d.host = c.zero_rows.data();
      d.dev = A->d.zero_rows;
      break;
    case YASPMV_ARR_CTA_SEG0:
      d.bytes = c.ntiles * 4;
      d.host = c.cta_seg0.data();
      d.dev = A->d.cta_seg0;
      break;
    case YASPMV_ARR_FRE:
      d.bytes = c.ntiles * p.C * 4;
      break;
    default: {
      if (which < YASPMV_ARR_BAND_FLAGS || which > YASPMV_ARR_BAND_FAR_BLK0) return fail(YASPMV_EINVAL, "unknown array id");
      if (!A->band_on) return fail(YASPMV_EINVAL, "no band stream: the handle is not panel-sliced (band = 0)");
      const PanelCanonical& q = A->pan;
      const PanelGeom& g = q.g;
      const int64_t NS = g.NS();
      if ((which == YASPMV_ARR_BAND_FAR_COL || which == YASPMV_ARR_BAND_FAR_BLK0) && !g.fip)
        return fail(YASPMV_EINVAL, "no far slices: the handle's band_far is YASPMV_FAR_SEPARATE");
      d.band = true;
      d.ntiles = q.nband_pad / PANEL_TC;
      d.C = PANEL_WT;
      switch (which) {
        case YASPMV_ARR_BAND_FLAGS:
          d.bytes = q.nband_pad / 8; d.host = q.flags.data(); d.dev = A->pd.flags; break;
        case YASPMV_ARR_BAND_COL16:
          d.bytes = (q.nband_pad - q.nfar_pad) * 2; d.host = q.col16.data(); d.dev = A->pd.col16; d.ptb = 2 * PANEL_BT;
          d.ntiles = (q.nband_pad - q.nfar_pad) / PANEL_TC;
          break;
        case YASPMV_ARR_BAND_FAR_COL:
          d.bytes = q.nfar_pad * 4; d.host = q.far_col.data(); d.dev = A->pd.far_col; d.ptb = 4 * PANEL_BT;
          d.ntiles = q.nfar_pad / PANEL_TC;
          break;
        case YASPMV_ARR_BAND_FAR_BLK0:
          d.bytes = (g.npanels + 1) * 8; d.host = q.far_blk0.data(); d.dev = A->pd.far_blk0; break;
        case YASPMV_ARR_BAND_VAL:
          d.bytes = q.nband_pad * A->vsize; d.host = q.val.data(); d.dev = A->pd.val; d.ptb = PANEL_BT * A->vsize;
          break;
        case YASPMV_ARR_BAND_PANEL_BLK0:
          d.bytes = (g.npanels + 1) * 8; d.host = q.panel_blk0.data(); d.dev = A->pd.panel_blk0; break;
        case YASPMV_ARR_BAND_SLICE_PTR:
          d.bytes = g.npanels * (NS + 1) * 4; d.host = q.slice_ptr.data(); d.dev = A->pd.slice_ptr; break;
        case YASPMV_ARR_BAND_STOP_PTR:
          d.bytes = g.npanels * (NS + 1) * 4; d.host = q.stop_ptr.data(); d.dev = A->pd.stop_ptr; break;
        case YASPMV_ARR_BAND_FIRST_ROW:
          d.bytes = g.npanels * NS * 4; d.host = q.first_row.data(); d.dev = A->pd.first_row; break;
        default:
          d.bytes = q.nband_pad / PANEL_TC * 4; d.host = q.tile_rank.data(); d.dev = A->pd.tile_rank; break;
      }
    }
  }
  return YASPMV_OK;
}

double now_s() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

}  // namespace

extern "C" {

yaspmv_status yaspmv_export(yaspmv_matrix A, int32_t which, void* dst, int64_t bytes, int64_t* nbytes) {
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  ArrDesc d;
  yaspmv_status st = describe(A, which, d);
  if (st != YASPMV_OK) return st;
  if (nbytes) *nbytes = d.bytes;
  if (!dst) return YASPMV_OK;
  if (bytes < d.bytes) return fail(YASPMV_EINVAL, "destination too small");
  if (which == YASPMV_ARR_FRE) {
    if (!A->have_host_arrays) return fail(YASPMV_EINVAL, "FRE needs the host flags (YASPMV_KEEP_HOST)");
    std::vector<int32_t> fre;
    compute_fre(A->can, A->can.flags.data(), A->can.cta_seg0.data(), fre);
    std::memcpy(dst, fre.data(), d.bytes);
    return YASPMV_OK;
  }
  if (d.band ? !A->have_pan_host : (!A->have_host_arrays && which != YASPMV_ARR_CTA_SEG0))
    return fail(YASPMV_EINVAL, "canonical host arrays released: build with YASPMV_KEEP_HOST");
  if (d.bytes) std::memcpy(dst, d.host, d.bytes);
  return YASPMV_OK;
}

yaspmv_status yaspmv_export_device(yaspmv_matrix A, int32_t which, void* dst, int64_t bytes, int64_t* nbytes) {
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle has no device arrays");
  ArrDesc d;
  yaspmv_status st = describe(A, which, d);
  if (st != YASPMV_OK) return st;
  if (nbytes) *nbytes = d.bytes;
  if (!dst) return YASPMV_OK;
  if (bytes < d.bytes) return fail(YASPMV_EINVAL, "destination too small");
  CUDA_TRY(cudaSetDevice(A->device));
  CUDA_TRY(cudaDeviceSynchronize());
  const Canonical& c = A->can;
  if (which == YASPMV_ARR_FRE) {
    std::vector<uint8_t> fl(c.nnzb_pad / 8);
    std::vector<int32_t> cs(c.ntiles);
    if (!fl.empty()) CUDA_TRY(cudaMemcpy(fl.data(), A->d.flags, fl.size(), cudaMemcpyDeviceToHost));
    if (!cs.empty()) CUDA_TRY(cudaMemcpy(cs.data(), A->d.cta_seg0, cs.size() * 4, cudaMemcpyDeviceToHost));
    std::vector<int32_t> fre;
    compute_fre(c, fl.data(), cs.data(), fre);
    std::memcpy(dst, fre.data(), d.bytes);
    return YASPMV_OK;
  }
  if (d.bytes == 0) return YASPMV_OK;
  if (d.ptb == 0) {
    CUDA_TRY(cudaMemcpy(dst, d.dev, d.bytes, cudaMemcpyDeviceToHost));
  } else {
    std::vector<uint8_t> tmp(d.bytes);
    CUDA_TRY(cudaMemcpy(tmp.data(), d.dev, d.bytes, cudaMemcpyDeviceToHost));
    permute_from_device_layout(tmp.data(), static_cast<uint8_t*>(dst), d.ntiles >= 0 ? d.ntiles : c.ntiles,
                               d.ntiles >= 0 ? d.C : c.p.C, d.ptb);
  }
  return YASPMV_OK;
}

yaspmv_status yaspmv_export_device_range(yaspmv_matrix A, int32_t which, int64_t first_tile, int64_t ntiles,
                                         void* dst, int64_t bytes, int64_t* nbytes) {
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle has no device arrays");
  ArrDesc d;
  yaspmv_status st = describe(A, which, d);
  if (st != YASPMV_OK) return st;
  const Canonical& c = A->can;
  // bytes of one workgroup tile of the array (per-tile arrays: one entry)
  int64_t tb = 0, total_tiles = 0;
  const bool band = which >= YASPMV_ARR_BAND_FLAGS;
  const int64_t TC = band ? PANEL_TC : (int64_t)c.p.T * c.p.C;
  const int64_t ntl = band ? (d.ntiles >= 0 ? d.ntiles : A->pan.nband_pad / PANEL_TC) : c.ntiles;
  switch (which) {
    case YASPMV_ARR_FLAGS:
    case YASPMV_ARR_BAND_FLAGS: tb = TC / 8; break;
    case YASPMV_ARR_CTA_SEG0:
    case YASPMV_ARR_BAND_TILE_RANK: tb = 4; break;
    case YASPMV_ARR_COL:
    case YASPMV_ARR_COL_DELTA:
    case YASPMV_ARR_VAL0:
    case YASPMV_ARR_VAL1:
    case YASPMV_ARR_VAL2:
    case YASPMV_ARR_VAL3:
    case YASPMV_ARR_BAND_COL16:
    case YASPMV_ARR_BAND_FAR_COL:
    case YASPMV_ARR_BAND_VAL: tb = ntl > 0 ? d.bytes / ntl : 0; break;
    default: return fail(YASPMV_EINVAL, "range export: per-block or per-tile arrays only");
  }
  total_tiles = ntl;
  if (first_tile < 0 || ntiles < 0 || first_tile + ntiles > total_tiles) return fail(YASPMV_EINVAL, "tile range out of bounds");
  const int64_t out = ntiles * tb;
  if (nbytes) *nbytes = out;
  if (!dst || out == 0) return YASPMV_OK;
  if (bytes < out) return fail(YASPMV_EINVAL, "destination too small");
  CUDA_TRY(cudaSetDevice(A->device));
  CUDA_TRY(cudaDeviceSynchronize());
  const uint8_t* src = static_cast<const uint8_t*>(d.dev) + first_tile * tb;
  if (d.ptb == 0) {
    CUDA_TRY(cudaMemcpy(dst, src, out, cudaMemcpyDeviceToHost));
  } else {
    std::vector<uint8_t> tmp(out);
    CUDA_TRY(cudaMemcpy(tmp.data(), src, out, cudaMemcpyDeviceToHost));
    permute_from_device_layout(tmp.data(), static_cast<uint8_t*>(dst), ntiles, d.ntiles >= 0 ? d.C : c.p.C, d.ptb);
  }
  return YASPMV_OK;
}

// ------------------------------------------------------------------ auto-tuner (§4)
yaspmv_status yaspmv_tune_ex(yaspmv_matrix A, void* stream, yaspmv_params* chosen, int32_t mode) {
  yaspmv::TraceRange tr_("yaspmv:tune_ex");
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "tuning times the kernels: needs a device handle");
  if (!A->have_csr) return fail(YASPMV_EINVAL, "handle was built with YASPMV_DROP_CSR");
  const double t0 = now_s();
  CUDA_TRY(cudaSetDevice(A->device));
  const CSR& M = A->csr;
  const int vs = A->vsize;
  int l2 = 0, sms = 0;
  cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, A->device);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, A->device);

  // (1) footprint of every Table-1 block shape; keep the 4 smallest
  struct Shape { int64_t fp; int h, w; };
  std::vector<Shape> shapes;
  // a panel-sliced BCCOO+ handle tunes its far part (1x1 blocks, band kept by re-encoding)
  const bool band = A->band_on;
  for (int h = 1; h <= (band ? 1 : 4); ++h)
    for (int w : {1, 2, 4, 8}) {
      if (band && w > 1) continue;
      bool any = false;
      for (int T : {4, 8, 16, 32}) any |= find_kernel(A->dtype, h, w, T, COL_I32) != nullptr;
      if (!any) continue;
      const int64_t NB = (M.n + w - 1) / w;
      const int sc = NB < 65535 ? 2 : 4;
      shapes.push_back({footprint_bytes(count_blocks(M, h, w), h, w, vs, sc), h, w});
    }
  std::sort(shapes.begin(), shapes.end(), [](const Shape& a, const Shape& b) {
    return std::tie(a.fp, a.h, a.w) < std::tie(b.fp, b.h, b.w);
  });
  if (mode == 0 && shapes.size() > 4) shapes.resize(4);  // P:321 pruning; mode 1 = exhaustive

  // (2) candidates: slices only when x is a large share of L2 (BCCOO+ helps x locality,
  // P:154; its temporary buffer costs traffic)
  std::vector<int> Ss = {1};
  // Table 1's slice counts up to 32; the larger ones only when x is several times L2
  if ((int64_t)M.n * vs * 2 > (int64_t)l2) Ss = {1, 2, 4, 8};
  if ((int64_t)M.n * vs > 4 * (int64_t)l2) Ss = {1, 2, 4, 8, 16, 32};

  // scratch x / y for timing
  void* x = nullptr;
  void* y = nullptr;
  CUDA_TRY(cudaMalloc(&x, std::max<int64_t>(M.n, 1) * vs + 16));
  CUDA_TRY(cudaMalloc(&y, std::max<int64_t>(M.m, 1) * vs));
  CUDA_TRY(cudaMemset(x, 0, std::max<int64_t>(M.n, 1) * vs));
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaStream_t st = (cudaStream_t)stream;

  struct Cand { float ms; int64_t bytes; Params p; int bfar; };
  std::vector<Cand> results;
  int results_extra = 0;
  const Params saved = A->can.p;
  const int keep_flags = saved.flags & ~YASPMV_DROP_CSR;
  auto time_spmv = [&]() {  // median of 7 after 3 warm-up calls (< 0: a call failed)
    for (int it = 0; it < 3; ++it)
      if (yaspmv_spmv(A, x, y, stream) != YASPMV_OK) return -1.0f;
    std::vector<float> ts;
    for (int it = 0; it < 7; ++it) {
      cudaEventRecord(e0, st);
      yaspmv_spmv(A, x, y, stream);
      cudaEventRecord(e1, st);
      cudaEventSynchronize(e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, e0, e1);
      ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    return ts[ts.size() / 2];
  };
  // a band handle also times its far entries inside the panels (reading P7) against every
  // separate far-part candidate below
  if (band) {
    yaspmv_params ap{saved.h, saved.w, saved.S, saved.T, saved.C, saved.col_mode, saved.empty_mode, keep_flags,
                     -1, 1};
    ap.band_far = YASPMV_FAR_IN_PANEL;
    if (yaspmv_reencode(A, &ap) == YASPMV_OK) {
      const float ms = time_spmv();
      yaspmv_info info;
      yaspmv_get_info(A, &info);
      if (ms >= 0) results.push_back({ms, info.format_bytes, A->can.p, YASPMV_FAR_IN_PANEL});
    }
  }
  for (const Shape& sh : shapes) {
    const int64_t NB = (M.n + sh.w - 1) / sh.w;
    std::vector<int> cms = {NB < 65535 ? (int)COL_U16 : (int)COL_I32};
    if (NB >= 65535) cms.push_back(COL_DELTA);
    for (int S : Ss) {
      if (S > std::max<int64_t>(NB, 1)) continue;
      for (int cm : cms) {
        // host: one encode per (h, w, S, col mode) at the largest tile, (T, C) variants
        // derived; GPU translation: a full encode per candidate on the device
        const bool gpu = (saved.flags & YASPMV_GPU_ENCODE) != 0 || band;
        Params bp0;
        bp0.h = sh.h; bp0.w = sh.w; bp0.S = S; bp0.T = 32; bp0.C = 512; bp0.col_mode = cm;
        bp0.empty_mode = saved.empty_mode;
        bp0.tpc = 1;
        Params rp;
        if (resolve_params(bp0, M.m, M.n, rp) != YASPMV_OK) continue;
        Canonical base;
        if (!gpu && encode(M, rp, base) != YASPMV_OK) continue;
        const int64_t nnzb_est = gpu ? count_blocks(M, sh.h, sh.w) : base.nnzb;
        for (int T : {4, 8, 16, 32}) {
          if (!find_kernel(A->dtype, sh.h, sh.w, T, cm)) continue;
          for (int C : {64, 128, 256, 512}) {
            // occupancy bound: at least 2 tiles per SM unless the tile is small
            const int64_t tiles = (nnzb_est + (int64_t)T * C - 1) / ((int64_t)T * C);
            if (tiles < 2 * sms && (T * C) > 1024) continue;
            if (gpu) {
              yaspmv_params ap{sh.h, sh.w, S, T, C, cm, saved.empty_mode,
                               (saved.flags & YASPMV_GPU_ENCODE) ? YASPMV_GPU_ENCODE : keep_flags, -1, 1};
              if (band) ap.band_far = YASPMV_FAR_SEPARATE;
              if (yaspmv_reencode(A, &ap) != YASPMV_OK) continue;
            } else {
              Canonical cand;
              if (derive_tc(base, T, C, cand) != YASPMV_OK) continue;
              if (install_canonical(A, std::move(cand), 0) != YASPMV_OK) continue;  // e.g. launch bound
            }
            bool ok = true;
            for (int it = 0; it < 3 && ok; ++it) ok = yaspmv_spmv(A, x, y, stream) == YASPMV_OK;
            if (!ok) continue;
            std::vector<float> ts;
            for (int it = 0; it < 7; ++it) {
              cudaEventRecord(e0, st);
              yaspmv_spmv(A, x, y, stream);
              cudaEventRecord(e1, st);
              cudaEventSynchronize(e1);
              float ms = 0;
              cudaEventElapsedTime(&ms, e0, e1);
              ts.push_back(ms);
            }
            std::sort(ts.begin(), ts.end());
            yaspmv_info info;
            yaspmv_get_info(A, &info);
            results.push_back({ts[ts.size() / 2], info.format_bytes, A->can.p, A->can.p.bfar});
            // strategy 2 with the paper's pinned result cache sizes 1 and 2: a
            // launch-time switch on the same encoding
            for (int rc : {1, 2}) {
              if (!find_kernel(A->dtype, sh.h, sh.w, T, cm, 2) || set_launch(A, rc, 1) != YASPMV_OK) continue;
              bool ok2 = true;
              for (int it = 0; it < 3 && ok2; ++it) ok2 = yaspmv_spmv(A, x, y, stream) == YASPMV_OK;
              if (ok2) {
                std::vector<float> t2;
                for (int it = 0; it < 7; ++it) {
                  cudaEventRecord(e0, st);
                  yaspmv_spmv(A, x, y, stream);
                  cudaEventRecord(e1, st);
                  cudaEventSynchronize(e1);
                  float ms = 0;
                  cudaEventElapsedTime(&ms, e0, e1);
                  t2.push_back(ms);
                }
                std::sort(t2.begin(), t2.end());
                results.push_back({t2[t2.size() / 2], info.format_bytes, A->can.p, A->can.p.bfar});
              }
              set_launch(A, 0, 1);
            }
          }
        }
      }
    }
  }
  auto release = [&]() {
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(x);
    cudaFree(y);
  };
  if (results.empty()) {
    release();
    yaspmv_params back{saved.h, saved.w, saved.S, saved.T, saved.C, saved.col_mode, saved.empty_mode, keep_flags,
                       saved.rc > 0 ? saved.rc : -1, saved.tpc};
    back.band_far = saved.bfar;
    yaspmv_reencode(A, &back);
    return fail(YASPMV_EUNSUPPORTED, "no tunable candidate could be launched");
  }
  // (3) fastest; ties within 1%: smaller footprint, then lexicographic (Q15)
  float best_ms = 1e30f;
  for (const Cand& c : results) best_ms = std::min(best_ms, c.ms);
  const Cand* best = nullptr;
  for (const Cand& c : results) {
    if (c.ms > best_ms * 1.01f) continue;
    if (!best) { best = &c; continue; }
    auto key = [](const Cand& q) { return std::make_tuple(q.bytes, q.p.h, q.p.w, q.p.T, q.p.C, q.p.S, q.p.rc); };
    if (key(c) < key(*best)) best = &c;
  }
  yaspmv_params bp{best->p.h, best->p.w, best->p.S, best->p.T, best->p.C, best->p.col_mode, best->p.empty_mode,
                   keep_flags, best->p.rc > 0 ? best->p.rc : -1, 1};
  bp.band_far = best->bfar;
  yaspmv_status rs = yaspmv_reencode(A, &bp);
  if (rs != YASPMV_OK) {
    release();
    return rs;
  }
  // (4) tiles per CTA for the winner (launch-time; bitwise-identical results): fastest,
  // ties within 1% to the smaller count
  {
    float tbest = 1e30f;
    int kbest = 1;
    for (int k : {1, 2, 4}) {
      if (set_launch(A, A->can.p.rc, k) != YASPMV_OK) continue;
      for (int it = 0; it < 3; ++it) yaspmv_spmv(A, x, y, stream);
      std::vector<float> tk;
      for (int it = 0; it < 7; ++it) {
        cudaEventRecord(e0, st);
        yaspmv_spmv(A, x, y, stream);
        cudaEventRecord(e1, st);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        tk.push_back(ms);
      }
      std::sort(tk.begin(), tk.end());
      const float med = tk[tk.size() / 2];
      if (med < tbest * 0.99f) {
        tbest = med;
        kbest = k;
      }
      ++results_extra;
    }
    set_launch(A, A->can.p.rc, kbest);
  }
  release();
  A->tune_s = now_s() - t0;
  A->tune_candidates = (int)results.size() + results_extra;
  if (chosen) {
    const Params& q = A->can.p;
    *chosen = yaspmv_params{q.h, q.w, q.S, q.T, q.C, q.col_mode, q.empty_mode, q.flags, q.rc, A->tpc};
    chosen->band = q.band;
    chosen->panel_rows = q.pR;
    chosen->slice_width = q.pW;
    chosen->band_col0 = q.col0;
    chosen->band_far = q.bfar;
  }
  return YASPMV_OK;
}

yaspmv_status yaspmv_tune(yaspmv_matrix A, void* stream, yaspmv_params* chosen) {
  return yaspmv_tune_ex(A, stream, chosen, 0);
}

// ------------------------------------------------------------------ power iteration
int64_t yaspmv_nrm2sq_scratch_bytes(int64_t n) { return nrm2sq_blocks(n) * (int64_t)sizeof(double); }

yaspmv_status yaspmv_nrm2sq(const void* v, int64_t n, yaspmv_dtype dtype, double* out_dev, void* scratch_dev,
                            void* stream) {
  if (n < 0 || !out_dev || !scratch_dev || (n > 0 && !v)) return fail(YASPMV_EINVAL, "bad nrm2sq arguments");
  if (dtype != YASPMV_F32 && dtype != YASPMV_F64) return fail(YASPMV_EINVAL, "bad dtype");
  launch_nrm2sq(v, n, dtype, out_dev, static_cast<double*>(scratch_dev), stream);
  CUDA_TRY(cudaGetLastError());
  return YASPMV_OK;
}

yaspmv_status yaspmv_scale(const void* src, void* dst, int64_t n, yaspmv_dtype dtype, const double* norm2_dev,
                           void* stream) {
  if (n < 0 || !norm2_dev || (n > 0 && (!src || !dst))) return fail(YASPMV_EINVAL, "bad scale arguments");
  if (dtype != YASPMV_F32 && dtype != YASPMV_F64) return fail(YASPMV_EINVAL, "bad dtype");
  launch_scale(src, dst, n, dtype, norm2_dev, stream);
  CUDA_TRY(cudaGetLastError());
  return YASPMV_OK;
}

}  // extern "C"
