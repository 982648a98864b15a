// capi.cpp — the C ABI of include/yaspmv.h: handles, upload to the device layout, SpMV
// launch, export/introspection, the auto-tuner of PAPER.md §4, power-iteration helpers.
#include <cuda_runtime.h>
#include <omp.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <memory>
#include <string>
#include <cstdlib>

#include "handle.hpp"
#include "trace.hpp"
#include "../../include/yaspmv_ablation.h"

using namespace yaspmv;

namespace yaspmv {
void GpuArrays::free_all() {
  void* ps[] = {val[0], val[1], val[2], val[3], col, col32, flags, cta_seg0, seg_row, zero_rows};
  for (void* p : ps)
    if (p) cudaFree(p);
  *this = GpuArrays();
}
static thread_local std::string g_err;
void set_error(const std::string& msg) { g_err = msg; }
yaspmv_status fail(yaspmv_status st, const std::string& msg) {
  g_err = msg;
  return st;
}
// Debug spin bound: YASPMV_SPIN_LIMIT=N (read once per process) makes a
// look-back that polls more than N times write its tile id to a mapped host slot and trap;
// the slot survives the sticky launch error and is read by yaspmv_debug_spin_tile().
long long debug_spin_limit() {
  static const long long lim = [] {
    const char* e = std::getenv("YASPMV_SPIN_LIMIT");
    return e ? std::atoll(e) : 0ll;
  }();
  return lim;
}
static long long* g_spin_slot = nullptr;
long long* debug_spin_slot() {
  if (debug_spin_limit() <= 0) return nullptr;
  static const bool ok = [] {
    void* p = nullptr;
    if (cudaHostAlloc(&p, sizeof(long long), cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) return false;
    g_spin_slot = static_cast<long long*>(p);
    *g_spin_slot = -1;
    return true;
  }();
  return ok ? g_spin_slot : nullptr;
}
}  // namespace yaspmv

extern "C" int64_t yaspmv_debug_spin_tile(void) {
  return yaspmv::g_spin_slot ? (int64_t) * (volatile long long*)yaspmv::g_spin_slot : -1;
}

namespace {
// run a call on the handle's device and restore the caller's current device afterwards
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (dev >= 0 && cudaGetDevice(&prev) == cudaSuccess && prev != dev) cudaSetDevice(dev);
    else prev = -1;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};
}  // namespace

#define CUDA_TRY(expr)                                                                       \
  do {                                                                                       \
    cudaError_t _e = (expr);                                                                 \
    if (_e != cudaSuccess)                                                                   \
      return fail(_e == cudaErrorMemoryAllocation ? YASPMV_ENOMEM : YASPMV_ECUDA,            \
                  std::string(#expr) + ": " + cudaGetErrorString(_e));                       \
  } while (0)

namespace {

double now_s() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

Params from_abi(const yaspmv_params* p) {
  Params q;
  if (p) {
    q.h = p->block_h;
    q.w = p->block_w;
    q.S = p->slices;
    q.T = p->thread_tile;
    q.C = p->cta_size;
    q.col_mode = p->col_mode;
    q.empty_mode = p->empty_mode;
    q.flags = p->flags;
    q.rc = p->result_cache;
    q.tpc = p->tiles_per_cta;
    q.band = p->band;
    q.pR = p->panel_rows;
    q.pW = p->slice_width;
    q.col0 = p->band_col0;
    q.bfar = p->band_far;
  }
  return q;
}

yaspmv_params to_abi(const Params& q) {
  yaspmv_params p;
  p.block_h = q.h;
  p.block_w = q.w;
  p.slices = q.S;
  p.thread_tile = q.T;
  p.cta_size = q.C;
  p.col_mode = q.col_mode;
  p.empty_mode = q.empty_mode;
  p.flags = q.flags;
  p.result_cache = q.rc;
  p.tiles_per_cta = q.tpc;
  p.band = q.band;
  p.panel_rows = q.pR;
  p.slice_width = q.pW;
  p.band_col0 = q.col0;
  p.band_far = q.bfar;
  return p;
}

template <typename T>
yaspmv_status upload(const T* src, size_t bytes, T** dst) {
  *dst = nullptr;
  if (bytes == 0) return YASPMV_OK;
  CUDA_TRY(cudaMalloc((void**)dst, bytes));
  CUDA_TRY(cudaMemcpy(*dst, src, bytes, cudaMemcpyHostToDevice));
  return YASPMV_OK;
}

yaspmv_status upload_permuted(const uint8_t* src, int64_t ntiles, int C, int ptb, void** dst) {
  *dst = nullptr;
  const size_t bytes = (size_t)ntiles * C * ptb;
  if (bytes == 0) return YASPMV_OK;
  std::unique_ptr<uint8_t[]> tmp;
  try {
    tmp.reset(new uint8_t[bytes]);
  } catch (const std::bad_alloc&) {
    return fail(YASPMV_ENOMEM, "host staging allocation failed");
  }
  permute_to_device_layout(src, tmp.get(), ntiles, C, ptb);
  CUDA_TRY(cudaMalloc(dst, bytes));
  CUDA_TRY(cudaMemcpy(*dst, tmp.get(), bytes, cudaMemcpyHostToDevice));
  return YASPMV_OK;
}

// Per-call scratch of an encoding: ticket counter, status words + carries, BCCOO+ buffer.
yaspmv_status alloc_scratch(const Canonical& c, int vsize, DevArrays& d) {
  const Params& p = c.p;
  CUDA_TRY(cudaMalloc((void**)&d.ticket, sizeof(unsigned long long)));
  CUDA_TRY(cudaMemset(d.ticket, 0, sizeof(unsigned long long)));
  const int64_t nt = std::max<int64_t>(c.ntiles, 1);
  CUDA_TRY(cudaMalloc((void**)&d.status, 2 * nt * sizeof(unsigned long long)));
  CUDA_TRY(cudaMemset(d.status, 0, 2 * nt * sizeof(unsigned long long)));
  CUDA_TRY(cudaMalloc((void**)&d.carry, nt * p.h * sizeof(double)));
  CUDA_TRY(cudaMalloc((void**)&d.bnd, 2 * (nt + 1) * sizeof(unsigned long long)));
  CUDA_TRY(cudaMemset(d.bnd, 0, 2 * (nt + 1) * sizeof(unsigned long long)));
  CUDA_TRY(cudaMalloc((void**)&d.pend_val, nt * p.h * sizeof(double)));
  CUDA_TRY(cudaMalloc((void**)&d.pend_row, nt * sizeof(long long)));
  if (p.S > 1) CUDA_TRY(cudaMalloc(&d.tmp, (size_t)p.S * c.MB * p.h * vsize));
  return YASPMV_OK;
}

// Encoded host arrays -> a fresh set of device arrays in the device layout.
yaspmv_status to_device_impl(const Canonical& c, int vsize, DevArrays& d, int64_t& n_escapes) {
  const Params& p = c.p;
  yaspmv_status st;
  const int vptb = p.T * p.w * vsize;
  for (int r = 0; r < p.h; ++r)
    if ((st = upload_permuted(c.val[r].data(), c.ntiles, p.C, vptb, &d.val[r])) != YASPMV_OK) return st;
  if (p.col_mode == COL_U16) {
    st = upload_permuted(reinterpret_cast<const uint8_t*>(c.col16.data()), c.ntiles, p.C, 2 * p.T, &d.col);
  } else if (p.col_mode == COL_I32) {
    st = upload_permuted(reinterpret_cast<const uint8_t*>(c.col32.data()), c.ntiles, p.C, 4 * p.T, &d.col);
  } else {
    st = upload_permuted(reinterpret_cast<const uint8_t*>(c.delta.data()), c.ntiles, p.C, 2 * p.T, &d.col);
    if (st == YASPMV_OK) st = upload(c.col32.data(), c.col32.size() * 4, &d.col32);
  }
  if (st != YASPMV_OK) return st;
  if ((st = upload(c.flags.data(), c.flags.size(), &d.flags)) != YASPMV_OK) return st;
  if ((st = upload(c.cta_seg0.data(), c.cta_seg0.size() * 4, &d.cta_seg0)) != YASPMV_OK) return st;
  if ((st = upload(c.seg_row.data(), c.seg_row.size() * 4, &d.seg_row)) != YASPMV_OK) return st;
  if ((st = upload(c.zero_rows.data(), c.zero_rows.size() * 4, &d.zero_rows)) != YASPMV_OK) return st;
  if ((st = alloc_scratch(c, vsize, d)) != YASPMV_OK) return st;
  // escapes of the int16 delta column array (only they read col32)
  n_escapes = 0;
  if (p.col_mode == COL_DELTA)
    for (int16_t v : c.delta) n_escapes += v == -1;
  CUDA_TRY(cudaDeviceSynchronize());
  return YASPMV_OK;
}

// Upload A->can; on success replace A's device arrays, on failure keep the old ones.
yaspmv_status to_device(yaspmv_matrix A) {
  CUDA_TRY(cudaSetDevice(A->device));
  DevArrays nd;
  int64_t esc = 0;
  yaspmv_status st = to_device_impl(A->can, A->vsize, nd, esc);
  if (st != YASPMV_OK) {
    nd.free_all();
    return st;
  }
  CUDA_TRY(cudaDeviceSynchronize());  // no launch may still use the old arrays
  A->d.free_all();
  A->d = nd;
  A->n_escapes = esc;
  return YASPMV_OK;
}

yaspmv_status select_kernel(yaspmv_matrix A) {
  const Params& p = A->can.p;
  if (A->device < 0) return YASPMV_OK;  // host-only handles never launch
  A->kern = find_kernel(A->dtype, p.h, p.w, p.T, p.col_mode, p.rc > 0 ? 2 : 1);
  if (!A->kern)
    return fail(YASPMV_EUNSUPPORTED, "no compiled kernel for dtype/h/w/T (values per thread exceed 512 bytes)");
  int regs = 0, maxt = 0, bps = 0;
  int e = A->kern->attr(p.C, p.rc, &regs, &maxt, &bps);
  if (e != 0) return fail(YASPMV_ECUDA, std::string("kernel attributes: ") + cudaGetErrorString((cudaError_t)e));
  if (p.C > maxt) return fail(YASPMV_EUNSUPPORTED, "cta_size exceeds the kernel's launch bound");
  if (bps <= 0) return fail(YASPMV_EUNSUPPORTED, "kernel does not fit on an SM with this cta_size");
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, A->device);
  // one CTA per tiles_per_cta consecutive workgroup-level tiles; auto: 2 once the
  // matrix spans >= 32 waves of resident CTAs (C5: 244,680 tiles; measured 4.17 vs 4.52 ms)
  if (p.tpc > 0) A->tpc = p.tpc;
  else A->tpc = A->can.ntiles >= 32LL * std::max(1, sms) * bps ? 2 : 1;
  if (p.flags & YASPMV_TICKET_IDS) A->tpc = 1;
  A->grid = std::max<int64_t>(1, (A->can.ntiles + A->tpc - 1) / A->tpc);
  A->regs = regs;
  return YASPMV_OK;
}

// Make `c` A's encoding: select the kernel, upload, release host arrays unless kept.
// On failure A keeps its previous encoding (host and device).
yaspmv_status install_canonical_impl(yaspmv_matrix A, Canonical&& c, int flags) {
  Canonical old;
  std::swap(old, A->can);
  A->can = std::move(c);
  const KernelEntry* oldk = A->kern;
  const int64_t oldgrid = A->grid;
  yaspmv_status st;
  if ((st = select_kernel(A)) != YASPMV_OK) {
    A->can = std::move(old);
    A->kern = oldk;
    A->grid = oldgrid;
    return st;
  }
  if (A->device >= 0) {
    if ((st = to_device(A)) != YASPMV_OK) {  // old device arrays are untouched
      A->can = std::move(old);
      A->kern = oldk;
      A->grid = oldgrid;
      return st;
    }
    if (!(flags & YASPMV_KEEP_HOST)) {
      A->can.release_arrays();
      A->have_host_arrays = false;
    } else {
      A->have_host_arrays = true;
    }
  } else {
    A->have_host_arrays = true;
  }
  return YASPMV_OK;
}

// panel-sliced BCCOO+: validate and resolve the band parameters (0 = default)
yaspmv_status resolve_band(yaspmv_matrix A, Params& p) {
  if (p.band < 0) return fail(YASPMV_EINVAL, "band must be >= 0");
  if (p.band == 0) {
    p.pR = p.pW = p.col0 = p.bfar = 0;
    return YASPMV_OK;
  }
  if (p.bfar == 0) p.bfar = YASPMV_FAR_SEPARATE;
  if (p.bfar != YASPMV_FAR_SEPARATE && p.bfar != YASPMV_FAR_IN_PANEL) return fail(YASPMV_EINVAL, "bad band_far");
  if (A->dtype != YASPMV_F32) return fail(YASPMV_EUNSUPPORTED, "panel-sliced BCCOO+ is compiled for fp32");
  if (p.h != 1 || p.w != 1) return fail(YASPMV_EUNSUPPORTED, "panel-sliced BCCOO+ needs 1x1 blocks");
  if (p.pR == 0) p.pR = 16384;  // defaults: one CTA per SM (PANEL_CTA threads), ~200 KB of shared memory
  if (p.pW == 0) p.pW = 16384;
  if (p.pR % 256 || p.pR <= 0 || p.pR > 32768) return fail(YASPMV_EINVAL, "panel_rows must be a multiple of 256 in [256, 32768]");
  if (p.pW % 4 || p.pW <= 0 || p.pW > 65532) return fail(YASPMV_EINVAL, "slice_width must be a multiple of 4 in [4, 65532]");
  if ((p.pR + 2LL * p.band + p.pW - 1) / p.pW > PANEL_MAX_KS)
    return fail(YASPMV_EINVAL, "panel-sliced BCCOO+: (panel_rows + 2*band) / slice_width exceeds 64 slices");
  if (A->device >= 0) {
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, A->device);
    if (panel_smem_bytes(p.pR, p.pW) + 2048 > (size_t)optin)
      return fail(YASPMV_EINVAL, "panel_rows / slice_width need more shared memory than a CTA has");
  }
  return YASPMV_OK;
}

// upload the band part into nd (the caller installs it)
yaspmv_status panel_to_device(yaspmv_matrix A, const PanelCanonical& pc, PanelDev& nd) {
  nd = PanelDev();
  auto up = [&](const void* src, size_t bytes, void** dst) -> yaspmv_status {
    *dst = nullptr;
    if (!bytes) return YASPMV_OK;
    CUDA_TRY(cudaMalloc(dst, bytes));
    CUDA_TRY(cudaMemcpy(*dst, src, bytes, cudaMemcpyHostToDevice));
    return YASPMV_OK;
  };
  const int64_t ntl = pc.nband_pad / PANEL_TC;
  yaspmv_status st;
  if ((st = upload_permuted(reinterpret_cast<const uint8_t*>(pc.col16.data()), (pc.nband_pad - pc.nfar_pad) / PANEL_TC,
                            PANEL_WT, 2 * PANEL_BT,
                            &nd.col16)) != YASPMV_OK ||
      (st = upload_permuted(pc.val.data(), ntl, PANEL_WT, PANEL_BT * A->vsize, &nd.val)) != YASPMV_OK ||
      (st = up(pc.tile_rank.data(), pc.tile_rank.size() * 4, (void**)&nd.tile_rank)) != YASPMV_OK ||
      (st = up(pc.flags.data(), pc.flags.size(), (void**)&nd.flags)) != YASPMV_OK ||
      (st = up(pc.panel_blk0.data(), pc.panel_blk0.size() * 8, (void**)&nd.panel_blk0)) != YASPMV_OK ||
      (st = up(pc.slice_ptr.data(), pc.slice_ptr.size() * 4, (void**)&nd.slice_ptr)) != YASPMV_OK ||
      (st = up(pc.stop_ptr.data(), pc.stop_ptr.size() * 4, (void**)&nd.stop_ptr)) != YASPMV_OK ||
      (st = up(pc.first_row.data(), pc.first_row.size() * 4, (void**)&nd.first_row)) != YASPMV_OK ||
      (st = upload_permuted(reinterpret_cast<const uint8_t*>(pc.far_col.data()), pc.nfar_pad / PANEL_TC, PANEL_WT,
                            4 * PANEL_BT, &nd.far_col)) != YASPMV_OK ||
      (st = up(pc.far_blk0.data(), pc.far_blk0.size() * 8, (void**)&nd.far_blk0)) != YASPMV_OK) {
    nd.free_all();
    return st;
  }
  const int64_t np = std::max<int64_t>(pc.g.npanels, 1);
  if (cudaMalloc((void**)&nd.part, np * sizeof(double)) != cudaSuccess ||
      cudaMalloc((void**)&nd.scratch, nrm2sq_blocks(np) * sizeof(double)) != cudaSuccess) {
    nd.free_all();
    return fail(YASPMV_ENOMEM, "panel scratch allocation failed");
  }
  int e = panel_attr(pc.g.R, pc.g.W, &A->pan_regs);
  if (e != 0) {
    nd.free_all();
    return fail(YASPMV_ECUDA, std::string("panel kernel attributes: ") + cudaGetErrorString((cudaError_t)e));
  }
  CUDA_TRY(cudaDeviceSynchronize());
  return YASPMV_OK;
}

yaspmv_status encode_plain_into(yaspmv_matrix A, const CSR& src, const Params& p, double t0);

// the plain part of a YASPMV_FAR_IN_PANEL handle: shape only (no blocks, tiles or arrays)
yaspmv_status install_empty_plain(yaspmv_matrix A, const CSR& src, const Params& p) {
  Canonical c;
  c.m = src.m;
  c.n = src.n;
  c.MB = src.m;
  c.NB = src.n;
  c.SW = std::max<int64_t>(src.n, 1);
  c.p = p;
  c.p.h = c.p.w = c.p.S = 1;
  c.p.empty_mode = EMPTY_FILLER;
  c.vsize = A->vsize;
  return install_canonical_impl(A, std::move(c), p.flags);
}

// (re-)encode A->csr with params and upload; on failure A is left unchanged
yaspmv_status encode_into(yaspmv_matrix A, const Params& want) {
  const double t0 = now_s();
  Params p;
  yaspmv_status st = resolve_params(want, A->csr.m, A->csr.n, p);
  if (st != YASPMV_OK) return st;
  if ((st = resolve_band(A, p)) != YASPMV_OK) return st;
  A->nnz_total = A->csr.nnz;
  if (p.band == 0) {
    if ((st = encode_plain_into(A, A->csr, p, t0)) != YASPMV_OK) return st;
    A->band_on = false;
    A->pan = PanelCanonical();
    A->have_pan_host = false;
    if (A->device >= 0) A->pd.free_all();
    return YASPMV_OK;
  }
  // panel-sliced BCCOO+: split into the far part (plain path) and the band stream
  PanelGeom g;
  g.R = p.pR;
  g.W = p.pW;
  g.B = p.band;
  g.col0 = p.col0;
  g.fip = p.bfar == YASPMV_FAR_IN_PANEL ? 1 : 0;
  CSR far;
  PanelCanonical pc;
  if ((st = encode_panel(A->csr, g, far, pc)) != YASPMV_OK) return st;
  PanelDev nd;
  if (A->device >= 0) {
    CUDA_TRY(cudaSetDevice(A->device));
    if ((st = panel_to_device(A, pc, nd)) != YASPMV_OK) return st;
  }
  // P7: no far part — the plain encoding is an empty m x n matrix (no tiles, no launch)
  if ((st = g.fip ? install_empty_plain(A, far, p) : encode_plain_into(A, far, p, t0)) != YASPMV_OK) {
    nd.free_all();
    return st;
  }
  if (A->device >= 0) {
    A->pd.free_all();
    A->pd = nd;
  }
  A->band_on = true;
  A->have_pan_host = A->device < 0 || (p.flags & YASPMV_KEEP_HOST);
  if (!A->have_pan_host) pc.release_arrays();
  A->pan = std::move(pc);
  A->build_s = now_s() - t0;
  return YASPMV_OK;
}

// the plain BCCOO/BCCOO+ encoding of `src` (A->csr, or the far part of a panel encoding)
yaspmv_status encode_plain_into(yaspmv_matrix A, const CSR& src, const Params& p, double t0) {
  yaspmv_status st;
  if (A->device >= 0 && !find_kernel(A->dtype, p.h, p.w, p.T, p.col_mode, p.rc > 0 ? 2 : 1))
    return fail(YASPMV_EUNSUPPORTED, "no compiled kernel for this (dtype, h, w, T): values per thread > 512 B");
  if ((p.flags & YASPMV_GPU_ENCODE) && A->device >= 0) {
    CUDA_TRY(cudaSetDevice(A->device));
    Canonical meta;
    GpuArrays g;
    int64_t esc = 0;
    if ((st = encode_gpu(src, p, meta, g, esc, nullptr)) != YASPMV_OK) return st;
    DevArrays nd;
    for (int r = 0; r < 4; ++r) nd.val[r] = g.val[r];
    nd.col = g.col;
    nd.col32 = g.col32;
    nd.flags = g.flags;
    nd.cta_seg0 = g.cta_seg0;
    nd.seg_row = g.seg_row;
    nd.zero_rows = g.zero_rows;
    if ((st = alloc_scratch(meta, A->vsize, nd)) != YASPMV_OK) {
      nd.free_all();
      return st;
    }
    Canonical old;
    std::swap(old, A->can);
    A->can = std::move(meta);
    const KernelEntry* oldk = A->kern;
    const int64_t oldgrid = A->grid;
    if ((st = select_kernel(A)) != YASPMV_OK) {
      nd.free_all();
      A->can = std::move(old);
      A->kern = oldk;
      A->grid = oldgrid;
      return st;
    }
    CUDA_TRY(cudaDeviceSynchronize());
    A->d.free_all();
    A->d = nd;
    A->n_escapes = esc;
    A->have_host_arrays = false;
    A->build_s = now_s() - t0;
    return YASPMV_OK;
  }
  Canonical c;
  if ((st = encode(src, p, c)) != YASPMV_OK) return st;
  if ((st = install_canonical_impl(A, std::move(c), p.flags)) != YASPMV_OK) return st;
  A->build_s = now_s() - t0;
  return YASPMV_OK;
}

yaspmv_status build_common(yaspmv_matrix A, const Params& p) {
  yaspmv_status st = encode_into(A, p);
  if (st != YASPMV_OK) return st;
  if (p.flags & YASPMV_DROP_CSR) {
    A->csr = CSR();
    A->have_csr = false;
  } else {
    A->csr.make_owned();
    A->have_csr = true;
  }
  return YASPMV_OK;
}

yaspmv_status check_device(int32_t device) {
  if (device < 0) return YASPMV_OK;
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess) return fail(YASPMV_ECUDA, std::string("no CUDA device: ") + cudaGetErrorString(e));
  if (device >= n) return fail(YASPMV_EINVAL, "device ordinal out of range");
  return YASPMV_OK;
}

// the band stream + its aux (readings P1-P6), read once per SpMV
int64_t band_format_bytes(const yaspmv_matrix A) {
  if (!A->band_on) return 0;
  const PanelCanonical& q = A->pan;
  const int64_t NS = q.g.NS();
  int64_t b = q.nband_pad * (int64_t)A->vsize + q.nband_pad / 8;           // values, flags
  b += (q.nband_pad - q.nfar_pad) * 2 + q.nfar_pad * 4;                     // col16, far columns (P7)
  b += (q.g.npanels + 1) * 8 * (q.g.fip ? 2 : 1);                           // panel_blk0 (+ far_blk0)
  b += q.g.npanels * (NS + 1) * 4 + q.g.npanels * NS * 4;                   // slice_ptr, first_row
  b += q.nband_pad / PANEL_TC * 4;                                          // tile_rank
  return b;
}

int64_t format_bytes(const yaspmv_matrix A) {
  const Canonical& c = A->can;
  const Params& p = c.p;
  int64_t b = c.nnzb_pad * (int64_t)p.h * p.w * A->vsize;       // values
  b += c.nnzb_pad * (int64_t)col_bytes(p.col_mode);             // col / delta
  b += A->n_escapes * 4;                                         // escape reads
  b += c.nnzb_pad / 8;                                           // bit flags
  b += c.ntiles * (4 + 16 + (p.h > 1 ? 8 * (int64_t)p.h : 0) + 16);  // cta_seg0, status(+carry), carries, hand-off
  if (c.has_seg_row) b += c.n_stops * 4;                         // seg_row
  b += c.n_zero * 4;                                             // zero-fill list
  return b + band_format_bytes(A);
}

int64_t alg_bytes(const yaspmv_matrix A) {
  const Canonical& c = A->can;
  const Params& p = c.p;
  int64_t b = format_bytes(A) + c.n * A->vsize;  // + x
  const int64_t part = (int64_t)p.S * c.MB * p.h * A->vsize;  // far part's output: y or the S slices
  if (A->band_on && A->pan.g.fip) return b + c.m * A->vsize;  // + y (one kernel, no partials)
  if (A->band_on) return b + part + part + c.m * A->vsize;   // written, re-read by the band kernel, + y
  if (p.S == 1) b += c.m * A->vsize;             // + y
  else b += part + (int64_t)p.S * c.m * A->vsize + c.m * A->vsize;
  return b;
}

yaspmv_status run_spmv_plain(yaspmv_matrix A, const void* x, void* y, void* stream, const double* in_norm2,
                             double* out_norm2, int ablate, const PeerOut* peers, bool skip_combine = false) {
  const Canonical& c = A->can;
  const Params& p = c.p;
  cudaStream_t cs = (cudaStream_t)stream;
  DeviceGuard dg(A->device);  // the handle's device, whatever the caller's current one is
  if (c.m == 0) {
    if (out_norm2) CUDA_TRY(cudaMemsetAsync(out_norm2, 0, sizeof(double), cs));
    return YASPMV_OK;
  }
  if (c.ntiles == 0) {
    if (peers && peers->mc)
      launch_mc_zero(peers->p[0], c.m, A->vsize == 4 ? 0 : 1, cs);
    else if (peers)
      for (int q = 0; q < peers->n; ++q) CUDA_TRY(cudaMemsetAsync(peers->p[q], 0, (size_t)c.m * A->vsize, cs));
    else
      CUDA_TRY(cudaMemsetAsync(y, 0, (size_t)c.m * A->vsize, cs));
    if (out_norm2) CUDA_TRY(cudaMemsetAsync(out_norm2, 0, sizeof(double), cs));
    return YASPMV_OK;
  }
  const int nw1 = p.C / 32 + 1;
  const int64_t npart = p.S == 1 ? c.ntiles * nw1 : combine_blocks(c.m);
  if (out_norm2 && A->npart < npart) {  // partial sums of y^2 + the reduction scratch
    if (A->d_part) cudaFree(A->d_part);
    if (A->d_scratch) cudaFree(A->d_scratch);
    A->d_part = nullptr;
    A->d_scratch = nullptr;
    A->npart = 0;
    CUDA_TRY(cudaMalloc((void**)&A->d_part, npart * sizeof(double)));
    CUDA_TRY(cudaMalloc((void**)&A->d_scratch, nrm2sq_blocks(npart) * sizeof(double)));
    A->npart = npart;
  }
  KArgs a;
  for (int r = 0; r < 4; ++r) a.val[r] = A->d.val[r];
  a.col = A->d.col;
  a.col32 = A->d.col32;
  a.flags = A->d.flags;
  a.cta_seg0 = A->d.cta_seg0;
  a.seg_row = A->d.seg_row;
  a.zero_rows = A->d.zero_rows;
  a.n_zero = c.n_zero;
  a.x = x;
  a.out = p.S == 1 ? y : A->d.tmp;
  a.out_limit = p.S == 1 ? c.m : (int64_t)p.S * c.MB * p.h;
  a.n = c.n;
  a.ntiles = c.ntiles;
  a.period = c.ntiles;
  a.ticket = A->d.ticket;
  a.status = A->d.status;
  a.carry = A->d.carry;
  a.bnd = A->d.bnd;
  a.pend_val = A->d.pend_val;
  a.pend_row = A->d.pend_row;
  a.force_handoff = (p.flags & YASPMV_FORCE_HANDOFF) ? 1 : 0;
  a.epi = 0;
  a.in_norm2 = in_norm2;
  a.part = A->d_part;
  a.ablate = ablate;
  a.block_ids = (p.flags & YASPMV_TICKET_IDS) ? 0 : 1;
  a.pdl = (p.flags & YASPMV_NO_PDL) ? 0 : 1;
  a.dep_row = nullptr;
  a.npeer = 0;
  a.peer_mc = 0;
  for (int q = 0; q < YASPMV_MAX_RANKS; ++q) a.peer_out[q] = nullptr;
  a.rcache = p.rc * p.C;
  a.tpc = A->tpc;
  {  // warp-staged y stores (strategy 1, h = 1, no seg_row map, <= 40 KB of staging): on by
     // default for the far part of a panel-sliced handle, whose slices hold ~1 block per row
     // (C5: one scattered 4-byte store per row made a third of the far kernel's L2 requests;
     // staged + streaming stores: 1.25 -> 1.13 ms); YASPMV_WSTAGE = 0 / 1 / 2 overrides
    const char* e = std::getenv("YASPMV_WSTAGE");
    // (also on for the fused exchange's peer stores: each warp's rows go to every peer as
    // contiguous runs instead of P scattered stores per row)
    const int want = e ? std::atoi(e) : ((A->band_on || peers) ? 2 : 0);
    a.wstage = (want && p.h == 1 && p.rc == 0 && !ablate && c.n_zero == 0 &&
                A->d.seg_row == nullptr && (int64_t)p.C * p.T * A->vsize <= 40 * 1024)
                   ? want
                   : 0;
  }
  a.spin_limit = debug_spin_limit();
  a.spin_tile = debug_spin_slot();
  if (ablate && p.rc > 0) return fail(YASPMV_EUNSUPPORTED, "ablation / probe variants are strategy-1 kernels");
  if (peers && p.S == 1) {  // S > 1: the kernel writes tmp, the combine writes the peers
    a.npeer = peers->n;
    a.peer_mc = peers->mc;
    for (int q = 0; q < peers->n; ++q) a.peer_out[q] = peers->p[q];
  }
  if (ablate & ABL_DEFER_CARRY) {
    if (p.h != 1 || p.S != 1) return fail(YASPMV_EUNSUPPORTED, "ablation variants need h = 1, S = 1");
    if (A->abl_ntiles < c.ntiles) {
      if (A->d_dep_row) cudaFree(A->d_dep_row);
      A->d_dep_row = nullptr;
      CUDA_TRY(cudaMalloc((void**)&A->d_dep_row, c.ntiles * sizeof(int64_t)));
      A->abl_ntiles = c.ntiles;
    }
    a.dep_row = (ablate & ABL_NO_FIXUP) ? nullptr : A->d_dep_row;
  }
  if (p.S == 1) a.epi = (in_norm2 ? 1 : 0) | (out_norm2 ? 2 : 0);
  // (npeer > 0 selects the EPI = 2 instance: epilogue + peer stores)
  A->kern->launch(a, p.C, A->grid, stream);
  CUDA_TRY(cudaGetLastError());
  if ((ablate & ABL_DEFER_CARRY) && !(ablate & ABL_NO_FIXUP)) {
    launch_carry_fixup(A->d.status, A->d.carry, A->d_dep_row, c.ntiles, y, A->dtype, stream, 2);
    CUDA_TRY(cudaGetLastError());
  }
  if (p.S > 1 && !skip_combine) {
    launch_combine(A->d.tmp, y, c.m, c.MB * p.h, p.S, A->dtype, stream, in_norm2, out_norm2 ? A->d_part : nullptr,
                   peers);
    CUDA_TRY(cudaGetLastError());
  }
  if (out_norm2) {
    launch_sum_f64(A->d_part, npart, out_norm2, A->d_scratch, stream);
    CUDA_TRY(cudaGetLastError());
  }
  return YASPMV_OK;
}

// y := A x: the plain path, or for a panel-sliced BCCOO+ handle the far part (plain path,
// y := A_far x) followed by the band kernel (y += slices, in order; epilogue on the result)
// profiling (yaspmv_profile_begin): events of the current call, recorded between the
// kernel groups on the launching stream (stage 0 plain/far part, 1 band kernel, 2 sum)
cudaEvent_t* prof_events(yaspmv_matrix A) {
  if (!A->prof_on) return nullptr;
  std::array<cudaEvent_t, 4> ev{};
  for (auto& e : ev)
    if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
  A->prof_ev.push_back(ev);
  return A->prof_ev.back().data();
}

yaspmv_status run_spmv(yaspmv_matrix A, const void* x, void* y, void* stream, const double* in_norm2 = nullptr,
                       double* out_norm2 = nullptr, int ablate = 0, const PeerOut* peers = nullptr) {
  cudaEvent_t* ev = prof_events(A);
  cudaStream_t cs = (cudaStream_t)stream;
  if (!A->band_on) {
    if (ev) cudaEventRecord(ev[0], cs);
    yaspmv_status st = run_spmv_plain(A, x, y, stream, in_norm2, out_norm2, ablate, peers);
    if (ev) {
      cudaEventRecord(ev[1], cs);
      cudaEventRecord(ev[2], cs);
      cudaEventRecord(ev[3], cs);
    }
    return st;
  }
  if (ablate) return fail(YASPMV_EUNSUPPORTED, "ablation variants run the plain format only");
  if (peers && !A->pan.g.fip && !(A->can.p.S > 1 && A->can.ntiles > 0))
    return fail(YASPMV_EUNSUPPORTED,
                "fused exchange of a panel-sliced handle: the far part needs S > 1 (its slices stay in tmp) or P7");
  if (A->can.m == 0) {
    if (out_norm2) CUDA_TRY(cudaMemsetAsync(out_norm2, 0, sizeof(double), (cudaStream_t)stream));
    return YASPMV_OK;
  }
  DeviceGuard dg(A->device);
  if (peers && peers->n > YASPMV_MAX_RANKS) return fail(YASPMV_EINVAL, "too many peers");
  if (ev) cudaEventRecord(ev[0], cs);
  // far part: BCCOO+ slices stay in tmp, the band kernel combines them (no combine kernel);
  // P7: the far entries are the panels' slice 0 — no far launch, acc starts at 0
  const bool fip = A->pan.g.fip != 0;
  const bool fold = !fip && A->can.p.S > 1 && A->can.ntiles > 0;
  if (!fip) {
    yaspmv_status st = run_spmv_plain(A, x, y, stream, nullptr, nullptr, 0, nullptr, fold);
    if (st != YASPMV_OK) return st;
  }
  if (ev) cudaEventRecord(ev[1], cs);
  const PanelGeom& g = A->pan.g;
  PanelArgs pa;
  pa.col16 = A->pd.col16;
  pa.val = A->pd.val;
  pa.flags = A->pd.flags;
  pa.panel_blk0 = A->pd.panel_blk0;
  pa.slice_ptr = A->pd.slice_ptr;
  pa.stop_ptr = A->pd.stop_ptr;
  pa.first_row = A->pd.first_row;
  pa.tile_rank = A->pd.tile_rank;
  pa.x = x;
  pa.y = y;
  pa.far_col = A->pd.far_col;
  pa.far_blk0 = A->pd.far_blk0;
  pa.fip = fip ? 1 : 0;
  pa.init = fold ? A->d.tmp : y;
  pa.ninit = fip ? 0 : fold ? A->can.p.S : 1;
  pa.init_stride = A->can.MB * A->can.p.h;
  pa.m = A->can.m;
  pa.n = A->can.n;
  pa.R = g.R;
  pa.W = g.W;
  pa.B = g.B;
  pa.col0 = g.col0;
  pa.KS = g.NS();
  pa.npanels = g.npanels;
  pa.epi = (in_norm2 ? 1 : 0) | (out_norm2 ? 2 : 0);
  // the band kernel as a programmatic dependent of the far kernel just launched (not after
  // a memset, not with P7, whose far phase gathers x at once)
  pa.pdl = (!fip && A->can.ntiles > 0 && !(A->can.p.flags & YASPMV_NO_PDL)) ? 1 : 0;
  pa.in_norm2 = in_norm2;
  pa.part = A->pd.part;
  if (peers) {  // fused exchange: the band kernel's epilogue writes every rank's copy of x
    pa.npeer = peers->n;
    pa.peer_mc = peers->mc;
    for (int q = 0; q < peers->n; ++q) pa.peer_out[q] = peers->p[q];
  }
  const int e = launch_panel(pa, A->dtype, stream);
  if (e != 0) return fail(YASPMV_ECUDA, std::string("panel kernel: ") + cudaGetErrorString((cudaError_t)e));
  if (ev) cudaEventRecord(ev[2], cs);
  if (out_norm2) {
    launch_sum_f64(A->pd.part, g.npanels, out_norm2, A->pd.scratch, stream);
    CUDA_TRY(cudaGetLastError());
  }
  if (ev) cudaEventRecord(ev[3], cs);
  return YASPMV_OK;
}

}  // namespace

// switch the launch-time parameters (strategy, tiles per CTA) of an encoded handle
yaspmv_status set_launch(yaspmv_matrix A, int rc, int tpc) {
  const int orc = A->can.p.rc, otpc = A->can.p.tpc, oldt = A->tpc;
  const KernelEntry* oldk = A->kern;
  const int64_t oldgrid = A->grid;
  A->can.p.rc = rc;
  A->can.p.tpc = tpc;
  yaspmv_status st = select_kernel(A);
  if (st != YASPMV_OK) {
    A->can.p.rc = orc;
    A->can.p.tpc = otpc;
    A->kern = oldk;
    A->grid = oldgrid;
    A->tpc = oldt;
  }
  return st;
}

yaspmv_status install_canonical(yaspmv_matrix A, Canonical&& c, int flags) {
  return install_canonical_impl(A, std::move(c), flags);
}

yaspmv_status run_spmv_peers(yaspmv_matrix A, const void* x, const double* in_norm2, double* out_norm2,
                             const yaspmv::PeerOut& peers, void* stream) {
  return run_spmv(A, x, nullptr, stream, in_norm2, out_norm2, 0, &peers);
}

// =====================================================================================
extern "C" {

const char* yaspmv_last_error(void) { return g_err.c_str(); }
const char* yaspmv_version(void) { return "yaspmv-b200 0.1 (sm_100a)"; }

yaspmv_status yaspmv_l2_persist(int32_t device, int64_t bytes, int64_t* set_bytes) {
  int ndev = 0;
  CUDA_TRY(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev || bytes < 0) return fail(YASPMV_EINVAL, "bad device or bytes");
  DeviceGuard dg(device);
  int mx = 0;
  CUDA_TRY(cudaDeviceGetAttribute(&mx, cudaDevAttrMaxPersistingL2CacheSize, device));
  const size_t want = (size_t)std::min<int64_t>(bytes, (int64_t)mx);
  CUDA_TRY(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, want));
  if (set_bytes) {
    size_t now = 0;
    CUDA_TRY(cudaDeviceGetLimit(&now, cudaLimitPersistingL2CacheSize));
    *set_bytes = (int64_t)now;
  }
  return YASPMV_OK;
}

yaspmv_status yaspmv_build_csr(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                               const void* vals, yaspmv_dtype dtype, const yaspmv_params* params,
                               int32_t device, yaspmv_matrix* out) {
  yaspmv::TraceRange tr_("yaspmv:build_csr");
  if (!out) return fail(YASPMV_EINVAL, "out is NULL");
  *out = nullptr;
  if (dtype != YASPMV_F32 && dtype != YASPMV_F64) return fail(YASPMV_EINVAL, "bad dtype");
  yaspmv_status st = check_device(device);
  if (st != YASPMV_OK) return st;
  std::unique_ptr<yaspmv_matrix_s> A(new (std::nothrow) yaspmv_matrix_s());
  if (!A) return fail(YASPMV_ENOMEM, "handle allocation failed");
  A->device = device;
  A->dtype = dtype;
  A->vsize = dtype == YASPMV_F32 ? 4 : 8;
  if ((st = normalize_csr(m, n, row_ptr, col_idx, vals, A->vsize, A->csr)) != YASPMV_OK) return st;
  if ((st = build_common(A.get(), from_abi(params))) != YASPMV_OK) return st;
  *out = A.release();
  return YASPMV_OK;
}

yaspmv_status yaspmv_build_coo(int64_t m, int64_t n, int64_t nnz, const int32_t* row_idx, const int32_t* col_idx,
                               const void* vals, yaspmv_dtype dtype, const yaspmv_params* params, int32_t device,
                               yaspmv_matrix* out) {
  yaspmv::TraceRange tr_("yaspmv:build_coo");
  if (!out) return fail(YASPMV_EINVAL, "out is NULL");
  *out = nullptr;
  if (dtype != YASPMV_F32 && dtype != YASPMV_F64) return fail(YASPMV_EINVAL, "bad dtype");
  yaspmv_status st = check_device(device);
  if (st != YASPMV_OK) return st;
  std::unique_ptr<yaspmv_matrix_s> A(new (std::nothrow) yaspmv_matrix_s());
  if (!A) return fail(YASPMV_ENOMEM, "handle allocation failed");
  A->device = device;
  A->dtype = dtype;
  A->vsize = dtype == YASPMV_F32 ? 4 : 8;
  if ((st = normalize_coo(m, n, nnz, row_idx, col_idx, vals, A->vsize, A->csr)) != YASPMV_OK) return st;
  if ((st = build_common(A.get(), from_abi(params))) != YASPMV_OK) return st;
  *out = A.release();
  return YASPMV_OK;
}

void yaspmv_free(yaspmv_matrix A) { delete A; }

yaspmv_status yaspmv_profile_begin(yaspmv_matrix A) {
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle");
  CUDA_TRY(cudaSetDevice(A->device));
  for (auto& ev : A->prof_ev)
    for (cudaEvent_t e : ev) cudaEventDestroy(e);
  A->prof_ev.clear();
  A->prof_on = true;
  return YASPMV_OK;
}

yaspmv_status yaspmv_profile_end(yaspmv_matrix A, double* ms, int32_t n, int64_t* calls) {
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  A->prof_on = false;
  double acc[3] = {0, 0, 0};
  yaspmv_status st = YASPMV_OK;
  if (!A->prof_ev.empty()) {
    cudaSetDevice(A->device);
    for (auto& ev : A->prof_ev) {
      if (cudaEventSynchronize(ev[3]) != cudaSuccess) st = fail(YASPMV_ECUDA, "profiling events failed");
      for (int s = 0; s < 3 && st == YASPMV_OK; ++s) {
        float t = 0;
        if (cudaEventElapsedTime(&t, ev[s], ev[s + 1]) == cudaSuccess) acc[s] += t;
      }
    }
  }
  if (calls) *calls = (int64_t)A->prof_ev.size();
  for (int s = 0; s < n && s < 3; ++s)
    if (ms) ms[s] = acc[s];
  for (auto& ev : A->prof_ev)
    for (cudaEvent_t e : ev) cudaEventDestroy(e);
  A->prof_ev.clear();
  return st;
}

yaspmv_status yaspmv_reencode(yaspmv_matrix A, const yaspmv_params* params) {
  yaspmv::TraceRange tr_("yaspmv:reencode");
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (!A->have_csr) return fail(YASPMV_EINVAL, "handle was built with YASPMV_DROP_CSR");
  Params want = from_abi(params);
  const Params& cur = A->can.p;
  if (!want.h) want.h = cur.h;
  if (!want.w) want.w = cur.w;
  if (!want.S) want.S = cur.S;
  if (!want.T) want.T = cur.T;
  if (!want.C) want.C = cur.C;
  if (!want.col_mode) want.col_mode = cur.col_mode;
  if (!want.empty_mode) want.empty_mode = cur.empty_mode;
  if (!params || !want.flags) want.flags = cur.flags;
  want.rc = want.rc == 0 ? cur.rc : (want.rc < 0 ? 0 : want.rc);
  if (!want.tpc) want.tpc = cur.tpc;
  // panel-sliced BCCOO+: 0 = keep the handle's band parameters, band = -1 = plain format
  if (want.band == 0) {
    want.band = cur.band;
    if (!want.pR) want.pR = cur.pR;
    if (!want.pW) want.pW = cur.pW;
    if (!want.col0) want.col0 = cur.col0;
    if (!want.bfar) want.bfar = cur.bfar;
  } else if (want.band < 0) {
    want.band = want.pR = want.pW = want.col0 = want.bfar = 0;
  }
  {  // only launch-time parameters change (strategy, tiles per CTA): no re-encode
    Params rp;
    if (A->device >= 0 && resolve_params(want, A->csr.m, A->csr.n, rp) == YASPMV_OK && rp.h == cur.h &&
        rp.w == cur.w && rp.S == cur.S && rp.T == cur.T && rp.C == cur.C && rp.col_mode == cur.col_mode &&
        (rp.empty_mode == 0 || rp.empty_mode == cur.empty_mode) && rp.flags == cur.flags && rp.band == cur.band &&
        rp.pR == cur.pR && rp.pW == cur.pW && rp.col0 == cur.col0 &&
        (rp.band == 0 || (rp.bfar ? rp.bfar : (int)YASPMV_FAR_SEPARATE) == cur.bfar))
      return set_launch(A, rp.rc, rp.tpc);
  }
  return encode_into(A, want);
}

yaspmv_status yaspmv_spmv(yaspmv_matrix A, const void* x, void* y, void* stream) {
  yaspmv::TraceRange tr_("yaspmv:spmv");
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle (built with device = -1): no CPU fallback");
  if (A->can.m > 0 && !y) return fail(YASPMV_EINVAL, "y is NULL");
  if (A->can.n > 0 && !x) return fail(YASPMV_EINVAL, "x is NULL");
  const int64_t xb = A->can.n * A->vsize, yb = A->can.m * A->vsize;
  const char* xc = static_cast<const char*>(x);
  const char* yc = static_cast<const char*>(y);
  if (xb > 0 && yb > 0 && xc < yc + yb && yc < xc + xb) return fail(YASPMV_EINVAL, "x and y overlap");
  if (((uintptr_t)x) % ((uintptr_t)A->can.p.w * A->vsize) != 0)
    return fail(YASPMV_EINVAL, "x must be aligned to w * sizeof(value) bytes");
  return run_spmv(A, x, y, stream);
}

yaspmv_status yaspmv_spmv_power(yaspmv_matrix A, const void* x, void* y, const double* in_norm2, double* out_norm2,
                                void* stream) {
  yaspmv::TraceRange tr_("yaspmv:spmv_power");
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle (built with device = -1): no CPU fallback");
  if (A->can.m > 0 && !y) return fail(YASPMV_EINVAL, "y is NULL");
  if (A->can.n > 0 && !x) return fail(YASPMV_EINVAL, "x is NULL");
  const int64_t xb = A->can.n * A->vsize, yb = A->can.m * A->vsize;
  const char* xc = static_cast<const char*>(x);
  const char* yc = static_cast<const char*>(y);
  if (xb > 0 && yb > 0 && xc < yc + yb && yc < xc + xb) return fail(YASPMV_EINVAL, "x and y overlap");
  if (((uintptr_t)x) % ((uintptr_t)A->can.p.w * A->vsize) != 0)
    return fail(YASPMV_EINVAL, "x must be aligned to w * sizeof(value) bytes");
  return run_spmv(A, x, y, stream, in_norm2, out_norm2);
}

yaspmv_status yaspmv_spmv_host(yaspmv_matrix A, const void* x_host, void* y_host, void* stream) {
  yaspmv::TraceRange tr_("yaspmv:spmv_host");
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle: no CPU fallback");
  const size_t xb = (size_t)A->can.n * A->vsize, yb = (size_t)A->can.m * A->vsize;
  CUDA_TRY(cudaSetDevice(A->device));
  if (!A->xs && xb) CUDA_TRY(cudaMalloc(&A->xs, xb));
  if (!A->ys && yb) CUDA_TRY(cudaMalloc(&A->ys, yb));
  cudaStream_t s = (cudaStream_t)stream;
  if (xb) CUDA_TRY(cudaMemcpyAsync(A->xs, x_host, xb, cudaMemcpyHostToDevice, s));
  yaspmv_status st = run_spmv(A, A->xs, A->ys, stream);
  if (st != YASPMV_OK) return st;
  if (yb) CUDA_TRY(cudaMemcpyAsync(y_host, A->ys, yb, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(cudaStreamSynchronize(s));
  return YASPMV_OK;
}

yaspmv_status yaspmv_spmv_host_async(yaspmv_matrix A, const void* x_host, void* y_host, void* stream) {
  yaspmv::TraceRange tr_("yaspmv:spmv_host_async");
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle: no CPU fallback");
  const size_t xb = (size_t)A->can.n * A->vsize, yb = (size_t)A->can.m * A->vsize;
  CUDA_TRY(cudaSetDevice(A->device));
  if (!A->s_in) {
    CUDA_TRY(cudaStreamCreateWithFlags(&A->s_in, cudaStreamNonBlocking));
    CUDA_TRY(cudaStreamCreateWithFlags(&A->s_out, cudaStreamNonBlocking));
    for (auto& s : A->hslot) {
      CUDA_TRY(cudaMalloc(&s.x, std::max<size_t>(xb, 16)));
      CUDA_TRY(cudaMalloc(&s.y, std::max<size_t>(yb, 16)));
      CUDA_TRY(cudaEventCreateWithFlags(&s.in, cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&s.comp, cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&s.done, cudaEventDisableTiming));
      CUDA_TRY(cudaEventRecord(s.done, A->s_out));
    }
  }
  auto& s = A->hslot[A->next_slot];
  A->next_slot = (A->next_slot + 1) % 3;
  cudaStream_t cs = (cudaStream_t)stream;
  CUDA_TRY(cudaStreamWaitEvent(A->s_in, s.done, 0));  // the slot's previous copy-out is done
  if (xb) CUDA_TRY(cudaMemcpyAsync(s.x, x_host, xb, cudaMemcpyHostToDevice, A->s_in));
  CUDA_TRY(cudaEventRecord(s.in, A->s_in));
  CUDA_TRY(cudaStreamWaitEvent(cs, s.in, 0));
  yaspmv_status st = run_spmv(A, s.x, s.y, stream);
  if (st != YASPMV_OK) return st;
  CUDA_TRY(cudaEventRecord(s.comp, cs));
  CUDA_TRY(cudaStreamWaitEvent(A->s_out, s.comp, 0));
  if (yb) CUDA_TRY(cudaMemcpyAsync(y_host, s.y, yb, cudaMemcpyDeviceToHost, A->s_out));
  CUDA_TRY(cudaEventRecord(s.done, A->s_out));
  return YASPMV_OK;
}

yaspmv_status yaspmv_host_sync(yaspmv_matrix A) {
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->s_out) {
    CUDA_TRY(cudaSetDevice(A->device));
    CUDA_TRY(cudaStreamSynchronize(A->s_out));
  }
  return YASPMV_OK;
}

int32_t yaspmv_launches_per_spmv(yaspmv_matrix A) {
  if (!A || A->can.m == 0) return 0;
  const int band = A->band_on && A->pan.g.npanels > 0 ? 1 : 0;
  if (A->band_on && A->pan.g.fip) return band;  // the band kernel alone (P7)
  if (A->can.ntiles == 0) return band;  // memset (+ the band kernel)
  if (band) return 2;                   // far part (its slices combined by the band kernel) + band
  return A->can.p.S > 1 ? 2 : 1;
}

yaspmv_status yaspmv_ablation_spmv(yaspmv_matrix A, int32_t variant, const void* x, void* y, void* stream) {
  if (!A) return fail(YASPMV_EINVAL, "NULL handle");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle");
  if (variant < 1 || variant > 12) return fail(YASPMV_EINVAL, "ablation variant must be in 1..12");
  if (variant != 3 && (A->can.p.h != 1 || A->can.p.w != 1))
    return fail(YASPMV_EUNSUPPORTED, "ablation variants / probes are compiled for 1x1 blocks only");
  const int ab = variant == 1   ? ABL_DEFER_CARRY
                 : variant == 2 ? ABL_NO_SKIP
                 : variant == 4 ? ABL_GATHER_ONLY
                 : variant == 5 ? ABL_STREAM_ONLY
                 : variant == 6 ? (ABL_GATHER_ONLY | ABL_GATHER_L2)
                 : variant == 7 ? (ABL_DEFER_CARRY | ABL_NO_FIXUP)
                 : variant == 8 ? ABL_STOP_SCAN
                 : variant == 9 ? (ABL_DEFER_CARRY | ABL_NO_FIXUP | ABL_NO_YSTORE)
                 : variant == 10 ? (ABL_STOP_SCAN | ABL_PROBE_PUB)
                 : variant == 11 ? (ABL_STOP_SCAN | ABL_PROBE_ST)
                 : variant == 12 ? ABL_NO_PUBLISH0
                                 : 0;
  return run_spmv(A, x, y, stream, nullptr, nullptr, ab);
}

int64_t yaspmv_ablation_tree_scratch_bytes(int64_t n_elem) {
  const int64_t ntiles = (n_elem + 1023) / 1024;
  return ntiles * (int64_t)(8 + 8 + 8);
}

yaspmv_status yaspmv_ablation_tree(const int32_t* rows, const uint8_t* flags, const int32_t* tile_seg0,
                                   const int32_t* col, const void* val, int64_t n_elem, const void* x, void* y,
                                   int64_t m, yaspmv_dtype dtype, void* scratch, int64_t scratch_bytes, void* stream) {
  if (n_elem < 0 || m < 0 || (!rows && (!flags || !tile_seg0))) return fail(YASPMV_EINVAL, "bad tree arguments");
  if (scratch_bytes < yaspmv_ablation_tree_scratch_bytes(n_elem)) return fail(YASPMV_EINVAL, "scratch too small");
  const int64_t ntiles = (n_elem + 1023) / 1024;
  unsigned long long* status = static_cast<unsigned long long*>(scratch);
  double* carry = reinterpret_cast<double*>(status + ntiles);
  int64_t* dep = reinterpret_cast<int64_t*>(carry + ntiles);
  int e = launch_tree_segsum(rows, flags, tile_seg0, col, val, n_elem, x, y, m, dtype, status, carry, dep, stream);
  if (e) return fail(YASPMV_ECUDA, std::string("tree kernel: ") + cudaGetErrorString((cudaError_t)e));
  return YASPMV_OK;
}

int32_t yaspmv_launches_per_power_step(yaspmv_matrix A) {
  if (!A || A->can.m == 0) return 0;
  if (A->band_on) return yaspmv_launches_per_spmv(A) + 2;  // far (+ combine) + band + the y^2 sum
  if (A->can.ntiles == 0) return 0;
  return yaspmv_launches_per_spmv(A) + 2;  // + the two-level sum of the y^2 partials
}

yaspmv_status yaspmv_get_info(yaspmv_matrix A, yaspmv_info* o) {
  if (!A || !o) return fail(YASPMV_EINVAL, "NULL argument");
  const Canonical& c = A->can;
  std::memset(o, 0, sizeof(*o));
  o->m = c.m;
  o->n = c.n;
  o->nnz = A->band_on ? A->nnz_total : c.nnz;
  o->MB = c.MB;
  o->NB = c.NB;
  o->SW = c.SW;
  o->nnzb = c.nnzb;
  o->nnzb_pad = c.nnzb_pad;
  o->ntiles = c.ntiles;
  o->n_stops = c.n_stops;
  o->n_filler = c.n_filler;
  o->n_zero_rows = c.n_zero;
  o->format_bytes = format_bytes(A);
  o->alg_bytes = alg_bytes(A);
  o->footprint_bytes = footprint_bytes(c.nnzb, c.p.h, c.p.w, A->vsize, col_bytes(c.p.col_mode));
  o->params = to_abi(c.p);
  if (A->device >= 0) o->params.tiles_per_cta = A->tpc;  // the resolved value
  o->dtype = A->dtype;
  o->device = A->device;
  o->has_seg_row = c.has_seg_row;
  o->regs_per_thread = A->regs;
  o->build_seconds = A->build_s;
  o->tune_seconds = A->tune_s;
  o->tune_candidates = A->tune_candidates;
  if (A->band_on) {
    o->band_blocks = A->pan.nband;
    o->band_blocks_pad = A->pan.nband_pad;
    o->band_panels = A->pan.g.npanels;
    o->band_slices = A->pan.g.KS;
    o->band_far_blocks_pad = A->pan.nfar_pad;
    o->band_stops = A->pan.n_stops;
    o->band_format_bytes = band_format_bytes(A);
  }
  return YASPMV_OK;
}

}  // extern "C"
