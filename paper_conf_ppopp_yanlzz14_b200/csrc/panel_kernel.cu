// panel_kernel.cu — K4, the band kernel of the panel-sliced BCCOO+ format (DESIGN.md §2.1,
// §6.6).  One CTA per row panel of R rows (PAPER.md's workgroup, walking the
// panel's band stream in workgroup-level tiles of BT*BC blocks):
//
//   prologue  acc[0..R) := y[panel rows] (the far part's result, already in y); the
//             panel's slice offsets to shared memory; x windows of the first three slices
//             (W values each, plus the slices' row-occupancy bitmaps) requested with
//             cp.async.bulk on an mbarrier each — the part of x one BCCOO+ slice uses
//             (P:154), staged in shared memory so that every gather of the slice is an
//             LDS instead of a 32-byte L2 request;
//   per tile  128-bit streaming loads of the thread tile (values, u16 column offsets, the
//             BT flag bits; the next tile's loads are issued before this tile's math),
//             gathers from the resident windows, products, the per-thread sequential
//             segmented sum (strategy 1), the workgroup segmented scan of
//             (has_stop, last partial sum), then the segment sums are
//             added to acc[row] slice by slice (ascending k: the BCCOO+ combine order,
//             P:184), rows found through the slice's occupancy bitmap (reading P6);
//             a segment that runs into the next tile carries its partial sum in the CTA
//             (the tiles of a panel run in order inside one workgroup, so the
//             adjacent-synchronization chain of P:295-298 never leaves the SM);
//   epilogue  y[panel rows] := acc (optionally scaled; per-panel sum of y^2).
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.hpp"
#include "panel.hpp"

namespace yaspmv {
namespace {

constexpr int BT = PANEL_BT, BC = PANEL_BC, NWARP = BC / 32;

__device__ __forceinline__ uint64_t pol_evict_first() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ void ld16(const void* p, uint64_t pol, uint32_t* w) {
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3])
               : "l"(p), "l"(pol));
}
__device__ __forceinline__ uint32_t ld_flags16(const uint8_t* p) {
  unsigned short v;
  asm volatile("ld.global.nc.L1::no_allocate.u16 %0, [%1];" : "=h"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_test(uint64_t* bar, unsigned parity) {
  uint32_t ok;
  asm volatile(
      "{ .reg .pred p; mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
  while (!mbar_test(bar, parity)) {
  }
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

// shared-memory layout (dynamic part): acc[R] | 3 x { window[W + 4] | occ[NW] | pre[NW] }
struct Layout {
  int64_t wbytes, bufbytes;
  __host__ __device__ Layout(int64_t R, int64_t W) {
    wbytes = ((W + 4) * 4 + 15) / 16 * 16;
    bufbytes = wbytes + (R / 32) * 4 + (R / 32) * 2;
    bufbytes = (bufbytes + 15) / 16 * 16;
  }
};

struct PanelShared {
  int sp[PANEL_MAX_KS + 1];   // slice_ptr of the panel
  int st[PANEL_MAX_KS + 1];   // stop_ptr of the panel
  uint64_t bar[PANEL_NBUF];
  float wv[NWARP];
  int wf[NWARP];
  int wn[NWARP];
  float cin;                  // carry into the next tile (partial sum of an open segment)
  int s_before;               // row stops of the panel before the current tile
  double ss[NWARP];
};

// the row (inside the panel) of the rank-th stop of a slice: the rank-th set bit of its
// occupancy bitmap (reading P6), through the per-word prefix counts
__device__ __forceinline__ int select_row(const uint32_t* occ, const uint16_t* pre, int nw, int rank) {
  int lo = 0, hi = nw - 1;  // largest w with pre[w] <= rank
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if ((int)pre[mid] <= rank) lo = mid;
    else hi = mid - 1;
  }
  const unsigned pos = __fns(occ[lo], 0, rank - (int)pre[lo] + 1);
  return lo * 32 + (int)pos;
}
// the next row after `row` that holds an entry of the slice
__device__ __forceinline__ int next_row(const uint32_t* occ, int row) {
  int w = (row + 1) >> 5;
  uint32_t bits = occ[w] & (0xFFFFFFFFu << ((row + 1) & 31));
  while (bits == 0) bits = occ[++w];
  return w * 32 + __ffs(bits) - 1;
}

template <typename VT>
__global__ void __launch_bounds__(BC, 1) panel_kernel(const PanelArgs a) {
  extern __shared__ __align__(16) unsigned char dsm[];
  __shared__ PanelShared sh;
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const int64_t p = blockIdx.x;
  const int R = (int)a.R, W = (int)a.W, KS = (int)a.KS, NW = R / 32;
  const Layout L(a.R, a.W);
  VT* acc = reinterpret_cast<VT*>(dsm);
  unsigned char* bufs = dsm + (int64_t)R * sizeof(VT);
  auto win = [&](int k) { return reinterpret_cast<VT*>(bufs + (k % PANEL_NBUF) * L.bufbytes); };
  auto occ_of = [&](int k) { return reinterpret_cast<uint32_t*>(bufs + (k % PANEL_NBUF) * L.bufbytes + L.wbytes); };
  auto pre_of = [&](int k) {
    return reinterpret_cast<uint16_t*>(bufs + (k % PANEL_NBUF) * L.bufbytes + L.wbytes + NW * 4);
  };
  const int64_t row0 = p * a.R;
  const int64_t cb = row0 + a.col0 - a.B;  // column base of the panel (P1)
  const VT* x = static_cast<const VT*>(a.x);
  VT* y = static_cast<VT*>(a.y);
  const int64_t xe = (int64_t)(reinterpret_cast<uintptr_t>(x) / sizeof(VT));
  // window of slice k: columns [cb + k*W, cb + (k+1)*W); element j of the window sits at
  // win[shift(k) + j], shift chosen so that shared and global addresses agree mod 16 B
  auto shift_of = [&](int k) { return (int)(((xe + cb + (int64_t)k * W) % 4 + 4) % 4); };

  // ---- prologue ---------------------------------------------------------------------
  for (int k = t; k <= KS; k += BC) {
    sh.sp[k] = a.slice_ptr[p * (KS + 1) + k];
    sh.st[k] = a.stop_ptr[p * (KS + 1) + k];
  }
  if (t == 0) {
    for (int b = 0; b < PANEL_NBUF; ++b) mbar_init(&sh.bar[b], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    sh.cin = 0.f;
    sh.s_before = 0;
  }
  const int rows = (int)min((int64_t)a.R, a.m - row0);
  for (int r = t; r < R; r += BC) acc[r] = r < rows ? y[row0 + r] : VT(0);
  __syncthreads();
  // thread 0 requests slice k into buffer k % 3 (W values of x + bitmap + prefix counts)
  auto issue = [&](int k) {
    uint64_t* bar = &sh.bar[k % PANEL_NBUF];
    if (k >= PANEL_NBUF) mbar_wait(bar, (unsigned)((k / PANEL_NBUF - 1) & 1));  // previous use landed
    VT* w = win(k);
    const int sh_k = shift_of(k);
    const int64_t base = cb + (int64_t)k * W;
    const int64_t lo = max((int64_t)0, base), hi = min((int64_t)a.n, base + W);
    unsigned tx = 0;
    int64_t alo = lo, ahi = lo;
    if (lo < hi) {
      alo = lo + ((4 - ((xe + lo) & 3)) & 3);
      ahi = hi - ((xe + hi) & 3);
      if (alo > ahi) alo = ahi = hi;
      for (int64_t j = lo; j < alo && j < hi; ++j) w[sh_k + (j - base)] = x[j];  // unaligned head
      for (int64_t j = max(ahi, alo); j < hi; ++j) w[sh_k + (j - base)] = x[j];  // unaligned tail
      tx += (unsigned)((ahi - alo) * sizeof(VT));
    }
    const int64_t rec = (p * KS + k) * (int64_t)NW;
    tx += NW * 4 + NW * 2;
    mbar_arrive_tx(bar, tx);
    if (ahi > alo) bulk_g2s(w + sh_k + (alo - base), x + alo, (unsigned)((ahi - alo) * sizeof(VT)), bar);
    bulk_g2s(occ_of(k), a.occ + rec, NW * 4, bar);
    bulk_g2s(pre_of(k), a.pre + rec, NW * 2, bar);
  };
  int issued = 0;  // slices requested so far (thread 0's count; every thread tracks it)
  if (t == 0)
    for (int k = 0; k < min(KS, PANEL_NBUF); ++k) issue(k);
  issued = min(KS, PANEL_NBUF);

  const int64_t pb0 = a.panel_blk0[p];
  const int ntl = (int)((a.panel_blk0[p + 1] - pb0) / PANEL_TC);
  const int nreal = sh.sp[KS];
  const uint64_t pol = pol_evict_first();
  const uint8_t* vbase = static_cast<const uint8_t*>(a.val);
  const uint8_t* cbase = static_cast<const uint8_t*>(a.col16);
  constexpr int VCH = BT * (int)sizeof(VT) / 16;  // 16-B chunks of values per thread
  constexpr int CCH = BT * 2 / 16;                 // 16-B chunks of u16 columns per thread
  uint32_t vn[VCH * 4], cn[CCH * 4], fn = 0;
  auto load_tile = [&](int j) {
    const int64_t tile = pb0 / PANEL_TC + j;
#pragma unroll
    for (int c = 0; c < VCH; ++c) ld16(vbase + (tile * (int64_t)BC * VCH + (int64_t)c * BC + t) * 16, pol, &vn[4 * c]);
#pragma unroll
    for (int c = 0; c < CCH; ++c) ld16(cbase + (tile * (int64_t)BC * CCH + (int64_t)c * BC + t) * 16, pol, &cn[4 * c]);
    fn = ld_flags16(a.flags + ((tile * PANEL_TC + (int64_t)t * BT) >> 3));
  };
  if (ntl > 0) load_tile(0);
  // slice containing panel block b (b < nreal)
  auto slice_of = [&](int b, int k) {
    while (b >= sh.sp[k + 1]) ++k;
    return k;
  };
  double ssq = 0.0;

  for (int j = 0; j < ntl; ++j) {
    uint32_t vw[VCH * 4], cw[CCH * 4];
#pragma unroll
    for (int q = 0; q < VCH * 4; ++q) vw[q] = vn[q];
#pragma unroll
    for (int q = 0; q < CCH * 4; ++q) cw[q] = cn[q];
    const uint32_t fl = fn;
    if (j + 1 < ntl) load_tile(j + 1);  // next tile's stream in flight during this one

    const int tb0 = j * PANEL_TC;               // first block of the tile (panel-relative)
    const int tb1 = min(tb0 + PANEL_TC, nreal);  // end of its real blocks
    const int bt0 = tb0 + t * BT;               // this thread's first block
    // slices of the tile: k_lo..k_hi (nothing if the tile is only padding)
    int k_lo = 0, k_hi = -1;
    if (tb0 < tb1) {
      int lo = 0, hi = KS - 1;  // largest k with sp[k] <= tb0
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (sh.sp[mid] <= tb0) lo = mid;
        else hi = mid - 1;
      }
      k_lo = slice_of(tb0, lo);
      k_hi = slice_of(tb1 - 1, k_lo);
    }
    // windows: slices below k_lo are finished; request up to k_lo + 2 into their buffers
    if (k_hi >= 0) {
      const int want = min(KS, k_lo + PANEL_NBUF);
      if (t == 0)
        for (int k = issued; k < want; ++k) issue(k);
      issued = max(issued, want);
      for (int k = k_lo; k <= min(k_hi, k_lo + PANEL_NBUF - 1); ++k) mbar_wait(&sh.bar[k % PANEL_NBUF], (k / PANEL_NBUF) & 1);
    }

    // ---- multiply: gathers from the resident windows (global x beyond them) ----------
    int kf = k_lo;
    if (bt0 < tb1) kf = slice_of(bt0, k_lo);
    VT pr[BT];
    {
      int k = kf;
      int sk = shift_of(k);
      const VT* wk = win(k);
#pragma unroll
      for (int i = 0; i < BT; ++i) {
        const int b = bt0 + i;
        VT v = VT(0);
        if (b < tb1) {
          if (b >= sh.sp[k + 1]) {
            k = slice_of(b, k);
            sk = shift_of(k);
            wk = win(k);
          }
          const int c = (int)((cw[i >> 1] >> (16 * (i & 1))) & 0xFFFFu);
          const VT xv = (k < k_lo + PANEL_NBUF) ? wk[sk + c] : __ldg(x + cb + (int64_t)k * W + c);
          v = __uint_as_float(vw[i]) * xv;
        }
        pr[i] = v;
      }
    }
    // ---- per-thread segmented sum: stops are '0' bits ------------------------
    const uint32_t stops = ~fl & 0xFFFFu;
    const int nst = __popc(stops);
    const int hs = nst > 0;
    VT tail = VT(0);
#pragma unroll
    for (int i = 0; i < BT; ++i) tail = ((stops >> i) & 1u) ? VT(0) : tail + pr[i];
    // ---- workgroup segmented scan of (has_stop, last partial sum) -------------
    int f = hs, nn = nst;
    VT v = tail;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int f2 = __shfl_up_sync(0xffffffffu, f, d);
      const int n2 = __shfl_up_sync(0xffffffffu, nn, d);
      const VT v2 = __shfl_up_sync(0xffffffffu, v, d);
      if (lane >= d) {
        if (!f) v = v2 + v;
        f |= f2;
        nn += n2;
      }
    }
    if (lane == 31) {
      sh.wf[wid] = f;
      sh.wn[wid] = nn;
      sh.wv[wid] = v;
    }
    int fx = __shfl_up_sync(0xffffffffu, f, 1);
    int nx = __shfl_up_sync(0xffffffffu, nn, 1);
    VT vx = __shfl_up_sync(0xffffffffu, v, 1);
    if (lane == 0) {
      fx = 0;
      nx = 0;
      vx = VT(0);
    }
    __syncthreads();
    int Fw = 0, Nw = 0, Fall = 0, Ntot = 0;
    VT Vw = VT(0), Vall = VT(0);
    for (int q = 0; q < NWARP; ++q) {
      const int fq = sh.wf[q];
      if (q < wid) {
        Vw = fq ? sh.wv[q] : Vw + sh.wv[q];
        Fw |= fq;
        Nw += sh.wn[q];
      }
      Vall = fq ? sh.wv[q] : Vall + sh.wv[q];
      Fall |= fq;
      Ntot += sh.wn[q];
    }
    const VT cin = sh.cin;
    const int sb = sh.s_before;
    const int Fex = Fw | fx;
    // exclusive carry into this thread's first segment: earlier threads of the tile, and
    // the open segment of the previous tile if no earlier thread of this tile has a stop
    const VT Vex = Fex ? (fx ? vx : Vw + vx) : cin + (Vw + vx);
    // ---- add the segment sums to acc[row], slice by slice (ascending k): one
    // phase per slice of the tile, a barrier between phases, so every acc[row] receives
    // its slices' sums in order (deterministic) and no two threads update a row at once
    {
      bool first = true;
      int s = sb + Nw + nx;  // panel stop index of this thread's next stop
      for (int kk = k_lo; kk <= k_hi; ++kk) {
        if (hs) {
          int k = kf, row = -1;
          VT run = VT(0);
#pragma unroll
          for (int i = 0; i < BT; ++i) {
            const int b = bt0 + i;
            if (b < tb1) {
              if (b >= sh.sp[k + 1]) k = slice_of(b, k);
              if (k == kk) {
                run = run + pr[i];
                if ((stops >> i) & 1u) {
                  const VT val = first ? run + Vex : run;
                  first = false;
                  const bool res = k < k_lo + PANEL_NBUF;
                  const int64_t rec = (p * KS + k) * (int64_t)NW;
                  const uint32_t* oc = res ? occ_of(k) : a.occ + rec;
                  row = row < 0 ? select_row(oc, res ? pre_of(k) : a.pre + rec, NW, s - sh.st[k]) : next_row(oc, row);
                  acc[row] = acc[row] + val;
                  ++s;
                  run = VT(0);
                }
              }
            }
          }
        }
        __syncthreads();
      }
    }
    if (t == 0) {
      sh.cin = Fall ? Vall : cin + Vall;  // the tile's open segment carries into the next tile
      sh.s_before = sb + Ntot;
    }
    __syncthreads();
  }

  // ---- epilogue: y := acc (scaled), sum of y^2 ----------------------------------------
  const double inv = (a.epi & 1) ? 1.0 / sqrt(a.in_norm2[0]) : 1.0;
  for (int r = t; r < rows; r += BC) {
    const VT o = (a.epi & 1) ? (VT)(acc[r] * inv) : acc[r];
    y[row0 + r] = o;
    ssq += (double)o * (double)o;
  }
  if (a.epi & 2) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ssq += __shfl_xor_sync(0xffffffffu, ssq, o);
    if (lane == 0) sh.ss[wid] = ssq;
    __syncthreads();
    if (t == 0) {
      double s2 = 0.0;
      for (int q = 0; q < NWARP; ++q) s2 += sh.ss[q];
      a.part[p] = s2;
    }
  }
}

}  // namespace

size_t panel_smem_bytes(int64_t R, int64_t W) {
  const Layout L(R, W);
  return (size_t)R * 4 + PANEL_NBUF * L.bufbytes;
}

int panel_attr(int64_t R, int64_t W, int* regs) {
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, panel_kernel<float>);
  if (e != cudaSuccess) return (int)e;
  *regs = fa.numRegs;
  int optin = 0, dev = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  const size_t need = panel_smem_bytes(R, W);
  if (need + fa.sharedSizeBytes > (size_t)optin) return (int)cudaErrorInvalidConfiguration;
  return (int)cudaFuncSetAttribute(panel_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                   optin - (int)fa.sharedSizeBytes);
}

int launch_panel(const PanelArgs& a, int dtype, void* stream) {
  if (dtype != 0) return (int)cudaErrorNotSupported;
  if (a.npanels == 0) return 0;
  panel_kernel<float><<<(unsigned)a.npanels, BC, panel_smem_bytes(a.R, a.W), (cudaStream_t)stream>>>(a);
  return (int)cudaGetLastError();
}

}  // namespace yaspmv
