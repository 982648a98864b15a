// panel_kernel.cu — K4, the band kernel of the panel-sliced BCCOO+ format (DESIGN.md §2.1,
// §6.6).  One CTA per row panel of R rows (PAPER.md's workgroup, walking the
// panel's band stream in workgroup-level tiles of BT*BC blocks):
//
//   prologue  acc[0..R) := 0; the panel's slice offsets to shared memory; the x windows
//             of the first two band slices (W values each) requested with cp.async.bulk
//             on an mbarrier — the part of x
//             one BCCOO+ slice uses, staged in shared memory so that every gather
//             of the slice is an LDS instead of a 32-byte L2 request;
//   P7        the far slice first: the same tiles with int32 columns, x gathered from
//             global memory (its latency overlaps the window loads and the other warps);
//   per slice the next slice's window is requested into the other buffer; the slice's
//             workgroup-level tiles (16 blocks x 32 threads = one warp; every slice is
//             padded to whole tiles, reading P4) go round-robin to the warps, which run
//             independently: 128-bit streaming loads of the thread tile (the warp's next
//             tile is already in flight), gathers from the window, products, the
//             per-thread sequential segmented sum (strategy 1), the warp's
//             segmented scan of (has_stop, last partial sum), and the carry into
//             the tile's first segment by adjacent synchronization with the slice's
//             earlier tiles — a decoupled look-back over per-tile records in shared
//             memory that stops at the nearest final carry-out; every segment
//             sum is added to acc[row], row = the slice's first row + the stop's rank
//             from the tile's first-result entry (reading P6).  Inside a slice every row has one segment, so no
//             two warps touch one row; a barrier between slices keeps each row's slice
//             sums in ascending order (the BCCOO+ combine order) — deterministic;
//   epilogue  y[panel rows] := the far part's result (its S slice vectors summed in fp64; none
//             with P7) + acc, optionally scaled; per-panel sum of y^2.
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

#include "common.hpp"
#include "panel.hpp"

namespace yaspmv {
namespace {

constexpr int BT = PANEL_BT;
#ifndef PANEL_ACC_RUN
#define PANEL_ACC_RUN 4  // positions per acc update chain (BT / RUN chains, RUN rounds)
#endif

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
__device__ __forceinline__ int ld_acquire_s32(const volatile int* p) {
  int v;
  asm volatile("ld.acquire.cta.shared::cta.b32 %0, [%1];" : "=r"(v) : "r"(smem_u32((const void*)p)) : "memory");
  return v;
}
// acc slot of panel row r (identity: padded or permuted layouts that spread the warp's
// stops, ~8 rows apart, over the banks cost more address arithmetic than the conflicts they
// remove — measured 2.26 / 2.43 ms vs 2.15 ms on C5)
__device__ __forceinline__ int swz(int r) { return r; }

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

// shared-memory layout (dynamic part): acc[R] | NBUF x window[W + 4] (window element j at
// shift + j; slot shift + W holds 0, the column of a FILLER block, reading P6)
struct Layout {
  int64_t wbytes, bufbytes;
  __host__ __device__ Layout(int64_t R, int64_t W) {
    (void)R;
    wbytes = ((W + 4) * 4 + 15) / 16 * 16;
    bufbytes = wbytes;
  }
};

constexpr int RING = 512, LAG = 128, MAXWARP = 32;
static_assert(PANEL_TC == 512, "tile index = block offset >> 9");
static_assert(RING > 2 * LAG + MAXWARP, "a look-back never reads a record slot that was reused");

struct PanelShared {
  int sp[PANEL_MAX_KS + 2];        // slice_ptr of the panel (NS + 1 entries)
  unsigned nemask[3];              // bit k: slice k is non-empty
  int fr[PANEL_MAX_KS + 1];        // first_row of every slice
  uint64_t bar[PANEL_NBUF];
  volatile int armed[PANEL_NBUF];  // window (non-empty band slice ordinal) armed on each buffer
  // carry records of the panel's tiles (decoupled look-back): rT = the tile's
  // aggregate (the tail after its last row stop, or its whole sum when it has none), rI =
  // its carry-out (= rT for a tile holding a stop or starting its slice, carry-in + rT
  // otherwise); tag 2(t+1): rT published, 2(t+1)+1: rI final as well
  float rT[RING];
  float rI[RING];
  volatile int rtag[RING];
  double ss[MAXWARP];
};

// Thread 0 requests the x window of the o-th non-empty band slice of the panel (slices
// kb0..KS-1; its slice id found from the slice offsets) into buffer o % NBUF: W values of x
// from column cb + (k - kb0)*W with cp.async.bulk on the buffer's mbarrier, the unaligned
// ends by plain loads, and the zero slot behind the window (a FILLER block's column, P6).
template <typename VT>
__device__ __forceinline__ void issue_window(PanelShared& sh, unsigned char* bufs, int64_t bufbytes, const VT* x,
                                          int64_t n, int64_t xe, int64_t cb, int W, int KS, int kb0, int o) {
  int k = kb0, oo = -1;
  for (; k < KS; ++k)
    if (sh.sp[k] != sh.sp[k + 1] && ++oo == o) break;
  if (k >= KS) return;
  uint64_t* bar = &sh.bar[o % PANEL_NBUF];
  if (o >= PANEL_NBUF) mbar_wait(bar, (unsigned)((o / PANEL_NBUF - 1) & 1));  // previous use landed
  VT* w = reinterpret_cast<VT*>(bufs + (o % PANEL_NBUF) * bufbytes);
  const int64_t base = cb + (int64_t)(k - kb0) * W;
  const int sh_k = (int)(((xe + base) % 4 + 4) % 4);
  const int64_t lo = max((int64_t)0, base), hi = min(n, base + W);
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
  w[sh_k + W] = VT(0);
  mbar_arrive_tx(bar, tx);
  if (ahi > alo) bulk_g2s(w + sh_k + (alo - base), x + alo, (unsigned)((ahi - alo) * sizeof(VT)), bar);
  __threadfence_block();
  sh.armed[o % PANEL_NBUF] = o;
}

template <typename VT, int NTH>
__global__ void __launch_bounds__(NTH, 1) panel_kernel(const PanelArgs a) {
  constexpr int NWARP = NTH / 32;
  static_assert(NWARP <= MAXWARP, "CTA size");
  extern __shared__ __align__(16) unsigned char dsm[];
  __shared__ PanelShared sh;
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const int64_t p = blockIdx.x;
  const int R = (int)a.R, W = (int)a.W, KS = (int)a.KS, fip = a.fip;
  const Layout L(a.R, a.W);
  VT* acc = reinterpret_cast<VT*>(dsm);
  unsigned char* bufs = dsm + (int64_t)R * sizeof(VT);
  auto win = [&](int o) { return reinterpret_cast<VT*>(bufs + (o % PANEL_NBUF) * L.bufbytes); };
  const int64_t row0 = p * a.R;
  const int64_t cb = row0 + a.col0 - a.B;  // column base of the panel (P1)
  const VT* x = static_cast<const VT*>(a.x);
  VT* y = static_cast<VT*>(a.y);
  const int64_t xe = (int64_t)(reinterpret_cast<uintptr_t>(x) / sizeof(VT));
  // window of band slice k (slice k - fip of the band): columns [cb + (k-fip)*W, + W);
  // element j of the window sits at win[shift(k) + j], shift chosen so that shared and
  // global addresses agree mod 16 B
  auto shift_of = [&](int k) { return (int)(((xe + cb + (int64_t)(k - fip) * W) % 4 + 4) % 4); };

  // ---- prologue ---------------------------------------------------------------------
  for (int k = t; k <= KS; k += NTH) {
    sh.sp[k] = a.slice_ptr[p * (KS + 1) + k];
    if (k < KS) sh.fr[k] = a.first_row[p * KS + k];
  }
  if (t < 96) {  // bit k: slice k holds blocks (KS <= 64 band slices + the P7 far slice)
    const bool ne = t < KS && a.slice_ptr[p * (KS + 1) + t] != a.slice_ptr[p * (KS + 1) + t + 1];
    const unsigned b = __ballot_sync(0xffffffffu, ne);
    if (lane == 0) sh.nemask[wid] = b;
  }
  for (int q = t; q < RING; q += NTH) sh.rtag[q] = 0;
  if (t == 0) {
    for (int b = 0; b < PANEL_NBUF; ++b) {
      mbar_init(&sh.bar[b], 1);
      sh.armed[b] = -1;
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  const int rows = (int)min((int64_t)a.R, a.m - row0);
  // acc := 0 (the far part's result joins in the epilogue, after this grid's wait on it)
  for (int r = t * (16 / (int)sizeof(VT)); r < R; r += NTH * (16 / (int)sizeof(VT)))
    *reinterpret_cast<uint4*>(acc + r) = make_uint4(0u, 0u, 0u, 0u);
  __syncthreads();
  const unsigned long long nemask = ((unsigned long long)sh.nemask[1] << 32) | sh.nemask[0];
  const unsigned nemask2 = sh.nemask[2];
  auto next_nonempty = [&](int k) {  // first slice >= k holding blocks (KS: none)
    const unsigned long long m = k < 64 ? nemask >> k : 0ull;
    if (m) return k + __ffsll((long long)m) - 1;
    const unsigned m2 = k < 96 ? nemask2 >> (max(k, 64) - 64) : 0u;
    return m2 ? max(k, 64) + __ffs((int)m2) - 1 : KS;
  };
  auto issue = [&](int ow) { issue_window<VT>(sh, bufs, L.bufbytes, x, a.n, xe, cb, W, KS, fip, ow); };
  const int hf = fip && sh.sp[0] != sh.sp[1];  // the panel has a non-empty far slice (P7)

  const int64_t pb0 = a.panel_blk0[p];
  const int64_t tile0 = pb0 / PANEL_TC;  // first tile of the panel
  // col16 holds band blocks only, far_col far-slice blocks only (P7)
  const int64_t c16_off = fip ? a.far_blk0[p + 1] / PANEL_TC : 0;
  const uint64_t pol = pol_evict_first();
  const uint8_t* vbase = static_cast<const uint8_t*>(a.val);
  const uint8_t* cbase = static_cast<const uint8_t*>(a.col16);
  constexpr int VCH = BT * (int)sizeof(VT) / 16;  // 16-B chunks of values per thread
  constexpr int CCH = BT * 2 / 16;                 // 16-B chunks of u16 columns per thread
  constexpr int FCH = BT * 4 / 16;                 // 16-B chunks of int32 far columns per thread

  double ssq = 0.0;
  int o = 0;  // non-empty ordinal of the current slice (the far slice included)

  // Warp NWARP-1 is the window producer; warps 0..NWARP-2 compute.  Between slices every
  // acc[row] must receive its slice o-1 sum before its slice o sum, and slice o-1's window
  // buffer may take a later band slice only when no warp reads it any more: named barrier
  // X_o (barrier.sync 1 + (o & 1), all NTH threads; the non-.aligned form: a warp may
  // arrive diverged after its lane-0 look-back or window requests).  A compute warp that is done with slice o-1
  // loads, multiplies and scans its first slice-o tile, and waits on X_o only before that
  // tile's first acc update; the producer passes X_o and requests the next window.  With P7
  // the far slice is slice 0 (no window; band window ordinal = o - hf).
  constexpr int NCW = NWARP - 1;
  if (wid == NWARP - 1) {
    int nne = 0;
    for (int kk = 0; kk < KS; ++kk) nne += sh.sp[kk] != sh.sp[kk + 1];
    if (lane == 0) {
      issue(0);
      issue(1);
    }
    for (int oo = 1; oo < nne; ++oo) {
      if (oo & 1) asm volatile("barrier.sync 2, %0;" ::"n"(NTH) : "memory");
      else asm volatile("barrier.sync 1, %0;" ::"n"(NTH) : "memory");
      if (lane == 0 && oo - 1 >= hf) issue(oo + 1 - hf);  // slice oo-1 held window oo-1-hf
    }
    // the far part's slice results of the panel rows, wanted by the epilogue: once the far
    // kernel is complete (programmatic dependent launch), pulled into L2 in the background
    if (a.ninit > 0 && rows > 0) {
      if (a.pdl) cudaGridDependencySynchronize();
      if (lane < a.ninit) {
        const VT* in = static_cast<const VT*>(a.init) + row0 + lane * a.init_stride;
        const uintptr_t b0 = reinterpret_cast<uintptr_t>(in) & ~(uintptr_t)15;
        const uintptr_t b1 = reinterpret_cast<uintptr_t>(in + rows) & ~(uintptr_t)15;
        if (b1 > b0)
          asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(b0), "r"((unsigned)(b1 - b0)) : "memory");
      }
    }
  }
  auto slice_barrier = [&](int oo) {
    if (oo & 1) asm volatile("barrier.sync 2, %0;" ::"n"(NTH) : "memory");
    else asm volatile("barrier.sync 1, %0;" ::"n"(NTH) : "memory");
  };

  // ---- one tile after its products: per-thread segmented sum, warp scan, carry record,
  // acc updates, look-back (shared by the far slice and the band slices) -----------------
  auto finish = [&](VT(&pr)[BT], const uint32_t fl_, const int tr, const int lt, const int u, const int frk,
                    bool& pending, auto&& prefetch) {
    const uint32_t stops = ~fl_ & 0xFFFFu;
    // per-thread segmented sum: pr[i] := sum of its segment up to block i
    const int nst = __popc(stops);
#pragma unroll
    for (int i = 1; i < BT; ++i) pr[i] = ((stops >> (i - 1)) & 1u) ? pr[i] : pr[i - 1] + pr[i];
    const VT tail = ((stops >> (BT - 1)) & 1u) ? VT(0) : pr[BT - 1];
    // warp segmented scan of (has_stop, last partial sum); the stop count rides in
    // the low 16 bits and the has-stop flag above (a sum of flags is non-zero iff their OR is)
    int fn_ = nst | ((nst > 0) << 16);
    VT v = tail;
    const bool allstop = __ballot_sync(0xffffffffu, nst > 0) == 0xffffffffu;
    int nx_fast = 0;
    if (allstop) {
      // every lane holds a stop (the common case): each lane's scanned value is its own
      // tail (the skip of P:222 at thread level), and the stops of the earlier lanes are
      // counted by bit planes of the per-lane counts (nst <= 16: five ballots + popc, no
      // shuffle chain)
      const unsigned ltm = (1u << lane) - 1u;
#pragma unroll
      for (int b = 0; b < 5; ++b) nx_fast += __popc(__ballot_sync(0xffffffffu, (nst >> b) & 1) & ltm) << b;
      fn_ = (nx_fast + nst) | (1 << 16);
    } else {
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const int g2 = __shfl_up_sync(0xffffffffu, fn_, d);
        const VT v2 = __shfl_up_sync(0xffffffffu, v, d);
        if (lane >= d) {
          if (!(fn_ >> 16)) v = v2 + v;
          fn_ += g2;
        }
      }
    }
    const int f = (fn_ >> 16) != 0;
    // publish the tile's carry record (before anything waits on others); its carry-out is
    // final at once when it holds a stop or starts its slice.  Before the next tile's loads
    // are issued: the fence would otherwise wait for them to land
    const bool final_now = f || u == 0;
    if (lane == 31) {
      sh.rT[lt % RING] = v;  // inclusive: the tail after the tile's last stop, or its sum
      if (final_now) sh.rI[lt % RING] = v;
      __threadfence_block();
      sh.rtag[lt % RING] = 2 * (lt + 1) + (final_now ? 1 : 0);
    }
    prefetch();  // the warp's next tile in flight during this tile's updates and look-back
    int fx, nx;
    if (allstop) {
      fx = lane > 0;
      nx = nx_fast;
    } else {
      const int gx = __shfl_up_sync(0xffffffffu, fn_, 1);
      fx = lane > 0 && (gx >> 16) != 0;
      nx = lane > 0 ? gx & 0xFFFF : 0;
    }
    VT vx = __shfl_up_sync(0xffffffffu, v, 1);
    if (lane == 0) vx = VT(0);
    if (pending) {  // every warp is done with slice o - 1 (acc order)
      slice_barrier(o);
      pending = false;
    }
    // add the segment sums to acc[row]: the s-th stop of the slice is row first_row + s
    // (reading P6), so this thread's stops take the rows from first_row + tile_rank + nx
    // on.  The first stop's row then also gets the earlier lanes' part (vx) — right away,
    // or, when the segment continues earlier tiles (dep), together with their carry after
    // the look-back: a fixed association, so y stays bitwise deterministic
    const bool dep = nst && !fx && u > 0;  // the warp's first stop continues earlier tiles
    const int row_first = frk + tr + nx;
    {
      // four independent update chains, one per quarter of the thread tile (positions
      // 4q..4q+3 own the rows from row_first + the stops before 4q on): their loads issue
      // back to back instead of one shared-memory round trip per stop; the chains touch
      // disjoint rows, so the result is the same as the sequential walk
      static_assert(BT == 16, "chains of PANEL_ACC_RUN positions");
      constexpr int RUN = PANEL_ACC_RUN, NQ = BT / RUN;
      VT* aq[NQ];
      {
        int c = 0;
#pragma unroll
        for (int q = 0; q < NQ; ++q) {
          aq[q] = acc + row_first + c;
          c += __popc(stops & (((1u << RUN) - 1u) << (RUN * q)));
        }
      }
#pragma unroll
      for (int r = 0; r < RUN; ++r) {
        VT l[NQ];
#pragma unroll
        for (int q = 0; q < NQ; ++q)
          if ((stops >> (RUN * q + r)) & 1u) l[q] = *aq[q];
#pragma unroll
        for (int q = 0; q < NQ; ++q)
          if ((stops >> (RUN * q + r)) & 1u) {
            *aq[q] = l[q] + pr[RUN * q + r];
            ++aq[q];
          }
      }
      if (nst && !dep) acc[swz(row_first)] = acc[swz(row_first)] + vx;
    }
    // carry-in of the tile's first segment: decoupled look-back over the slice's earlier
    // tiles back to the nearest one whose carry-out is final, then summed
    // forward — the same left-to-right sum from the segment's start whichever record the
    // walk stops at, so y is bitwise deterministic.  Needed by the warp's first stop (dep)
    // and, for a tile without a stop, by its own carry-out (a row spanning many tiles walks
    // O(warps) records per tile, not O(its length))
    const bool nostop = !allstop && !__shfl_sync(0xffffffffu, f, 31);
    const unsigned dball = __ballot_sync(0xffffffffu, dep);
    if (dball || (nostop && u > 0)) {
      VT carry = VT(0);
      if (lane == 0) {
        int q = lt - 1;
        for (;; --q) {
          int tg;
          while ((tg = ld_acquire_s32(&sh.rtag[q % RING])) < 2 * (q + 1)) __nanosleep(16);
          if (tg & 1) break;
        }
        // acquire loads of the tags order the record reads (no fence: it would wait for
        // the next tile's loads in flight)
        carry = sh.rI[q % RING];
        for (int r = q + 1; r < lt; ++r) carry = carry + sh.rT[r % RING];
      }
      carry = __shfl_sync(0xffffffffu, carry, 0);
      if (dep) acc[swz(row_first)] = acc[swz(row_first)] + (carry + vx);
      if (nostop && lane == 31) {  // v of lane 31 = the tile's whole sum
        sh.rI[lt % RING] = carry + v;
        __threadfence_block();
        sh.rtag[lt % RING] = 2 * (lt + 1) + 1;
      }
    }
  };
  // flow control (slices of more than LAG tiles only): the record slot of this tile must
  // have been released — the tile LAG before it has a final carry-out
  auto flow = [&](int lt, int u, int ntile_k) {
    if (ntile_k > LAG && u >= LAG) {
      if (lane == 0)
        while (sh.rtag[(lt - LAG) % RING] != 2 * (lt - LAG + 1) + 1) __nanosleep(32);
      __syncwarp();
    }
  };

  // ---- P7: the far slice (slice 0): int32 columns, gathers of x from global memory -------
  if (hf && wid < NCW) {
    const int ntile_f = sh.sp[1] >> 9;
    const int frk = sh.fr[0];
    const int64_t ft0 = a.far_blk0[p] / PANEL_TC;  // the panel's first far-slice tile
    const uint8_t* fcbase = static_cast<const uint8_t*>(a.far_col);
    bool pending = false;
    for (int u = wid; u < ntile_f; u += NCW) {
      flow(u, u, ntile_f);
      const int64_t tile = tile0 + u, ftile = ft0 + u;
      uint32_t fc[BT], fv[VCH * 4];
#pragma unroll
      for (int c = 0; c < FCH; ++c)
        ld16(fcbase + (ftile * (int64_t)32 * FCH + (int64_t)c * 32 + lane) * 16, pol, &fc[4 * c]);
#pragma unroll
      for (int c = 0; c < VCH; ++c)
        ld16(vbase + (tile * (int64_t)32 * VCH + (int64_t)c * 32 + lane) * 16, pol, &fv[4 * c]);
      const uint32_t flf = ld_flags16(a.flags + ((tile * PANEL_TC + (int64_t)lane * BT) >> 3));
      const int trf = __ldg(a.tile_rank + tile);
      VT pr[BT];
#pragma unroll
      for (int i = 0; i < BT; ++i)  // column n: a FILLER block, reads 0 (P7)
        pr[i] = fc[i] < (uint32_t)a.n ? __uint_as_float(fv[i]) * __ldg(x + fc[i]) : VT(0);
      finish(pr, flf, trf, u, u, frk, pending, [] {});
    }
  }

  // ---- the band slices -------------------------------------------------------------------
  int k = wid < NCW ? next_nonempty(fip) : KS;  // no band tiles for the producer
  o = hf;
  uint32_t vw[VCH * 4], cw[CCH * 4], fl = 0;
  int trank = 0;
  auto load_tile = [&](int lt) {  // panel-local tile: the thread's run (device layout)
    const int64_t tile = tile0 + lt, ctile = tile - c16_off;
#pragma unroll
    for (int c = 0; c < CCH; ++c) ld16(cbase + (ctile * (int64_t)32 * CCH + (int64_t)c * 32 + lane) * 16, pol, &cw[4 * c]);
#pragma unroll
    for (int c = 0; c < VCH; ++c) ld16(vbase + (tile * (int64_t)32 * VCH + (int64_t)c * 32 + lane) * 16, pol, &vw[4 * c]);
    fl = ld_flags16(a.flags + ((tile * PANEL_TC + (int64_t)lane * BT) >> 3));
    trank = __ldg(a.tile_rank + tile);
  };
  // this warp's first tile in slice kk or a later non-empty slice that has one: its
  // panel-local tile index, -1 if none
  // Tiles go to the compute warps round-robin over the panel's whole tile sequence (tile lt
  // to warp lt mod NCW, continuing across slice boundaries), not restarting at warp 0 in
  // every slice: the warps that finish slice o first take slice o+1's first tiles, so the
  // per-slice remainder does not pile up on the same warps (balance at the slice barriers)
  auto first_u = [&](int kk) {  // this warp's first slice-local tile index in slice kk
    const int l0 = sh.sp[kk] >> 9;
    return (wid - l0 % NCW + NCW) % NCW;
  };
  auto first_tile_from = [&](int kk) {
    kk = next_nonempty(kk);
    while (kk < KS && (sh.sp[kk + 1] - sh.sp[kk]) >> 9 <= first_u(kk)) kk = next_nonempty(kk + 1);
    return kk < KS ? (sh.sp[kk] >> 9) + first_u(kk) : -1;
  };
  if (k < KS) {  // the warp's first band tile in flight before the first window wait
    const int f = first_tile_from(k);
    if (f >= 0) load_tile(f);
  }
  while (k < KS) {
    const int ltile_k = sh.sp[k] >> 9;                     // panel-local first tile of the slice
    const int ntile_k = (sh.sp[k + 1] - sh.sp[k]) >> 9;    // tiles of the slice
    const int ow = o - hf;                                 // its window ordinal
    // window ow of slice k resident (a buffer two requests behind would alias the awaited
    // parity: wait until the request is armed first)
    while (sh.armed[ow % PANEL_NBUF] != ow) {
    }
    mbar_wait(&sh.bar[ow % PANEL_NBUF], (ow / PANEL_NBUF) & 1);
    const VT* wk = win(ow) + shift_of(k);
    const uint32_t wk_s = smem_u32(wk);
    const int frk = sh.fr[k];
    bool pending = o > 0;  // X_o still ahead of this warp
    for (int u = first_u(k); u < ntile_k; u += NCW) {
      const int lt = ltile_k + u;       // panel-local tile index (tag of its carry record)
      flow(lt, u, ntile_k);
      // ---- multiply: gathers from the slice's window --------------------------------
      VT pr[BT];
#pragma unroll
      for (int i = 0; i < BT; ++i) {
        // byte offset of the column in the window, added to the window's 32-bit shared address
        // (one shift-and-mask + one add per gather; measured 1.763 -> 1.757 ms against wk[c])
        const uint32_t cb4 = (i & 1) ? (cw[i >> 1] >> 16) << 2 : (cw[i >> 1] & 0xFFFFu) << 2;
        float xv;
        asm volatile("ld.shared.f32 %0, [%1];" : "=f"(xv) : "r"(wk_s + cb4));
        pr[i] = __uint_as_float(vw[i]) * xv;
      }
      const uint32_t flc = fl;
      const int trc = trank;
      finish(pr, flc, trc, lt, u, frk, pending, [&] {  // the warp's next tile
        if (u + NCW < ntile_k) {
          load_tile(lt + NCW);
        } else {
          const int f = first_tile_from(k + 1);
          if (f >= 0) load_tile(f);
        }
      });
    }
    if (pending) slice_barrier(o);  // no tile of this slice: still part of X_o
    k = next_nonempty(k + 1);
    ++o;
  }
  __syncthreads();  // the last slice's sums are in acc

  // ---- epilogue: y := far part + acc (scaled), sum of y^2 -------------------------------
  // y[r] = (s_0 + ... + s_{S-1}) + band, the far part's S slice results summed in ascending
  // order in fp64 (the BCCOO+ combine, Q11) and the band slices' fp32 sum added to it
  // in fp64: a fixed association, bitwise deterministic
  if (a.pdl && a.ninit > 0) cudaGridDependencySynchronize();  // the far kernel is complete
  const double inv = (a.epi & 1) ? 1.0 / sqrt(a.in_norm2[0]) : 1.0;
  const VT* in = static_cast<const VT*>(a.init) + row0;
  // the output: y, or in a fused exchange every rank's copy of the next x (peer stores, or one
  // store through a multicast mapping)
  auto store_y = [&](int64_t i, VT v) {
    if (a.peer_mc) {
      multimem_store(static_cast<VT*>(a.peer_out[0]) + i, v);
    } else if (a.npeer > 0) {
      for (int q = 0; q < a.npeer; ++q) static_cast<VT*>(a.peer_out[q])[i] = v;
    } else {
      y[i] = v;
    }
  };
  auto store_y4 = [&](int64_t i, float4 v) {
    if (a.peer_mc) {
      asm volatile("multimem.st.relaxed.sys.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(static_cast<float*>(a.peer_out[0]) + i),
                   "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
                   : "memory");
    } else if (a.npeer > 0) {
      for (int q = 0; q < a.npeer; ++q) *reinterpret_cast<float4*>(static_cast<float*>(a.peer_out[q]) + i) = v;
    } else {
      *reinterpret_cast<float4*>(y + i) = v;
    }
  };
  // y[r] = (VT)((s_0 + ... + s_{S-1} in fp64, ascending) + acc[r]) * inv)
  auto out_row = [&](int r, double s) {
    const VT o2 = a.ninit > 0 ? (VT)((s + (double)acc[swz(r)]) * inv)
                              : ((a.epi & 1) ? (VT)(acc[swz(r)] * inv) : acc[swz(r)]);
    store_y(row0 + r, o2);
    ssq += (double)o2 * (double)o2;
  };
  int rdone = 0;
  uintptr_t oal = a.npeer > 0 ? 0 : reinterpret_cast<uintptr_t>(y + row0);
  for (int q = 0; q < a.npeer; ++q) oal |= reinterpret_cast<uintptr_t>(static_cast<VT*>(a.peer_out[q]) + row0);
  if (sizeof(VT) == 4 && ((reinterpret_cast<uintptr_t>(in) | oal) & 15) == 0 && (a.init_stride & 3) == 0) {
    // 128-bit loads of the far part's slice results, every slice of two row quads in flight
    // at once (the epilogue runs with no other CTA on the SM to hide its latency)
    const int ng = rows >> 2;
    for (int g0 = t; g0 < ng; g0 += 2 * NTH) {
      double s[2][4];
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int j = 0; j < 4; ++j) s[h][j] = 0.0;
      for (int q0 = 0; q0 < a.ninit; q0 += 4) {
        float4 v[4][2];
#pragma unroll
        for (int dq = 0; dq < 4; ++dq)
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int g = g0 + h * NTH;
            v[dq][h] = (q0 + dq < a.ninit && g < ng)
                           ? __ldcs(reinterpret_cast<const float4*>(in + (int64_t)(q0 + dq) * a.init_stride) + g)
                           : make_float4(0.f, 0.f, 0.f, 0.f);
          }
#pragma unroll
        for (int dq = 0; dq < 4; ++dq)
          if (q0 + dq < a.ninit)
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              s[h][0] += (double)v[dq][h].x;
              s[h][1] += (double)v[dq][h].y;
              s[h][2] += (double)v[dq][h].z;
              s[h][3] += (double)v[dq][h].w;
            }
      }
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int g = g0 + h * NTH;
        if (g < ng) {
          const float4 ac = *reinterpret_cast<const float4*>(acc + 4 * g);
          float4 o;
          const float ai[4] = {ac.x, ac.y, ac.z, ac.w};
          float oi[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            oi[j] = a.ninit > 0 ? (float)((s[h][j] + (double)ai[j]) * inv) : ((a.epi & 1) ? (float)(ai[j] * inv) : ai[j]);
            ssq += (double)oi[j] * (double)oi[j];
          }
          o = make_float4(oi[0], oi[1], oi[2], oi[3]);
          store_y4(row0 + 4 * g, o);
        }
      }
    }
    rdone = ng * 4;
  }
  for (int r = rdone + t; r < rows; r += NTH) {  // unaligned rows (scalar)
    double s = 0.0;
    for (int q = 0; q < a.ninit; ++q) s += (double)__ldcs(in + q * a.init_stride + r);
    out_row(r, s);
  }
  if (a.epi & 2) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) ssq += __shfl_xor_sync(0xffffffffu, ssq, d);
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

// CTA size of the band kernel: PANEL_CTA, or YASPMV_PANEL_CTA in {512, 640, 704, 768, 896, 1024}
// (exploration; registers per thread = 64K / size)
static int panel_cta() {
  static int c = [] {
    const char* e = std::getenv("YASPMV_PANEL_CTA");
    const int v = e ? std::atoi(e) : PANEL_CTA;
    return (v == 512 || v == 640 || v == 704 || v == 768 || v == 896 || v == 1024) ? v : PANEL_CTA;
  }();
  return c;
}
template <typename F>
static auto with_kernel(int nth, F&& f) {
  switch (nth) {
    case 512: return f(panel_kernel<float, 512>);
    case 640: return f(panel_kernel<float, 640>);
    case 704: return f(panel_kernel<float, 704>);
    case 896: return f(panel_kernel<float, 896>);
    case 1024: return f(panel_kernel<float, 1024>);
    default: return f(panel_kernel<float, 768>);
  }
}

int panel_attr(int64_t R, int64_t W, int* regs) {
  return with_kernel(panel_cta(), [&](auto kern) -> int {
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, kern);
    if (e != cudaSuccess) return (int)e;
    *regs = fa.numRegs;
    int optin = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    const size_t need = panel_smem_bytes(R, W);
    if (need + fa.sharedSizeBytes > (size_t)optin) return (int)cudaErrorInvalidConfiguration;
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, optin - (int)fa.sharedSizeBytes);
    if (e != cudaSuccess) return (int)e;
    // two CTAs per SM when the windows allow it: the whole unified carve-out as shared memory
    return (int)cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  });
}

int launch_panel(const PanelArgs& a, int dtype, void* stream) {
  if (dtype != 0) return (int)cudaErrorNotSupported;
  if (a.npanels == 0) return 0;
  // programmatic dependent launch (a.pdl): the CTAs may start while the far kernel's last
  // wave runs — that kernel lets dependents launch only after each of its CTAs has waited
  // for its own predecessors, so x is final; its results are read after this grid waits
  const int nth = panel_cta();
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)a.npanels);
  cfg.blockDim = dim3(nth);
  cfg.dynamicSmemBytes = panel_smem_bytes(a.R, a.W);
  cfg.stream = (cudaStream_t)stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = a.pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return with_kernel(nth, [&](auto kern) -> int { return (int)cudaLaunchKernelEx(&cfg, kern, a); });
}

}  // namespace yaspmv
