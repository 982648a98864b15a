// spmv_kernel.cuh — the fused BCCOO / BCCOO+ SpMV kernel for sm_100a.
//
// One CTA per workgroup-level tile of T*C consecutive non-zero blocks, one thread per
// thread-level tile of T blocks (§3.2.1, Fig. 8).  The three logical
// steps of P:226 run in ONE kernel:
//   (1) stream the tile (values, column indices, bit flags) with 128-bit coalesced loads
//       from the offline-transposed device layout, L2 evict-first; gather x
//       through the read-only path with L2 evict-last (the texture path of P:302/P:322);
//       multiply;
//   (2) per-thread sequential segmented sum driven by the bit flags (P:262, P:267:
//       "strategy 1" with intermediate sums in registers, ShM_size = 0 as the tuner pins,
//       P:322); CTA-level segmented scan of the per-thread last partial sums with start
//       flag = "tile holds a row stop" as warp shuffles + one shared-memory
//       pass, skipped per warp when every thread has a stop;
//   (3) carries across workgroups: the paper's adjacent synchronization
//       rendered as decoupled look-back — a tile WITH a row stop publishes its last partial
//       sum at once (the paper's "directly updates Grp_sum[X]"), a tile without one
//       publishes its aggregate; the tile whose first row stop needs the carry folds the
//       predecessors' published values back to the nearest tile with a stop.  Logical
//       tile ids come from an atomic ticket, so waiting is only ever on CTAs that
//       started earlier.  Status words carry an epoch (no per-call memset, no sentinel
//       value, Q9); carries are fp64 (Q12).  Write-back of y (or of the BCCOO+ partial
//       result) happens in the same kernel.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "common.hpp"

namespace yaspmv {
namespace dev {

__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}

// streaming loads of the matrix arrays: read-only, no L1 allocation, L2 evict-first
__device__ __forceinline__ void ld_stream16(const void* p, uint64_t pol, uint32_t* w) {
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
      : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3])
      : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ld_stream8(const void* p, uint64_t pol, uint32_t* w) {
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.u32 {%0,%1}, [%2], %3;"
      : "=r"(w[0]), "=r"(w[1])
      : "l"(p), "l"(pol));
}

// x gathers: read-only path, evict-last in L1 and L2 (x is reused by every row, P:32;
// measured on C5: L1 evict-last 4.49 ms, default 4.60, L1 no-allocate / .cg 4.83)
#define YASPMV_XLD "ld.global.nc.L1::evict_last.L2::cache_hint.f32"

__device__ __forceinline__ float ldx(const float* p, uint64_t pol) {
  float v;
  asm(YASPMV_XLD " %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ double ldx(const double* p, uint64_t pol) {
  double v;
  asm("ld.global.nc.L1::evict_last.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void ldx2(const float* p, uint64_t pol, float* v) {
  asm("ld.global.nc.L1::evict_last.L2::cache_hint.v2.f32 {%0,%1}, [%2], %3;" : "=f"(v[0]), "=f"(v[1]) : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ldx4(const float* p, uint64_t pol, float* v) {
  asm("ld.global.nc.L1::evict_last.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
      : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3])
      : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ldx2(const double* p, uint64_t pol, double* v) {
  asm("ld.global.nc.L1::evict_last.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;" : "=d"(v[0]), "=d"(v[1]) : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ldx4(const double* p, uint64_t pol, double* v) {
  ldx2(p, pol, v);
  ldx2(p + 2, pol, v + 2);
}

__device__ __forceinline__ unsigned long long ld_acquire(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// per-thread run of PTB bytes of a tile in the device layout -> PTB/4 words
template <int PTB>
__device__ __forceinline__ void load_run(const void* base, int64_t tile, int C, int t, uint64_t pol,
                                         uint32_t (&w)[PTB / 4]) {
  constexpr int CH = PTB < 16 ? PTB : 16;
  constexpr int NCH = PTB / CH;
  const char* b = static_cast<const char*>(base) + tile * (int64_t)C * PTB;
#pragma unroll
  for (int j = 0; j < NCH; ++j) {
    const char* a = b + ((int64_t)j * C + t) * CH;
    if constexpr (CH == 16) ld_stream16(a, pol, &w[4 * j]);
    else ld_stream8(a, pol, &w[2 * j]);
  }
}

// T bit flags of the thread tile starting at block blk0 (canonical LSB-first stream),
// streamed like the other matrix arrays (no L1 allocation: L1 is kept for x)
__device__ __forceinline__ uint32_t ld_stream_u32(const void* p) {
  uint32_t v;
  asm("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint32_t ld_stream_u16(const void* p) {
  unsigned short v;
  asm("ld.global.nc.L1::no_allocate.u16 %0, [%1];" : "=h"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ uint32_t ld_stream_u8(const void* p) {
  unsigned short v;
  asm("ld.global.nc.L1::no_allocate.u8 %0, [%1];" : "=h"(v) : "l"(p));
  return v & 0xFFu;
}
template <int T>
__device__ __forceinline__ uint32_t load_flags(const uint8_t* f, int64_t blk0) {
  if constexpr (T == 32) return ld_stream_u32(f + (blk0 >> 3));
  else if constexpr (T == 16) return ld_stream_u16(f + (blk0 >> 3));
  else if constexpr (T == 8) return ld_stream_u8(f + (blk0 >> 3));
  else return (ld_stream_u8(f + (blk0 >> 3)) >> (blk0 & 4)) & 0xFu;
}

template <typename VT>
__device__ __forceinline__ VT word_val(const uint32_t* w, int i) {
  if constexpr (sizeof(VT) == 4) return __uint_as_float(w[i]);
  else return __hiloint2double((int)w[2 * i + 1], (int)w[2 * i]);
}

template <typename VT, int W>
__device__ __forceinline__ void gather_x(const VT* x, int64_t cb, int64_t n, uint64_t pol, VT (&xs)[W]) {
  if constexpr (W == 1) {
    // predicated: a FILLER block sits in block column NB (Q3) and reads 0, never x
    xs[0] = cb < n ? ldx(x + cb, pol) : VT(0);
  } else {
    const int64_t i0 = cb * W;
    if (i0 + W <= n) {
      if constexpr (W == 2) ldx2(x + i0, pol, xs);
      else if constexpr (W == 4) ldx4(x + i0, pol, xs);
      else {
        ldx4(x + i0, pol, xs);
        ldx4(x + i0 + 4, pol, xs + 4);
      }
    } else {  // last block column of a matrix whose width is not a multiple of w (Q4)
#pragma unroll
      for (int c = 0; c < W; ++c) xs[c] = (i0 + c < n) ? ldx(x + i0 + c, pol) : VT(0);
    }
  }
}

__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long atom_exch_acq_rel(unsigned long long* p, unsigned long long v) {
  unsigned long long o;
  asm volatile("atom.acq_rel.gpu.global.exch.b64 %0, [%1], %2;" : "=l"(o) : "l"(p), "l"(v) : "memory");
  return o;
}
// 16-byte status / hand-off words: single 128-bit accesses (LDG/STG.E.128, ATOMG.EXCH.128),
// so a status word and the value published with it are observed together
__device__ __forceinline__ void ld_relaxed_16(const unsigned long long* p, unsigned long long& lo,
                                              unsigned long long& hi) {
  asm volatile("ld.relaxed.gpu.global.v2.b64 {%0, %1}, [%2];" : "=l"(lo), "=l"(hi) : "l"(p) : "memory");
}
__device__ __forceinline__ void st_relaxed_16(unsigned long long* p, unsigned long long lo, unsigned long long hi) {
  asm volatile("st.relaxed.gpu.global.v2.b64 [%0], {%1, %2};" ::"l"(p), "l"(lo), "l"(hi) : "memory");
}
__device__ __forceinline__ void atom_exch_16(unsigned long long* p, unsigned long long lo, unsigned long long hi,
                                             unsigned long long& olo, unsigned long long& ohi) {
  asm volatile(
      "{ .reg .b128 d, s; mov.b128 s, {%2, %3}; atom.relaxed.gpu.global.exch.b128 d, [%4], s; "
      "mov.b128 {%0, %1}, d; }"
      : "=l"(olo), "=l"(ohi)
      : "l"(lo), "l"(hi), "l"(p)
      : "memory");
}
__device__ __forceinline__ double ld_relaxed_f64(const double* p) {
  double v;
  asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
  return v;
}
}  // namespace dev

// the launch epoch of this CTA (block-id mode): set by thread 0 at its first tile's scan
__device__ __forceinline__ unsigned long long& cta_epoch_slot() {
  __shared__ unsigned long long e;
  return e;
}

// Output store.  In a fused exchange (EPI == 2 instances) the element goes to
// every rank's copy of the next x over peer memory (NVLink P2P stores through IPC
// mappings; the rank's own buffer is one of them), so the all-gather overlaps the SpMV.
template <typename VT, int EPI>
__device__ __forceinline__ void store_out(const KArgs& a, VT* out, int64_t i, VT v) {
  if constexpr (EPI == 2) {
    if (a.peer_mc) {  // NVSwitch multicast: one store, every rank's copy
      multimem_store(static_cast<VT*>(a.peer_out[0]) + i, v);
      return;
    }
#pragma unroll
    for (int q = 0; q < YASPMV_MAX_RANKS; ++q)
      if (q < a.npeer) static_cast<VT*>(a.peer_out[q])[i] = v;
  } else {
    out[i] = v;
  }
}

template <typename VT, int H, int W, int T, int CM>
struct KTraits {
  static constexpr int VB = T * W * (int)sizeof(VT);      // value bytes per thread per array
  static constexpr int CB = T * (CM == COL_I32 ? 4 : 2);  // column bytes per thread
  static constexpr int MAXC = (VB * H > 256) ? 256 : 512;
  // register cap: 96 for the fp32 scalar-row instances (32 values + 32 x in registers) so
  // that the C5-class kernel keeps 5 CTAs of 128 threads per SM (104 registers would
  // allow 4: allocation is per warp in units of 8 per thread); otherwise what C <= MAXC
  // needs (the former __launch_bounds__(MAXC, 1))
  static constexpr int MAXREG = (sizeof(VT) == 4 && H == 1 && T * W <= 32) ? 96 : (MAXC == 512 ? 128 : 255);
  __host__ __device__ static size_t smem_bytes(int) { return 0; }  // L1 keeps the whole carve-out
};

template <typename VT, int H>
struct ScanShared {
  long long tile;
  unsigned long long epoch;
  double inv;  // power-iteration epilogue scale 1/sqrt(*in_norm2), computed once per CTA
  VT wv[16][H];
  int wf[16];
  int wn[16];
};

// Carry-in of tile k's first segment (adjacent synchronization, as a decoupled
// look-back): the fold of the published tails of tiles k-1, k-2, ... back to the nearest
// tile holding a row stop (state 2), 32 predecessors per window, fixed association (Q10).
// Warp-collective; waits only on predecessors nearer than that stop.  Polled with relaxed
// loads (an acquire would invalidate L1 and with it the cached x); a carry value is read
// only after its tile's epoch-tagged status word was seen (written before the release).
// Forward progress rests on in-order dispatch or on ticket ids; a debug bound
// (KArgs::spin_limit, YASPMV_SPIN_LIMIT) turns a hang into a trap naming the tile.
template <int H>
__device__ __forceinline__ void lookback(const KArgs& a, int64_t k, unsigned long long epoch, int lane,
                                         double (&carry)[H]) {
#pragma unroll
  for (int r = 0; r < H; ++r) carry[r] = 0.0;
  int64_t jw = k - 1;
  long long spins = 0;
  while (true) {
    const int64_t idx = jw - lane;
    int state = idx >= 0 ? 0 : 2;  // before tile 0: an inclusive prefix of 0
    unsigned long long vbits = 0;  // h = 1: the carry-out, read with its status word
    unsigned p2, lim;
    while (true) {
      if (state == 0) {
        unsigned long long sv;
        if constexpr (H == 1) dev::ld_relaxed_16(a.status + 2 * idx, sv, vbits);
        else sv = dev::ld_relaxed(a.status + 2 * idx);
        if ((sv >> 2) == epoch) state = (int)(sv & 3ull);
      }
      p2 = __ballot_sync(0xffffffffu, state == 2);
      const unsigned p0 = __ballot_sync(0xffffffffu, state == 0);
      const unsigned nearer = p2 ? ((p2 & (0u - p2)) - 1u) : 0xffffffffu;
      if ((p0 & nearer) == 0) {
        lim = p2 ? __ffs(p2) - 1 : 31;  // nearest tile with a row stop
        break;
      }
      if (a.spin_limit > 0 && ++spins > a.spin_limit) {  // debug bound: report the tile, trap
        if (lane == 0) *(volatile long long*)a.spin_tile = (long long)k;
        __threadfence_system();
        __trap();
      }
    }
    // h > 1: the carries are separate words written before a release of the status word;
    // an acquire-release fence orders this warp's carry reads after the status reads
    if constexpr (H > 1) asm volatile("fence.acq_rel.gpu;" ::: "memory");
#pragma unroll
    for (int r = 0; r < H; ++r) {
      double cv = 0.0;
      if (lane <= (int)lim && idx >= 0) {
        if constexpr (H == 1) cv = __longlong_as_double((long long)vbits);
        else cv = dev::ld_relaxed_f64(a.carry + idx * H + r);
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) cv += __shfl_xor_sync(0xffffffffu, cv, o);  // fixed tree
      carry[r] += __shfl_sync(0xffffffffu, cv, 0);
    }
    if (p2) break;
    jw -= 32;
  }
}

// y of tile k's carried first segment = (partial + carry-in) scaled; its y^2 partial slot
template <typename VT, int H, int EPI>
__device__ __forceinline__ void write_carried(const KArgs& a, VT* out, int64_t k, int64_t row, const double (&dep)[H],
                                              const double (&carry)[H], double inv, int NW) {
  double ds = 0.0;
#pragma unroll
  for (int r = 0; r < H; ++r)
    if (row * H + r < a.out_limit) {
      const VT o = (VT)((dep[r] + carry[r]) * inv);
      store_out<VT, EPI>(a, out, row * H + r, o);
      ds += (double)o * (double)o;
    }
  if ((EPI == 1 || EPI == 2) && (a.epi & 2)) a.part[k * (NW + 1) + NW] = ds;
}

// hand-off word tags (bnd[k], per launch epoch): tile k left its carried segment pending /
// tile k-1 has published its carry-out
__device__ __forceinline__ unsigned long long bnd_tag(unsigned long long epoch, unsigned who) {
  return ((epoch & 0x3FFFFFFFull) << 2) | who;  // low 32 bits; h = 1 packs the row above
}
constexpr unsigned BND_PENDING = 1, BND_DONE = 2;

// Step 3a of a tile (thread C-1): publish the tile's carry-out — its status word with the
// inclusive value when the tile holds a row stop (the paper's "directly updates"),
// else its aggregate — and take over the successor's carried segment if the successor
// already left it behind (non-blocking hand-off, see resolve_carries).
template <typename VT, int H, int EPI>
__device__ __forceinline__ void publish_carry(const KArgs& a, const int64_t tile, const unsigned long long epoch,
                                              const int Fall, const int hs, const VT (&acc)[H], const VT (&Vex)[H],
                                              bool& succ_pending, unsigned long long& succ_lo,
                                              unsigned long long& succ_hi) {
  // state 2 = inclusive prefix known (tile holds a stop), 1 = aggregate only
  const unsigned long long sw = (epoch << 2) | (Fall ? 2ull : 1ull);
  if constexpr (H == 1) {
    const double cv0 = (double)(hs ? acc[0] : Vex[0] + acc[0]);
    dev::st_relaxed_16(a.status + 2 * tile, sw, (unsigned long long)__double_as_longlong(cv0));
    if constexpr (EPI == 3) __stcg(a.carry + tile, cv0);  // the ablation's carry kernel
  } else {
    double* cv = a.carry + tile * H;
#pragma unroll
    for (int r = 0; r < H; ++r) __stcg(cv + r, (double)(hs ? acc[r] : Vex[r] + acc[r]));
    dev::st_release(a.status + 2 * tile, sw);
  }
  if (!(EPI == 3 && (a.ablate & ABL_DEFER_CARRY)) && tile + 1 < a.ntiles) {
    if constexpr (H == 1) {
      dev::atom_exch_16(a.bnd + 2 * (tile + 1), bnd_tag(epoch, BND_DONE), 0ull, succ_lo, succ_hi);
      succ_pending = (succ_lo & 0xFFFFFFFFull) == bnd_tag(epoch, BND_PENDING);
    } else {
      succ_pending = (dev::atom_exch_acq_rel(a.bnd + 2 * (tile + 1), bnd_tag(epoch, BND_DONE)) & 0xFFFFFFFFull) ==
                     bnd_tag(epoch, BND_PENDING);
    }
  }
}

// Step 3c of a tile: the carry-in of its first row stop (decoupled look-back) and the
// successor's carried segment if it was handed to this tile.
template <typename VT, int H, int EPI>
__device__ __forceinline__ void resolve_carries(const KArgs& a, VT* out, const int64_t tile,
                                                const unsigned long long epoch, const int lane, const int wid,
                                                const int NW, const bool dependent, const VT (&dep)[H],
                                                const int64_t dep_row, const double inv, const bool succ_pending,
                                                const unsigned long long succ_lo, const unsigned long long succ_hi) {
  // The warp holding the tile's first row stop needs the carry-in.  Non-blocking hand-off:
  // if the predecessor has not published yet, leave the partial and its row behind and
  // exchange the tile's hand-off word; whichever of the two tiles arrives second
  // completes the segment (the other returns at once), so a tile never holds its SM
  // slot waiting for a slower predecessor in the common case.  Same arithmetic either
  // way: (fp64 partial + look-back fold) * inv, rounded once.
  const unsigned dep_ballot = __ballot_sync(0xffffffffu, dependent);
  if (dep_ballot) {
    const int dep_lane = __ffs(dep_ballot) - 1;
    unsigned long long sv = 0;
    if (lane == 0) sv = dev::ld_relaxed(a.status + 2 * (tile - 1));
    sv = __shfl_sync(0xffffffffu, sv, 0);
    bool mine = true;
    const bool can_pack = H > 1 || a.out_limit < (1ll << 32);  // h = 1 packs the row in 32 bits
    if (((sv >> 2) != epoch || a.force_handoff) && can_pack) {  // predecessor still running: hand off
      unsigned long long old = 0;
      if (lane == dep_lane) {
        if constexpr (H == 1) {
          unsigned long long ohi;
          dev::atom_exch_16(a.bnd + 2 * tile, ((unsigned long long)dep_row << 32) | bnd_tag(epoch, BND_PENDING),
                            (unsigned long long)__double_as_longlong((double)dep[0]), old, ohi);
        } else {
#pragma unroll
          for (int r = 0; r < H; ++r) a.pend_val[tile * H + r] = (double)dep[r];
          a.pend_row[tile] = dep_row;
          old = dev::atom_exch_acq_rel(a.bnd + 2 * tile, bnd_tag(epoch, BND_PENDING));
        }
      }
      old = __shfl_sync(0xffffffffu, old, dep_lane);
      mine = (old & 0xFFFFFFFFull) == bnd_tag(epoch, BND_DONE);  // it published meanwhile: finish here
    }
    if (mine) {
      double carry[H];
      lookback<H>(a, tile, epoch, lane, carry);
      if (lane == dep_lane) {
        double d[H];
#pragma unroll
        for (int r = 0; r < H; ++r) d[r] = (double)dep[r];
        write_carried<VT, H, EPI>(a, out, tile, dep_row, d, carry, inv, NW);
      }
    }
  }
  // the next tile handed its carried segment to this one (its predecessor)
  if (wid == NW - 1 && __shfl_sync(0xffffffffu, succ_pending ? 1 : 0, 31)) {
    double carry[H];
    lookback<H>(a, tile + 1, epoch, lane, carry);
    if (lane == 31) {
      double d[H];
      int64_t row;
      if constexpr (H == 1) {  // carried in the exchanged word
        d[0] = __longlong_as_double((long long)succ_hi);
        row = (int64_t)(succ_lo >> 32);
      } else {  // lane 31's acquire (the exchange) made tile+1's pending data visible
#pragma unroll
        for (int r = 0; r < H; ++r) d[r] = a.pend_val[(tile + 1) * H + r];
        row = (int64_t)a.pend_row[tile + 1];
      }
      write_carried<VT, H, EPI>(a, out, tile + 1, row, d, carry, inv, NW);
    }
  }
}

// Step 1 of a tile: stream the thread tile — bit flags,
// block columns, values (128-bit loads of the offline-transposed layout, L2 evict-first)
// and the tile's first-result entry — then, after the programmatic-dependent-launch wait,
// take the epoch ticket, zero-fill empty stacked rows (Q1) and issue all T gathers of x.
template <typename VT, int H, int W, int T, int CM, int EPI>
__device__ __forceinline__ void stream_tile(const KArgs& a, const int64_t tile, ScanShared<VT, H>& sh, const int t,
                                            const int C, uint32_t& fl,
                                            uint32_t (&vw)[H][KTraits<VT, H, W, T, CM>::VB / 4], VT (&xs)[T][W],
                                            int& cta_seg0, unsigned long long& tk) {
  using TR = KTraits<VT, H, W, T, CM>;
  constexpr int VB = TR::VB, CB = TR::CB;
  const uint64_t pol_s = dev::policy_evict_first();
  const uint64_t pol_x = dev::policy_evict_last();
  // ---- step 1: stream the thread tile (128-bit loads, offline-transposed layout) ----
  const int64_t blk0 = tile * (int64_t)C * T + (int64_t)t * T;
  fl = dev::load_flags<T>(a.flags, blk0);
  uint32_t cw[CB / 4];
  dev::load_run<CB>(a.col, tile, C, t, pol_s, cw);
#pragma unroll
  for (int r = 0; r < H; ++r) dev::load_run<VB>(a.val[r], tile, C, t, pol_s, vw[r]);
  // the tile's first-result entry: matrix data too, so issued with the stream
  // instead of after the scan, where its latency would sit on the critical path
  cta_seg0 = __ldg(a.cta_seg0 + tile);

  VT* out = static_cast<VT*>(a.out);
  // Programmatic dependent launch: everything above reads only the encoded matrix (never
  // written by other kernels) and overlaps the previous kernel's tail; x, y, the status
  // words and the ticket may depend on earlier kernels in the stream.
  if (a.block_ids) {
    // the next kernel may launch once every CTA is past this wait: whatever it reads that
    // an earlier kernel wrote (x) is then final (the panel kernel reads x before it waits
    // for this grid's own results)
    if (a.pdl) {
      cudaGridDependencySynchronize();
      cudaTriggerProgrammaticLaunchCompletion();
    }
    if (t == 0) {
      // one ticket per CTA, advanced by the CTA's tile count (a launch still adds ntiles): the
      // launch epoch, consumed only at the scan barrier; later tiles of the CTA reuse it
      const int64_t c0 = (int64_t)blockIdx.x * max(a.tpc, 1);
      if (tile == c0) tk = atomicAdd(a.ticket, (unsigned long long)(min(a.ntiles, c0 + max(a.tpc, 1)) - c0));
      if constexpr (EPI == 1 || EPI == 2) sh.inv = (a.epi & 1) ? 1.0 / sqrt(a.in_norm2[0]) : 1.0;
    }
  }
  // zero-fill of stacked rows that hold no block (empty_mode MAP, Q1)
  if (a.n_zero > 0) {
    const int64_t per = (a.n_zero + a.ntiles - 1) / a.ntiles;
    const int64_t z0 = tile * per, z1 = min(a.n_zero, z0 + per);
    for (int64_t z = z0 + t; z < z1; z += C) {
      const int64_t sr = a.zero_rows[z];
#pragma unroll
      for (int r = 0; r < H; ++r)
        if (sr * H + r < a.out_limit) store_out<VT, EPI>(a, out, sr * H + r, VT(0));
    }
  }
  // block columns, then all T gathers of x in flight
  int colb[T];
#pragma unroll
  for (int b = 0; b < T; ++b) {
    if constexpr (CM == COL_I32) {
      colb[b] = (int)cw[b];
    } else {
      const uint32_t hw = (cw[b >> 1] >> (16 * (b & 1))) & 0xFFFFu;
      if constexpr (CM == COL_U16) colb[b] = (int)hw;
      else {  // segmented int16 difference, -1 = escape to the int32 array
        const int d = (int)(int16_t)hw;
        const int base = (b == 0) ? 0 : colb[b - 1];
        colb[b] = (d == -1) ? __ldg(a.col32 + blk0 + b) : base + d;
      }
    }
  }
  const VT* x = static_cast<const VT*>(a.x);
#pragma unroll
  for (int b = 0; b < T; ++b)
    dev::gather_x<VT, W>(x,
                         (EPI == 3 && (a.ablate & (ABL_STREAM_ONLY | ABL_GATHER_L2)))
                             ? (colb[b] & ((a.ablate & ABL_STREAM_ONLY) ? 15 : 0xFFFFF))
                             : colb[b],
                         a.n, pol_x, xs[b]);
}

// The work of one workgroup-level tile (T*C consecutive blocks): steps 1-3
// of P:226 plus the cross-tile carry.
template <typename VT, int H, int W, int T, int CM, int EPI>
__device__ __forceinline__ void tile_body(const KArgs& a, const int64_t tile, ScanShared<VT, H>& sh) {
  using TR = KTraits<VT, H, W, T, CM>;
  constexpr int VB = TR::VB;
  constexpr uint32_t TMASK = (T == 32) ? 0xffffffffu : ((1u << T) - 1u);
  auto& s_wv = sh.wv;
  auto& s_wf = sh.wf;
  auto& s_wn = sh.wn;
  const int t = threadIdx.x, C = blockDim.x, lane = t & 31, wid = t >> 5, NW = C >> 5;
  // ---- step 1: stream the thread tile, gather x ------------------------------------
  uint32_t fl;
  uint32_t vw[H][VB / 4];
  VT xs[T][W];
  int cta_seg0;
  unsigned long long tk = 0;
  stream_tile<VT, H, W, T, CM, EPI>(a, tile, sh, t, C, fl, vw, xs, cta_seg0, tk);
  VT* out = static_cast<VT*>(a.out);
  // warp-staged y stores (KArgs::wstage): this warp's slice of the dynamic shared memory
  extern __shared__ __align__(16) unsigned char s1_stage[];
  // (not in the T = 32 peer-store instance: its registers would spill)
  VT* const wbuf = (H == 1 && (EPI == 0 || EPI == 1 || (EPI == 2 && T <= 16)) && a.wstage && a.seg_row == nullptr)
                       ? reinterpret_cast<VT*>(s1_stage) + wid * 32 * T
                       : nullptr;
  const bool STG = wbuf != nullptr;
  // row stops: '0' bits; one popc gives their count
  const uint32_t stops = ~fl & TMASK;
  const int nst = __popc(stops);
  const int hs = nst > 0;

  // ---- step 2a: multiply + per-thread sequential segmented sum ------
  // Strategy 1: the per-block products stay in registers ("intermediate_sums",
  // Reg_size = T, ShM_size = 0 as the tuner pins); the running sum after the last
  // stop is the thread's last partial sum.
  VT pr[T][H];
  VT acc[H];
#pragma unroll
  for (int r = 0; r < H; ++r) acc[r] = VT(0);
#pragma unroll
  for (int b = 0; b < T; ++b) {
    const bool stop = (stops >> b) & 1u;
#pragma unroll
    for (int r = 0; r < H; ++r) {
      VT p = dev::word_val<VT>(vw[r], b * W) * xs[b][0];
#pragma unroll
      for (int c = 1; c < W; ++c) p = fma(dev::word_val<VT>(vw[r], b * W + c), xs[b][c], p);
      pr[b][r] = p;
      acc[r] = stop ? VT(0) : acc[r] + p;
    }
  }

  if (EPI == 3 && (a.ablate & (ABL_GATHER_ONLY | ABL_STREAM_ONLY))) {  // roofline probes: loads only
    VT s = VT(0);
#pragma unroll
    for (int b = 0; b < T; ++b)
#pragma unroll
      for (int r = 0; r < H; ++r) s += pr[b][r];
    if (s == VT(-1.25e-30) || fl == 0x9e3779b9u) out[t] = s;  // keeps every load live
    return;
  }

  // ---- step 2b: CTA segmented scan of (has_stop, last partial sum) --
  int f = hs, nn = nst;
  VT v[H];
#pragma unroll
  for (int r = 0; r < H; ++r) v[r] = acc[r];
  const unsigned hs_ballot = __ballot_sync(0xffffffffu, hs);
  // lanes 1..31 all hold a stop: every in-warp segment has size 1 -> skip
  const bool warp_all_stop = (hs_ballot | 1u) == 0xffffffffu && !(EPI == 3 && (a.ablate & ABL_NO_SKIP));
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int f2 = __shfl_up_sync(0xffffffffu, f, d);
    const int n2 = __shfl_up_sync(0xffffffffu, nn, d);
    if (!warp_all_stop) {
#pragma unroll
      for (int r = 0; r < H; ++r) {
        const VT v2 = __shfl_up_sync(0xffffffffu, v[r], d);
        if (lane >= d && !f) v[r] = v2 + v[r];
      }
    }
    if (lane >= d) { f |= f2; nn += n2; }
  }
  if (lane == 31) {
    s_wf[wid] = f;
    s_wn[wid] = nn;
#pragma unroll
    for (int r = 0; r < H; ++r) s_wv[wid][r] = v[r];
  }
  int fx = __shfl_up_sync(0xffffffffu, f, 1);
  int nx = __shfl_up_sync(0xffffffffu, nn, 1);
  VT vx[H];
#pragma unroll
  for (int r = 0; r < H; ++r) vx[r] = __shfl_up_sync(0xffffffffu, v[r], 1);
  if (lane == 0) {
    fx = 0;
    nx = 0;
#pragma unroll
    for (int r = 0; r < H; ++r) vx[r] = VT(0);
  }
  // block-id mode (in-order dispatch): the ticket only yields the launch epoch,
  // needed from here on, so its atomic latency hides behind the tile's loads
  if (a.block_ids && t == 0) {  // the CTA's first tile took the ticket (stream_tile)
    if (tile == (int64_t)blockIdx.x * max(a.tpc, 1)) cta_epoch_slot() = tk / (unsigned long long)a.period + 1ull;
    sh.epoch = cta_epoch_slot();
  }
  __syncthreads();
  const unsigned long long epoch = sh.epoch;
  int Fw = 0, Nw = 0, Fall = 0;
  VT Vw[H];
#pragma unroll
  for (int r = 0; r < H; ++r) Vw[r] = VT(0);
  for (int q = 0; q < NW; ++q) {
    const int fq = s_wf[q];
    if (q < wid) {  // prefix over earlier warps, folded left to right (deterministic)
#pragma unroll
      for (int r = 0; r < H; ++r) Vw[r] = fq ? s_wv[q][r] : Vw[r] + s_wv[q][r];
      Fw |= fq;
      Nw += s_wn[q];
    }
    Fall |= fq;
  }
  const int Fex = Fw | fx;
  const int Nex = Nw + nx;
  VT Vex[H];
#pragma unroll
  for (int r = 0; r < H; ++r) Vex[r] = fx ? vx[r] : Vw[r] + vx[r];
  if (EPI == 3 && (a.ablate & ABL_STOP_SCAN)) {  // roofline probe: everything up to the scan
    if (a.ablate & ABL_PROBE_PUB) {
      if (t == C - 1)
        dev::st_relaxed_16(a.status + 2 * tile, (epoch << 2) | (Fall ? 2ull : 1ull),
                           (unsigned long long)__double_as_longlong((double)Vex[0]));
    } else if (a.ablate & ABL_PROBE_ST) {
      out[(tile * C + t) % a.out_limit] = Vex[0] + VT(Nex);
    } else if (Vex[0] == VT(-1.25e-30) || Nex == -7) {
      out[t] = Vex[0];
    }
    return;
  }

  // ---- step 3a: publish this tile's carry-out (adjacent sync) -----------
  bool succ_pending = false;
  unsigned long long succ_lo = 0, succ_hi = 0;
  if (t == C - 1 && !(EPI == 3 && (a.ablate & ABL_NO_PUBLISH0) && tile == 0))
    publish_carry<VT, H, EPI>(a, tile, epoch, Fall, hs, acc, Vex, succ_pending, succ_lo, succ_hi);

  // ---- step 2c/3b: combine and write back -----------------------------
  const bool dependent = hs && !Fex && tile > 0;  // the tile's first stop needs the carry
  const int64_t seg0 = (int64_t)cta_seg0 + Nex;  // first-result entry
  // optional power-iteration epilogue: y scaled by 1/sqrt(in_norm2), sum y^2 partials
  const double inv = (EPI == 1 || EPI == 2) ? sh.inv : 1.0;
  const VT invv = (VT)inv;
  VT ssv = VT(0);
  VT dep[H];
  int64_t dep_row = 0;
  if (hs) {
    // Strategy 1 combine: walk the intermediate sums; the first stop adds the
    // scanned last partial sums of earlier threads (Vex), later stops are complete.  The
    // tile's very first segment (dependent) is handed to the look-back below.
    VT run[H];
#pragma unroll
    for (int r = 0; r < H; ++r) run[r] = Vex[r];
    bool first = dependent;
    if constexpr (H == 1 && (EPI == 0 || EPI == 1 || (EPI == 2 && T <= 16))) {
      if (STG) {  // warp-staged stores: the j-th stop of the thread goes to slot nx + j
        VT rr = run[0];
        int j = nx;
#pragma unroll
        for (int b = 0; b < T; ++b) {
          rr = rr + pr[b][0];
          if ((stops >> b) & 1u) {
            if (first) {
              dep[0] = rr;
              dep_row = seg0;
            } else {
              const VT o = (EPI == 1 || EPI == 2) ? rr * invv : rr;
              wbuf[j] = o;
              if constexpr (EPI == 1 || EPI == 2) ssv = fma(o, o, ssv);
            }
            first = false;
            ++j;
            rr = VT(0);
          }
        }
      }
    }
    if (STG) {
      // done above (H = 1, EPI 0/1 only: STG is false otherwise)
    } else if (a.seg_row == nullptr) {  // segment k is stacked row k: rows are consecutive
      int64_t row = seg0;
#pragma unroll
      for (int b = 0; b < T; ++b) {
#pragma unroll
        for (int r = 0; r < H; ++r) run[r] = run[r] + pr[b][r];
        if ((stops >> b) & 1u) {
          if (first) {
#pragma unroll
            for (int r = 0; r < H; ++r) dep[r] = run[r];
            dep_row = row;
          } else {
#pragma unroll
            for (int r = 0; r < H; ++r)
              if (H == 1 || row * H + r < a.out_limit) {
                const VT o = (EPI == 1 || EPI == 2) ? run[r] * invv : run[r];
                if (EPI == 3 && (a.ablate & ABL_NO_YSTORE)) {  // probe: the cost of the y stores
                  if (o == VT(-1.25e-30)) out[row * H + r] = o;
                } else {
                  store_out<VT, EPI>(a, out, row * H + r, o);
                }
                if constexpr (EPI == 1 || EPI == 2) ssv = fma(o, o, ssv);
              }
          }
          first = false;
          ++row;
#pragma unroll
          for (int r = 0; r < H; ++r) run[r] = VT(0);
        }
      }
    } else {  // seg_row map (empty_mode MAP, Q1)
      int64_t seg = seg0;
#pragma unroll
      for (int b = 0; b < T; ++b) {
#pragma unroll
        for (int r = 0; r < H; ++r) run[r] = run[r] + pr[b][r];
        if ((stops >> b) & 1u) {
          const int64_t sr = (int64_t)__ldg(a.seg_row + seg);
          if (first) {
#pragma unroll
            for (int r = 0; r < H; ++r) dep[r] = run[r];
            dep_row = sr;
          } else {
#pragma unroll
            for (int r = 0; r < H; ++r)
              if (sr * H + r < a.out_limit) {
                const VT o = (EPI == 1 || EPI == 2) ? run[r] * invv : run[r];
                store_out<VT, EPI>(a, out, sr * H + r, o);
                if constexpr (EPI == 1 || EPI == 2) ssv = fma(o, o, ssv);
              }
          }
          first = false;
          ++seg;
#pragma unroll
          for (int r = 0; r < H; ++r) run[r] = VT(0);
        }
      }
    }
  }
  if (STG) {  // the warp's rows [cta_seg0 + Nw, + its stop count) as one contiguous run
    __syncwarp();
    const int wcnt = __shfl_sync(0xffffffffu, nn, 31);
    const int skip = __ballot_sync(0xffffffffu, dependent) != 0u;  // slot 0: the carried segment
    const int64_t wrow0 = (int64_t)cta_seg0 + Nw;
    if (EPI != 2 && a.wstage == 2) {  // streaming stores (the slice results are read by a later kernel)
      for (int i = lane + skip; i < wcnt; i += 32) __stcs(out + wrow0 + i, wbuf[i]);
    } else {
      for (int i = lane + skip; i < wcnt; i += 32) store_out<VT, EPI>(a, out, wrow0 + i, wbuf[i]);
    }
    __syncwarp();
  }
  double ss = (double)ssv;

  // ---- step 3c: look back for the carry-in (decoupled look-back) --------
  // by the warp holding the tile's first row stop; a window of 32 predecessors per
  // round, polled with relaxed loads (no L1 invalidation: x stays cached in L1)
  if ((EPI == 1 || EPI == 2) && (a.epi & 2)) {  // per-warp partial of sum y^2, fixed tree (deterministic)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
    if (lane == 0) a.part[tile * (NW + 1) + wid] = ss;
    if (t == 0 && !(Fall && tile > 0)) a.part[tile * (NW + 1) + NW] = 0.0;  // no carried segment
  }
  if (EPI == 3 && (a.ablate & ABL_DEFER_CARRY)) {  // ablation: carries by a second kernel
    // (dep_row == NULL: the "no carries" probe — the carried segments stay incomplete)
    if (a.dep_row && t == 0 && !(Fall && tile > 0)) a.dep_row[tile] = -1;
    if (dependent) {
#pragma unroll
      for (int r = 0; r < H; ++r)
        if (dep_row * H + r < a.out_limit) out[dep_row * H + r] = dep[r];
      if (a.dep_row) a.dep_row[tile] = dep_row;
    }
    return;
  }
  resolve_carries<VT, H, EPI>(a, out, tile, epoch, lane, wid, NW, dependent, dep, dep_row, inv, succ_pending,
                              succ_lo, succ_hi);
}

// Strategy 2 (Fig. 10/12): no per-thread intermediate sums array.  The
// first-result entries — stops before each thread in the tile, derived in-kernel
// by a count scan instead of stored per thread — place every segment sum in a
// per-workgroup result cache of RC = k*C entries in shared memory (k = result cache size,
// Table 1); the thread walks its tile once, writing each completed segment straight
// to its cache slot and keeping only the sum up to its first stop and its last partial
// sum.  After the CTA scan the first stop's entry receives the scanned last partial sums
// of the earlier threads, and the whole cache is written to y in a coalesced way.
// Entries at or beyond RC ("more row stops than the result cache size") are complete
// sums and go straight to y (the paper parks them in a global result array for a later
// pass; on B200 the final value is already known).  The tile's first segment still
// travels the cross-tile carry path of strategy 1 (thread 0's entry 0).
template <typename VT, int H, int W, int T, int CM, int EPI>
__device__ __forceinline__ void tile_body_s2(const KArgs& a, const int64_t tile, ScanShared<VT, H>& sh, VT* rcache) {
  using TR = KTraits<VT, H, W, T, CM>;
  constexpr int VB = TR::VB;
  constexpr uint32_t TMASK = (T == 32) ? 0xffffffffu : ((1u << T) - 1u);
  const int t = threadIdx.x, C = blockDim.x, lane = t & 31, wid = t >> 5, NW = C >> 5;
  const int RC = a.rcache;
  uint32_t fl;
  uint32_t vw[H][VB / 4];
  VT xs[T][W];
  int cta_seg0;
  unsigned long long tk = 0;
  stream_tile<VT, H, W, T, CM, EPI>(a, tile, sh, t, C, fl, vw, xs, cta_seg0, tk);
  VT* out = static_cast<VT*>(a.out);
  const uint32_t stops = ~fl & TMASK;
  const int nst = __popc(stops);
  const int hs = nst > 0;

  // first-result entries: inclusive count scan in the warp, warp totals through smem
  int nin = nst;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int n2 = __shfl_up_sync(0xffffffffu, nin, d);
    if (lane >= d) nin += n2;
  }
  if (lane == 31) sh.wn[wid] = nin;
  __syncthreads();
  int Nw = 0, Ntot = 0;
  for (int q = 0; q < NW; ++q) {
    const int c = sh.wn[q];
    if (q < wid) Nw += c;
    Ntot += c;
  }
  const int fre = Nw + nin - nst;  // this thread's first stop, relative to the tile's first
  const double inv = (EPI == 1 || EPI == 2) ? sh.inv : 1.0;
  const VT invv = (VT)inv;
  VT ssv = VT(0);
  // a segment sum that is final: to its cache slot, or past the cache straight to y
  auto emit = [&](const int e, const VT (&v)[H]) {
    if (e < RC) {
#pragma unroll
      for (int r = 0; r < H; ++r) rcache[e * H + r] = v[r];
    } else {
      const int64_t row = a.seg_row ? (int64_t)__ldg(a.seg_row + cta_seg0 + e) : (int64_t)cta_seg0 + e;
#pragma unroll
      for (int r = 0; r < H; ++r)
        if (row * H + r < a.out_limit) {
          const VT o = (EPI == 1 || EPI == 2) ? v[r] * invv : v[r];
          store_out<VT, EPI>(a, out, row * H + r, o);
          if constexpr (EPI == 1 || EPI == 2) ssv = fma(o, o, ssv);
        }
    }
  };

  // ---- multiply + sequential segmented sum straight into the result cache ----------
  VT run[H], head[H];
#pragma unroll
  for (int r = 0; r < H; ++r) run[r] = head[r] = VT(0);
  int j = 0;
#pragma unroll
  for (int b = 0; b < T; ++b) {
#pragma unroll
    for (int r = 0; r < H; ++r) {
      VT p = dev::word_val<VT>(vw[r], b * W) * xs[b][0];
#pragma unroll
      for (int c = 1; c < W; ++c) p = fma(dev::word_val<VT>(vw[r], b * W + c), xs[b][c], p);
      run[r] = run[r] + p;
    }
    if ((stops >> b) & 1u) {
      if (j == 0) {
#pragma unroll
        for (int r = 0; r < H; ++r) head[r] = run[r];
      } else {
        emit(fre + j, run);
      }
      ++j;
#pragma unroll
      for (int r = 0; r < H; ++r) run[r] = VT(0);
    }
  }

  // ---- CTA segmented scan of (has_stop, last partial sum) ----------
  int f = hs;
  VT v[H];
#pragma unroll
  for (int r = 0; r < H; ++r) v[r] = run[r];
  const unsigned hs_ballot = __ballot_sync(0xffffffffu, hs);
  const bool warp_all_stop = (hs_ballot | 1u) == 0xffffffffu;  // skip
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int f2 = __shfl_up_sync(0xffffffffu, f, d);
    if (!warp_all_stop) {
#pragma unroll
      for (int r = 0; r < H; ++r) {
        const VT v2 = __shfl_up_sync(0xffffffffu, v[r], d);
        if (lane >= d && !f) v[r] = v2 + v[r];
      }
    }
    if (lane >= d) f |= f2;
  }
  if (lane == 31) {
    sh.wf[wid] = f;
#pragma unroll
    for (int r = 0; r < H; ++r) sh.wv[wid][r] = v[r];
  }
  int fx = __shfl_up_sync(0xffffffffu, f, 1);
  VT vx[H];
#pragma unroll
  for (int r = 0; r < H; ++r) vx[r] = __shfl_up_sync(0xffffffffu, v[r], 1);
  if (lane == 0) {
    fx = 0;
#pragma unroll
    for (int r = 0; r < H; ++r) vx[r] = VT(0);
  }
  if (a.block_ids && t == 0) {  // the CTA's first tile took the ticket (stream_tile)
    if (tile == (int64_t)blockIdx.x * max(a.tpc, 1)) cta_epoch_slot() = tk / (unsigned long long)a.period + 1ull;
    sh.epoch = cta_epoch_slot();
  }
  __syncthreads();
  const unsigned long long epoch = sh.epoch;
  int Fw = 0, Fall = 0;
  VT Vw[H];
#pragma unroll
  for (int r = 0; r < H; ++r) Vw[r] = VT(0);
  for (int q = 0; q < NW; ++q) {
    const int fq = sh.wf[q];
    if (q < wid) {
#pragma unroll
      for (int r = 0; r < H; ++r) Vw[r] = fq ? sh.wv[q][r] : Vw[r] + sh.wv[q][r];
      Fw |= fq;
    }
    Fall |= fq;
  }
  const int Fex = Fw | fx;
  VT Vex[H];
#pragma unroll
  for (int r = 0; r < H; ++r) Vex[r] = fx ? vx[r] : Vw[r] + vx[r];

  bool succ_pending = false;
  unsigned long long succ_lo = 0, succ_hi = 0;
  if (t == C - 1) publish_carry<VT, H, EPI>(a, tile, epoch, Fall, hs, run, Vex, succ_pending, succ_lo, succ_hi);

  // ---- the first stop's entry gets the earlier threads' scanned partial sums --
  const bool dependent = hs && !Fex && tile > 0;  // the tile's first segment: carry path
  VT dep[H];
  int64_t dep_row = 0;
  if (hs) {
#pragma unroll
    for (int r = 0; r < H; ++r) dep[r] = head[r] + Vex[r];
    if (dependent) dep_row = a.seg_row ? (int64_t)__ldg(a.seg_row + cta_seg0 + fre) : (int64_t)cta_seg0 + fre;
    else emit(fre, dep);
  }
  __syncthreads();
  // ---- coalesced write-back of the result cache (entry 0 of tiles > 0 is carried) ----
  const int lim = min(Ntot, RC);
  for (int e = (tile > 0 ? 1 : 0) + t; e < lim; e += C) {
    const int64_t row = a.seg_row ? (int64_t)__ldg(a.seg_row + cta_seg0 + e) : (int64_t)cta_seg0 + e;
#pragma unroll
    for (int r = 0; r < H; ++r)
      if (row * H + r < a.out_limit) {
        const VT o = (EPI == 1 || EPI == 2) ? rcache[e * H + r] * invv : rcache[e * H + r];
        store_out<VT, EPI>(a, out, row * H + r, o);
        if constexpr (EPI == 1 || EPI == 2) ssv = fma(o, o, ssv);
      }
  }
  if ((EPI == 1 || EPI == 2) && (a.epi & 2)) {  // per-warp partial of sum y^2, fixed tree (deterministic)
    double ss = (double)ssv;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
    if (lane == 0) a.part[tile * (NW + 1) + wid] = ss;
    if (t == 0 && !(Fall && tile > 0)) a.part[tile * (NW + 1) + NW] = 0.0;  // no carried segment
  }
  resolve_carries<VT, H, EPI>(a, out, tile, epoch, lane, wid, NW, dependent, dep, dep_row, inv, succ_pending,
                              succ_lo, succ_hi);
}

// One CTA per workgroup-level tile; logical tile ids from an atomic ticket.
template <typename VT, int H, int W, int T, int CM, int EPI>
__global__ void __maxnreg__((KTraits<VT, H, W, T, CM>::MAXREG)) spmv_bccoo_kernel(const KArgs a) {
  __shared__ ScanShared<VT, H> shb[2];
  ScanShared<VT, H>& sh = shb[0];
  if (a.block_ids) {  // tile = workgroup id: workgroups dispatch in order — the default
    if (a.tpc <= 1) {
      tile_body<VT, H, W, T, CM, EPI>(a, (int64_t)blockIdx.x, sh);
      return;
    }
    // tpc consecutive tiles per workgroup: a warp done with one tile issues the next
    // tile's loads at once (no barrier between tiles) while the tile's stores drain and its
    // look-back completes.  The scan state alternates between two buffers: the scan barrier
    // of tile k+1 is passed only when every warp has finished tile k, so tile k+2 can
    // reuse tile k's buffer.
    const int64_t t0 = (int64_t)blockIdx.x * a.tpc, t1 = min(a.ntiles, t0 + a.tpc);
    for (int64_t tile = t0; tile < t1; ++tile) tile_body<VT, H, W, T, CM, EPI>(a, tile, shb[tile & 1]);
    return;
  }
  if (a.pdl) {
    cudaGridDependencySynchronize();
    cudaTriggerProgrammaticLaunchCompletion();
  }
  if (threadIdx.x == 0) {  // logical workgroup id from an atomic ticket
    const unsigned long long tk = atomicAdd(a.ticket, 1ull);
    const unsigned long long q = tk / (unsigned long long)a.period;
    sh.tile = (long long)(tk - q * (unsigned long long)a.period);
    sh.epoch = q + 1ull;  // launches so far: tags this launch's status words (Q9)
    if constexpr (EPI == 1 || EPI == 2) sh.inv = (a.epi & 1) ? 1.0 / sqrt(a.in_norm2[0]) : 1.0;
  }
  __syncthreads();
  tile_body<VT, H, W, T, CM, EPI>(a, sh.tile, sh);
}

// Strategy-2 kernel (result cache in dynamic shared memory: KArgs::rcache entries of h values)
template <typename VT, int H, int W, int T, int CM, int EPI>
__global__ void __maxnreg__((KTraits<VT, H, W, T, CM>::MAXREG)) spmv_bccoo_s2_kernel(const KArgs a) {
  __shared__ ScanShared<VT, H> sh;
  extern __shared__ __align__(16) unsigned char s2_rcache[];
  VT* rcache = reinterpret_cast<VT*>(s2_rcache);
  if (a.block_ids) {
    // consecutive tiles without a barrier in between: each state (counts, scan values,
    // result cache) is written in tile k+1 only after a barrier that every warp reaches
    // after its last read of that state in tile k (count scan -> B1, walk -> B2, cache
    // write-back -> next tile's B1)
    const int64_t t0 = (int64_t)blockIdx.x * max(a.tpc, 1), t1 = min(a.ntiles, t0 + max(a.tpc, 1));
    for (int64_t tile = t0; tile < t1; ++tile) tile_body_s2<VT, H, W, T, CM, EPI>(a, tile, sh, rcache);
    return;
  }
  if (a.pdl) {
    cudaGridDependencySynchronize();
    cudaTriggerProgrammaticLaunchCompletion();
  }
  if (threadIdx.x == 0) {
    const unsigned long long tk = atomicAdd(a.ticket, 1ull);
    const unsigned long long q = tk / (unsigned long long)a.period;
    sh.tile = (long long)(tk - q * (unsigned long long)a.period);
    sh.epoch = q + 1ull;
    if constexpr (EPI == 1 || EPI == 2) sh.inv = (a.epi & 1) ? 1.0 / sqrt(a.in_norm2[0]) : 1.0;
  }
  __syncthreads();
  tile_body_s2<VT, H, W, T, CM, EPI>(a, sh.tile, sh, rcache);
}

template <typename VT, int H, int W, int T, int CM>
void launch_spmv(const KArgs& a, int C, int64_t grid, void* stream) {
  using TR = KTraits<VT, H, W, T, CM>;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(C);
  const size_t stage = a.wstage ? (size_t)C * T * H * sizeof(VT) : 0;
  cfg.dynamicSmemBytes = TR::smem_bytes(C) + stage;
  cfg.stream = (cudaStream_t)stream;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = a.pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  {  // staged stores need enough of the unified carve-out as shared memory for a full SM of
     // CTAs (the instances prefer L1 otherwise, which would cap the CTAs per SM): set as a
     // launch attribute and, for tools that replay kernels without it (ncu), as the function
     // attribute of the EPI 0/1 instances — changed only when a launch needs another split
    size_t pct = 0;
    if (stage) {
      const size_t need = (size_t)(2048 / C) * (stage + 2048);
      pct = (need * 100 + 228 * 1024 - 1) / (228 * 1024);
      if (pct > 100) pct = 100;
      attr[1].id = cudaLaunchAttributePreferredSharedMemoryCarveout;
      attr[1].val.sharedMemCarveout = (unsigned)pct;
      cfg.numAttrs = 2;
    }
    static int set_pct[3] = {0, 0, 0};  // per EPI 0/1/2 instance of this template; attr_spmv starts at 0
    const int e = a.npeer > 0 ? 2 : a.epi ? 1 : 0;
    if (!a.ablate && set_pct[e] != (int)pct) {
      if (e == 2) cudaFuncSetAttribute(spmv_bccoo_kernel<VT, H, W, T, CM, 2>, cudaFuncAttributePreferredSharedMemoryCarveout, (int)pct);
      else if (e) cudaFuncSetAttribute(spmv_bccoo_kernel<VT, H, W, T, CM, 1>, cudaFuncAttributePreferredSharedMemoryCarveout, (int)pct);
      else cudaFuncSetAttribute(spmv_bccoo_kernel<VT, H, W, T, CM, 0>, cudaFuncAttributePreferredSharedMemoryCarveout, (int)pct);
      set_pct[e] = (int)pct;
    }
  }
  // EPI: 0 plain SpMV, 1 power-iteration epilogue, 2 epilogue + peer stores (fused
  // exchange), 3 ablation / roofline probes (h = w = 1 only); separate instances so that
  // neither the peer loop nor the probes cost the production kernel registers
  if (a.ablate) {
    if constexpr (H == 1 && W == 1) cudaLaunchKernelEx(&cfg, spmv_bccoo_kernel<VT, H, W, T, CM, 3>, a);
  } else if (a.npeer > 0) cudaLaunchKernelEx(&cfg, spmv_bccoo_kernel<VT, H, W, T, CM, 2>, a);
  else if (a.epi) cudaLaunchKernelEx(&cfg, spmv_bccoo_kernel<VT, H, W, T, CM, 1>, a);
  else cudaLaunchKernelEx(&cfg, spmv_bccoo_kernel<VT, H, W, T, CM, 0>, a);
}

template <typename VT, int H, int W, int T, int CM>
int attr_spmv(int C, int /*rc*/, int* regs, int* max_threads, int* blocks_per_sm) {
  using TR = KTraits<VT, H, W, T, CM>;
  auto k = spmv_bccoo_kernel<VT, H, W, T, CM, 0>;
  auto k2 = spmv_bccoo_kernel<VT, H, W, T, CM, 1>;
  auto k3 = spmv_bccoo_kernel<VT, H, W, T, CM, 2>;
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, k);
  if (e != cudaSuccess) return (int)e;
  *regs = fa.numRegs;
  *max_threads = fa.maxThreadsPerBlock;
  *blocks_per_sm = 0;
  if (C > 0 && C <= *max_threads) {
    int optin = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    if (TR::smem_bytes(C) + fa.sharedSizeBytes > (size_t)optin) return 0;
    // the warp-staged y stores (KArgs::wstage) take up to 48 KB of dynamic shared memory on
    // the EPI 0/1 instances: a fixed per-instance cap, whichever handle selects it
    const int stage_cap = (int)(48 * 1024 - fa.sharedSizeBytes);
    e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, max((int)TR::smem_bytes(C), stage_cap));
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(k2, cudaFuncAttributeMaxDynamicSharedMemorySize, max((int)TR::smem_bytes(C), stage_cap));
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(k3, cudaFuncAttributeMaxDynamicSharedMemorySize, max((int)TR::smem_bytes(C), stage_cap));
    if (e != cudaSuccess) return (int)e;
    // x gathers are the L1 traffic: give L1 the whole unified carve-out
    e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, 0);
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(k2, cudaFuncAttributePreferredSharedMemoryCarveout, 0);
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(k3, cudaFuncAttributePreferredSharedMemoryCarveout, 0);
    if (e != cudaSuccess) return (int)e;
    if constexpr (H == 1 && W == 1) {
      e = cudaFuncSetAttribute(spmv_bccoo_kernel<VT, H, W, T, CM, 3>, cudaFuncAttributePreferredSharedMemoryCarveout,
                               0);
      if (e != cudaSuccess) return (int)e;
    }
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k, C, TR::smem_bytes(C));
    if (e != cudaSuccess) return (int)e;
  }
  return 0;
}

template <typename VT, int H, int W, int T, int CM>
void launch_spmv_s2(const KArgs& a, int C, int64_t grid, void* stream) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(C);
  cfg.dynamicSmemBytes = (size_t)a.rcache * H * sizeof(VT);
  cfg.stream = (cudaStream_t)stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = a.pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  if (a.npeer > 0) cudaLaunchKernelEx(&cfg, spmv_bccoo_s2_kernel<VT, H, W, T, CM, 2>, a);
  else if (a.epi) cudaLaunchKernelEx(&cfg, spmv_bccoo_s2_kernel<VT, H, W, T, CM, 1>, a);
  else cudaLaunchKernelEx(&cfg, spmv_bccoo_s2_kernel<VT, H, W, T, CM, 0>, a);
}

template <typename VT, int H, int W, int T, int CM>
int attr_spmv_s2(int C, int rc, int* regs, int* max_threads, int* blocks_per_sm) {
  auto k0 = spmv_bccoo_s2_kernel<VT, H, W, T, CM, 0>;
  auto k1 = spmv_bccoo_s2_kernel<VT, H, W, T, CM, 1>;
  auto k2 = spmv_bccoo_s2_kernel<VT, H, W, T, CM, 2>;
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, k0);
  if (e != cudaSuccess) return (int)e;
  *regs = fa.numRegs;
  *max_threads = fa.maxThreadsPerBlock;
  *blocks_per_sm = 0;
  if (C > 0 && C <= *max_threads) {
    const size_t dyn = (size_t)rc * C * H * sizeof(VT);
    int optin = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    if (dyn + fa.sharedSizeBytes > (size_t)optin) return 0;
    for (auto k : {k0, k1, k2}) {
      // the cap is a property of the kernel instance, shared by every handle using it: set
      // it to the opt-in limit once, never to this handle's size (a smaller later handle
      // would otherwise lower it under an earlier handle's launches)
      e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, optin - (int)fa.sharedSizeBytes);
      if (e != cudaSuccess) return (int)e;
      e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, 0);  // the rest stays L1
      if (e != cudaSuccess) return (int)e;
    }
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k0, C, dyn);
    if (e != cudaSuccess) return (int)e;
  }
  return 0;
}

template <typename VT, int H, int W, int T>
void reg_t(std::vector<KernelEntry>& R) {
  if constexpr (T * H * W * (int)sizeof(VT) <= 512) {
    const int dt = sizeof(VT) == 4 ? 0 : 1;
    R.push_back({dt, H, W, T, COL_U16, 1, &launch_spmv<VT, H, W, T, COL_U16>, &attr_spmv<VT, H, W, T, COL_U16>});
    R.push_back({dt, H, W, T, COL_I32, 1, &launch_spmv<VT, H, W, T, COL_I32>, &attr_spmv<VT, H, W, T, COL_I32>});
    R.push_back({dt, H, W, T, COL_DELTA, 1, &launch_spmv<VT, H, W, T, COL_DELTA>, &attr_spmv<VT, H, W, T, COL_DELTA>});
  }
}

template <typename VT, int H, int W>
void reg_w(std::vector<KernelEntry>& R) {
  reg_t<VT, H, W, 4>(R);
  reg_t<VT, H, W, 8>(R);
  reg_t<VT, H, W, 16>(R);
  reg_t<VT, H, W, 32>(R);
}

template <typename VT, int H>
void reg_h(std::vector<KernelEntry>& R) {
  reg_w<VT, H, 1>(R);
  reg_w<VT, H, 2>(R);
  reg_w<VT, H, 4>(R);
  reg_w<VT, H, 8>(R);
}

// strategy-2 instances (compiled in inst_s2_*.cu)
template <typename VT, int H, int W, int T>
void reg_t_s2(std::vector<KernelEntry>& R) {
  if constexpr (T * H * W * (int)sizeof(VT) <= 512) {
    const int dt = sizeof(VT) == 4 ? 0 : 1;
    R.push_back({dt, H, W, T, COL_U16, 2, &launch_spmv_s2<VT, H, W, T, COL_U16>, &attr_spmv_s2<VT, H, W, T, COL_U16>});
    R.push_back({dt, H, W, T, COL_I32, 2, &launch_spmv_s2<VT, H, W, T, COL_I32>, &attr_spmv_s2<VT, H, W, T, COL_I32>});
    R.push_back(
        {dt, H, W, T, COL_DELTA, 2, &launch_spmv_s2<VT, H, W, T, COL_DELTA>, &attr_spmv_s2<VT, H, W, T, COL_DELTA>});
  }
}

template <typename VT, int H, int W>
void reg_w_s2(std::vector<KernelEntry>& R) {
  reg_t_s2<VT, H, W, 4>(R);
  reg_t_s2<VT, H, W, 8>(R);
  reg_t_s2<VT, H, W, 16>(R);
  reg_t_s2<VT, H, W, 32>(R);
}

template <typename VT, int H>
void reg_h_s2(std::vector<KernelEntry>& R) {
  reg_w_s2<VT, H, 1>(R);
  reg_w_s2<VT, H, 2>(R);
  reg_w_s2<VT, H, 4>(R);
  reg_w_s2<VT, H, 8>(R);
}

}  // namespace yaspmv
