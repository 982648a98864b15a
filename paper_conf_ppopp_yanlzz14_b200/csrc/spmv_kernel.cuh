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

// x gathers: read-only path, L2 evict-last (x is reused by every row)
__device__ __forceinline__ float ldx(const float* p, uint64_t pol) {
  float v;
  asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ double ldx(const double* p, uint64_t pol) {
  double v;
  asm("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ void ldx2(const float* p, uint64_t pol, float* v) {
  asm("ld.global.nc.L2::cache_hint.v2.f32 {%0,%1}, [%2], %3;" : "=f"(v[0]), "=f"(v[1]) : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ldx4(const float* p, uint64_t pol, float* v) {
  asm("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
      : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3])
      : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ldx2(const double* p, uint64_t pol, double* v) {
  asm("ld.global.nc.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;" : "=d"(v[0]), "=d"(v[1]) : "l"(p), "l"(pol));
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

// T bit flags of the thread tile starting at block blk0 (canonical LSB-first stream)
template <int T>
__device__ __forceinline__ uint32_t load_flags(const uint8_t* f, int64_t blk0) {
  if constexpr (T == 32) return __ldg(reinterpret_cast<const unsigned int*>(f + (blk0 >> 3)));
  else if constexpr (T == 16) return __ldg(reinterpret_cast<const unsigned short*>(f + (blk0 >> 3)));
  else if constexpr (T == 8) return __ldg(f + (blk0 >> 3));
  else return (__ldg(f + (blk0 >> 3)) >> (blk0 & 4)) & 0xFu;
}

template <typename VT>
__device__ __forceinline__ VT word_val(const uint32_t* w, int i) {
  if constexpr (sizeof(VT) == 4) return __uint_as_float(w[i]);
  else return __hiloint2double((int)w[2 * i + 1], (int)w[2 * i]);
}

template <typename VT, int W>
__device__ __forceinline__ void gather_x(const VT* x, int64_t cb, int64_t n, uint64_t pol, VT (&xs)[W]) {
  if constexpr (W == 1) {
    xs[0] = ldx(x + cb, pol);
  } else {
    const int64_t i0 = cb * W;
    if (i0 + W <= n) {
      if constexpr (W == 2) ldx2(x + i0, pol, xs);
      else ldx4(x + i0, pol, xs);
    } else {  // last block column of a matrix whose width is not a multiple of w (Q4)
#pragma unroll
      for (int c = 0; c < W; ++c) xs[c] = (i0 + c < n) ? ldx(x + i0 + c, pol) : VT(0);
    }
  }
}

// ---- mbarrier + TMA bulk copy (sm_90+ / sm_100a) ----------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// 1-D bulk copy global -> shared, completion counted on an mbarrier, L2 evict-first
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::
          "r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ void lds16(const void* p, uint32_t* w) {
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]) : "r"(smem_u32(p)));
}
__device__ __forceinline__ void lds8(const void* p, uint32_t* w) {
  asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(w[0]), "=r"(w[1]) : "r"(smem_u32(p)));
}
__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ double ld_relaxed_f64(const double* p) {
  double v;
  asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void consumer_bar(int nthreads) {
  asm volatile("bar.sync 1, %0;" ::"r"(nthreads) : "memory");
}

// per-thread run of PTB bytes of a tile held in shared memory in the device layout
template <int PTB>
__device__ __forceinline__ void lds_run(const unsigned char* base, int C, int t, uint32_t (&w)[PTB / 4]) {
  constexpr int CH = PTB < 16 ? PTB : 16;
  constexpr int NCH = PTB / CH;
#pragma unroll
  for (int j = 0; j < NCH; ++j) {
    const unsigned char* a = base + ((int)j * C + t) * CH;
    if constexpr (CH == 16) lds16(a, &w[4 * j]);
    else lds8(a, &w[2 * j]);
  }
}

template <int T>
__device__ __forceinline__ uint32_t lds_flags(const unsigned char* f, int t) {
  if constexpr (T == 32) return *reinterpret_cast<const uint32_t*>(f + 4 * t);
  else if constexpr (T == 16) return *reinterpret_cast<const uint16_t*>(f + 2 * t);
  else if constexpr (T == 8) return f[t];
  else return (f[t >> 1] >> ((t & 1) * 4)) & 0xFu;
}

}  // namespace dev

template <typename VT, int H, int W, int T, int CM>
struct KTraits {
  static constexpr int VB = T * W * (int)sizeof(VT);      // value bytes per thread per array
  static constexpr int CB = T * (CM == COL_I32 ? 4 : 2);  // column bytes per thread
  static constexpr int MAXC = (VB * H > 256) ? 256 : 512;  // consumer threads
  static constexpr int SLOT = T + 1;                       // result-cache slots per thread (odd stride)
  static constexpr int NST_MAX = 4;
  static constexpr int QK = 32;                            // carry fix-up queue entries
  __host__ __device__ static size_t stage_bytes(int C) { return (size_t)C * (H * VB + CB) + (size_t)C * T / 8; }
  __host__ __device__ static size_t cache_bytes(int C) { return (size_t)C * SLOT * H * sizeof(VT); }
  // stages: as many as fit two CTAs per SM (~110 KB each), between 2 and NST_MAX
  __host__ __device__ static int stages(int C) {
    const size_t per = stage_bytes(C);
    const size_t cb = cache_bytes(C);
    const size_t budget = cb < 110 * 1024 ? 110 * 1024 - cb : 0;
    const int n = (int)(budget / per);
    return n < 2 ? 2 : (n > NST_MAX ? NST_MAX : n);
  }
  __host__ __device__ static size_t smem_bytes(int C) { return stages(C) * stage_bytes(C) + cache_bytes(C); }
};

// Persistent and warp-specialised.  Threads [0, C) consume tiles; warp C/32 is the
// producer (one lane takes tile tickets and streams each tile's arrays into a shared-
// memory stage with TMA bulk copies tracked by mbarriers); warp C/32+1 is the carry
// fix-up warp that completes, off the consumers' critical path, the one segment per tile
// that continues from earlier tiles (decoupled look-back over the published carries).
template <typename VT, int H, int W, int T, int CM>
__global__ void __launch_bounds__(KTraits<VT, H, W, T, CM>::MAXC + 64)
    spmv_bccoo_kernel(const KArgs a) {
  using TR = KTraits<VT, H, W, T, CM>;
  constexpr int VB = TR::VB, CB = TR::CB, SLOT = TR::SLOT, QK = TR::QK;
  constexpr uint32_t TMASK = (T == 32) ? 0xffffffffu : ((1u << T) - 1u);
  extern __shared__ __align__(128) unsigned char smem_raw[];
  __shared__ __align__(8) uint64_t full_bar[TR::NST_MAX];
  __shared__ __align__(8) uint64_t empty_bar[TR::NST_MAX];
  __shared__ long long s_tile[TR::NST_MAX];
  __shared__ unsigned long long s_epoch[TR::NST_MAX];
  __shared__ VT s_wv[2][16][H];
  __shared__ int s_wf[2][16];
  __shared__ int s_wn[2][16];
  // fix-up queue: pending first segments of tiles that need the carry from earlier tiles
  __shared__ long long q_tile[QK];  // -1 = end of work
  __shared__ long long q_row[QK];
  __shared__ VT q_val[QK][H];
  __shared__ unsigned long long q_epoch;
  __shared__ volatile int q_seq[QK];
  __shared__ volatile int q_consumed;

  const int C = blockDim.x - 64;  // consumer threads
  const int NWC = C >> 5;
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5;
  const int NST = TR::stages(C);
  const size_t SB = TR::stage_bytes(C);
  unsigned char* stage0 = smem_raw;
  VT* cache = reinterpret_cast<VT*>(smem_raw + NST * SB);  // per-thread segment sums

  if (t == 0) {
    for (int s = 0; s < NST; ++s) {
      dev::mbar_init(&full_bar[s], 1);
      dev::mbar_init(&empty_bar[s], NWC);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (t < QK) q_seq[t] = 0;
  if (t == 0) q_consumed = 0;
  __syncthreads();

  // ================================================================ producer warp
  if (wid == NWC) {
    if (lane == 0) {
      const uint64_t pol = dev::policy_evict_first();
      const size_t vbytes = (size_t)C * VB, cbytes = (size_t)C * CB, fbytes = (size_t)C * T / 8;
      int s = 0;
      uint32_t phase = 0;
      for (;;) {
        dev::mbar_wait(&empty_bar[s], phase ^ 1u);
        const unsigned long long tk = atomicAdd(a.ticket, 1ull);  // logical workgroup id
        const unsigned long long q = tk / (unsigned long long)a.period;
        const long long tile = (long long)(tk - q * (unsigned long long)a.period);
        unsigned char* st = stage0 + s * SB;
        s_epoch[s] = q + 1ull;
        if (tile >= a.ntiles) {
          s_tile[s] = -1;
          dev::mbar_arrive(&full_bar[s]);
          break;
        }
        s_tile[s] = tile;
        dev::mbar_arrive_expect_tx(&full_bar[s], (uint32_t)SB);
#pragma unroll
        for (int r = 0; r < H; ++r)
          dev::bulk_g2s(st + r * vbytes, static_cast<const unsigned char*>(a.val[r]) + tile * vbytes,
                        (uint32_t)vbytes, &full_bar[s], pol);
        dev::bulk_g2s(st + H * vbytes, static_cast<const unsigned char*>(a.col) + tile * cbytes, (uint32_t)cbytes,
                      &full_bar[s], pol);
        dev::bulk_g2s(st + H * vbytes + cbytes, a.flags + tile * fbytes, (uint32_t)fbytes, &full_bar[s], pol);
        if (++s == NST) { s = 0; phase ^= 1u; }
      }
    }
    return;
  }

  VT* out = static_cast<VT*>(a.out);

  // ================================================================ carry fix-up warp
  if (wid == NWC + 1) {
    int head = 0;
    bool done = false;
    while (!done) {
      const int e = head + lane;
      const bool ready = q_seq[e % QK] == e + 1;
      const unsigned rm = __ballot_sync(0xffffffffu, ready);
      const int n = __ffs(~rm) - 1 < 0 ? 32 : __ffs(~rm) - 1;  // leading ready entries
      if (n == 0) {
        __nanosleep(64);
        continue;
      }
      __threadfence_block();
      long long tile = -2, row = 0;
      VT dv[H];
      if (lane < n) {
        tile = q_tile[e % QK];
        row = q_row[e % QK];
#pragma unroll
        for (int r = 0; r < H; ++r) dv[r] = q_val[e % QK][r];
      }
      const unsigned long long epoch = q_epoch;
      done = __any_sync(0xffffffffu, lane < n && tile == -1);
      __syncwarp();
      if (lane == 0) q_consumed = head + n;  // slots may be refilled
      if (tile >= 0) {
        // look back from tile-1 to the nearest tile holding a row stop (adjacent
        // synchronization); relaxed polling of the epoch-tagged status words
        // (no L1 invalidation); each value is read from L2 only after its tag is seen
        double carry[H];
#pragma unroll
        for (int r = 0; r < H; ++r) carry[r] = 0.0;
        for (long long idx = tile - 1; idx >= 0; --idx) {
          unsigned long long sv;
          do { sv = dev::ld_relaxed(a.status + idx); } while ((sv >> 2) != epoch);
#pragma unroll
          for (int r = 0; r < H; ++r) carry[r] += dev::ld_relaxed_f64(a.carry + idx * H + r);
          if ((sv & 3ull) == 2ull) break;  // inclusive prefix reached
        }
#pragma unroll
        for (int r = 0; r < H; ++r)
          if (row * H + r < a.out_limit) out[row * H + r] = (VT)((double)dv[r] + carry[r]);
      }
      head += n;
    }
    return;
  }

  // ================================================================ consumers
  const uint64_t pol_x = dev::policy_evict_last();
  const VT* x = static_cast<const VT*>(a.x);
  VT* my = cache + (size_t)t * SLOT * H;
  int s = 0;
  uint32_t phase = 0;
  int npush = 0;  // fix-up entries pushed (uniform over the consumers)
  for (int it = 0;; ++it) {
    dev::mbar_wait(&full_bar[s], phase);
    const int64_t tile = s_tile[s];
    const unsigned long long epoch = s_epoch[s];
    if (tile < 0) {
      if (t == 0) {  // end marker for the fix-up warp
        while (q_consumed <= npush - QK) {}
        q_tile[npush % QK] = -1;
        q_epoch = epoch;
        __threadfence_block();
        q_seq[npush % QK] = npush + 1;
      }
      break;
    }
    // ---- step 1: the thread tile from the stage (offline-transposed layout)
    const unsigned char* st = stage0 + s * SB;
    uint32_t vw[H][VB / 4];
#pragma unroll
    for (int r = 0; r < H; ++r) dev::lds_run<VB>(st + r * (size_t)C * VB, C, t, vw[r]);
    uint32_t cw[CB / 4];
    dev::lds_run<CB>(st + (size_t)H * C * VB, C, t, cw);
    const uint32_t fl = dev::lds_flags<T>(st + (size_t)H * C * VB + (size_t)C * CB, t);
    __syncwarp();
    if (lane == 0) dev::mbar_arrive(&empty_bar[s]);  // the stage may be refilled
    if (++s == NST) { s = 0; phase ^= 1u; }

    const int64_t blk0 = tile * (int64_t)C * T + (int64_t)t * T;
    // zero-fill of stacked rows that hold no block (empty_mode MAP, Q1)
    if (a.n_zero > 0) {
      const int64_t per = (a.n_zero + a.ntiles - 1) / a.ntiles;
      const int64_t z0 = tile * per, z1 = min(a.n_zero, z0 + per);
      for (int64_t z = z0 + t; z < z1; z += C) {
        const int64_t sr = a.zero_rows[z];
#pragma unroll
        for (int r = 0; r < H; ++r)
          if (sr * H + r < a.out_limit) out[sr * H + r] = VT(0);
      }
    }
    // row stops: '0' bits; one popc gives their count
    const uint32_t stops = ~fl & TMASK;
    const int nst = __popc(stops);
    const int hs = nst > 0;

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
    VT xs[T][W];
#pragma unroll
    for (int b = 0; b < T; ++b) dev::gather_x<VT, W>(x, colb[b], a.n, pol_x, xs[b]);

    // ---- step 2a: multiply + per-thread sequential segmented sum ----
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
        acc[r] += p;
        if (stop) {
          my[b * H + r] = acc[r];  // segment closed inside the thread tile
          acc[r] = VT(0);
        }
      }
    }

    // ---- step 2b: CTA segmented scan of (has_stop, last partial sum) -
    const int pb = it & 1;
    int f = hs, nn = nst;
    VT v[H];
#pragma unroll
    for (int r = 0; r < H; ++r) v[r] = acc[r];
    const unsigned hs_ballot = __ballot_sync(0xffffffffu, hs);
    // lanes 1..31 all hold a stop: every in-warp segment has size 1 -> skip
    const bool warp_all_stop = (hs_ballot | 1u) == 0xffffffffu;
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
      s_wf[pb][wid] = f;
      s_wn[pb][wid] = nn;
#pragma unroll
      for (int r = 0; r < H; ++r) s_wv[pb][wid][r] = v[r];
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
    dev::consumer_bar(C);
    int Fw = 0, Nw = 0, Fall = 0;
    VT Vw[H];
#pragma unroll
    for (int r = 0; r < H; ++r) Vw[r] = VT(0);
    for (int q = 0; q < NWC; ++q) {
      const int fq = s_wf[pb][q];
      if (q < wid) {  // prefix over earlier warps, folded left to right (deterministic)
#pragma unroll
        for (int r = 0; r < H; ++r) Vw[r] = fq ? s_wv[pb][q][r] : Vw[r] + s_wv[pb][q][r];
        Fw |= fq;
        Nw += s_wn[pb][q];
      }
      Fall |= fq;
    }
    const int Fex = Fw | fx;
    const int Nex = Nw + nx;
    VT Vex[H];
#pragma unroll
    for (int r = 0; r < H; ++r) Vex[r] = fx ? vx[r] : Vw[r] + vx[r];

    // ---- step 3a: publish this tile's carry-out (adjacent sync) ---------
    if (t == C - 1) {
      double* cv = a.carry + tile * H;
#pragma unroll
      for (int r = 0; r < H; ++r) __stcg(cv + r, (double)(hs ? acc[r] : Vex[r] + acc[r]));
      // state 2 = inclusive prefix known (tile holds a stop), 1 = aggregate only
      dev::st_release(a.status + tile, (epoch << 2) | (Fall ? 2ull : 1ull));
    }

    // ---- step 2c/3b: combine and write back ---------------------------
    const bool has_dep = Fall && tile > 0;          // uniform: this tile pushes one fix-up
    const bool dependent = hs && !Fex && tile > 0;  // the thread holding the tile's first stop
    const int64_t seg0 = (int64_t)__ldg(a.cta_seg0 + tile) + Nex;  // first-result entry
    {
      uint32_t sm = stops;
      int j = 0;
      while (sm) {
        const int b = __ffs(sm) - 1;
        sm &= sm - 1;
        const int64_t seg = seg0 + j;
        const int64_t sr = a.seg_row ? (int64_t)__ldg(a.seg_row + seg) : seg;
        VT o[H];
#pragma unroll
        for (int r = 0; r < H; ++r) o[r] = my[b * H + r];
        if (j == 0) {
#pragma unroll
          for (int r = 0; r < H; ++r) o[r] = Vex[r] + o[r];
        }
        if (j == 0 && dependent) {  // hand the segment to the fix-up warp
          while (q_consumed <= npush - QK) {}
          const int qi = npush % QK;
          q_tile[qi] = tile;
          q_row[qi] = sr;
#pragma unroll
          for (int r = 0; r < H; ++r) q_val[qi][r] = o[r];
          q_epoch = epoch;
          __threadfence_block();
          q_seq[qi] = npush + 1;
        } else {
#pragma unroll
          for (int r = 0; r < H; ++r)
            if (sr * H + r < a.out_limit) out[sr * H + r] = o[r];
        }
        ++j;
      }
    }
    npush += has_dep ? 1 : 0;
  }
}

template <typename VT, int H, int W, int T, int CM>
void launch_spmv(const KArgs& a, int C, int64_t grid, void* stream) {
  using TR = KTraits<VT, H, W, T, CM>;
  spmv_bccoo_kernel<VT, H, W, T, CM><<<(unsigned)grid, C + 64, TR::smem_bytes(C), (cudaStream_t)stream>>>(a);
}

template <typename VT, int H, int W, int T, int CM>
int attr_spmv(int C, int* regs, int* max_threads, int* blocks_per_sm) {
  using TR = KTraits<VT, H, W, T, CM>;
  auto k = spmv_bccoo_kernel<VT, H, W, T, CM>;
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, k);
  if (e != cudaSuccess) return (int)e;
  *regs = fa.numRegs;
  *max_threads = fa.maxThreadsPerBlock - 64;
  *blocks_per_sm = 0;
  if (C > 0 && C <= *max_threads) {
    int optin = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    const size_t need = TR::smem_bytes(C) + fa.sharedSizeBytes;
    if (need > (size_t)optin) return 0;  // does not fit: blocks_per_sm stays 0
    e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)TR::smem_bytes(C));
    if (e != cudaSuccess) return (int)e;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k, C + 32, TR::smem_bytes(C));
    if (e != cudaSuccess) return (int)e;
  }
  return 0;
}

template <typename VT, int H, int W, int T>
void reg_t(std::vector<KernelEntry>& R) {
  if constexpr (T * H * W * (int)sizeof(VT) <= 512) {
    const int dt = sizeof(VT) == 4 ? 0 : 1;
    R.push_back({dt, H, W, T, COL_U16, &launch_spmv<VT, H, W, T, COL_U16>, &attr_spmv<VT, H, W, T, COL_U16>});
    R.push_back({dt, H, W, T, COL_I32, &launch_spmv<VT, H, W, T, COL_I32>, &attr_spmv<VT, H, W, T, COL_I32>});
    R.push_back({dt, H, W, T, COL_DELTA, &launch_spmv<VT, H, W, T, COL_DELTA>, &attr_spmv<VT, H, W, T, COL_DELTA>});
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
}

}  // namespace yaspmv
