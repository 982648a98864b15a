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

}  // namespace dev

template <typename VT, int H, int W, int T, int CM>
struct KTraits {
  static constexpr int VB = T * W * (int)sizeof(VT);      // value bytes per thread per array
  static constexpr int CB = T * (CM == COL_I32 ? 4 : 2);  // column bytes per thread
  static constexpr int MAXC = (VB * H > 256) ? 256 : 512;
};

template <typename VT, int H, int W, int T, int CM>
__global__ void __launch_bounds__(KTraits<VT, H, W, T, CM>::MAXC)
    spmv_bccoo_kernel(const KArgs a) {
  using TR = KTraits<VT, H, W, T, CM>;
  constexpr int VB = TR::VB, CB = TR::CB;
  __shared__ unsigned long long s_ticket;
  __shared__ VT s_wv[16][H];
  __shared__ int s_wf[16];
  __shared__ int s_wn[16];
  __shared__ VT s_dep[H];
  __shared__ int64_t s_dep_row;

  const int t = threadIdx.x, C = blockDim.x, lane = t & 31, wid = t >> 5;
  if (t == 0) s_ticket = atomicAdd(a.ticket, 1ull);  // logical workgroup id
  __syncthreads();
  const unsigned long long tk = s_ticket;
  const int64_t tile = (int64_t)(tk % (unsigned long long)a.ntiles);
  const unsigned long long epoch = tk / (unsigned long long)a.ntiles + 1ull;
  const uint64_t pol_s = dev::policy_evict_first();
  const uint64_t pol_x = dev::policy_evict_last();

  // ---- step 1: stream the thread tile --------------------------------------------
  const int64_t blk0 = tile * (int64_t)C * T + (int64_t)t * T;
  const uint32_t fl = dev::load_flags<T>(a.flags, blk0);
  uint32_t cw[CB / 4];
  dev::load_run<CB>(a.col, tile, C, t, pol_s, cw);
  uint32_t vw[H][VB / 4];
#pragma unroll
  for (int r = 0; r < H; ++r) dev::load_run<VB>(a.val[r], tile, C, t, pol_s, vw[r]);

  // zero-fill of stacked rows that hold no block (empty_mode MAP, Q1)
  if (a.n_zero > 0) {
    const int64_t per = (a.n_zero + a.ntiles - 1) / a.ntiles;
    const int64_t z0 = tile * per, z1 = min(a.n_zero, z0 + per);
    VT* out = static_cast<VT*>(a.out);
    for (int64_t z = z0 + t; z < z1; z += C) {
      const int64_t sr = a.zero_rows[z];
#pragma unroll
      for (int r = 0; r < H; ++r)
        if (sr * H + r < a.out_limit) out[sr * H + r] = VT(0);
    }
  }

  // block columns
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

  // multiply: p[b][r] = sum_c val[r][b*w + c] * x[col_b*w + c]
  const VT* x = static_cast<const VT*>(a.x);
  VT p[T][H];
#pragma unroll
  for (int b = 0; b < T; ++b) {
    VT xs[W];
    dev::gather_x<VT, W>(x, colb[b], a.n, pol_x, xs);
#pragma unroll
    for (int r = 0; r < H; ++r) {
      VT s = dev::word_val<VT>(vw[r], b * W) * xs[0];
#pragma unroll
      for (int c = 1; c < W; ++c) s = fma(dev::word_val<VT>(vw[r], b * W + c), xs[c], s);
      p[b][r] = s;
    }
  }

  // ---- step 2a: per-thread sequential segmented sum ----------------
  VT tail[H];
#pragma unroll
  for (int r = 0; r < H; ++r) tail[r] = VT(0);
  int nst = 0;
#pragma unroll
  for (int b = 0; b < T; ++b) {
    const bool stop = !((fl >> b) & 1u);  // '0' = row stop
#pragma unroll
    for (int r = 0; r < H; ++r) tail[r] = stop ? VT(0) : tail[r] + p[b][r];
    nst += stop;
  }
  // tail = the thread's last partial sum: the running sum after its last row stop
  // (0 when the tile ends in a stop)
  const int hs = nst > 0;

  // ---- step 2b: CTA segmented scan of (has_stop, last partial sum) --
  int f = hs, nn = nst;
  VT v[H];
#pragma unroll
  for (int r = 0; r < H; ++r) v[r] = tail[r];
  const bool warp_all_stop = __all_sync(0xffffffffu, hs || t == 0);  // skip check
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
  // lane-exclusive values (inclusive of lane-1)
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
  __syncthreads();
  // prefix over earlier warps, folded left to right (deterministic)
  int Fw = 0, Nw = 0;
  VT Vw[H];
#pragma unroll
  for (int r = 0; r < H; ++r) Vw[r] = VT(0);
  for (int q = 0; q < wid; ++q) {
    const int fq = s_wf[q];
#pragma unroll
    for (int r = 0; r < H; ++r) Vw[r] = fq ? s_wv[q][r] : Vw[r] + s_wv[q][r];
    Fw |= fq;
    Nw += s_wn[q];
  }
  // exclusive prefix of this thread = (earlier warps) (+) (earlier lanes)
  const int Fex = Fw | fx;
  const int Nex = Nw + nx;
  VT Vex[H];
#pragma unroll
  for (int r = 0; r < H; ++r) Vex[r] = fx ? vx[r] : Vw[r] + vx[r];

  // ---- step 3a: publish this tile's carry-out (adjacent sync) -----------
  const int tile_has_stop = __syncthreads_or(hs);
  if (t == C - 1) {
    double* cv = a.carry + tile * H;
#pragma unroll
    for (int r = 0; r < H; ++r) {
      const VT incl = hs ? tail[r] : Vex[r] + tail[r];
      __stcg(cv + r, (double)incl);
    }
    // state 2 = inclusive prefix known (tile holds a stop), 1 = aggregate only
    dev::st_release(a.status + tile, (epoch << 2) | (tile_has_stop ? 2ull : 1ull));
  }

  // ---- step 2c/3b: combine and write back -----------------------------
  VT* out = static_cast<VT*>(a.out);
  const bool dependent_here = hs && !Fex && tile > 0;  // first stop of the tile needs the carry
  if (hs) {
    int64_t seg = (int64_t)__ldg(a.cta_seg0 + tile) + Nex;  // first-result entry
    VT acc[H];
#pragma unroll
    for (int r = 0; r < H; ++r) acc[r] = VT(0);
    bool first = true;
#pragma unroll
    for (int b = 0; b < T; ++b) {
#pragma unroll
      for (int r = 0; r < H; ++r) acc[r] += p[b][r];
      if (!((fl >> b) & 1u)) {
        const int64_t sr = a.seg_row ? (int64_t)__ldg(a.seg_row + seg) : seg;
        if (first) {
#pragma unroll
          for (int r = 0; r < H; ++r) acc[r] = Vex[r] + acc[r];
        }
        if (first && dependent_here) {
#pragma unroll
          for (int r = 0; r < H; ++r) s_dep[r] = acc[r];
          s_dep_row = sr;
        } else {
#pragma unroll
          for (int r = 0; r < H; ++r)
            if (sr * H + r < a.out_limit) out[sr * H + r] = acc[r];
        }
        first = false;
        ++seg;
#pragma unroll
        for (int r = 0; r < H; ++r) acc[r] = VT(0);
      }
    }
  }
  if (!tile_has_stop || tile == 0) return;  // nothing waits for a carry
  __syncthreads();

  // ---- step 3c: look back for the carry-in (decoupled look-back) --------
  if (wid == 0) {
    double carry[H];
#pragma unroll
    for (int r = 0; r < H; ++r) carry[r] = 0.0;
    int64_t j = tile - 1;
    while (true) {
      const int64_t idx = j - lane;
      int state = 2;  // before tile 0: an inclusive prefix of 0
      if (idx >= 0) {
        unsigned long long s;
        do { s = dev::ld_acquire(a.status + idx); } while ((s >> 2) != epoch);
        state = (int)(s & 3ull);
      }
      const unsigned pm = __ballot_sync(0xffffffffu, state == 2);
      const int lim = pm ? __ffs(pm) - 1 : 31;  // nearest tile with a row stop
#pragma unroll
      for (int r = 0; r < H; ++r) {
        double cv = (lane <= lim && idx >= 0) ? __ldcg(a.carry + idx * H + r) : 0.0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) cv += __shfl_xor_sync(0xffffffffu, cv, o);  // fixed tree
        carry[r] += cv;
      }
      if (pm) break;
      j -= 32;
    }
    if (lane == 0) {
      const int64_t sr = s_dep_row;
#pragma unroll
      for (int r = 0; r < H; ++r)
        if (sr * H + r < a.out_limit) out[sr * H + r] = (VT)((double)s_dep[r] + carry[r]);
    }
  }
}

template <typename VT, int H, int W, int T, int CM>
void launch_spmv(const KArgs& a, int C, int64_t grid, void* stream) {
  spmv_bccoo_kernel<VT, H, W, T, CM><<<(unsigned)grid, C, 0, (cudaStream_t)stream>>>(a);
}

template <typename VT, int H, int W, int T, int CM>
int attr_spmv(int* regs, int* max_threads) {
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, spmv_bccoo_kernel<VT, H, W, T, CM>);
  if (e != cudaSuccess) return (int)e;
  *regs = fa.numRegs;
  *max_threads = fa.maxThreadsPerBlock;
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
