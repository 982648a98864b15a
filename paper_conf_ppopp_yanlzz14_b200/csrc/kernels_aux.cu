// kernels_aux.cu — BCCOO+ slice combine, power-iteration helpers, and the
// registry of precompiled SpMV instances.
#include <cuda_runtime.h>

#include <algorithm>
#include <mutex>

#include "common.hpp"

namespace yaspmv {

// ---------------------------------------------------------------- BCCOO+ combine
// y[i] = sum_{s=0..S-1} tmp[s*stride + i], ascending s (Fig. 5; Q11), fp64
// accumulation then one rounding.  Vectorised 4 elements per thread when aligned.
__device__ __forceinline__ double block_sum256(double v);

// optional power-iteration epilogue: y scaled by 1/sqrt(*in_norm2), block partials of y^2
template <typename VT>
__global__ void combine_kernel(const VT* __restrict__ tmp, VT* __restrict__ y, int64_t m, int64_t stride, int S,
                               const double* __restrict__ in_norm2, double* __restrict__ part, const PeerOut peers) {
  cudaTriggerProgrammaticLaunchCompletion();
  const int64_t nthreads = (int64_t)gridDim.x * blockDim.x;
  const double inv = in_norm2 ? 1.0 / sqrt(in_norm2[0]) : 1.0;
  double ss = 0.0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += nthreads) {
    double s = (double)__ldcs(tmp + i);
    for (int q = 1; q < S; ++q) s += (double)__ldcs(tmp + (int64_t)q * stride + i);
    const VT o = in_norm2 ? (VT)((VT)s * inv) : (VT)s;
    if (peers.mc) {  // fused exchange through an NVSwitch multicast mapping
      multimem_store(static_cast<VT*>(peers.p[0]) + i, o);
    } else if (peers.n > 0) {  // fused exchange: every rank's copy of the next x (yaspmv_power_step_fused)
#pragma unroll
      for (int q = 0; q < YASPMV_MAX_RANKS; ++q)
        if (q < peers.n) static_cast<VT*>(peers.p[q])[i] = o;
    } else {
      y[i] = o;
    }
    ss += (double)o * (double)o;
  }
  if (part) {
    ss = block_sum256(ss);
    if (threadIdx.x == 0) part[blockIdx.x] = ss;
  }
}

static int num_sms() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  return sms;
}

int64_t combine_blocks(int64_t m) {
  int64_t blocks = (m + 255) / 256;
  const int64_t cap = (int64_t)num_sms() * 16;
  if (blocks > cap) blocks = cap;
  return blocks < 1 ? 1 : blocks;
}

void launch_combine(const void* tmp, void* y, int64_t m, int64_t stride, int S, int dtype, void* stream,
                    const double* in_norm2, double* part, const PeerOut* peers) {
  if (m <= 0) return;
  const int64_t blocks = combine_blocks(m);
  const PeerOut po = peers ? *peers : PeerOut();
  if (dtype == 0)
    combine_kernel<float><<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>((const float*)tmp, (float*)y, m,
                                                                             stride, S, in_norm2, part, po);
  else
    combine_kernel<double><<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>((const double*)tmp, (double*)y, m,
                                                                               stride, S, in_norm2, part, po);
}

// zeros through a multicast mapping (an empty matrix in a fused step: cudaMemset does not take
// multicast addresses)
template <typename VT>
__global__ void mc_zero_kernel(VT* p, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    multimem_store(p + i, VT(0));
}
void launch_mc_zero(void* p, int64_t n, int dtype, void* stream) {
  if (n <= 0) return;
  const unsigned blocks = (unsigned)std::min<int64_t>((n + 255) / 256, 1184);
  if (dtype == 0) mc_zero_kernel<float><<<blocks, 256, 0, (cudaStream_t)stream>>>((float*)p, n);
  else mc_zero_kernel<double><<<blocks, 256, 0, (cudaStream_t)stream>>>((double*)p, n);
}

// ---------------------------------------------------------------- ||v||^2
// Deterministic two-pass reduction: fixed grid, fixed per-block partials, one final block.
static constexpr int NRM_THREADS = 256;
static constexpr int NRM_MAX_BLOCKS = 1184;  // 8 x 148

int64_t nrm2sq_blocks(int64_t n) {
  int64_t b = (n + NRM_THREADS * 4 - 1) / (NRM_THREADS * 4);
  if (b < 1) b = 1;
  if (b > NRM_MAX_BLOCKS) b = NRM_MAX_BLOCKS;
  return b;
}

__device__ __forceinline__ double block_sum(double v) {
  __shared__ double sh[NRM_THREADS / 32];
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = v;
  __syncthreads();
  double r = 0.0;
  if (threadIdx.x == 0)
    for (int q = 0; q < NRM_THREADS / 32; ++q) r += sh[q];
  return r;
}

template <typename VT>
__global__ void nrm2sq_partial(const VT* __restrict__ v, int64_t n, double* __restrict__ partials) {
  double s = 0.0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    const double a = (double)v[i];
    s = fma(a, a, s);
  }
  s = block_sum(s);
  if (threadIdx.x == 0) partials[blockIdx.x] = s;
}

__device__ __forceinline__ double block_sum256(double v) { return block_sum(v); }

__global__ void sum_f64_partial(const double* __restrict__ v, int64_t n, double* __restrict__ partials) {
  cudaTriggerProgrammaticLaunchCompletion();
  double s = 0.0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) s += v[i];
  s = block_sum(s);
  if (threadIdx.x == 0) partials[blockIdx.x] = s;
}

__global__ void nrm2sq_final(const double* __restrict__ partials, int nb, double* __restrict__ out) {
  cudaTriggerProgrammaticLaunchCompletion();
  double s = 0.0;
  for (int i = threadIdx.x; i < nb; i += blockDim.x) s += partials[i];
  s = block_sum(s);
  if (threadIdx.x == 0) out[0] = s;
}

void launch_nrm2sq(const void* v, int64_t n, int dtype, double* out, double* partials, void* stream) {
  const int64_t nb = nrm2sq_blocks(n);
  cudaStream_t st = (cudaStream_t)stream;
  if (dtype == 0) nrm2sq_partial<float><<<(unsigned)nb, NRM_THREADS, 0, st>>>((const float*)v, n, partials);
  else nrm2sq_partial<double><<<(unsigned)nb, NRM_THREADS, 0, st>>>((const double*)v, n, partials);
  nrm2sq_final<<<1, NRM_THREADS, 0, st>>>(partials, (int)nb, out);
}

// deterministic sum of n doubles (fixed grid for a given n): out[0] = sum v
void launch_sum_f64(const double* v, int64_t n, double* out, double* partials, void* stream) {
  const int64_t nb = nrm2sq_blocks(n);
  cudaStream_t st = (cudaStream_t)stream;
  sum_f64_partial<<<(unsigned)nb, NRM_THREADS, 0, st>>>(v, n, partials);
  nrm2sq_final<<<1, NRM_THREADS, 0, st>>>(partials, (int)nb, out);
}

// ---------------------------------------------------------------- dst = src / ||.||
template <typename VT>
__global__ void scale_kernel(const VT* src, VT* dst, int64_t n, const double* __restrict__ norm2) {
  const double inv = 1.0 / sqrt(norm2[0]);
  const VT f = (VT)inv;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) dst[i] = src[i] * f;
}

void launch_scale(const void* src, void* dst, int64_t n, int dtype, const double* norm2, void* stream) {
  if (n <= 0) return;
  int64_t blocks = (n + 255) / 256;
  const int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  cudaStream_t st = (cudaStream_t)stream;
  if (dtype == 0) scale_kernel<float><<<(unsigned)blocks, 256, 0, st>>>((const float*)src, (float*)dst, n, norm2);
  else scale_kernel<double><<<(unsigned)blocks, 256, 0, st>>>((const double*)src, (double*)dst, n, norm2);
}

// ---------------------------------------------------------------- registry
void register_s1_f32_h1(std::vector<KernelEntry>&);
void register_s1_f32_h2(std::vector<KernelEntry>&);
void register_s1_f32_h3(std::vector<KernelEntry>&);
void register_s1_f32_h4(std::vector<KernelEntry>&);
void register_s1_f64_h1(std::vector<KernelEntry>&);
void register_s1_f64_h2(std::vector<KernelEntry>&);
void register_s1_f64_h3(std::vector<KernelEntry>&);
void register_s1_f64_h4(std::vector<KernelEntry>&);
void register_s2_f32_h1(std::vector<KernelEntry>&);
void register_s2_f32_h2(std::vector<KernelEntry>&);
void register_s2_f32_h3(std::vector<KernelEntry>&);
void register_s2_f32_h4(std::vector<KernelEntry>&);
void register_s2_f64_h1(std::vector<KernelEntry>&);
void register_s2_f64_h2(std::vector<KernelEntry>&);
void register_s2_f64_h3(std::vector<KernelEntry>&);
void register_s2_f64_h4(std::vector<KernelEntry>&);

const std::vector<KernelEntry>& all_kernels() {
  static std::vector<KernelEntry> R;
  static std::once_flag once;
  std::call_once(once, [] {
    register_s1_f32_h1(R);
    register_s1_f32_h2(R);
    register_s1_f32_h3(R);
    register_s1_f32_h4(R);
    register_s1_f64_h1(R);
    register_s1_f64_h2(R);
    register_s1_f64_h3(R);
    register_s1_f64_h4(R);
    register_s2_f32_h1(R);
    register_s2_f32_h2(R);
    register_s2_f32_h3(R);
    register_s2_f32_h4(R);
    register_s2_f64_h1(R);
    register_s2_f64_h2(R);
    register_s2_f64_h3(R);
    register_s2_f64_h4(R);
  });
  return R;
}

const KernelEntry* find_kernel(int dtype, int h, int w, int T, int cm, int strat) {
  for (const KernelEntry& e : all_kernels())
    if (e.dtype == dtype && e.h == h && e.w == w && e.T == T && e.cm == cm && e.strat == strat) return &e;
  return nullptr;
}

}  // namespace yaspmv
