// mb_gather.cu — microbenchmark: throughput of random 4-byte gathers on B200 from
// (a) global memory (L2-resident window), (b) the CTA's own shared memory, (c) distributed
// shared memory across a thread-block cluster (ld.shared::cluster).  Decides where C5's
// band gathers of x can be served.  Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb_gather tools/mb_gather.cu
#include <cooperative_groups.h>
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

namespace cg = cooperative_groups;

#define CK(x)                                                                          \
  do {                                                                                 \
    cudaError_t e_ = (x);                                                              \
    if (e_ != cudaSuccess) {                                                           \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      exit(1);                                                                         \
    }                                                                                  \
  } while (0)

__device__ __forceinline__ uint32_t hsh(uint32_t a) {
  a ^= a >> 16;
  a *= 0x7feb352du;
  a ^= a >> 15;
  return a;
}

constexpr int U = 16;  // independent gathers in flight per thread per iteration

__global__ void k_global(const float* __restrict__ x, uint32_t mask, int iters, float* out) {
  uint32_t s = hsh(blockIdx.x * blockDim.x + threadIdx.x + 1);
  float acc = 0.f;
  for (int it = 0; it < iters; ++it) {
    float v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      s = s * 1664525u + 1013904223u;
      v[u] = __ldg(x + ((s >> 7) & mask));
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc += v[u];
  }
  if (acc == 1.2345f) out[0] = acc;
}

// local shared memory: NW words per CTA
__global__ void k_smem(int nwords_log2, int iters, float* out) {
  extern __shared__ float sm[];
  const uint32_t n = 1u << nwords_log2, mask = n - 1;
  for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) sm[i] = (float)i;
  __syncthreads();
  uint32_t s = hsh(blockIdx.x * blockDim.x + threadIdx.x + 1);
  float acc = 0.f;
  for (int it = 0; it < iters; ++it) {
    float v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      s = s * 1664525u + 1013904223u;
      v[u] = sm[(s >> 7) & mask];
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc += v[u];
  }
  if (acc == 1.2345f) out[0] = acc;
}

// distributed shared memory: random word of a random CTA of the cluster (csz CTAs)
__global__ void k_dsmem(int nwords_log2, int csz_log2, int iters, int local_only, float* out) {
  extern __shared__ float sm[];
  cg::cluster_group cl = cg::this_cluster();
  const uint32_t n = 1u << nwords_log2, mask = n - 1;
  for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) sm[i] = (float)i;
  cl.sync();
  uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
  uint32_t rbase[8];
#pragma unroll
  for (int r = 0; r < 8; ++r) {
    uint32_t ra = 0;
    if (r < (1 << csz_log2)) asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(base), "r"(r));
    rbase[r] = ra;
  }
  const uint32_t me = cl.block_rank();
  uint32_t s = hsh(blockIdx.x * blockDim.x + threadIdx.x + 1);
  float acc = 0.f;
  const uint32_t rmask = (1u << csz_log2) - 1;
  for (int it = 0; it < iters; ++it) {
    float v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      s = s * 1664525u + 1013904223u;
      const uint32_t r = local_only ? me : ((s >> 27) & rmask);
      uint32_t a = 0;
      // select without local memory indexing
#pragma unroll
      for (int q = 0; q < 8; ++q) a = (q == (int)r) ? rbase[q] : a;
      a += ((s >> 7) & mask) * 4u;
      asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v[u]) : "r"(a));
    }
#pragma unroll
    for (int u = 0; u < U; ++u) acc += v[u];
  }
  cl.sync();
  if (acc == 1.2345f) out[0] = acc;
}

int main() {
  int dev = 0, nsm = 0;
  CK(cudaGetDevice(&dev));
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  float *x, *out;
  const size_t NX = 64u << 20;  // 256 MB
  CK(cudaMalloc(&x, NX * 4));
  CK(cudaMemset(x, 0, NX * 4));
  CK(cudaMalloc(&out, 4));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  auto timeit = [&](auto launch) {
    launch();
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(e0));
    for (int r = 0; r < 5; ++r) launch();
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    CK(cudaGetLastError());
    return ms / 5;
  };
  const int iters = 64;
  // (a) global: windows of 512 KB .. 256 MB, 8 CTAs x 256 threads per SM
  for (int lg : {17, 20, 22, 24, 26}) {
    const int th = 256, grid = nsm * 8;
    float ms = timeit([&] { k_global<<<grid, th>>>(x, (1u << lg) - 1, iters, out); });
    double g = (double)grid * th * iters * U / (ms * 1e-3) / 1e9;
    printf("global  window %8.1f KB : %8.1f G gathers/s  (%.3f ms)\n", (4.0 * (1u << lg)) / 1024, g, ms);
  }
  // (b) smem: 128 KB per CTA, 1 CTA/SM, 1024 threads; and 2 CTAs x 64 KB
  for (int cfg = 0; cfg < 3; ++cfg) {
    int lg = cfg == 0 ? 15 : 14, th = cfg == 2 ? 512 : 1024, per = cfg == 0 ? 1 : 2;
    size_t sb = (size_t)4 << lg;
    CK(cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sb));
    const int grid = nsm * per;
    float ms = timeit([&] { k_smem<<<grid, th, sb>>>(lg, iters, out); });
    double g = (double)grid * th * iters * U / (ms * 1e-3) / 1e9;
    printf("smem    %3d KB x %d CTA/SM, %4d thr : %8.1f G gathers/s  (%.3f ms)\n", (int)(sb >> 10), per, th, g, ms);
  }
  // (c) dsmem: cluster 2/4/8, 128 KB per CTA (and 64 KB with 2 CTAs per SM)
  for (int lc : {1, 2, 3}) {
    for (int local = 0; local < 2; ++local) {
      int lg = 15, th = 1024;
      size_t sb = (size_t)4 << lg;
      CK(cudaFuncSetAttribute(k_dsmem, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sb));
      if (lc == 3) CK(cudaFuncSetAttribute(k_dsmem, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
      const int csz = 1 << lc;
      int grid = (nsm / csz) * csz;
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(grid);
      cfg.blockDim = dim3(th);
      cfg.dynamicSmemBytes = sb;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeClusterDimension;
      at[0].val.clusterDim.x = csz;
      at[0].val.clusterDim.y = 1;
      at[0].val.clusterDim.z = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      int ncl = 0;
      CK(cudaOccupancyMaxActiveClusters(&ncl, (void*)k_dsmem, &cfg));
      float ms = timeit([&] { CK(cudaLaunchKernelEx(&cfg, k_dsmem, lg, lc, iters, local, out)); });
      double g = (double)grid * th * iters * U / (ms * 1e-3) / 1e9;
      printf("dsmem   cluster %d (%d active clusters) %s : %8.1f G gathers/s  (%.3f ms)\n", csz, ncl,
             local ? "own-CTA addr via mapa" : "random CTA        ", g, ms);
    }
  }
  return 0;
}
