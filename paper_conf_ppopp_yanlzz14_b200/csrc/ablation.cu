// ablation.cu — the baselines of the paper's Fig. 14 ablation, rebuilt on B200
// for measurement only (tools/ablation.py; include/yaspmv_ablation.h):
//   "COO"   : COO format + a tree-based segmented sum [5] (Blelloch/Hillis-Steele levels
//             with a barrier between levels) + a second kernel for the carries
//   "BCCOO" : the same tree-based segmented sum over the BCCOO bit flags
// and the second-kernel carry fix-up used by "Efficient segmented sum/scan" (our kernel
// with ABL_DEFER_CARRY) before adjacent synchronization replaces it.
#include <cuda_runtime.h>

#include "common.hpp"

namespace yaspmv {

// carry fix-up: tile k's first segment continues from earlier tiles; its carry is the sum
// of the published values back to the nearest tile holding a segment end (state 2),
// folded newest to oldest (fixed order, deterministic).  Runs after all tiles published.
template <typename VT>
__global__ void carry_fixup_kernel(const unsigned long long* status, int sstride, const double* carry,
                                   const int64_t* dep_row, int64_t ntiles, VT* y) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < ntiles; k += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = dep_row[k];
    if (r < 0) continue;
    double c = 0.0;
    for (int64_t i = k - 1; i >= 0; --i) {
      c += carry[i];
      if ((status[i * sstride] & 3ull) == 2ull) break;
    }
    y[r] = (VT)((double)y[r] + c);
  }
}

void launch_carry_fixup(const unsigned long long* status, const double* carry, const int64_t* dep_row,
                        int64_t ntiles, void* y, int dtype, void* stream, int sstride) {
  int64_t g = (ntiles + 255) / 256;
  if (g < 1) g = 1;
  if (g > 65535) g = 65535;
  if (dtype == 0)
    carry_fixup_kernel<float><<<(unsigned)g, 256, 0, (cudaStream_t)stream>>>(status, sstride, carry, dep_row, ntiles,
                                                                               (float*)y);
  else
    carry_fixup_kernel<double><<<(unsigned)g, 256, 0, (cudaStream_t)stream>>>(status, sstride, carry, dep_row, ntiles,
                                                                                (double*)y);
}

// Tree-based segmented sum over 1024-element tiles (256 threads x 4 elements): products
// and head flags in shared memory, log2(1024) = 10 levels of a segmented Hillis-Steele scan
// with barriers, then every segment end writes its row.  COO: row index per element
// (rows != NULL); BCCOO: bit flags + the per-tile stop offset (tile_seg0).
constexpr int TR_NT = 256, TR_EPT = 4, TR_TILE = TR_NT * TR_EPT;

template <typename VT, bool COO>
__global__ void __launch_bounds__(TR_NT) tree_segsum_kernel(const int32_t* rows, const uint8_t* flags,
                                                            const int32_t* tile_seg0, const int32_t* col,
                                                            const VT* val, int64_t n_elem, const VT* x, VT* y,
                                                            int64_t m, unsigned long long* status, double* carry,
                                                            int64_t* dep_row) {
  __shared__ VT sv[2][TR_TILE];
  __shared__ int sf[2][TR_TILE];  // segment-start flags (scanned with OR)
  __shared__ int sn[2][TR_TILE];  // ends before (BCCOO row numbers)
  __shared__ unsigned char se[TR_TILE];
  const int t = threadIdx.x;
  const int64_t tile = blockIdx.x, base = tile * TR_TILE;
  for (int k = 0; k < TR_EPT; ++k) {
    const int i = k * TR_NT + t;
    const int64_t e = base + i;
    VT p = VT(0);
    int start = 0, end = 0;
    if (e < n_elem) {
      p = val[e] * x[col[e]];
      if (COO) {
        start = (e == 0 || rows[e] != rows[e - 1]);
        end = (e == n_elem - 1 || rows[e + 1] != rows[e]);
      } else {
        start = (e == 0) || !((flags[(e - 1) >> 3] >> ((e - 1) & 7)) & 1);
        end = !((flags[e >> 3] >> (e & 7)) & 1);
      }
    }
    sv[0][i] = p;
    sf[0][i] = start;
    sn[0][i] = end;
    se[i] = (unsigned char)end;
  }
  __syncthreads();
  int cur = 0;
  for (int d = 1; d < TR_TILE; d <<= 1) {  // one tree level per iteration, barrier between
    for (int k = 0; k < TR_EPT; ++k) {
      const int i = k * TR_NT + t;
      VT v = sv[cur][i];
      int f = sf[cur][i], nn = sn[cur][i];
      if (i >= d) {
        if (!f) v = sv[cur][i - d] + v;
        f |= sf[cur][i - d];
        nn += sn[cur][i - d];
      }
      sv[cur ^ 1][i] = v;
      sf[cur ^ 1][i] = f;
      sn[cur ^ 1][i] = nn;
    }
    __syncthreads();
    cur ^= 1;
  }
  // write segment ends; the tile's first segment may continue from earlier tiles
  bool dep_here = false;
  for (int k = 0; k < TR_EPT; ++k) {
    const int i = k * TR_NT + t;
    const int64_t e = base + i;
    if (e >= n_elem || !se[i]) continue;
    const int64_t row = COO ? (int64_t)rows[e] : (int64_t)tile_seg0[tile] + sn[cur][i] - 1;
    if (row < m) y[row] = sv[cur][i];
    if (!sf[cur][i] && tile > 0) {  // no segment start at or before i in this tile
      dep_row[tile] = row;
      dep_here = true;
    }
  }
  (void)dep_here;
  if (t == TR_NT - 1) {
    const int i = TR_TILE - 1;
    const int has_end = sn[cur][i] > 0;
    // tail = the open segment after the last end (the whole tile without an end)
    carry[tile] = (double)(se[i] ? VT(0) : sv[cur][i]);
    status[tile] = has_end ? 2ull : 1ull;
  }
}

__global__ void fill_i64(int64_t* a, int64_t n, int64_t v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) a[i] = v;
}

int launch_tree_segsum(const int32_t* rows, const uint8_t* flags, const int32_t* tile_seg0, const int32_t* col,
                       const void* val, int64_t n_elem, const void* x, void* y, int64_t m, int dtype,
                       unsigned long long* status, double* carry, int64_t* dep_row, void* stream) {
  const int64_t ntiles = (n_elem + TR_TILE - 1) / TR_TILE;
  if (ntiles == 0) return 0;
  cudaStream_t st = (cudaStream_t)stream;
  fill_i64<<<(unsigned)((ntiles + 255) / 256 > 65535 ? 65535 : (ntiles + 255) / 256), 256, 0, st>>>(dep_row, ntiles, -1);
  const bool coo = rows != nullptr;
  if (dtype == 0) {
    if (coo) tree_segsum_kernel<float, true><<<(unsigned)ntiles, TR_NT, 0, st>>>(rows, flags, tile_seg0, col, (const float*)val, n_elem, (const float*)x, (float*)y, m, status, carry, dep_row);
    else tree_segsum_kernel<float, false><<<(unsigned)ntiles, TR_NT, 0, st>>>(rows, flags, tile_seg0, col, (const float*)val, n_elem, (const float*)x, (float*)y, m, status, carry, dep_row);
  } else {
    if (coo) tree_segsum_kernel<double, true><<<(unsigned)ntiles, TR_NT, 0, st>>>(rows, flags, tile_seg0, col, (const double*)val, n_elem, (const double*)x, (double*)y, m, status, carry, dep_row);
    else tree_segsum_kernel<double, false><<<(unsigned)ntiles, TR_NT, 0, st>>>(rows, flags, tile_seg0, col, (const double*)val, n_elem, (const double*)x, (double*)y, m, status, carry, dep_row);
  }
  launch_carry_fixup(status, carry, dep_row, ntiles, y, dtype, stream);
  return (int)cudaGetLastError();
}

}  // namespace yaspmv
