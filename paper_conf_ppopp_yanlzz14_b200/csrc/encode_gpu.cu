// encode_gpu.cu — GPU-accelerated COO/CSR -> BCCOO/BCCOO+ translation (PAPER.md P:321:
// "we use GPUs to accelerate the translation from the COO format to the BCCOO/BCCOO+
// format").  Produces exactly the arrays of the host encoder (encode.cpp, E1-E9 of
// DESIGN.md), written straight into the device layout; parity is checked against the
// oracle through yaspmv_export_device (tests/test_encode_gpu.py).
//
//   1. row id of every entry: scatter row starts + inclusive max-scan
//   2. key = stacked block row * NB + block column (sr = (bc div SW)*MB + br);
//      sorted already for h = 1, S = 1 (CSR order), else a stable radix sort of (key, entry)
//   3. first entry of each distinct key = a block; exclusive scan -> block rank (E3 order)
//   4. blocks per stacked row -> offsets with / without FILLER blocks (Q1)
//   5. scatter columns, stop bits, values into the offline-transposed layout
//   6. column storage (u16 / i32 / int16 delta), stops per tile
#include <cuda_runtime.h>

#include <cub/cub.cuh>

#include <algorithm>
#include <string>

#include "common.hpp"

namespace yaspmv {

#define GTRY(expr)                                                                          \
  do {                                                                                      \
    cudaError_t _e = (expr);                                                                \
    if (_e != cudaSuccess) {                                                                \
      pool.release();                                                                       \
      out.free_all();                                                                       \
      return fail(_e == cudaErrorMemoryAllocation ? YASPMV_ENOMEM : YASPMV_ECUDA,           \
                  std::string("encode_gpu: ") + #expr + ": " + cudaGetErrorString(_e));     \
    }                                                                                       \
  } while (0)

namespace {

struct Pool {  // temporaries freed at the end (or on failure)
  std::vector<void*> ptrs;
  cudaStream_t st = nullptr;
  template <typename T>
  cudaError_t get(T** p, size_t n) {
    void* q = nullptr;
    cudaError_t e = cudaMalloc(&q, std::max<size_t>(n, 1) * sizeof(T));
    if (e == cudaSuccess) ptrs.push_back(q);
    *p = static_cast<T*>(q);
    return e;
  }
  void release() {
    for (void* p : ptrs) cudaFree(p);
    ptrs.clear();
  }
};

inline unsigned grid_for(int64_t n, int threads = 256) {
  int64_t g = (n + threads - 1) / threads;
  if (g > 1048576) g = 1048576;
  return (unsigned)std::max<int64_t>(g, 1);
}

__global__ void k_mark_rows(const int64_t* rp, int64_t m, int32_t* rowid) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x)
    if (rp[i] < rp[i + 1]) rowid[rp[i]] = (int32_t)i;
}

__global__ void k_keys(const int32_t* rowid, const int32_t* ci, int64_t nnz, int h, int w, int64_t MB, int64_t NB,
                       int64_t SW, unsigned long long* key, int64_t* idx) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t br = rowid[e] / h, bc = ci[e] / w;
    const int64_t sr = (bc / SW) * MB + br;
    key[e] = (unsigned long long)(sr * NB + bc);
    if (idx) idx[e] = e;
  }
}

__global__ void k_newblock(const unsigned long long* key, int64_t nnz, int64_t* flag) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x)
    flag[e] = (e == 0 || key[e] != key[e - 1]) ? 1 : 0;
}

__global__ void k_block_keys(const unsigned long long* key, const int64_t* flag, const int64_t* rank, int64_t nnz,
                             int64_t NB, unsigned long long* bkey, int32_t* cnt) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x)
    if (flag[e]) {
      bkey[rank[e]] = key[e];
      atomicAdd(cnt + key[e] / NB, 1);
    }
}

__global__ void k_rowcnt(const int32_t* cnt, int64_t nsr, int filler, int64_t* cnt_real, int64_t* cnt_full,
                         int64_t* empty) {
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < nsr; s += (int64_t)gridDim.x * blockDim.x) {
    cnt_real[s] = cnt[s];
    cnt_full[s] = (filler && cnt[s] == 0) ? 1 : cnt[s];
    empty[s] = cnt[s] == 0 ? 1 : 0;
  }
}

__device__ __forceinline__ void clear_bit(uint8_t* flags, int64_t b) {
  unsigned int* w = reinterpret_cast<unsigned int*>(flags) + (b >> 5);
  atomicAnd(w, ~(1u << (b & 31)));
}

__global__ void k_fill_blocks(const unsigned long long* bkey, int64_t nreal, int64_t NB, const int64_t* off_real,
                              const int64_t* off_full, const int32_t* cnt, int32_t* colb, uint8_t* flags) {
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nreal; b += (int64_t)gridDim.x * blockDim.x) {
    const int64_t sr = (int64_t)(bkey[b] / NB), bc = (int64_t)(bkey[b] % NB);
    const int64_t pos = off_full[sr] + (b - off_real[sr]);
    colb[pos] = (int32_t)bc;                                        // E5
    if (b == off_real[sr] + cnt[sr] - 1) clear_bit(flags, pos);     // E6: last block of its row
  }
}

__global__ void k_fillers(const int32_t* cnt, int64_t nsr, const int64_t* off_real, const int64_t* off_full,
                          const unsigned long long* bkey, int64_t NB, int32_t* colb, uint8_t* flags) {
  for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < nsr; s += (int64_t)gridDim.x * blockDim.x)
    if (cnt[s] == 0) {  // Q1 R1 / Q3: zero block in block column NB (x reads 0 there, Q4)
      const int64_t pos = off_full[s];
      colb[pos] = (int32_t)NB;
      clear_bit(flags, pos);
    }
}

__global__ void k_pad_cols(int32_t* colb, int64_t nnzb, int64_t np) {
  const int32_t last = nnzb > 0 ? colb[nnzb - 1] : 0;
  for (int64_t b = nnzb + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < np; b += (int64_t)gridDim.x * blockDim.x)
    colb[b] = last;
}

// device-layout byte address of byte `ob` of thread t's run in tile k (run = ptb bytes)
__device__ __forceinline__ int64_t dev_addr(int64_t k, int t, int C, int ptb, int ob) {
  const int ch = ptb < 16 ? ptb : 16;
  return k * (int64_t)C * ptb + ((int64_t)(ob / ch) * C + t) * ch + (ob % ch);
}

__global__ void k_values(const int64_t* order, const int64_t* rank, const int64_t* flag,
                         const unsigned long long* key, int64_t nnz,
                         const int32_t* rowid, const int32_t* ci, const uint8_t* v, int vs, int h, int w, int64_t NB,
                         const int64_t* off_real, const int64_t* off_full, int T, int C, uint8_t* val0,
                         uint8_t* val1, uint8_t* val2, uint8_t* val3) {
  const int64_t TC = (int64_t)T * C;
  const int ptb = T * w * vs;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nnz; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t o = order ? order[e] : e;  // original entry
    const int64_t sr = (int64_t)(key[e] / NB);
    const int64_t blk = rank[e] + flag[e] - 1;  // exclusive scan -> block index of entry e
    const int64_t pos = off_full[sr] + (blk - off_real[sr]);
    const int r = rowid[o] % h, c = ci[o] % w;
    const int64_t k = pos / TC;
    const int t = (int)((pos % TC) / T);
    const int ob = (int)(((pos % T) * w + c) * vs);
    uint8_t* dst = (r == 0 ? val0 : r == 1 ? val1 : r == 2 ? val2 : val3) + dev_addr(k, t, C, ptb, ob);
    if (vs == 4) *reinterpret_cast<uint32_t*>(dst) = reinterpret_cast<const uint32_t*>(v)[o];  // E4
    else *reinterpret_cast<unsigned long long*>(dst) = reinterpret_cast<const unsigned long long*>(v)[o];
  }
}

__global__ void k_cols(const int32_t* colb, int64_t np, int T, int C, int mode, void* dcol) {
  const int64_t TC = (int64_t)T * C;
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < np; b += (int64_t)gridDim.x * blockDim.x) {
    const int64_t k = b / TC;
    const int t = (int)((b % TC) / T), i = (int)(b % T);
    if (mode == COL_I32) {
      *reinterpret_cast<int32_t*>(static_cast<uint8_t*>(dcol) + dev_addr(k, t, C, 4 * T, 4 * i)) = colb[b];
    } else {
      int16_t v;
      if (mode == COL_U16) {
        v = (int16_t)(uint16_t)colb[b];
      } else {  // segmented int16 difference per thread tile, -1 = escape (Q7)
        const int64_t d = (int64_t)colb[b] - (i == 0 ? 0 : colb[b - 1]);
        v = (d < -32768 || d > 32767 || d == -1) ? (int16_t)-1 : (int16_t)d;
      }
      *reinterpret_cast<int16_t*>(static_cast<uint8_t*>(dcol) + dev_addr(k, t, C, 2 * T, 2 * i)) = v;
    }
  }
}

__global__ void k_tile_stops(const uint8_t* flags, int64_t ntiles, int64_t tb, int32_t* out) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < ntiles; k += (int64_t)gridDim.x * blockDim.x) {
    int z = 0;
    const unsigned int* w = reinterpret_cast<const unsigned int*>(flags + k * tb);
    for (int64_t q = 0; q < tb / 4; ++q) z += 32 - __popc(w[q]);
    out[k] = z;
  }
}

__global__ void k_iota(int32_t* a, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    a[i] = (int32_t)i;
}

__global__ void k_escapes(const int32_t* colb, int64_t np, int T, unsigned long long* n) {
  unsigned long long z = 0;
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < np; b += (int64_t)gridDim.x * blockDim.x) {
    const int64_t d = (int64_t)colb[b] - (b % T == 0 ? 0 : colb[b - 1]);
    z += (d < -32768 || d > 32767 || d == -1);
  }
  if (z) atomicAdd(n, z);
}

}  // namespace

yaspmv_status encode_gpu(const CSR& A, const Params& p, Canonical& meta, GpuArrays& outarr, int64_t& n_escapes,
                         void* stream) {
  Pool pool;
  cudaStream_t st = (cudaStream_t)stream;
  const int h = p.h, w = p.w, S = p.S, T = p.T, C = p.C, vs = A.vsize;
  const int64_t TC = (int64_t)T * C, m = A.m, n = A.n, nnz = A.nnz;
  meta = Canonical();
  meta.m = m;
  meta.n = n;
  meta.nnz = nnz;
  meta.vsize = vs;
  meta.MB = (m + h - 1) / h;
  meta.NB = (n + w - 1) / w;
  meta.SW = meta.NB > 0 ? (meta.NB + S - 1) / S : 1;
  const int64_t MB = meta.MB, NB = std::max<int64_t>(meta.NB, 1), SW = meta.SW, nsr = (int64_t)S * MB;
  GpuArrays out;
  (void)n;

  // inputs
  int64_t* rp = nullptr;
  int32_t *ci = nullptr, *rowid = nullptr;
  uint8_t* v = nullptr;
  GTRY(pool.get(&rp, m + 1));
  GTRY(pool.get(&ci, nnz));
  GTRY(pool.get(&v, (size_t)nnz * vs));
  GTRY(pool.get(&rowid, nnz));
  GTRY(cudaMemcpyAsync(rp, A.rp, (m + 1) * sizeof(int64_t), cudaMemcpyHostToDevice, st));
  if (nnz) {
    GTRY(cudaMemcpyAsync(ci, A.ci, nnz * sizeof(int32_t), cudaMemcpyHostToDevice, st));
    GTRY(cudaMemcpyAsync(v, A.v, (size_t)nnz * vs, cudaMemcpyHostToDevice, st));
  }
  void* tmp = nullptr;
  size_t tmp_bytes = 0, need = 0;
  auto ensure_tmp = [&](size_t b) -> cudaError_t {
    if (b <= tmp_bytes) return cudaSuccess;
    uint8_t* q = nullptr;
    cudaError_t e = pool.get(&q, b);
    tmp = q;
    tmp_bytes = b;
    return e;
  };
  // 1. row ids
  GTRY(cudaMemsetAsync(rowid, 0, std::max<int64_t>(nnz, 1) * sizeof(int32_t), st));
  k_mark_rows<<<grid_for(m), 256, 0, st>>>(rp, m, rowid);
  if (nnz) {
    GTRY(cub::DeviceScan::InclusiveScan(nullptr, need, rowid, rowid, cub::Max(), nnz, st));
    GTRY(ensure_tmp(need));
    GTRY(cub::DeviceScan::InclusiveScan(tmp, need, rowid, rowid, cub::Max(), nnz, st));
  }
  // 2. keys (+ sort unless already in order)
  unsigned long long *key = nullptr, *key2 = nullptr;
  int64_t *idx = nullptr, *idx2 = nullptr;
  const bool sorted = (h == 1 && S == 1);
  GTRY(pool.get(&key, nnz));
  if (!sorted) GTRY(pool.get(&idx, nnz));
  k_keys<<<grid_for(nnz), 256, 0, st>>>(rowid, ci, nnz, h, w, MB, NB, SW, key, sorted ? nullptr : idx);
  const int64_t* order = nullptr;
  if (!sorted && nnz) {
    GTRY(pool.get(&key2, nnz));
    GTRY(pool.get(&idx2, nnz));
    int end_bit = 1;
    while (end_bit < 64 && ((unsigned long long)nsr * (unsigned long long)NB) >> end_bit) ++end_bit;
    GTRY(cub::DeviceRadixSort::SortPairs(nullptr, need, key, key2, idx, idx2, nnz, 0, end_bit, st));
    GTRY(ensure_tmp(need));
    GTRY(cub::DeviceRadixSort::SortPairs(tmp, need, key, key2, idx, idx2, nnz, 0, end_bit, st));
    std::swap(key, key2);
    order = idx2;
  }
  // 3. blocks
  int64_t *flag = nullptr, *rank = nullptr;
  GTRY(pool.get(&flag, nnz));
  GTRY(pool.get(&rank, nnz));
  int64_t nreal = 0;
  if (nnz) {
    k_newblock<<<grid_for(nnz), 256, 0, st>>>(key, nnz, flag);
    GTRY(cub::DeviceScan::ExclusiveSum(nullptr, need, flag, rank, nnz, st));
    GTRY(ensure_tmp(need));
    GTRY(cub::DeviceScan::ExclusiveSum(tmp, need, flag, rank, nnz, st));
    int64_t last_rank = 0, last_flag = 0;
    GTRY(cudaMemcpyAsync(&last_rank, rank + nnz - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    GTRY(cudaMemcpyAsync(&last_flag, flag + nnz - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    GTRY(cudaStreamSynchronize(st));
    nreal = last_rank + last_flag;
  }
  unsigned long long* bkey = nullptr;
  int32_t* cnt = nullptr;
  GTRY(pool.get(&bkey, nreal));
  GTRY(pool.get(&cnt, nsr));
  GTRY(cudaMemsetAsync(cnt, 0, std::max<int64_t>(nsr, 1) * sizeof(int32_t), st));
  if (nnz) k_block_keys<<<grid_for(nnz), 256, 0, st>>>(key, flag, rank, nnz, NB, bkey, cnt);
  // 4. empty stacked rows -> empty mode (Q1), offsets
  int64_t *cr = nullptr, *cf = nullptr, *emp = nullptr, *off_real = nullptr, *off_full = nullptr, *sum1 = nullptr;
  GTRY(pool.get(&cr, nsr));
  GTRY(pool.get(&cf, nsr));
  GTRY(pool.get(&emp, nsr));
  GTRY(pool.get(&off_real, nsr + 1));
  GTRY(pool.get(&off_full, nsr + 1));
  GTRY(pool.get(&sum1, 1));
  int64_t n_empty = 0;
  if (nsr) {
    k_rowcnt<<<grid_for(nsr), 256, 0, st>>>(cnt, nsr, 0, cr, cf, emp);
    GTRY(cub::DeviceReduce::Sum(nullptr, need, emp, sum1, nsr, st));
    GTRY(ensure_tmp(need));
    GTRY(cub::DeviceReduce::Sum(tmp, need, emp, sum1, nsr, st));
    GTRY(cudaMemcpyAsync(&n_empty, sum1, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    GTRY(cudaStreamSynchronize(st));
  }
  Params rp_ = p;
  const int s_c = col_bytes(p.col_mode);
  if (rp_.empty_mode == 0) {  // same rule as the host encoder (Q1)
    const int64_t r1 = n_empty * (int64_t)(h * w * vs + s_c);
    const int64_t r2 = 4 * (nsr - n_empty) + 4 * n_empty;
    rp_.empty_mode = (n_empty == 0 || r1 <= r2) ? EMPTY_FILLER : EMPTY_MAP;
  }
  const bool filler = rp_.empty_mode == EMPTY_FILLER;
  if (nsr) {
    k_rowcnt<<<grid_for(nsr), 256, 0, st>>>(cnt, nsr, filler ? 1 : 0, cr, cf, emp);
    GTRY(cub::DeviceScan::ExclusiveSum(nullptr, need, cr, off_real, nsr + 0, st));
    GTRY(ensure_tmp(need));
    GTRY(cub::DeviceScan::ExclusiveSum(tmp, need, cr, off_real, nsr, st));
    GTRY(cub::DeviceScan::ExclusiveSum(tmp, need, cf, off_full, nsr, st));
  }
  int64_t nnzb = nreal + (filler ? n_empty : 0);
  const int64_t np = (nnzb + TC - 1) / TC * TC, ntiles = np / TC;
  meta.p = rp_;
  meta.nnzb = nnzb;
  meta.nnzb_pad = np;
  meta.ntiles = ntiles;
  meta.n_filler = filler ? n_empty : 0;

  // 5. outputs in the device layout
  int32_t* colb = nullptr;
  GTRY(pool.get(&colb, np));
  const int vptb = T * w * vs;
  for (int r = 0; r < h; ++r) {
    GTRY(cudaMalloc(&out.val[r], std::max<int64_t>(ntiles * C * vptb, 16)));
    GTRY(cudaMemsetAsync(out.val[r], 0, std::max<int64_t>(ntiles * C * vptb, 16), st));
  }
  GTRY(cudaMalloc((void**)&out.flags, std::max<int64_t>(np / 8, 16)));
  GTRY(cudaMemsetAsync(out.flags, 0xFF, std::max<int64_t>(np / 8, 16), st));
  if (nreal)
    k_fill_blocks<<<grid_for(nreal), 256, 0, st>>>(bkey, nreal, NB, off_real, off_full, cnt, colb, out.flags);
  if (filler && n_empty)
    k_fillers<<<grid_for(nsr), 256, 0, st>>>(cnt, nsr, off_real, off_full, bkey, NB, colb, out.flags);
  if (np > nnzb) k_pad_cols<<<grid_for(np - nnzb), 256, 0, st>>>(colb, nnzb, np);
  if (nnz)
    k_values<<<grid_for(nnz), 256, 0, st>>>(order, rank, flag, key, nnz, rowid, ci, v, vs, h, w, NB, off_real, off_full, T,
                                            C, static_cast<uint8_t*>(out.val[0]), static_cast<uint8_t*>(out.val[1]),
                                            static_cast<uint8_t*>(out.val[2]), static_cast<uint8_t*>(out.val[3]));
  // 6. column storage, stops per tile
  const int cptb = T * col_bytes(rp_.col_mode);
  GTRY(cudaMalloc(&out.col, std::max<int64_t>(ntiles * C * cptb, 16)));
  if (np) k_cols<<<grid_for(np), 256, 0, st>>>(colb, np, T, C, rp_.col_mode, out.col);
  n_escapes = 0;
  if (rp_.col_mode == COL_DELTA) {
    GTRY(cudaMalloc((void**)&out.col32, std::max<int64_t>(np, 1) * sizeof(int32_t)));
    GTRY(cudaMemcpyAsync(out.col32, colb, np * sizeof(int32_t), cudaMemcpyDeviceToDevice, st));
    unsigned long long* ne = nullptr;
    GTRY(pool.get(&ne, 1));
    GTRY(cudaMemsetAsync(ne, 0, sizeof(unsigned long long), st));
    if (np) k_escapes<<<grid_for(np), 256, 0, st>>>(colb, np, T, ne);
    unsigned long long hne = 0;
    GTRY(cudaMemcpyAsync(&hne, ne, sizeof(hne), cudaMemcpyDeviceToHost, st));
    GTRY(cudaStreamSynchronize(st));
    n_escapes = (int64_t)hne;
  }
  int32_t* tstops = nullptr;
  GTRY(pool.get(&tstops, ntiles + 1));
  GTRY(cudaMalloc((void**)&out.cta_seg0, std::max<int64_t>(ntiles, 1) * sizeof(int32_t)));
  int64_t n_stops = 0;
  if (ntiles) {
    k_tile_stops<<<grid_for(ntiles), 256, 0, st>>>(out.flags, ntiles, TC / 8, tstops);
    GTRY(cub::DeviceScan::ExclusiveSum(nullptr, need, tstops, out.cta_seg0, ntiles, st));
    GTRY(ensure_tmp(need));
    GTRY(cub::DeviceScan::ExclusiveSum(tmp, need, tstops, out.cta_seg0, ntiles, st));
    int32_t a = 0, b = 0;
    GTRY(cudaMemcpyAsync(&a, out.cta_seg0 + ntiles - 1, 4, cudaMemcpyDeviceToHost, st));
    GTRY(cudaMemcpyAsync(&b, tstops + ntiles - 1, 4, cudaMemcpyDeviceToHost, st));
    GTRY(cudaStreamSynchronize(st));
    n_stops = (int64_t)a + b;
  }
  meta.n_stops = n_stops;
  // Q1 R2: seg_row (non-empty stacked rows in order) and zero_rows (the others)
  if (!filler && n_empty) {
    int32_t* ids = nullptr;
    int64_t* nsel = nullptr;
    GTRY(pool.get(&ids, nsr));
    GTRY(pool.get(&nsel, 1));
    k_iota<<<grid_for(nsr), 256, 0, st>>>(ids, nsr);
    GTRY(cudaMalloc((void**)&out.seg_row, std::max<int64_t>(nsr - n_empty, 1) * sizeof(int32_t)));
    GTRY(cudaMalloc((void**)&out.zero_rows, std::max<int64_t>(n_empty, 1) * sizeof(int32_t)));
    // flags: emp (1 = empty) and cr (>0 = non-empty)
    GTRY(cub::DeviceSelect::Flagged(nullptr, need, ids, cr, out.seg_row, nsel, nsr, st));
    GTRY(ensure_tmp(need));
    GTRY(cub::DeviceSelect::Flagged(tmp, need, ids, cr, out.seg_row, nsel, nsr, st));
    GTRY(cub::DeviceSelect::Flagged(tmp, need, ids, emp, out.zero_rows, nsel, nsr, st));
    meta.has_seg_row = 1;
    meta.n_zero = n_empty;
  }
  GTRY(cudaStreamSynchronize(st));
  pool.release();
  outarr = out;
  return YASPMV_OK;
}

}  // namespace yaspmv
