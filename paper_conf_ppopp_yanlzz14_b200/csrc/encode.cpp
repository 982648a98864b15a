// encode.cpp — host BCCOO / BCCOO+ encoder (multi-threaded C++).
//
// Implements SURVEY §8(a) steps a1-a4 (build time) following PAPER.md §2:
//   a1 normalise input: sort by (row, col), sum duplicates, keep explicit zeros
//   a2 h x w blocking and BCCOO+ vertical slices stacked top-down
//   a3 canonical arrays: bit flags, 0 = row stop, padded with 1s to the workgroup
//      tile, original block columns, h value arrays,
//      u16 / int32 / int16-delta column storage
//   a4 aux: row stops before every workgroup tile (the first-result entry)
// and the device layout (offline transpose).  Readings of silent or garbled
// passages are DESIGN.md Q1-Q16; this file shares no code with oracle/ (the oracle's
// encoder is an independent numpy program checked against this one bit for bit).
#include <omp.h>

#include <algorithm>
#include <atomic>
#include <cstring>
#include <numeric>

#include "common.hpp"

namespace yaspmv {

void CSR::make_owned() {
  if (owned()) return;
  rp_own.assign(rp, rp + m + 1);
  ci_own.assign(ci, ci + nnz);
  v_own.assign(v, v + (size_t)nnz * vsize);
  adopt_owned();
}

void Canonical::release_arrays() {
  std::vector<uint8_t>().swap(flags);
  std::vector<uint16_t>().swap(col16);
  std::vector<int32_t>().swap(col32);
  std::vector<int16_t>().swap(delta);
  for (auto& v : val) std::vector<uint8_t>().swap(v);
  std::vector<int32_t>().swap(seg_row);
  std::vector<int32_t>().swap(zero_rows);
}

int64_t footprint_bytes(int64_t nnzb, int h, int w, int vsize, int s_c) {
  // Table 3's footprint: the sum of the array sizes: values, col_index, bit flags
  return nnzb * (int64_t)(h * w * vsize + s_c) + (nnzb + 7) / 8;
}

// ------------------------------------------------------------------------- a1
namespace {

template <typename VT>
void sum_dups_row(const int32_t* ci, const VT* v, int64_t len, std::vector<int64_t>& idx,
                  std::vector<int32_t>& oc, std::vector<VT>& ov) {
  idx.resize(len);
  std::iota(idx.begin(), idx.end(), 0);
  std::stable_sort(idx.begin(), idx.end(), [&](int64_t a, int64_t b) { return ci[a] < ci[b]; });
  oc.clear();
  ov.clear();
  for (int64_t k = 0; k < len; ++k) {
    int32_t c = ci[idx[k]];
    VT x = v[idx[k]];
    if (!oc.empty() && oc.back() == c) ov.back() = ov.back() + x;  // input order (Q14)
    else { oc.push_back(c); ov.push_back(x); }
  }
}

template <typename VT>
yaspmv_status normalize_rows(int64_t m, int64_t n, const int64_t* rp, const int32_t* ci, const VT* v, CSR& out) {
  // per row: stable sort by column, sum duplicates in input order
  std::vector<int64_t> newlen(m);
#pragma omp parallel
  {
    std::vector<int64_t> idx;
    std::vector<int32_t> oc;
    std::vector<VT> ov;
#pragma omp for schedule(dynamic, 1024)
    for (int64_t i = 0; i < m; ++i) {
      sum_dups_row<VT>(ci + rp[i], v + rp[i], rp[i + 1] - rp[i], idx, oc, ov);
      newlen[i] = (int64_t)oc.size();
    }
  }
  out.m = m;
  out.n = n;
  out.vsize = sizeof(VT);
  out.rp_own.assign(m + 1, 0);
  for (int64_t i = 0; i < m; ++i) out.rp_own[i + 1] = out.rp_own[i] + newlen[i];
  out.nnz = out.rp_own[m];
  out.ci_own.resize(out.nnz);
  out.v_own.resize((size_t)out.nnz * sizeof(VT));
  VT* ovals = reinterpret_cast<VT*>(out.v_own.data());
#pragma omp parallel
  {
    std::vector<int64_t> idx;
    std::vector<int32_t> oc;
    std::vector<VT> ov;
#pragma omp for schedule(dynamic, 1024)
    for (int64_t i = 0; i < m; ++i) {
      sum_dups_row<VT>(ci + rp[i], v + rp[i], rp[i + 1] - rp[i], idx, oc, ov);
      std::copy(oc.begin(), oc.end(), out.ci_own.begin() + out.rp_own[i]);
      std::copy(ov.begin(), ov.end(), ovals + out.rp_own[i]);
    }
  }
  out.adopt_owned();
  return YASPMV_OK;
}

}  // namespace

yaspmv_status normalize_csr(int64_t m, int64_t n, const int64_t* rp, const int32_t* ci, const void* v,
                            int vsize, CSR& out) {
  if (m < 0 || n < 0) return fail(YASPMV_EINVAL, "m and n must be >= 0");
  if (m > INT32_MAX || n > INT32_MAX) return fail(YASPMV_EINVAL, "m and n must fit int32 (column indices are int32)");
  if (!rp) return fail(YASPMV_EINVAL, "row_ptr is NULL");
  if (rp[0] != 0) return fail(YASPMV_EINVAL, "row_ptr[0] must be 0");
  const int64_t nnz = rp[m];
  if (nnz > 0 && (!ci || !v)) return fail(YASPMV_EINVAL, "col_idx / vals NULL with nnz > 0");
  std::atomic<int> bad_mono{0}, bad_range{0}, unsorted{0};
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < m; ++i) {
    if (rp[i + 1] < rp[i]) { bad_mono = 1; continue; }
    for (int64_t k = rp[i]; k < rp[i + 1]; ++k) {
      if (ci[k] < 0 || ci[k] >= n) bad_range = 1;
      if (k > rp[i] && ci[k] <= ci[k - 1]) unsorted = 1;
    }
  }
  if (bad_mono) return fail(YASPMV_EINVAL, "row_ptr is not non-decreasing");
  if (bad_range) return fail(YASPMV_EINVAL, "column index out of range [0, n)");
  out = CSR();
  out.m = m;
  out.n = n;
  out.vsize = vsize;
  out.nnz = nnz;
  if (!unsorted) {  // already normalised: view the caller's arrays
    out.rp = rp;
    out.ci = ci;
    out.v = static_cast<const uint8_t*>(v);
    return YASPMV_OK;
  }
  if (vsize == 4) return normalize_rows<float>(m, n, rp, ci, static_cast<const float*>(v), out);
  return normalize_rows<double>(m, n, rp, ci, static_cast<const double*>(v), out);
}

yaspmv_status normalize_coo(int64_t m, int64_t n, int64_t nnz, const int32_t* ri, const int32_t* ci,
                            const void* v, int vsize, CSR& out) {
  if (m < 0 || n < 0 || nnz < 0) return fail(YASPMV_EINVAL, "m, n, nnz must be >= 0");
  if (m > INT32_MAX || n > INT32_MAX) return fail(YASPMV_EINVAL, "m and n must fit int32");
  if (nnz > 0 && (!ri || !ci || !v)) return fail(YASPMV_EINVAL, "NULL COO arrays with nnz > 0");
  for (int64_t k = 0; k < nnz; ++k)
    if (ri[k] < 0 || ri[k] >= m || ci[k] < 0 || ci[k] >= n)
      return fail(YASPMV_EINVAL, "COO index out of range");
  // stable counting sort by row -> CSR in input order inside each row
  std::vector<int64_t> rp(m + 1, 0);
  for (int64_t k = 0; k < nnz; ++k) rp[ri[k] + 1]++;
  for (int64_t i = 0; i < m; ++i) rp[i + 1] += rp[i];
  std::vector<int64_t> pos(rp.begin(), rp.end() - 1);
  std::vector<int32_t> c(nnz);
  std::vector<uint8_t> vv((size_t)nnz * vsize);
  const uint8_t* vb = static_cast<const uint8_t*>(v);
  for (int64_t k = 0; k < nnz; ++k) {
    int64_t d = pos[ri[k]]++;
    c[d] = ci[k];
    std::memcpy(&vv[(size_t)d * vsize], vb + (size_t)k * vsize, vsize);
  }
  CSR tmp;
  yaspmv_status st = normalize_csr(m, n, rp.data(), c.data(), vv.data(), vsize, tmp);
  if (st != YASPMV_OK) return st;
  tmp.make_owned();
  out = std::move(tmp);
  out.adopt_owned();
  return YASPMV_OK;
}

// ------------------------------------------------------------------------- params
yaspmv_status resolve_params(const Params& in, int64_t m, int64_t n, Params& out) {
  out = in;
  if (out.h == 0) out.h = 1;
  if (out.w == 0) out.w = 1;
  if (out.S == 0) out.S = 1;
  if (out.T == 0) out.T = 16;
  if (out.C == 0) out.C = 256;
  if (out.h < 1 || out.h > 4) return fail(YASPMV_EINVAL, "block_h must be in {1,2,3,4} (Table 1)");
  // Table 1 has w in {1,2,4}; 8 is the extension the paper's Dense result asks for
  // (clSpMV's 2x8 BCSR beat yaSpMV there)
  if (out.w != 1 && out.w != 2 && out.w != 4 && out.w != 8)
    return fail(YASPMV_EINVAL, "block_w must be in {1,2,4,8} (Table 1 + the w = 8 extension)");
  if (out.T != 4 && out.T != 8 && out.T != 16 && out.T != 32)
    return fail(YASPMV_EINVAL, "thread_tile must be in {4,8,16,32}");
  if (out.C != 64 && out.C != 128 && out.C != 256 && out.C != 512)
    return fail(YASPMV_EINVAL, "cta_size must be in {64,128,256,512} (Table 1)");
  const int64_t NB = (n + out.w - 1) / out.w;
  if (out.S < 1 || (NB > 0 && out.S > NB)) return fail(YASPMV_EINVAL, "slices must satisfy 1 <= S <= ceil(n/w)");
  if (out.col_mode == 0) out.col_mode = NB < 65535 ? COL_U16 : COL_I32;  // P:302, Q6
  if (out.col_mode < 1 || out.col_mode > 3) return fail(YASPMV_EINVAL, "bad col_mode");
  if (out.col_mode == COL_U16 && NB >= 65535)
    return fail(YASPMV_EINVAL, "u16 column storage needs ceil(n/w) < 65535 (P:302)");
  if (out.empty_mode < 0 || out.empty_mode > 2) return fail(YASPMV_EINVAL, "bad empty_mode");
  if (out.rc < 0) out.rc = 0;  // -1 = strategy 1 explicitly (yaspmv_reencode)
  if (out.rc != 0 && out.rc != 1 && out.rc != 2 && out.rc != 4)
    return fail(YASPMV_EINVAL, "result_cache must be 0 (strategy 1) or 1, 2, 4 (x C entries, strategy 2)");
  if (out.tpc < 0 || out.tpc > 64) return fail(YASPMV_EINVAL, "tiles_per_cta must be 0 (auto) or in 1..64");
  (void)m;
  return YASPMV_OK;
}

// ------------------------------------------------------------------------- a2-a4
namespace {

// sorted unique block columns of block row br (merging its h sorted rows)
inline void block_cols_of(const CSR& A, int h, int w, int64_t br, std::vector<int32_t>& out) {
  out.clear();
  const int64_t r0 = br * h, r1 = std::min<int64_t>(A.m, r0 + h);
  if (r1 - r0 == 1) {
    for (int64_t k = A.rp[r0]; k < A.rp[r0 + 1]; ++k) {
      int32_t bc = A.ci[k] / w;
      if (out.empty() || out.back() != bc) out.push_back(bc);
    }
    return;
  }
  int64_t ptr[4], end[4];
  int nr = (int)(r1 - r0);
  for (int q = 0; q < nr; ++q) { ptr[q] = A.rp[r0 + q]; end[q] = A.rp[r0 + q + 1]; }
  while (true) {
    int32_t best = INT32_MAX;
    for (int q = 0; q < nr; ++q)
      if (ptr[q] < end[q]) best = std::min(best, A.ci[ptr[q]] / w);
    if (best == INT32_MAX) break;
    out.push_back(best);
    for (int q = 0; q < nr; ++q)
      while (ptr[q] < end[q] && A.ci[ptr[q]] / w == best) ++ptr[q];
  }
}

}  // namespace

int64_t count_blocks(const CSR& A, int h, int w) {
  const int64_t MB = (A.m + h - 1) / h;
  int64_t total = 0;
#pragma omp parallel reduction(+ : total)
  {
    std::vector<int32_t> bcs;
#pragma omp for schedule(dynamic, 256)
    for (int64_t br = 0; br < MB; ++br) {
      block_cols_of(A, h, w, br, bcs);
      total += (int64_t)bcs.size();
    }
  }
  return total;
}

namespace {

inline void clear_bit(uint8_t* flags, int64_t b) {
  __atomic_fetch_and(&flags[b >> 3], (uint8_t)~(1u << (b & 7)), __ATOMIC_RELAXED);
}

}  // namespace

yaspmv_status encode(const CSR& A, const Params& p, Canonical& out) {
  out = Canonical();
  const int h = p.h, w = p.w, S = p.S, T = p.T, C = p.C, vs = A.vsize;
  const int64_t TC = (int64_t)T * C;
  out.m = A.m;
  out.n = A.n;
  out.nnz = A.nnz;
  out.vsize = vs;
  out.MB = (A.m + h - 1) / h;
  out.NB = (A.n + w - 1) / w;
  out.SW = out.NB > 0 ? (out.NB + S - 1) / S : 1;
  const int64_t MB = out.MB, SW = out.SW, nsr = (int64_t)S * MB;

  // a2 pass 1: blocks per stacked block row sr = s*MB + br
  std::vector<int64_t> cnt(nsr + 1, 0);
#pragma omp parallel
  {
    std::vector<int32_t> bcs;
#pragma omp for schedule(dynamic, 256)
    for (int64_t br = 0; br < MB; ++br) {
      block_cols_of(A, h, w, br, bcs);
      for (int32_t bc : bcs) cnt[(bc / SW) * MB + br]++;
    }
  }
  int64_t n_empty = 0, n_real = 0;
  for (int64_t sr = 0; sr < nsr; ++sr) { n_empty += cnt[sr] == 0; n_real += cnt[sr]; }
  const int s_c = col_bytes(p.col_mode);
  Params rp = p;
  if (rp.empty_mode == 0) {  // Q1: the cheaper of filler blocks (R1) and a seg_row map (R2)
    const int64_t r1 = n_empty * (int64_t)(h * w * vs + s_c);
    const int64_t r2 = 4 * (nsr - n_empty) + 4 * n_empty;
    rp.empty_mode = (n_empty == 0 || r1 <= r2) ? EMPTY_FILLER : EMPTY_MAP;
  }
  out.p = rp;
  const bool filler = rp.empty_mode == EMPTY_FILLER;
  // offsets of every stacked row in the block stream (E3 order: (sr, bc))
  std::vector<int64_t> off(nsr + 1, 0);
  for (int64_t sr = 0; sr < nsr; ++sr) off[sr + 1] = off[sr] + ((filler && cnt[sr] == 0) ? 1 : cnt[sr]);
  out.nnzb = off[nsr];
  out.n_filler = filler ? n_empty : 0;
  out.nnzb_pad = (out.nnzb + TC - 1) / TC * TC;
  out.ntiles = out.nnzb_pad / TC;
  const int64_t NP = out.nnzb_pad;

  // a3: arrays
  try {
    out.flags.assign(NP / 8, 0xFF);  // E6/E7: 1 = continue; pad bits stay 1
    std::vector<int32_t> colb(NP, 0);
    for (int r = 0; r < h; ++r) out.val[r].assign((size_t)NP * w * vs, 0);

    // a2 pass 2: fill columns, values, and clear the stop bit of each stacked row
#pragma omp parallel
    {
      std::vector<int32_t> bcs;
      std::vector<int64_t> pos;
#pragma omp for schedule(dynamic, 256)
      for (int64_t br = 0; br < MB; ++br) {
        block_cols_of(A, h, w, br, bcs);
        pos.resize(bcs.size());
        int64_t k = 0;
        for (int s = 0; s < S; ++s) {
          const int64_t sr = (int64_t)s * MB + br;
          int64_t b = off[sr];
          while (k < (int64_t)bcs.size() && bcs[k] / SW == s) {
            pos[k] = b;
            colb[b] = bcs[k];  // E5: ORIGINAL block column
            ++b;
            ++k;
          }
        }
        for (int r = 0; r < h; ++r) {
          const int64_t i = br * h + r;
          if (i >= A.m) break;
          uint8_t* vdst = out.val[r].data();
          int64_t q = 0;
          for (int64_t e = A.rp[i]; e < A.rp[i + 1]; ++e) {
            const int32_t c = A.ci[e];
            const int32_t bc = c / w;
            while (bcs[q] != bc) ++q;
            std::memcpy(vdst + ((size_t)pos[q] * w + (c % w)) * vs, A.v + (size_t)e * vs, vs);  // E4
          }
        }
        for (int s = 0; s < S; ++s) {
          const int64_t sr = (int64_t)s * MB + br;
          if (off[sr + 1] > off[sr]) clear_bit(out.flags.data(), off[sr + 1] - 1);  // E6
        }
      }
    }
    // R1 fillers take block column NB, past the last one: x reads 0 there (Q4), so an
    // empty row is 0 for every x, +-Inf included; pad blocks repeat the last column (Q3)
    if (filler && n_empty) {
      for (int64_t sr = 0; sr < nsr; ++sr)
        if (cnt[sr] == 0) colb[off[sr]] = (int32_t)out.NB;
    }
    for (int64_t b = out.nnzb; b < NP; ++b) colb[b] = out.nnzb > 0 ? colb[out.nnzb - 1] : 0;

    // E9: column storage
    if (rp.col_mode == COL_U16) {
      out.col16.resize(NP);
#pragma omp parallel for schedule(static)
      for (int64_t b = 0; b < NP; ++b) out.col16[b] = (uint16_t)colb[b];
    } else {
      if (rp.col_mode == COL_DELTA) {
        out.delta.resize(NP);
#pragma omp parallel for schedule(static)
        for (int64_t b = 0; b < NP; ++b) {
          const int64_t base = (b % T == 0) ? 0 : colb[b - 1];  // segmented per thread tile
          const int64_t d = (int64_t)colb[b] - base;
          out.delta[b] = (d < -32768 || d > 32767 || d == -1) ? (int16_t)-1 : (int16_t)d;  // -1 = escape
        }
      }
      out.col32.swap(colb);
    }

    // Q1 R2: stop -> stacked row map and the zero-fill list
    if (!filler && n_empty) {
      out.seg_row.reserve(nsr - n_empty);
      out.zero_rows.reserve(n_empty);
      for (int64_t sr = 0; sr < nsr; ++sr) {
        if (cnt[sr]) out.seg_row.push_back((int32_t)sr);
        else out.zero_rows.push_back((int32_t)sr);
      }
      out.has_seg_row = 1;
      out.n_zero = n_empty;
    }

    // a4: row stops before each workgroup tile
    out.cta_seg0.assign(out.ntiles, 0);
    std::vector<int64_t> per_tile(out.ntiles, 0);
    const int64_t tb = TC / 8;
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < out.ntiles; ++k) {
      int64_t z = 0;
      for (int64_t q = 0; q < tb; ++q) z += 8 - __builtin_popcount(out.flags[k * tb + q]);
      per_tile[k] = z;
    }
    int64_t acc = 0;
    for (int64_t k = 0; k < out.ntiles; ++k) {
      if (acc > INT32_MAX) return fail(YASPMV_EUNSUPPORTED, "more than 2^31 row stops");
      out.cta_seg0[k] = (int32_t)acc;
      acc += per_tile[k];
    }
    out.n_stops = acc;
  } catch (const std::bad_alloc&) {
    out = Canonical();
    return fail(YASPMV_ENOMEM, "host allocation failed while encoding");
  }
  return YASPMV_OK;
}

// ------------------------------------------------------------------------- tuner helper
// The canonical arrays of the same (h, w, S, col mode) for another (T, C): T*C divides the
// base tile, so the arrays are prefixes of the base ones (padding has the same content),
// except the per-thread delta array and the per-tile stop counts, which are recomputed.
yaspmv_status derive_tc(const Canonical& base, int T, int C, Canonical& out) {
  const int64_t TC = (int64_t)T * C, BTC = (int64_t)base.p.T * base.p.C;
  if (BTC % TC != 0) return fail(YASPMV_EINVAL, "derive_tc: tile does not divide the base tile");
  out = Canonical();
  out.m = base.m; out.n = base.n; out.nnz = base.nnz; out.MB = base.MB; out.NB = base.NB; out.SW = base.SW;
  out.nnzb = base.nnzb; out.n_stops = base.n_stops; out.n_filler = base.n_filler; out.n_zero = base.n_zero;
  out.has_seg_row = base.has_seg_row; out.vsize = base.vsize;
  out.p = base.p;
  out.p.T = T;
  out.p.C = C;
  out.nnzb_pad = (out.nnzb + TC - 1) / TC * TC;
  out.ntiles = out.nnzb_pad / TC;
  const int64_t NP = out.nnzb_pad;
  const int w = base.p.w, vs = base.vsize;
  try {
    out.flags.assign(base.flags.begin(), base.flags.begin() + NP / 8);
    if (!base.col16.empty()) out.col16.assign(base.col16.begin(), base.col16.begin() + NP);
    if (!base.col32.empty()) out.col32.assign(base.col32.begin(), base.col32.begin() + NP);
    for (int r = 0; r < base.p.h; ++r) out.val[r].assign(base.val[r].begin(), base.val[r].begin() + (size_t)NP * w * vs);
    out.seg_row = base.seg_row;
    out.zero_rows = base.zero_rows;
    if (base.p.col_mode == COL_DELTA) {
      out.delta.resize(NP);
#pragma omp parallel for schedule(static)
      for (int64_t b = 0; b < NP; ++b) {
        const int64_t prev = (b % T == 0) ? 0 : out.col32[b - 1];
        const int64_t d = (int64_t)out.col32[b] - prev;
        out.delta[b] = (d < -32768 || d > 32767 || d == -1) ? (int16_t)-1 : (int16_t)d;
      }
    }
    out.cta_seg0.assign(out.ntiles, 0);
    int64_t acc = 0;
    const int64_t tb = TC / 8;
    for (int64_t k = 0; k < out.ntiles; ++k) {
      out.cta_seg0[k] = (int32_t)acc;
      for (int64_t q = 0; q < tb; ++q) acc += 8 - __builtin_popcount(out.flags[k * tb + q]);
    }
  } catch (const std::bad_alloc&) {
    out = Canonical();
    return fail(YASPMV_ENOMEM, "host allocation failed in derive_tc");
  }
  return YASPMV_OK;
}

// ------------------------------------------------------------------------- layout
void permute_to_device_layout(const uint8_t* src, uint8_t* dst, int64_t ntiles, int C, int ptb) {
  const int ch = ptb < 16 ? ptb : 16, nch = ptb / ch;
#pragma omp parallel for schedule(static)
  for (int64_t k = 0; k < ntiles; ++k) {
    const uint8_t* s = src + k * (int64_t)C * ptb;
    uint8_t* d = dst + k * (int64_t)C * ptb;
    for (int j = 0; j < nch; ++j)
      for (int t = 0; t < C; ++t) std::memcpy(d + ((int64_t)j * C + t) * ch, s + (int64_t)t * ptb + j * ch, ch);
  }
}

void permute_from_device_layout(const uint8_t* src, uint8_t* dst, int64_t ntiles, int C, int ptb) {
  const int ch = ptb < 16 ? ptb : 16, nch = ptb / ch;
#pragma omp parallel for schedule(static)
  for (int64_t k = 0; k < ntiles; ++k) {
    const uint8_t* s = src + k * (int64_t)C * ptb;
    uint8_t* d = dst + k * (int64_t)C * ptb;
    for (int j = 0; j < nch; ++j)
      for (int t = 0; t < C; ++t) std::memcpy(d + (int64_t)t * ptb + j * ch, s + ((int64_t)j * C + t) * ch, ch);
  }
}

}  // namespace yaspmv
