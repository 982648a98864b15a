// panel.cpp — host encoder of the panel-sliced BCCOO+ part (P1-P6; the
// independent reference is oracle/panel.py).  Panels are independent, so every pass runs
// in parallel over panels (OpenMP); each panel's blocks, flag bytes and bitmap words are
// disjoint ranges.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "common.hpp"
#include "panel.hpp"

namespace yaspmv {

void PanelDev::free_all() {
  void* ps[] = {col16, val, flags, panel_blk0, slice_ptr, stop_ptr, first_row, tile_rank, part, scratch};
  for (void* q : ps)
    if (q) cudaFree(q);
  *this = PanelDev();
}

namespace {
inline int32_t clamp32(int64_t v) { return (int32_t)std::min<int64_t>(std::max<int64_t>(v, INT32_MIN), INT32_MAX); }
}  // namespace

yaspmv_status encode_panel(const CSR& A, const PanelGeom& g0, CSR& far, PanelCanonical& out) {
  PanelGeom g = g0;
  g.KS = (g.R + 2 * g.B + g.W - 1) / g.W;
  g.npanels = (A.m + g.R - 1) / g.R;
  if (g.KS > PANEL_MAX_KS) return fail(YASPMV_EINVAL, "panel: (R + 2B) / W must not exceed 64 slices");
  if (g.W >= 65535) return fail(YASPMV_EINVAL, "panel: slice width must be < 65535 (u16 offsets, W = filler)");
  const int64_t KS = g.KS, NP = g.npanels, R = g.R, W = g.W;
  const int vs = A.vsize;
  out = PanelCanonical();
  out.g = g;

  // P1/P2: a row's band entries are one contiguous run of its (column-sorted) CSR entries
  // [lo, hi): columns in [cb, cb + KS*W); per slice: entries, occupied rows, first/last row
  std::vector<int64_t> band_lo(A.m), band_hi(A.m);
  std::vector<int64_t> pcnt(NP, 0);                      // band entries per panel
  std::vector<int32_t> scnt((size_t)NP * KS, 0);         // entries per (panel, slice)
  std::vector<int32_t> socc((size_t)NP * KS, 0);         // occupied rows per (panel, slice)
  std::vector<int32_t> sfirst((size_t)NP * KS, -1), slast((size_t)NP * KS, -1);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t p = 0; p < NP; ++p) {
    const int64_t cb = p * R + g.col0 - g.B, ce = cb + KS * W;
    const int64_t r1 = std::min(A.m, (p + 1) * R);
    int64_t cnt = 0;
    int32_t* sc = scnt.data() + p * KS;
    int32_t* so = socc.data() + p * KS;
    int32_t* sf = sfirst.data() + p * KS;
    int32_t* sl = slast.data() + p * KS;
    for (int64_t i = p * R; i < r1; ++i) {
      const int32_t* c0 = A.ci + A.rp[i];
      const int32_t* c1 = A.ci + A.rp[i + 1];
      const int32_t* lo = std::lower_bound(c0, c1, clamp32(cb));
      const int32_t* hi = ce > INT32_MAX ? c1 : std::lower_bound(lo, c1, clamp32(ce));
      band_lo[i] = lo - A.ci;
      band_hi[i] = hi - A.ci;
      cnt += hi - lo;
      int64_t kprev = -1;
      for (const int32_t* c = lo; c < hi; ++c) {
        const int64_t k = (*c - cb) / W;
        sc[k]++;
        if (k != kprev) {
          so[k]++;
          if (sf[k] < 0) sf[k] = (int32_t)(i - p * R);
          sl[k] = (int32_t)(i - p * R);
          kprev = k;
        }
      }
    }
    pcnt[p] = cnt;
  }
  // P6 fillers, P4 padding of every slice to a multiple of the workgroup tile
  out.panel_blk0.assign(NP + 1, 0);
  for (int64_t p = 0; p < NP; ++p) {
    int64_t sz = 0;
    for (int64_t k = 0; k < KS; ++k) {
      const int64_t q = p * KS + k;
      const int64_t fill = slast[q] >= 0 ? (int64_t)(slast[q] - sfirst[q] + 1) - socc[q] : 0;
      out.nfill += fill;
      sz += ((int64_t)scnt[q] + fill + PANEL_TC - 1) / PANEL_TC * PANEL_TC;
    }
    out.panel_blk0[p + 1] = out.panel_blk0[p] + sz;
    out.nband += pcnt[p];
  }
  out.nband_pad = out.panel_blk0[NP];
  // far part: the remaining entries of every row, as a CSR of the same shape
  far = CSR();
  far.m = A.m;
  far.n = A.n;
  far.vsize = vs;
  far.rp_own.assign(A.m + 1, 0);
  for (int64_t i = 0; i < A.m; ++i)
    far.rp_own[i + 1] = far.rp_own[i] + (A.rp[i + 1] - A.rp[i]) - (band_hi[i] - band_lo[i]);
  far.nnz = far.rp_own[A.m];
  try {
    far.ci_own.resize(far.nnz);
    far.v_own.resize((size_t)far.nnz * vs);
    out.flags.assign(out.nband_pad / 8, 0xFF);
    out.col16.assign(out.nband_pad, 0);
    out.val.assign((size_t)out.nband_pad * vs, 0);
    out.slice_ptr.assign((size_t)NP * (KS + 1), 0);
    out.stop_ptr.assign((size_t)NP * (KS + 1), 0);
    out.first_row.assign((size_t)NP * KS, 0);
    out.tile_rank.assign(out.nband_pad / PANEL_TC, 0);
  } catch (const std::bad_alloc&) {
    return fail(YASPMV_ENOMEM, "panel encoder: host allocation failed");
  }
  far.adopt_owned();

#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t p = 0; p < NP; ++p) {
    const int64_t cb = p * R + g.col0 - g.B;
    const int64_t r0 = p * R, r1 = std::min(A.m, (p + 1) * R);
    int32_t* sp = out.slice_ptr.data() + p * (KS + 1);
    int32_t* st = out.stop_ptr.data() + p * (KS + 1);
    const int64_t b0 = out.panel_blk0[p];
    std::vector<int64_t> gsz(KS), fillp(KS), lastrow(KS);
    for (int64_t k = 0; k < KS; ++k) {
      const int64_t q = p * KS + k;
      const int64_t nst = slast[q] >= 0 ? slast[q] - sfirst[q] + 1 : 0;
      gsz[k] = scnt[q] + (nst - socc[q]);                                          // entries + fillers
      sp[k + 1] = sp[k] + (int32_t)((gsz[k] + PANEL_TC - 1) / PANEL_TC * PANEL_TC);
      st[k + 1] = st[k] + (int32_t)nst;
      out.first_row[q] = sfirst[q] >= 0 ? sfirst[q] : 0;
      fillp[k] = b0 + sp[k];                                                       // P3 cursor
      lastrow[k] = sfirst[q] >= 0 ? sfirst[q] - 1 : 0;
    }
    auto stop_at = [&](int64_t pos) { out.flags[pos >> 3] &= (uint8_t)~(1u << (pos & 7)); };
    for (int64_t i = r0; i < r1; ++i) {
      const int64_t lr = i - r0;
      // far entries: before and after the band run (column order kept)
      int64_t f = far.rp_own[i];
      for (int64_t e = A.rp[i]; e < band_lo[i]; ++e, ++f) {
        far.ci_own[f] = A.ci[e];
        std::memcpy(&far.v_own[(size_t)f * vs], A.v + (size_t)e * vs, vs);
      }
      for (int64_t e = band_hi[i]; e < A.rp[i + 1]; ++e, ++f) {
        far.ci_own[f] = A.ci[e];
        std::memcpy(&far.v_own[(size_t)f * vs], A.v + (size_t)e * vs, vs);
      }
      // band entries, slice by slice (a slice's entries of one row are consecutive)
      for (int64_t e = band_lo[i]; e < band_hi[i]; ++e) {
        const int64_t rel = (int64_t)A.ci[e] - cb;
        const int64_t k = rel / W;
        if (lastrow[k] < lr) {  // first entry of row i in slice k: fillers for the empty rows before it
          for (int64_t rr = lastrow[k] + 1; rr < lr; ++rr) {
            const int64_t pos = fillp[k]++;
            out.col16[pos] = (uint16_t)W;  // value 0 (zero-initialised), the zero slot of the window
            stop_at(pos);
          }
          lastrow[k] = lr;
        }
        const int64_t pos = fillp[k]++;
        out.col16[pos] = (uint16_t)(rel - k * W);                                   // P5
        std::memcpy(&out.val[(size_t)pos * vs], A.v + (size_t)e * vs, vs);
        if (e + 1 == band_hi[i] || ((int64_t)A.ci[e + 1] - cb) / W != k) stop_at(pos);  // P4: row stop
      }
    }
    // pad entries repeat their slice's last stored column (Q3); stops before every tile
    // inside its slice (the per-tile first-result entry)
    for (int64_t k = 0; k < KS; ++k) {
      if (gsz[k] > 0)
        for (int64_t b = b0 + sp[k] + gsz[k]; b < b0 + sp[k + 1]; ++b) out.col16[b] = out.col16[b0 + sp[k] + gsz[k] - 1];
      int32_t before = 0;
      for (int64_t tt = (b0 + sp[k]) / PANEL_TC; tt < (b0 + sp[k + 1]) / PANEL_TC; ++tt) {
        out.tile_rank[tt] = before;
        int ones = 0;
        for (int q = 0; q < PANEL_TC / 8; ++q) ones += __builtin_popcount(out.flags[tt * (PANEL_TC / 8) + q]);
        before += PANEL_TC - ones;
      }
    }
  }
  for (int64_t p = 0; p < NP; ++p) out.n_stops += out.stop_ptr[p * (KS + 1) + KS];
  return YASPMV_OK;
}

}  // namespace yaspmv
