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
  void* ps[] = {col16, val, flags, panel_blk0, slice_ptr, stop_ptr, first_row, tile_rank, far_col, far_blk0,
                part, scratch};
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
  const int64_t fip = g.fip ? 1 : 0;
  const int64_t KS = g.KS, NS = KS + fip, NP = g.npanels, R = g.R, W = g.W;
  const int vs = A.vsize;
  out = PanelCanonical();
  out.g = g;

  // P1/P2: a row's band entries are one contiguous run of its (column-sorted) CSR entries
  // [lo, hi): columns in [cb, cb + KS*W); per slice (slice fip + k = band slice k, slice 0
  // = the far slice with P7): entries, occupied rows, first/last row
  std::vector<int64_t> band_lo(A.m), band_hi(A.m);
  std::vector<int64_t> pcnt(NP, 0);                      // band entries per panel
  std::vector<int32_t> scnt((size_t)NP * NS, 0);         // entries per (panel, slice)
  std::vector<int32_t> socc((size_t)NP * NS, 0);         // occupied rows per (panel, slice)
  std::vector<int32_t> sfirst((size_t)NP * NS, -1), slast((size_t)NP * NS, -1);
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t p = 0; p < NP; ++p) {
    const int64_t cb = p * R + g.col0 - g.B, ce = cb + KS * W;
    const int64_t r1 = std::min(A.m, (p + 1) * R);
    int64_t cnt = 0;
    int32_t* sc = scnt.data() + p * NS;
    int32_t* so = socc.data() + p * NS;
    int32_t* sf = sfirst.data() + p * NS;
    int32_t* sl = slast.data() + p * NS;
    for (int64_t i = p * R; i < r1; ++i) {
      const int32_t* c0 = A.ci + A.rp[i];
      const int32_t* c1 = A.ci + A.rp[i + 1];
      const int32_t* lo = std::lower_bound(c0, c1, clamp32(cb));
      const int32_t* hi = ce > INT32_MAX ? c1 : std::lower_bound(lo, c1, clamp32(ce));
      band_lo[i] = lo - A.ci;
      band_hi[i] = hi - A.ci;
      cnt += hi - lo;
      const int32_t lr = (int32_t)(i - p * R);
      if (fip && (c1 - c0) > (hi - lo)) {  // P7: the row's far entries, slice 0
        sc[0] += (int32_t)((c1 - c0) - (hi - lo));
        so[0]++;
        if (sf[0] < 0) sf[0] = lr;
        sl[0] = lr;
      }
      int64_t kprev = -1;
      for (const int32_t* c = lo; c < hi; ++c) {
        const int64_t k = (*c - cb) / W + fip;
        sc[k]++;
        if (k != kprev) {
          so[k]++;
          if (sf[k] < 0) sf[k] = lr;
          sl[k] = lr;
          kprev = k;
        }
      }
    }
    pcnt[p] = cnt;
  }
  // P6 fillers, P4 padding of every slice to a multiple of the workgroup tile
  auto padded = [&](int64_t q) {
    const int64_t fill = slast[q] >= 0 ? (int64_t)(slast[q] - sfirst[q] + 1) - socc[q] : 0;
    return ((int64_t)scnt[q] + fill + PANEL_TC - 1) / PANEL_TC * PANEL_TC;
  };
  out.panel_blk0.assign(NP + 1, 0);
  if (fip) out.far_blk0.assign(NP + 1, 0);
  for (int64_t p = 0; p < NP; ++p) {
    int64_t sz = 0;
    for (int64_t k = 0; k < NS; ++k) {
      const int64_t q = p * NS + k;
      out.nfill += slast[q] >= 0 ? (int64_t)(slast[q] - sfirst[q] + 1) - socc[q] : 0;
      sz += padded(q);
    }
    out.panel_blk0[p + 1] = out.panel_blk0[p] + sz;
    if (fip) out.far_blk0[p + 1] = out.far_blk0[p] + padded(p * NS);
    out.nband += pcnt[p];
  }
  out.nband_pad = out.panel_blk0[NP];
  out.nfar_pad = fip ? out.far_blk0[NP] : 0;
  // far part: the remaining entries of every row, as a CSR of the same shape (P7: none)
  far = CSR();
  far.m = A.m;
  far.n = A.n;
  far.vsize = vs;
  far.rp_own.assign(A.m + 1, 0);
  if (!fip)
    for (int64_t i = 0; i < A.m; ++i)
      far.rp_own[i + 1] = far.rp_own[i] + (A.rp[i + 1] - A.rp[i]) - (band_hi[i] - band_lo[i]);
  far.nnz = far.rp_own[A.m];
  try {
    far.ci_own.resize(far.nnz);
    far.v_own.resize((size_t)far.nnz * vs);
    out.flags.assign(out.nband_pad / 8, 0xFF);
    out.col16.assign(out.nband_pad - out.nfar_pad, 0);
    out.far_col.assign(out.nfar_pad, 0);
    out.val.assign((size_t)out.nband_pad * vs, 0);
    out.slice_ptr.assign((size_t)NP * (NS + 1), 0);
    out.stop_ptr.assign((size_t)NP * (NS + 1), 0);
    out.first_row.assign((size_t)NP * NS, 0);
    out.tile_rank.assign(out.nband_pad / PANEL_TC, 0);
  } catch (const std::bad_alloc&) {
    return fail(YASPMV_ENOMEM, "panel encoder: host allocation failed");
  }
  far.adopt_owned();

#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t p = 0; p < NP; ++p) {
    const int64_t cb = p * R + g.col0 - g.B;
    const int64_t r0 = p * R, r1 = std::min(A.m, (p + 1) * R);
    int32_t* sp = out.slice_ptr.data() + p * (NS + 1);
    int32_t* st = out.stop_ptr.data() + p * (NS + 1);
    const int64_t b0 = out.panel_blk0[p];
    // stored column of unified block pos: col16 holds the band blocks, far_col the far ones
    const int64_t c16_0 = fip ? out.far_blk0[p + 1] : 0;           // far blocks up to panel p
    const int64_t fc_0 = fip ? b0 - out.far_blk0[p] : 0;            // band blocks before panel p
    std::vector<int64_t> gsz(NS), fillp(NS), lastrow(NS);
    for (int64_t k = 0; k < NS; ++k) {
      const int64_t q = p * NS + k;
      const int64_t nst = slast[q] >= 0 ? slast[q] - sfirst[q] + 1 : 0;
      gsz[k] = scnt[q] + (nst - socc[q]);                                          // entries + fillers
      sp[k + 1] = sp[k] + (int32_t)((gsz[k] + PANEL_TC - 1) / PANEL_TC * PANEL_TC);
      st[k + 1] = st[k] + (int32_t)nst;
      out.first_row[q] = sfirst[q] >= 0 ? sfirst[q] : 0;
      fillp[k] = b0 + sp[k];                                                       // P3 cursor
      lastrow[k] = sfirst[q] >= 0 ? sfirst[q] - 1 : 0;
    }
    auto stop_at = [&](int64_t pos) { out.flags[pos >> 3] &= (uint8_t)~(1u << (pos & 7)); };
    auto put = [&](int64_t k, int64_t col, const void* v) {  // next block of slice k
      const int64_t pos = fillp[k]++;
      if (k < fip) out.far_col[pos - fc_0] = (int32_t)col;
      else out.col16[pos - c16_0] = (uint16_t)col;
      if (v) std::memcpy(&out.val[(size_t)pos * vs], v, vs);
      return pos;
    };
    auto fill_to = [&](int64_t k, int64_t lr) {  // fillers for the empty rows before row lr of slice k
      if (lastrow[k] < lr) {
        for (int64_t rr = lastrow[k] + 1; rr < lr; ++rr) stop_at(put(k, k < fip ? A.n : W, nullptr));
        lastrow[k] = lr;
      }
    };
    for (int64_t i = r0; i < r1; ++i) {
      const int64_t lr = i - r0;
      if (fip) {  // P7: the far entries, before and after the band run (column order kept)
        const int64_t nf = (A.rp[i + 1] - A.rp[i]) - (band_hi[i] - band_lo[i]);
        if (nf > 0) {
          fill_to(0, lr);
          int64_t left = nf;
          for (int64_t e = A.rp[i]; e < band_lo[i]; ++e)
            if (const int64_t pos = put(0, A.ci[e], A.v + (size_t)e * vs); --left == 0) stop_at(pos);
          for (int64_t e = band_hi[i]; e < A.rp[i + 1]; ++e)
            if (const int64_t pos = put(0, A.ci[e], A.v + (size_t)e * vs); --left == 0) stop_at(pos);
        }
      } else {  // far entries: before and after the band run (column order kept)
        int64_t f = far.rp_own[i];
        for (int64_t e = A.rp[i]; e < band_lo[i]; ++e, ++f) {
          far.ci_own[f] = A.ci[e];
          std::memcpy(&far.v_own[(size_t)f * vs], A.v + (size_t)e * vs, vs);
        }
        for (int64_t e = band_hi[i]; e < A.rp[i + 1]; ++e, ++f) {
          far.ci_own[f] = A.ci[e];
          std::memcpy(&far.v_own[(size_t)f * vs], A.v + (size_t)e * vs, vs);
        }
      }
      // band entries, slice by slice (a slice's entries of one row are consecutive)
      for (int64_t e = band_lo[i]; e < band_hi[i]; ++e) {
        const int64_t rel = (int64_t)A.ci[e] - cb;
        const int64_t kb = rel / W, k = kb + fip;
        fill_to(k, lr);
        const int64_t pos = put(k, rel - kb * W, A.v + (size_t)e * vs);              // P5
        if (e + 1 == band_hi[i] || ((int64_t)A.ci[e + 1] - cb) / W != kb) stop_at(pos);  // P4: row stop
      }
    }
    // pad entries repeat their slice's last stored column (Q3); stops before every tile
    // inside its slice (the per-tile first-result entry)
    for (int64_t k = 0; k < NS; ++k) {
      if (gsz[k] > 0) {
        const int64_t lastp = b0 + sp[k] + gsz[k] - 1;
        for (int64_t b = lastp + 1; b < b0 + sp[k + 1]; ++b) {
          if (k < fip) out.far_col[b - fc_0] = out.far_col[lastp - fc_0];
          else out.col16[b - c16_0] = out.col16[lastp - c16_0];
        }
      }
      int32_t before = 0;
      for (int64_t tt = (b0 + sp[k]) / PANEL_TC; tt < (b0 + sp[k + 1]) / PANEL_TC; ++tt) {
        out.tile_rank[tt] = before;
        int ones = 0;
        for (int q = 0; q < PANEL_TC / 8; ++q) ones += __builtin_popcount(out.flags[tt * (PANEL_TC / 8) + q]);
        before += PANEL_TC - ones;
      }
    }
  }
  for (int64_t p = 0; p < NP; ++p) out.n_stops += out.stop_ptr[p * (NS + 1) + NS];
  return YASPMV_OK;
}

}  // namespace yaspmv
