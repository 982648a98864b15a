// common.hpp — internal declarations shared by the encoder, kernels, tuner and C ABI.
// Nothing here crosses the ABI (include/yaspmv.h is the boundary).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "../../include/yaspmv.h"

namespace yaspmv {

enum ColMode { COL_U16 = 1, COL_I32 = 2, COL_DELTA = 3 };
enum EmptyMode { EMPTY_FILLER = 1, EMPTY_MAP = 2 };
// ablation switches (Fig. 14); never set by yaspmv_spmv
enum Ablate {
  ABL_DEFER_CARRY = 1,
  ABL_NO_SKIP = 2,
  // roofline probes (not steps of the method): the tile's loads exactly as K1 issues them,
  // then only a per-thread sum kept live; GATHER_ONLY keeps the x gathers, STREAM_ONLY
  // redirects them to x[col & 15] (L1 hits) so only the format stream remains
  ABL_GATHER_ONLY = 4,
  ABL_STREAM_ONLY = 8,
  ABL_GATHER_L2 = 16,  // with GATHER_ONLY: gathers of x[col & (2^20-1)] (4-8 MB: L2 hits, L1 misses)
  ABL_STOP_SCAN = 32,  // probe: return right after the CTA scan (no publish, stores, carries)
  ABL_NO_FIXUP = 64,  // host side, with DEFER_CARRY: no carry kernel ("no carries" probe)
  ABL_NO_YSTORE = 256,  // probe: y stores of the FILLER write-back skipped
  // with STOP_SCAN: after the scan, thread C-1 stores the tile's status word (PUB) / every
  // thread stores one value, coalesced (ST) — the cost of a CTA ending in stores
  ABL_PROBE_PUB = 512,
  ABL_PROBE_ST = 1024,
  // testing the debug spin bound: tile 0 never publishes its carry-out, so a look-back
  // that reaches it polls forever (until YASPMV_SPIN_LIMIT traps)
  ABL_NO_PUBLISH0 = 2048
};

struct Params {
  int h = 1, w = 1, S = 1, T = 16, C = 256, col_mode = 0, empty_mode = 0, flags = 0;
  int rc = 0;  // result cache size in units of C: 0 = strategy 1, k > 0 = strategy 2 (Table 1)
  int tpc = 0;  // tiles per CTA (0 = auto)
  // panel-sliced BCCOO+ (panel.hpp): band half-width (0 = plain format), panel rows,
  // slice width, column of row 0
  int band = 0, pR = 0, pW = 0, col0 = 0;
  int bfar = 0;  // YASPMV_FAR_SEPARATE / YASPMV_FAR_IN_PANEL (0: resolved by resolve_band)
};

inline int col_bytes(int mode) { return mode == COL_I32 ? 4 : 2; }

// Normalised CSR (sorted, distinct columns per row).  Either owns its arrays or views
// the caller's (when the input already is normalised).
struct CSR {
  int64_t m = 0, n = 0, nnz = 0;
  int vsize = 4;
  const int64_t* rp = nullptr;
  const int32_t* ci = nullptr;
  const uint8_t* v = nullptr;
  std::vector<int64_t> rp_own;
  std::vector<int32_t> ci_own;
  std::vector<uint8_t> v_own;
  void adopt_owned() {
    rp = rp_own.data();
    ci = ci_own.data();
    v = v_own.data();
  }
  void make_owned();  // copy a view into owned storage
  bool owned() const { return rp == rp_own.data() && !rp_own.empty(); }
};

// Canonical BCCOO / BCCOO+ arrays, host side.
struct Canonical {
  int64_t m = 0, n = 0, nnz = 0, MB = 0, NB = 0, SW = 1;
  int64_t nnzb = 0, nnzb_pad = 0, ntiles = 0, n_stops = 0, n_filler = 0;
  int64_t n_zero = 0;   // zero-filled stacked rows (EMPTY_MAP)
  int has_seg_row = 0;  // seg_row map present (EMPTY_MAP with empty rows)
  Params p;
  int vsize = 4;
  std::vector<uint8_t> flags;     // nnzb_pad/8, LSB-first, 0 = row stop
  std::vector<uint16_t> col16;    // COL_U16
  std::vector<int32_t> col32;     // COL_I32, or the escape array of COL_DELTA
  std::vector<int16_t> delta;     // COL_DELTA
  std::vector<uint8_t> val[4];    // h arrays of nnzb_pad*w values (raw bytes)
  std::vector<int32_t> seg_row;   // EMPTY_MAP with empty rows
  std::vector<int32_t> zero_rows; // EMPTY_MAP with empty rows
  std::vector<int32_t> cta_seg0;  // ntiles
  void release_arrays();
};

// encoded arrays resident on the device, in the device layout (encode_gpu.cu)
struct GpuArrays {
  void* val[4] = {nullptr, nullptr, nullptr, nullptr};
  void* col = nullptr;
  int32_t* col32 = nullptr;
  uint8_t* flags = nullptr;
  int32_t* cta_seg0 = nullptr;
  int32_t* seg_row = nullptr;
  int32_t* zero_rows = nullptr;
  void free_all();
};

// status helpers ------------------------------------------------------------------
void set_error(const std::string& msg);
yaspmv_status fail(yaspmv_status st, const std::string& msg);
long long debug_spin_limit();   // YASPMV_SPIN_LIMIT (0 = unbounded look-back polling)
long long* debug_spin_slot();   // mapped host slot for the trapped tile id (nullable)

// encoder (encode.cpp) ---------------------------------------------------------------
yaspmv_status normalize_csr(int64_t m, int64_t n, const int64_t* rp, const int32_t* ci, const void* v,
                            int vsize, CSR& out);
yaspmv_status normalize_coo(int64_t m, int64_t n, int64_t nnz, const int32_t* ri, const int32_t* ci,
                            const void* v, int vsize, CSR& out);
yaspmv_status resolve_params(const Params& in, int64_t m, int64_t n, Params& out);
yaspmv_status encode(const CSR& A, const Params& p, Canonical& out);
yaspmv_status derive_tc(const Canonical& base, int T, int C, Canonical& out);
// GPU translation: A is the normalised host CSR, p resolved (empty_mode may be 0)
yaspmv_status encode_gpu(const CSR& A, const Params& p, Canonical& meta, GpuArrays& out, int64_t& n_escapes,
                         void* stream);
// device layout: per workgroup tile, the per-thread byte runs (ptb bytes each) are
// transposed into chunks of min(16, ptb) bytes so that chunk j of thread t lives at
// (tile*C*nch + j*C + t) — the offline transpose of PAPER.md P:269-273.
void permute_to_device_layout(const uint8_t* src, uint8_t* dst, int64_t ntiles, int C, int ptb);
void permute_from_device_layout(const uint8_t* src, uint8_t* dst, int64_t ntiles, int C, int ptb);
int64_t footprint_bytes(int64_t nnzb, int h, int w, int vsize, int s_c);
int64_t count_blocks(const CSR& A, int h, int w);  // h x w blocks holding >= 1 entry (S = 1)

// kernels (spmv_kernel.cuh / inst_*.cu / kernels_aux.cu) -----------------------------
struct KArgs {
  const void* val[4];
  const void* col;         // device layout: u16 / i32 block columns or int16 deltas
  const int32_t* col32;    // canonical int32 columns (escape path of COL_DELTA)
  const uint8_t* flags;    // canonical packed bit flags
  const int32_t* cta_seg0; // row stops before each tile
  const int32_t* seg_row;  // nullable: stop -> stacked block row
  const int32_t* zero_rows;
  int64_t n_zero;
  const void* x;
  void* out;               // y (S == 1) or the BCCOO+ partial buffer tmp[S*MB*h]
  int64_t out_limit;       // valid output elements
  int64_t n;               // columns of A (x length)
  int64_t ntiles;
  int64_t period;          // tickets per launch = ntiles + grid (persistent CTAs)
  unsigned long long* ticket;
  // per tile, 16 B: [0] status word (epoch << 2 | state), [1] (h = 1) the carry-out as fp64
  // bits, written together by one 128-bit store and read by one 128-bit load, so no fence
  // orders value and status; h > 1 keeps the carries in `carry` (release/relaxed pair)
  unsigned long long* status;
  double* carry;           // ntiles * h
  // non-blocking carries: bnd[2k..2k+1] is the 16-byte hand-off word between tile k-1 and
  // tile k (epoch-tagged; whichever of the two arrives second completes tile k's carried
  // segment).  h = 1: the pending partial and its row travel inside the word (one 128-bit
  // atomic exchange per side, no fence); h > 1: in pend_val[k*h..] / pend_row[k], ordered
  // by acquire-release exchanges
  unsigned long long* bnd;
  double* pend_val;
  long long* pend_row;
  int force_handoff;       // YASPMV_FORCE_HANDOFF (tests): never take the ready-predecessor fast path
  // power-iteration epilogue (yaspmv_spmv_power): bit 0 scale y by 1/sqrt(*in_norm2),
  // bit 1 write per-warp partials of sum y^2 to part[tile*(C/32+1) + warp] (+ carried seg)
  int epi;
  const double* in_norm2;
  double* part;
  int ablate;              // Ablate bits (0 in production)
  int block_ids;           // 1: tile = blockIdx (in-order dispatch), ticket only for the epoch
  int pdl;                 // launched with programmatic dependent launch
  int64_t* dep_row;        // ABL_DEFER_CARRY: per tile, row of the carried segment or -1
  // fused exchange (yaspmv_power_step_fused, EPI instances only): npeer > 0 writes every
  // output element to peer_out[q][i] for q < npeer (every rank's copy of the next x,
  // pre-offset to this rank's chunk) instead of out[i]
  int npeer;
  void* peer_out[YASPMV_MAX_RANKS];
  int peer_mc;             // 1: peer_out[0] is a multicast address (npeer = 1, multimem.st)
  int rcache;              // strategy 2: result cache entries (rc * C); 0 for strategy 1
  int tpc;                 // consecutive tiles per workgroup (block-id mode); grid = ceil(ntiles / tpc)
  // debug spin bound: > 0 = a look-back that polls more than spin_limit times
  // writes the waiting tile id to *spin_tile (mapped host memory) and traps
  long long spin_limit;
  long long* spin_tile;
  // strategy 1, h = 1, no seg_row map: each warp stages its finished row sums in its slice of
  // C*T values of dynamic shared memory and writes them as one contiguous run (the rows of a
  // warp's stops are consecutive) instead of one scattered 4-byte store per row
  int wstage;
};

// destinations of a fused exchange (combine kernel of BCCOO+, S > 1); mc = 1: p[0] is an
// NVSwitch multicast address (n = 1) — one multimem.st reaches every rank's buffer
struct PeerOut {
  int n = 0;
  int mc = 0;
  void* p[YASPMV_MAX_RANKS] = {};
};

#ifdef __CUDACC__
// one store through a multicast mapping (multimem.st, sm_90+): the switch writes it into
// every bound buffer
template <typename VT>
__device__ __forceinline__ void multimem_store(VT* p, VT v) {
  if constexpr (sizeof(VT) == 4)
    asm volatile("multimem.st.relaxed.sys.global.f32 [%0], %1;" ::"l"(p), "f"((float)v) : "memory");
  else
    asm volatile("multimem.st.relaxed.sys.global.f64 [%0], %1;" ::"l"(p), "d"((double)v) : "memory");
}
#endif

typedef void (*LaunchFn)(const KArgs& a, int C, int64_t grid, void* stream);
typedef int (*AttrFn)(int C, int rc, int* regs, int* max_threads, int* blocks_per_sm);

struct KernelEntry {
  int dtype, h, w, T, cm;
  int strat;  // segmented-sum strategy (P:267 / P:274): 1 registers, 2 result cache
  LaunchFn launch;
  AttrFn attr;
};

const KernelEntry* find_kernel(int dtype, int h, int w, int T, int cm, int strat = 1);
const std::vector<KernelEntry>& all_kernels();

void launch_mc_zero(void* p, int64_t n, int dtype, void* stream);
void launch_combine(const void* tmp, void* y, int64_t m, int64_t stride, int S, int dtype, void* stream,
                    const double* in_norm2 = nullptr, double* part = nullptr, const PeerOut* peers = nullptr);
int64_t combine_blocks(int64_t m);
void launch_sum_f64(const double* v, int64_t n, double* out, double* partials, void* stream);
// sstride: u64 words per tile in `status` (2 for a matrix's status words, 1 for the tree
// ablation's scratch)
void launch_carry_fixup(const unsigned long long* status, const double* carry, const int64_t* dep_row,
                        int64_t ntiles, void* y, int dtype, void* stream, int sstride = 1);
int launch_tree_segsum(const int32_t* rows, const uint8_t* flags, const int32_t* tile_seg0, const int32_t* col,
                       const void* val, int64_t n_elem, const void* x, void* y, int64_t m, int dtype,
                       unsigned long long* status, double* carry, int64_t* dep_row, void* stream);
void launch_nrm2sq(const void* v, int64_t n, int dtype, double* out, double* partials, void* stream);
int64_t nrm2sq_blocks(int64_t n);
void launch_scale(const void* src, void* dst, int64_t n, int dtype, const double* norm2, void* stream);

}  // namespace yaspmv
