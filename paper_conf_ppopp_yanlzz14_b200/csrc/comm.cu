// comm.cu — the fused multi-GPU power step: SpMV write-back straight into every rank's copy
// of the replicated x over peer memory, plus the signal-pad protocol that replaces the
// NCCL all-reduce + all-gather of the unfused loop (include/yaspmv.h "fused multi-GPU
// power step"; not in the paper, which is single-GPU).
//
// One device allocation per rank (so one cudaIpcMemHandle maps all of it on a peer):
//   [ xbuf0 : n_pad*vsize | xbuf1 : n_pad*vsize | signal pad ]
// signal pad (written by the peers):
//   uint64 flag[MAX]          flag[q] = number of steps rank q has completed (epoch)
//   double norm[2][MAX]       norm[k%2][q] = ||z_k restricted to rank q's rows||^2
// Step k on rank r: (k > begin) wait until flag[q] >= k for all q, total = sum_q norm[(k-1)%2][q]
// (rank order, fp64: identical on every rank) -> SpMV with the 1/sqrt(total) epilogue and
// peer stores into xbuf[(k+1)%2] of every rank -> ||z_k||^2 of the rank's rows -> publish
// kernel: norm + flag = k+1 into every peer's pad, system-scope release after a
// system-scope fence (the SpMV's peer stores precede it in stream order).
#include <cuda.h>
#include <cuda_runtime.h>
#include <sys/syscall.h>
#include <cerrno>
#include <unistd.h>

#include <algorithm>
#include <cstring>
#include <string>

#include "handle.hpp"
#include "trace.hpp"

using namespace yaspmv;

#define CUDA_TRY(expr)                                                                       \
  do {                                                                                       \
    cudaError_t _e = (expr);                                                                 \
    if (_e != cudaSuccess)                                                                   \
      return fail(_e == cudaErrorMemoryAllocation ? YASPMV_ENOMEM : YASPMV_ECUDA,            \
                  std::string(#expr) + ": " + cudaGetErrorString(_e));                       \
  } while (0)

namespace {
constexpr int MAXR = YASPMV_MAX_RANKS;
constexpr size_t SIG_FLAG_OFF = 0;
constexpr size_t SIG_NORM_OFF = 8 * MAXR;
constexpr size_t SIG_BYTES = 8 * MAXR + 16 * MAXR;

size_t round_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

struct PeerSig {
  int n = 0;
  char* p[MAXR] = {};
};

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Posts this rank's ||z_k||^2 partial and its completed-step count into every rank's pad.
__global__ void publish_kernel(PeerSig ps, int rank, unsigned long long epoch, int parity,
                               const double* __restrict__ norm_local) {
  const int q = threadIdx.x;
  if (q >= ps.n) return;
  const double nv = norm_local[0];
  double* ns = reinterpret_cast<double*>(ps.p[q] + SIG_NORM_OFF) + parity * MAXR + rank;
  *reinterpret_cast<volatile double*>(ns) = nv;
  __threadfence_system();  // the SpMV's peer stores (earlier in stream order) and the norm
  st_release_sys(reinterpret_cast<unsigned long long*>(ps.p[q] + SIG_FLAG_OFF) + rank, epoch);
}

// One thread polls every rank's flag in this rank's pad (acquire, system scope) until it
// reaches `target`, then sums the norm partials in rank order.  Bounded by timeout_ns: a
// lost peer sets *err and the kernel returns instead of hanging the GPU.
__global__ void wait_kernel(const char* __restrict__ sig, int world, unsigned long long target, int parity,
                            double* __restrict__ total, int* __restrict__ err, unsigned long long timeout_ns) {
  if (threadIdx.x != 0) return;
  const unsigned long long* flag = reinterpret_cast<const unsigned long long*>(sig + SIG_FLAG_OFF);
  const unsigned long long t0 = globaltimer_ns();
  bool ok = true;
  for (int q = 0; q < world && ok; ++q) {
    while (ld_acquire_sys(flag + q) < target) {
      if (globaltimer_ns() - t0 > timeout_ns) {
        ok = false;
        break;
      }
      __nanosleep(256);
    }
  }
  if (!ok) {
    atomicExch(err, 1);
    total[0] = __longlong_as_double(0x7ff8000000000000ll);  // NaN: the step's result is invalid
    return;
  }
  const volatile double* norm = reinterpret_cast<const volatile double*>(sig + SIG_NORM_OFF) + parity * MAXR;
  double s = 0.0;
  for (int q = 0; q < world; ++q) s += norm[q];
  total[0] = s;
}
}  // namespace

namespace {
// CUDA driver entry points of the multicast path, resolved at run time through the runtime
// (no link-time libcuda dependency)
struct Drv {
  bool ok = false;
  CUresult (*devattr)(int*, CUdevice_attribute, CUdevice) = nullptr;
  CUresult (*devget)(CUdevice*, int) = nullptr;
  CUresult (*mc_gran)(size_t*, const CUmulticastObjectProp*, CUmulticastGranularity_flags) = nullptr;
  CUresult (*mc_create)(CUmemGenericAllocationHandle*, const CUmulticastObjectProp*) = nullptr;
  CUresult (*mc_add)(CUmemGenericAllocationHandle, CUdevice) = nullptr;
  CUresult (*mc_bind)(CUmemGenericAllocationHandle, size_t, CUmemGenericAllocationHandle, size_t, size_t,
                      unsigned long long) = nullptr;
  CUresult (*mc_unbind)(CUmemGenericAllocationHandle, CUdevice, size_t, size_t) = nullptr;
  CUresult (*mem_gran)(size_t*, const CUmemAllocationProp*, CUmemAllocationGranularity_flags) = nullptr;
  CUresult (*mem_create)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*,
                         unsigned long long) = nullptr;
  CUresult (*mem_release)(CUmemGenericAllocationHandle) = nullptr;
  CUresult (*addr_reserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long) = nullptr;
  CUresult (*addr_free)(CUdeviceptr, size_t) = nullptr;
  CUresult (*mem_map)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long) = nullptr;
  CUresult (*mem_unmap)(CUdeviceptr, size_t) = nullptr;
  CUresult (*set_access)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t) = nullptr;
  CUresult (*export_h)(void*, CUmemGenericAllocationHandle, CUmemAllocationHandleType, unsigned long long) = nullptr;
  CUresult (*import_h)(CUmemGenericAllocationHandle*, void*, CUmemAllocationHandleType) = nullptr;
};
template <typename F>
bool entry(const char* name, F& f) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess ||
      !p)
    return false;
  f = reinterpret_cast<F>(p);
  return true;
}
const Drv& drv() {
  static Drv d = [] {
    Drv x;
    x.ok = entry("cuDeviceGetAttribute", x.devattr) && entry("cuDeviceGet", x.devget) &&
           entry("cuMulticastGetGranularity", x.mc_gran) && entry("cuMulticastCreate", x.mc_create) &&
           entry("cuMulticastAddDevice", x.mc_add) && entry("cuMulticastBindMem", x.mc_bind) &&
           entry("cuMulticastUnbind", x.mc_unbind) && entry("cuMemGetAllocationGranularity", x.mem_gran) &&
           entry("cuMemCreate", x.mem_create) && entry("cuMemRelease", x.mem_release) &&
           entry("cuMemAddressReserve", x.addr_reserve) && entry("cuMemAddressFree", x.addr_free) &&
           entry("cuMemMap", x.mem_map) && entry("cuMemUnmap", x.mem_unmap) && entry("cuMemSetAccess", x.set_access) &&
           entry("cuMemExportToShareableHandle", x.export_h) &&
           entry("cuMemImportFromShareableHandle", x.import_h);
    return x;
  }();
  return d;
}
}  // namespace

#define CU_TRY(expr)                                                                         \
  do {                                                                                       \
    CUresult _r = (expr);                                                                    \
    if (_r != CUDA_SUCCESS) return fail(YASPMV_ECUDA, std::string(#expr) + ": CUresult " + std::to_string((int)_r)); \
  } while (0)

struct yaspmv_comm_s {
  int device = -1, rank = 0, world = 1, dtype = 0, vsize = 4;
  int64_t chunk = 0, n_pad = 0;
  unsigned long long timeout_ns = 0;
  char* base = nullptr;  // own allocation: xbuf0 | xbuf1 | signal pad
  size_t xbytes = 0;     // one x buffer, rounded to 256 B
  size_t total = 0;
  char* peer[MAXR] = {};   // base of every rank's allocation as mapped here (peer[rank] = base)
  bool ipc[MAXR] = {};     // opened with cudaIpcOpenMemHandle (closed on free)
  bool connected = false;
  int64_t seq = 0;         // steps issued on this comm
  bool fresh = true;       // the next step reads x_0 unscaled and does not wait
  double* d_norm_local = nullptr;  // [0] this rank's ||z||^2, [1] the total, [2..] reduction scratch
  int* d_err = nullptr;
  int64_t scratch_n = 0;
  double* d_scratch = nullptr;
  // NVSwitch multicast (yaspmv_comm_mc_*): the two x buffers live in a VMM allocation bound
  // to a multicast object of all ranks; the SpMV stores z through the multicast mapping
  bool mc = false;                         // bound: steps use mc_va / loc_va
  bool mc_have = false, mc_added = false, mem_have = false;
  CUmemGenericAllocationHandle mc_h = 0, mem_h = 0;
  size_t mc_size = 0;
  CUdeviceptr mc_va = 0, loc_va = 0;
  int mc_fd = -1;
  ~yaspmv_comm_s() {
    if (device < 0) return;
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(device);
    if (mc_have || mem_have) {
      cudaDeviceSynchronize();
      const Drv& d = drv();
      CUdevice dev = 0;
      d.devget(&dev, device);
      if (mc_va) { d.mem_unmap(mc_va, mc_size); d.addr_free(mc_va, mc_size); }
      if (loc_va) { d.mem_unmap(loc_va, mc_size); d.addr_free(loc_va, mc_size); }
      if (mc && mc_have) d.mc_unbind(mc_h, dev, 0, mc_size);
      if (mem_have) d.mem_release(mem_h);
      if (mc_have) d.mem_release(mc_h);
    }
    if (mc_fd >= 0) close(mc_fd);
    for (int q = 0; q < MAXR; ++q)
      if (ipc[q] && peer[q]) cudaIpcCloseMemHandle(peer[q]);
    if (base) cudaFree(base);
    if (d_norm_local) cudaFree(d_norm_local);
    if (d_err) cudaFree(d_err);
    if (d_scratch) cudaFree(d_scratch);
    cudaSetDevice(cur);
  }
  char* xbuf(const char* b, int64_t k) const { return const_cast<char*>(b) + (size_t)(k & 1) * xbytes; }
  char* xown() const { return mc ? reinterpret_cast<char*>(loc_va) : base; }  // this rank's x buffers
  char* sig(const char* b) const { return const_cast<char*>(b) + 2 * xbytes; }
};

extern "C" {

yaspmv_status yaspmv_comm_create(int32_t device, int32_t rank, int32_t world, int64_t chunk, yaspmv_dtype dtype,
                                 int32_t timeout_ms, yaspmv_comm* out) {
  if (!out) return fail(YASPMV_EINVAL, "out is NULL");
  *out = nullptr;
  if (world < 1 || world > MAXR) return fail(YASPMV_EINVAL, "world must be in [1, YASPMV_MAX_RANKS]");
  if (rank < 0 || rank >= world) return fail(YASPMV_EINVAL, "rank out of range");
  if (chunk < 0) return fail(YASPMV_EINVAL, "chunk < 0");
  if (dtype != YASPMV_F32 && dtype != YASPMV_F64) return fail(YASPMV_EINVAL, "bad dtype");
  if (device < 0) return fail(YASPMV_EINVAL, "a comm needs a CUDA device (no CPU fallback)");
  int ndev = 0;
  CUDA_TRY(cudaGetDeviceCount(&ndev));
  if (device >= ndev) return fail(YASPMV_EINVAL, "device ordinal out of range");
  CUDA_TRY(cudaSetDevice(device));
  auto* c = new yaspmv_comm_s();
  c->device = device;
  c->rank = rank;
  c->world = world;
  c->dtype = dtype;
  c->vsize = dtype == YASPMV_F32 ? 4 : 8;
  c->chunk = chunk;
  c->n_pad = chunk * world;
  c->timeout_ns = (unsigned long long)(timeout_ms > 0 ? timeout_ms : 60000) * 1000000ull;
  c->xbytes = round_up(std::max<size_t>((size_t)c->n_pad * c->vsize, 16), 256);
  c->total = 2 * c->xbytes + SIG_BYTES;
  cudaError_t e = cudaMalloc((void**)&c->base, c->total);
  if (e == cudaSuccess) e = cudaMemset(c->base, 0, c->total);  // x pads, flags = 0 (no step done)
  if (e == cudaSuccess) e = cudaMalloc((void**)&c->d_norm_local, 2 * sizeof(double));
  if (e == cudaSuccess) e = cudaMemset(c->d_norm_local, 0, 2 * sizeof(double));
  if (e == cudaSuccess) e = cudaMalloc((void**)&c->d_err, sizeof(int));
  if (e == cudaSuccess) e = cudaMemset(c->d_err, 0, sizeof(int));
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  if (e != cudaSuccess) {
    delete c;
    return fail(e == cudaErrorMemoryAllocation ? YASPMV_ENOMEM : YASPMV_ECUDA,
                std::string("comm allocation: ") + cudaGetErrorString(e));
  }
  c->peer[rank] = c->base;
  if (world == 1) c->connected = true;
  *out = c;
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_ipc_handle(yaspmv_comm c, void* out, int64_t bytes) {
  if (!c || !out) return fail(YASPMV_EINVAL, "NULL argument");
  if (bytes < (int64_t)sizeof(cudaIpcMemHandle_t)) return fail(YASPMV_EINVAL, "handle buffer < 64 bytes");
  CUDA_TRY(cudaSetDevice(c->device));
  cudaIpcMemHandle_t h;
  CUDA_TRY(cudaIpcGetMemHandle(&h, c->base));
  std::memcpy(out, &h, sizeof(h));
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_open_ipc(yaspmv_comm c, const void* handles, int64_t bytes) {
  if (!c || !handles) return fail(YASPMV_EINVAL, "NULL argument");
  const size_t hs = sizeof(cudaIpcMemHandle_t);
  if (bytes < (int64_t)(hs * c->world)) return fail(YASPMV_EINVAL, "handles must hold world * 64 bytes");
  if (c->connected && c->world > 1) return fail(YASPMV_EINVAL, "comm already connected");
  CUDA_TRY(cudaSetDevice(c->device));
  for (int q = 0; q < c->world; ++q) {
    if (q == c->rank) continue;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, static_cast<const char*>(handles) + q * hs, hs);
    void* p = nullptr;
    CUDA_TRY(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
    c->peer[q] = static_cast<char*>(p);
    c->ipc[q] = true;
  }
  c->connected = true;
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_connect_local(yaspmv_comm c, const yaspmv_comm* peers, int32_t world) {
  if (!c || !peers) return fail(YASPMV_EINVAL, "NULL argument");
  if (world != c->world) return fail(YASPMV_EINVAL, "world mismatch");
  for (int q = 0; q < world; ++q) {
    const yaspmv_comm p = peers[q];
    if (!p || p->rank != q || p->world != world || p->dtype != c->dtype || p->chunk != c->chunk)
      return fail(YASPMV_EINVAL, "peer comms must be rank-ordered with equal world, dtype and chunk");
    if (p->device != c->device) {  // another GPU of this process: needs peer access
      int can = 0;
      CUDA_TRY(cudaDeviceCanAccessPeer(&can, c->device, p->device));
      if (!can) return fail(YASPMV_EUNSUPPORTED, "no peer access between the devices");
      CUDA_TRY(cudaSetDevice(c->device));
      cudaError_t e = cudaDeviceEnablePeerAccess(p->device, 0);
      if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled)
        return fail(YASPMV_ECUDA, std::string("cudaDeviceEnablePeerAccess: ") + cudaGetErrorString(e));
      cudaGetLastError();
    }
    c->peer[q] = p->base;
  }
  c->connected = true;
  return YASPMV_OK;
}

void* yaspmv_comm_x(yaspmv_comm c, int32_t which) {
  if (!c) return nullptr;
  return c->xbuf(c->xown(), c->seq + (which & 1));
}

// ---- NVSwitch multicast: one multimem.st per element instead of P stores
int32_t yaspmv_comm_mc_supported(int32_t device) {
  const Drv& d = drv();
  if (!d.ok) return 0;
  CUdevice dev = 0;
  int v = 0;
  if (d.devget(&dev, device) != CUDA_SUCCESS) return 0;
  if (d.devattr(&v, CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev) != CUDA_SUCCESS) return 0;
  return v ? 1 : 0;
}

static size_t mc_bytes(yaspmv_comm c, size_t* gran_out) {
  const Drv& d = drv();
  CUmulticastObjectProp mp = {};
  mp.numDevices = (unsigned)c->world;
  mp.size = 2 * c->xbytes;
  mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  size_t g1 = 0, g2 = 0;
  d.mc_gran(&g1, &mp, CU_MULTICAST_GRANULARITY_RECOMMENDED);
  CUmemAllocationProp ap = {};
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = c->device;
  d.mem_gran(&g2, &ap, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
  size_t g = std::max<size_t>(std::max(g1, g2), 2u << 20);
  *gran_out = g;
  return round_up(2 * c->xbytes, g);
}

yaspmv_status yaspmv_comm_mc_create(yaspmv_comm c, int64_t* fd_out) {
  if (!c || !fd_out) return fail(YASPMV_EINVAL, "NULL argument");
  if (!yaspmv_comm_mc_supported(c->device)) return fail(YASPMV_EUNSUPPORTED, "device has no switch multicast");
  if (c->mc_have) return fail(YASPMV_EINVAL, "multicast object already present");
  const Drv& d = drv();
  CUDA_TRY(cudaSetDevice(c->device));
  size_t g = 0;
  c->mc_size = mc_bytes(c, &g);
  CUmulticastObjectProp mp = {};
  mp.numDevices = (unsigned)c->world;
  mp.size = c->mc_size;
  mp.handleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  CU_TRY(d.mc_create(&c->mc_h, &mp));
  c->mc_have = true;
  int fd = -1;
  CU_TRY(d.export_h(&fd, c->mc_h, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0));
  c->mc_fd = fd;
  *fd_out = fd;
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_mc_import(yaspmv_comm c, int64_t pid, int64_t fd) {
  if (!c) return fail(YASPMV_EINVAL, "NULL comm");
  if (c->mc_have) return fail(YASPMV_EINVAL, "multicast object already present");
  const Drv& d = drv();
  if (!d.ok) return fail(YASPMV_EUNSUPPORTED, "driver multicast entry points unavailable");
  CUDA_TRY(cudaSetDevice(c->device));
  size_t g = 0;
  c->mc_size = mc_bytes(c, &g);
  int local = -1;
  if (pid <= 0 || pid == (int64_t)getpid()) {
    local = dup((int)fd);
  } else {  // the creator's descriptor, duplicated into this process (Linux >= 5.6)
    const int pfd = (int)syscall(SYS_pidfd_open, (pid_t)pid, 0);
    if (pfd < 0) return fail(YASPMV_ECUDA, "pidfd_open failed (errno " + std::to_string(errno) + ")");
    local = (int)syscall(SYS_pidfd_getfd, pfd, (int)fd, 0);
    close(pfd);
  }
  if (local < 0) return fail(YASPMV_ECUDA, "could not obtain the multicast descriptor (errno " + std::to_string(errno) + ")");
  c->mc_fd = local;
  CU_TRY(d.import_h(&c->mc_h, (void*)(uintptr_t)local, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR));
  c->mc_have = true;
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_mc_add_device(yaspmv_comm c) {
  if (!c || !c->mc_have) return fail(YASPMV_EINVAL, "no multicast object (mc_create / mc_import first)");
  if (c->mc_added) return YASPMV_OK;
  const Drv& d = drv();
  CUDA_TRY(cudaSetDevice(c->device));
  CUdevice dev = 0;
  CU_TRY(d.devget(&dev, c->device));
  CU_TRY(d.mc_add(c->mc_h, dev));
  c->mc_added = true;
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_mc_bind(yaspmv_comm c) {
  if (!c || !c->mc_added) return fail(YASPMV_EINVAL, "mc_add_device first (on every rank)");
  if (c->mc) return YASPMV_OK;
  const Drv& d = drv();
  CUDA_TRY(cudaSetDevice(c->device));
  CUdevice dev = 0;
  CU_TRY(d.devget(&dev, c->device));
  size_t g = 0;
  const size_t sz = mc_bytes(c, &g);
  if (sz != c->mc_size) return fail(YASPMV_EINVAL, "multicast size mismatch between ranks");
  CUmemAllocationProp ap = {};
  ap.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  ap.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  ap.location.id = c->device;
  CU_TRY(d.mem_create(&c->mem_h, sz, &ap, 0));
  c->mem_have = true;
  CU_TRY(d.mc_bind(c->mc_h, 0, c->mem_h, 0, sz, 0));
  CUmemAccessDesc acc = {};
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = c->device;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  CU_TRY(d.addr_reserve(&c->loc_va, sz, g, 0, 0));
  CU_TRY(d.mem_map(c->loc_va, sz, 0, c->mem_h, 0));
  CU_TRY(d.set_access(c->loc_va, sz, &acc, 1));
  CU_TRY(d.addr_reserve(&c->mc_va, sz, g, 0, 0));
  CU_TRY(d.mem_map(c->mc_va, sz, 0, c->mc_h, 0));
  CU_TRY(d.set_access(c->mc_va, sz, &acc, 1));
  // the current x buffers move into the bound memory; from here on steps read loc_va and
  // store through mc_va
  CUDA_TRY(cudaMemcpy(reinterpret_cast<void*>(c->loc_va), c->base, 2 * c->xbytes, cudaMemcpyDeviceToDevice));
  CUDA_TRY(cudaDeviceSynchronize());
  c->mc = true;
  return YASPMV_OK;
}

int32_t yaspmv_comm_mc_active(yaspmv_comm c) { return c && c->mc ? 1 : 0; }

yaspmv_status yaspmv_comm_mc_release(yaspmv_comm c) {
  if (!c) return fail(YASPMV_EINVAL, "NULL comm");
  if (c->mc) {  // back to the peer-mapped buffers (the bound ones stay mapped until free)
    CUDA_TRY(cudaSetDevice(c->device));
    CUDA_TRY(cudaDeviceSynchronize());
    CUDA_TRY(cudaMemcpy(c->base, reinterpret_cast<void*>(c->loc_va), 2 * c->xbytes, cudaMemcpyDeviceToDevice));
    c->mc = false;
  }
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_begin(yaspmv_comm c) {
  if (!c) return fail(YASPMV_EINVAL, "NULL comm");
  c->fresh = true;
  return YASPMV_OK;
}

double* yaspmv_comm_norm2_device(yaspmv_comm c) { return c ? c->d_norm_local + 1 : nullptr; }
int64_t yaspmv_comm_seq(yaspmv_comm c) { return c ? c->seq : -1; }

int32_t yaspmv_launches_per_fused_step(yaspmv_matrix A) {
  if (!A) return 0;
  // wait + SpMV (+ combine) + 2 reduction kernels + publish
  return 1 + (A->can.ntiles > 0 ? (A->can.p.S > 1 ? 2 : 1) : 0) + 2 + 1;
}

static yaspmv_status launch_wait(yaspmv_comm c, cudaStream_t s) {
  wait_kernel<<<1, 32, 0, s>>>(c->sig(c->base), c->world, (unsigned long long)c->seq, (int)((c->seq - 1) & 1),
                               c->d_norm_local + 1, c->d_err, c->timeout_ns);
  CUDA_TRY(cudaGetLastError());
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_wait(yaspmv_comm c, void* stream) {
  if (!c) return fail(YASPMV_EINVAL, "NULL comm");
  if (!c->connected) return fail(YASPMV_EINVAL, "comm not connected (open_ipc / connect_local)");
  CUDA_TRY(cudaSetDevice(c->device));
  if (c->seq == 0 || c->fresh) return YASPMV_OK;  // nothing issued since begin
  return launch_wait(c, (cudaStream_t)stream);
}

yaspmv_status yaspmv_power_step_fused(yaspmv_matrix A, yaspmv_comm c, void* stream) {
  yaspmv::TraceRange tr_("yaspmv:power_step_fused");
  if (!A || !c) return fail(YASPMV_EINVAL, "NULL argument");
  if (A->device < 0) return fail(YASPMV_EINVAL, "host-only handle: no CPU fallback");
  if (!c->connected) return fail(YASPMV_EINVAL, "comm not connected (open_ipc / connect_local)");
  if (A->device != c->device) return fail(YASPMV_EINVAL, "matrix and comm on different devices");
  if (A->dtype != c->dtype) return fail(YASPMV_EINVAL, "matrix and comm dtypes differ");
  if (A->can.n != c->n_pad) return fail(YASPMV_EINVAL, "matrix columns must equal world * chunk (padded x)");
  if (A->can.m > c->chunk) return fail(YASPMV_EINVAL, "matrix rows exceed the comm chunk");
  CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = (cudaStream_t)stream;
  const bool scaled = !c->fresh;
  if (scaled) {
    yaspmv_status st = launch_wait(c, s);
    if (st != YASPMV_OK) return st;
  }
  PeerOut po;
  if (c->mc) {  // one multimem.st per element: the switch writes every rank's buffer
    po.n = 1;
    po.mc = 1;
    po.p[0] = c->xbuf(reinterpret_cast<const char*>(c->mc_va), c->seq + 1) + (size_t)c->rank * c->chunk * c->vsize;
  } else {
    po.n = c->world;
    for (int q = 0; q < c->world; ++q)
      po.p[q] = c->xbuf(c->peer[q], c->seq + 1) + (size_t)c->rank * c->chunk * c->vsize;
  }
  yaspmv_status st = run_spmv_peers(A, c->xbuf(c->xown(), c->seq), scaled ? c->d_norm_local + 1 : nullptr,
                                    c->d_norm_local, po, stream);
  if (st != YASPMV_OK) return st;
  PeerSig ps;
  ps.n = c->world;
  for (int q = 0; q < c->world; ++q) ps.p[q] = c->sig(c->peer[q]);
  publish_kernel<<<1, 32, 0, s>>>(ps, c->rank, (unsigned long long)(c->seq + 1), (int)(c->seq & 1),
                                  c->d_norm_local);
  CUDA_TRY(cudaGetLastError());
  c->seq += 1;
  c->fresh = false;
  return YASPMV_OK;
}

yaspmv_status yaspmv_comm_check(yaspmv_comm c) {
  if (!c) return fail(YASPMV_EINVAL, "NULL comm");
  CUDA_TRY(cudaSetDevice(c->device));
  int err = 0;
  CUDA_TRY(cudaMemcpy(&err, c->d_err, sizeof(int), cudaMemcpyDeviceToHost));
  if (err) {
    CUDA_TRY(cudaMemset(c->d_err, 0, sizeof(int)));
    return fail(YASPMV_ECUDA, "fused power step: a peer's signal did not arrive within the timeout");
  }
  return YASPMV_OK;
}

void yaspmv_comm_free(yaspmv_comm c) { delete c; }

}  // extern "C"
