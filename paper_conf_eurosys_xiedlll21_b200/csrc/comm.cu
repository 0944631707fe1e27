// comm.cu — fused cross-GPU reduce + finalisation for tree-sharded prediction.
//
// Tree sharding (dist.py, P:2441-2456 scale the path over GPUs; the C5 forest does not fit one
// CTA's staging) leaves every rank with raw fp64 per-sample sums of its own trees.  Instead of a
// separate ncclReduce followed by a finalize launch, the partials are written straight into an
// NCCL symmetric-memory window and ONE kernel per rank
//   1. synchronises with the same CTA on every peer through an LSA barrier (NCCL device API),
//   2. loads the peers' partials of its rows directly over NVLink (load/store-accessible peer
//      memory), sums them in rank order 0..world-1 — fixed order, so every rank that finalises a
//      row produces the same bits — and applies the full forest's aggregation (base score,
//      average, class margin / argmax) exactly like k_finalize,
//   3. passes a second barrier so no peer overwrites its window while others still read it.
// NCCL is loaded at run time (dlopen): libtahoe.so does not link against it, and everything else
// in the library works without it.  The peer-pointer variant (tahoe_reduce_partials) runs the same
// row kernel over caller-provided device pointers (same device, P2P or CUDA-IPC mappings).
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>

#include <nccl.h>
#include <nccl_device.h>

#include "internal.hpp"

using namespace tahoe;

namespace {

constexpr int kMaxPeers = 64;        // tahoe_reduce_partials: peers passed by value
constexpr int kReduceBlock = 256;

// ------------------------------------------------------------------ NCCL, loaded at run time
struct NcclApi {
  bool ok = false;
  std::string why;
  int version = 0;
  decltype(&ncclGetVersion) GetVersion = nullptr;
  decltype(&ncclGetErrorString) GetErrorString = nullptr;
  decltype(&ncclGetUniqueId) GetUniqueId = nullptr;
  decltype(&ncclCommInitRank) CommInitRank = nullptr;
  decltype(&ncclCommFinalize) CommFinalize = nullptr;
  decltype(&ncclCommDestroy) CommDestroy = nullptr;
  decltype(&ncclMemAlloc) MemAlloc = nullptr;
  decltype(&ncclMemFree) MemFree = nullptr;
  decltype(&ncclCommWindowRegister) WindowRegister = nullptr;
  decltype(&ncclCommWindowDeregister) WindowDeregister = nullptr;
  ncclResult_t (*DevCommCreate)(ncclComm_t, ncclDevCommRequirements_t const*, ncclDevComm_t*) = nullptr;
  ncclResult_t (*DevCommDestroy)(ncclComm_t, ncclDevComm_t const*) = nullptr;
};

template <class F>
static bool sym(void* h, const char* name, F& f, std::string& why) {
  f = reinterpret_cast<F>(dlsym(h, name));
  if (!f) why = std::string("NCCL symbol missing: ") + name;
  return f != nullptr;
}

static NcclApi load_nccl() {
  NcclApi a;
  void* h = nullptr;
  const char* env = std::getenv("TAHOE_NCCL_LIB");
  if (env && *env) h = dlopen(env, RTLD_NOW | RTLD_GLOBAL);
  // the copy torch already loaded (same process) comes first, then the loader's search path
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    a.why = std::string("cannot load NCCL (set TAHOE_NCCL_LIB): ") + (dlerror() ? dlerror() : "");
    return a;
  }
  bool ok = sym(h, "ncclGetVersion", a.GetVersion, a.why) &&
            sym(h, "ncclGetErrorString", a.GetErrorString, a.why) &&
            sym(h, "ncclGetUniqueId", a.GetUniqueId, a.why) &&
            sym(h, "ncclCommInitRank", a.CommInitRank, a.why) &&
            sym(h, "ncclCommFinalize", a.CommFinalize, a.why) &&
            sym(h, "ncclCommDestroy", a.CommDestroy, a.why) &&
            sym(h, "ncclMemAlloc", a.MemAlloc, a.why) && sym(h, "ncclMemFree", a.MemFree, a.why) &&
            sym(h, "ncclCommWindowRegister", a.WindowRegister, a.why) &&
            sym(h, "ncclCommWindowDeregister", a.WindowDeregister, a.why) &&
            sym(h, "ncclDevCommCreate", a.DevCommCreate, a.why) &&
            sym(h, "ncclDevCommDestroy", a.DevCommDestroy, a.why);
  if (!ok) return a;
  a.GetVersion(&a.version);
  // the device-side structures (window, barrier) are compiled from the 2.28 headers
  if (a.version / 100 != NCCL_VERSION_CODE / 100) {
    a.why = "NCCL " + std::to_string(a.version) + " loaded, the device API was compiled against " +
            std::to_string(NCCL_VERSION_CODE);
    return a;
  }
  a.ok = true;
  return a;
}

static NcclApi& nccl_api() {
  static NcclApi api = load_nccl();
  return api;
}

static tahoe_status nccl_fail(ncclResult_t r, const char* what) {
  return fail(TAHOE_E_CUDA, std::string(what) + ": " + nccl_api().GetErrorString(r));
}

static tahoe_status cuda_err(cudaError_t e, const char* what) {
  return fail(TAHOE_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

struct DevScope {  // restores the caller's current device
  int prev = -1;
  explicit DevScope(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DevScope() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

// ------------------------------------------------------------------ kernels
struct ReduceArgs {
  int32_t world = 1;
  int32_t C = 1;                 // outputs per row
  int32_t agg = 0;
  float base = 0.0f;
  int32_t n_trees_full = 1;
  int64_t lo = 0, hi = 0;        // rows this rank finalises
  float* out = nullptr;          // [(hi - lo) x C]
  int32_t* out_class = nullptr;  // [hi - lo] or nullptr
};

struct PeerPtrs {
  const double* p[kMaxPeers];
};

// Rows [lo, hi): s = sum_p partial_p[i][c] in rank order, then the finalisation of k_finalize
// (readings Z16-Z18: fp64 sum, RN to fp32, argmax ties to the lowest class).
template <class Peer>
__device__ __forceinline__ void reduce_finalize_rows(const ReduceArgs& a, Peer peer) {
  const int32_t C = a.C;
  for (int64_t i = a.lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.hi;
       i += (int64_t)gridDim.x * blockDim.x) {
    int best = 0;
    double bv = 0.0;
    for (int32_t c = 0; c < C; c++) {
      double s = 0.0;
      for (int32_t p = 0; p < a.world; p++) s += peer(p)[i * C + c];
      double v;
      if (a.agg == TAHOE_AGG_VOTE) v = s;
      else if (a.agg == TAHOE_AGG_AVERAGE) v = s / (double)a.n_trees_full + (double)a.base;
      else v = s + (double)a.base;
      a.out[(i - a.lo) * C + c] = (float)v;
      if (c == 0 || v > bv) { best = c; bv = v; }
    }
    if (a.out_class) {
      int32_t k = 0;
      if (a.agg == TAHOE_AGG_BINARY) k = bv > 0.0 ? 1 : 0;
      else if (a.agg == TAHOE_AGG_CLASS_SUM || a.agg == TAHOE_AGG_VOTE) k = best;
      a.out_class[i - a.lo] = k;
    }
  }
}

__global__ void __launch_bounds__(kReduceBlock) k_reduce_ptrs(const ReduceArgs a, const PeerPtrs P) {
  reduce_finalize_rows(a, [&](int p) { return P.p[p]; });
}

// One LSA barrier per CTA index (barrier b pairs CTA b of every rank).  acq_rel: the arrive
// releases this rank's partials (written by the preceding kernel in stream order) and, on the
// second barrier, orders this CTA's peer loads before any peer's later overwrite.
__global__ void __launch_bounds__(kReduceBlock) k_reduce_lsa(const ReduceArgs a,
                                                            const __grid_constant__ ncclDevComm dc,
                                                            ncclWindow_t win) {
  ncclLsaBarrierSession<ncclCoopCta> bar(ncclCoopCta(), dc, ncclTeamLsa(dc), dc.lsaBarrier, blockIdx.x);
  bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
  reduce_finalize_rows(a, [&](int p) {
    return reinterpret_cast<const double*>(ncclGetPeerPointer(win, 0, p));
  });
  bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
}

// NVLS variant (opt-in, TAHOE_REDUCE_NVLS=1 at tahoe_comm_init, world > 1 on an NVSwitch system
// with multicast): the per-class sum over ranks is one multimem.ld_reduce of the window's
// multicast address — the switch adds the G ranks' fp64 partials and returns the sum, so each row
// costs one NVLink load per class instead of G peer loads.  The switch's addition order is not
// specified, so reading R5's rank order (bit-reproducible run to run) does not hold; the sum stays
// within reading Z17's fp64 bound (dyadic forests: exact).
__global__ void __launch_bounds__(kReduceBlock) k_reduce_nvls(const ReduceArgs a,
                                                             const __grid_constant__ ncclDevComm dc,
                                                             ncclWindow_t win) {
  ncclLsaBarrierSession<ncclCoopCta> bar(ncclCoopCta(), dc, ncclTeamLsa(dc), dc.lsaBarrier, blockIdx.x);
  bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
  const double* mc = reinterpret_cast<const double*>(ncclGetLsaMultimemPointer(win, 0, dc));
  const int32_t C = a.C;
  for (int64_t i = a.lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.hi;
       i += (int64_t)gridDim.x * blockDim.x) {
    int best = 0;
    double bv = 0.0;
    for (int32_t c = 0; c < C; c++) {
      double s;
      asm volatile("multimem.ld_reduce.relaxed.sys.global.add.f64 %0, [%1];"
                   : "=d"(s) : "l"(mc + i * C + c) : "memory");
      double v;
      if (a.agg == TAHOE_AGG_VOTE) v = s;
      else if (a.agg == TAHOE_AGG_AVERAGE) v = s / (double)a.n_trees_full + (double)a.base;
      else v = s + (double)a.base;
      a.out[(i - a.lo) * C + c] = (float)v;
      if (c == 0 || v > bv) { best = c; bv = v; }
    }
    if (a.out_class) {
      int32_t k = 0;
      if (a.agg == TAHOE_AGG_BINARY) k = bv > 0.0 ? 1 : 0;
      else if (a.agg == TAHOE_AGG_CLASS_SUM || a.agg == TAHOE_AGG_VOTE) k = best;
      a.out_class[i - a.lo] = k;
    }
  }
  bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
}

static tahoe_status rows_of(int64_t n, int32_t world, int32_t rank, int32_t mode, int64_t* lo,
                            int64_t* hi) {
  if (n < 0) return fail(TAHOE_E_INVAL, "n < 0");
  if (world < 1 || rank < 0 || rank >= world) return fail(TAHOE_E_INVAL, "bad rank / world");
  if (mode == TAHOE_REDUCE_ALL) { *lo = 0; *hi = n; return TAHOE_OK; }
  if (mode != TAHOE_REDUCE_SCATTER) return fail(TAHOE_E_INVAL, "unknown reduce mode");
  // same split as dist.shard_rows: sizes differ by at most one
  *lo = (int64_t)((__int128)n * rank / world);
  *hi = (int64_t)((__int128)n * (rank + 1) / world);
  return TAHOE_OK;
}

// A shard carries the full forest's aggregation, base score and tree count (make_shard).
static ReduceArgs reduce_args(const tahoe_forest* f, int32_t world, int64_t lo, int64_t hi,
                              float* out, int32_t* out_class) {
  const Forest& H = f->host;
  ReduceArgs a;
  a.world = world;
  a.C = H.n_out();
  a.agg = H.agg;
  a.base = H.base;
  a.n_trees_full = H.n_trees_full;
  a.lo = lo;
  a.hi = hi;
  a.out = out;
  a.out_class = out_class;
  return a;
}

static int reduce_grid(int64_t rows, int sms) {
  int64_t g = (rows + kReduceBlock - 1) / kReduceBlock;
  if (g > (int64_t)sms * 4) g = (int64_t)sms * 4;
  return (int)(g < 1 ? 1 : g);
}

}  // namespace

struct tahoe_comm {
  ncclComm_t comm = nullptr;
  ncclDevComm dev{};
  bool dev_ok = false;
  bool nvls = false;              // devComm created with lsaMultimem (k_reduce_nvls)
  int32_t world = 1, rank = 0, device = 0;
  int32_t grid = 0;               // CTAs of k_reduce_lsa == LSA barriers requested
  void* buf = nullptr;            // symmetric window (partials of this rank)
  size_t bytes = 0;
  ncclWindow_t win = nullptr;
};

static void release_window(tahoe_comm* c) {
  if (c->win) nccl_api().WindowDeregister(c->comm, c->win);
  if (c->buf) nccl_api().MemFree(c->buf);
  c->win = nullptr;
  c->buf = nullptr;
  c->bytes = 0;
}

#define TAHOE_COMM_GUARD_BEGIN try {
#define TAHOE_COMM_GUARD_END                                                    \
  }                                                                             \
  catch (const std::bad_alloc&) { return fail(TAHOE_E_NOMEM, "host allocation failed"); } \
  catch (const std::exception& ex) { return fail(TAHOE_E_INVAL, ex.what()); }

extern "C" {

__attribute__((visibility("default"))) tahoe_status tahoe_comm_unique_id(uint8_t* id) {
  if (!id) return fail(TAHOE_E_INVAL, "NULL id");
  if (!nccl_api().ok) return fail(TAHOE_E_UNSUPPORTED, nccl_api().why);
  static_assert(sizeof(ncclUniqueId) == TAHOE_COMM_ID_BYTES, "ncclUniqueId size");
  ncclUniqueId u;
  ncclResult_t r = nccl_api().GetUniqueId(&u);
  if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
  std::memcpy(id, &u, sizeof u);
  return TAHOE_OK;
}

__attribute__((visibility("default"))) tahoe_status tahoe_comm_init(const uint8_t* id, int32_t world,
                                                                    int32_t rank, int32_t device,
                                                                    tahoe_comm** out) {
  TAHOE_COMM_GUARD_BEGIN
  if (!id || !out) return fail(TAHOE_E_INVAL, "NULL argument");
  *out = nullptr;
  if (world < 1 || rank < 0 || rank >= world) return fail(TAHOE_E_INVAL, "bad rank / world");
  if (world > kMaxPeers) return fail(TAHOE_E_INVAL, "world > 64");
  if (device < 0) return fail(TAHOE_E_INVAL, "device < 0");
  if (!nccl_api().ok) return fail(TAHOE_E_UNSUPPORTED, nccl_api().why);
  DevScope ds(device);
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || cur != device) return fail(TAHOE_E_CUDA, "cannot select device");
  tahoe_comm* c = new tahoe_comm();
  c->world = world;
  c->rank = rank;
  c->device = device;
  cudaDeviceGetAttribute(&c->grid, cudaDevAttrMultiProcessorCount, device);
  if (c->grid < 1) c->grid = 1;
  ncclUniqueId u;
  std::memcpy(&u, id, sizeof u);
  ncclResult_t r = nccl_api().CommInitRank(&c->comm, world, u, rank);
  if (r != ncclSuccess) { delete c; return nccl_fail(r, "ncclCommInitRank"); }
  ncclDevCommRequirements reqs;
  std::memset(&reqs, 0, sizeof reqs);
  reqs.lsaBarrierCount = c->grid;
  const char* nv = std::getenv("TAHOE_REDUCE_NVLS");
  if (world > 1 && nv && std::strcmp(nv, "1") == 0) {
    // multicast (NVLS) team memory; without NVSwitch multicast the creation fails and the
    // peer-load kernel is used
    reqs.lsaMultimem = true;
    r = nccl_api().DevCommCreate(c->comm, &reqs, &c->dev);
    c->nvls = r == ncclSuccess && c->dev.lsaMultimem.mcBasePtr != nullptr;
    if (r == ncclSuccess && !c->nvls) nccl_api().DevCommDestroy(c->comm, &c->dev);
    reqs.lsaMultimem = false;
  }
  if (!c->nvls) r = nccl_api().DevCommCreate(c->comm, &reqs, &c->dev);
  if (r != ncclSuccess) {
    nccl_api().CommDestroy(c->comm);
    delete c;
    return nccl_fail(r, "ncclDevCommCreate");
  }
  c->dev_ok = true;
  if (c->dev.lsaSize != world) {
    const int ls = c->dev.lsaSize;
    nccl_api().DevCommDestroy(c->comm, &c->dev);
    nccl_api().CommDestroy(c->comm);
    delete c;
    return fail(TAHOE_E_UNSUPPORTED, "ranks are not all load/store-reachable (LSA team " +
                                         std::to_string(ls) + " of " + std::to_string(world) +
                                         "): use the ncclReduce path");
  }
  *out = c;
  return TAHOE_OK;
  TAHOE_COMM_GUARD_END
}

__attribute__((visibility("default"))) void tahoe_comm_free(tahoe_comm* c) {
  if (!c) return;
  DevScope ds(c->device);
  cudaDeviceSynchronize();
  release_window(c);
  if (c->dev_ok) nccl_api().DevCommDestroy(c->comm, &c->dev);
  if (c->comm) {
    nccl_api().CommFinalize(c->comm);
    nccl_api().CommDestroy(c->comm);
  }
  delete c;
}

__attribute__((visibility("default"))) tahoe_status tahoe_reduce_rows(int64_t n, int32_t world,
                                                                      int32_t rank, int32_t mode,
                                                                      int64_t* lo, int64_t* hi) {
  if (!lo || !hi) return fail(TAHOE_E_INVAL, "NULL argument");
  return rows_of(n, world, rank, mode, lo, hi);
}

__attribute__((visibility("default"))) tahoe_status tahoe_predict_reduce(
    const tahoe_forest* shard, tahoe_comm* c, const float* X, int64_t n, int32_t d, int32_t mode,
    float* out, int32_t* out_class, tahoe_stream stream) {
  TAHOE_COMM_GUARD_BEGIN
  if (!shard || !c) return fail(TAHOE_E_INVAL, "NULL forest or comm");
  if (shard->device < 0) return fail(TAHOE_E_STATE, "host-only forest handle");
  if (shard->device != c->device) return fail(TAHOE_E_INVAL, "forest and comm live on different devices");
  int64_t lo = 0, hi = 0;
  tahoe_status st = rows_of(n, c->world, c->rank, mode, &lo, &hi);
  if (st != TAHOE_OK) return st;
  if (n == 0) return TAHOE_OK;
  if (!X || (!out && hi > lo)) return fail(TAHOE_E_INVAL, "NULL X or output pointer");
  DevScope ds(c->device);
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  const size_t need = (size_t)n * (size_t)shard->host.n_out() * sizeof(double);
  if (need > c->bytes) {
    // collective on every rank (same n on every rank): drain in-flight users, then re-register
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_err(e, "synchronize before window growth");
    release_window(c);
    size_t bytes = std::max<size_t>(need, (size_t)2 << 20);
    bytes = (bytes + ((size_t)2 << 20) - 1) & ~(((size_t)2 << 20) - 1);
    ncclResult_t r = nccl_api().MemAlloc(&c->buf, bytes);
    if (r != ncclSuccess) { c->buf = nullptr; return nccl_fail(r, "ncclMemAlloc"); }
    r = nccl_api().WindowRegister(c->comm, c->buf, bytes, &c->win, NCCL_WIN_COLL_SYMMETRIC);
    if (r != ncclSuccess) {
      nccl_api().MemFree(c->buf);
      c->buf = nullptr;
      c->win = nullptr;
      return nccl_fail(r, "ncclCommWindowRegister");
    }
    c->bytes = bytes;
  }
  st = tahoe_predict_partial(shard, X, n, d, static_cast<double*>(c->buf), stream);
  if (st != TAHOE_OK) return st;
  ReduceArgs a = reduce_args(shard, c->world, lo, hi, out, out_class);
  if (c->nvls) k_reduce_nvls<<<c->grid, kReduceBlock, 0, s>>>(a, c->dev, c->win);
  else k_reduce_lsa<<<c->grid, kReduceBlock, 0, s>>>(a, c->dev, c->win);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_err(e, c->nvls ? "k_reduce_nvls launch" : "k_reduce_lsa launch");
  return TAHOE_OK;
  TAHOE_COMM_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_reduce_partials(
    const tahoe_forest* full, const double* const* partials, int32_t world, int32_t rank,
    int32_t mode, int64_t n, float* out, int32_t* out_class, tahoe_stream stream) {
  TAHOE_COMM_GUARD_BEGIN
  if (!full) return fail(TAHOE_E_INVAL, "NULL forest");
  if (full->device < 0) return fail(TAHOE_E_STATE, "host-only forest handle");
  if (world > kMaxPeers) return fail(TAHOE_E_INVAL, "world > 64");
  int64_t lo = 0, hi = 0;
  tahoe_status st = rows_of(n, world, rank, mode, &lo, &hi);
  if (st != TAHOE_OK) return st;
  if (hi == lo) return TAHOE_OK;
  if (!partials || !out) return fail(TAHOE_E_INVAL, "NULL partials or output pointer");
  PeerPtrs P{};
  for (int32_t p = 0; p < world; p++) {
    if (!partials[p]) return fail(TAHOE_E_INVAL, "NULL partial of rank " + std::to_string(p));
    P.p[p] = partials[p];
  }
  DevScope ds(full->device);
  ReduceArgs a = reduce_args(full, world, lo, hi, out, out_class);
  k_reduce_ptrs<<<reduce_grid(hi - lo, std::max(1, full->num_sms)), kReduceBlock, 0,
                  reinterpret_cast<cudaStream_t>(stream)>>>(a, P);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_err(e, "k_reduce_ptrs launch");
  return TAHOE_OK;
  TAHOE_COMM_GUARD_END
}

}  // extern "C"
