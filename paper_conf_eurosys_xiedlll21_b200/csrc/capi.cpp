// capi.cpp — the extern "C" boundary of libtahoe.so (include/tahoe.h), Algorithm 1's online
// steps: layout on the host once per forest, strategy choice + launch per batch.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <climits>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <new>
#include <sstream>
#include <string>

#include "internal.hpp"

namespace tahoe {

static thread_local std::string g_err;

tahoe_status fail(tahoe_status st, const std::string& msg) {
  g_err = msg;
  return st;
}

static tahoe_status cuda_fail(cudaError_t e, const char* what) {
  return fail(TAHOE_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

// Restores the caller's current device on scope exit (torch owns the thread's device state).
struct DeviceGuard {
  int prev = -1;
  bool ok = true;
  explicit DeviceGuard(int dev) {
    if (dev < 0) return;
    cudaGetDevice(&prev);
    if (prev != dev) ok = cudaSetDevice(dev) == cudaSuccess;
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

constexpr int32_t kDefaultMaxSmem = kMaxSmemOptin;

// Stream-ordered scratch (fp64 partials) comes from a library-owned pool per device that keeps
// its memory across synchronisations (release threshold = max), so a predict call never waits
// for the driver to map fresh pages.
static cudaError_t scratch_alloc(void** p, size_t bytes, cudaStream_t st) {
  static std::mutex mu;
  static cudaMemPool_t pools[64] = {};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaMallocAsync(p, bytes, st);
  {
    std::lock_guard<std::mutex> g(mu);
    if (!pools[dev]) {
      cudaMemPoolProps props = {};
      props.allocType = cudaMemAllocationTypePinned;
      props.location.type = cudaMemLocationTypeDevice;
      props.location.id = dev;
      e = cudaMemPoolCreate(&pools[dev], &props);
      if (e != cudaSuccess) { pools[dev] = nullptr; return cudaMallocAsync(p, bytes, st); }
      uint64_t thr = UINT64_MAX;
      cudaMemPoolSetAttribute(pools[dev], cudaMemPoolAttrReleaseThreshold, &thr);
    }
  }
  return cudaMallocFromPoolAsync(p, bytes, pools[dev], st);
}

// Slot rows (32 nodes each) of the per-CTA forest slice: the opt-in shared memory minus the
// sample-tile ring for rows of n_features attributes (none when rows stay in global memory).
static int32_t slot_budget_for(int32_t max_smem, int32_t n_features) {
  const int32_t fb = feature_bits(n_features + 1);
  const bool padded = n_features % 4 == 0;   // predict with d == n_features takes the 2-D TMA path
  int64_t ring = std::max<int64_t>(0, sliced_ring_bytes(n_features, fb, padded)) + kSlicedBarrierBytes;
  // forests that can take the u16 rank codes (reading R7) keep room for their (minimum, 3-deep)
  // code-tile ring, control block and staged partials too (rows of ~100-127 attributes are too wide
  // for the fp32 ring, which would otherwise leave the whole of shared memory to the slice)
  if (fb <= kCodeMaxFbits) ring = std::max<int64_t>(ring, coded_ring_smem(kSlicedRing, code_tile_stride(fb)));
  // the slice region is rounded up to 1 KB so the ring's row bases stay aligned
  return (int32_t)std::max<int64_t>(0, ((max_smem - ring) & ~1023LL) / kSlotBytes);
}

static void free_host_pipe(tahoe_forest* f) {
  auto& h = f->hp;
  if (!h.ready) return;
  cudaStreamDestroy(h.s_in);
  cudaStreamDestroy(h.s_cmp);
  cudaStreamDestroy(h.s_cmp2);
  cudaStreamDestroy(h.s_out);
  cudaEventDestroy(h.ev_start);
  for (int b = 0; b < 3; b++) { cudaEventDestroy(h.ev_in[b]); cudaEventDestroy(h.ev_cmp[b]); cudaEventDestroy(h.ev_out[b]); }
  h = tahoe_forest::HostPipe();
}

static cudaError_t init_host_pipe(tahoe_forest* f) {
  auto& h = f->hp;
  if (h.ready) return cudaSuccess;
  cudaError_t e = cudaStreamCreateWithFlags(&h.s_in, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h.s_cmp, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h.s_cmp2, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h.s_out, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h.ev_start, cudaEventDisableTiming);
  for (int b = 0; b < 3 && e == cudaSuccess; b++) {
    e = cudaEventCreateWithFlags(&h.ev_in[b], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h.ev_cmp[b], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h.ev_out[b], cudaEventDisableTiming);
  }
  h.ready = e == cudaSuccess;
  return e;
}

static void free_device(tahoe_forest* f) {
  if (f->device < 0) return;
  DeviceGuard g(f->device);
  free_host_pipe(f);
  cudaFree((void*)f->dd.nodes);
  cudaFree((void*)f->dd.root);
  cudaFree((void*)f->dd.cls);
  cudaFree((void*)f->dd.tree_orig);
  cudaFree((void*)f->dd.slot_orig);
  cudaFree((void*)f->dd.cls_seg);
  cudaFree((void*)f->ds.nodes);
  cudaFree((void*)f->ds.col_len);
  cudaFree((void*)f->ds.slots);
  cudaFree((void*)f->ds.leaf_meta);
  cudaFree((void*)f->ds.cnodes);
  cudaFree((void*)f->ds.thr_tab);
  cudaFree((void*)f->ds.thr_off);
  cudaFree((void*)f->ds.cb_img);
  cudaFree((void*)f->ds.cb_desc);
  cudaFree((void*)f->ds.slot_attr);
  cudaFree((void*)f->ds.v_src);
  cudaFree((void*)f->ds.c8_img);
  cudaFree((void*)f->ds.c8_grp);
  cudaFree((void*)f->ds.c8_band);
  cudaFree((void*)f->ds.slice_w);
  cudaFree((void*)f->ds.col_mid);
  cudaFree(f->d_class_ptr);
  cudaFree(f->d_class_parts);
  cudaFree(f->d_cta_start);
  f->d_cta_start = nullptr;
  f->dd = DevDirect();
  f->ds = DevSliced();
  f->d_class_ptr = f->d_class_parts = nullptr;
}

template <class T>
static tahoe_status upload(const std::vector<T>& v, const T** dst) {
  if (v.empty()) { *dst = nullptr; return TAHOE_OK; }
  void* p = nullptr;
  // padded to 64 bytes (zeros), so kernels may load whole aligned node groups past the last node
  const size_t bytes = v.size() * sizeof(T), padded = (bytes + 63) & ~(size_t)63;
  cudaError_t e = cudaMalloc(&p, padded);
  if (e != cudaSuccess) return fail(TAHOE_E_NOMEM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
  if (padded > bytes) e = cudaMemset(static_cast<char*>(p) + bytes, 0, padded - bytes);
  if (e == cudaSuccess) e = cudaMemcpy(p, v.data(), bytes, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) { cudaFree(p); return cuda_fail(e, "cudaMemcpy"); }
  *dst = static_cast<const T*>(p);
  return TAHOE_OK;
}

// encode both images with the current layout state and (re)upload them (Algorithm 1 line 7)
// Direct image chunking (reading R4): B200's L2 is 126 MB; a direct image larger than
// kDirectChunkMin is walked in chunks of whole trees of at most kDirectChunkBytes (one launch per
// chunk, fp64 partials accumulated in chunk order), so the nodes every row visits come from L2
// rather than HBM.  $TAHOE_DIRECT_CHUNK_KB overrides the chunk size (0 = never chunk).
static void direct_chunks(tahoe_forest* f) {
  int64_t chunk = (int64_t)20 << 20, min_total = (int64_t)64 << 20;
  if (const char* e = std::getenv("TAHOE_DIRECT_CHUNK_KB")) {
    chunk = (int64_t)std::atoll(e) << 10;
    min_total = chunk;
  }
  const std::vector<int32_t>& root = f->di.root;
  const int64_t N = (int64_t)f->di.nodes.size() / 2;
  const int32_t T = (int32_t)root.size();
  f->direct_chunks.assign(1, 0);
  if (chunk > 0 && N * 8 > min_total) {
    int64_t acc = 0;
    for (int32_t t = 0; t < T; t++) {
      const int64_t sz = (int64_t)((t + 1 < T ? root[t + 1] : N) - root[t]) * 8;
      if (acc > 0 && acc + sz > chunk) {
        f->direct_chunks.push_back(t);
        acc = 0;
      }
      acc += sz;
    }
  }
  f->direct_chunks.push_back(T);
}

static tahoe_status encode_and_upload(tahoe_forest* f) {
  tahoe_status st = encode_direct(f->host, f->di);
  if (st != TAHOE_OK) return st;
  direct_chunks(f);
  st = encode_sliced(f->host, f->slot_budget, f->sl, f->max_smem);
  if (st != TAHOE_OK) return st;
  if (f->device < 0) return TAHOE_OK;
  DeviceGuard g(f->device);
  if (!g.ok) return fail(TAHOE_E_CUDA, "cannot select device");
  free_device(f);
  if ((st = upload(f->di.nodes, &f->dd.nodes)) != TAHOE_OK) return st;
  if ((st = upload(f->di.root, &f->dd.root)) != TAHOE_OK) return st;
  if ((st = upload(f->di.cls, &f->dd.cls)) != TAHOE_OK) return st;
  if ((st = upload(f->di.tree_orig, &f->dd.tree_orig)) != TAHOE_OK) return st;
  if ((st = upload(f->di.slot_orig, &f->dd.slot_orig)) != TAHOE_OK) return st;
  if ((st = upload(f->di.cls_seg, &f->dd.cls_seg)) != TAHOE_OK) return st;
  f->dd.n_slots = (int32_t)f->di.root.size();
  f->dd.fbits = f->di.fbits;
  f->dd.n_nodes = (int64_t)f->di.nodes.size() / 2;
  if (f->sl.valid) {
    if ((st = upload(f->sl.nodes, &f->ds.nodes)) != TAHOE_OK) return st;
    if ((st = upload(f->sl.col_len, &f->ds.col_len)) != TAHOE_OK) return st;
    if ((st = upload(f->sl.slots, &f->ds.slots)) != TAHOE_OK) return st;
    if ((st = upload(f->sl.leaf_meta, &f->ds.leaf_meta)) != TAHOE_OK) return st;
    const int32_t* cp = nullptr;
    const int32_t* cq = nullptr;
    if ((st = upload(f->sl.class_ptr, &cp)) != TAHOE_OK) return st;
    if ((st = upload(f->sl.class_parts, &cq)) != TAHOE_OK) return st;
    f->d_class_ptr = const_cast<int32_t*>(cp);
    f->d_class_parts = const_cast<int32_t*>(cq);
    f->ds.n_slices = f->sl.n_slices;
    f->ds.slots_max = f->sl.slots_max;
    f->ds.fbits = f->sl.fbits;
    // weighted CTA shares of a full-GPU launch (largest remainder, at least one CTA per slice)
    const int32_t ns = f->sl.n_slices;
    f->cta_start.clear();
    if (ns >= 1 && ns <= f->num_sms && (int32_t)f->sl.slice_work.size() == ns) {
      double tot = 0;
      for (double w : f->sl.slice_work) tot += w;
      std::vector<int32_t> c(ns, 1);
      int32_t left = f->num_sms - ns;
      std::vector<std::pair<double, int32_t>> rem;
      for (int32_t q = 0; q < ns; q++) {
        const double share = (double)f->num_sms * f->sl.slice_work[q] / tot - 1.0;
        const int32_t k = std::max(0, std::min(left, (int32_t)std::floor(share)));
        c[q] += k;
        left -= k;
        rem.push_back({share - k, q});
      }
      std::sort(rem.begin(), rem.end(), [](const std::pair<double, int32_t>& u, const std::pair<double, int32_t>& v) {
        return u.first != v.first ? u.first > v.first : u.second < v.second; });
      for (size_t q = 0; left > 0; q = (q + 1) % rem.size(), left--) c[rem[q].second]++;
      f->cta_start.assign(ns + 1, 0);
      for (int32_t q = 0; q < ns; q++) f->cta_start[q + 1] = f->cta_start[q] + c[q];
      const int32_t* dp = nullptr;
      if ((st = upload(f->cta_start, &dp)) != TAHOE_OK) return st;
      f->d_cta_start = const_cast<int32_t*>(dp);
    }
    if (f->sl.code_valid) {
      if ((st = upload(f->sl.cnodes, &f->ds.cnodes)) != TAHOE_OK) return st;
      if ((st = upload(f->sl.thr_tab, &f->ds.thr_tab)) != TAHOE_OK) return st;
      if ((st = upload(f->sl.thr_off, &f->ds.thr_off)) != TAHOE_OK) return st;
      if (!f->sl.code8 && (st = upload(f->sl.slot_attr, &f->ds.slot_attr)) != TAHOE_OK) return st;
      if ((st = upload(f->sl.col_mid, &f->ds.col_mid)) != TAHOE_OK) return st;
      f->ds.n_features = f->host.n_features;
      f->ds.n_thr = f->sl.thr_off.back();
      if (!f->sl.cb_img.empty()) {
        if ((st = upload(f->sl.cb_img, &f->ds.cb_img)) != TAHOE_OK) return st;
        if ((st = upload(f->sl.cb_desc, &f->ds.cb_desc)) != TAHOE_OK) return st;
        f->ds.cb_rows = f->sl.cb_rows;
        f->ds.cb_passes = f->sl.cb_passes;
      }
      if (f->sl.code8) {   // wide codes (reading R8)
        const int32_t* grp = nullptr;
        const int32_t* band = nullptr;
        if ((st = upload(f->sl.v_src, &f->ds.v_src)) != TAHOE_OK) return st;
        if ((st = upload(f->sl.c8_img, &f->ds.c8_img)) != TAHOE_OK) return st;
        if ((st = upload(f->sl.c8_grp, &grp)) != TAHOE_OK) return st;
        if ((st = upload(f->sl.c8_band, &band)) != TAHOE_OK) return st;
        f->ds.c8_grp = reinterpret_cast<const int4x*>(grp);
        f->ds.c8_band = reinterpret_cast<const int4x*>(band);
        f->ds.c8_bands = f->sl.c8_bands;
        // the TMA-staged pre-pass: every band at most kCode8BandGroups groups, its tables at most
        // kCode8TmaTables bytes and its source attributes one kCode8BoxW-float box (an imported layout
        // may come from another band plan)
        f->ds.c8_tma = 1;
        for (int32_t b = 0; b < f->sl.c8_bands; b++) {
          const int32_t* bd = &f->sl.c8_band[(size_t)b * 4];
          int32_t lo = INT32_MAX, hi = -1;
          for (int32_t v = bd[2] * 32; v < bd[3] * 32 && v < (int32_t)f->sl.v_src.size(); v++)
            if (f->sl.v_src[v] >= 0) { lo = std::min(lo, f->sl.v_src[v]); hi = std::max(hi, f->sl.v_src[v]); }
          if (bd[3] - bd[2] > kCode8BandGroups || bd[1] > kCode8TmaTables || (hi >= 0 && hi - (lo & ~3) >= kCode8BoxW) ||
              (hi >= 0 && f->sl.v_src[(size_t)bd[2] * 32] != lo))
            f->ds.c8_tma = 0;
        }
        f->ds.vfbits = f->sl.vfbits;
        f->ds.code8 = 1;
      }
      // slice weights for the coded kernels' slice switching (simulated lane-steps per row)
      std::vector<float> w(f->sl.slice_work.begin(), f->sl.slice_work.end());
      if (w.size() != (size_t)f->sl.n_slices) w.assign((size_t)f->sl.n_slices, 1.0f);
      if ((st = upload(w, &f->ds.slice_w)) != TAHOE_OK) return st;
    }
  }
  return TAHOE_OK;
}

static tahoe_status init_handle(tahoe_forest* f, int32_t device) {
  f->device = device;
  f->num_sms = 148;
  f->max_smem = kDefaultMaxSmem;
  if (device >= 0) {
    int cnt = 0;
    cudaError_t e = cudaGetDeviceCount(&cnt);
    if (e != cudaSuccess || device >= cnt) return fail(TAHOE_E_CUDA, "no such CUDA device");
    int v = 0;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device) == cudaSuccess) f->num_sms = v;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, device) == cudaSuccess) f->max_smem = v;
  }
  f->slot_budget = slot_budget_for(f->max_smem, f->host.n_features);
  if (const char* e = std::getenv("TAHOE_SLOT_BUDGET")) f->slot_budget = std::atoi(e);  // experiments
  return TAHOE_OK;
}

static PlanStats plan_stats(const tahoe_forest* f, int32_t d = -1) {
  PlanStats st;
  if (d < 0) d = f->host.n_features;
  st.wide_rows = d > 256;
  if (f->sl.valid) {
    const int64_t room = (int64_t)f->max_smem - (((f->sl.slots_max * kSlotBytes) + 1023) & ~1023) - kSlicedBarrierBytes;
    const int64_t ring = std::min<int64_t>(sliced_ring_bytes(d, f->sl.fbits, false) < 0 ? INT64_MAX : sliced_ring_bytes(d, f->sl.fbits, false),
                                           sliced_ring_bytes(d, f->sl.fbits, true) < 0 ? INT64_MAX : sliced_ring_bytes(d, f->sl.fbits, true));
    st.rows_global = ring > room;
  }
  for (double v : f->host.exp_reads) st.V += v;
  st.sliced_ok = f->sl.valid;
  static const bool codes_off = std::getenv("TAHOE_CODES") && std::string(std::getenv("TAHOE_CODES")) == "0";
  st.coded_ok = f->sl.valid && f->sl.code_valid && !codes_off;
  st.code_passes = std::max(1, (1 << f->sl.fbits) / 32);
  st.code8 = f->sl.code8;
  if (st.code8) st.code_passes = (1 << f->sl.vfbits) / 32;
  st.sliced_eff = f->sl.eff_sim;
  st.n_slices = f->sl.n_slices;
  st.num_sms = f->num_sms;
  st.n_trees = (int32_t)f->di.root.size();
  st.d = d;
  st.n_out = f->host.n_out();
  st.scalar = st.n_out == 1 && f->host.agg != TAHOE_AGG_VOTE;
  const int64_t rs = rows_smem_bytes(d, st.n_trees, f->host.n_out());
  st.rows_ok = rs <= (int64_t)f->max_smem - 1024;
  st.rows_per_sm = (int32_t)std::max<int64_t>(1, std::min<int64_t>(4, 232448 / (rs + 1024)));
  return st;
}

static int32_t choose(const tahoe_forest* f, int64_t n, int32_t d, int32_t forced) {
  if (forced < 0) {
    const char* env = std::getenv("TAHOE_FORCE_STRATEGY");
    if (env && *env) forced = std::atoi(env);
  }
  if (forced == TAHOE_STRATEGY_DIRECT) return TAHOE_STRATEGY_DIRECT;
  if (forced == TAHOE_STRATEGY_ROWS) return plan_stats(f, d).rows_ok ? TAHOE_STRATEGY_ROWS : -4;
  if (forced == TAHOE_STRATEGY_SLICED) return f->sl.valid ? TAHOE_STRATEGY_SLICED : -2;
  if (forced == TAHOE_STRATEGY_SLICED_CODED)
    return !f->sl.valid ? -2 : (f->ds.cnodes ? TAHOE_STRATEGY_SLICED_CODED : -3);
  // the cost model weighs the rank-coded twin of the sliced strategy (reading R7) wherever the
  // forest qualifies; $TAHOE_CODES=0 leaves it out (experiments)
  return select_strategy(plan_stats(f, d), n, d, f->host.agg);
}

static SlicedPlan sliced_plan(const tahoe_forest* f, const float* X, int64_t n, int32_t d) {
  SlicedPlan p;
  p.forest_smem = ((f->sl.slots_max * kSlotBytes) + 1023) & ~1023;
  const int32_t fb = f->sl.fbits;
  const int64_t room = (int64_t)f->max_smem - p.forest_smem - kSlicedBarrierBytes;
  const int64_t ring_p = padded_rows_possible(X, d) ? sliced_ring_bytes(d, fb, true) : -1;
  const int64_t ring_d = sliced_ring_bytes(d, fb, false);
  int64_t ring = 0;
  if (ring_p >= 0 && ring_p <= room) { p.rows = 2; ring = ring_p; }
  else if (ring_d >= 0 && ring_d <= room) { p.rows = 1; ring = ring_d; }
  else p.rows = 0;
  p.tile_rows = kSlicedTileRows;
  p.buf_floats = p.rows ? sliced_buf_floats(d, fb, p.rows == 2) : 0;
  p.row_stride = sliced_row_stride(d, fb, p.rows == 2);
  p.smem_bytes = p.forest_smem + (int32_t)ring + kSlicedBarrierBytes;
  const int32_t ns = f->sl.n_slices;
  if (ns <= f->num_sms) {
    // no more CTAs per slice than there are tiles: a small batch should not make 148 CTAs each
    // stage a ~200 KB slice for nothing
    const int64_t tiles = (n + p.tile_rows - 1) / p.tile_rows;
    p.cps = (int32_t)std::max<int64_t>(1, std::min<int64_t>(f->num_sms / ns, tiles));
    p.grid = ns * p.cps;
  } else {
    p.cps = 1;
    p.grid = f->num_sms;
  }
  p.block = 1024;
  return p;
}

// One batch on the device.  mode 0: final outputs; mode 1: raw fp64 partial [n x n_out].
static tahoe_status run(const tahoe_forest* f, const float* X, int64_t n, int32_t d, float* out,
                        int32_t* out_class, int32_t* out_leaf, uint64_t* out_fp, double* raw_user,
                        int32_t forced, cudaStream_t st, void* ev_b = nullptr, void* ev_e = nullptr,
                        double* prof = nullptr) {
  const Forest& H = f->host;
  const int32_t C = H.n_out();
  int32_t strat = choose(f, n, d, forced);
  if (strat == -2) return fail(TAHOE_E_UNSUPPORTED, "sliced strategy unavailable: " + f->sl.why_invalid);
  if (strat == -3) return fail(TAHOE_E_UNSUPPORTED, "rank-coded slices unavailable: " + f->sl.code_why);
  if (strat == -4) return fail(TAHOE_E_UNSUPPORTED, "rows strategy: row + per-tree values exceed shared memory");
  if (strat == TAHOE_STRATEGY_SLICED_CODED && !f->sl.code8) {
    // the code-tile ring (+ trailers and staged partials) must fit next to the slice
    const int64_t need = (((int64_t)f->sl.slots_max * kSlotBytes + 1023) & ~1023LL) +
                         coded_ring_smem(kSlicedRing, code_tile_stride(f->sl.fbits));
    if (need > f->max_smem) {
      if (forced == TAHOE_STRATEGY_SLICED_CODED)
        return fail(TAHOE_E_UNSUPPORTED, "rank-coded slices: code-tile ring does not fit shared memory");
      strat = TAHOE_STRATEGY_SLICED;
    }
  }
  cudaError_t e;
  if (out_fp && (e = cudaMemsetAsync(out_fp, 0, (size_t)n * 8, st)) != cudaSuccess) return cuda_fail(e, "memset");
  OutArgs o;
  o.out = out;
  o.out_class = out_class;
  o.out_leaf = out_leaf;
  o.out_fp = out_fp;
  o.agg = H.agg;
  o.base = H.base;
  o.n_trees_full = H.n_trees_full;
  o.n_classes = C;
  o.T_leaf = H.n_trees_full;
  FinalizeArgs fa;
  fa.n_classes = C;
  fa.agg = H.agg;
  fa.base = H.base;
  fa.n_trees_full = H.n_trees_full;
  fa.n = n;
  fa.out = out;
  fa.out_class = out_class;
  fa.raw_out = raw_user;
  const bool scalar = C == 1 && H.agg != TAHOE_AGG_VOTE;
  if (strat == TAHOE_STRATEGY_ROWS) {   // one launch: walk + combine + finalize (or raw sums)
    o.raw = raw_user;
    if (ev_b) cudaEventRecord(static_cast<cudaEvent_t>(ev_b), st);
    const int rc = launch_rows(f->dd, X, n, d, o, f->num_sms, st);
    if (ev_e) cudaEventRecord(static_cast<cudaEvent_t>(ev_e), st);
    if (rc) return cuda_fail((cudaError_t)rc, "rows kernel");
    return TAHOE_OK;
  }
  if (strat == TAHOE_STRATEGY_DIRECT) {
    const size_t nchunks = f->direct_chunks.size() - 1;
    if (scalar && !raw_user && nchunks == 1) {
      if (ev_b) cudaEventRecord(static_cast<cudaEvent_t>(ev_b), st);
      int rc = launch_direct(f->dd, X, n, d, o, true, f->num_sms, st);
      if (ev_e) cudaEventRecord(static_cast<cudaEvent_t>(ev_e), st);
      if (rc) return cuda_fail((cudaError_t)rc, "direct kernel");
      return TAHOE_OK;
    }
    double* raw = raw_user;
    if (!raw && (e = scratch_alloc((void**)&raw, (size_t)n * C * 8, st)) != cudaSuccess)
      return fail(TAHOE_E_NOMEM, "cudaMallocAsync partial");
    if ((e = cudaMemsetAsync(raw, 0, (size_t)n * C * 8, st)) != cudaSuccess) {
      if (!raw_user) cudaFreeAsync(raw, st);
      return cuda_fail(e, "memset");
    }
    o.raw = raw;
    if (ev_b) cudaEventRecord(static_cast<cudaEvent_t>(ev_b), st);
    int rc = 0;
    for (size_t c = 0; c < nchunks && !rc; c++) {   // raw += each chunk's per-class sums
      DevDirect dc = f->dd;
      const int32_t s0 = f->direct_chunks[c], s1 = f->direct_chunks[c + 1];
      dc.root += s0;
      dc.cls += s0;
      dc.tree_orig += s0;
      dc.n_slots = s1 - s0;
      rc = launch_direct(dc, X, n, d, o, false, f->num_sms, st);
    }
    if (ev_e) cudaEventRecord(static_cast<cudaEvent_t>(ev_e), st);
    if (rc) {
      if (!raw_user) cudaFreeAsync(raw, st);
      return cuda_fail((cudaError_t)rc, "direct kernel");
    }
    if (!raw_user) {
      fa.partial = raw;
      fa.part_stride = 1;
      fa.row_stride = C;
      rc = launch_finalize(fa, st);
      cudaFreeAsync(raw, st);
      if (rc) return cuda_fail((cudaError_t)rc, "finalize kernel");
    }
    return TAHOE_OK;
  }
  // sliced
  const SlicedPlan plan = sliced_plan(f, X, n, d);
  const bool fused = scalar && !raw_user && f->sl.n_slices == 1;
  double* part = nullptr;
  if (!fused) {
    if ((e = scratch_alloc((void**)&part, (size_t)f->sl.n_slices * n * 8, st)) != cudaSuccess)
      return fail(TAHOE_E_NOMEM, "cudaMallocAsync partial");
    o.raw = part;
  }
  int rc;
  fa.partial = part;
  fa.part_stride = n;
  fa.row_stride = 1;
  fa.class_ptr = f->d_class_ptr;
  fa.class_parts = f->d_class_parts;
  if (strat == TAHOE_STRATEGY_SLICED_CODED && f->sl.code8) {
    // wide codes (reading R8): u8 code tiles + NaN flags from the library pool
    const int64_t ntiles = (code8_chunk_rows(f->sl.vfbits, n) + kCode8TileRows - 1) / kCode8TileRows;
    const size_t cbytes = (size_t)ntiles * (size_t)(code8_tile_bytes(f->sl.vfbits) + 16) +
                          (size_t)f->sl.n_slices * 8;
    void* cbuf = nullptr;
    if ((e = scratch_alloc(&cbuf, cbytes, st)) != cudaSuccess) {
      if (part) cudaFreeAsync(part, st);
      return fail(TAHOE_E_NOMEM, "cudaMallocAsync code tiles");
    }
    SlicedPlan cp = plan;
    cp.cta_start = f->d_cta_start;   // used per chunk once it has a few tiles per CTA
    rc = launch_sliced_codes8(f->ds, cp, X, n, d, static_cast<uint8_t*>(cbuf), o, fused,
                              f->num_sms, st, ev_b, ev_e);
    cudaFreeAsync(cbuf, st);
  } else if (strat == TAHOE_STRATEGY_SLICED_CODED) {
    const int64_t ntiles = (n + kSlicedTileRows - 1) / kSlicedTileRows;
    // code tiles, then per-slice tile / CTA counters (dynamic tile claiming, slice switching)
    const size_t cbytes = (size_t)ntiles * code_tile_stride(f->sl.fbits) + (size_t)f->sl.n_slices * 8;
    void* cbuf = nullptr;
    if ((e = scratch_alloc(&cbuf, cbytes, st)) != cudaSuccess) {
      if (part) cudaFreeAsync(part, st);
      return fail(TAHOE_E_NOMEM, "cudaMallocAsync code tiles");
    }
    SlicedPlan cp = plan;
    // a full GPU of CTAs, shared out among the slices by their simulated work, once every CTA has
    // at least a few tiles
    if (f->d_cta_start && ntiles >= 4LL * f->num_sms) {
      cp.grid = f->num_sms;
      cp.cta_start = f->d_cta_start;
    }
    rc = launch_sliced_codes(f->ds, cp, X, n, d, static_cast<uint16_t*>(cbuf), o, fused,
                             f->num_sms, st, ev_b, ev_e, prof);
    cudaFreeAsync(cbuf, st);
  } else {
    if (ev_b) cudaEventRecord(static_cast<cudaEvent_t>(ev_b), st);
    rc = launch_sliced(f->ds, plan, X, n, d, o, fused, st);
    if (ev_e) cudaEventRecord(static_cast<cudaEvent_t>(ev_e), st);
  }
  if (rc) { if (part) cudaFreeAsync(part, st); return cuda_fail((cudaError_t)rc, "sliced kernel"); }
  if (!fused) {
    rc = launch_finalize(fa, st);
    cudaFreeAsync(part, st);
    if (rc) return cuda_fail((cudaError_t)rc, "finalize kernel");
  }
  return TAHOE_OK;
}

static tahoe_status check_predict(const tahoe_forest* f, const float* X, int64_t n, int32_t d,
                                  const void* out) {
  if (!f) return fail(TAHOE_E_INVAL, "NULL forest");
  if (n < 0) return fail(TAHOE_E_INVAL, "n < 0");
  if (f->device < 0) return fail(TAHOE_E_STATE, "host-only forest handle (device = -1)");
  if (n == 0) return TAHOE_OK;
  if (!X || !out) return fail(TAHOE_E_INVAL, "NULL X or output pointer");
  if (d < f->host.max_feature + 1 || d < 1)
    return fail(TAHOE_E_INVAL, "d = " + std::to_string(d) + " < largest attribute index + 1 (" +
                                   std::to_string(f->host.max_feature + 1) + ")");
  return TAHOE_OK;
}

}  // namespace tahoe

using namespace tahoe;

#define TAHOE_GUARD_BEGIN try {
#define TAHOE_GUARD_END                                                         \
  }                                                                             \
  catch (const std::bad_alloc&) { return fail(TAHOE_E_NOMEM, "host allocation failed"); } \
  catch (const std::exception& ex) { return fail(TAHOE_E_INVAL, ex.what()); }  \
  catch (...) { return fail(TAHOE_E_INVAL, "unknown exception"); }

// ---- layout state export / import (ship a laid-out forest to other ranks without re-running
// calibration, similarity detection and balancing; SURVEY §8(e) tree sharding)
namespace {
struct BlobW {
  std::vector<uint8_t> b;
  template <class T> void put(const T& v) { const uint8_t* p = reinterpret_cast<const uint8_t*>(&v); b.insert(b.end(), p, p + sizeof(T)); }
  template <class T> void vec(const std::vector<T>& v) {
    put<int64_t>((int64_t)v.size());
    const uint8_t* p = reinterpret_cast<const uint8_t*>(v.data());
    b.insert(b.end(), p, p + v.size() * sizeof(T));
  }
};
struct BlobR {
  const uint8_t* p; int64_t n, o = 0;
  template <class T> bool get(T& v) { if (o + (int64_t)sizeof(T) > n) return false; std::memcpy(&v, p + o, sizeof(T)); o += sizeof(T); return true; }
  template <class T> bool vec(std::vector<T>& v) {
    int64_t k;
    if (!get(k) || k < 0 || o + k * (int64_t)sizeof(T) > n) return false;
    v.resize((size_t)k);
    std::memcpy(v.data(), p + o, (size_t)k * sizeof(T));
    o += k * (int64_t)sizeof(T);
    return true;
  }
};
constexpr uint32_t kLayoutMagic = 0x59414c54u;   // "TLAY"
}  // namespace

extern "C" {

__attribute__((visibility("default"))) const char* tahoe_last_error(void) { return g_err.c_str(); }

__attribute__((visibility("default"))) tahoe_status tahoe_forest_build(
    int32_t n_trees, const int32_t* root, int32_t n_nodes, const int32_t* feature,
    const float* threshold, const int32_t* left, const int32_t* right, const float* leaf_value,
    const uint8_t* default_left, const int32_t* tree_class, int32_t n_features, int32_t n_classes,
    tahoe_agg agg, float base_score, int32_t device, tahoe_forest** out) {
  TAHOE_GUARD_BEGIN
  if (!out) return fail(TAHOE_E_INVAL, "NULL out");
  *out = nullptr;
  tahoe_forest* f = new tahoe_forest();
  tahoe_status st = build_forest(f->host, n_trees, root, n_nodes, feature, threshold, left, right,
                                 leaf_value, default_left, tree_class, n_features, n_classes,
                                 (int32_t)agg, base_score);
  if (st == TAHOE_OK) st = init_handle(f, device);
  if (st == TAHOE_OK) st = encode_and_upload(f);
  if (st != TAHOE_OK) { free_device(f); delete f; return st; }
  *out = f;
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_forest_layout(
    tahoe_forest* f, const float* X_calib_host, int64_t n_calib, int32_t d,
    const tahoe_layout_opts* opts) {
  TAHOE_GUARD_BEGIN
  if (!f) return fail(TAHOE_E_INVAL, "NULL forest");
  if (n_calib < 0 || (n_calib > 0 && !X_calib_host)) return fail(TAHOE_E_INVAL, "bad calibration set");
  if (n_calib > 0 && d < f->host.max_feature + 1) return fail(TAHOE_E_INVAL, "calibration d too small");
  tahoe_layout_opts o{};
  if (opts) o = *opts;
  else { o.node_reorder = 1; o.tree_group = 1; }
  if (o.t_nodes <= 0) o.t_nodes = 4;
  if (o.l_hash <= 0) o.l_hash = 128;
  if (o.m_chunks <= 0) o.m_chunks = 64;
  if (o.m_chunks > o.l_hash) return fail(TAHOE_E_INVAL, "m_chunks > l_hash");
  Forest& F = f->host;
  F.opts = o;
  if (n_calib > 0) {
    calibrate(F, X_calib_host, n_calib, d);
    // keep an evenly spaced subsample of the calibration rows for the lockstep simulation
    const int64_t m = std::min<int64_t>(n_calib, 1024);
    F.dsim = d;
    F.Xsim.resize((size_t)m * d);
    for (int64_t r = 0; r < m; r++)
      std::memcpy(&F.Xsim[(size_t)r * d], X_calib_host + (r * n_calib / m) * d, (size_t)d * 4);
  }
  reorder_nodes(F, o.node_reorder != 0);
  order_trees(F);
  return encode_and_upload(f);
  TAHOE_GUARD_END
}

static tahoe_status layout_opts_fill(const tahoe_layout_opts* opts, tahoe_layout_opts* o) {
  *o = tahoe_layout_opts{};
  if (opts) *o = *opts;
  else { o->node_reorder = 1; o->tree_group = 1; }
  if (o->t_nodes <= 0) o->t_nodes = 4;
  if (o->l_hash <= 0) o->l_hash = 128;
  if (o->m_chunks <= 0) o->m_chunks = 64;
  if (o->m_chunks > o->l_hash) return fail(TAHOE_E_INVAL, "m_chunks > l_hash");
  return TAHOE_OK;
}


__attribute__((visibility("default"))) tahoe_status tahoe_forest_layout_export(
    const tahoe_forest* f, void* buf, int64_t cap, int64_t* size) {
  TAHOE_GUARD_BEGIN
  if (!f || !size) return fail(TAHOE_E_INVAL, "NULL argument");
  const Forest& F = f->host;
  BlobW w;
  w.put<uint32_t>(kLayoutMagic);
  w.put<int32_t>(1);                                     // version
  w.put<int32_t>(F.n_trees);
  w.put<int64_t>((int64_t)F.feat.size());
  w.put(F.opts);
  w.put<int32_t>(F.calibrated ? 1 : 0);
  w.put<int64_t>(F.n_cal);
  w.put<int32_t>(F.dsim);
  w.vec(F.count);
  w.vec(F.hot_left);
  w.vec(F.exp_reads);
  w.vec(F.order);
  w.vec(F.Xsim);
  *size = (int64_t)w.b.size();
  if (!buf) return TAHOE_OK;
  if (cap < *size) return fail(TAHOE_E_INVAL, "buffer too small");
  std::memcpy(buf, w.b.data(), w.b.size());
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_forest_layout_import(
    tahoe_forest* f, const void* buf, int64_t size) {
  TAHOE_GUARD_BEGIN
  if (!f || !buf || size <= 0) return fail(TAHOE_E_INVAL, "bad argument");
  Forest& F = f->host;
  BlobR r{static_cast<const uint8_t*>(buf), size};
  uint32_t magic = 0;
  int32_t ver = 0, T = 0, cal = 0, dsim = 0;
  int64_t N = 0, ncal = 0;
  tahoe_layout_opts opts{};
  Forest G = F;   // applied only when the whole blob parses and matches this forest
  bool ok = r.get(magic) && magic == kLayoutMagic && r.get(ver) && ver == 1 && r.get(T) &&
            r.get(N) && r.get(opts) && r.get(cal) && r.get(ncal) && r.get(dsim) &&
            r.vec(G.count) && r.vec(G.hot_left) && r.vec(G.exp_reads) && r.vec(G.order) &&
            r.vec(G.Xsim) && r.o == size;
  if (!ok) return fail(TAHOE_E_INVAL, "not a layout state blob");
  if (T != F.n_trees || N != (int64_t)F.feat.size() || (int64_t)G.count.size() != N ||
      (int64_t)G.hot_left.size() != N || (int64_t)G.exp_reads.size() != T || (int64_t)G.order.size() != T ||
      (dsim > 0 && (int64_t)G.Xsim.size() % dsim != 0))
    return fail(TAHOE_E_INVAL, "layout state does not match this forest");
  std::vector<int32_t> seen((size_t)T, 0);
  for (int32_t t : G.order) {
    if (t < 0 || t >= T || seen[t]++) return fail(TAHOE_E_INVAL, "layout state: bad tree order");
  }
  G.opts = opts;
  G.calibrated = cal != 0;
  G.n_cal = ncal;
  G.dsim = dsim;
  F = std::move(G);
  return encode_and_upload(f);
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_count_visits(
    const tahoe_forest* f, const float* X, int64_t n, int32_t d, uint32_t* counts,
    tahoe_stream stream) {
  TAHOE_GUARD_BEGIN
  tahoe_status st = check_predict(f, X, n, d, counts);
  if (st != TAHOE_OK || n == 0) return st;
  DeviceGuard g(f->device);
  int rc = launch_count_visits(f->dd, X, n, d, counts, f->num_sms, reinterpret_cast<cudaStream_t>(stream));
  if (rc) return cuda_fail((cudaError_t)rc, "visit-count kernel");
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_forest_layout_counts(
    tahoe_forest* f, const uint64_t* counts, int64_t n_calib, const float* X_sim_host,
    int64_t n_sim, int32_t d, const tahoe_layout_opts* opts) {
  TAHOE_GUARD_BEGIN
  if (!f || !counts || n_calib < 1) return fail(TAHOE_E_INVAL, "bad argument");
  if (n_sim > 0 && (!X_sim_host || d < f->host.max_feature + 1)) return fail(TAHOE_E_INVAL, "bad simulation rows");
  tahoe_layout_opts o;
  tahoe_status st = layout_opts_fill(opts, &o);
  if (st != TAHOE_OK) return st;
  Forest& F = f->host;
  F.opts = o;
  set_counts(F, counts, n_calib);
  F.Xsim.clear();
  F.dsim = 0;
  if (n_sim > 0) {
    const int64_t m = std::min<int64_t>(n_sim, 1024);
    F.dsim = d;
    F.Xsim.resize((size_t)m * d);
    for (int64_t r = 0; r < m; r++)
      std::memcpy(&F.Xsim[(size_t)r * d], X_sim_host + (r * n_sim / m) * d, (size_t)d * 4);
  }
  reorder_nodes(F, o.node_reorder != 0);
  order_trees(F);
  return encode_and_upload(f);
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_forest_l2_persist(
    const tahoe_forest* f, tahoe_stream stream, float hit_ratio) {
  TAHOE_GUARD_BEGIN
  if (!f) return fail(TAHOE_E_INVAL, "NULL forest");
  if (f->device < 0) return fail(TAHOE_E_STATE, "host-only forest handle");
  DeviceGuard g(f->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const void* base = f->sl.valid ? (const void*)f->ds.nodes : (const void*)f->dd.nodes;
  size_t bytes = f->sl.valid ? (size_t)f->sl.bytes() : (size_t)f->di.bytes();
  int max_persist = 0, max_window = 0;
  cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, f->device);
  cudaDeviceGetAttribute(&max_window, cudaDevAttrMaxAccessPolicyWindowSize, f->device);
  cudaStreamAttrValue v = {};
  if (hit_ratio > 0.0f && max_persist > 0 && max_window > 0) {
    bytes = std::min(bytes, (size_t)max_window);
    cudaError_t e = cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min(bytes, (size_t)max_persist));
    if (e != cudaSuccess) return cuda_fail(e, "cudaDeviceSetLimit");
    v.accessPolicyWindow.base_ptr = const_cast<void*>(base);
    v.accessPolicyWindow.num_bytes = bytes;
    v.accessPolicyWindow.hitRatio = std::min(1.0f, hit_ratio);
    v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
    v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
  }
  cudaError_t e = cudaStreamSetAttribute(st, cudaStreamAttributeAccessPolicyWindow, &v);
  if (e != cudaSuccess) return cuda_fail(e, "cudaStreamSetAttribute");
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_predict_ex(
    const tahoe_forest* f, const float* X, int64_t n, int32_t d, float* out,
    const tahoe_predict_opts* opts, tahoe_stream stream) {
  TAHOE_GUARD_BEGIN
  tahoe_status st = check_predict(f, X, n, d, out);
  if (st != TAHOE_OK || n == 0) return st;
  DeviceGuard g(f->device);
  tahoe_predict_opts o{};
  o.force_strategy = -1;
  if (opts) o = *opts;
  return run(f, X, n, d, out, o.out_class, o.out_leaf, o.out_fingerprint, nullptr, o.force_strategy,
             reinterpret_cast<cudaStream_t>(stream), o.ev_main_begin, o.ev_main_end);
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_profile_walk(
    const tahoe_forest* f, const float* X, int64_t n, int32_t d, float* out, double* stats,
    tahoe_stream stream) {
  TAHOE_GUARD_BEGIN
  tahoe_status st = check_predict(f, X, n, d, out);
  if (st != TAHOE_OK || n == 0) return st;
  if (!stats) return fail(TAHOE_E_INVAL, "NULL stats");
  if (!f->sl.valid || !f->ds.cnodes || f->sl.code8)
    return fail(TAHOE_E_UNSUPPORTED, "walk profiling needs the u16 rank-coded slices");
  DeviceGuard g(f->device);
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  double* dev = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&dev, 8 * sizeof(double), s);
  if (e == cudaSuccess) e = cudaMemsetAsync(dev, 0, 8 * sizeof(double), s);
  if (e != cudaSuccess) return cuda_fail(e, "profile buffer");
  st = run(f, X, n, d, out, nullptr, nullptr, nullptr, nullptr, TAHOE_STRATEGY_SLICED_CODED, s,
           nullptr, nullptr, dev);
  if (st == TAHOE_OK) {
    e = cudaMemcpyAsync(stats, dev, 8 * sizeof(double), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  }
  cudaFreeAsync(dev, s);
  if (st != TAHOE_OK) return st;
  if (e != cudaSuccess) return cuda_fail(e, "profile readback");
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_predict(
    const tahoe_forest* f, const float* X, int64_t n, int32_t d, float* out, tahoe_stream stream) {
  return tahoe_predict_ex(f, X, n, d, out, nullptr, stream);
}

__attribute__((visibility("default"))) tahoe_status tahoe_predict_host(
    const tahoe_forest* f, const float* X_host, int64_t n, int32_t d, float* out_host,
    int32_t* class_host, tahoe_stream stream) {
  TAHOE_GUARD_BEGIN
  tahoe_status st = check_predict(f, X_host, n, d, out_host);
  if (st != TAHOE_OK || n == 0) return st;
  DeviceGuard g(f->device);
  cudaStream_t user = reinterpret_cast<cudaStream_t>(stream);
  const int32_t C = f->host.n_out();
  // Chunks overlap H2D / compute / D2H on three streams: 8 chunks of >= 64K rows.  The time is
  // about H2D of every row plus the compute of the last chunk, as long as a chunk's compute (fixed
  // launch / tail cost + per-row cost) stays below its H2D; 16 equal chunks, and 8 chunks followed
  // by halving tail chunks, measured slower (more fixed per-chunk cost).  Three buffers, so a copy
  // never waits for the compute of the chunk before the previous one.
  int64_t chunk = std::min<int64_t>(n, std::max<int64_t>(65536, (n + 7) / 8));
  std::vector<int64_t> cuts;
  // ramp ($TAHOE_HOST_RAMP, default on for >= 1M rows; C2's 1M rows: 365-368 -> 374-391 M samples/s
  // same box): the pipeline's fill (H2D of the first
  // chunk) and drain (compute of the last) are what the overlap cannot hide, so the first and last
  // chunks are small (n/64, n/32, ... doubling up to n/16 in the middle): a few more launches,
  // each worth its fixed cost only when the batch is large
  static const int ramp_env = std::getenv("TAHOE_HOST_RAMP") ? std::atoi(std::getenv("TAHOE_HOST_RAMP")) : -1;
  const bool ramp = ramp_env >= 0 ? ramp_env != 0 : n >= 1000000;
  if (ramp) {
    chunk = std::max<int64_t>(65536, (n + 15) / 16);
    std::vector<int64_t> head, tail;
    int64_t left = n;
    for (int64_t s = std::max<int64_t>(65536, n / 64); s < chunk && left > 4 * s; s *= 2) {
      head.push_back(s);
      tail.push_back(s);
      left -= 2 * s;
    }
    std::vector<int64_t> sizes(head);
    for (; left > 0; left -= std::min(left, chunk)) sizes.push_back(std::min(left, chunk));
    sizes.insert(sizes.end(), tail.rbegin(), tail.rend());
    int64_t r = 0;
    for (int64_t z : sizes) { cuts.push_back(r); r += z; }
  } else {
    for (int64_t r = 0; r < n; r += chunk) cuts.push_back(r);
  }
  cuts.push_back(n);
  const int64_t nchunks = (int64_t)cuts.size() - 1;
  constexpr int NB = 3;
  tahoe_forest* fm = const_cast<tahoe_forest*>(f);   // the pipe is handle-owned scratch state
  std::lock_guard<std::mutex> lock(fm->host_mu);
  if (cudaError_t ie = init_host_pipe(fm)) return cuda_fail(ie, "tahoe_predict_host streams");
  // chunks alternate between two compute streams, so the next chunk's pre-pass and walk start on
  // the SMs the previous walk's tail releases (one compute stream: every chunk's tail idled the GPU)
  cudaStream_t s_in = fm->hp.s_in, s_out = fm->hp.s_out;
  cudaStream_t s_cmps[2] = {fm->hp.s_cmp, fm->hp.s_cmp2};
  static const int two_env = std::getenv("TAHOE_HOST_STREAMS") ? std::atoi(std::getenv("TAHOE_HOST_STREAMS")) : 2;
  const int ncmp = two_env == 1 ? 1 : 2;
  cudaEvent_t ev_start = fm->hp.ev_start;
  cudaEvent_t* ev_in = fm->hp.ev_in;
  cudaEvent_t* ev_cmp = fm->hp.ev_cmp;
  cudaEvent_t* ev_out = fm->hp.ev_out;
  const int64_t nbuf = std::min<int64_t>(NB, nchunks);
  float* dX = nullptr;
  float* dO = nullptr;
  int32_t* dC = nullptr;
  cudaError_t e = scratch_alloc((void**)&dX, (size_t)nbuf * chunk * d * 4, user);
  if (e == cudaSuccess) e = scratch_alloc((void**)&dO, (size_t)nbuf * chunk * C * 4, user);
  if (e == cudaSuccess && class_host) e = scratch_alloc((void**)&dC, (size_t)nbuf * chunk * 4, user);
  cudaEventRecord(ev_start, user);
  cudaStreamWaitEvent(s_in, ev_start, 0);
  cudaStreamWaitEvent(s_cmps[0], ev_start, 0);
  cudaStreamWaitEvent(s_cmps[1], ev_start, 0);
  cudaStreamWaitEvent(s_out, ev_start, 0);
  for (int64_t c = 0; c < nchunks && e == cudaSuccess && st == TAHOE_OK; c++) {
    const int b = (int)(c % NB);
    cudaStream_t s_cmp = s_cmps[c % ncmp];
    const int64_t r0 = cuts[c], nr = cuts[c + 1] - cuts[c];
    float* xb = dX + (size_t)b * chunk * d;
    float* ob = dO + (size_t)b * chunk * C;
    int32_t* cb = dC ? dC + (size_t)b * chunk : nullptr;
    if (c >= NB) cudaStreamWaitEvent(s_in, ev_cmp[b], 0);    // X buffer consumed by chunk c-NB
    e = cudaMemcpyAsync(xb, X_host + r0 * d, (size_t)nr * d * 4, cudaMemcpyHostToDevice, s_in);
    cudaEventRecord(ev_in[b], s_in);
    cudaStreamWaitEvent(s_cmp, ev_in[b], 0);
    if (c >= NB) cudaStreamWaitEvent(s_cmp, ev_out[b], 0);   // out buffer drained by chunk c-NB
    if (e == cudaSuccess)
      st = run(f, xb, nr, d, ob, cb, nullptr, nullptr, nullptr, -1, s_cmp);
    cudaEventRecord(ev_cmp[b], s_cmp);
    cudaStreamWaitEvent(s_out, ev_cmp[b], 0);
    if (e == cudaSuccess) e = cudaMemcpyAsync(out_host + r0 * C, ob, (size_t)nr * C * 4, cudaMemcpyDeviceToHost, s_out);
    if (e == cudaSuccess && cb) e = cudaMemcpyAsync(class_host + r0, cb, (size_t)nr * 4, cudaMemcpyDeviceToHost, s_out);
    cudaEventRecord(ev_out[b], s_out);
  }
  cudaEventRecord(ev_in[0], s_in);
  cudaEventRecord(ev_cmp[0], s_cmps[0]);
  cudaEventRecord(ev_cmp[1], s_cmps[1]);
  cudaEventRecord(ev_out[0], s_out);
  cudaStreamWaitEvent(user, ev_in[0], 0);
  cudaStreamWaitEvent(user, ev_cmp[0], 0);
  cudaStreamWaitEvent(user, ev_cmp[1], 0);
  cudaStreamWaitEvent(user, ev_out[0], 0);
  if (dX) cudaFreeAsync(dX, user);
  if (dO) cudaFreeAsync(dO, user);
  if (dC) cudaFreeAsync(dC, user);
  if (st != TAHOE_OK) return st;
  if (e != cudaSuccess) return cuda_fail(e, "tahoe_predict_host");
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_measure_visit_rate(
    int32_t device, int32_t variant, int32_t steps, int32_t reps, double* node_reads_per_s,
    double* smem_bytes_per_clk) {
  TAHOE_GUARD_BEGIN
  // variant 0 tests its exit every four steps per chain (walk_coded2): steps a multiple of 4;
  // variant 1 walks each half column (steps / 2 slots) four steps per exit test: a multiple of 8
  if (variant < 0 || variant > 2 || steps < 2 || (steps & 1) || (variant == 0 && (steps & 3)) ||
      (variant == 1 && (steps & 7)) || steps > 600 ||
      reps < 1 || !node_reads_per_s)
    return fail(TAHOE_E_INVAL, "bad microbenchmark arguments");
  DeviceGuard g(device);
  if (!g.ok) return fail(TAHOE_E_CUDA, "cannot select device");
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
  cudaStream_t st;
  cudaError_t e = cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  if (e != cudaSuccess) return cuda_fail(e, "stream");
  double* sink = nullptr;
  unsigned long long* cyc = nullptr;
  uint32_t* sink2 = nullptr;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  e = cudaMalloc(&sink, (size_t)sms * 8);
  if (e == cudaSuccess) e = cudaMalloc(&cyc, (size_t)sms * 8);
  if (e == cudaSuccess) e = cudaMalloc(&sink2, (size_t)sms * 4);
  int rc = e == cudaSuccess ? 0 : (int)e;
  float ms = 0.0f;
  if (variant == 2) {
    // the direct walk: 4096 internal nodes whose hot child is the next one (attribute = slot % 100,
    // threshold +inf so "x < b" holds, hot = left), 4 CTAs of 512 threads per SM
    std::vector<uint32_t> h(2 * 4096);
    for (uint32_t q = 0; q < 4096; q++) {
      h[2 * q] = 0x7f800000u;
      h[2 * q + 1] = kHotLeftBit | (1u << 7) | (q % 100u);
    }
    void* nodes = nullptr;
    if (!rc) rc = (int)cudaMalloc(&nodes, h.size() * 4);
    if (!rc) rc = (int)cudaMemcpy(nodes, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    const int grid = sms * 4, total = steps * reps;
    if (!rc) rc = launch_visit_peak_direct(nodes, total / 8, grid, sink, st);   // warm-up
    if (!rc) {
      cudaEventRecord(a, st);
      rc = launch_visit_peak_direct(nodes, total, grid, sink, st);
      cudaEventRecord(b, st);
    }
    if (!rc) rc = (int)cudaStreamSynchronize(st);
    if (!rc) {
      cudaEventElapsedTime(&ms, a, b);
      *node_reads_per_s = (double)grid * 512.0 * (double)total / (ms / 1000.0);
    }
    cudaFree(nodes);
  } else {
    if (!rc) rc = launch_visit_peak(variant, steps, std::max(1, reps / 8), sms, sink, st);   // warm-up
    if (!rc) {
      cudaEventRecord(a, st);
      rc = launch_visit_peak(variant, steps, reps, sms, sink, st);
      cudaEventRecord(b, st);
    }
    if (!rc) rc = (int)cudaStreamSynchronize(st);
    if (!rc) {
      cudaEventElapsedTime(&ms, a, b);
      *node_reads_per_s = (double)sms * 1024.0 * 2.0 * steps * (double)reps / (ms / 1000.0);
    }
  }
  if (!rc && smem_bytes_per_clk) {
    const int iters = 4096;
    rc = launch_smem_bw(iters, sms, cyc, sink2, st);
    if (!rc) rc = (int)cudaStreamSynchronize(st);
    if (!rc) {
      std::vector<unsigned long long> c((size_t)sms);
      rc = (int)cudaMemcpy(c.data(), cyc, (size_t)sms * 8, cudaMemcpyDeviceToHost);
      double mean = 0.0;
      for (unsigned long long v : c) mean += (double)v / sms;
      *smem_bytes_per_clk = 1024.0 * 16.0 * 8.0 * iters / mean;
    }
  }
  cudaFree(sink);
  cudaFree(cyc);
  cudaFree(sink2);
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaStreamDestroy(st);
  if (rc) return cuda_fail((cudaError_t)rc, "microbenchmark");
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_forest_shard(
    const tahoe_forest* f, int32_t rank, int32_t world, int32_t device, tahoe_forest** shard) {
  TAHOE_GUARD_BEGIN
  if (!f || !shard) return fail(TAHOE_E_INVAL, "NULL argument");
  if (world < 1 || rank < 0 || rank >= world) return fail(TAHOE_E_INVAL, "bad rank/world");
  *shard = nullptr;
  tahoe_forest* s = new tahoe_forest();
  s->host = make_shard(f->host, rank, world);
  if (s->host.n_trees == 0) { delete s; return fail(TAHOE_E_INVAL, "shard has no trees (world > n_trees)"); }
  tahoe_status st = init_handle(s, device);
  if (st == TAHOE_OK) st = encode_and_upload(s);
  if (st != TAHOE_OK) { free_device(s); delete s; return st; }
  *shard = s;
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_predict_partial(
    const tahoe_forest* shard, const float* X, int64_t n, int32_t d, double* partial,
    tahoe_stream stream) {
  TAHOE_GUARD_BEGIN
  tahoe_status st = check_predict(shard, X, n, d, partial);
  if (st != TAHOE_OK || n == 0) return st;
  DeviceGuard g(shard->device);
  return run(shard, X, n, d, nullptr, nullptr, nullptr, nullptr, partial, -1,
             reinterpret_cast<cudaStream_t>(stream));
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_finalize(
    const tahoe_forest* full, const double* partial, int64_t n, float* out, int32_t* out_class,
    tahoe_stream stream) {
  TAHOE_GUARD_BEGIN
  if (!full) return fail(TAHOE_E_INVAL, "NULL forest");
  if (n < 0) return fail(TAHOE_E_INVAL, "n < 0");
  if (full->device < 0) return fail(TAHOE_E_STATE, "host-only forest handle");
  if (n == 0) return TAHOE_OK;
  if (!partial || !out) return fail(TAHOE_E_INVAL, "NULL pointer");
  DeviceGuard g(full->device);
  const Forest& H = full->host;
  FinalizeArgs fa;
  fa.partial = partial;
  fa.part_stride = 1;
  fa.row_stride = H.n_out();
  fa.n_classes = H.n_out();
  fa.agg = H.agg;
  fa.base = H.base;
  fa.n_trees_full = H.n_trees_full;
  fa.n = n;
  fa.out = out;
  fa.out_class = out_class;
  int rc = launch_finalize(fa, reinterpret_cast<cudaStream_t>(stream));
  if (rc) return cuda_fail((cudaError_t)rc, "finalize kernel");
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) int32_t tahoe_forest_n_outputs(const tahoe_forest* f) {
  return f ? f->host.n_out() : -1;
}
__attribute__((visibility("default"))) int32_t tahoe_forest_n_trees(const tahoe_forest* f) {
  return f ? f->host.n_trees : -1;
}

__attribute__((visibility("default"))) int32_t tahoe_select_strategy(const tahoe_forest* f,
                                                                     int64_t n, int32_t d) {
  if (!f) return -1;
  return choose(f, n, d, -1);
}

__attribute__((visibility("default"))) double tahoe_predict_cost_us(const tahoe_forest* f,
                                                                   int32_t strategy, int64_t n) {
  if (!f) return -1.0;
  return predict_us(plan_stats(f), strategy, n);
}

__attribute__((visibility("default"))) tahoe_status tahoe_forest_stats(const tahoe_forest* f,
                                                                       char* buf, int64_t len) {
  TAHOE_GUARD_BEGIN
  if (!f || !buf || len <= 0) return fail(TAHOE_E_INVAL, "bad argument");
  const Forest& H = f->host;
  int64_t leaves = 0;
  int32_t maxd = 0;
  for (size_t k = 0; k < H.feat.size(); k++) {
    leaves += H.feat[k] < 0;
    maxd = std::max(maxd, H.depth[k]);
  }
  double V = 0;
  for (double v : H.exp_reads) V += v;
  std::ostringstream js;
  js.precision(6);
  js << "{\"n_trees\":" << H.n_trees << ",\"n_trees_full\":" << H.n_trees_full
     << ",\"nodes\":" << H.feat.size() << ",\"leaves\":" << leaves << ",\"max_depth\":" << maxd
     << ",\"n_features\":" << H.n_features << ",\"n_classes\":" << H.n_classes
     << ",\"agg\":" << H.agg << ",\"calibrated\":" << (H.calibrated ? "true" : "false")
     << ",\"n_calib\":" << H.n_cal << ",\"expected_node_reads_per_sample\":" << V
     << ",\"expected_visits_per_sample\":" << (V - H.n_trees)
     << ",\"feature_bits\":" << f->di.fbits << ",\"direct_bytes\":" << f->di.bytes()
     << ",\"direct_chunks\":" << (f->direct_chunks.empty() ? 0 : f->direct_chunks.size() - 1)
     << ",\"bytes_fixed_index\":" << (int64_t)H.feat.size() * 12
     << ",\"sliced_valid\":" << (f->sl.valid ? "true" : "false")
     << ",\"sliced_why\":\"" << f->sl.why_invalid << "\""
     << ",\"coded_valid\":" << (f->sl.code_valid ? "true" : "false")
     << ",\"coded_why\":\"" << f->sl.code_why << "\"" << ",\"coded_thresholds\":"
     << (f->sl.thr_off.empty() ? 0 : f->sl.thr_off.back())
     << ",\"code8\":" << (f->sl.code8 ? "true" : "false") << ",\"code8_vfbits\":" << f->sl.vfbits
     << ",\"code8_virtual\":" << f->sl.n_virtual << ",\"code8_bands\":" << f->sl.c8_bands
     << ",\"code_bank_rows\":" << f->sl.cb_rows << ",\"code_bank_passes\":" << f->sl.cb_passes
     << ",\"code_bank_desc\":[" << [&] {
          std::string r;
          for (size_t q = 0; q < f->sl.cb_desc.size(); q++) r += (q ? "," : "") + std::to_string(f->sl.cb_desc[q]);
          return r; }() << "]"
     << ",\"code_slot\":[" << [&] {
          std::string r;
          if (f->sl.code_valid && !f->sl.code8)
            for (size_t q = 0; q < f->sl.code_slot.size(); q++) r += (q ? "," : "") + std::to_string(f->sl.code_slot[q]);
          return r; }() << "]"
     << ",\"sliced_fbits\":" << f->sl.fbits << ",\"cta_split\":[" << [&] {
          std::string r;
          for (size_t q = 0; q + 1 < f->cta_start.size(); q++)
            r += (q ? "," : "") + std::to_string(f->cta_start[q + 1] - f->cta_start[q]);
          return r; }() << "]"
     << ",\"n_slices\":" << f->sl.n_slices << ",\"slots_max\":" << f->sl.slots_max
     << ",\"slot_budget\":" << f->slot_budget << ",\"sliced_bytes\":" << f->sl.bytes()
     << ",\"column_balance_expected\":" << f->sl.eff << ",\"lockstep_eff_sim\":" << f->sl.eff_sim
     << ",\"trees_per_lane\":" << f->sl.trees_per_lane << ",\"cost_fitted\":"
     << (cost_params().fitted ? "true" : "false")
     << ",\"rows_ok\":" << (plan_stats(f).rows_ok ? "true" : "false")
     << ",\"sliced_rows_global\":" << (plan_stats(f).rows_global ? "true" : "false")
     << ",\"num_sms\":" << f->num_sms << ",\"max_smem\":" << f->max_smem << "}";
  std::string s = js.str();
  if ((int64_t)s.size() + 1 > len) return fail(TAHOE_E_INVAL, "buffer too small");
  std::memcpy(buf, s.c_str(), s.size() + 1);
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) void tahoe_forest_free(tahoe_forest* f) {
  if (!f) return;
  free_device(f);
  delete f;
}

// ------------------------------------------------------------------ introspection
__attribute__((visibility("default"))) tahoe_status tahoe_forest_layout_info(
    const tahoe_forest* f, uint64_t* count, uint8_t* hot_left, double* exp_reads, int32_t* order) {
  TAHOE_GUARD_BEGIN
  if (!f) return fail(TAHOE_E_INVAL, "NULL forest");
  const Forest& H = f->host;
  if (count) std::fill(count, count + H.n_nodes_user, 0);
  if (hot_left) std::fill(hot_left, hot_left + H.n_nodes_user, 1);
  for (size_t k = 0; k < H.feat.size(); k++) {
    if (count) count[H.orig[k]] = H.count[k];
    if (hot_left) hot_left[H.orig[k]] = H.hot_left[k];
  }
  if (exp_reads) for (int32_t t = 0; t < H.n_trees; t++) exp_reads[t] = H.exp_reads[t];
  if (order) for (int32_t i = 0; i < H.n_trees; i++) order[i] = H.tree_orig[H.order[i]];
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_tree_tokens(
    const tahoe_forest* f, int32_t t, int32_t t_nodes, int32_t* token_nodes, double* weights,
    int32_t cap, int32_t* n_tokens) {
  TAHOE_GUARD_BEGIN
  if (!f || t < 0 || t >= f->host.n_trees || t_nodes < 1 || !n_tokens) return fail(TAHOE_E_INVAL, "bad argument");
  std::vector<int32_t> tok;
  std::vector<double> w;
  tree_tokens(f->host, t, t_nodes, tok, w);
  *n_tokens = (int32_t)w.size();
  for (int32_t i = 0; i < std::min<int32_t>(cap, (int32_t)w.size()); i++) {
    for (int32_t j = 0; j < t_nodes; j++) {
      int32_t k = tok[(size_t)i * t_nodes + j];
      if (token_nodes) token_nodes[(size_t)i * t_nodes + j] = k < 0 ? -1 : f->host.orig[k];
    }
    if (weights) weights[i] = w[i];
  }
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_tree_simhash(
    const tahoe_forest* f, int32_t t, int32_t t_nodes, int32_t l_hash, double* checksum, uint8_t* bits) {
  TAHOE_GUARD_BEGIN
  if (!f || t < 0 || t >= f->host.n_trees || t_nodes < 1 || l_hash < 1) return fail(TAHOE_E_INVAL, "bad argument");
  std::vector<double> cs;
  std::vector<uint8_t> b;
  tree_simhash(f->host, t, t_nodes, l_hash, cs, b);
  if (checksum) std::copy(cs.begin(), cs.end(), checksum);
  if (bits) std::copy(b.begin(), b.end(), bits);
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_simhash(
    const int8_t* strings, const double* weights, int32_t n_str, int32_t l_hash, double* checksum,
    uint8_t* bits) {
  TAHOE_GUARD_BEGIN
  if (!strings || !weights || !checksum || !bits || n_str < 0 || l_hash < 1) return fail(TAHOE_E_INVAL, "bad argument");
  simhash(strings, weights, n_str, l_hash, checksum, bits);
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_lsh_order(
    const uint8_t* bits, int32_t n_trees, int32_t l_hash, int32_t m_chunks, int32_t* collisions,
    int32_t* order) {
  TAHOE_GUARD_BEGIN
  if (!bits || n_trees < 1 || l_hash < 1 || m_chunks < 1 || m_chunks > l_hash || !order)
    return fail(TAHOE_E_INVAL, "bad argument");
  std::vector<uint8_t> b(bits, bits + (size_t)n_trees * l_hash);
  std::vector<uint16_t> col;
  std::vector<int32_t> ord = lsh_order(b, n_trees, l_hash, m_chunks, &col);
  std::copy(ord.begin(), ord.end(), order);
  if (collisions) for (size_t i = 0; i < col.size(); i++) collisions[i] = col[i];
  return TAHOE_OK;
  TAHOE_GUARD_END
}

__attribute__((visibility("default"))) tahoe_status tahoe_sha1(const uint8_t* msg, int64_t len,
                                                               uint8_t digest[20]) {
  if ((!msg && len > 0) || len < 0 || !digest) return fail(TAHOE_E_INVAL, "bad argument");
  sha1(msg, (size_t)len, digest);
  return TAHOE_OK;
}

__attribute__((visibility("default"))) tahoe_status tahoe_forest_export_sliced(
    const tahoe_forest* f, int32_t* header, int32_t* slice_info, int32_t* col_len, uint32_t* nodes,
    int32_t* leaf_meta) {
  TAHOE_GUARD_BEGIN
  if (!f || !header) return fail(TAHOE_E_INVAL, "bad argument");
  const SlicedImage& S = f->sl;
  int32_t h[8] = {S.valid ? S.n_slices : 0, S.slots_max, S.fbits, f->host.n_trees, f->host.n_classes,
                  kSlicedCols, kSlotBytes, 0};
  std::copy(h, h + 8, header);
  if (!S.valid) return TAHOE_OK;
  if (slice_info)
    for (int32_t s = 0; s < S.n_slices; s++) {
      slice_info[4 * s] = S.slots[s];
      slice_info[4 * s + 1] = S.cls[s];
      slice_info[4 * s + 2] = S.ntrees[s];
      slice_info[4 * s + 3] = 0;
    }
  if (col_len) std::copy(S.col_len.begin(), S.col_len.end(), col_len);
  if (nodes) std::copy(S.nodes.begin(), S.nodes.end(), nodes);
  if (leaf_meta) std::copy(S.leaf_meta.begin(), S.leaf_meta.end(), leaf_meta);
  return TAHOE_OK;
  TAHOE_GUARD_END
}

}  // extern "C"
