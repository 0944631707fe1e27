// kernels.cu — the traversal + combine kernels for sm_100a.
//
// Every (sample, tree) pair walks root -> leaf on "x_j < b_i"; NaN takes the node's
// default path; leaf values are combined per sample in fp64 (reading Z17) and rounded
// once to fp32.  Two strategies (Algorithm 1 line 15, re-targeted):
//
//  k_direct  — the paper's "direct method": one thread per sample walks every tree
//              of a forest image that stays in HBM / L2; no shared memory, no reduction.
//  k_sliced  — the paper's "shared forest" / "splitting shared forest" re-designed:
//              a persistent CTA keeps one forest SLICE resident in shared memory (cp.async.bulk +
//              mbarrier), streams sample tiles into shared memory with double-buffered TMA bulk
//              copies, and a warp evaluates one sample with its 32 lanes walking 32 lane columns
//              of trees (conflict-free 8-byte node loads, one-row feature loads), then reduces the
//              32 fp64 lane sums with a shuffle butterfly.  Slices write fp64 partials that a
//              fixed-order finalize kernel combines; a single-slice forest finalizes in-kernel.
//  k_finalize — fixed-order fp64 sum of parts per class, base / average / argmax, RN to fp32.
#include <cuda_runtime.h>
#include <cstdint>

#include "kernels.hpp"
#include "tahoe.h"

namespace tahoe {

// ------------------------------------------------------------------ device helpers
__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
// 1-D TMA bulk copy global -> shared, completion counted on an mbarrier (bytes % 16 == 0,
// 16-byte aligned addresses).  SASS: UBLKCP.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}
// issue a (possibly > 64 KB) bulk copy in 64 KB pieces on one barrier; caller did expect_tx(total)
__device__ __forceinline__ void bulk_g2s_big(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  const uint32_t kPiece = 65536;
  for (uint32_t off = 0; off < bytes; off += kPiece) {
    uint32_t b = bytes - off < kPiece ? bytes - off : kPiece;
    bulk_g2s(static_cast<char*>(dst) + off, static_cast<const char*>(src) + off, b, bar);
  }
}

// The node test of one internal node: left iff x < b, NaN -> default path.
// Returns the slot/node delta to the next node: +1 for the hot child, +cold delta otherwise.
__device__ __forceinline__ uint32_t step(uint32_t thr_bits, uint32_t y, float v, int fbits,
                                         uint32_t offmask) {
  const float thr = __uint_as_float(thr_bits);
  const bool nan = v != v;
  const bool go_left = nan ? ((y & kDefaultLeftBit) != 0) : (v < thr);
  const bool hot = go_left == ((y & kHotLeftBit) != 0);
  return hot ? 1u : ((y >> fbits) & offmask);
}

// Scalar aggregations finalised in fp64, then one round-to-nearest (Z14, Z17).
__device__ __forceinline__ void write_scalar(const OutArgs& o, int64_t i, double s) {
  double v;
  if (o.agg == TAHOE_AGG_AVERAGE) v = s / (double)o.n_trees_full + (double)o.base;
  else v = s + (double)o.base;
  o.out[i] = (float)v;
  if (o.out_class) o.out_class[i] = (o.agg == TAHOE_AGG_BINARY && v > 0.0) ? 1 : 0;
}

// ------------------------------------------------------------------ direct strategy
struct DirectKArgs {
  DevDirect img;
  const float* X;
  int64_t n;
  int32_t d;
  OutArgs o;
};

template <bool LEAF, bool FUSED>
__global__ void __launch_bounds__(256) k_direct(const DirectKArgs a) {
  const uint2* __restrict__ nodes = reinterpret_cast<const uint2*>(a.img.nodes);
  const int fbits = a.img.fbits;
  const uint32_t fmask = (1u << fbits) - 1u;
  const uint32_t offmask = (1u << (kOffsetTop - fbits)) - 1u;
  const int32_t C = a.o.n_classes;
  const bool vote = a.o.agg == TAHOE_AGG_VOTE;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const float* __restrict__ x = a.X + i * a.d;
    int32_t t = 0;
    uint32_t k = (uint32_t)__ldg(&a.img.root[0]);
    int32_t cls = __ldg(&a.img.cls[0]);
    double acc = 0.0;
    uint64_t fp = 0;
    for (;;) {
      const uint2 nd = __ldg(&nodes[k]);
      if ((int32_t)nd.y < 0) {  // leaf: combine
        const float v = __uint_as_float(nd.x);
        if (vote) a.o.raw[i * C + (int32_t)v] += 1.0;
        else acc += (double)v;
        if (LEAF) {
          const int32_t tree = __ldg(&a.img.tree_orig[t]);
          const uint32_t leaf = nd.y & 0x7fffffffu;
          a.o.out_leaf[i * a.o.T_leaf + tree] = (int32_t)leaf;
          fp += mix64(((uint64_t)(uint32_t)tree << 32) | leaf);
        }
        if (++t == a.img.n_slots) break;
        k = (uint32_t)__ldg(&a.img.root[t]);
        if (!FUSED) {
          const int32_t c2 = __ldg(&a.img.cls[t]);
          if (c2 != cls) {
            if (!vote) a.o.raw[i * C + cls] = acc;
            acc = 0.0;
            cls = c2;
          }
        }
      } else {  // internal node: "x_j < b_i"
        const float v = __ldg(&x[nd.y & fmask]);
        k += step(nd.x, nd.y, v, fbits, offmask);
      }
    }
    if (FUSED) write_scalar(a.o, i, acc);
    else if (!vote) a.o.raw[i * C + cls] = acc;
    if (LEAF && a.o.out_fp) atomicAdd(reinterpret_cast<unsigned long long*>(&a.o.out_fp[i]),
                                     (unsigned long long)fp);
  }
}

// ------------------------------------------------------------------ sliced strategy
struct SlicedKArgs {
  DevSliced img;
  const float* X;
  int64_t n;
  int32_t d;
  int32_t tile_rows;
  int32_t cps;           // CTAs per slice (single-pass)
  int32_t forest_smem;   // bytes reserved for the slice
  int32_t tile_floats;   // floats per tile buffer
  int32_t tma_ok;        // X is 16-byte aligned and tile_rows*d*4 % 16 == 0
  OutArgs o;
};

template <bool LEAF, bool FUSED, bool ROWS_SMEM>
__global__ void __launch_bounds__(1024, 1) k_sliced(const SlicedKArgs a) {
  extern __shared__ __align__(128) unsigned char smem[];
  uint2* s_nodes = reinterpret_cast<uint2*>(smem);
  float* s_tile = reinterpret_cast<float*>(smem + a.forest_smem);
  uint64_t* s_bar = reinterpret_cast<uint64_t*>(
      smem + a.forest_smem + (ROWS_SMEM ? 2 * (size_t)a.tile_floats * sizeof(float) : 0));
  const int lane = threadIdx.x & 31;
  const int warp = threadIdx.x >> 5;
  const int nwarps = blockDim.x >> 5;
  const int fbits = a.img.fbits;
  const uint32_t fmask = (1u << fbits) - 1u;
  const uint32_t offmask = (1u << (kOffsetTop - fbits)) - 1u;
  const int32_t ns = a.img.n_slices;
  const int32_t G = gridDim.x;
  const bool multipass = ns > G;
  const int64_t R = a.tile_rows;
  const int64_t ntiles = (a.n + R - 1) / R;
  const size_t tile_bytes_full = (size_t)R * a.d * sizeof(float);

  if (threadIdx.x == 0) {
    mbar_init(&s_bar[0], 1);
    mbar_init(&s_bar[1], 1);
    mbar_init(&s_bar[2], 1);
    fence_mbar_init();
  }
  __syncthreads();
  uint32_t ph_forest = 0, ph0 = 0, ph1 = 0;

  auto tile_tma = [&](int64_t tile) -> bool {
    return ROWS_SMEM && a.tma_ok && (tile + 1) * R <= a.n;
  };
  auto issue_tile = [&](int64_t tile, int buf) {  // thread 0 only
    fence_proxy_async_smem();
    mbar_expect_tx(&s_bar[1 + buf], (uint32_t)tile_bytes_full);
    bulk_g2s_big(s_tile + (size_t)buf * a.tile_floats, a.X + tile * R * a.d,
                 (uint32_t)tile_bytes_full, &s_bar[1 + buf]);
  };

  for (int32_t sl = multipass ? (int32_t)blockIdx.x : (int32_t)blockIdx.x % ns; sl < ns;
       sl += multipass ? G : ns) {
    const int64_t t0 = multipass ? 0 : blockIdx.x / ns;
    const int64_t ts = multipass ? 1 : a.cps;
    // stage the slice (a7): one bulk copy of slots*32*8 bytes
    if (threadIdx.x == 0) {
      const uint32_t bytes = (uint32_t)a.img.slots[sl] * 256u;
      fence_proxy_async_smem();
      mbar_expect_tx(&s_bar[0], bytes);
      bulk_g2s_big(s_nodes, a.img.nodes + (size_t)sl * a.img.slots_max * 64, bytes, &s_bar[0]);
      if (t0 < ntiles && tile_tma(t0)) issue_tile(t0, 0);
    }
    const uint32_t end = (uint32_t)a.img.col_len[sl * 32 + lane];
    const int32_t* __restrict__ leaf_meta = a.img.leaf_meta + (size_t)sl * a.img.slots_max * 64;
    mbar_wait(&s_bar[0], ph_forest);
    ph_forest ^= 1;

    int64_t it = 0;
    for (int64_t tile = t0; tile < ntiles; tile += ts, ++it) {
      const int buf = (int)(it & 1);
      const int64_t r0 = tile * R;
      const int nr = (int)((a.n - r0) < R ? (a.n - r0) : R);
      const float* tbuf = s_tile + (size_t)buf * a.tile_floats;
      if (ROWS_SMEM) {
        const int64_t nxt = tile + ts;
        if (threadIdx.x == 0 && nxt < ntiles && tile_tma(nxt)) issue_tile(nxt, buf ^ 1);
        if (tile_tma(tile)) {
          if (buf == 0) { mbar_wait(&s_bar[1], ph0); ph0 ^= 1; }
          else { mbar_wait(&s_bar[2], ph1); ph1 ^= 1; }
        } else {  // ragged or unaligned tile: cooperative copy (a6 fallback)
          float* dst = s_tile + (size_t)buf * a.tile_floats;
          const float* src = a.X + r0 * a.d;
          const int64_t cnt = (int64_t)nr * a.d;
          for (int64_t q = threadIdx.x; q < cnt; q += blockDim.x) dst[q] = __ldg(&src[q]);
          __syncthreads();
        }
      }
      for (int r = warp; r < nr; r += nwarps) {
        const int64_t i = r0 + r;
        const float* __restrict__ row = ROWS_SMEM ? tbuf + (size_t)r * a.d : a.X + i * a.d;
        double acc = 0.0;
        uint64_t fp = 0;
        uint32_t s = 0;
        // a8: each lane walks the trees of its column for sample i; leaves jump to the next root
        while (s < end) {
          const uint2 nd = s_nodes[s * 32 + lane];
          if ((int32_t)nd.y < 0) {
            acc += (double)__uint_as_float(nd.x);
            if (LEAF) {
              const int2 m = *reinterpret_cast<const int2*>(&leaf_meta[2 * (s * 32 + lane)]);
              a.o.out_leaf[i * a.o.T_leaf + m.x] = m.y;
              fp += mix64(((uint64_t)(uint32_t)m.x << 32) | (uint32_t)m.y);
            }
            s += nd.y & 0x7fffffffu;
          } else {
            const float v = ROWS_SMEM ? row[nd.y & fmask] : __ldg(&row[nd.y & fmask]);
            s += step(nd.x, nd.y, v, fbits, offmask);
          }
        }
        // a9: fp64 butterfly over the 32 lane sums (lane 0's order is fixed)
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
        if (LEAF) {
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) fp += __shfl_xor_sync(0xffffffffu, fp, o);
        }
        if (lane == 0) {
          if (FUSED) write_scalar(a.o, i, acc);
          else a.o.raw[(size_t)sl * a.n + i] = acc;
          if (LEAF && a.o.out_fp)
            atomicAdd(reinterpret_cast<unsigned long long*>(&a.o.out_fp[i]), (unsigned long long)fp);
        }
      }
      __syncthreads();  // the tile buffer is free for the next prefetch
    }
    __syncthreads();  // the slice buffer is free for the next slice (multi-pass)
  }
}

// ------------------------------------------------------------------ finalize
__global__ void __launch_bounds__(256) k_finalize(const FinalizeArgs a) {
  const int32_t C = a.n_classes;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.n;
       i += (int64_t)gridDim.x * blockDim.x) {
    int best = 0;
    double bv = 0.0;
    for (int32_t c = 0; c < C; c++) {
      double s = 0.0;
      if (a.class_ptr) {
        for (int32_t p = a.class_ptr[c]; p < a.class_ptr[c + 1]; p++)
          s += a.partial[(int64_t)a.class_parts[p] * a.part_stride + i * a.row_stride];
      } else {
        s = a.partial[(int64_t)c * a.part_stride + i * a.row_stride];
      }
      if (a.raw_out) { a.raw_out[i * C + c] = s; continue; }
      double v;
      if (a.agg == TAHOE_AGG_VOTE) v = s;
      else if (a.agg == TAHOE_AGG_AVERAGE) v = s / (double)a.n_trees_full + (double)a.base;
      else v = s + (double)a.base;
      a.out[i * C + c] = (float)v;
      if (c == 0 || v > bv) { best = c; bv = v; }
    }
    if (!a.raw_out && a.out_class) {
      if (a.agg == TAHOE_AGG_BINARY) a.out_class[i] = bv > 0.0 ? 1 : 0;
      else if (a.agg == TAHOE_AGG_CLASS_SUM || a.agg == TAHOE_AGG_VOTE) a.out_class[i] = best;
      else a.out_class[i] = 0;
    }
  }
}

// ------------------------------------------------------------------ launchers
static int grid_for(int64_t n, int block, int num_sms, int per_sm) {
  int64_t g = (n + block - 1) / block;
  int64_t cap = (int64_t)num_sms * per_sm;
  if (g > cap) g = cap;
  return (int)(g < 1 ? 1 : g);
}

int launch_direct(const DevDirect& img, const float* X, int64_t n, int32_t d, const OutArgs& o,
                  bool fused, int32_t num_sms, void* stream) {
  DirectKArgs a{img, X, n, d, o};
  const int block = 256;
  const int grid = grid_for(n, block, num_sms, 8);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const bool leaf = o.out_leaf != nullptr || o.out_fp != nullptr;
  if (leaf) {
    if (fused) k_direct<true, true><<<grid, block, 0, st>>>(a);
    else k_direct<true, false><<<grid, block, 0, st>>>(a);
  } else {
    if (fused) k_direct<false, true><<<grid, block, 0, st>>>(a);
    else k_direct<false, false><<<grid, block, 0, st>>>(a);
  }
  return (int)cudaGetLastError();
}

template <bool L, bool F, bool R>
static cudaError_t sliced_one(const SlicedKArgs& a, const SlicedPlan& p, cudaStream_t st) {
  auto kern = k_sliced<L, F, R>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, p.smem_bytes);
  if (e != cudaSuccess) return e;
  kern<<<p.grid, p.block, p.smem_bytes, st>>>(a);
  return cudaGetLastError();
}

int launch_sliced(const DevSliced& img, const SlicedPlan& plan, const float* X, int64_t n,
                  int32_t d, const OutArgs& o, bool fused, void* stream) {
  SlicedKArgs a{};
  a.img = img;
  a.X = X;
  a.n = n;
  a.d = d;
  a.tile_rows = plan.tile_rows;
  a.cps = plan.cps;
  a.forest_smem = plan.forest_smem;
  a.tile_floats = plan.tile_rows * d;
  a.tma_ok = ((reinterpret_cast<uintptr_t>(X) & 15) == 0) &&
             (((int64_t)plan.tile_rows * d * 4) % 16 == 0);
  a.o = o;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const bool leaf = o.out_leaf != nullptr || o.out_fp != nullptr;
  cudaError_t e;
  if (plan.rows_in_smem) {
    if (leaf) e = fused ? sliced_one<true, true, true>(a, plan, st) : sliced_one<true, false, true>(a, plan, st);
    else e = fused ? sliced_one<false, true, true>(a, plan, st) : sliced_one<false, false, true>(a, plan, st);
  } else {
    if (leaf) e = fused ? sliced_one<true, true, false>(a, plan, st) : sliced_one<true, false, false>(a, plan, st);
    else e = fused ? sliced_one<false, true, false>(a, plan, st) : sliced_one<false, false, false>(a, plan, st);
  }
  return (int)e;
}

int launch_finalize(const FinalizeArgs& a, void* stream) {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int block = 256;
  k_finalize<<<grid_for(a.n, block, sms, 8), block, 0, static_cast<cudaStream_t>(stream)>>>(a);
  return (int)cudaGetLastError();
}

}  // namespace tahoe
