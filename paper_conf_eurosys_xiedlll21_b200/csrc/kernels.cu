// kernels.cu — the traversal + combine kernels for sm_100a.
//
// Every (sample, tree) pair walks root -> leaf on "x_j < b_i"; NaN takes the node's
// default path; leaf values are combined per sample in fp64 (reading Z17) and rounded
// once to fp32.  Strategies (Algorithm 1 line 15, re-targeted):
//
//  k_direct*        — the paper's "direct method": threads walk trees of a forest
//                     image that stays in HBM / L2 (one thread per sample, or eight per sample over
//                     rows staged in shared memory for large batches); images over 64 MB are walked
//                     in L2-sized chunks of trees (reading R4).
//  k_sliced         — "shared forest" / "splitting shared forest" re-designed: a
//                     persistent CTA keeps one forest SLICE (16 lane columns of trees) resident in
//                     shared memory, streams 64-row sample tiles through a 3-deep TMA ring, and a
//                     half-warp walks one sample (lane = lane column), two samples per lane.
//  k_sliced_codes   — the same walk over exact u16 rank codes of the rows (reading R7), produced by
//                     a pre-pass (k_encode_rows_banks); a producer warp stages the slice and the
//                     code tiles (cp.async.bulk into a ring of up to 8 tiles, full / empty mbarriers),
//                     31 consumer warps claim 4-row work units; LEAF / PROF instantiations add leaf
//                     ids + fingerprints / per-lane timing.
//  k_sliced_codes8  — wide rows (reading R8): u8 codes over virtual attributes, dynamic tile claiming
//                     across ~30 slices, four chains per lane.
//  k_rows           — small batches (f1): one CTA per sample, lane = tree over the direct image,
//                     fixed-order block reduction and finalize in one launch.
//  k_finalize       — fixed-order fp64 sum of parts per class, base / average / argmax, RN to fp32.
//  k_visit_peak / k_smem_bw — the microbenchmarks of Algorithm 1 line 4 (the roofline peak).
#include <cuda.h>
#include <cuda_runtime.h>
#include <algorithm>
#include <atomic>
#include <numeric>
#include <cstdlib>
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
  // try_wait with a suspend-time hint: a waiting warp sleeps in hardware instead of re-issuing
  // the probe (a plain try_wait loop spent a fifth of all issue slots on spinning)
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(phase), "r"(20000u)
      : "memory");
}
// Ring-wrap guard of the dynamically claimed tile rings (k_sliced, k_sliced_codes): a ring of
// kRing buffers uses 2 * kRing "full" mbarriers, tile sequence number seq on barrier seq % (2 kRing)
// with parity (seq / (2 kRing)) & 1.  A warp claiming a unit of tile seq therefore waits on a
// parity two phases of THAT barrier apart only if tile seq - 2 kRing has not arrived; but then tile
// seq - kRing (same buffer) cannot have been issued, so the 2 x 16 units of those two tiles are
// claimed by 32 blocked warps and no warp is left to claim seq (a CTA has 32 warps; a tile has 16
// units).  With one barrier per buffer a warp could claim tile seq + 2 kRing while tile seq was still
// held by one slow unit, and its parity wait would return at once on the old data.
constexpr int kRingBars = 2 * kSlicedRing;
__device__ __forceinline__ uint32_t ring_bar(uint32_t seq) { return seq % (uint32_t)kRingBars; }
__device__ __forceinline__ uint32_t ring_parity(uint32_t seq) { return (seq / (uint32_t)kRingBars) & 1u; }

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
          if (a.o.out_leaf) a.o.out_leaf[i * a.o.T_leaf + tree] = (int32_t)leaf;
          fp += mix64(((uint64_t)(uint32_t)tree << 32) | leaf);
        }
        if (++t == a.img.n_slots) break;
        k = (uint32_t)__ldg(&a.img.root[t]);
        if (!FUSED) {
          const int32_t c2 = __ldg(&a.img.cls[t]);
          if (c2 != cls) {
            if (!vote) a.o.raw[i * C + cls] += acc;
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
    else if (!vote) a.o.raw[i * C + cls] += acc;
    if (LEAF && a.o.out_fp) atomicAdd(reinterpret_cast<unsigned long long*>(&a.o.out_fp[i]),
                                     (unsigned long long)fp);
  }
}

// Direct strategy with staged rows: a CTA copies a tile of BLOCK rows into shared memory (odd
// row stride, so lanes reading different rows at random attributes spread over the banks), then
// each thread walks every tree for its row.  The tree loop is warp-uniform: the lanes of a warp
// stay in the same tree, so with hot-child-next ordering their node loads fall on few
// L1 lines ("nodes that tend to be accessed at the same time ... contiguous").
template <bool LEAF, bool FUSED, int BLOCK, bool LOCKSTEP>
__global__ void __launch_bounds__(BLOCK) k_direct_tiled(const DirectKArgs a, int32_t rs) {
  extern __shared__ __align__(16) float s_rows[];
  const uint2* __restrict__ nodes = reinterpret_cast<const uint2*>(a.img.nodes);
  const int fbits = a.img.fbits;
  const uint32_t fmask = (1u << fbits) - 1u;
  const uint32_t offmask = (1u << (kOffsetTop - fbits)) - 1u;
  const int32_t C = a.o.n_classes;
  const bool vote = a.o.agg == TAHOE_AGG_VOTE;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t ntiles = (a.n + BLOCK - 1) / BLOCK;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * BLOCK;
    const int nr = (int)((a.n - r0) < BLOCK ? (a.n - r0) : BLOCK);
    __syncthreads();
    for (int r = warp; r < nr; r += BLOCK / 32) {
      const float* src = a.X + (r0 + r) * a.d;
      for (int c = lane; c < a.d; c += 32) s_rows[r * rs + c] = __ldg(&src[c]);
    }
    __syncthreads();
    const bool active = threadIdx.x < nr;
    const int64_t i = r0 + threadIdx.x;
    const float* row = s_rows + threadIdx.x * rs;
    double acc = 0.0;
    uint64_t fp = 0;
    int32_t cls = __ldg(&a.img.cls[0]);
    if (LOCKSTEP) {
      for (int32_t t = 0; t < a.img.n_slots; t++) {
        uint32_t k = (uint32_t)__ldg(&a.img.root[t]);
        if (!FUSED) {
          const int32_t c2 = __ldg(&a.img.cls[t]);
          if (c2 != cls) {
            if (active && !vote) a.o.raw[i * C + cls] += acc;
            acc = 0.0;
            cls = c2;
          }
        }
        if (!active) continue;
        uint2 nd = __ldg(&nodes[k]);
        while ((int32_t)nd.y >= 0) {
          k += step(nd.x, nd.y, row[nd.y & fmask], fbits, offmask);
          nd = __ldg(&nodes[k]);
        }
        const float v = __uint_as_float(nd.x);
        if (vote) a.o.raw[i * C + (int32_t)v] += 1.0;
        else acc += (double)v;
        if (LEAF) {
          const int32_t tree = __ldg(&a.img.tree_orig[t]);
          const uint32_t leaf = nd.y & 0x7fffffffu;
          if (a.o.out_leaf) a.o.out_leaf[i * a.o.T_leaf + tree] = (int32_t)leaf;
          fp += mix64(((uint64_t)(uint32_t)tree << 32) | leaf);
        }
      }
    } else if (active) {
      // free-running: each thread moves to its next tree as soon as it reaches a leaf
      int32_t t = 0;
      uint32_t k = (uint32_t)__ldg(&a.img.root[0]);
      for (;;) {
        const uint2 nd = __ldg(&nodes[k]);
        if ((int32_t)nd.y < 0) {
          const float v = __uint_as_float(nd.x);
          if (vote) a.o.raw[i * C + (int32_t)v] += 1.0;
          else acc += (double)v;
          if (LEAF) {
            const int32_t tree = __ldg(&a.img.tree_orig[t]);
            const uint32_t leaf = nd.y & 0x7fffffffu;
            if (a.o.out_leaf) a.o.out_leaf[i * a.o.T_leaf + tree] = (int32_t)leaf;
            fp += mix64(((uint64_t)(uint32_t)tree << 32) | leaf);
          }
          if (++t == a.img.n_slots) break;
          k = (uint32_t)__ldg(&a.img.root[t]);
          if (!FUSED) {
            const int32_t c2 = __ldg(&a.img.cls[t]);
            if (c2 != cls) {
              if (!vote) a.o.raw[i * C + cls] += acc;
              acc = 0.0;
              cls = c2;
            }
          }
        } else {
          k += step(nd.x, nd.y, row[nd.y & fmask], fbits, offmask);
        }
      }
    }
    if (active) {
      if (FUSED) write_scalar(a.o, i, acc);
      else if (!vote) a.o.raw[i * C + cls] += acc;
      if (LEAF && a.o.out_fp)
        atomicAdd(reinterpret_cast<unsigned long long*>(&a.o.out_fp[i]), (unsigned long long)fp);
    }
  }
}

// Direct strategy, staged rows, P threads per row (scalar outputs, no leaf ids): thread j of a row
// walks trees j, j+P, j+2P, ... free-running; the P partial sums are added in a fixed order
// through shuffles.  P x more threads over the same staged rows hide more node-load latency.
// GRP > 1: node loads fetch the aligned group of GRP slots (16 B or 32 B) holding the node into
// registers, and the next node is taken from them when it lies in the same group (the hot child
// sits in the next slot), so a walk down a hot chain costs one L1/L2 request per group
// instead of one per node.  The device image is padded to 64 bytes (upload()).
template <bool FUSED, int ROWS, int P, int GRP = 1>
__global__ void __launch_bounds__(ROWS * P) k_direct_tlp(const DirectKArgs a, int32_t rs) {
  extern __shared__ __align__(16) float s_rows[];
  const uint2* __restrict__ nodes = reinterpret_cast<const uint2*>(a.img.nodes);
  const int fbits = a.img.fbits;
  const uint32_t fmask = (1u << fbits) - 1u;
  const uint32_t offmask = (1u << (kOffsetTop - fbits)) - 1u;
  const int32_t T = a.img.n_slots;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int r = threadIdx.x / P, j = threadIdx.x % P;
  const int64_t ntiles = (a.n + ROWS - 1) / ROWS;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * ROWS;
    const int nr = (int)((a.n - r0) < ROWS ? (a.n - r0) : ROWS);
    __syncthreads();
    for (int q = warp; q < nr; q += ROWS * P / 32) {
      const float* src = a.X + (r0 + q) * a.d;
      for (int c = lane; c < a.d; c += 32) s_rows[q * rs + c] = __ldg(&src[c]);
    }
    __syncthreads();
    const bool active = r < nr;
    const float* row = s_rows + (active ? r : 0) * rs;
    double acc = 0.0;
    if (active && j < T) {
      int32_t t = j;
      uint32_t k = (uint32_t)__ldg(&a.img.root[t]);
      uint4 g0 = make_uint4(0u, 0u, 0u, 0u), g1 = g0;
      uint32_t gbase = 0xffffffffu;
      for (;;) {
        uint2 nd;
        if constexpr (GRP == 1) {
          nd = __ldg(&nodes[k]);
        } else {
          if ((k & ~(uint32_t)(GRP - 1)) != gbase) {
            gbase = k & ~(uint32_t)(GRP - 1);
            const uint4* gp = reinterpret_cast<const uint4*>(nodes + gbase);
            g0 = __ldg(gp);
            if constexpr (GRP == 4) g1 = __ldg(gp + 1);
          }
          const uint32_t w = k & (uint32_t)(GRP - 1);
          if constexpr (GRP == 4) {
            const uint4 g = (w & 2u) ? g1 : g0;
            nd = (w & 1u) ? make_uint2(g.z, g.w) : make_uint2(g.x, g.y);
          } else {
            nd = w ? make_uint2(g0.z, g0.w) : make_uint2(g0.x, g0.y);
          }
        }
        if ((int32_t)nd.y < 0) {
          acc += (double)__uint_as_float(nd.x);
          t += P;
          if (t >= T) break;
          k = (uint32_t)__ldg(&a.img.root[t]);
        } else {
          k += step(nd.x, nd.y, row[nd.y & fmask], fbits, offmask);
        }
      }
    }
    // fixed-order combine of the row's P chains (lanes j = 0..P-1 are adjacent)
#pragma unroll
    for (int o = 1; o < P; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (active && j == 0) {
      const int64_t i = r0 + r;
      if (FUSED) write_scalar(a.o, i, acc);
      else a.o.raw[i] += acc;
    }
  }
}

// Direct strategy with tree heads in shared memory (scalar outputs, no leaf ids): k_direct_tlp's
// walk, but the first `kh` node slots of every tree of the image (the root and the hot-first
// preorder prefix below it, reading R1 / P:616-628) are copied once per CTA into shared memory
// and read from there; the rest of each tree is read through L1/L2 as before.  A tree's slots are
// contiguous from root[t] (encode_direct), so slot k of tree t is a head iff k - root[t] < kh.
template <bool FUSED, int ROWS, int P>
__global__ void __launch_bounds__(ROWS * P) k_direct_heads(const DirectKArgs a, int32_t rs, int32_t kh) {
  extern __shared__ __align__(16) uint2 s_heads[];
  const uint2* __restrict__ nodes = reinterpret_cast<const uint2*>(a.img.nodes);
  const int fbits = a.img.fbits;
  const uint32_t fmask = (1u << fbits) - 1u;
  const uint32_t offmask = (1u << (kOffsetTop - fbits)) - 1u;
  const int32_t T = a.img.n_slots;
  float* s_rows = reinterpret_cast<float*>(s_heads + (size_t)T * kh);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int r = threadIdx.x / P, j = threadIdx.x % P;
  for (int32_t q = threadIdx.x; q < T * kh; q += ROWS * P) {
    const int32_t t = q / kh;
    const int64_t g = (int64_t)__ldg(&a.img.root[t]) + (q - t * kh);
    s_heads[q] = g < a.img.n_nodes ? __ldg(&nodes[g]) : make_uint2(0u, 0u);
  }
  const int64_t ntiles = (a.n + ROWS - 1) / ROWS;
  for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const int64_t r0 = tile * ROWS;
    const int nr = (int)((a.n - r0) < ROWS ? (a.n - r0) : ROWS);
    __syncthreads();
    for (int q = warp; q < nr; q += ROWS * P / 32) {
      const float* src = a.X + (r0 + q) * a.d;
      for (int c = lane; c < a.d; c += 32) s_rows[q * rs + c] = __ldg(&src[c]);
    }
    __syncthreads();
    const bool active = r < nr;
    const float* row = s_rows + (active ? r : 0) * rs;
    double acc = 0.0;
    if (active && j < T) {
      int32_t t = j;
      uint32_t hb = (uint32_t)(j * kh);
      uint32_t rt = (uint32_t)__ldg(&a.img.root[t]);
      uint32_t k = rt;
      for (;;) {
        const uint32_t rel = k - rt;
        const uint2 nd = rel < (uint32_t)kh ? s_heads[hb + rel] : __ldg(&nodes[k]);
        if ((int32_t)nd.y < 0) {
          acc += (double)__uint_as_float(nd.x);
          t += P;
          if (t >= T) break;
          hb += (uint32_t)(P * kh);
          rt = k = (uint32_t)__ldg(&a.img.root[t]);
        } else {
          k += step(nd.x, nd.y, row[nd.y & fmask], fbits, offmask);
        }
      }
    }
#pragma unroll
    for (int o = 1; o < P; o <<= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (active && j == 0) {
      const int64_t i = r0 + r;
      if (FUSED) write_scalar(a.o, i, acc);
      else a.o.raw[i] += acc;
    }
  }
}

// ------------------------------------------------------------------ sliced strategy
// Sliced node words (encode.cpp): x = threshold (internal) or leaf value;
//   internal y = off_bytes << (F+3) | default_left << (F+2) | attribute << 2   (left child next)
//   leaf     y = next_root_bytes << (F+3) | (2^F - 1) << 2            (all-ones attribute field)
// A slice has 16 lane columns; slot s of column c is the word pair 16*s + c, one slot row is
// 16 x 8 B = 128 B and offsets are byte distances between slots.  Lane l walks column l & 15 for
// the rows of its half-warp (l >> 4): an 8-byte load is served per half-warp, whose 16 lanes sit
// in 16 different bank pairs.  The attribute is stored as a byte offset; staged rows sit at a
// power-of-two stride >= 2^F floats, so its shared address is one LOP3: (y & amask) | row_base,
// and a leaf is the one address row_base | amask.  Every lane column ends with a self-looping leaf
// of value 0.0, so a lane that has finished its trees keeps stepping harmlessly.
struct alignas(64) SlicedKArgs {
  CUtensorMap tmap;      // PADDED rows: X as a 2-D tensor [n][d], box [row_stride][tile_rows]
  DevSliced img;
  const float* X;
  int64_t n;
  int32_t d;
  int32_t tile_rows;
  int32_t cps;           // CTAs per slice (single-pass)
  int32_t forest_smem;   // bytes reserved for the slice (multiple of 1024)
  int32_t row_stride;    // floats between staged rows (PADDED: multiple of 2^F; DENSE: d)
  int32_t buf_floats;    // floats per ring buffer
  int32_t x_aligned;     // DENSE rows: X 16-byte aligned (one 1-D bulk copy per tile)
  OutArgs o;
};

// Row staging layouts of k_sliced (SlicedPlan::rows)
constexpr int kRowsGlobal = 0;  // rows read from global memory (too wide to stage)
constexpr int kRowsDense = 1;   // rows at stride d, one 1-D bulk copy per tile
constexpr int kRowsPadded = 2;  // rows at stride 2^F*k via one 2-D tensor TMA per tile

constexpr int kRing = kSlicedRing;  // sample-tile ring depth

struct StepConsts {
  uint32_t amask;   // attribute byte-offset mask (2^F - 1) << 2
  uint32_t dlbit;   // default-left bit
  uint32_t shmul;   // 2^(32 - (F+3)): y >> (F+3) == umulhi(y, shmul)
};

// One step of one lane: read the node at shared address p, test "x_j < b_i", move to
// the left child (next slot row) or the right child (+off); return the leaf value met (0.0f at
// internal nodes).  A leaf jumps to the lane's next tree root.  NAN_AWARE: NaN takes the node's
// default path.
template <bool NAN_AWARE, bool PADDED>
__device__ __forceinline__ float sliced_step_v(uint32_t& p, uint32_t rowaddr, uint32_t leafaddr,
                                               const StepConsts& k) {
  uint32_t x, y;
  float v;
  asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(p));
  // PADDED: row bases are aligned to the attribute field, so OR == ADD and the leaf is the one
  // address row | amask; DENSE: add, and test the attribute field itself
  const uint32_t off = y & k.amask;
  const uint32_t addr = PADDED ? ((y & k.amask) | rowaddr) : (rowaddr + off);
  asm("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr));
  bool go_left = v < __uint_as_float(x);
  if (NAN_AWARE) go_left = go_left || ((v != v) && (y & k.dlbit));
  const bool leaf = PADDED ? (addr == leafaddr) : (off == k.amask);
  // y >> (F+3) as a high multiply: IMAD.HI runs on the FMA pipe, relieving the ALU pipe
  p += (go_left && !leaf) ? (uint32_t)kSlotBytes : __umulhi(y, k.shmul);
  return __uint_as_float(leaf ? x : 0u);
}

// fp32 sum of two consecutive step values of one chain, then ONE fp64 add: exact, because two
// consecutive steps never both meet a nonzero leaf (every tree has an internal root in the sliced
// encoding, and the terminal leaf is 0.0), so the fp32 add is x + 0 = x.  Internal nodes add
// +0.0, which leaves an fp64 sum that started at +0.0 unchanged.
__device__ __forceinline__ void add_pair(double& acc, float v1, float v2) {
  double dv;
  asm("cvt.f64.f32 %0, %1;" : "=d"(dv) : "f"(__fadd_rn(v1, v2)));
  acc += dv;
}

template <bool NAN_AWARE, bool PADDED>
__device__ __forceinline__ void walk_columns2(uint32_t pA, uint32_t pB, uint32_t pe,
                                              uint32_t rowA, uint32_t rowB, const StepConsts& k,
                                              double& accA, double& accB) {
  // two independent samples per lane (ILP): while one chain waits on shared memory the other
  // issues; a chain that reached its terminal self-loop steps harmlessly
  const uint32_t leafA = rowA | k.amask, leafB = rowB | k.amask;
  accA = 0.0;
  accB = 0.0;
  while ((pA != pe) | (pB != pe)) {
    const float a1 = sliced_step_v<NAN_AWARE, PADDED>(pA, rowA, leafA, k);
    const float b1 = sliced_step_v<NAN_AWARE, PADDED>(pB, rowB, leafB, k);
    const float a2 = sliced_step_v<NAN_AWARE, PADDED>(pA, rowA, leafA, k);
    const float b2 = sliced_step_v<NAN_AWARE, PADDED>(pB, rowB, leafB, k);
    add_pair(accA, a1, a2);
    add_pair(accB, b1, b2);
  }
}

// One chain with the per-leaf diagnostics (caller leaf ids, fingerprint).
template <bool NAN_AWARE, bool PADDED>
__device__ __forceinline__ double walk_columns_leaf(uint32_t p, uint32_t pe, uint32_t rowaddr,
                                                    const StepConsts& k, uint32_t sbase,
                                                    const SlicedKArgs& a,
                                                    const int32_t* __restrict__ leaf_meta,
                                                    int64_t i, uint64_t& fp) {
  const uint32_t leafaddr = rowaddr | k.amask;
  double acc = 0.0;
  while (p != pe) {
    const uint32_t lp = p;
    uint32_t yy;
    asm("ld.shared.u32 %0, [%1];" : "=r"(yy) : "r"(lp + 4));
    const float v = sliced_step_v<NAN_AWARE, PADDED>(p, rowaddr, leafaddr, k);
    add_pair(acc, v, 0.0f);
    if ((yy & k.amask) == k.amask) {
      const uint32_t slot_word = (lp - sbase) >> 3;
      const int2 m = *reinterpret_cast<const int2*>(&leaf_meta[2 * slot_word]);
      if (a.o.out_leaf) a.o.out_leaf[i * a.o.T_leaf + m.x] = m.y;
      fp += mix64(((uint64_t)(uint32_t)m.x << 32) | (uint32_t)m.y);
    }
  }
  return acc;
}

// Rows too wide to stage (e.g. 2000 attributes) are read from global memory through L1; this walk
// is always NaN-aware and never reads past the row for a leaf.
template <bool LEAF>
__device__ __forceinline__ double walk_columns_global(uint32_t p, uint32_t pe,
                                                      const float* __restrict__ row,
                                                      const StepConsts& k, uint32_t sbase,
                                                      const SlicedKArgs& a,
                                                      const int32_t* __restrict__ leaf_meta,
                                                      int64_t i, uint64_t& fp) {
  double acc = 0.0;
  const char* rowb = reinterpret_cast<const char*>(row);
  while (p != pe) {
    uint32_t x, y;
    asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(p));
    const uint32_t off = y & k.amask;
    const bool leaf = off == k.amask;
    const float v = __ldg(reinterpret_cast<const float*>(rowb + (leaf ? 0u : off)));
    const bool go_left = (v < __uint_as_float(x)) || ((v != v) && (y & k.dlbit));
    const uint32_t delta = (go_left && !leaf) ? (uint32_t)kSlotBytes : __umulhi(y, k.shmul);
    if (leaf) {
      acc += (double)__uint_as_float(x);
      if (LEAF && delta) {
        const int2 m = *reinterpret_cast<const int2*>(&leaf_meta[2 * ((p - sbase) >> 3)]);
        if (a.o.out_leaf) a.o.out_leaf[i * a.o.T_leaf + m.x] = m.y;
        fp += mix64(((uint64_t)(uint32_t)m.x << 32) | (uint32_t)m.y);
      }
    }
    p += delta;
  }
  return acc;
}

// Two chains over rows in global memory (always NaN-aware; a leaf reads the row's first float,
// which is in bounds, and discards it).
__device__ __forceinline__ float global_step_v(uint32_t& p, const char* __restrict__ row,
                                               const StepConsts& k) {
  uint32_t x, y;
  asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(p));
  const uint32_t off = y & k.amask;
  const bool leaf = off == k.amask;
  const float v = __ldg(reinterpret_cast<const float*>(row + (leaf ? 0u : off)));
  const bool go_left = (v < __uint_as_float(x)) || ((v != v) && (y & k.dlbit));
  p += (go_left && !leaf) ? (uint32_t)kSlotBytes : __umulhi(y, k.shmul);
  return __uint_as_float(leaf ? x : 0u);
}

__device__ __forceinline__ void walk_columns2_global(uint32_t pA, uint32_t pB, uint32_t pe,
                                                     const float* rowA, const float* rowB,
                                                     const StepConsts& k, double& accA,
                                                     double& accB) {
  const char* ra = reinterpret_cast<const char*>(rowA);
  const char* rb = reinterpret_cast<const char*>(rowB);
  accA = 0.0;
  accB = 0.0;
  while ((pA != pe) | (pB != pe)) {
    const float a1 = global_step_v(pA, ra, k);
    const float b1 = global_step_v(pB, rb, k);
    const float a2 = global_step_v(pA, ra, k);
    const float b2 = global_step_v(pB, rb, k);
    add_pair(accA, a1, a2);
    add_pair(accB, b1, b2);
  }
}

template <bool LEAF, bool FUSED, int ROWS>
__global__ void __launch_bounds__(1024, 1) k_sliced(const __grid_constant__ SlicedKArgs a) {
  constexpr bool ROWS_SMEM = ROWS != kRowsGlobal;
  constexpr bool PADDED = ROWS == kRowsPadded;
  constexpr int C = kSlicedCols;
  extern __shared__ __align__(1024) unsigned char smem[];
  float* s_ring = reinterpret_cast<float*>(smem + a.forest_smem);
  uint64_t* s_full = reinterpret_cast<uint64_t*>(
      smem + a.forest_smem + (ROWS_SMEM ? (size_t)kRing * a.buf_floats * sizeof(float) : 0));
  // control block (kSlicedBarrierBytes): [kRingBars] full barriers, the slice barrier, the unit
  // counter at +64 B, the per-buffer release counters at +72 B
  uint64_t* s_forest = s_full + kRingBars;
  unsigned long long* s_next = reinterpret_cast<unsigned long long*>(s_full) + 8;  // +64 B
  int* s_cnt = reinterpret_cast<int*>(reinterpret_cast<unsigned char*>(s_full) + 72);
  static_assert(8 * (kRingBars + 1) <= 64 && 72 + 4 * kRing <= kSlicedBarrierBytes, "control block");
  const int lane = threadIdx.x & 31;
  const int warp = threadIdx.x >> 5;
  const int nwarps = blockDim.x >> 5;
  const int col = lane & (C - 1);   // lane column walked by this lane
  const int half = lane >> 4;       // half-warp: which rows of the work unit this lane walks
  const uint32_t F = (uint32_t)a.img.fbits;
  StepConsts k;
  k.amask = ((1u << F) - 1u) << 2;
  k.dlbit = 1u << (F + 2);
  k.shmul = 1u << (32 - (F + 3));
  const int32_t ns = a.img.n_slices;
  const int32_t G = gridDim.x;
  const bool multipass = ns > G;
  const int64_t R = a.tile_rows;
  const int64_t ntiles = (a.n + R - 1) / R;
  const int rs = a.row_stride;

  if (threadIdx.x == 0) {
    // full barriers: one arrive.expect_tx per TMA fill, or 32 cp.async arrivals (misaligned X)
    const uint32_t arrivals = (ROWS == kRowsDense && !a.x_aligned) ? 32u : 1u;
    for (int b = 0; b < kRingBars; b++) mbar_init(&s_full[b], arrivals);
    for (int b = 0; b < kRing; b++) s_cnt[b] = 0;
    *s_next = 0ull;
    mbar_init(s_forest, 1);
    fence_mbar_init();
  }
  __syncthreads();

  // a6: stage tile `tile` (CTA-wide tile sequence number seq) into ring buffer b; called by one
  // whole warp
  auto issue_tile = [&](int64_t tile, int b, uint32_t seq) {
    const int64_t r0 = tile * R;
    float* dst = s_ring + (size_t)b * a.buf_floats;
    uint64_t* bar = &s_full[ring_bar(seq)];
    if (PADDED) {
      // one 2-D tensor copy: box [row_stride][R] at (0, r0); columns >= d and rows >= n are
      // zero-filled by the TMA unit and still counted in the transaction bytes
      if (lane == 0) {
        fence_proxy_async_smem();
        mbar_expect_tx(bar, (uint32_t)(R * rs * sizeof(float)));
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
            " [%0], [%1, {%2, %3}], [%4];" ::"r"(smem_u32(dst)),
            "l"(reinterpret_cast<uint64_t>(&a.tmap)), "r"(0), "r"((int32_t)r0), "r"(smem_u32(bar))
            : "memory");
      }
    } else {
      const int64_t nr = (a.n - r0) < R ? (a.n - r0) : R;
      const uint32_t bytes = (uint32_t)(nr * a.d * sizeof(float));
      const float* src = a.X + r0 * a.d;
      if (a.x_aligned) {
        if (lane == 0) {
          const uint32_t body = bytes & ~15u;
          for (uint32_t q = body / 4; q < bytes / 4; q++) dst[q] = __ldg(&src[q]);  // <= 3 floats
          fence_proxy_async_smem();
          mbar_expect_tx(bar, body);
          if (body) bulk_g2s_big(dst, src, body, bar);
        }
      } else {
        // misaligned X: 4-byte cp.async copies by the warp, each lane's completion counted on the
        // buffer's mbarrier (initialised with 32 arrivals for this path)
        const uint32_t cnt = bytes / 4;
        for (uint32_t q = lane; q < cnt; q += 32)
          asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst + q)), "l"(src + q)
                       : "memory");
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(bar))
                     : "memory");
      }
    }
    __syncwarp();
  };

  // release ring buffer b after one work unit; the warp finishing the tile's last unit refills it
  // with the tile kRing ahead (acquire fence after observing the counter)
  auto release = [&](int b, int units, int64_t it, int64_t my_tiles, int64_t t0, int64_t ts,
                     uint32_t seq) {   // seq: the tile sequence number of the released tile
    __syncwarp();
    int last = 0;
    if (lane == 0) {
      __threadfence_block();
      last = atomicAdd(&s_cnt[b], 1) == units - 1;
      if (last) { atomicExch(&s_cnt[b], 0); __threadfence_block(); }
    }
    last = __shfl_sync(0xffffffffu, last, 0);
    if (last && it + kRing < my_tiles) issue_tile(t0 + (it + kRing) * ts, b, seq + (uint32_t)kRing);
  };

  uint32_t g = 0;  // tiles this CTA has consumed so far (identical in every warp)
  uint32_t ph_forest = 0;
  for (int32_t sl = multipass ? (int32_t)blockIdx.x : (int32_t)blockIdx.x % ns; sl < ns;
       sl += multipass ? G : ns) {
    const int64_t t0 = multipass ? 0 : blockIdx.x / ns;
    const int64_t ts = multipass ? 1 : a.cps;
    const int64_t my_tiles = t0 < ntiles ? (ntiles - t0 + ts - 1) / ts : 0;
    if (warp == 0) {
      if (lane == 0) {  // a7: the slice, one bulk copy of slots x 128 bytes
        const uint32_t bytes = (uint32_t)a.img.slots[sl] * (uint32_t)kSlotBytes;
        fence_proxy_async_smem();
        mbar_expect_tx(s_forest, bytes);
        bulk_g2s_big(smem, a.img.nodes + (size_t)sl * a.img.slots_max * C * 2, bytes, s_forest);
      }
      if (ROWS_SMEM)
        for (int64_t q = 0; q < kRing && q < my_tiles; q++)
          issue_tile(t0 + q * ts, (int)((g + q) % kRing), g + (uint32_t)q);
    }
    const uint32_t sbase = smem_u32(smem);
    const uint32_t p0 = sbase + (uint32_t)col * 8u;
    const uint32_t pe = sbase + ((uint32_t)a.img.col_len[sl * C + col] * C + (uint32_t)col) * 8u;
    const int32_t* __restrict__ leaf_meta = a.img.leaf_meta + (size_t)sl * a.img.slots_max * C * 2;
    mbar_wait(s_forest, ph_forest);
    ph_forest ^= 1u;

    if (!LEAF) {
      // Dynamic schedule over work units of 4 rows {u, u+16, u+32, u+48} of a 64-row tile: half h
      // of the warp walks rows u+16h (chain A) and u+32+16h (chain B).  Warps grab units from a CTA
      // counter, so a slow unit delays nobody (claims may run ahead of the ring: see ring_bar).
      // Rows too wide to stage are read from global memory with the same schedule.
      constexpr int kUnits = kSlicedTileRows / 4;
      const uint64_t total = (uint64_t)my_tiles * kUnits;
      for (;;) {
        unsigned long long q = 0;
        if (lane == 0) q = atomicAdd(s_next, 1ull);
        q = __shfl_sync(0xffffffffu, q, 0);
        if (q >= total) break;
        const int64_t it = (int64_t)(q / kUnits);
        const int u = (int)(q % kUnits);
        const uint32_t gt = g + (uint32_t)it;
        const int b = (int)(gt % kRing);
        const int64_t r0 = (t0 + it * ts) * R;
        const int nr = (int)((a.n - r0) < R ? (a.n - r0) : R);
        if (ROWS_SMEM) mbar_wait(&s_full[ring_bar(gt)], ring_parity(gt));
        if (u < nr) {
          const int rA = u + 16 * half, rB = rA + 32;
          const bool okA = rA < nr, okB = rB < nr;
          const uint32_t pA = okA ? p0 : pe, pB = okB ? p0 : pe;
          double accA, accB;
          if (ROWS_SMEM) {
            const float* tbuf = s_ring + (size_t)b * a.buf_floats;
            const float* rowA = tbuf + (size_t)(okA ? rA : u) * rs;
            const float* rowB = tbuf + (size_t)(okB ? rB : u) * rs;
            bool has_nan = false;
            for (int j = col; j < a.d; j += C) has_nan |= (rowA[j] != rowA[j]) | (rowB[j] != rowB[j]);
            if (__any_sync(0xffffffffu, has_nan))
              walk_columns2<true, PADDED>(pA, pB, pe, smem_u32(rowA), smem_u32(rowB), k, accA, accB);
            else
              walk_columns2<false, PADDED>(pA, pB, pe, smem_u32(rowA), smem_u32(rowB), k, accA, accB);
          } else {
            walk_columns2_global(pA, pB, pe, a.X + (r0 + (okA ? rA : u)) * a.d,
                                 a.X + (r0 + (okB ? rB : u)) * a.d, k, accA, accB);
          }
          // a9: one butterfly for the four rows: after the first exchange (xor 8) lanes with bit 3
          // clear hold chain-A pair sums and lanes with bit 3 set chain-B pair sums; three more
          // steps finish all four (fixed order).  Lanes 0, 8, 16, 24 own rows u, u+32, u+16, u+48.
          const bool b3 = lane & 8;
          double v = (b3 ? accB : accA) + __shfl_xor_sync(0xffffffffu, b3 ? accA : accB, 8);
#pragma unroll
          for (int o = 4; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
          const int rr = b3 ? rB : rA;
          if ((lane & 7) == 0 && (b3 ? okB : okA)) {
            const int64_t i = r0 + rr;
            if (FUSED) write_scalar(a.o, i, v);
            else a.o.raw[(size_t)sl * a.n + i] = v;
          }
        }
        if (ROWS_SMEM) release(b, kUnits, it, my_tiles, t0, ts, gt);
      }
      g += (uint32_t)my_tiles;
    } else {
      // static schedule (leaf / fingerprint diagnostics): warp w walks rows
      // w (half 0) and w + 32 (half 1) of every tile, one chain per lane
      for (int64_t it = 0; it < my_tiles; it++, g++) {
        const int b = (int)(g % kRing);
        const int64_t tile = t0 + it * ts;
        const int64_t r0 = tile * R;
        const int nr = (int)((a.n - r0) < R ? (a.n - r0) : R);
        const float* tbuf = s_ring + (size_t)b * a.buf_floats;
        if (ROWS_SMEM) mbar_wait(&s_full[ring_bar(g)], ring_parity(g));
        for (int r = warp; r < (int)(R / 2); r += nwarps) {
          const int rr = r + 32 * half;
          const bool ok = rr < nr;
          const int64_t i = r0 + (ok ? rr : 0);
          uint64_t fp = 0;
          double acc = 0.0;
          if (ROWS_SMEM) {
            const float* row = tbuf + (size_t)(ok ? rr : 0) * rs;
            bool has_nan = false;
            if (ok)
              for (int j = col; j < a.d; j += C) has_nan |= row[j] != row[j];
            const uint32_t p = ok ? p0 : pe;
            if (__any_sync(0xffffffffu, has_nan))
              acc = walk_columns_leaf<true, PADDED>(p, pe, smem_u32(row), k, sbase, a, leaf_meta, i, fp);
            else
              acc = walk_columns_leaf<false, PADDED>(p, pe, smem_u32(row), k, sbase, a, leaf_meta, i, fp);
          } else if (ok) {
            acc = walk_columns_global<LEAF>(p0, pe, a.X + i * a.d, k, sbase, a, leaf_meta, i, fp);
          }
          // a9: butterfly within each half-warp (16 lane sums, fixed order); lanes 0 and 16 write
#pragma unroll
          for (int o = 8; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
          if (LEAF) {
#pragma unroll
            for (int o = 8; o > 0; o >>= 1) fp += __shfl_xor_sync(0xffffffffu, fp, o);
          }
          if (col == 0 && ok) {
            if (FUSED) write_scalar(a.o, i, acc);
            else a.o.raw[(size_t)sl * a.n + i] = acc;
            if (LEAF && a.o.out_fp)
              atomicAdd(reinterpret_cast<unsigned long long*>(&a.o.out_fp[i]), (unsigned long long)fp);
          }
        }
        if (ROWS_SMEM) release(b, nwarps, it, my_tiles, t0, ts, g);
      }
    }
    __syncthreads();  // every warp is done with this slice (multi-pass reload)
    if (threadIdx.x == 0) *s_next = 0ull;
    __syncthreads();
  }
}

// ------------------------------------------------------------------ rank-coded sliced strategy
// Reading R7: "x_j < b_i" is evaluated on exact order-preserving codes.  Per attribute
// the forest's distinct thresholds are sorted (tab); a row value x becomes
// code(x) = #{k : tab[k] <= x}, and a node whose threshold is tab[j] stores t = j + 1, so that
// x < tab[j]  <=>  code(x) < t  — the same decision, bit for bit, for every x (NaN is coded
// kCodeNan and takes the default path; ties and signed zeros follow IEEE <=).  Two things get
// cheaper on the hot loop: an attribute read is 2 bytes, so the two rows a warp walks at once share
// one 128-byte bank line (1 shared-memory wavefront instead of 2), and an internal node word
// (t < 2^15) is a subnormal float, so "add the leaf value" becomes an unconditional
// flush-to-zero fp32 add of the word just read (internal words add exactly 0).

// k_encode_rows: X (n x d fp32 row-major) -> code tiles.  One thread per (row, code slot); the
// attribute's threshold table is searched by bisection in shared memory (or L2 when too large).
struct EncodeRowsArgs {
  const float* X;
  int64_t n;
  int32_t d, nf, fbits, rb, n_thr;
  const float* tab;
  const int32_t* off;
  uint16_t* codes;
  int32_t tstride;   // bytes per code tile (rows + trailer)
  int64_t ntiles;
  const int32_t* slot_attr;   // [2^fbits] attribute of each code slot, -1 = pad (R10)
};

__device__ __forceinline__ uint32_t code_row_off(int r, int rb) {
  return rb == 64 ? (((uint32_t)(r & 15) << 7) | ((uint32_t)((r >> 4) & 1) << 6) | ((uint32_t)(r >> 5) << 11))
                  : (uint32_t)r * (uint32_t)rb;
}
// Rows of >= 128 bytes: the rows walked by the second half-warp (r & 16) store attribute slot j at
// slot j ^ 32 (their 64-byte halves swapped), so the low, most-tested attributes of the two rows
// one warp reads at once sit in different banks (C3 ncu before: 25 % of shared wavefronts were
// bank-conflict replays between the two half-warps' rows).  Returned in u16 slots.
__device__ __forceinline__ uint32_t code_slot_swz(int r, int rb) {
  return (rb >= 128 && (r & 16)) ? 32u : 0u;
}

template <bool SMEM>
__global__ void __launch_bounds__(1024) k_encode_rows(const EncodeRowsArgs a) {
  extern __shared__ __align__(16) float s_tab[];
  const float* __restrict__ tab = a.tab;
  const int32_t* __restrict__ off = a.off;
  if (SMEM) {
    int32_t* s_off = reinterpret_cast<int32_t*>(s_tab + a.n_thr);
    for (int i = threadIdx.x; i < a.n_thr; i += blockDim.x) s_tab[i] = __ldg(&a.tab[i]);
    for (int i = threadIdx.x; i <= a.nf; i += blockDim.x) s_off[i] = __ldg(&a.off[i]);
    __syncthreads();
    tab = s_tab;
    off = s_off;
  }
  const int64_t total = a.ntiles * 64 << a.fbits;
  const int smask = (1 << a.fbits) - 1;
  const int64_t tile_u16 = a.tstride >> 1;
  const int32_t flag_u16 = 32 * a.rb;   // trailer word (after the rows)
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = e >> a.fbits;
    const int j = (int)(e & smask);            // code slot
    const int att = __ldg(&a.slot_attr[j]);    // attribute coded there
    uint16_t code = kCodePad;
    if (r < a.n && att >= 0) {
      const float x = __ldg(&a.X[r * a.d + att]);
      if (x != x) {
        code = kCodeNan;
        *reinterpret_cast<int32_t*>(a.codes + (r >> 6) * tile_u16 + flag_u16) = 1;
      } else {
        const int32_t b0 = off[att];
        int32_t lo = b0, len = off[att + 1] - b0;
        while (len > 0) {   // lo := first index with tab[lo] > x
          const int32_t h = len >> 1;
          if (tab[lo + h] <= x) { lo += h + 1; len -= h + 1; }
          else len = h;
        }
        code = (uint16_t)(lo - b0);
      }
    }
    a.codes[(r >> 6) * tile_u16 + (code_row_off((int)(r & 63), a.rb) >> 1) + (j ^ code_slot_swz((int)(r & 63), a.rb))] = code;
  }
}

// k_encode_rows_banks: the same codes from bank-private tables (encode.cpp build_code_banks): the
// CTA bulk-copies the table image into shared memory once; warp w codes rows w, w + W, ... one pass
// at a time, lane l of pass p bisecting attribute desc[p][l] inside its own banks (one wavefront
// per probe for the whole warp).
struct EncodeBanksArgs {
  const float* X;
  int64_t n;
  int32_t d, rb, passes, img_bytes;
  const float* img;
  const int4* desc;
  uint16_t* codes;
  int32_t tstride;   // bytes per code tile (rows + trailer)
  int64_t nrows;   // ntiles * 64
};

template <bool RB64>
__global__ void __launch_bounds__(1024, 1) k_encode_rows_banks(const EncodeBanksArgs a) {
  extern __shared__ __align__(1024) float s_img[];
  __shared__ uint64_t s_bar;
  const int lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    mbar_init(&s_bar, 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    fence_proxy_async_smem();
    mbar_expect_tx(&s_bar, (uint32_t)a.img_bytes);
    bulk_g2s_big(s_img, a.img, (uint32_t)a.img_bytes, &s_bar);
  }
  mbar_wait(&s_bar, 0);
  const int rb = RB64 ? 64 : a.rb;
  const int64_t tile_u16 = a.tstride >> 1;
  const int32_t flag_u16 = 32 * rb;   // trailer word (after the rows)
  // a warp codes kR consecutive rows at once (independent bisections interleaved).  Work units
  // are (row group, pass) with the pass fastest: all passes of a row group run back to back, so
  // the row's X lines are still in L1 / L2 for its later passes and its code row is written whole
  // (passes outermost read X once per pass from HBM: C3 ncu 2.95 GB of DRAM traffic for 1.4 GB
  // algorithmic).  The next unit's attribute values are loaded before this unit is searched.
  constexpr int kR = 8;
  static_assert(64 % kR == 0, "a row group stays inside one tile");
  const int64_t wstride = (int64_t)gridDim.x * (blockDim.x >> 5) * kR;
  const int64_t w0 = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * kR;
  const uint32_t d = (uint32_t)a.d;
  const int P = a.passes;
  auto load_x = [&](int64_t r0, int feat, float* x) {
    const float* xr = a.X + (feat >= 0 ? feat : 0) + r0 * a.d;
    if (feat >= 0 && r0 + kR <= a.n) {
#pragma unroll
      for (int q = 0; q < kR; q++) x[q] = __ldg(xr + q * d);
    } else {
#pragma unroll
      for (int q = 0; q < kR; q++) x[q] = (feat >= 0 && r0 + q < a.n) ? __ldg(xr + q * d) : 0.0f;
    }
  };
  float xn[kR];
  int4 dn = __ldg(&a.desc[lane]);
  if (w0 < a.nrows) load_x(w0, dn.y, xn);
  int64_t r0 = w0;
  int p = 0;
  while (r0 < a.nrows) {
    const int4 dsc = dn;
    float x[kR];
#pragma unroll
    for (int q = 0; q < kR; q++) x[q] = xn[q];
    // next unit: pass p + 1 of this group, or pass 0 of the next group
    int64_t r1 = r0;
    int p1 = p + 1;
    if (p1 == P) { p1 = 0; r1 += wstride; }
    if (r1 < a.nrows) {
      dn = __ldg(&a.desc[p1 * 32 + lane]);
      load_x(r1, dn.y, xn);
    }
    const int slot = dsc.x, feat = dsc.y;
    const uint32_t base = smem_u32(s_img) + (uint32_t)dsc.z;   // element 0 of this lane's table
    const uint32_t stride = (uint32_t)dsc.w >> 16;               // bytes between elements
    const uint32_t lstride = 31u - __clz(stride | 1u);           // stride is a power of two
    const int K = dsc.w & 0xffff;
    const int top = K > 0 ? 1 << (31 - __clz(K)) : 0;            // largest power of two <= K
    // pos := #{thresholds <= x} by Shar's bisection (uniform trip count for every row of this
    // lane, every probe in range, no bounds tests): after the first probe at top - 1 the count
    // lies in [pos, pos + top]; each halving step keeps it in [pos, pos + step]; a last probe
    // at pos decides between pos and pos + 1.  Positions are byte offsets (pos * stride).
    // rows kept as absolute probe addresses ad = base + pos; one probe = address add, LDS,
    // FSETP, predicated add (4 instructions; the select + add the compiler emitted made it 5)
    uint32_t pos[kR];
#pragma unroll
    for (int q = 0; q < kR; q++) pos[q] = 0;
    if (top > 0) {
      float v0;
      asm("ld.shared.f32 %0, [%1];" : "=f"(v0) : "r"(base + (uint32_t)(top - 1) * stride));
      const uint32_t hi = (uint32_t)(K - top) * stride;
      uint32_t ad[kR];
#pragma unroll
      for (int q = 0; q < kR; q++) ad[q] = base + (v0 <= x[q] ? hi : 0u);
      for (uint32_t stepb = ((uint32_t)top >> 1) * stride; stepb >= stride; stepb >>= 1) {
        const uint32_t off = stepb - stride;
#pragma unroll
        for (int q = 0; q < kR; q++)
          asm("{\n\t.reg .f32 t;\n\t.reg .pred p;\n\t.reg .u32 a;\n\t"
              "add.u32 a, %0, %2;\n\t"
              "ld.shared.f32 t, [a];\n\t"
              "setp.le.f32 p, t, %1;\n\t"
              "@p add.u32 %0, %0, %3;\n\t}"
              : "+r"(ad[q]) : "f"(x[q]), "r"(off), "r"(stepb));
      }
#pragma unroll
      for (int q = 0; q < kR; q++) {
        float v;
        asm("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(ad[q]));
        pos[q] = ((ad[q] - base) >> lstride) + (v <= x[q] ? 1u : 0u);
      }
    }
    if (slot >= 0) {
      // the kR rows r0 .. r0+kR-1 of a group (r0 % kR == 0) sit at a constant stride in the
      // tile: 128 bytes apart in the 64-byte-row layout (same bits 4-5 of r), rb otherwise
      uint16_t* tb = a.codes + (r0 >> 6) * tile_u16;
      uint16_t* p0 = tb + (code_row_off((int)(r0 & 63), rb) >> 1) + (slot ^ code_slot_swz((int)(r0 & 63), rb));
      const int rstride = RB64 ? 64 : (rb >> 1);
      bool nan = false;
      if (feat >= 0 && r0 + kR <= a.n) {
#pragma unroll
        for (int q = 0; q < kR; q++) {
          const bool isnan_q = x[q] != x[q];
          nan |= isnan_q;
          p0[q * rstride] = isnan_q ? kCodeNan : (uint16_t)pos[q];
        }
      } else {
#pragma unroll
        for (int q = 0; q < kR; q++) {
          uint16_t code = (uint16_t)pos[q];
          if (feat < 0 || r0 + q >= a.n) code = kCodePad;
          else if (x[q] != x[q]) { code = kCodeNan; nan = true; }
          p0[q * rstride] = code;
        }
      }
      if (nan) *reinterpret_cast<int32_t*>(tb + flag_u16) = 1;
    }
    r0 = r1;
    p = p1;
  }
}

// One row: fixed-order fp64 sum of the row's parts per class, then base / average / argmax and one
// round to fp32 (Z14, Z17).  Parts are read through L2 (they may have been written by other SMs).
// The row's parts are walked in CSR order (class by class, each class's parts in slice order) in
// batches of kFinBatch independent loads issued before any is added, so a thread waits for one
// memory round trip per batch instead of one per part; the additions keep the same order.
constexpr int kFinBatch = 8;
__device__ __forceinline__ void finalize_row(const FinalizeArgs& a, int64_t i) {
  const int32_t C = a.n_classes;
  const int32_t np = a.class_ptr ? __ldg(&a.class_ptr[C]) : C;
  int best = 0;
  double bv = 0.0;
  auto emit = [&](int32_t c, double s) {
    if (a.raw_out) { a.raw_out[i * C + c] = s; return; }
    double v;
    if (a.agg == TAHOE_AGG_VOTE) v = s;
    else if (a.agg == TAHOE_AGG_AVERAGE) v = s / (double)a.n_trees_full + (double)a.base;
    else v = s + (double)a.base;
    a.out[i * C + c] = (float)v;
    if (c == 0 || v > bv) { best = c; bv = v; }
  };
  int32_t c = 0;
  int32_t cend = a.class_ptr ? __ldg(&a.class_ptr[1]) : 1;   // first part of class c + 1
  double s = 0.0;
  for (int32_t p0 = 0; p0 < np; p0 += kFinBatch) {
    double v[kFinBatch];
#pragma unroll
    for (int k = 0; k < kFinBatch; k++) {
      const int32_t p = p0 + k;
      v[k] = 0.0;
      if (p < np) {
        const int64_t part = a.class_ptr ? (int64_t)__ldg(&a.class_parts[p]) : (int64_t)p;
        v[k] = __ldcg(&a.partial[part * a.part_stride + i * a.row_stride]);
      }
    }
#pragma unroll
    for (int k = 0; k < kFinBatch; k++) {
      const int32_t p = p0 + k;
      if (p < np) {
        while (p == cend) {   // classes ending before part p (empty classes included)
          emit(c, s);
          s = 0.0;
          c++;
          cend = a.class_ptr ? __ldg(&a.class_ptr[c + 1]) : c + 1;
        }
        s += v[k];
      }
    }
  }
  for (; c < C; c++) {
    emit(c, s);
    s = 0.0;
  }
  if (!a.raw_out && a.out_class) {
    if (a.agg == TAHOE_AGG_BINARY) a.out_class[i] = bv > 0.0 ? 1 : 0;
    else if (a.agg == TAHOE_AGG_CLASS_SUM || a.agg == TAHOE_AGG_VOTE) a.out_class[i] = best;
    else a.out_class[i] = 0;
  }
}

struct CodedKArgs {
  DevSliced img;
  const uint16_t* codes;
  int64_t n;
  int32_t forest_smem;   // bytes reserved for the slice (multiple of 1024)
  int32_t tile_bytes;    // the 64 code rows of a tile (its NaN flag follows them)
  int32_t tstride;       // bytes per tile (rows + trailer of max(128, row bytes)), in HBM and in the ring
  int32_t rb;            // bytes per code row
  int32_t cps;           // CTAs per slice (single-pass, no cta_start)
  const int32_t* cta_start;  // or: slice s is worked by CTAs [cta_start[s], cta_start[s+1])
  int32_t prefetch;      // entries of the CTA's tile sequence to prefetch into L2 ahead (0 = none)
  int32_t ring;          // ring depth (kSlicedRing .. kCodedRingMax): as many tiles as shared memory holds
  uint32_t ring_m, bars_m;   // ceil(2^32 / ring), ceil(2^32 / (2 ring)): division by multiply-high
  double* prof;          // PROF instantiation: load-balance statistics (prof_unit), else null
  int32_t* tile_next;    // [ns] next unclaimed tile of each slice (zeroed per launch)
  int32_t* cta_on;       // [ns] CTAs currently on each slice (zeroed per launch)
  const float* work;     // [ns] simulated lane-steps per row of each slice (slice choice weights)
  OutArgs o;
};

// x / d and x % d for a small runtime divisor d (<= 16) and x < 2^24: q = umulhi(x, ceil(2^32 / d))
// is exact there (error term x (m d - 2^32) / 2^32 < x d / 2^32 < 1 / d)
__device__ __forceinline__ uint32_t fdiv_small(uint32_t x, uint32_t m) { return __umulhi(x, m); }
__device__ __forceinline__ uint32_t fmod_small(uint32_t x, uint32_t d, uint32_t m) {
  return x - __umulhi(x, m) * d;
}

// One step on a coded slice: node {x = t or leaf value, y}, attribute code at (y & amask) | row,
// left iff code < t (NaN-aware: or NaN and default-left), right / next root at +(y >> (F+2)).
// Returns the node word as a float: the leaf value, or a subnormal (flushed to 0 by the add).
// yout (diagnostic walks only): receives the node word's y, so the caller can tell a leaf.
template <bool NAN_AWARE, bool SWZ>
__device__ __forceinline__ float coded_step(uint32_t& p, uint32_t rowaddr, uint32_t amask,
                                            uint32_t dlbit, uint32_t shmul,
                                            uint32_t* yout = nullptr) {
  uint32_t x, y;
  int32_t c;
  asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(p));
  if (yout) *yout = y;
  // SWZ: rowaddr carries the swizzle (code_slot_swz), XORed into the attribute offset
  asm("ld.shared.s16 %0, [%1];" : "=r"(c) : "r"(SWZ ? ((y & amask) ^ rowaddr) : ((y & amask) | rowaddr)));
  bool go_left = (uint32_t)c < x;
  if (NAN_AWARE) go_left = go_left || ((c == (int32_t)(int16_t)kCodeNan) && (y & dlbit));
  p += go_left ? (uint32_t)kSlotBytes : __umulhi(y, shmul);
  return __uint_as_float(x);
}

// flush-to-zero fp32 add of two consecutive step words (internal words are subnormal -> +0; at
// most one of two consecutive steps meets a leaf), then one fp64 add: exact.
__device__ __forceinline__ void add_pair_ftz(double& acc, float v1, float v2) {
  float s;
  asm("add.rn.ftz.f32 %0, %1, %2;" : "=f"(s) : "f"(v1), "f"(v2));
  double dv;
  asm("cvt.f64.f32 %0, %1;" : "=d"(dv) : "f"(s));
  acc += dv;
}

#ifndef TAHOE_CODED_EXIT
#define TAHOE_CODED_EXIT 4   // steps per chain between exit tests of walk_coded2 (even)
#endif
constexpr int kCodedExit = TAHOE_CODED_EXIT;
template <bool NAN_AWARE, bool SWZ>
__device__ __forceinline__ void walk_coded2(uint32_t pA, uint32_t pB, uint32_t pe, uint32_t rowA,
                                            uint32_t rowB, uint32_t amask, uint32_t dlbit,
                                            uint32_t shmul, double& accA, double& accB) {
  accA = 0.0;
  accB = 0.0;
  // kCodedExit steps per chain between exit tests (a finished chain idles on its column's
  // self-looping terminal leaf of value 0): the test costs 3 of ~37 instructions per two-step round
  while ((pA != pe) | (pB != pe)) {
#pragma unroll
    for (int k = 0; k < kCodedExit / 2; k++) {
      const float a1 = coded_step<NAN_AWARE, SWZ>(pA, rowA, amask, dlbit, shmul);
      const float b1 = coded_step<NAN_AWARE, SWZ>(pB, rowB, amask, dlbit, shmul);
      const float a2 = coded_step<NAN_AWARE, SWZ>(pA, rowA, amask, dlbit, shmul);
      const float b2 = coded_step<NAN_AWARE, SWZ>(pB, rowB, amask, dlbit, shmul);
      add_pair_ftz(accA, a1, a2);
      add_pair_ftz(accB, b1, b2);
    }
  }
}

// Leaf diagnostics of a coded walk (per-(sample, tree) leaf ids, fingerprint): the node word just
// read at q was a leaf iff its attribute field is all ones (the pad code) and q is not the
// column's terminal self-loop pe; its caller {tree, node} ids sit in leaf_meta at the same word
// index as in the slice.
__device__ __forceinline__ void record_leaf(uint32_t q, uint32_t y, uint32_t pe, uint32_t amask,
                                            uint32_t sbase, const int2* __restrict__ meta,
                                            int32_t* out_row, uint64_t& fp) {
  if ((y & amask) == amask && q != pe) {
    const int2 m = __ldg(&meta[(q - sbase) >> 3]);
    if (out_row) out_row[m.x] = m.y;
    fp += mix64(((uint64_t)(uint32_t)m.x << 32) | (uint32_t)m.y);
  }
}

// walk_coded2 with the leaf diagnostics: the same steps in the same order and the same fp32 / fp64
// additions; after every step the node just read is checked for a leaf.
template <bool NAN_AWARE, bool SWZ>
__device__ __forceinline__ void walk_coded2_leaf(uint32_t pA, uint32_t pB, uint32_t pe,
                                                 uint32_t rowA, uint32_t rowB, uint32_t amask,
                                                 uint32_t dlbit, uint32_t shmul, double& accA,
                                                 double& accB, uint32_t sbase,
                                                 const int2* __restrict__ meta, int32_t* outA,
                                                 int32_t* outB, uint64_t& fpA, uint64_t& fpB) {
  accA = 0.0;
  accB = 0.0;
  fpA = 0;
  fpB = 0;
  while ((pA != pe) | (pB != pe)) {
    uint32_t y, q;
    q = pA; const float a1 = coded_step<NAN_AWARE, SWZ>(pA, rowA, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outA, fpA);
    q = pB; const float b1 = coded_step<NAN_AWARE, SWZ>(pB, rowB, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outB, fpB);
    q = pA; const float a2 = coded_step<NAN_AWARE, SWZ>(pA, rowA, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outA, fpA);
    q = pB; const float b2 = coded_step<NAN_AWARE, SWZ>(pB, rowB, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outB, fpB);
    add_pair_ftz(accA, a1, a2);
    add_pair_ftz(accB, b1, b2);
  }
}

// walk_coded2 with per-lane timing (load-balance measurement, Table 3 analog): the
// same steps; each iteration records the SM clock, so `span` = cycles from the walk's start to the
// start of the lane's last iteration (a lane leaves the loop when both its chains are done).
template <bool NAN_AWARE, bool SWZ>
__device__ __forceinline__ void walk_coded2_prof(uint32_t pA, uint32_t pB, uint32_t pe, uint32_t rowA,
                                                 uint32_t rowB, uint32_t amask, uint32_t dlbit,
                                                 uint32_t shmul, double& accA, double& accB,
                                                 uint32_t& span) {
  accA = 0.0;
  accB = 0.0;
  const uint32_t t0 = (uint32_t)clock();
  uint32_t tl = t0;
  while ((pA != pe) | (pB != pe)) {
    tl = (uint32_t)clock();
    const float a1 = coded_step<NAN_AWARE, SWZ>(pA, rowA, amask, dlbit, shmul);
    const float b1 = coded_step<NAN_AWARE, SWZ>(pB, rowB, amask, dlbit, shmul);
    const float a2 = coded_step<NAN_AWARE, SWZ>(pA, rowA, amask, dlbit, shmul);
    const float b2 = coded_step<NAN_AWARE, SWZ>(pB, rowB, amask, dlbit, shmul);
    add_pair_ftz(accA, a1, a2);
    add_pair_ftz(accB, b1, b2);
  }
  span = tl - t0;
}

// Per-unit and per-lane load-balance statistics of a profiled walk (prof[8], device doubles):
// [0] sum over units of the CV of lane spans, [1] sum of mean/max lane span (lockstep efficiency),
// [2] units, [3] sum of mean lane span (cycles), [4] sum over warps of the CV of the lanes' total
// spans over the whole launch, [5] warps.
__device__ __forceinline__ void prof_unit(double* prof, uint32_t span) {
  const double x = (double)span;
  double s = x, q = x * x, m = x;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    s += __shfl_xor_sync(0xffffffffu, s, o);
    q += __shfl_xor_sync(0xffffffffu, q, o);
    m = fmax(m, __shfl_xor_sync(0xffffffffu, m, o));
  }
  if ((threadIdx.x & 31) == 0 && m > 0.0) {
    const double mean = s / 32.0, var = fmax(0.0, q / 32.0 - mean * mean);
    atomicAdd(&prof[0], sqrt(var) / mean);
    atomicAdd(&prof[1], mean / m);
    atomicAdd(&prof[2], 1.0);
    atomicAdd(&prof[3], mean);
  }
}
__device__ __forceinline__ void prof_lanes(double* prof, double total) {
  double s = total, q = total * total;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    s += __shfl_xor_sync(0xffffffffu, s, o);
    q += __shfl_xor_sync(0xffffffffu, q, o);
  }
  if ((threadIdx.x & 31) == 0 && s > 0.0) {
    const double mean = s / 32.0, var = fmax(0.0, q / 32.0 - mean * mean);
    atomicAdd(&prof[4], sqrt(var) / mean);
    atomicAdd(&prof[5], 1.0);
  }
}

// k_sliced_codes: k_sliced's persistent slice-stationary schedule (slice in shared memory, 3-deep
// ring of 64-row tiles refilled by the warp that finishes a tile, dynamic 4-row work units, one
// half-warp per row, two chains per lane) over code tiles (one 1-D bulk copy per tile).
// LEAF: the same schedule and walk, also writing per-(sample, tree) caller leaf ids (out_leaf, may
// be null) and accumulating fingerprints (out_fp, u64 atomic adds per slice).
// MODE 0: production; 1: LEAF (leaf ids / fingerprints); 2: PROF (per-lane spans, prof_unit)
template <bool FUSED, bool SWZ, int MODE>
__global__ void __launch_bounds__(1024, 1) k_sliced_codes(const __grid_constant__ CodedKArgs a) {
  constexpr bool LEAF = MODE == 1, PROF = MODE == 2;
  double lane_total = 0.0;   // PROF: this lane's spans over the launch
  constexpr int C = kSlicedCols;
  extern __shared__ __align__(1024) unsigned char smem[];
  unsigned char* s_ring = smem + a.forest_smem;
  // Producer / consumer ring (mbarrier hand-off only): warp PW (the last) stages the slice, claims
  // the slice's tiles from its global counter (so every CTA on a slice finishes with the slice) and
  // issues them into the ring, refilling buffer b once the kUnits units of its previous tile have
  // all arrived on empty[b] (and writing that tile's slice partials out first); the other 31 warps
  // claim 4-row work units from a CTA counter, wait on the tile's full barrier, walk, and arrive on
  // empty[b].  Entry e (of the CTA's stay on a slice) uses buffer e % ring and full barrier
  // e % (2 ring) with parity (e / (2 ring)) & 1: a consumer claiming e could only see a stale phase
  // if entry e - 2 ring had not arrived, but then e - ring is not issued either, and the 2 x 16
  // units of those two entries would hold 32 blocked consumers — there are 31 (the ring-wrap guard
  // of ring_bar, with a runtime depth).  Past the slice's last tile the producer issues kTerm
  // terminator entries (tile -1, no data: 2 x 16 units reach all 31 consumers' next claims); the
  // CTA then moves to the slice with the most remaining work per CTA (re-staging it), and the
  // barriers are re-initialised.
  const uint32_t ring = (uint32_t)a.ring, nbars = 2u * ring;
  constexpr int kUnits = kSlicedTileRows / 4;
  // control block (kCodedCtlBytes): [2 ring] full barriers, [ring] empty barriers, slice barrier,
  // unit counter (u32)
  uint64_t* s_full = reinterpret_cast<uint64_t*>(s_ring + (size_t)ring * a.tstride);
  uint64_t* s_empty = s_full + nbars;
  uint64_t* s_forest = s_empty + ring;
  unsigned int* s_next = reinterpret_cast<unsigned int*>(s_forest + 1);
  // slice partials of the tiles in the ring (consumers write, the producer stores them coalesced)
  double* s_part = reinterpret_cast<double*>(reinterpret_cast<unsigned char*>(s_full) + kCodedCtlBytes);
  const int lane = threadIdx.x & 31;
  const int warp = threadIdx.x >> 5;
  const int PW = (int)(blockDim.x >> 5) - 1;   // producer warp
  const int col = lane & (C - 1);
  const int half = lane >> 4;
  const uint32_t F = (uint32_t)a.img.fbits;
  const uint32_t amask = ((1u << F) - 1u) << 1;
  const uint32_t dlbit = 1u << (F + 1);
  const uint32_t shmul = 1u << (32 - (F + 2));
  const int32_t ns = a.img.n_slices;
  const int32_t G = gridDim.x;
  const bool multipass = ns > G;
  const int64_t R = kSlicedTileRows;
  const int64_t ntiles = (a.n + R - 1) / R;

  constexpr uint32_t kTerm = 2;
  static_assert(kTerm * kUnits >= 31 && kTerm <= kSlicedRing, "terminators reach every consumer");
  uint32_t ph_forest = 0;
  const uint32_t ring0 = smem_u32(s_ring);
  const uint32_t sbase = smem_u32(smem);
  int32_t* s_slice = reinterpret_cast<int32_t*>(s_next + 1);
  int32_t* s_tile = s_slice + 1;   // [ring] tile of the entry in each buffer (-1: terminator)
  if (threadIdx.x == 0) {
    // first slice: the weighted CTA map (or round-robin; CTA b of a multi-pass launch takes slice b)
    int32_t sl = (int32_t)blockIdx.x % ns;
    if (!multipass && a.cta_start) {
      sl = 0;
      while (sl + 1 < ns && __ldg(&a.cta_start[sl + 1]) <= (int32_t)blockIdx.x) sl++;
    } else if (multipass) {
      sl = (int32_t)blockIdx.x;
    }
    *s_slice = sl;
    atomicAdd(&a.cta_on[sl], 1);
  }
  for (bool first = true;; first = false) {
    // (re)initialise the barriers for this slice: every wait of the previous slice has returned.
    // Every lane of the producer arrives on a full barrier (lane 0 with the transaction bytes)
    // and every consumer lane on an empty barrier: each lane's own shared-memory accesses are
    // released by its own arrival.
    if (threadIdx.x == 0) {
      for (uint32_t b = 0; b < nbars + ring + 1; b++) {
        if (!first) asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(&s_full[b])) : "memory");
        mbar_init(&s_full[b], b < nbars ? 32u : (b < nbars + ring ? (uint32_t)(kUnits * 32) : 1u));
      }
      *s_next = 0u;
      fence_mbar_init();
    }
    __syncthreads();
    const int32_t sl = *s_slice;
    if (sl < 0) break;
    if (warp == PW) {
      // ---- producer
      if (lane == 0) {   // a7: the slice, one bulk copy of slots x 128 bytes
        const uint32_t bytes = (uint32_t)a.img.slots[sl] * (uint32_t)kSlotBytes;
        fence_proxy_async_smem();
        mbar_expect_tx(s_forest, bytes);
        bulk_g2s_big(smem, a.img.cnodes + (size_t)sl * a.img.slots_max * C * 2, bytes, s_forest);
      }
      // entry x (valid) consumed: store its 64 slice partials (two coalesced 256-byte stores;
      // non-fused launches)
      auto drain = [&](uint32_t x) {
        const uint32_t b = fmod_small(x, ring, a.ring_m);
        mbar_wait(&s_empty[b], fdiv_small(x, a.ring_m) & 1u);
        if (!FUSED) {
          const int64_t r0 = (int64_t)s_tile[b] * R;
          const int nr = (int)((a.n - r0) < R ? (a.n - r0) : R);
          const double* sp = s_part + b * kSlicedTileRows;
          double* dst = a.o.raw + (size_t)sl * a.n + r0;
          if (lane < nr) dst[lane] = sp[lane];
          if (lane + 32 < nr) dst[lane + 32] = sp[lane + 32];
        }
        __syncwarp();
      };
      // tiles are claimed one at a time from the slice's counter, the next claim issued before
      // this one is used (its latency overlaps the drain and the issue)
      int32_t next = 0;
      if (lane == 0) next = atomicAdd(&a.tile_next[sl], 1);
      uint32_t e = 0, n_valid = 0, terms = 0;
      while (terms < kTerm) {
        if (e >= ring && e - ring < n_valid) drain(e - ring);   // buffer e % ring is free again
        int32_t tile = -1;
        if (terms == 0) {
          tile = __shfl_sync(0xffffffffu, next, 0);
          if (tile >= (int32_t)ntiles) tile = -1;
          else if (lane == 0) next = atomicAdd(&a.tile_next[sl], 1);
        }
        const uint32_t b = fmod_small(e, ring, a.ring_m);
        uint64_t* bar = &s_full[fmod_small(e, nbars, a.bars_m)];
        if (lane == 0) {
          s_tile[b] = tile;
          if (tile >= 0) {
            const int64_t ahead = a.prefetch ? (int64_t)tile + a.prefetch : -1;
            if (ahead >= 0 && ahead < ntiles)   // optional L2 prefetch of a later tile
              asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(reinterpret_cast<const unsigned char*>(a.codes) + ahead * a.tstride),
                           "r"((uint32_t)a.tstride) : "memory");
            fence_proxy_async_smem();
            mbar_expect_tx(bar, (uint32_t)a.tstride);
            bulk_g2s(s_ring + (size_t)b * a.tstride,
                     reinterpret_cast<const unsigned char*>(a.codes) + (int64_t)tile * a.tstride, (uint32_t)a.tstride, bar);
          } else {
            asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
          }
        } else {
          asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
        }
        if (tile >= 0) n_valid++;
        else terms++;
        e++;
      }
      // the valid entries not yet drained (the last ring - kTerm of them at most)
      for (uint32_t x = e > ring ? e - ring : 0; x < n_valid; x++) drain(x);
    } else {
      // ---- consumers
      const uint32_t p0 = sbase + (uint32_t)col * 8u;
      const uint32_t pe = sbase + ((uint32_t)a.img.col_len[sl * C + col] * C + (uint32_t)col) * 8u;
      const int2* __restrict__ meta =
          LEAF ? reinterpret_cast<const int2*>(a.img.leaf_meta) + (size_t)sl * a.img.slots_max * C : nullptr;
      mbar_wait(s_forest, 0u);
      for (;;) {
        uint32_t q = 0;
        if (lane == 0) q = atomicAdd(s_next, 1u);   // 32-bit: a native ATOMS.ADD (64-bit was a CAS loop)
        q = __shfl_sync(0xffffffffu, q, 0);
        const uint32_t gt = q / kUnits;
        const int u = (int)(q % kUnits);
        const int b = (int)fmod_small(gt, ring, a.ring_m);
        mbar_wait(&s_full[fmod_small(gt, nbars, a.bars_m)], fdiv_small(gt, a.bars_m) & 1u);
        const int32_t tile = s_tile[b];
        if (tile < 0) break;   // terminator: the slice's tiles are exhausted
        const int64_t r0 = (int64_t)tile * R;
        const int nr = (int)((a.n - r0) < R ? (a.n - r0) : R);
        if (u < nr) {
          const int rA = u + 16 * half, rB = rA + 32;
          const bool okA = rA < nr, okB = rB < nr;
          const uint32_t pA = okA ? p0 : pe, pB = okB ? p0 : pe;
          const uint32_t tb = ring0 + (uint32_t)b * (uint32_t)a.tstride;
          // row base | swizzle (code_slot_swz in bytes): the attribute offset is XORed into it
          const int qA = okA ? rA : u, qB = okB ? rB : u;
          const uint32_t rowA = SWZ ? (tb + code_row_off(qA, a.rb)) | (code_slot_swz(qA, a.rb) << 1)
                                    : tb + code_row_off(qA, a.rb);
          const uint32_t rowB = SWZ ? (tb + code_row_off(qB, a.rb)) | (code_slot_swz(qB, a.rb) << 1)
                                    : tb + code_row_off(qB, a.rb);
          uint32_t nan_flag;
          asm volatile("ld.shared.u32 %0, [%1];" : "=r"(nan_flag) : "r"(tb + (uint32_t)a.tile_bytes));
          double accA, accB;
          uint64_t fpA = 0, fpB = 0;
          if (LEAF) {
            int32_t* oA = (a.o.out_leaf && okA) ? a.o.out_leaf + (r0 + rA) * (int64_t)a.o.T_leaf : nullptr;
            int32_t* oB = (a.o.out_leaf && okB) ? a.o.out_leaf + (r0 + rB) * (int64_t)a.o.T_leaf : nullptr;
            if (nan_flag)
              walk_coded2_leaf<true, SWZ>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB, sbase, meta, oA, oB, fpA, fpB);
            else
              walk_coded2_leaf<false, SWZ>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB, sbase, meta, oA, oB, fpA, fpB);
          } else if (PROF) {
            uint32_t span;
            if (nan_flag) walk_coded2_prof<true, SWZ>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB, span);
            else walk_coded2_prof<false, SWZ>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB, span);
            prof_unit(a.prof, span);
            lane_total += (double)span;
          } else if (nan_flag) {
            walk_coded2<true, SWZ>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB);
          } else {
            walk_coded2<false, SWZ>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB);
          }
          // a9: the k_sliced butterfly (lanes 0, 8, 16, 24 own rows u, u+32, u+16, u+48)
          const bool b3 = lane & 8;
          double v = (b3 ? accB : accA) + __shfl_xor_sync(0xffffffffu, b3 ? accA : accB, 8);
#pragma unroll
          for (int o = 4; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
          uint64_t fv = 0;
          if (LEAF) {
            fv = (b3 ? fpB : fpA) + __shfl_xor_sync(0xffffffffu, b3 ? fpA : fpB, 8);
#pragma unroll
            for (int o = 4; o > 0; o >>= 1) fv += __shfl_xor_sync(0xffffffffu, fv, o);
          }
          const int rr = b3 ? rB : rA;
          if ((lane & 7) == 0 && (b3 ? okB : okA)) {
            if (FUSED) write_scalar(a.o, r0 + rr, v);
            else s_part[b * kSlicedTileRows + rr] = v;
            if (LEAF && a.o.out_fp)
              atomicAdd(reinterpret_cast<unsigned long long*>(&a.o.out_fp[r0 + rr]), (unsigned long long)fv);
          }
        }
        // the unit is done with buffer b (its partials are in s_part): every lane release-arrives on
        // empty[b], so each lane's own reads of the tile and writes of s_part are ordered before the
        // producer's refill (one arrival per lane rather than one per warp after __syncwarp: the same
        // ordering, and the form compute-sanitizer racecheck tracks)
        asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&s_empty[b])) : "memory");
      }
    }
    (void)ph_forest;
    __syncthreads();   // every valid entry of this slice is consumed and drained
    if (threadIdx.x == 0) {
      atomicSub(&a.cta_on[sl], 1);
      // next slice: the most remaining work per CTA already on it (a slice nobody works on is
      // always taken while it has tiles)
      int32_t best = -1;
      float bw = 0.0f;
      for (int32_t s2 = 0; s2 < ns; s2++) {
        const int32_t rem = (int32_t)ntiles - *reinterpret_cast<volatile int32_t*>(&a.tile_next[s2]);
        const int32_t on = *reinterpret_cast<volatile int32_t*>(&a.cta_on[s2]);
        if (rem < 1 || (on > 0 && rem < 2)) continue;
        const float w = (float)rem * __ldg(&a.work[s2]) / (float)(1 + on);
        if (w > bw) { bw = w; best = s2; }
      }
      if (best >= 0) atomicAdd(&a.cta_on[best], 1);
      *s_slice = best;
    }
    __syncthreads();
  }
  if (PROF && warp != PW) prof_lanes(a.prof, lane_total);
}

static int grid_for(int64_t n, int block, int num_sms, int per_sm);

// ------------------------------------------------------------------ visit counting
// Algorithm 1 line 16 ("Count edge probabilities during inference"): every node a sample
// passes through (leaves included) gets +1 on the counter of its caller node id.  Edge probability
// of (parent -> child) = count[child] / count[parent].  Lanes meeting the same node in
// the same step are aggregated into one atomic.
__global__ void __launch_bounds__(256) k_count_visits(const DevDirect img, const float* X,
                                                      int64_t n, int32_t d, uint32_t* counts) {
  const uint2* __restrict__ nodes = reinterpret_cast<const uint2*>(img.nodes);
  const int fbits = img.fbits;
  const uint32_t fmask = (1u << fbits) - 1u;
  const uint32_t offmask = (1u << (kOffsetTop - fbits)) - 1u;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t n_pad = ((n + 31) / 32) * 32;  // whole warps iterate together
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_pad; i += stride) {
    const bool active = i < n;
    const float* __restrict__ x = X + (active ? i : 0) * d;
    for (int32_t t = 0; t < img.n_slots; t++) {
      uint32_t k = (uint32_t)__ldg(&img.root[t]);
      bool going = active;
      for (;;) {
        const unsigned m = __ballot_sync(0xffffffffu, going);
        if (!m) break;
        if (going) {
          const unsigned same = __match_any_sync(m, k);
          if ((__ffs(same) - 1) == (int)(threadIdx.x & 31))
            atomicAdd(&counts[__ldg(&img.slot_orig[k])], (uint32_t)__popc(same));
          const uint2 nd = __ldg(&nodes[k]);
          if ((int32_t)nd.y < 0) going = false;
          else k += step(nd.x, nd.y, __ldg(&x[nd.y & fmask]), fbits, offmask);
        }
      }
    }
  }
}

int launch_count_visits(const DevDirect& img, const float* X, int64_t n, int32_t d,
                        uint32_t* counts, int32_t num_sms, void* stream) {
  const int block = 256;
  k_count_visits<<<grid_for(n, block, num_sms, 8), block, 0, static_cast<cudaStream_t>(stream)>>>(
      img, X, n, d, counts);
  return (int)cudaGetLastError();
}

// ------------------------------------------------------------------ finalize
__global__ void __launch_bounds__(256) k_finalize(const FinalizeArgs a) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.n;
       i += (int64_t)gridDim.x * blockDim.x)
    finalize_row(a, i);
}

// ------------------------------------------------------------------ launchers
static int grid_for(int64_t n, int block, int num_sms, int per_sm) {
  int64_t g = (n + block - 1) / block;
  int64_t cap = (int64_t)num_sms * per_sm;
  if (g > cap) g = cap;
  return (int)(g < 1 ? 1 : g);
}

template <bool L, bool F, int B, bool LS>
static cudaError_t direct_tiled_one(const DirectKArgs& a, int32_t rs, int32_t num_sms,
                                    cudaStream_t st) {
  auto kern = k_direct_tiled<L, F, B, LS>;
  const int smem = B * rs * 4;
  static std::atomic<int> configured[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64 && configured[dev].load() < smem) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin);
    if (e != cudaSuccess) return e;
    configured[dev].store(kMaxSmemOptin);
  }
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, B, smem);
  if (per_sm < 1) per_sm = 1;
  const int64_t ntiles = (a.n + B - 1) / B;
  const int grid = (int)std::min<int64_t>(ntiles, (int64_t)num_sms * per_sm);
  kern<<<grid, B, smem, st>>>(a, rs);
  return cudaGetLastError();
}

template <bool F, int P, int kRows = 128, int GRP = 1>
static cudaError_t direct_tlp_one(const DirectKArgs& a, int32_t rs, int32_t num_sms,
                                  cudaStream_t st) {
  auto kern = k_direct_tlp<F, kRows, P, GRP>;
  const int smem = kRows * rs * 4;
  static std::atomic<int> configured[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64 && configured[dev].load() < smem) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin);
    if (e != cudaSuccess) return e;
    configured[dev].store(kMaxSmemOptin);
  }
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kRows * P, smem);
  if (per_sm < 1) per_sm = 1;
  // experiments: $TAHOE_DIRECT_PERSM caps the resident CTAs per SM and hands the rest of the
  // unified L1 / shared memory to L1 (node reads)
  static const int cap = std::getenv("TAHOE_DIRECT_PERSM") ? std::atoi(std::getenv("TAHOE_DIRECT_PERSM")) : 0;
  if (cap > 0 && cap < per_sm) {
    per_sm = cap;
    const int pct = (int)std::min<int64_t>(100, ((int64_t)per_sm * (smem + 1024) * 100 + 233471) / 233472);
    cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
  }
  const int64_t ntiles = (a.n + kRows - 1) / kRows;
  const int grid = (int)std::min<int64_t>(ntiles, (int64_t)num_sms * per_sm);
  kern<<<grid, kRows * P, smem, st>>>(a, rs);
  return cudaGetLastError();
}

template <bool F, int P, int kRows>
static cudaError_t direct_heads_one(const DirectKArgs& a, int32_t rs, int32_t kh, int32_t num_sms,
                                    cudaStream_t st) {
  auto kern = k_direct_heads<F, kRows, P>;
  const int smem = kRows * rs * 4 + a.img.n_slots * kh * 8;
  static std::atomic<int> configured[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64 && configured[dev].load() < smem) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin);
    if (e != cudaSuccess) return e;
    configured[dev].store(kMaxSmemOptin);
  }
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kRows * P, smem);
  if (per_sm < 1) per_sm = 1;
  const int64_t ntiles = (a.n + kRows - 1) / kRows;
  const int grid = (int)std::min<int64_t>(ntiles, (int64_t)num_sms * per_sm);
  kern<<<grid, kRows * P, smem, st>>>(a, rs, kh);
  return cudaGetLastError();
}

int launch_direct(const DevDirect& img, const float* X, int64_t n, int32_t d, const OutArgs& o,
                  bool fused, int32_t num_sms, void* stream) {
  DirectKArgs a{img, X, n, d, o};
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const bool leaf = o.out_leaf != nullptr || o.out_fp != nullptr;
  // 0 = rows read from global memory; 1 = staged rows, warp-lockstep over trees;
  // 2 = staged rows, free-running over trees; 3 / 4 = staged rows (128 per CTA), 2 / 4 threads
  // per row; 5 = 64 staged rows, 8 threads per row; 6 = 64 rows x 4; 7 = 32 rows x 16.
  // Default for large batches: staged rows — attribute reads from shared memory leave L1/L2 to
  // the nodes — with 8 threads per row over 64-row CTAs for scalar outputs (5) and one thread per
  // row, free-running, otherwise (2).  C5 500-tree shard, 300K rows: rows-global 10.05 ms ->
  // staged 9.75 -> 2 threads per row 5.96 -> 8 threads per row over 64 rows 4.05 ms: more node
  // loads in flight, while the smaller row tiles leave ~150 KB of the unified L1 to the nodes
  // (4 threads per row over 128-row CTAs at 4 CTAs/SM leave ~50 KB: 8.04 ms; 16 per row 4.65 ms).
  // Rows from global memory (0) for small batches (lower launch cost) and for rows too wide to
  // stage.
  const bool scalar = o.n_classes == 1 && o.agg != TAHOE_AGG_VOTE;
  const char* env = std::getenv("TAHOE_DIRECT_VARIANT");
  int variant = env ? std::atoi(env) : (n >= 32768 ? (scalar && !leaf ? 5 : 2) : 0);
  if (d > 256) variant = 0;  // 128 staged rows must fit shared memory
  // 8 / 9: variant 5 / 128 rows x 8 with the first kh slots of every tree in shared memory
  // ($TAHOE_DIRECT_HEADS slots per tree, capped by a 48 KB budget; < 2 slots => variant 5)
  if ((variant == 8 || variant == 9) && scalar && !leaf) {
    const int32_t rs = d | 1;
    const char* khe = std::getenv("TAHOE_DIRECT_HEADS");
    int32_t kh = khe ? std::atoi(khe) : 8;
    while (kh > 1 && (int64_t)img.n_slots * kh * 8 > 49152) kh >>= 1;
    if (kh >= 2) {
      cudaError_t e;
      if (variant == 8) e = fused ? direct_heads_one<true, 8, 64>(a, rs, kh, num_sms, st) : direct_heads_one<false, 8, 64>(a, rs, kh, num_sms, st);
      else e = fused ? direct_heads_one<true, 8, 128>(a, rs, kh, num_sms, st) : direct_heads_one<false, 8, 128>(a, rs, kh, num_sms, st);
      return (int)e;
    }
    variant = 5;
  }
  if ((variant == 10 || variant == 11) && scalar && !leaf) {   // variant 5 over node groups
    const int32_t rs = d | 1;
    cudaError_t e;
    if (variant == 10) e = fused ? direct_tlp_one<true, 8, 64, 4>(a, rs, num_sms, st) : direct_tlp_one<false, 8, 64, 4>(a, rs, num_sms, st);
    else e = fused ? direct_tlp_one<true, 8, 64, 2>(a, rs, num_sms, st) : direct_tlp_one<false, 8, 64, 2>(a, rs, num_sms, st);
    return (int)e;
  }
  if (variant >= 3 && variant <= 7 && scalar && !leaf) {
    const int32_t rs = d | 1;
    cudaError_t e;
    if (variant == 3) e = fused ? direct_tlp_one<true, 2>(a, rs, num_sms, st) : direct_tlp_one<false, 2>(a, rs, num_sms, st);
    else if (variant == 4) e = fused ? direct_tlp_one<true, 4>(a, rs, num_sms, st) : direct_tlp_one<false, 4>(a, rs, num_sms, st);
    else if (variant == 5) e = fused ? direct_tlp_one<true, 8, 64>(a, rs, num_sms, st) : direct_tlp_one<false, 8, 64>(a, rs, num_sms, st);
    else if (variant == 6) e = fused ? direct_tlp_one<true, 4, 64>(a, rs, num_sms, st) : direct_tlp_one<false, 4, 64>(a, rs, num_sms, st);
    else e = fused ? direct_tlp_one<true, 16, 32>(a, rs, num_sms, st) : direct_tlp_one<false, 16, 32>(a, rs, num_sms, st);
    return (int)e;
  }
  if (variant == 1 || variant == 2) {
    const int32_t rs = d | 1;  // odd stride: lanes on different rows spread over the banks
    cudaError_t e;
    if (variant == 1) {
      if (leaf) e = fused ? direct_tiled_one<true, true, 128, true>(a, rs, num_sms, st) : direct_tiled_one<true, false, 128, true>(a, rs, num_sms, st);
      else e = fused ? direct_tiled_one<false, true, 128, true>(a, rs, num_sms, st) : direct_tiled_one<false, false, 128, true>(a, rs, num_sms, st);
    } else {
      if (leaf) e = fused ? direct_tiled_one<true, true, 128, false>(a, rs, num_sms, st) : direct_tiled_one<true, false, 128, false>(a, rs, num_sms, st);
      else e = fused ? direct_tiled_one<false, true, 128, false>(a, rs, num_sms, st) : direct_tiled_one<false, false, 128, false>(a, rs, num_sms, st);
    }
    return (int)e;
  }
  const int block = 256;
  const int grid = grid_for(n, block, num_sms, 8);
  if (leaf) {
    if (fused) k_direct<true, true><<<grid, block, 0, st>>>(a);
    else k_direct<true, false><<<grid, block, 0, st>>>(a);
  } else {
    if (fused) k_direct<false, true><<<grid, block, 0, st>>>(a);
    else k_direct<false, false><<<grid, block, 0, st>>>(a);
  }
  return (int)cudaGetLastError();
}

template <bool L, bool F, int R>
static cudaError_t sliced_one(const SlicedKArgs& a, const SlicedPlan& p, cudaStream_t st) {
  auto kern = k_sliced<L, F, R>;
  // raise the dynamic shared-memory limit once per process and device (not per launch)
  static std::atomic<int> configured[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64 && configured[dev].load() < p.smem_bytes) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin);
    if (e != cudaSuccess) return e;
    configured[dev].store(kMaxSmemOptin);
  }
  kern<<<p.grid, p.block, p.smem_bytes, st>>>(a);
  return cudaGetLastError();
}

template <bool L, bool F>
static cudaError_t sliced_rows(const SlicedKArgs& a, const SlicedPlan& p, cudaStream_t st) {
  if (p.rows == kRowsPadded) return sliced_one<L, F, kRowsPadded>(a, p, st);
  if (p.rows == kRowsDense) return sliced_one<L, F, kRowsDense>(a, p, st);
  return sliced_one<L, F, kRowsGlobal>(a, p, st);
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda needed)
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFn encode_tiled_fn() {
  static EncodeTiledFn fn = [] {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return (EncodeTiledFn) nullptr;
    return reinterpret_cast<EncodeTiledFn>(ptr);
  }();
  return fn;
}

bool padded_rows_possible(const float* X, int32_t d) {
  return ((reinterpret_cast<uintptr_t>(X) & 15) == 0) && (d % 4 == 0) && encode_tiled_fn() != nullptr;
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
  a.buf_floats = plan.buf_floats;
  a.row_stride = plan.row_stride;
  a.x_aligned = ((reinterpret_cast<uintptr_t>(X) & 15) == 0) &&
                (((int64_t)plan.tile_rows * d * 4) % 16 == 0);
  a.o = o;
  if (plan.rows == kRowsPadded) {
    EncodeTiledFn enc = encode_tiled_fn();
    if (!enc) return (int)cudaErrorNotSupported;
    const cuuint64_t gdim[2] = {(cuuint64_t)d, (cuuint64_t)n};
    const cuuint64_t gstride[1] = {(cuuint64_t)d * 4};
    const cuuint32_t box[2] = {(cuuint32_t)plan.row_stride, (cuuint32_t)plan.tile_rows};
    const cuuint32_t estride[2] = {1, 1};
    CUresult r = enc(&a.tmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(X), gdim, gstride,
                     box, estride, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return (int)cudaErrorInvalidValue;
  }
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const bool leaf = o.out_leaf != nullptr || o.out_fp != nullptr;
  cudaError_t e;
  if (leaf) e = fused ? sliced_rows<true, true>(a, plan, st) : sliced_rows<true, false>(a, plan, st);
  else e = fused ? sliced_rows<false, true>(a, plan, st) : sliced_rows<false, false>(a, plan, st);
  return (int)e;
}

int launch_sliced_codes(const DevSliced& img, const SlicedPlan& plan, const float* X, int64_t n,
                        int32_t d, uint16_t* codes, const OutArgs& o, bool fused, int32_t num_sms,
                        void* stream, void* ev_b, void* ev_e, double* prof) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int64_t ntiles = (n + kSlicedTileRows - 1) / kSlicedTileRows;
  const int32_t tstride = code_tile_stride(img.fbits);
  const int32_t tbytes = code_tile_bytes(img.fbits);
  // zero every tile's NaN flag (the trailer word after its rows) and the per-slice tile / CTA
  // counters after the tiles
  cudaError_t e = cudaMemset2DAsync(reinterpret_cast<char*>(codes) + tbytes, (size_t)tstride, 0, 4,
                                    (size_t)ntiles, st);
  if (e != cudaSuccess) return (int)e;
  int32_t* counters = reinterpret_cast<int32_t*>(reinterpret_cast<char*>(codes) + ntiles * tstride);
  e = cudaMemsetAsync(counters, 0, (size_t)img.n_slices * 8, st);
  if (e != cudaSuccess) return (int)e;
  EncodeRowsArgs ea;
  ea.X = X;
  ea.n = n;
  ea.d = d;
  ea.nf = img.n_features;
  ea.fbits = img.fbits;
  ea.rb = code_row_bytes(img.fbits);
  ea.n_thr = img.n_thr;
  ea.tab = img.thr_tab;
  ea.off = img.thr_off;
  ea.codes = codes;
  ea.tstride = tstride;
  ea.ntiles = ntiles;
  ea.slot_attr = img.slot_attr;
  const int64_t tab_bytes = (int64_t)img.n_thr * 4 + (int64_t)(img.n_features + 1) * 4;
  const int64_t elems = ntiles * kSlicedTileRows << img.fbits;
  const int blk = 1024;
  // $TAHOE_CODE_BANKS=0: bisect through L2 instead (tests cover both pre-pass kernels)
  const bool banks_off = std::getenv("TAHOE_CODE_BANKS") && std::atoi(std::getenv("TAHOE_CODE_BANKS")) == 0;
  if (img.cb_img && !banks_off) {
    EncodeBanksArgs ba;
    ba.X = X;
    ba.n = n;
    ba.d = d;
    ba.rb = code_row_bytes(img.fbits);
    ba.passes = img.cb_passes;
    ba.img_bytes = img.cb_rows * 128;
    ba.img = img.cb_img;
    ba.desc = reinterpret_cast<const int4*>(img.cb_desc);
    ba.codes = codes;
    ba.tstride = tstride;
    ba.nrows = ntiles * kSlicedTileRows;
    static std::atomic<int> configured[64];
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && !configured[dev].load()) {
      // static + dynamic shared memory must stay within the opt-in limit (the kernel's mbarrier
      // is static)
      e = cudaFuncSetAttribute(k_encode_rows_banks<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               kMaxSmemOptin - 1024);
      if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_encode_rows_banks<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 kMaxSmemOptin - 1024);
      if (e != cudaSuccess) return (int)e;
      configured[dev].store(1);
    }
    const int64_t warps_needed = (ba.nrows + 7) / 8;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(num_sms, (warps_needed + 31) / 32));
    if (ba.rb == 64) k_encode_rows_banks<true><<<grid, blk, ba.img_bytes, st>>>(ba);
    else k_encode_rows_banks<false><<<grid, blk, ba.img_bytes, st>>>(ba);
  } else if (tab_bytes <= 200 * 1024) {
    static std::atomic<int> configured[64];
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && !configured[dev].load()) {
      e = cudaFuncSetAttribute(k_encode_rows<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin);
      if (e != cudaSuccess) return (int)e;
      configured[dev].store(1);
    }
    const int smem = (int)((tab_bytes + 15) & ~15LL);
    const int per_sm = smem <= 100 * 1024 ? 2 : 1;
    k_encode_rows<true><<<grid_for((elems + 0) , blk, num_sms, per_sm), blk, smem, st>>>(ea);
  } else {
    k_encode_rows<false><<<grid_for(elems, blk, num_sms, 2), blk, 0, st>>>(ea);
  }
  if ((e = cudaGetLastError()) != cudaSuccess) return (int)e;

  CodedKArgs a{};
  a.img = img;
  a.codes = codes;
  a.n = n;
  a.forest_smem = plan.forest_smem;
  a.tile_bytes = tbytes;
  a.tstride = tstride;
  a.rb = code_row_bytes(img.fbits);
  a.cps = plan.cps;
  a.cta_start = plan.cta_start;
  a.prefetch = std::getenv("TAHOE_CODES_PREFETCH") ? std::atoi(std::getenv("TAHOE_CODES_PREFETCH")) : 0;
  a.o = o;
  // ring depth: every tile the shared memory next to the slice holds (3 .. kCodedRingMax); a deeper
  // ring lets the warps that claimed the next tile's units work instead of sleeping on its copy
  a.ring = coded_ring_depth(plan.forest_smem, tstride);
  if (const char* e = std::getenv("TAHOE_CODES_RING"))   // experiments (capped by what fits)
    a.ring = std::max(kSlicedRing, std::min(a.ring, std::atoi(e)));
  a.ring_m = (uint32_t)((0x100000000ULL + a.ring - 1) / a.ring);
  a.bars_m = (uint32_t)((0x100000000ULL + 2 * a.ring - 1) / (2 * a.ring));
  const int smem = plan.forest_smem + coded_ring_smem(a.ring, tstride);
  // rows of >= 128 bytes are stored swizzled (code_slot_swz); the others keep the plain walk;
  // leaf ids / fingerprints take the LEAF instantiation of the same walk
  const bool leaf = o.out_leaf != nullptr || o.out_fp != nullptr;
  a.prof = prof;
  a.tile_next = counters;
  a.cta_on = counters + img.n_slices;
  a.work = img.slice_w;
  using KFn = void (*)(CodedKArgs);
  // [mode][swz][fused]
  static const KFn table[3][2][2] = {
      {{k_sliced_codes<false, false, 0>, k_sliced_codes<true, false, 0>},
       {k_sliced_codes<false, true, 0>, k_sliced_codes<true, true, 0>}},
      {{k_sliced_codes<false, false, 1>, k_sliced_codes<true, false, 1>},
       {k_sliced_codes<false, true, 1>, k_sliced_codes<true, true, 1>}},
      {{k_sliced_codes<false, false, 2>, k_sliced_codes<true, false, 2>},
       {k_sliced_codes<false, true, 2>, k_sliced_codes<true, true, 2>}}};
  const int mode = prof ? 2 : (leaf ? 1 : 0);
  auto kern = table[mode][a.rb >= 128 ? 1 : 0][fused ? 1 : 0];
  {
    static std::atomic<int> configured[64];
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && !configured[dev].load()) {
      for (const auto& m : table)
        for (const auto& w : m)
          for (KFn k : w) {
            e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin);
            if (e != cudaSuccess) return (int)e;
          }
      configured[dev].store(1);
    }
  }
  if (ev_b) cudaEventRecord(static_cast<cudaEvent_t>(ev_b), st);
  kern<<<plan.grid, 1024, smem, st>>>(a);
  e = cudaGetLastError();
  if (ev_e) cudaEventRecord(static_cast<cudaEvent_t>(ev_e), st);
  return (int)e;
}

// ------------------------------------------------------------------ wide rank codes (reading R8)
// Rows of more than 127 attributes (C4: 2000).  A row becomes 2^V u8 codes over virtual
// attributes (kernels.hpp "wide codes"): 2 KB for C4 instead of 8 KB of fp32, so 16-row tiles fit
// in shared memory next to a slice and the walk's attribute reads stop going to L2.

// k_encode_rows8: CTA = (band b, row chunk).  The CTA bulk-copies band b's bank-private tables
// (encode.cpp build_code8_banks) into shared memory; a warp then codes kR rows at a time, group by
// group of the band: lane a bisects virtual attribute 32g + a with the group's uniform probe count
// (one conflict-free LDS per probe for the warp) and writes its code byte (32 consecutive bytes
// per row and group).  A tile's NaN flag is set by whichever band meets a NaN.
struct Encode8Args {
  const float* X;
  int64_t n;
  int32_t d, vfbits, bands, chunks;
  const float* img;
  const int4* grp;
  const int4* band;
  const int32_t* v_src;
  uint8_t* codes;
  uint32_t* flags;   // 4 words per tile, word 0 = NaN flag
};

// pos[q] := #{tab <= x[q]} over a lane's 2^K - 1 table elements at base + i * 128 bytes (NaN pads
// compare false): probe at pos + step - 1 for step = 2^(K-1) .. 1.  The running address a[q] =
// base + pos[q] * 128 makes every probe one LDS with an immediate offset, one FSETP and one
// predicated add.
// one bisection level of bisect8 (probe offset and step are immediates: LDS [ad + imm]; FSETP;
// predicated IADD: three instructions per probe), then the next level
#ifndef TAHOE_CODE8_UROWS
#define TAHOE_CODE8_UROWS 2
#endif
constexpr int kCode8URows = TAHOE_CODE8_UROWS;
// Wide-code rows walked by the second half-warp (tile row bit kCode8SwzBit set: rows u + 4 with
// two-row units, u + 2 and u + 6 with four-row units) keep code byte v at v ^ s, s = 64 (16 banks
// over; rows of 2^V < 128 bytes: half the row, which keeps it inside the row):
// the two half-warps walk the same lane columns, so at the top of every tree and at every leaf
// (the pad byte) they read the same byte offset of two different rows — one bank, two addresses.
// The walk XORs the attribute offset into the row base (`(y & amask) ^ row`, one LOP3 as before).
constexpr uint32_t kCode8SwzBit = kCode8URows == 2 ? 4u : 2u;
__device__ __forceinline__ uint32_t code8_swz(uint32_t r, uint32_t V) {
  return (r & kCode8SwzBit) ? min(64u, (1u << V) >> 1) : 0u;
}

template <int ST, int kR>
__device__ __forceinline__ void probe8(uint32_t* ad, const float* x) {
#pragma unroll
  for (int q = 0; q < kR; q++)
    asm("{\n\t.reg .f32 t;\n\t.reg .pred p;\n\t"
        "ld.shared.f32 t, [%0+%2];\n\t"
        "setp.le.f32 p, t, %1;\n\t"
        "@p add.u32 %0, %0, %3;\n\t}"
        : "+r"(ad[q]) : "f"(x[q]), "n"(((1u << ST) - 1u) << 7), "n"((1u << ST) << 7));
  if constexpr (ST > 0) probe8<ST - 1, kR>(ad, x);
}

template <int K, int kR>
__device__ __forceinline__ void bisect8(uint32_t base, const float* x, uint32_t* pos) {
  uint32_t ad[kR];
#pragma unroll
  for (int q = 0; q < kR; q++) ad[q] = base;
  probe8<K - 1, kR>(ad, x);
#pragma unroll
  for (int q = 0; q < kR; q++) pos[q] = (ad[q] - base) >> 7;
}

// 1024 threads x 4 rows per warp step (64 registers, no spills): C4 pre-pass 2.12 ms per 500K
// rows; 8 rows per step spill at 1024 threads (2.60 ms) and at 512 threads lack the warps to
// cover the X loads (3.02 ms)
constexpr int kEncode8Threads = 1024;
constexpr int kEncode8Rows = 4;
template <int THREADS, int kR>
__global__ void __launch_bounds__(THREADS, 1) k_encode_rows8(const Encode8Args a) {
  extern __shared__ __align__(1024) float s_img[];
  __shared__ uint64_t s_bar;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, W = blockDim.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(&s_bar, 1);
    fence_mbar_init();
  }
  __syncthreads();
  // persistent CTAs over (band, chunk) items, band-major: the launcher makes the item count a
  // multiple of the grid, so every CTA codes the same number of equal row chunks
  const int items = a.bands * a.chunks;
  uint32_t phase = 0;
  for (int item = blockIdx.x; item < items; item += gridDim.x) {
    const int b = item / a.chunks;
    const int64_t chunk = item % a.chunks;
    const int4 bd = __ldg(&a.band[b]);
    __syncthreads();   // every warp is done with the previous item's table
    if (bd.y > 0) {
      if (threadIdx.x == 0) {
        fence_proxy_async_smem();
        mbar_expect_tx(&s_bar, (uint32_t)bd.y);
        bulk_g2s_big(s_img, reinterpret_cast<const unsigned char*>(a.img) + bd.x, (uint32_t)bd.y, &s_bar);
      }
      mbar_wait(&s_bar, phase);
      phase ^= 1u;
    }
    static_assert(kCode8TileRows % kR == 0, "a row group stays inside one tile");
    // this chunk's rows, in whole groups of kR
    const int64_t groups = (a.n + kR - 1) / kR;
    const int64_t per = (groups + a.chunks - 1) / a.chunks;
    const int64_t r_lo = chunk * per * kR;
    const int64_t r_hi = min(a.n, (chunk + 1) * per * kR);
    const uint32_t V = (uint32_t)a.vfbits;
    const int64_t tile_bytes = (int64_t)kCode8TileRows << V;
    const uint32_t sbase = smem_u32(s_img) + (uint32_t)lane * 4u;
    static_assert(kR == 4, "the quad byte transpose below stores 4 rows");
    const int quad = lane & 3;   // after the transpose: this lane stores row `quad` ...
    const uint32_t qoff = (uint32_t)(lane >> 2) * 4u;   // ... bytes qoff .. qoff + 3 of the group
    for (int64_t r0 = r_lo + (int64_t)warp * kR; r0 < r_hi; r0 += (int64_t)W * kR) {
      const int nq = (int)min((int64_t)kR, r_hi - r0);   // rows of this group (the tail is ragged)
      bool nan_any = false;
      uint8_t* row0 = a.codes + (r0 / kCode8TileRows) * tile_bytes + ((r0 % kCode8TileRows) << V);
      // the group's rows as 32-bit offsets from one 64-bit base (rows past the tail re-read the
      // last row; their codes are not stored)
      const float* xb = a.X + r0 * a.d;
      uint32_t roff[kR];
#pragma unroll
      for (int q = 0; q < kR; q++) roff[q] = (uint32_t)(q < nq ? q : nq - 1) * (uint32_t)a.d;
      // the next group's attribute values are loaded before this group is searched
      auto load_x = [&](int g, float* x, int& src) {
        src = g < bd.w ? __ldg(&a.v_src[g * 32 + lane]) : -1;
        const uint32_t so = src >= 0 ? (uint32_t)src : 0u;
#pragma unroll
        for (int q = 0; q < kR; q++) x[q] = __ldg(xb + (roff[q] + so));
      };
      float xn[kR];
      int srcn;
      load_x(bd.z, xn, srcn);
      for (int g = bd.z; g < bd.w; g++) {
        const int src = srcn;
        float x[kR];
#pragma unroll
        for (int q = 0; q < kR; q++) x[q] = xn[q];
        load_x(g + 1, xn, srcn);
        uint32_t pos[kR];
        bisect8<7, kR>(sbase + (uint32_t)__ldg(&a.grp[g]).x * 4u, x, pos);
        // this lane's codes of rows 0..3 as the bytes of one word, then a 4 x 4 byte transpose
        // inside each quad of lanes (two exchanges): lane 4j + k ends with row k's codes of the
        // group's attributes 4j .. 4j + 3, one 32-bit store (four byte stores before)
        uint32_t w = 0;
#pragma unroll
        for (int q = 0; q < kR; q++) {
          const bool isnan_q = src >= 0 && x[q] != x[q];
          nan_any |= isnan_q && q < nq;
          const int8_t c = src < 0 ? kCode8Pad : (isnan_q ? kCode8Nan : (int8_t)pos[q]);
          w |= (uint32_t)(uint8_t)c << (8 * q);
        }
        uint32_t p = __shfl_xor_sync(0xffffffffu, w, 1);
        w = (lane & 1) ? __byte_perm(w, p, 0x3715) : __byte_perm(w, p, 0x6240);
        p = __shfl_xor_sync(0xffffffffu, w, 2);
        w = (lane & 2) ? __byte_perm(w, p, 0x3276) : __byte_perm(w, p, 0x5410);
        if (quad < nq)
          *reinterpret_cast<uint32_t*>(row0 + ((uint32_t)quad << V) + (((uint32_t)g * 32u + qoff) ^ code8_swz((uint32_t)(r0 + quad), V))) = w;
      }
      if (__any_sync(0xffffffffu, nan_any) && lane == 0) a.flags[(r0 / kCode8TileRows) * 4] = 1u;
    }
  }
}

// k_encode_rows8_tma: k_encode_rows8 with the rows staged by TMA.  ncu of k_encode_rows8 put 35 %
// of its stall samples on the X loads (the consumer of each group's LDGs); here thread 0 loads
// 128-row x kCode8BoxW-float boxes of X (the band's source attributes, one 2-D tensor copy per
// stage) into a two-stage ring, and warp w codes the stage's rows 4w .. 4w + 3 over the band's
// groups from shared memory.  Codes, stores and NaN flags as k_encode_rows8.
struct alignas(64) Encode8TmaArgs {
  CUtensorMap tmap;   // X as a 2-D tensor [n][d] fp32, box [kCode8BoxW][kCode8StageRows]
  Encode8Args e;
};

template <int kR>
__global__ void __launch_bounds__(1024, 1) k_encode_rows8_tma(const __grid_constant__ Encode8TmaArgs ta) {
  const Encode8Args& a = ta.e;
  const uint64_t tmap = reinterpret_cast<uint64_t>(&ta.tmap);   // in the parameter space
  extern __shared__ __align__(1024) float s_img[];
  float* s_x = s_img + kCode8TmaTables / 4;   // [2][kCode8StageRows][kCode8BoxW]
  // barriers after the stages: no static shared memory, so the dynamic block starts at the
  // window's base and the stages keep the 128-byte alignment tensor copies need (a static barrier
  // in front shifted them: illegal instruction)
  uint64_t* s_bars = reinterpret_cast<uint64_t*>(s_x + 2 * (kCode8StageBytes / 4));
  uint64_t& s_tab = s_bars[0];
  uint64_t* s_full = s_bars + 1;
  uint64_t* s_empty = s_bars + 3;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, W = blockDim.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(&s_tab, 1);
    for (int b = 0; b < 2; b++) {
      mbar_init(&s_full[b], 1);
      mbar_init(&s_empty[b], (uint32_t)W);
    }
    fence_mbar_init();
  }
  __syncthreads();
  static_assert(kR == 4 && kCode8StageRows % kCode8TileRows == 0 && kCode8StageRows == 4 * 32,
                "one 4-row group per warp, whole tiles per stage");
  const uint32_t V = (uint32_t)a.vfbits;
  const int64_t tile_bytes = (int64_t)kCode8TileRows << V;
  const uint32_t sbase = smem_u32(s_img) + (uint32_t)lane * 4u;
  const int quad = lane & 3;
  const uint32_t qoff = (uint32_t)(lane >> 2) * 4u;
  const int items = a.bands * a.chunks;
  const int64_t groups = (a.n + kR - 1) / kR;
  const int64_t per = (groups + a.chunks - 1) / a.chunks;
  uint32_t ph_tab = 0, sc = 0;   // table loads so far; stages issued so far (CTA-uniform)
  for (int item = blockIdx.x; item < items; item += gridDim.x) {
    const int b = item / a.chunks;
    const int64_t chunk = item % a.chunks;
    const int4 bd = __ldg(&a.band[b]);
    const int64_t r_lo = chunk * per * kR;
    const int64_t r_hi = min(a.n, (chunk + 1) * per * kR);
    const int nst = r_hi > r_lo ? (int)((r_hi - r_lo + kCode8StageRows - 1) / kCode8StageRows) : 0;
    // the band's first source attribute, rounded down to a 16-byte boundary (the box start)
    const int32_t s_lo = __ldg(&a.v_src[bd.z * 32]) & ~3;
    __syncthreads();   // every warp is done with the previous item's table and stages
    auto issue = [&](uint32_t k, int st) {   // stage st of this item as ring stage k
      uint64_t* bar = &s_full[k & 1];
      fence_proxy_async_smem();
      mbar_expect_tx(bar, (uint32_t)kCode8StageBytes);
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
          " [%0], [%1, {%2, %3}], [%4];" ::"r"(smem_u32(s_x + (size_t)(k & 1) * (kCode8StageBytes / 4))),
          "l"(tmap), "r"(s_lo), "r"((int32_t)(r_lo + (int64_t)st * kCode8StageRows)),
          "r"(smem_u32(bar))
          : "memory");
    };
    if (threadIdx.x == 0) {
      if (bd.y > 0) {
        fence_proxy_async_smem();
        mbar_expect_tx(&s_tab, (uint32_t)bd.y);
        bulk_g2s_big(s_img, reinterpret_cast<const unsigned char*>(a.img) + bd.x, (uint32_t)bd.y, &s_tab);
      }
      for (int st = 0; st < nst && st < 2; st++) issue(sc + (uint32_t)st, st);
    }
    if (bd.y > 0) {
      mbar_wait(&s_tab, ph_tab);
      ph_tab ^= 1u;
    }
    // this lane's source attribute and table base of each of the band's (<= 4) groups, once per
    // item instead of two global loads per group and stage
    int g_src[kCode8BandGroups];
    uint32_t g_tab[kCode8BandGroups];
#pragma unroll
    for (int j = 0; j < kCode8BandGroups; j++) {
      const int g = bd.z + j;
      g_src[j] = g < bd.w ? __ldg(&a.v_src[g * 32 + lane]) : -1;
      g_tab[j] = g < bd.w ? sbase + (uint32_t)__ldg(&a.grp[g]).x * 4u : sbase;
    }
    for (int st = 0; st < nst; st++, sc++) {
      const uint32_t k = sc & 1u;
      mbar_wait(&s_full[k], (sc >> 1) & 1u);
      const float* sx = s_x + (size_t)k * (kCode8StageBytes / 4) + warp * kR * kCode8BoxW;
      const int64_t rs0 = r_lo + (int64_t)st * kCode8StageRows;
      const int64_t r0 = rs0 + warp * kR;
      const int nq = r0 < r_hi ? (int)min((int64_t)kR, r_hi - r0) : 0;
      bool nan_any = false;
      uint8_t* row0 = a.codes + (r0 / kCode8TileRows) * tile_bytes + ((r0 % kCode8TileRows) << V);
#pragma unroll
      for (int j = 0; j < kCode8BandGroups; j++) {
        const int g = bd.z + j;
        if (nq <= 0 || g >= bd.w) break;
        const int src = g_src[j];
        const int col = src >= 0 ? src - s_lo : 0;
        float x[kR];
#pragma unroll
        for (int q = 0; q < kR; q++) x[q] = sx[q * kCode8BoxW + col];
        uint32_t pos[kR];
        bisect8<7, kR>(g_tab[j], x, pos);
        uint32_t w = 0;
#pragma unroll
        for (int q = 0; q < kR; q++) {
          const bool isnan_q = src >= 0 && x[q] != x[q];
          nan_any |= isnan_q && q < nq;
          const int8_t c = src < 0 ? kCode8Pad : (isnan_q ? kCode8Nan : (int8_t)pos[q]);
          w |= (uint32_t)(uint8_t)c << (8 * q);
        }
        uint32_t p = __shfl_xor_sync(0xffffffffu, w, 1);
        w = (lane & 1) ? __byte_perm(w, p, 0x3715) : __byte_perm(w, p, 0x6240);
        p = __shfl_xor_sync(0xffffffffu, w, 2);
        w = (lane & 2) ? __byte_perm(w, p, 0x3276) : __byte_perm(w, p, 0x5410);
        if (quad < nq)
          *reinterpret_cast<uint32_t*>(row0 + ((uint32_t)quad << V) + (((uint32_t)g * 32u + qoff) ^ code8_swz((uint32_t)(r0 + quad), V))) = w;
      }
      if (__any_sync(0xffffffffu, nan_any) && lane == 0) a.flags[(r0 / kCode8TileRows) * 4] = 1u;
      // the warp is done with stage k: one arrival per warp (after its lanes' reads)
      __syncwarp();
      if (lane == 0) asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&s_empty[k])) : "memory");
      // thread 0 refills the stage once every warp has left it
      if (threadIdx.x == 0 && st + 2 < nst) {
        mbar_wait(&s_empty[k], (sc >> 1) & 1u);
        issue(sc + 2, st + 2);
      }
    }
  }
}

struct Coded8KArgs {
  DevSliced img;
  const uint8_t* codes;
  const uint32_t* flags;
  int32_t* tile_next;    // [ns] next unclaimed tile of each slice (zeroed per launch)
  int32_t* cta_on;       // [ns] CTAs currently working on each slice (zeroed per launch)
  const float* work;     // [ns] simulated lane-steps per row of each slice (slice choice weights)
  int64_t n;
  int32_t forest_smem;   // bytes reserved for the slice (multiple of 1024)
  const int32_t* cta_start;  // initial CTA -> slice map (prefix), or nullptr: blockIdx % ns
  int64_t row0;          // first row of this launch's chunk (outputs are indexed row0 + r)
  int64_t n_all;         // rows of the whole batch (row stride of the raw partials)
  int32_t switch_slices; // 1: a CTA whose slice is exhausted moves to another (0: experiments)
  int32_t prefetch;      // tiles ahead of a claim to prefetch into L2 (0 = none)
  int32_t split;         // 1: four chains per lane (each column walked as two halves)
  int32_t claim;         // tiles one ring buffer claims per global atomic (>= 1)
  OutArgs o;
};

// One step on a wide-coded slice: node {x = t or leaf value, y}, code byte at (y & amask) | row,
// left iff code < t (NaN-aware: or NaN and default-left), right / next root at +(y >> (V+1)).
template <bool NAN_AWARE>
__device__ __forceinline__ float coded8_step(uint32_t& p, uint32_t rowaddr, uint32_t amask,
                                             uint32_t dlbit, uint32_t shmul,
                                             uint32_t* yout = nullptr) {
  uint32_t x, y;
  int32_t c;
  asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(p));
  if (yout) *yout = y;
  asm("ld.shared.s8 %0, [%1];" : "=r"(c) : "r"((y & amask) ^ rowaddr));
  bool go_left = (uint32_t)c < x;
  if (NAN_AWARE) go_left = go_left || ((c == (int32_t)kCode8Nan) && (y & dlbit));
  p += go_left ? (uint32_t)kSlotBytes : __umulhi(y, shmul);
  return __uint_as_float(x);
}

template <bool NAN_AWARE>
__device__ __forceinline__ void walk_coded8(uint32_t pA, uint32_t pB, uint32_t pe, uint32_t rowA,
                                            uint32_t rowB, uint32_t amask, uint32_t dlbit,
                                            uint32_t shmul, double& accA, double& accB) {
  accA = 0.0;
  accB = 0.0;
  while ((pA != pe) | (pB != pe)) {
    const float a1 = coded8_step<NAN_AWARE>(pA, rowA, amask, dlbit, shmul);
    const float b1 = coded8_step<NAN_AWARE>(pB, rowB, amask, dlbit, shmul);
    const float a2 = coded8_step<NAN_AWARE>(pA, rowA, amask, dlbit, shmul);
    const float b2 = coded8_step<NAN_AWARE>(pB, rowB, amask, dlbit, shmul);
    add_pair_ftz(accA, a1, a2);
    add_pair_ftz(accB, b1, b2);
  }
}

// Four chains per lane: each row's column is walked as two halves (split at col_mid, the tree
// root that halves the column's expected work), so a lane keeps four independent node chains in
// flight over the same two staged rows.  A first-half chain freezes at its split slot (it keeps
// re-reading that internal node, whose word adds +0).
template <bool NAN_AWARE>
__device__ __forceinline__ void walk_coded8_split(uint32_t pA1, uint32_t mA, uint32_t pA2, uint32_t pB1,
                                                  uint32_t mB, uint32_t pB2, uint32_t pe,
                                                  uint32_t rowA, uint32_t rowB, uint32_t amask,
                                                  uint32_t dlbit, uint32_t shmul, double& accA,
                                                  double& accB) {
  double a1 = 0.0, a2 = 0.0, b1 = 0.0, b2 = 0.0;
  while ((pA1 != mA) | (pA2 != pe) | (pB1 != mB) | (pB2 != pe)) {
    uint32_t q;
    q = pA1; const float x1 = coded8_step<NAN_AWARE>(q, rowA, amask, dlbit, shmul); pA1 = pA1 == mA ? pA1 : q;
    q = pB1; const float y1 = coded8_step<NAN_AWARE>(q, rowB, amask, dlbit, shmul); pB1 = pB1 == mB ? pB1 : q;
    const float x3 = coded8_step<NAN_AWARE>(pA2, rowA, amask, dlbit, shmul);
    const float y3 = coded8_step<NAN_AWARE>(pB2, rowB, amask, dlbit, shmul);
    q = pA1; const float x2 = coded8_step<NAN_AWARE>(q, rowA, amask, dlbit, shmul); pA1 = pA1 == mA ? pA1 : q;
    q = pB1; const float y2 = coded8_step<NAN_AWARE>(q, rowB, amask, dlbit, shmul); pB1 = pB1 == mB ? pB1 : q;
    const float x4 = coded8_step<NAN_AWARE>(pA2, rowA, amask, dlbit, shmul);
    const float y4 = coded8_step<NAN_AWARE>(pB2, rowB, amask, dlbit, shmul);
    add_pair_ftz(a1, x1, x2);
    add_pair_ftz(b1, y1, y2);
    add_pair_ftz(a2, x3, x4);
    add_pair_ftz(b2, y3, y4);
  }
  accA = a1 + a2;
  accB = b1 + b2;
}

// Two chains per lane over one row (two-row work units, TAHOE_CODE8_UROWS=2): the row's column
// walked as two halves split at col_mid, kCode8Exit steps per chain between exit tests.
#ifndef TAHOE_CODE8_EXIT
#define TAHOE_CODE8_EXIT 4
#endif
constexpr int kCode8Exit = TAHOE_CODE8_EXIT;
template <bool NAN_AWARE>
__device__ __forceinline__ void walk_coded8_split1(uint32_t pA1, uint32_t mA, uint32_t pA2, uint32_t pe,
                                                   uint32_t rowA, uint32_t amask, uint32_t dlbit,
                                                   uint32_t shmul, double& accA) {
  double a1 = 0.0, a2 = 0.0;
  while ((pA1 != mA) | (pA2 != pe)) {
#pragma unroll
    for (int k = 0; k < kCode8Exit / 2; k++) {
      uint32_t q;
      q = pA1; const float x1 = coded8_step<NAN_AWARE>(q, rowA, amask, dlbit, shmul); pA1 = pA1 == mA ? pA1 : q;
      const float x3 = coded8_step<NAN_AWARE>(pA2, rowA, amask, dlbit, shmul);
      q = pA1; const float x2 = coded8_step<NAN_AWARE>(q, rowA, amask, dlbit, shmul); pA1 = pA1 == mA ? pA1 : q;
      const float x4 = coded8_step<NAN_AWARE>(pA2, rowA, amask, dlbit, shmul);
      add_pair_ftz(a1, x1, x2);
      add_pair_ftz(a2, x3, x4);
    }
  }
  accA = a1 + a2;
}

// Leaf-diagnostic twins of the two wide-code walks (same steps, same order, same additions; the
// node read before each step is checked for a leaf, record_leaf).  A first-half chain frozen at its
// split slot re-reads a tree root, which is never a leaf.
template <bool NAN_AWARE>
__device__ __forceinline__ void walk_coded8_leaf(uint32_t pA, uint32_t pB, uint32_t pe, uint32_t rowA,
                                                 uint32_t rowB, uint32_t amask, uint32_t dlbit,
                                                 uint32_t shmul, double& accA, double& accB,
                                                 uint32_t sbase, const int2* __restrict__ meta,
                                                 int32_t* outA, int32_t* outB, uint64_t& fpA,
                                                 uint64_t& fpB) {
  accA = 0.0;
  accB = 0.0;
  fpA = 0;
  fpB = 0;
  while ((pA != pe) | (pB != pe)) {
    uint32_t y, q;
    q = pA; const float a1 = coded8_step<NAN_AWARE>(pA, rowA, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outA, fpA);
    q = pB; const float b1 = coded8_step<NAN_AWARE>(pB, rowB, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outB, fpB);
    q = pA; const float a2 = coded8_step<NAN_AWARE>(pA, rowA, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outA, fpA);
    q = pB; const float b2 = coded8_step<NAN_AWARE>(pB, rowB, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outB, fpB);
    add_pair_ftz(accA, a1, a2);
    add_pair_ftz(accB, b1, b2);
  }
}

template <bool NAN_AWARE>
__device__ __forceinline__ void walk_coded8_split_leaf(uint32_t pA1, uint32_t mA, uint32_t pA2, uint32_t pB1,
                                                       uint32_t mB, uint32_t pB2, uint32_t pe,
                                                       uint32_t rowA, uint32_t rowB, uint32_t amask,
                                                       uint32_t dlbit, uint32_t shmul, double& accA,
                                                       double& accB, uint32_t sbase,
                                                       const int2* __restrict__ meta, int32_t* outA,
                                                       int32_t* outB, uint64_t& fpA, uint64_t& fpB) {
  double a1 = 0.0, a2 = 0.0, b1 = 0.0, b2 = 0.0;
  fpA = 0;
  fpB = 0;
  while ((pA1 != mA) | (pA2 != pe) | (pB1 != mB) | (pB2 != pe)) {
    uint32_t q, y;
    q = pA1; const float x1 = coded8_step<NAN_AWARE>(q, rowA, amask, dlbit, shmul, &y);
    record_leaf(pA1, y, pe, amask, sbase, meta, outA, fpA); pA1 = pA1 == mA ? pA1 : q;
    q = pB1; const float y1 = coded8_step<NAN_AWARE>(q, rowB, amask, dlbit, shmul, &y);
    record_leaf(pB1, y, pe, amask, sbase, meta, outB, fpB); pB1 = pB1 == mB ? pB1 : q;
    q = pA2; const float x3 = coded8_step<NAN_AWARE>(pA2, rowA, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outA, fpA);
    q = pB2; const float y3 = coded8_step<NAN_AWARE>(pB2, rowB, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outB, fpB);
    q = pA1; const float x2 = coded8_step<NAN_AWARE>(q, rowA, amask, dlbit, shmul, &y);
    record_leaf(pA1, y, pe, amask, sbase, meta, outA, fpA); pA1 = pA1 == mA ? pA1 : q;
    q = pB1; const float y2 = coded8_step<NAN_AWARE>(q, rowB, amask, dlbit, shmul, &y);
    record_leaf(pB1, y, pe, amask, sbase, meta, outB, fpB); pB1 = pB1 == mB ? pB1 : q;
    q = pA2; const float x4 = coded8_step<NAN_AWARE>(pA2, rowA, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outA, fpA);
    q = pB2; const float y4 = coded8_step<NAN_AWARE>(pB2, rowB, amask, dlbit, shmul, &y);
    record_leaf(q, y, pe, amask, sbase, meta, outB, fpB);
    add_pair_ftz(a1, x1, x2);
    add_pair_ftz(b1, y1, y2);
    add_pair_ftz(a2, x3, x4);
    add_pair_ftz(b2, y3, y4);
  }
  accA = a1 + a2;
  accB = b1 + b2;
}

// k_sliced_codes8: k_sliced_codes' walk (slice resident in shared memory, dynamic 4-row work
// units, half-warp per row, two / four chains per lane) over 8-row tiles of u8 code rows; unit u of
// a tile: half h walks rows u + 2h (chain A) and u + 4 + 2h (chain B).  Tiles are claimed
// dynamically from a per-slice global counter (so the ~30 slices sweep the code rows together); a
// CTA whose slice runs out of tiles moves to the slice with the most remaining work per CTA
// (re-staging it), so no SM idles while another slice still has tiles.
// Ring hand-off with mbarriers only: entry e of a slice lives in buffer e % kR8 and completes full
// barrier e % kFull8 (parity (e / kFull8) & 1); every lane that worked on a unit of entry e arrives
// on the buffer's empty barrier, and the warp that releases the entry's LAST unit (elected by a
// per-buffer counter) waits on that empty phase, stores the entry's partials and issues entry
// e + kR8 into the buffer (all its lanes arrive on the new entry's full barrier, lane 0 with the
// transaction bytes) — the refill follows the release at once, with no producer warp to wake.  A
// consumer could wait on a stale full phase only if entry e - kFull8 had not arrived; then the
// kFull8 / kR8 later entries of that buffer are not issued and their units would hold every other
// consumer (static_assert below).  Past the slice's last tile an issue is a terminator (tile -1,
// no data); a buffer that issued one issues only terminators; consumers keep releasing entries
// and leave once every buffer has issued a terminator and every valid entry has been drained.  The
// barriers are re-initialised for the next slice.
// Work units of 2 rows (one per half-warp, the row's column walked as two halves: two chains per
// lane) and 20 warps: the ring holds 6 x 4 two-row units, so four units are loading while twenty
// are walked, and a warp's loop waits for the slowest of 64 half-column walks instead of 128.
// Same-box C4 walk: four-row units (four chains per lane) with 10 warps 5.52 ms, two-row units
// with 20 warps 5.38 ms, with 16 warps 5.56 ms (round 2; before, four-row units: 8 warps 6.42 ms,
// 10 warps 5.88 ms, 12 warps 6.11 ms).  -DTAHOE_CODE8_UROWS=4 -DTAHOE_CODE8_THREADS=320 restores
// the four-row units (experiments).
#ifndef TAHOE_CODE8_THREADS
#define TAHOE_CODE8_THREADS 640
#endif
constexpr int kCode8Threads = TAHOE_CODE8_THREADS;
constexpr int kFull8 = 6 * kCode8Ring;         // full barriers (6 per ring buffer)
template <bool FUSED, int R, int kR8, bool LEAF>
__global__ void __launch_bounds__(1024, 1) k_sliced_codes8(const __grid_constant__ Coded8KArgs a) {
  constexpr int C = kSlicedCols;
  constexpr int FS = R / kCode8TileRows;   // pre-pass tiles (NaN flags) per walked tile
  static_assert(R % kCode8TileRows == 0 && R * kR8 == kCode8TileRows * kCode8Ring, "ring rows");
  constexpr int kUnits = R / kCode8URows;
  constexpr int kWarps = kCode8Threads / 32;
  static_assert(kCode8URows == 4 || kCode8URows == 2, "unit rows");
  static_assert(kFull8 % kR8 == 0 && (kFull8 / kR8) * kUnits >= kWarps, "ring-wrap guard");
  extern __shared__ __align__(1024) unsigned char smem[];
  const uint32_t V = (uint32_t)a.img.vfbits;
  const uint32_t RB = 1u << V;
  const uint32_t tile_bytes = (uint32_t)R << V;
  const uint32_t sbase = smem_u32(smem);
  const uint32_t ring_off = ((sbase + (uint32_t)a.forest_smem + RB - 1u) & ~(RB - 1u)) - sbase;
  unsigned char* s_ring = smem + ring_off;
  uint32_t* s_flag = reinterpret_cast<uint32_t*>(s_ring + (size_t)kR8 * tile_bytes);
  double* s_part = reinterpret_cast<double*>(s_flag + kR8 * FS * 4);
  // control block (kCode8Ctl bytes): barriers, counters, tiles of the ring entries, slice
  uint64_t* s_full = reinterpret_cast<uint64_t*>(s_part + kR8 * R);   // [kFull8] entry arrived
  uint64_t* s_empty = s_full + kFull8;                                  // [kR8] entry released
  uint64_t* s_forest = s_empty + kR8;                                   // slice staged
  unsigned int* s_next = reinterpret_cast<unsigned int*>(s_forest + 1); // unit counter
  int32_t* s_cnt = reinterpret_cast<int32_t*>(s_next + 1);              // [kR8] units released
  int32_t* s_tile = s_cnt + kR8;                                        // [kR8] tile of the entry
  int32_t* s_vis = s_tile + kR8;                                        // valid entries issued
  int32_t* s_vdone = s_vis + 1;                                         // valid entries drained
  int32_t* s_dead = s_vis + 2;                                          // buffers that issued a terminator
  int32_t* s_slice = s_vis + 3;
  int32_t* s_cnext = s_vis + 4;                                         // [kR8] buffer's next claimed tile
  int32_t* s_cleft = s_cnext + kR8;                                     // [kR8] claimed tiles left
  static_assert(8 * (kFull8 + kR8 + 1) + 4 * (1 + 4 * kR8 + 4) <= kCode8Ctl, "control block");
  const int lane = threadIdx.x & 31;
  const int col = lane & (C - 1);
  const int half = lane >> 4;
  const uint32_t amask = RB - 1u;
  const uint32_t dlbit = RB;
  const uint32_t shmul = 1u << (32 - (V + 1));
  const int32_t ns = a.img.n_slices;
  const int32_t ntiles = (int32_t)((a.n + R - 1) / R);

  if (threadIdx.x == 0) {
    int32_t sl = (int32_t)blockIdx.x % ns;
    if (a.cta_start) {
      sl = 0;
      while (sl + 1 < ns && __ldg(&a.cta_start[sl + 1]) <= (int32_t)blockIdx.x) sl++;
    }
    *s_slice = sl;
    atomicAdd(&a.cta_on[sl], 1);
  }
  // issue entry e of slice sl into buffer e % kR8 (one whole warp); prev_dead: the buffer already
  // issued a terminator (then this is one too, without claiming)
  auto issue = [&](int sl, uint32_t e, bool prev_dead) {
    const int b = (int)(e % kR8);
    uint64_t* bar = &s_full[e % kFull8];
    if (lane == 0) {
      // a buffer claims a.claim consecutive tiles per global atomic and issues them one by one
      // (its issues are serialised by the ring, so the pair s_cnext / s_cleft needs no lock); a
      // chunk is used up before the buffer claims again, so a CTA leaving the slice (every buffer
      // past the last tile) holds no unprocessed claimed tile
      int32_t tile = -1;
      if (!prev_dead) {
        if (s_cleft[b] == 0) {
          s_cnext[b] = atomicAdd(&a.tile_next[sl], a.claim);
          s_cleft[b] = a.claim;
        }
        tile = s_cnext[b]++;
        s_cleft[b]--;
        if (tile >= ntiles) tile = -1;
      }
      s_tile[b] = tile;
      if (tile >= 0) {
        atomicAdd(s_vis, 1);
        // warm L2 with the tile this slice's CTAs will claim a few claims from now
        if (a.prefetch > 0 && tile + a.prefetch < ntiles)
          asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a.codes + (int64_t)(tile + a.prefetch) * tile_bytes),
                       "r"(tile_bytes) : "memory");
        fence_proxy_async_smem();
        mbar_expect_tx(bar, tile_bytes + 16u * FS);
        bulk_g2s(s_ring + (size_t)b * tile_bytes, a.codes + (int64_t)tile * tile_bytes, tile_bytes, bar);
        bulk_g2s(s_flag + b * FS * 4, a.flags + (int64_t)tile * FS * 4, 16u * FS, bar);
      } else {
        if (!prev_dead) atomicAdd(s_dead, 1);
        asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
      }
    } else {
      asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
    }
  };

  for (bool first = true;; first = false) {
    // (re)initialise the barriers and counters for this slice: every wait of the previous slice
    // has returned
    if (threadIdx.x == 0) {
      for (int b = 0; b < kFull8 + kR8 + 1; b++) {
        if (!first) asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(smem_u32(&s_full[b])) : "memory");
        mbar_init(&s_full[b], b < kFull8 ? 32u : (b < kFull8 + kR8 ? (uint32_t)(kUnits * 32) : 1u));
      }
      *s_next = 0u;
      for (int b = 0; b < kR8; b++) s_cnt[b] = s_cleft[b] = 0;
      *s_vis = 0;
      *s_vdone = 0;
      *s_dead = 0;
      fence_mbar_init();
    }
    __syncthreads();
    const int32_t sl = *s_slice;
    if (sl < 0) break;
    if (threadIdx.x < 32) {
      if (lane == 0) {   // a7: the slice
        const uint32_t bytes = (uint32_t)a.img.slots[sl] * (uint32_t)kSlotBytes;
        fence_proxy_async_smem();
        mbar_expect_tx(s_forest, bytes);
        bulk_g2s_big(smem, a.img.cnodes + (size_t)sl * a.img.slots_max * C * 2, bytes, s_forest);
      }
      for (uint32_t q = 0; q < (uint32_t)kR8; q++) issue(sl, q, false);
    }
    const uint32_t p0 = sbase + (uint32_t)col * 8u;
    const uint32_t pe = sbase + ((uint32_t)a.img.col_len[sl * C + col] * C + (uint32_t)col) * 8u;
    // the column's split slot (first tree of its second half), once per slice
    const uint32_t pm_sl = a.split ? sbase + ((uint32_t)__ldg(&a.img.col_mid[sl * C + col]) * C + (uint32_t)col) * 8u : pe;
    const int2* __restrict__ meta =
        LEAF ? reinterpret_cast<const int2*>(a.img.leaf_meta) + (size_t)sl * a.img.slots_max * C : nullptr;
    mbar_wait(s_forest, 0u);
    for (;;) {
      uint32_t q = 0;
      if (lane == 0) q = atomicAdd(s_next, 1u);
      q = __shfl_sync(0xffffffffu, q, 0);
      const uint32_t e = q / kUnits;
      const int u = (int)(q % kUnits);
      const int b = (int)(e % kR8);
      mbar_wait(&s_full[e % kFull8], (e / kFull8) & 1u);
      const int32_t tile = s_tile[b];
      if (tile >= 0) {
        const int64_t r0 = (int64_t)tile * R;
        const int nr = (int)((a.n - r0) < R ? (a.n - r0) : R);
        if (u < nr) {
          // four-row units: half h walks rows u + R/4 h (chain A) and + R/2 (chain B); two-row
          // units: half h walks row u + R/2 h only (chain B idle)
          const int rA = u + (R / kCode8URows) * half, rB = rA + R / 2;
          const bool okA = rA < nr, okB = kCode8URows == 4 && rB < nr;
          const uint32_t pA = okA ? p0 : pe, pB = okB ? p0 : pe;
          const uint32_t tb = sbase + ring_off + (uint32_t)b * tile_bytes;
          const uint32_t qA = (uint32_t)(okA ? rA : u), qB = (uint32_t)(okB ? rB : u);
          const uint32_t rowA = (tb + (qA << V)) | code8_swz(qA, V);   // XORed with the byte offset
          const uint32_t rowB = (tb + (qB << V)) | code8_swz(qB, V);
          uint32_t nan_flag = 0;
#pragma unroll
          for (int k = 0; k < FS; k++) {
            uint32_t fk;
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(fk) : "r"(smem_u32(s_flag + (b * FS + k) * 4)));
            nan_flag |= fk;
          }
          double accA, accB;
          uint64_t fpA = 0, fpB = 0;
          int32_t* oA = nullptr;
          int32_t* oB = nullptr;
          if (LEAF && a.o.out_leaf) {
            if (okA) oA = a.o.out_leaf + (a.row0 + r0 + rA) * (int64_t)a.o.T_leaf;
            if (okB) oB = a.o.out_leaf + (a.row0 + r0 + rB) * (int64_t)a.o.T_leaf;
          }
          if (kCode8URows == 2 && !LEAF && a.split) {
            const uint32_t pm = pm_sl;
            const uint32_t mA = okA ? pm : pe;
            accB = 0.0;
            if (nan_flag) walk_coded8_split1<true>(pA, mA, mA, pe, rowA, amask, dlbit, shmul, accA);
            else walk_coded8_split1<false>(pA, mA, mA, pe, rowA, amask, dlbit, shmul, accA);
          } else if (a.split) {
            const uint32_t pm = pm_sl;
            const uint32_t mA = okA ? pm : pe, mB = okB ? pm : pe;
            if (LEAF) {
              if (nan_flag) walk_coded8_split_leaf<true>(pA, mA, mA, pB, mB, mB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB, sbase, meta, oA, oB, fpA, fpB);
              else walk_coded8_split_leaf<false>(pA, mA, mA, pB, mB, mB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB, sbase, meta, oA, oB, fpA, fpB);
            } else {
              if (nan_flag) walk_coded8_split<true>(pA, mA, mA, pB, mB, mB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB);
              else walk_coded8_split<false>(pA, mA, mA, pB, mB, mB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB);
            }
          } else if (LEAF) {
            if (nan_flag) walk_coded8_leaf<true>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB, sbase, meta, oA, oB, fpA, fpB);
            else walk_coded8_leaf<false>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB, sbase, meta, oA, oB, fpA, fpB);
          } else if (nan_flag) {
            walk_coded8<true>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB);
          } else {
            walk_coded8<false>(pA, pB, pe, rowA, rowB, amask, dlbit, shmul, accA, accB);
          }
          // butterfly over the 16 lane columns: after the xor-8 exchange lanes with bit 3 clear
          // hold chain A, set hold chain B (lanes 0, 8, 16, 24 own rows rA(h=0), rB(h=0), rA(h=1),
          // rB(h=1))
          // (two-row units: chain B is empty, the lanes with bit 3 set add their chain A sums too,
          // in the same xor-8 first order; lanes 0 and 16 own the two rows)
          const bool b3 = kCode8URows == 4 && (lane & 8);
          double v = kCode8URows == 4 ? (b3 ? accB : accA) + __shfl_xor_sync(0xffffffffu, b3 ? accA : accB, 8)
                                      : accA + __shfl_xor_sync(0xffffffffu, accA, 8);
#pragma unroll
          for (int o = 4; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
          uint64_t fv = 0;
          if (LEAF) {
            fv = kCode8URows == 4 ? (b3 ? fpB : fpA) + __shfl_xor_sync(0xffffffffu, b3 ? fpA : fpB, 8)
                                  : fpA + __shfl_xor_sync(0xffffffffu, fpA, 8);
#pragma unroll
            for (int o = 4; o > 0; o >>= 1) fv += __shfl_xor_sync(0xffffffffu, fv, o);
          }
          const int rr = b3 ? rB : rA;
          if ((lane & (kCode8URows == 4 ? 7 : 15)) == 0 && (b3 ? okB : okA)) {
            if (FUSED) write_scalar(a.o, a.row0 + r0 + rr, v);
            else s_part[b * R + rr] = v;
            if (LEAF && a.o.out_fp)
              atomicAdd(reinterpret_cast<unsigned long long*>(&a.o.out_fp[a.row0 + r0 + rr]), (unsigned long long)fv);
          }
        }
    }
      // release the unit: every lane arrives on the buffer's empty barrier; the warp releasing the
      // entry's last unit waits for the whole entry, stores its partials and issues entry e + kR8
      asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(&s_empty[b])) : "memory");
      int last = 0;
      if (lane == 0) {
        last = atomicAdd(&s_cnt[b], 1) == kUnits - 1;
        if (last) atomicExch(&s_cnt[b], 0);
      }
      last = __shfl_sync(0xffffffffu, last, 0);
      if (last) {
        mbar_wait(&s_empty[b], (e / kR8) & 1u);
        if (tile >= 0 && !FUSED) {
          const int64_t r0 = (int64_t)tile * R;
          const int nr = (int)((a.n - r0) < R ? (a.n - r0) : R);
          if (lane < nr) a.o.raw[(size_t)sl * a.n_all + a.row0 + r0 + lane] = s_part[b * R + lane];
        }
        __syncwarp();
        issue(sl, e + kR8, tile < 0);
        if (tile >= 0 && lane == 0) atomicAdd(s_vdone, 1);
      }
      if (tile < 0) {
        int done = 0;
        if (lane == 0)
          done = *reinterpret_cast<volatile int32_t*>(s_dead) == kR8 &&
                 *reinterpret_cast<volatile int32_t*>(s_vdone) == *reinterpret_cast<volatile int32_t*>(s_vis);
        if (__shfl_sync(0xffffffffu, done, 0)) break;
      }
    }
    __syncthreads();   // every valid entry of this slice is consumed and drained
    if (threadIdx.x == 0) {
      atomicSub(&a.cta_on[sl], 1);
      // next slice: the most remaining work per CTA already on it
      int32_t best = -1;
      float bw = 0.0f;
      for (int32_t s2 = 0; s2 < ns; s2++) {
        const int32_t rem = ntiles - *reinterpret_cast<volatile int32_t*>(&a.tile_next[s2]);
        const int32_t on = *reinterpret_cast<volatile int32_t*>(&a.cta_on[s2]);
        if (rem < 1 || (on > 0 && rem < 2)) continue;   // a slice nobody works on is always taken
        const float w = (float)rem * __ldg(&a.work[s2]) / (float)(1 + on);
        if (w > bw) { bw = w; best = s2; }
      }
      if (!a.switch_slices) best = -1;
      if (best >= 0) atomicAdd(&a.cta_on[best], 1);
      *s_slice = best;
    }
    __syncthreads();
  }
}

int launch_sliced_codes8(const DevSliced& img, const SlicedPlan& plan, const float* X, int64_t n,
                         int32_t d, uint8_t* codes, const OutArgs& o, bool fused, int32_t num_sms,
                         void* stream, void* ev_b, void* ev_e) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const int64_t tbytes = code8_tile_bytes(img.vfbits);
  const int64_t chunk = code8_chunk_rows(img.vfbits, n);
  const int64_t ctiles = (chunk + kCode8TileRows - 1) / kCode8TileRows;
  uint32_t* flags = reinterpret_cast<uint32_t*>(codes + ctiles * tbytes);
  cudaError_t e = cudaSuccess;
  {
    static std::atomic<int> configured[64];
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev >= 0 && dev < 64 && !configured[dev].load()) {
      e = cudaFuncSetAttribute(k_encode_rows8<kEncode8Threads, kEncode8Rows>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin - 1024);
      if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_encode_rows8_tma<kEncode8Rows>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 kMaxSmemOptin - 1024);
      for (auto k : {k_sliced_codes8<true, kCode8TileRows, kCode8Ring, false>, k_sliced_codes8<false, kCode8TileRows, kCode8Ring, false>,
                     k_sliced_codes8<true, kCode8TileRows, kCode8Ring, true>, k_sliced_codes8<false, kCode8TileRows, kCode8Ring, true>})
        if (e == cudaSuccess) e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin);
      if (e != cudaSuccess) return (int)e;
      configured[dev].store(1);
    }
  }
  const int smem = plan.forest_smem + (int)code8_ring_smem(img.vfbits);
  const int threads = kCode8Threads;
  // Optional chunks of rows ($TAHOE_CODE8_CHUNK_MB) bound the code scratch; the default is one
  // launch pair for the whole batch (chunks small enough for the chunk's tiles to stay in L2
  // between the pre-pass and the ~30 slices were measured slower: each chunk pays a tail).  The
  // kernel events bracket the walk kernel, or the whole chunk loop when there are several chunks.
  const bool one = chunk >= n;
  if (ev_b && !one) cudaEventRecord(static_cast<cudaEvent_t>(ev_b), st);
  for (int64_t c0 = 0; c0 < n; c0 += chunk) {
    const int64_t cn = std::min(chunk, n - c0);
    const int64_t ntiles = (cn + kCode8TileRows - 1) / kCode8TileRows;
    // NaN flags (16 bytes per tile), then the per-slice tile counters and CTA counts
    e = cudaMemsetAsync(flags, 0, (size_t)ntiles * 16 + (size_t)img.n_slices * 8, st);
    if (e != cudaSuccess) return (int)e;
    Encode8Args ea;
    ea.X = X + c0 * d;
    ea.n = cn;
    ea.d = d;
    ea.vfbits = img.vfbits;
    ea.bands = img.c8_bands;
    // lcm(bands, SMs) items of equal rows: one persistent CTA per SM, bands / gcd items each
    ea.chunks = num_sms / std::gcd(std::max(1, img.c8_bands), num_sms);
    ea.img = img.c8_img;
    ea.grp = reinterpret_cast<const int4*>(img.c8_grp);
    ea.band = reinterpret_cast<const int4*>(img.c8_band);
    ea.v_src = img.v_src;
    ea.codes = codes;
    ea.flags = flags;
    // TMA-staged rows when X is a valid 2-D tensor (16-byte aligned rows) and every band fits one
    // box; else the rows through L1 ($TAHOE_CODE8_TMA=0 forces that path: experiments, tests)
    const bool tma_off = std::getenv("TAHOE_CODE8_TMA") && std::atoi(std::getenv("TAHOE_CODE8_TMA")) == 0;
    EncodeTiledFn enc = encode_tiled_fn();
    const bool tma = !tma_off && enc && img.c8_tma && (reinterpret_cast<uintptr_t>(X) & 15) == 0 && d % 4 == 0;
    if (tma) {
      Encode8TmaArgs ta{};
      ta.e = ea;
      const cuuint64_t gdim[2] = {(cuuint64_t)d, (cuuint64_t)cn};   // this chunk's rows
      const cuuint64_t gstride[1] = {(cuuint64_t)d * 4};
      const cuuint32_t box[2] = {(cuuint32_t)kCode8BoxW, (cuuint32_t)kCode8StageRows};
      const cuuint32_t estride[2] = {1, 1};
      CUresult r = enc(&ta.tmap, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(X + c0 * d), gdim,
                       gstride, box, estride, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                       CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) return (int)cudaErrorInvalidValue;
      k_encode_rows8_tma<kEncode8Rows><<<num_sms, kEncode8Threads, kCode8TmaTables + 2 * kCode8StageBytes + 64, st>>>(ta);
    } else {
      k_encode_rows8<kEncode8Threads, kEncode8Rows><<<num_sms, kEncode8Threads, kCode8BandBudget, st>>>(ea);
    }
    if ((e = cudaGetLastError()) != cudaSuccess) return (int)e;
    Coded8KArgs a{};
    a.img = img;
    a.codes = codes;
    a.flags = flags;
    a.tile_next = reinterpret_cast<int32_t*>(flags + ntiles * 4);
    a.cta_on = a.tile_next + img.n_slices;
    a.work = img.slice_w;
    a.n = cn;
    a.row0 = c0;
    a.n_all = n;
    a.forest_smem = plan.forest_smem;
    a.switch_slices = !(std::getenv("TAHOE_CODE8_SWITCH") && std::atoi(std::getenv("TAHOE_CODE8_SWITCH")) == 0);
    // L2 prefetch 32 tiles ahead of each issued tile (round 1, one tile per claim: 8 ahead, C4 walk
    // 7.27 -> 6.88 ms); $TAHOE_CODE8_PREFETCH overrides (experiments)
    a.prefetch = std::getenv("TAHOE_CODE8_PREFETCH") ? std::atoi(std::getenv("TAHOE_CODE8_PREFETCH")) : 32;
    // four chains per lane (C4 walk 6.43 -> 6.22 ms); $TAHOE_CODE8_SPLIT=0: two (experiments)
    a.split = img.col_mid ? (std::getenv("TAHOE_CODE8_SPLIT") ? std::atoi(std::getenv("TAHOE_CODE8_SPLIT")) : 1) : 0;
    // 8 tiles per claim: the global atomic's round trip sat in front of every refill (ncu: 4 % of
    // warp samples on its result, 19 % on the full barrier of entries it delayed).  Same-box C4
    // walk, tiles per claim 1 / 2 / 4 / 8 / 16 / 32: 5.95 / 5.71 / 5.59 / 5.53 / 5.56 / 5.61 ms
    // (prefetch 32; 8 per claim with prefetch 8 / 0: 5.55 / 5.62)
    a.claim = std::getenv("TAHOE_CODE8_CLAIM") ? std::max(1, std::atoi(std::getenv("TAHOE_CODE8_CLAIM"))) : 8;
    // a full GPU of CTAs (shared out among the slices by simulated work) once the chunk gives
    // every CTA a few tiles, else the plan's grid
    const bool full = plan.cta_start && ntiles >= 4LL * num_sms;
    a.cta_start = full ? plan.cta_start : nullptr;
    const int grid = full ? num_sms : plan.grid;
    a.o = o;
    // (16-row tiles in a 3-deep ring and 512 / 1024-thread CTAs measured within 2 %)
    const bool leaf = o.out_leaf != nullptr || o.out_fp != nullptr;
    auto kern = leaf ? (fused ? k_sliced_codes8<true, kCode8TileRows, kCode8Ring, true>
                              : k_sliced_codes8<false, kCode8TileRows, kCode8Ring, true>)
                     : (fused ? k_sliced_codes8<true, kCode8TileRows, kCode8Ring, false>
                              : k_sliced_codes8<false, kCode8TileRows, kCode8Ring, false>);
    if (ev_b && one) cudaEventRecord(static_cast<cudaEvent_t>(ev_b), st);
    kern<<<grid, threads, smem, st>>>(a);
    if ((e = cudaGetLastError()) != cudaSuccess) return (int)e;
  }
  if (ev_e) cudaEventRecord(static_cast<cudaEvent_t>(ev_e), st);
  return 0;
}

// ------------------------------------------------------------------ ROWS strategy (f1)
// Small batches (the paper's low-parallelism workload, batch 100): the sliced
// strategies stage a ~200 KB slice per CTA and need a finalize launch, which dominates a 100-row
// batch.  Here a CTA takes one sample: it stages the row in shared memory, each thread walks trees
// j = tid, tid + B, ... of the DIRECT image (hot child next; kept L2-resident across
// calls by tahoe_forest_l2_persist) and parks the tree's leaf value in shared memory; then every
// class's fp64 sum is formed by a fixed-order block reduction (each thread a contiguous chunk of the
// class's tree slots, then a fixed butterfly), and the block finalises the row (reading Z14/Z17).
// One launch, no scratch: CUDA-graph capturable.
template <bool LEAF>
__global__ void __launch_bounds__(kRowsThreads) k_rows(const DirectKArgs a) {
  extern __shared__ __align__(1024) unsigned char smem[];
  float* s_row = reinterpret_cast<float*>(smem);
  float* s_val = reinterpret_cast<float*>(smem + ((size_t)a.d * 4 + 15) / 16 * 16);
  double* s_red = reinterpret_cast<double*>(reinterpret_cast<unsigned char*>(s_val) +
                                            ((size_t)a.img.n_slots * 4 + 15) / 16 * 16);
  __shared__ unsigned long long s_fp[kRowsThreads / 32];
  const uint2* __restrict__ nodes = reinterpret_cast<const uint2*>(a.img.nodes);
  const int fbits = a.img.fbits;
  const uint32_t fmask = (1u << fbits) - 1u;
  const uint32_t offmask = (1u << (kOffsetTop - fbits)) - 1u;
  const int32_t T = a.img.n_slots, C = a.o.n_classes, B = blockDim.x;
  const bool vote = a.o.agg == TAHOE_AGG_VOTE;
  // the first tree's root node is fetched before the row is staged (two dependent L2 reads that
  // overlap the staging); it is the same for every row of this CTA
  const uint32_t k0 = threadIdx.x < T ? (uint32_t)__ldg(&a.img.root[threadIdx.x]) : 0u;
  const uint2 nd0 = threadIdx.x < T ? __ldg(&nodes[k0]) : make_uint2(0u, 0u);
  for (int64_t i = blockIdx.x; i < a.n; i += gridDim.x) {
    __syncthreads();   // the previous row's values and reductions are consumed
    const float* __restrict__ x = a.X + i * a.d;
    for (int c = threadIdx.x; c < a.d; c += B) s_row[c] = __ldg(&x[c]);
    __syncthreads();
    uint64_t fp = 0;
    for (int32_t j = threadIdx.x; j < T; j += B) {
      uint32_t k = j == (int32_t)threadIdx.x ? k0 : (uint32_t)__ldg(&a.img.root[j]);
      uint2 nd = j == (int32_t)threadIdx.x ? nd0 : __ldg(&nodes[k]);
      while ((int32_t)nd.y >= 0) {   // internal: "x_j < b_i", NaN -> default
        k += step(nd.x, nd.y, s_row[nd.y & fmask], fbits, offmask);
        nd = __ldg(&nodes[k]);
      }
      s_val[j] = __uint_as_float(nd.x);
      if (LEAF) {
        const int32_t tree = __ldg(&a.img.tree_orig[j]);
        const uint32_t leaf = nd.y & 0x7fffffffu;
        if (a.o.out_leaf) a.o.out_leaf[i * a.o.T_leaf + tree] = (int32_t)leaf;
        fp += mix64(((uint64_t)(uint32_t)tree << 32) | leaf);
      }
    }
    __syncthreads();
    // a9 combine: per class a fixed-order fp64 sum of its tree slots (VOTE: exact counts) — each
    // thread a contiguous chunk, a warp butterfly, the warps' values summed in warp order; all
    // classes share the two block barriers
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, W = B >> 5;
    for (int32_t c = 0; c < C; c++) {
      const int32_t s0 = vote ? 0 : __ldg(&a.img.cls_seg[c]), s1 = vote ? T : __ldg(&a.img.cls_seg[c + 1]);
      const int32_t chunk = (s1 - s0 + B - 1) / B;
      const int32_t q0 = s0 + threadIdx.x * chunk, q1 = min(s1, q0 + chunk);
      double part = 0.0;
      for (int32_t q = q0; q < q1; q++)
        part += vote ? (s_val[q] == (float)c ? 1.0 : 0.0) : (double)s_val[q];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
      if (lane == 0) s_red[c * W + warp] = part;
    }
    __syncthreads();
    double* s_cls = s_red + (size_t)C * W;
    for (int32_t c = threadIdx.x; c < C; c += B) {
      double sum = 0.0;
      for (int w = 0; w < W; w++) sum += s_red[c * W + w];
      s_cls[c] = sum;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      int best = 0;
      double bv = 0.0;
      for (int32_t c = 0; c < C; c++) {
        const double sum = s_cls[c];
        if (a.o.raw) {
          a.o.raw[i * C + c] = sum;
          continue;
        }
        // a10 finalize (as finalize_row / write_scalar)
        double v;
        if (vote) v = sum;
        else if (a.o.agg == TAHOE_AGG_AVERAGE) v = sum / (double)a.o.n_trees_full + (double)a.o.base;
        else v = sum + (double)a.o.base;
        a.o.out[i * C + c] = (float)v;
        if (c == 0 || v > bv) { best = c; bv = v; }
      }
      if (!a.o.raw && a.o.out_class) {
        if (a.o.agg == TAHOE_AGG_BINARY) a.o.out_class[i] = bv > 0.0 ? 1 : 0;
        else if (a.o.agg == TAHOE_AGG_CLASS_SUM || vote) a.o.out_class[i] = best;
        else a.o.out_class[i] = 0;
      }
    }
    if (LEAF && a.o.out_fp) {
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) fp += __shfl_xor_sync(0xffffffffu, fp, o);
      if ((threadIdx.x & 31) == 0) s_fp[threadIdx.x >> 5] = fp;
      __syncthreads();
      if (threadIdx.x == 0) {
        unsigned long long t = 0;
        for (int w = 0; w < (B >> 5); w++) t += s_fp[w];
        a.o.out_fp[i] += t;   // the launcher zeroed out_fp; chunked images add per launch
      }
    }
  }
}

int launch_rows(const DevDirect& img, const float* X, int64_t n, int32_t d, const OutArgs& o,
                int32_t num_sms, void* stream) {
  const int64_t smem = rows_smem_bytes(d, img.n_slots, o.n_classes);
  if (smem > kMaxSmemOptin - 1024) return (int)cudaErrorInvalidValue;
  DirectKArgs a{img, X, n, d, o};
  const bool leaf = o.out_leaf != nullptr || o.out_fp != nullptr;
  auto kern = leaf ? k_rows<true> : k_rows<false>;
  static std::atomic<int> configured[64];
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev >= 0 && dev < 64 && configured[dev].load() < smem) {
    cudaError_t e = cudaFuncSetAttribute(k_rows<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin - 1024);
    if (e == cudaSuccess) e = cudaFuncSetAttribute(k_rows<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxSmemOptin - 1024);
    if (e != cudaSuccess) return (int)e;
    configured[dev].store(kMaxSmemOptin);
  }
  int per_sm = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kRowsThreads, (size_t)smem);
  if (per_sm < 1) per_sm = 1;
  const int grid = (int)std::min<int64_t>(n, (int64_t)num_sms * per_sm);
  kern<<<grid, kRowsThreads, (size_t)smem, static_cast<cudaStream_t>(stream)>>>(a);
  return (int)cudaGetLastError();
}

// ------------------------------------------------------------------ microbenchmarks
// "Measure hardware parameters by a microbenchmark" (Algorithm 1 line 4), re-targeted:
// the walk is bound by the shared-memory (LSU) data pipe, so the peak it is measured against is the
// node-read rate of the production walk itself on ideal data — every lane walks a column of L
// internal nodes (the same node words, the same walk_coded2 / walk_coded8_split code) that all
// go left, the two half-warps on different slot rows (an 8-byte node load of a warp is 2
// wavefronts, its minimum), the code loads conflict-free, perfect lockstep, no tile traffic.
// A warp-step is then 2 wavefronts of node + 1 of code.  VAR 0: u16 codes, two chains per lane
// (k_sliced_codes); VAR 1: u8 codes over 2 KB rows, four chains per lane (k_sliced_codes8).
template <int VAR>
__global__ void __launch_bounds__(1024, 1) k_visit_peak(int32_t L, int32_t reps, double* sink) {
  extern __shared__ __align__(1024) unsigned char smem[];
  constexpr int C = kSlicedCols;
  const int lane = threadIdx.x & 31, col = lane & (C - 1), half = lane >> 4;
  // two synthetic slices of L + 1 slots (one per half-warp), then the code rows
  const uint32_t slice_bytes = (uint32_t)(L + 1) * kSlotBytes;
  uint32_t* w = reinterpret_cast<uint32_t*>(smem);
  const uint32_t F = VAR == 0 ? 5u : 11u;                       // attribute field bits
  const uint32_t sh = VAR == 0 ? F + 2 : F + 1;                 // offset shift
  const uint32_t amask = VAR == 0 ? ((1u << F) - 1u) << 1 : (1u << F) - 1u;
  const uint32_t dlbit = VAR == 0 ? 1u << (F + 1) : 1u << F;
  const uint32_t shmul = 1u << (32 - sh);
  for (uint32_t q = threadIdx.x; q < 2 * (uint32_t)(L + 1) * C; q += blockDim.x) {
    const uint32_t slot = (q / C) % (uint32_t)(L + 1), c = q % C;
    const bool term = slot == (uint32_t)L;
    // internal: rank t larger than every code (left, next slot); attribute: column c's own code
    // (u16: bytes 2c of a 64-byte row; u8: byte 4c); terminal: self-loop, all-ones attribute
    const uint32_t attr = VAR == 0 ? (c << 1) : (c << 2);
    w[2 * q] = term ? 0u : (VAR == 0 ? 0x7FFFu : 127u);
    w[2 * q + 1] = term ? amask : attr;
  }
  unsigned char* rows = smem + 2 * slice_bytes;
  for (uint32_t q = threadIdx.x; q < 8192 / 4; q += blockDim.x) reinterpret_cast<uint32_t*>(rows)[q] = 0u;
  __syncthreads();
  const uint32_t sb = smem_u32(smem) + (uint32_t)half * slice_bytes;
  const uint32_t p0 = sb + (uint32_t)col * 8u;
  const uint32_t pe = sb + ((uint32_t)L * C + (uint32_t)col) * 8u;
  const uint32_t rb = smem_u32(rows);
  double tot = 0.0;
  for (int r = 0; r < reps; r++) {
    double accA, accB;
    if (VAR == 0) {
      // chain A rows of the two halves share one 128-byte line (rows u and u+16), chain B likewise
      const uint32_t rowA = rb + (uint32_t)half * 64u, rowB = rb + 128u + (uint32_t)half * 64u;
      walk_coded2<false, false>(p0, p0, pe, rowA, rowB, amask, dlbit, shmul, accA, accB);
    } else {
      const uint32_t rowA = rb + (uint32_t)half * 64u, rowB = rb + 2048u + (uint32_t)half * 64u;
      const uint32_t pm = sb + ((uint32_t)(L / 2) * C + (uint32_t)col) * 8u;
      if (kCode8URows == 2) {   // the production walk: one row per half-warp, two chains per lane
        walk_coded8_split1<false>(p0, pm, pm, pe, rowA, amask, dlbit, shmul, accA);
        walk_coded8_split1<false>(p0, pm, pm, pe, rowB, amask, dlbit, shmul, accB);
      } else {
        walk_coded8_split<false>(p0, pm, pm, p0, pm, pm, pe, rowA, rowB, amask, dlbit, shmul, accA, accB);
      }
    }
    double v = accA + accB;
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    tot += v;
  }
  if (tot != 0.0) sink[blockIdx.x] = tot;   // never true (internal words add +0); keeps the walk
}

// VAR 2: the direct walk's peak (k_direct_tlp's step: an 8-byte node through L1 with __ldg, the
// attribute from a row staged in shared memory, the hot child next): every thread walks a chain of
// internal nodes that all go to their hot child, in a node array small enough to stay L1-resident
// (`nodes`, 4096 nodes = 32 KB), eight threads per row over 64 staged rows per CTA as the
// production kernel — i.e. the node-read rate when every node read hits L1.
__global__ void __launch_bounds__(512) k_visit_peak_direct(const uint2* __restrict__ nodes, int32_t steps,
                                                           uint32_t mask, double* sink) {
  __shared__ float s_rows[64 * 101];
  for (int q = threadIdx.x; q < 64 * 101; q += blockDim.x) s_rows[q] = (float)(q % 7);
  __syncthreads();
  const int fbits = 7;
  const uint32_t fmask = (1u << fbits) - 1u;
  const uint32_t offmask = (1u << (kOffsetTop - fbits)) - 1u;
  const float* row = s_rows + (threadIdx.x >> 3) * 101;
  uint32_t k = (threadIdx.x * 37u) & mask;   // mask (4095) is a kernel argument: the chain is live
  for (int i = 0; i < steps; i++) {
    const uint2 nd = __ldg(&nodes[k]);
    k = (k + step(nd.x, nd.y, row[nd.y & fmask], fbits, offmask)) & mask;
  }
  if (k == 0xFFFFFFFFu) sink[blockIdx.x] = (double)k;   // never (mask < 2^32 - 1)
}

// Raw shared-memory load bandwidth: every warp issues conflict-free 16-byte loads (a warp = 512 B =
// 4 wavefronts) in independent chains; bytes per SM clock from clock64 around the loop.
__global__ void __launch_bounds__(1024, 1) k_smem_bw(int32_t iters, unsigned long long* cycles, uint32_t* sink) {
  extern __shared__ __align__(1024) unsigned char smem[];
  uint4* v = reinterpret_cast<uint4*>(smem);
  for (int q = threadIdx.x; q < 4096; q += blockDim.x) v[q] = make_uint4(q, q + 1, q + 2, q + 3);
  __syncthreads();
  const uint32_t base = smem_u32(smem) + (uint32_t)(threadIdx.x & 31) * 16u;
  uint32_t acc = 0;
  const unsigned long long t0 = clock64();
  for (int i = 0; i < iters; i++) {
#pragma unroll
    for (int k = 0; k < 8; k++) {
      uint4 r;
      asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                   : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
                   : "r"(base + (uint32_t)(((i * 8 + k) & 63) * 512)));
      acc ^= r.x ^ r.w;
    }
  }
  __syncthreads();
  const unsigned long long t1 = clock64();
  if (threadIdx.x == 0) cycles[blockIdx.x] = t1 - t0;
  if (acc == 0x12345678u) sink[blockIdx.x] = acc;
}

int launch_visit_peak(int32_t variant, int32_t L, int32_t reps, int32_t grid, double* sink, void* stream) {
  const int smem = 2 * (L + 1) * kSlotBytes + 8192;
  auto kern = variant == 0 ? k_visit_peak<0> : k_visit_peak<1>;
  // at least 120 KB of dynamic shared memory: one CTA per SM, as the production walk
  const int dyn = std::max(smem, 120 * 1024);
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, dyn);
  if (e != cudaSuccess) return (int)e;
  kern<<<grid, 1024, dyn, static_cast<cudaStream_t>(stream)>>>(L, reps, sink);
  return (int)cudaGetLastError();
}

int launch_visit_peak_direct(const void* nodes, int32_t steps, int32_t grid, double* sink, void* stream) {
  k_visit_peak_direct<<<grid, 512, 0, static_cast<cudaStream_t>(stream)>>>(static_cast<const uint2*>(nodes), steps, 4095u, sink);
  return (int)cudaGetLastError();
}

int launch_smem_bw(int32_t iters, int32_t grid, unsigned long long* cycles, uint32_t* sink, void* stream) {
  const int dyn = 120 * 1024;
  cudaError_t e = cudaFuncSetAttribute(k_smem_bw, cudaFuncAttributeMaxDynamicSharedMemorySize, dyn);
  if (e != cudaSuccess) return (int)e;
  k_smem_bw<<<grid, 1024, dyn, static_cast<cudaStream_t>(stream)>>>(iters, cycles, sink);
  return (int)cudaGetLastError();
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
