// kernels.hpp — device images and launch arguments shared by the host code and kernels.cu.
// Plain structs of raw pointers and sizes (no CUDA types), so host .cpp files compile with g++.
#pragma once
#include <cstdint>

namespace tahoe {

// ------------------------------------------------------------------ node word encoding
// 8-byte node {x, y} (variable-length attribute index P:1006-1015):
//   internal: x = fp32 threshold bits;
//             y = [31] 0 | [30] default_left | [29] hot_is_left | [28:F] cold delta | [F-1:0] feature
//   leaf:     x = fp32 leaf value bits;
//             y = [31] 1 | [30:0] sliced image: slot delta to the lane's next tree root
//                                 direct image: caller node id
// The hot child (the more probable one) is always the next node/slot (+1); the cold
// child is at +cold delta.  F = feature_bits(n_features).
constexpr uint32_t kLeafBit = 0x80000000u;
constexpr uint32_t kDefaultLeftBit = 0x40000000u;
constexpr uint32_t kHotLeftBit = 0x20000000u;
constexpr int kOffsetTop = 29;   // cold delta occupies bits [28:F]

struct DevDirect {
  const uint32_t* nodes = nullptr;   // uint2 per node
  const int32_t* root = nullptr;     // per tree slot (class-major order)
  const int32_t* cls = nullptr;      // per tree slot
  const int32_t* tree_orig = nullptr;
  const int32_t* slot_orig = nullptr; // caller node id of every node slot (visit counting)
  const int32_t* cls_seg = nullptr;   // [n_classes + 1] tree-slot range of each class (class-major)
  int32_t n_slots = 0;
  int32_t fbits = 0;
  int64_t n_nodes = 0;
};

struct int4x { int32_t x, y, z, w; };   // host-side stand-in for CUDA's int4 (same layout)

struct DevSliced {
  const uint32_t* nodes = nullptr;   // [ns][slots_max][32] uint2
  const int32_t* col_len = nullptr;  // [ns][32]
  const int32_t* slots = nullptr;    // [ns]
  const int32_t* leaf_meta = nullptr;// [ns][slots_max][32] int2 {caller tree, caller node}
  int32_t n_slices = 0;
  int32_t slots_max = 0;
  int32_t fbits = 0;
  // rank-coded twin (reading R7); cnodes == nullptr when the forest does not qualify
  const uint32_t* cnodes = nullptr;  // [ns][slots_max][16] uint2
  const float* thr_tab = nullptr;    // sorted distinct thresholds, attribute after attribute
  const int32_t* thr_off = nullptr;  // [n_features + 1]
  int32_t n_features = 0;            // attributes coded per row
  int32_t n_thr = 0;                 // thr_off[n_features]
  const float* cb_img = nullptr;     // bank-private tables (cb_rows x 32 words) or nullptr
  const int32_t* cb_desc = nullptr;  // [cb_passes][32] int4
  const int32_t* slot_attr = nullptr; // [2^fbits] attribute coded in each u16 slot (-1 = pad; R10)
  int32_t cb_rows = 0, cb_passes = 0;
  // wide rank codes (reading R8): cnodes hold u8-code node words when code8 != 0
  int32_t code8 = 0;
  int32_t vfbits = 0;                // code row = 2^vfbits bytes
  const int32_t* v_src = nullptr;    // [2^vfbits] source column of each code byte, -1 = pad
  const float* c8_img = nullptr;     // pre-pass tables (bank-private, band after band)
  const int4x* c8_grp = nullptr;     // [2^vfbits / 32] {word offset in band, probes, band, 0}
  const int4x* c8_band = nullptr;    // [bands] {byte offset, bytes, first group, end group}
  int32_t c8_bands = 0;
  int32_t c8_tma = 0;                // every band fits k_encode_rows8_tma (<= 8 groups, 256 sources)
  const float* slice_w = nullptr;    // [ns] simulated lane-steps per row (dynamic slice choice)
  const int32_t* col_mid = nullptr;  // [ns][16] split slot of each column (two chains per row)
};

// ------------------------------------------------------------------ rank-coded rows (reading R7)
// A sample row becomes u16 codes: code(x) = #{distinct thresholds of the attribute <= x}
// (< kCodeMaxRank), NaN -> kCodeNan; slots n_features .. 2^F - 1 hold kCodePad.  Loaded
// sign-extended, kCodeNan / kCodePad are 0xFFFFFFFE / 0xFFFFFFFF, larger than every node word,
// so "code < t" sends NaN right (its default path is applied separately) and a leaf's pad read
// never goes left.  A 64-row tile of code rows is kCodeTileRows * code_row_bytes(F) bytes; with
// 64-byte rows, row r sits at ((r & 15) << 7) | (((r >> 4) & 1) << 6) | ((r >> 5) << 11), so
// the rows u and u + 16 that the two half-warps of a warp walk together occupy the two halves of
// one 128-byte bank line (conflict-free attribute loads).
constexpr int32_t kCodeMaxRank = 32000;
constexpr int32_t kCodeMaxFbits = 7;
constexpr int32_t kCodeBankBudget = 216 * 1024;   // shared memory for the bank-private tables
constexpr uint16_t kCodeNan = 0xFFFEu;
constexpr uint16_t kCodePad = 0xFFFFu;
inline int32_t code_row_bytes(int32_t fbits) { return (2 << fbits) < 64 ? 64 : (2 << fbits); }
inline int32_t code_tile_bytes(int32_t fbits) { return 64 * code_row_bytes(fbits); }
// a code tile in HBM and in the ring: the rows, then a trailer whose first word is the tile's NaN
// flag (1 if any of its codes is kCodeNan; it arrives with the tile's bulk copy).  The trailer is
// max(128, row bytes) long so that every ring buffer's rows stay aligned to the row size: a code
// address is formed by OR-ing the attribute's byte offset into the row base.
inline int32_t code_tile_stride(int32_t fbits) {
  return code_tile_bytes(fbits) + (code_row_bytes(fbits) > 128 ? code_row_bytes(fbits) : 128);
}

// ------------------------------------------------------------------ wide codes (reading R8)
// Rows of more than 127 attributes: an attribute with K distinct thresholds becomes ceil(K / 127)
// VIRTUAL attributes; piece k codes thresholds tab[127k .. 127k + 126] as
// code_k(x) = #{i in the piece : tab[i] <= x} = clamp(code(x) - 127k, 0, 127), and a node whose
// threshold is tab[i] reads piece k = i / 127 with t = i - 127k + 1, so that
// x < tab[i]  <=>  code(x) < i + 1  <=>  code_k(x) < t  (R7's exactness, piece by piece).  Codes are
// s8: 0 .. 127, NaN kCode8Nan (-2), pad kCode8Pad (-1); loaded sign-extended they exceed every node
// word like R7's u16 codes.  A code row is 2^V bytes (V = vfbits, all-ones byte = the pad a leaf
// reads); node words: internal x = t, y = off_bytes << (V+1) | default_left << V | virtual
// attribute; leaf x = value, y = off_bytes << (V+1) | (2^V - 1).  Tiles of kCode8TileRows rows;
// the tiles' NaN flags sit in a separate array (16 bytes per tile) that rides along with each
// tile's bulk copy.
constexpr int32_t kCode8MaxRank = 127;
constexpr int32_t kCode8MaxFbits = 12;           // rows of <= 4 KB
constexpr int32_t kCode8TileRows = 8;
#ifndef TAHOE_CODE8_RING
#define TAHOE_CODE8_RING 6   // -DTAHOE_CODE8_RING for experiments
#endif
constexpr int32_t kCode8Ring = TAHOE_CODE8_RING;
constexpr int32_t kCode8BandBudget = 200 * 1024; // pre-pass tables per CTA
// TMA-staged pre-pass (k_encode_rows8_tma): a band is at most 4 groups (128 virtual attributes, so
// at most 128 source attributes; from the first one rounded down to a 16-byte boundary — a box
// start off that boundary is an illegal instruction — they fit one 2-D tensor box of 132 floats
// per row, 528 bytes, a multiple of 16) and its tables at most 4 x 127 x 128 bytes; two 128-row
// stages of X (one 4-row group per warp of the 1024-thread CTA) follow the tables in shared
// memory (65 + 135 KB).  C4: 16 bands read 2112 floats per 2000-float row (3-group bands of
// 128-float boxes: 22 bands, 2816 floats, 1.41x the row bytes from HBM)
constexpr int32_t kCode8BandGroups = 4;
constexpr int32_t kCode8BoxW = 132;
constexpr int32_t kCode8StageRows = 128;
constexpr int32_t kCode8StageBytes = kCode8StageRows * kCode8BoxW * 4;
constexpr int32_t kCode8TmaTables = kCode8BandGroups * 127 * 128;
constexpr int8_t kCode8Nan = -2;
constexpr int8_t kCode8Pad = -1;
inline int64_t code8_tile_bytes(int32_t vfbits) { return (int64_t)kCode8TileRows << vfbits; }
// rows per launch: the chunk's code tiles (~48 MB) stay in the 126 MB L2 between the pre-pass
// and the slices
int64_t code8_chunk_mb();   // $TAHOE_CODE8_CHUNK_MB (experiments); default 0 = one launch
inline int64_t code8_chunk_rows(int32_t vfbits, int64_t n) {
  if (code8_chunk_mb() <= 0) return n > 0 ? n : 1;
  int64_t c = (code8_chunk_mb() << 20) >> vfbits;
  c -= c % kCode8TileRows;
  if (c < kCode8TileRows) c = kCode8TileRows;
  return n < c ? n : c;
}
// mbarriers (6 full per buffer, one empty per buffer, slice), counters, entry tiles and claims
constexpr int32_t kCode8Ctl = kCode8Ring <= 6 ? 512 : 1024;
// shared memory next to the slice: the ring (aligned to the row size), the flags, staged partials,
// the control block
inline int64_t code8_ring_smem(int32_t vfbits) {
  return (int64_t)kCode8Ring * code8_tile_bytes(vfbits) + (1LL << vfbits) + kCode8Ring * 16 +
         kCode8Ring * kCode8TileRows * 8 + kCode8Ctl;
}

struct OutArgs {
  float* out = nullptr;          // final scores (fused finalize) or nullptr
  int32_t* out_class = nullptr;
  int32_t* out_leaf = nullptr;   // [n][T_leaf] caller tree order
  uint64_t* out_fp = nullptr;    // fingerprint (atomic u64 adds; zeroed by the launcher)
  double* raw = nullptr;         // fp64 parts (layout chosen by the strategy)
  int32_t agg = 0;
  float base = 0.0f;
  int32_t n_trees_full = 1;      // AVERAGE divisor
  int32_t n_classes = 1;
  int32_t T_leaf = 0;            // row stride of out_leaf
};

struct FinalizeArgs {
  const double* partial = nullptr;
  int64_t part_stride = 0;       // element stride between parts
  int64_t row_stride = 0;        // element stride between samples
  const int32_t* class_ptr = nullptr;    // device CSR class -> parts, or nullptr: part c == class c
  const int32_t* class_parts = nullptr;
  int32_t n_classes = 1;
  int32_t agg = 0;
  float base = 0.0f;
  int32_t n_trees_full = 1;
  int64_t n = 0;
  float* out = nullptr;          // FINAL mode
  int32_t* out_class = nullptr;
  double* raw_out = nullptr;     // RAW mode (n x C fp64, no base) if non-null
};

// Launchers (kernels.cu).  Return a cudaError_t value as int (0 = success).
constexpr int32_t kMaxSmemOptin = 232448;   // sharedMemPerBlockOptin on sm_100 (227 KB)
constexpr int32_t kSlicedCols = 16;         // lane columns per slice (one per half-warp lane)
constexpr int32_t kSlotBytes = kSlicedCols * 8;  // one slot row: 16 columns x 8-byte nodes
constexpr int32_t kSlicedRing = 3;          // sample-tile ring depth of k_sliced
constexpr int32_t kSlicedTileRows = 64;     // rows per tile (two per warp of a 1024-thread CTA)
constexpr int32_t kSlicedBarrierBytes = 128;
// rank-coded slices (k_sliced_codes): ring of `ring` code tiles (3 .. kCodedRingMax, as many as fit),
// a control block, `ring` x 64 staged fp64 partials
constexpr int32_t kCodedRingMax = 8;
constexpr int32_t kCodedCtlBytes = 256;
inline int32_t coded_ring_smem(int32_t ring, int32_t tstride) {
  return ring * tstride + kCodedCtlBytes + ring * kSlicedTileRows * 8;
}
inline int32_t coded_ring_depth(int32_t forest_smem, int32_t tstride) {
  int32_t r = kCodedRingMax;
  while (r > kSlicedRing && forest_smem + coded_ring_smem(r, tstride) > kMaxSmemOptin) r--;
  return r;
}

// PADDED staging: rows at a stride that is a multiple of 2^fbits floats (>= d, >= 4), so that row
// bases are aligned to the attribute byte-offset field and a leaf's all-ones attribute stays
// inside the row.  DENSE staging: rows at stride d plus a tail pad for the last row's leaf read.
inline int32_t sliced_row_stride(int32_t d, int32_t fbits, bool padded) {
  if (!padded) return d;
  int32_t q = 1 << fbits;
  if (q < 4) q = 4;
  return ((d + q - 1) / q) * q;
}
inline int32_t sliced_buf_floats(int32_t d, int32_t fbits, bool padded) {
  if (padded) return kSlicedTileRows * sliced_row_stride(d, fbits, true);
  const int64_t f = (int64_t)kSlicedTileRows * d + (1 << fbits);
  return (int32_t)((f + 255) & ~255LL);  // keep every buffer 1 KB aligned
}
// Shared memory of the sample-tile ring, or -1 when rows are too wide to stage (> 64 KB).
inline int64_t sliced_ring_bytes(int32_t d, int32_t fbits, bool padded) {
  int64_t b = (int64_t)kSlicedRing * sliced_buf_floats(d, fbits, padded) * 4;
  return b <= 64 * 1024 ? b : -1;
}
bool padded_rows_possible(const float* X, int32_t d);  // kernels.cu

struct SlicedPlan {
  int32_t grid = 0, block = 1024, tile_rows = 0, cps = 1;
  int32_t smem_bytes = 0, forest_smem = 0, buf_floats = 0, row_stride = 0;
  int32_t rows = 0;  // 0 global, 1 dense, 2 padded (kernels.cu kRows*)
  const int32_t* cta_start = nullptr;  // coded slices: CTA -> slice prefix (grid == its total),
                                       // or nullptr: CTA b works on slice b % n_slices
};
int launch_direct(const DevDirect& img, const float* X, int64_t n, int32_t d, const OutArgs& o,
                  bool fused, int32_t num_sms, void* stream);
int launch_sliced(const DevSliced& img, const SlicedPlan& plan, const float* X, int64_t n,
                  int32_t d, const OutArgs& o, bool fused, void* stream);
// rank-coded sliced strategy: encode X into code tiles (codes: device scratch of
// ntiles * code_tile_stride bytes), then walk the coded slices
// prof != nullptr: the PROF instantiation (per-lane walk spans -> prof[6], load-balance statistics)
int launch_sliced_codes(const DevSliced& img, const SlicedPlan& plan, const float* X, int64_t n,
                        int32_t d, uint16_t* codes, const OutArgs& o, bool fused, int32_t num_sms,
                        void* stream, void* ev_b, void* ev_e, double* prof = nullptr);
// wide rank codes (reading R8): per chunk of code8_chunk_rows rows, u8 code tiles (codes: scratch
// of ctiles * code8_tile_bytes + ctiles * 16 bytes of NaN flags + n_slices * 8 bytes of counters,
// ctiles = the chunk's tiles), then the coded slices over them
int launch_sliced_codes8(const DevSliced& img, const SlicedPlan& plan, const float* X, int64_t n,
                         int32_t d, uint8_t* codes, const OutArgs& o, bool fused, int32_t num_sms,
                         void* stream, void* ev_b, void* ev_e);
int launch_finalize(const FinalizeArgs& a, void* stream);
// ROWS strategy (small batches): one CTA per sample, lane = tree over the direct
// image, fixed-order block reduction and in-kernel finalize; one launch, no scratch.  Returns
// cudaErrorInvalidValue when the row + per-tree values exceed the shared memory it may use.
constexpr int32_t kRowsThreads = 512;
// row | per-tree values | per-(class, warp) partials + per-class sums
inline int64_t rows_smem_bytes(int32_t d, int32_t n_slots, int32_t n_out = 1) {
  return ((int64_t)d * 4 + 15) / 16 * 16 + ((int64_t)n_slots * 4 + 15) / 16 * 16 +
         (int64_t)n_out * (kRowsThreads / 32 + 1) * 8;
}
int launch_rows(const DevDirect& img, const float* X, int64_t n, int32_t d, const OutArgs& o,
                int32_t num_sms, void* stream);
int launch_count_visits(const DevDirect& img, const float* X, int64_t n, int32_t d,
                        uint32_t* counts, int32_t num_sms, void* stream);
int set_sliced_smem_limit(int32_t bytes);
// microbenchmarks (Algorithm 1 line 4): the coded walk on ideal data; raw shared-memory loads
int launch_visit_peak(int32_t variant, int32_t L, int32_t reps, int32_t grid, double* sink, void* stream);
int launch_smem_bw(int32_t iters, int32_t grid, unsigned long long* cycles, uint32_t* sink, void* stream);
int launch_visit_peak_direct(const void* nodes, int32_t steps, int32_t grid, double* sink, void* stream);

}  // namespace tahoe
