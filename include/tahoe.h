/*
 * include/tahoe.h — C ABI of the B200-native Tahoe forest-inference engine (libtahoe.so).
 *
 * The path (BASELINE.json north_star): for every (sample, tree) pair walk
 * root -> leaf by the node test "x_j < b_i", then combine the
 * per-tree leaf values per sample.  The calls follow the paper's Algorithm 1
 * (P:1360-1419): an online CPU step that rearranges nodes and trees once per forest
 * (tahoe_forest_layout, lines 5-7) and an online GPU step per batch that picks a strategy with a
 * cost model and launches it (tahoe_predict, lines 8-15).
 *
 * Conventions
 *  - Every symbol is extern "C"; no C++ exception crosses the boundary.  Every call returns a
 *    tahoe_status; tahoe_last_error() gives a thread-local message for the last failure.
 *  - Node arrays use GLOBAL node indices: tree t's root is root[t]; children index the same arrays.
 *  - X is row-major float32, n rows x d columns; sample i's attribute j is X[i*d + j].
 *  - Device pointers are raw CUDA device pointers on the forest's device; `stream` is a
 *    cudaStream_t (NULL = legacy default stream).  All GPU work is enqueued asynchronously; device
 *    faults surface at the caller's next synchronisation.
 *  - Results never depend on the layout: leaf ids are the caller's node ids and sums are fp64
 *    (reading Z17); with dyadic leaf values every output is bit-identical across layouts.
 *  - There is no CPU fallback: prediction runs only in this library's sm_100a kernels.
 */
#ifndef TAHOE_H
#define TAHOE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tahoe_forest tahoe_forest;   /* opaque; owns its host and device images */
typedef struct CUstream_st* tahoe_stream;   /* == cudaStream_t */

typedef enum {
  TAHOE_OK = 0,
  TAHOE_E_INVAL = 1,        /* invalid argument or invalid forest                          */
  TAHOE_E_NOMEM = 2,        /* host or device allocation failed                            */
  TAHOE_E_CUDA = 3,         /* CUDA runtime error (launch, copy, no device)                */
  TAHOE_E_UNSUPPORTED = 4,  /* valid input outside what the encoding supports              */
  TAHOE_E_STATE = 5         /* call not allowed in this handle state (e.g. host-only)     */
} tahoe_status;

/* How per-tree leaf values v(i,t) are combined per sample (north star; reading Z14). */
typedef enum {
  TAHOE_AGG_SUM = 0,        /* out[i]     = base + sum_t v(i,t)                                 */
  TAHOE_AGG_AVERAGE = 1,    /* out[i]     = base + (sum_t v(i,t)) / T        (fp64 divide)      */
  TAHOE_AGG_BINARY = 2,     /* out[i]     = base + sum_t v(i,t); class = out > 0 (fp64; 0 -> 0)  */
  TAHOE_AGG_CLASS_SUM = 3,  /* out[i*C+c] = base + sum_{t: class(t)=c} v(i,t); class = argmax,
                               ties -> lowest c                                               */
  TAHOE_AGG_VOTE = 4        /* out[i*C+c] = #{t : v(i,t) == c}; class = argmax, ties -> lowest */
} tahoe_agg;

/* Strategies (Algorithm 1 line 15, re-targeted to B200). */
typedef enum {
  TAHOE_STRATEGY_AUTO = -1,   /* cost model (Algorithm 1 lines 8-13)                          */
  TAHOE_STRATEGY_DIRECT = 0,  /* lane = sample; forest image in HBM/L2 (paper's "direct")     */
  TAHOE_STRATEGY_SLICED = 1,  /* lane = tree; forest slices resident in shared memory, sample
                                 tiles staged by TMA ("shared forest" / "splitting shared
                                 forest")                                        */
  TAHOE_STRATEGY_SLICED_CODED = 2, /* SLICED over exact rank codes of the attributes (DESIGN.md
                                 reading R7; same results bit for bit): a pre-pass turns each
                                 row into u16 codes, the slices compare codes with threshold
                                 ranks.  AUTO takes it instead of SLICED when the forest
                                 qualifies (<= 127 attributes, <= 32000 distinct thresholds per
                                 attribute, no subnormal leaf value); leaf ids and fingerprints
                                 come from the same walk's diagnostic instantiation; forcing it
                                 on a forest that does not qualify returns E_UNSUPPORTED.
                                 Forests over more than 127 attributes get the
                                 WIDE codes instead (reading R8): u8 codes over virtual
                                 attributes (<= 127 thresholds each), 2^V-byte code rows staged
                                 in shared memory next to slices packed for that room; they
                                 qualify while the used attributes need <= 4 KB rows and every
                                 tree fits the smaller lane column                            */
  TAHOE_STRATEGY_ROWS = 3     /* small batches (the paper's batch-100 workload
                                 P:1714-1717): one CTA per sample, lane = tree over the direct
                                 image, fixed-order block reduction and finalize in the same
                                 kernel (one launch, no scratch: CUDA-graph capturable).  Needs
                                 4 d + 4 n_trees + 512 bytes of shared memory (E_UNSUPPORTED
                                 when forced beyond that)                                     */
} tahoe_strategy;

/*
 * tahoe_forest_build — validate and copy a forest, encode it with the default layout (input tree
 * order, left child first), upload it to `device`.  Passage: P:181-192 (binary trees, node =
 * attribute index + threshold), P:397-399 (default path D).
 *
 *  n_trees, root[n_trees]      global index of each tree's root
 *  n_nodes                     length of the node arrays
 *  feature[n_nodes]            attribute index; < 0 marks a leaf
 *  threshold[n_nodes]          internal node: go LEFT iff x[feature] < threshold (IEEE fp32)
 *  left/right[n_nodes]         children (ignored for leaves)
 *  leaf_value[n_nodes]         leaf value (VOTE: the class id, an integer in [0, n_classes))
 *  default_left[n_nodes]|NULL  NaN goes left iff 1; NULL => NaN follows the comparison (right)
 *  tree_class[n_trees]|NULL    class of each tree for CLASS_SUM; NULL => t % n_classes
 *  n_features                  attributes per sample the forest may address (feature < it)
 *  n_classes                   1 for SUM/AVERAGE/BINARY; C >= 1 for CLASS_SUM/VOTE
 *  device                      CUDA device ordinal, or -1 for a HOST-ONLY handle (layout and
 *                              introspection only; prediction returns TAHOE_E_STATE)
 * Ownership: every array is copied; the caller keeps its buffers.  *out is owned by the caller
 * and released with tahoe_forest_free.
 * Errors: E_INVAL on n_trees < 1, n_classes < 1, a feature outside [0, n_features), a child
 * outside [0, n_nodes), a node reachable twice (shared or cyclic), a NaN threshold, tree_class
 * out of range, VOTE leaves that are not integers in [0, n_classes), NULL required pointers.
 * Unreachable nodes are ignored.  E_CUDA if `device` is not usable.
 */
tahoe_status tahoe_forest_build(int32_t n_trees, const int32_t* root, int32_t n_nodes,
                                const int32_t* feature, const float* threshold,
                                const int32_t* left, const int32_t* right,
                                const float* leaf_value, const uint8_t* default_left,
                                const int32_t* tree_class, int32_t n_features, int32_t n_classes,
                                tahoe_agg agg, float base_score, int32_t device,
                                tahoe_forest** out);

/* Layout options; zero fields take the paper's defaults T_nodes=4, L_hash=128, M=64.
 * node_reorder / tree_group: 1 = on (default), 0 = off (ablation switches, EX8).            */
typedef struct {
  int32_t t_nodes, l_hash, m_chunks;
  int32_t node_reorder, tree_group;
  int32_t _reserved;
  uint64_t seed;
} tahoe_layout_opts;

/*
 * tahoe_forest_layout — Algorithm 1 lines 5-7 on the host: count how many of the
 * n_calib calibration rows take each edge (edge / node probability), put the more
 * probable child of every node next to it (probability-based node rearrangement),
 * order trees by SimHash/LSH similarity and deal them into balanced work units
 * (expected-work packing, then a local search on the measured paths of up to 1024 of the rows,
 * reading R6), then re-encode and re-upload.  X_calib_host: HOST pointer, n_calib x d row-major
 * float32.
 * opts may be NULL (defaults).  Mutates the handle: must not overlap predictions on it.
 * Results of later predictions are unchanged bit for bit (leaf ids, classes; sums are fp64).
 */
tahoe_status tahoe_forest_layout(tahoe_forest* f, const float* X_calib_host, int64_t n_calib,
                                 int32_t d, const tahoe_layout_opts* opts);

/*
 * tahoe_count_visits — Algorithm 1 line 16, "Count edge probabilities during inference":
 * for every row of X (DEVICE, n x d) and every tree, add 1 to counts[k] for each node k the row's
 * path passes through (root and leaf included); k is the CALLER's node id.  counts: DEVICE
 * uint32[n_nodes] (the build's array length), accumulated (zero it first), not thread-safe against
 * concurrent layouts.  Edge probability (parent -> child) = counts[child] / counts[parent]
 * (P:399-406).  Errors as tahoe_predict.
 */
tahoe_status tahoe_count_visits(const tahoe_forest* f, const float* X, int64_t n, int32_t d,
                                uint32_t* counts, tahoe_stream stream);

/*
 * tahoe_forest_layout_counts — tahoe_forest_layout driven by visit counts measured elsewhere
 * (e.g. tahoe_count_visits on live traffic; re-layout for incremental updates).
 * counts: HOST uint64[n_nodes] by caller node id over n_calib rows.  X_sim_host (n_sim x d, may be
 * NULL; up to 1024 rows are kept) feeds the lockstep simulation of the cost model and the
 * measured-path balancing of lane columns (reading R6).
 */
tahoe_status tahoe_forest_layout_counts(tahoe_forest* f, const uint64_t* counts, int64_t n_calib,
                                        const float* X_sim_host, int64_t n_sim, int32_t d,
                                        const tahoe_layout_opts* opts);

/*
 * tahoe_predict — Algorithm 1 lines 8-15 per batch: cost model, launch.  X: DEVICE pointer
 * n x d row-major float32 (d >= largest attribute index used by the forest + 1; extra columns are
 * ignored); out: DEVICE float32 n x n_out (n_out = tahoe_forest_n_outputs).  n == 0 is a no-op.
 * Returns E_INVAL on a too-small d or NULL pointers with n > 0, E_STATE on a host-only handle,
 * E_CUDA on launch failure.
 * X and out are borrowed and must stay valid until the work enqueued on `stream` completes.
 * Concurrent predictions on one handle from several threads/streams are allowed.
 */
tahoe_status tahoe_predict(const tahoe_forest* f, const float* X, int64_t n, int32_t d,
                           float* out, tahoe_stream stream);

typedef struct {
  int32_t* out_class;         /* DEVICE int32[n] (BINARY / CLASS_SUM / VOTE), or NULL           */
  int32_t* out_leaf;          /* DEVICE int32[n*T]: leaf reached in tree t (caller's node id),
                                 caller's tree order, or NULL                                  */
  uint64_t* out_fingerprint;  /* DEVICE uint64[n]: sum_t mix64(((u64)t << 32) | leaf) mod 2^64,
                                 mix64 = splitmix64 finaliser, or NULL                         */
  int32_t force_strategy;     /* tahoe_strategy; -1 = cost model                                */
  int32_t _reserved;
  void* ev_main_begin;        /* cudaEvent_t or NULL: recorded on `stream` right before / after  */
  void* ev_main_end;          /*   the main traversal kernel (bench-side kernel timing)          */
} tahoe_predict_opts;

/* tahoe_predict with optional class / leaf / fingerprint outputs and a forced strategy. */
tahoe_status tahoe_predict_ex(const tahoe_forest* f, const float* X, int64_t n, int32_t d,
                              float* out, const tahoe_predict_opts* opts, tahoe_stream stream);

/*
 * tahoe_predict_host — the end-to-end call with HOST buffers: X_host (n x d float32), out_host
 * (n x n_out float32) and class_host (int32[n] or NULL) are host pointers (pinned memory gives
 * overlapped copies).  The batch is cut into chunks; host->device copies, prediction and
 * device->host copies of consecutive chunks overlap on internal streams; `stream` is made to
 * wait for all of it, so events recorded on `stream` bracket the whole transfer + compute.
 * The host buffers must stay valid until `stream` reaches that point.
 */
tahoe_status tahoe_predict_host(const tahoe_forest* f, const float* X_host, int64_t n, int32_t d,
                                float* out_host, int32_t* class_host, tahoe_stream stream);

/*
 * tahoe_forest_l2_persist — low-latency serving (the paper's batch-100 workload,
 * P:1714-1717): mark the forest image the strategy reads as an L2-persisting access-policy window
 * on `stream` (hit_ratio in (0, 1]; 0 removes the window), so small batches do not re-fetch it
 * from HBM between calls.  Mutates the stream's attributes and the device's persisting-L2 limit.
 */
tahoe_status tahoe_forest_l2_persist(const tahoe_forest* f, tahoe_stream stream, float hit_ratio);

/*
 * tahoe_forest_layout_export / _import — the layout state of a handle (calibration counts, hot
 * children, expected reads, tree order, the kept simulation rows, the options) as an opaque byte
 * blob, so one rank lays a forest out (Algorithm 1 lines 5-7) and the others apply the result to
 * their own build of the same node arrays (e.g. before tahoe_forest_shard) instead of repeating
 * it.  export: *size = blob bytes; buf may be NULL (size query), else cap >= *size (E_INVAL
 * otherwise).  import: E_INVAL unless the blob came from a forest with the same trees and nodes;
 * then re-encodes and re-uploads the images (must not overlap predictions on the handle).
 */
tahoe_status tahoe_forest_layout_export(const tahoe_forest* f, void* buf, int64_t cap, int64_t* size);
tahoe_status tahoe_forest_layout_import(tahoe_forest* f, const void* buf, int64_t size);

/* ---------------- hardware parameters (Algorithm 1 line 4) ---------------- */

/*
 * tahoe_measure_visit_rate — "Measure hardware parameters by a microbenchmark" (Algorithm 1 line
 * 4), re-targeted to the walk's bound (DESIGN.md §5 Roofline): the node-read rate of
 * the production coded walk on ideal data (every lane walks `steps` internal nodes of its own
 * column, perfect lockstep, conflict-free code loads, no tile traffic), one 1024-thread CTA per SM
 * on all SMs of `device`, `reps` walks per lane.  variant 0: u16 codes, two chains per lane (the
 * walk of the rank-coded slices); variant 1: u8 codes, four chains per lane (the wide codes);
 * variant 2: the direct walk (8-byte nodes through L1 by __ldg, attributes from staged rows, hot
 * child next, eight threads per row, 4 CTAs of 512 threads per SM) over a 32 KB node array that
 * stays L1-resident: steps x reps node reads per thread.
 * Writes *node_reads_per_s (node reads = visits, leaf reads included, per second); optionally
 * *smem_bytes_per_clk (NULL to skip): conflict-free 16-byte shared-memory loads measured with
 * clock64, bytes per SM clock.  E_INVAL on a bad variant / steps < 2 / odd steps (variant 0: steps
 * not a multiple of 4; variant 1: of 8) / reps < 1;
 * E_CUDA on launch failure.  Synchronous (own stream).
 */
tahoe_status tahoe_measure_visit_rate(int32_t device, int32_t variant, int32_t steps, int32_t reps,
                                      double* node_reads_per_s, double* smem_bytes_per_clk);

/*
 * tahoe_profile_walk — load-balance measurement (Table 3 "A.C.V.", the
 * coefficient of variation of execution time across threads, Fig. 2(c)):
 * predicts X (device, n x d) with the u16 rank-coded slices through an instrumented copy of their
 * walk that reads the SM clock every iteration, writing out (device, n x n_out) as tahoe_predict
 * does and stats[8] (HOST doubles):
 *   stats[0] / stats[2]  mean over work units of the CV of the 32 lanes' walk spans,
 *   stats[1] / stats[2]  mean over work units of mean/max lane span (lockstep efficiency),
 *   stats[3] / stats[2]  mean lane span in SM cycles,
 *   stats[4] / stats[5]  mean over warps of the CV of the lanes' total spans over the launch.
 * E_UNSUPPORTED unless the forest has the u16 coded slices; synchronous (waits on `stream`).
 */
tahoe_status tahoe_profile_walk(const tahoe_forest* f, const float* X, int64_t n, int32_t d,
                                float* out, double* stats, tahoe_stream stream);

/* ---------------- tree sharding (multi-GPU) ---------------- */

/* Sub-forest of the trees assigned to `rank` of `world` (balanced by expected visits per tree,
 * deterministic), encoded and uploaded to `device` (-1 = host-only).  The shard keeps the full
 * forest's layout decisions.  Caller frees *shard. */
tahoe_status tahoe_forest_shard(const tahoe_forest* f, int32_t rank, int32_t world,
                                int32_t device, tahoe_forest** shard);

/* Raw fp64 sums of the shard's trees, DEVICE partial[n * n_out] (no base, no average, no argmax;
 * VOTE: vote counts).  Summing the partials of all shards (e.g. NCCL reduce) and finalising with
 * the full forest reproduces tahoe_predict. */
tahoe_status tahoe_predict_partial(const tahoe_forest* shard, const float* X, int64_t n, int32_t d,
                                   double* partial, tahoe_stream stream);

/* out[n * n_out] (+ out_class[n] or NULL) from summed raw partials, using the FULL forest's
 * aggregation, base score and tree count. */
tahoe_status tahoe_finalize(const tahoe_forest* full, const double* partial, int64_t n,
                            float* out, int32_t* out_class, tahoe_stream stream);

/* ---------------- fused cross-GPU reduce (tree sharding over NVLink) ----------
 * The paper scales the path over GPUs.  When the forest is split by trees
 * (tahoe_forest_shard), every rank holds the SAME rows and computes the raw fp64 sums of its own
 * trees; tahoe_predict_reduce writes them straight into an NCCL symmetric-memory window and ONE
 * kernel then (1) meets the same CTA of every peer at an LSA barrier (NCCL device API), (2) loads
 * the peers' partials of its rows over NVLink, sums them in rank order 0..world-1 (fixed order:
 * identical bits on every rank that finalises a row) and applies the full forest's aggregation as
 * tahoe_finalize does, (3) passes a second barrier before any rank may reuse its window.  No
 * separate ncclReduce and no separate finalize launch.
 *
 * NCCL >= 2.28 (device API) is loaded at run time with dlopen: the copy already loaded in the
 * process (torch's) is used, else $TAHOE_NCCL_LIB, else "libnccl.so.2" from the loader path.  The
 * rest of libtahoe.so never needs NCCL; without it these calls return TAHOE_E_UNSUPPORTED.  All
 * ranks must be load/store-reachable (one NVLink domain), else TAHOE_E_UNSUPPORTED at init. */
typedef struct tahoe_comm tahoe_comm;
#define TAHOE_COMM_ID_BYTES 128
enum tahoe_reduce_mode {
  TAHOE_REDUCE_SCATTER = 0,   /* rank r finalises rows [n*r/world, n*(r+1)/world)             */
  TAHOE_REDUCE_ALL = 1        /* every rank finalises all n rows                               */
};

/* A fresh communicator id (ncclGetUniqueId) on one rank; the caller broadcasts the 128 bytes. */
tahoe_status tahoe_comm_unique_id(uint8_t id[TAHOE_COMM_ID_BYTES]);

/* Collective over `world` processes, one per GPU: ncclCommInitRank on `device`, plus a device
 * communicator with one LSA barrier per SM.  *comm is owned by the caller (tahoe_comm_free).
 * Environment TAHOE_REDUCE_NVLS=1 (world > 1): the device communicator also maps the window's
 * NVLS multicast address and tahoe_predict_reduce sums the ranks' partials in the switch
 * (multimem.ld_reduce; addition order unspecified, within reading Z17's fp64 bound); where
 * multicast is unavailable the peer-load kernel (rank-order sum, reading R5) is used. */
tahoe_status tahoe_comm_init(const uint8_t id[TAHOE_COMM_ID_BYTES], int32_t world, int32_t rank,
                             int32_t device, tahoe_comm** comm);
void tahoe_comm_free(tahoe_comm* comm);   /* synchronises the device first; NULL is a no-op     */

/* Rows [*lo, *hi) that `rank` finalises under `mode` (host arithmetic, no GPU). */
tahoe_status tahoe_reduce_rows(int64_t n, int32_t world, int32_t rank, int32_t mode, int64_t* lo,
                               int64_t* hi);

/* Collective: every rank calls it with the same n, d and mode and its own shard of the forest
 * (tahoe_forest_shard(full, rank, world, device)); a shard carries the full forest's aggregation,
 * base score and tree count.  X: DEVICE [n x d] fp32, the same rows on every rank.  out: DEVICE [(hi-lo) x n_out] fp32 and out_class [(hi-lo)] (or NULL) for this rank's
 * rows [lo, hi) (tahoe_reduce_rows).  Stream-ordered; the window grows (collectively) on the first
 * call with a larger n, which synchronises the device. */
tahoe_status tahoe_predict_reduce(const tahoe_forest* shard, tahoe_comm* comm, const float* X,
                                  int64_t n, int32_t d, int32_t mode, float* out,
                                  int32_t* out_class, tahoe_stream stream);

/* The same fused sum + finalisation over caller-provided partials, with the aggregation of `full`
 * (the full forest or any of its shards): partials is a HOST array of `world` DEVICE pointers to
 * fp64 [n x n_out] partial sums (tahoe_predict_partial), each readable from full's device (same device, peer access or CUDA-IPC mappings); the caller orders the
 * producers before this call.  out / out_class as in tahoe_predict_reduce.  world <= 64. */
tahoe_status tahoe_reduce_partials(const tahoe_forest* full, const double* const* partials,
                                   int32_t world, int32_t rank, int32_t mode, int64_t n,
                                   float* out, int32_t* out_class, tahoe_stream stream);

/* ---------------- queries ---------------- */
int32_t tahoe_forest_n_outputs(const tahoe_forest* f);   /* 1 or n_classes; -1 on NULL        */
int32_t tahoe_forest_n_trees(const tahoe_forest* f);
/* JSON object with realised forest and layout statistics (nodes, leaves, depths, expected
 * visits per sample, encoded bytes, slices, chosen strategy for a batch size, ...). */
tahoe_status tahoe_forest_stats(const tahoe_forest* f, char* buf, int64_t buf_len);
/* Strategy the cost model picks for a batch of n rows of width d (Algorithm 1 lines 8-13). */
int32_t tahoe_select_strategy(const tahoe_forest* f, int64_t n, int32_t d);
/* The cost model's predicted time (microseconds) of `strategy` for a batch of n rows; +inf when the
 * strategy is unavailable for this forest, -1 on NULL.  Constants: costmodel_b200.json next to the
 * library (fitted by scripts/fit_costmodel.py) or $TAHOE_COSTMODEL. */
double tahoe_predict_cost_us(const tahoe_forest* f, int32_t strategy, int64_t n);
void tahoe_forest_free(tahoe_forest* f);                  /* synchronise in-flight work first  */
const char* tahoe_last_error(void);                       /* thread-local, never NULL          */

/* ---------------- layout introspection (host-only; used by tests, no GPU needed) ----------- */

/* Per ORIGINAL node: calibration visit count and hot_is_left (1 = left child stays next to the
 * node); per tree: expected nodes read per sample; the similarity tree order.  Any pointer may be
 * NULL.  Arrays: count[n_nodes], hot_left[n_nodes], exp_reads[n_trees], order[n_trees]. */
tahoe_status tahoe_forest_layout_info(const tahoe_forest* f, uint64_t* count, uint8_t* hot_left,
                                      double* exp_reads, int32_t* order);

/* Tokens of tree t (reading Z6): windows of t_nodes caller node ids (-1 padded), each with the
 * node probability of its last node; ordered by last node in hot-first preorder.  Writes at most
 * cap tokens and sets *n_tokens to the total. */
tahoe_status tahoe_tree_tokens(const tahoe_forest* f, int32_t t, int32_t t_nodes,
                               int32_t* token_nodes, double* weights, int32_t cap,
                               int32_t* n_tokens);

/* The L_hash-bit SimHash of tree t: checksum[l_hash] and normalised bits[l_hash]. */
tahoe_status tahoe_tree_simhash(const tahoe_forest* f, int32_t t, int32_t t_nodes, int32_t l_hash,
                                double* checksum, uint8_t* bits);

/* Pure SimHash of given +-1 strings (n_str x l_hash int8) and weights. */
tahoe_status tahoe_simhash(const int8_t* strings, const double* weights, int32_t n_str,
                           int32_t l_hash, double* checksum, uint8_t* bits);

/* LSH: bits[n_trees x l_hash] -> collisions[n_trees x n_trees] (or NULL) and the
 * greedy similarity order[n_trees] (reading Z11). */
tahoe_status tahoe_lsh_order(const uint8_t* bits, int32_t n_trees, int32_t l_hash,
                             int32_t m_chunks, int32_t* collisions, int32_t* order);

/* SHA1 digest (FIPS 180-4) used by tokenisation. */
tahoe_status tahoe_sha1(const uint8_t* msg, int64_t len, uint8_t digest[20]);

/* Export of the encoded SLICED image for host-side decoding in tests (C = lane columns = 16):
 *   header[0..7] = {n_slices, slots_max, feature_bits, n_trees, n_classes, C, slot_bytes, 0}
 *   slice_info[n_slices*4] = {slots, class, n_trees_in_slice, 0}
 *   col_len[n_slices*C], nodes[n_slices*slots_max*C] (uint2 as uint32 pairs),
 *   leaf_meta[n_slices*slots_max*C*2] = {caller tree index, caller node id} at leaf slots.
 * Any array pointer may be NULL (then only header is filled). */
tahoe_status tahoe_forest_export_sliced(const tahoe_forest* f, int32_t* header,
                                        int32_t* slice_info, int32_t* col_len, uint32_t* nodes,
                                        int32_t* leaf_meta);

#ifdef __cplusplus
}
#endif
#endif /* TAHOE_H */
