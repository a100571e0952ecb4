// internal.h — host-side definition of griffin_index and launcher prototypes.
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/griffin.h"
#include "griffin_dev.cuh"

namespace griffin {

void set_error(const std::string &msg);

#define GRIFFIN_CUDA_TRY(expr)                                                          \
  do {                                                                                   \
    cudaError_t _e = (expr);                                                             \
    if (_e != cudaSuccess) {                                                             \
      ::griffin::set_error(std::string(#expr) + ": " + cudaGetErrorString(_e));          \
      return _e == cudaErrorMemoryAllocation ? GRIFFIN_ERR_OOM : GRIFFIN_ERR_CUDA;        \
    }                                                                                    \
  } while (0)

// Device status bits (set by kernels, read by griffin_sync_status).
enum : int { kStatusBadTerm = 1, kStatusOverflow = 2, kStatusTooManyTerms = 4 };

// Query modes per (query, round).
enum : uint32_t { kModeNone = 0, kModeMerge = 1, kModeGallop = 2, kModeAll = 3, kModeProbe = 4,
                  kModeBitmap = 5, kModeBitAnd = 6 };
// word-AND units (both lists of a round-1 pair decoded into bitvectors): words per unit
constexpr uint32_t kAndWords = 512;
// Per-term batch decode-once kind (Workspace::tdec): not decoded, decoded into
// the docID arena, or decoded into a docID bitvector with rank (dense lists).
enum : uint8_t { kDecNone = 0, kDecArena = 1, kDecBitmap = 2 };

// Grow-only device buffer.
struct DevBuf {
  void *p = nullptr;
  size_t bytes = 0;
  cudaError_t reserve(size_t want) {
    if (want <= bytes) return cudaSuccess;
    if (p) cudaFree(p);
    p = nullptr;
    bytes = 0;
    // small buffers grow with 25% headroom (fewer re-allocations); large ones
    // (intermediates, arena, candidates: GBs at C5) are sized exactly
    size_t nb = want < (64ull << 20) ? want + want / 4 + 256 : want + 256;
    cudaError_t e = cudaMalloc(&p, nb);
    if (e == cudaSuccess) bytes = nb;
    return e;
  }
  void release() {
    if (p) cudaFree(p);
    p = nullptr;
    bytes = 0;
  }
  template <class T> T *as() const { return static_cast<T *>(p); }
};

// Query workspace (all grow-only; sized by griffin_reserve / the host API).
struct Workspace {
  DevBuf plan_terms, plan_m, cap, cap_off, rcount, rsel, qmode, unit_base;  // per query
  DevBuf unit_off, unit_cnt, unit_dst, urec, uperm;                         // per unit
  DevBuf rbuf0, rbuf1, bump, cand, tkstate;                                 // per survivor
  DevBuf flt, fstate;   // top-k sampled-threshold pre-filter: kept keys, per-query state
  DevBuf scal;       // scalars: counters, status, bump ctr, unit ctr
  DevBuf keys, counts, docids, scores, qoffs, qterms;  // host-API staging on device
  DevBuf demand, tdec, runs, run_base, vtmp, run_term; // per term / run (batch reuse)
  DevBuf arena;                                        // decoded lists, nblocks * B u32
  DevBuf bmap;                                         // decoded dense lists: bitvector + rank
  DevBuf qtau;                                         // per query: top-k key threshold (bitand_tau_kernel)
  DevBuf sbkt_cnt, sbkt_pos, sbkt_tmp;                 // S-locality unit order buckets
  size_t nq_cap = 0, unit_cap = 0, entry_cap = 0;
  // pinned host staging; a grown buffer's predecessors stay allocated until the
  // workspace is freed (zero-copy result views may still point into them)
  void *h_pinned = nullptr;
  size_t h_pinned_bytes = 0;
  std::vector<void *> old_pinned;
  // griffin_query_batch_submit/collect: the batch in flight on this workspace
  cudaEvent_t done = nullptr;
  cudaStream_t pend_stream = nullptr;
  uint32_t pend_nq = 0, pend_k = 0;
  size_t pend_out = 0;   // byte offset of the results in h_pinned
  // a submitted batch not yet collected; read by synchronous calls under the
  // index mutex, cleared by collect only after the results were read out
  std::atomic<bool> pending{false};
  bool results_valid = false;   // the last collect succeeded (griffin_query_batch_results)
};

// Offsets of the scalar block (u64 slots).
enum : int {
  kScalCounters = 0,  // 4 x u64: alg bytes, payload bytes, decoded postings, survivors
  kScalBump = 4,      // u64 bump counter
  kScalUnitCtr = 5,   // u32 unit ticket counter (in a u64 slot)
  kScalStatus = 6,    // int status
  kScalTotals = 7,    // u64 x2: sum cap, sum units (written by plan kernels)
  kScalDec = 10,      // 3 x u64: decode-once alg bytes, payload bytes, postings
  kScalPerm = 13,     // 2 x u64: unit order list head (merge units) / tail (the rest)
  kScalArena = 15,    // 2 x u64: decoded-arena postings read by intersect, their compressed bytes
  kScalDecC8d = 17,   // u64: decode-once compressed bytes read (payload + skip/meta)
  kScalRoundTot = 18, // u64: survivors of the current round (compaction scan total)
  kScalDiag = 19,     // 4 x u64 (counting mode): merge units, merged elements, gallop units, galloped elements
  kScalUnitCtr2 = 23, // u64 ticket counter of the round-1 gallop/single-term kernel
  kScalDiag2 = 24,    // 4 x u64 (counting mode): bitvector units, their R elements, word-AND units, their words
  kScalCount = 28
};

#ifndef GRIFFIN_BUMP_CHUNK
#define GRIFFIN_BUMP_CHUNK 1024
#endif
constexpr uint32_t kBumpChunk = GRIFFIN_BUMP_CHUNK;   // bump-area entries grabbed per warp atomic
constexpr uint32_t kBmBucketShift = 13;   // 8192 docs (2 KB of bitvector) per bucket

struct RoundArgs {
  uint32_t nq, round, D, T, Tdec;
  int forced_mode;
  int probe;
  int nextgeq;   // gallop into compressed S by EF NextGEQ (no block decode)
  int count;     // maintain the algorithmic-byte / postings counters (profiling)
  uint32_t pchunk;   // probe pass: survivors per unit (multiple of 32, <= B)
  const uint32_t *plan_terms;
  const uint32_t *plan_m;
  const uint32_t *cap;
  uint64_t *cap_off;      // per query, per buffer: region offset ([0,nq] rbuf0, [nq+1,2nq+1] rbuf1)
  const uint64_t *roff_prev;   // this round's input offsets (buffer (round-1)&1)
  uint64_t *roff_next;         // this round's output offsets (buffer round&1)
  uint32_t *rcount;
  uint8_t *rsel;
  uint32_t *qmode;
  uint64_t *unit_base;
  uint64_t *unit_off;
  uint32_t *unit_cnt;
  uint64_t unit_cap;
  const uint2 *rprev;
  uint2 *rnext;
  uint2 *bump;
  uint64_t entry_cap;
  uint64_t bump_cap;      // entries of the bump area (entry_cap + per-warp chunk slack)
  unsigned long long *scal;
  uint4 *urec;            // per unit: {q, i0|lu, j0, lo docID} (partition stage)
  uint4 *uperm;           // processing order of the units (merge units first, then the rest):
                          // {unit, query | mode << 29, R term, S term} (uperm_entry)
  uint32_t *sbkt_cnt;     // S-locality order: merge units per bucket of S blocks (or null)
  unsigned long long *sbkt_pos;   // bucket cursors (exclusive scan of sbkt_cnt)
  uint32_t sbkt_shift;    // bucket = global S block of the unit's start >> shift
  // bitvector units follow the merge buckets: bucket = sbkt_nm + S slot * sbkt_nbb
  // + (first R docID >> kBmBucketShift), so units probing the same bitvector
  // region run together (L2 reuse across queries)
  uint64_t sbkt_nm;
  uint32_t sbkt_nbb;
  const uint32_t *dec;    // batch decoded arena (global block * B + i), or null
  const uint8_t *tdec;    // per term: kDecArena / kDecBitmap this batch (else kDecNone)
  const uint2 *bm;        // bitvector area: slot s at bm + s * bm_words
  const uint32_t *bm_slot;   // per term: its bitvector slot (kNone: not eligible)
  uint32_t bm_words;      // words per bitvector = ceil(n_docs / 32)
  const uint64_t *qtau;   // per query: round-1 key threshold of 2-term word-AND queries (or null)
};

}  // namespace griffin

namespace griffin {
struct Cluster;
}

struct griffin_index {
  std::mutex mu;
  // multi-GPU handle (griffin_build_opts.num_gpus > 1): the shards and their
  // exchange state; every query call goes through multi.cu
  std::vector<griffin_index *> shards;
  griffin::Cluster *cl = nullptr;
  int device = 0;
  cudaStream_t stream = nullptr;
  // options
  uint32_t B = 128, T = 128, Tdec = 16, D = 8;
  double k1 = 1.2, bm25_b = 0.75;
  uint32_t shard = 0, nshards = 1, doc_base = 0, doc_end = 0, N = 0, V = 0;
  float k1p1 = 0.f;
  // device index
  griffin::TermInfo *d_terms = nullptr;
  uint32_t *d_first = nullptr;
  uint2 *d_meta = nullptr;
  uint4 *d_payload = nullptr;
  uint32_t *d_tfw = nullptr;
  float *d_norm = nullptr;
  uint64_t nblocks = 0, payload16 = 0, tf_words = 0, postings = 0;
  std::vector<griffin::TermInfo> h_terms;
  // query state
  griffin::Workspace ws;
  griffin::Workspace qws;   // griffin_query's CUDA-graph path (sized for one query)
  std::vector<griffin::Workspace *> extra_ws;  // griffin_workspace_create
  int mode = 0;
  int reuse = 2;
  // single-query CUDA graphs, keyed by (distinct terms, k, mode, workspace identity)
  struct QueryGraph {
    uint32_t mt, k;
    int mode;
    uint64_t ws_id;
    cudaGraphExec_t exec;
  };
  std::vector<QueryGraph> graphs;
  bool single_ws = false;
  int use_graphs = 1;
  int probe = 1;
  int nextgeq = 1;
  int topk_filter = 1;   // sampled-threshold pre-filter for large candidate sets
  int sorder = 1;   // merge units ordered by the S blocks they read (L2 reuse across queries)
  uint32_t sorder_shift = 6;
  uint32_t P = 0;   // probe chunk (0 = B)
  // dense lists decoded once per batch into a bitvector + rank (kDecBitmap):
  // eligible iff df_local * bm_inv >= n_docs (density >= 1 / bm_inv); 0 = off.
  // Slots are per eligible term (host-assigned when the knob changes).
  uint32_t bm_inv = 32, bm_slots_inv = 0, bm_nslots = 0;
  uint32_t *d_bm_slot = nullptr, *d_bm_term = nullptr;
  // batches of at least this many queries get the R7 subset top-k threshold
  uint32_t tau_min_queries = 4096;
  uint64_t entry_budget = 0;   // griffin_set_entry_budget: intermediate entries per workspace (0 = exact bound)
  int profiling = 0;   // bit 0: per-stage CUDA events, bit 1: algorithmic-byte counters
  griffin_profile prof{};
  std::vector<cudaEvent_t> ev_pool;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> pending;  // stage, events
  size_t ev_next = 0;
  uint64_t launch_count = 0;  // kernels launched by this handle (always on)

  griffin::DevIndex dev() const {
    griffin::DevIndex d;
    d.terms = d_terms;
    d.first = d_first;
    d.meta = d_meta;
    d.payload = d_payload;
    d.tfw = d_tfw;
    d.norm = d_norm;
    d.num_terms = V;
    d.doc_base = doc_base;
    d.n_docs = doc_end - doc_base;
    d.B = B;
    d.log2B = 0;
    d.k1p1 = k1p1;
    return d;
  }
};

namespace griffin {

// encode.cu
griffin_status encode_index(griffin_index *ix, const uint32_t *h_docids_local,
                            const uint32_t *h_tfs, const std::vector<uint64_t> &post_off);
// query.cu
griffin_status run_batch(griffin_index *ix, Workspace &w, uint32_t nq, const uint32_t *d_qoffs,
                         const uint32_t *d_terms, uint32_t max_terms, uint32_t k,
                         uint64_t *d_keys, uint32_t *d_counts, cudaStream_t st, bool final_topk,
                         int forced_mode);
griffin_status reserve_ws(griffin_index *ix, Workspace &w, uint32_t nq, uint64_t units,
                          uint64_t entries);
griffin_status reserve_topk(griffin_index *ix, Workspace &w, uint32_t nq, uint32_t k);
griffin_status launch_merge_topk(griffin_index *ix, uint32_t G, uint32_t nq, uint32_t k,
                                 const uint64_t *d_keys, const uint32_t *d_counts,
                                 uint64_t *d_out_keys, uint32_t *d_out_counts, cudaStream_t st);
griffin_status launch_keys_to_results(griffin_index *ix, uint32_t nq, uint32_t k,
                                      const uint64_t *d_keys, const uint32_t *d_counts,
                                      uint32_t *d_docids, float *d_scores, cudaStream_t st);
griffin_status launch_decode_list(griffin_index *ix, uint32_t term, uint32_t *d_out,
                                  cudaStream_t st);
griffin_status launch_decode_all(griffin_index *ix, unsigned long long *d_acc, cudaStream_t st);
// copies the final survivor docIDs (global) of query 0 after run_batch(final_topk=false)
griffin_status copy_final_docids(griffin_index *ix, uint32_t *h_out, uint64_t cap, uint64_t *count);
// per-query bounds used to size the workspace (same rule as the device plan kernel)
// probe-pass survivors per unit: the griffin_set_probe_chunk value, else B/2
// (>= 32): measured 4.5 % faster than B on the C2 batch (more, shorter units)
inline uint32_t probe_chunk(const griffin_index *ix) {
  return ix->P ? ix->P : (ix->B / 2 >= 32 ? ix->B / 2 : 32u);
}
void host_query_bounds(const griffin_index *ix, uint32_t *ts, uint32_t n, uint64_t *cap,
                       uint64_t *units);
griffin_status launch_merge_topk_peer(griffin_index *ix, uint32_t G, uint32_t nq, uint32_t k,
                                      const uint64_t *const *keys, const uint32_t *const *counts,
                                      uint64_t *d_out_keys, uint32_t *d_out_counts, cudaStream_t st);
// api.cu helpers used by multi.cu
griffin_status reserve_for(griffin_index *ix, Workspace &w, uint32_t nq, const uint32_t *qoffs,
                           const uint32_t *terms, uint32_t k, uint32_t *max_terms);
griffin_status ensure_pinned_ws(Workspace &w, size_t bytes);
// SM count of a device (cached).
int num_sms(int dev);
// Process-wide dynamic-smem attribute (grow-only) + cached occupancy of a kernel.
cudaError_t launch_config(const void *fn, int dev, size_t smem, int threads, int *per_sm);
// Host copy of results out of pinned staging: large copies (a C5 batch's
// 80 MB of docIDs + scores) are split over a few threads.
void par_memcpy(void *dst, const void *src, size_t bytes);
// multi.cu
griffin_status cluster_init(griffin_index *cx, int exchange);
void cluster_destroy(griffin_index *cx);
griffin_status cluster_query_batch(griffin_index *cx, uint32_t nq, const uint32_t *qoffs,
                                   const uint32_t *terms, uint32_t k, uint32_t *out_docids,
                                   float *out_scores, uint32_t *out_counts);
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

}  // namespace griffin
