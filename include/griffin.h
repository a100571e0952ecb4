/*
 * griffin.h — C ABI of the B200-native Griffin-GPU conjunctive query path.
 *
 * The path (Liu, Wang, Swanson, "Griffin", PPoPP'18; /root/reference/PAPER.md,
 * cited P:<line>):
 *   block-parallel Elias-Fano decode (§3.1.1, Alg. 1)
 *   -> SvS list intersection, merge-path partitioned (§3.1.2) or
 *      skip-pointer galloping for skewed lengths
 *   -> BM25 scoring of the survivors (§2.1.3)
 *   -> top-k selection (§3.1.3)
 * with docID-range sharding across GPUs (not in the paper).
 *
 * Conventions (all entry points):
 *  - No exceptions cross this boundary; every call returns a griffin_status.
 *    On failure no output is written and griffin_last_error() returns a
 *    thread-local message.
 *  - "host" pointers are ordinary CPU memory, borrowed for the duration of the
 *    call; the library keeps no input pointer after returning.
 *  - "device" pointers are CUDA global memory on the index's device; calls that
 *    take them are asynchronous on the given stream (cudaStream_t passed as
 *    void*; NULL = the legacy default stream).
 *  - One call at a time per index handle (calls are serialised by a mutex).
 *  - docIDs are uint32 in [0, num_docs), num_docs < 2^32 - 1; 0xFFFFFFFF is
 *    the "no result" sentinel.
 *  - Results are ordered by score descending, ties by docID ascending
 *    (SURVEY A16); slots [count, k) hold docID 0xFFFFFFFF and score -inf.
 *  - Scores are fp32 BM25 with k1/b from griffin_build_opts,
 *    idf_t = ln(1 + (N - df_t + 0.5)/(df_t + 0.5)) and
 *    w = idf_t * (tf*(k1+1)) / (tf + k1*((1-b) + b*dl/avgdl)), each term's w
 *    accumulated in (global df asc, termID asc) order.
 *
 * This header is the only interface between the product and its callers; it is
 * not shared with the test oracle (oracle/), which has its own.
 */
#ifndef GRIFFIN_H_
#define GRIFFIN_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GRIFFIN_MAX_TERMS 16   /* distinct terms per query */
#define GRIFFIN_MAX_K 4096     /* largest k accepted */
#define GRIFFIN_MAX_SHARDS 8

typedef struct griffin_index griffin_index; /* opaque; owns device memory + stream */

typedef enum {
  GRIFFIN_OK = 0,
  GRIFFIN_ERR_INVALID_ARG = 1, /* bad sizes, term >= V, k == 0 or > GRIFFIN_MAX_K, ... */
  GRIFFIN_ERR_UNSORTED = 2,    /* a list not strictly increasing or a docID >= N */
  GRIFFIN_ERR_OOM = 3,         /* device allocation failed / workspace too small */
  GRIFFIN_ERR_CUDA = 4,        /* CUDA runtime error (message in griffin_last_error) */
  GRIFFIN_ERR_NCCL = 5,        /* NCCL missing or a collective failed (multi-GPU handles) */
  GRIFFIN_ERR_UNSUPPORTED = 6  /* no CUDA device / not sm_100 */
} griffin_status;

/* Corpus in CSR form (host pointers).  Term t's postings are
 * docids[list_offsets[t] .. list_offsets[t+1]) with matching tfs; docIDs strictly
 * increasing and < num_docs; tfs >= 1 (the per-posting "document frequency" of
 * P:357-361 / P:1009-1010 read as term frequency), any value up to
 * 2^32-1, stored losslessly.  doc_lengths[num_docs] are the BM25 document lengths
 * (SURVEY A13); their sum must be > 0. */
typedef struct {
  uint32_t num_docs;
  uint32_t num_terms;
  const uint64_t *list_offsets; /* [num_terms + 1] */
  const uint32_t *docids;
  const uint32_t *tfs;
  const uint32_t *doc_lengths;  /* [num_docs] */
} griffin_corpus;

typedef struct {
  uint32_t block_size;   /* EF block length B: 64..512, multiple of 32; 0 -> 128 */
  double bm25_k1;        /* BM25 k1 (paper silent); <= 0 -> 1.2 */
  double bm25_b;         /* BM25 b; < 0 -> 0.75 */
  uint32_t gallop_ratio; /* T: a round gallops iff |S| > T*|R|; 0 -> max(4, block_size/8),
                            the B200 crossover measured in DESIGN.md (the paper's T = B) */
  int32_t device;        /* CUDA device ordinal to build on; < 0 -> current device */
  uint32_t shard_index;  /* docID-range shard g of num_shards */
  uint32_t num_shards;   /* 0 or 1 -> unsharded */
  uint32_t gallop_ratio_decoded; /* T for rounds whose S list was decoded once into the batch
                                    arena (griffin_set_reuse): galloping there costs ~log2(B)
                                    probes per R element instead of a block decode, so the
                                    crossover is lower; 0 -> max(4, block_size/8) */
  /* ---- one handle over several GPUs ----
   * num_gpus G > 1: the handle builds G docID-range shards itself (shard g owns
   * [g*ceil(N/G), min(N,(g+1)*ceil(N/G))), global N/df/avgdl/idf everywhere, so
   * each doc's score is bit-identical to the unsharded one) on devices[g]
   * (NULL -> 0..G-1), owns their streams and NCCL communicators, and
   * griffin_query / griffin_query_batch return the GLOBAL top-k: per-shard top-k
   * keys are exchanged and k-way merged on the devices (exact: keys are unique,
   * so a global top-k key is in its shard's top-k).  num_shards must then be 0/1.
   * INVALID_ARG if G > 8 or a device ordinal is >= the visible device count;
   * GRIFFIN_ERR_NCCL if an NCCL exchange is requested and NCCL (libnccl.so.2,
   * loaded at run time) is missing or fails.  Devices may repeat (several
   * shards on one GPU), which only the peer exchange supports. */
  uint32_t num_gpus;       /* 0/1 -> a single shard (unless exchange != 0) */
  const int32_t *devices;  /* [num_gpus] device ordinals, borrowed for the call; NULL -> 0..G-1 */
  int32_t exchange;        /* griffin_exchange: how per-shard top-k lists meet */
} griffin_build_opts;

/* Exchange of per-shard top-k lists for a multi-GPU handle.
 *  AUTO: PEER.  NCCL_ALLGATHER: ncclAllGather of every shard's keys/counts (one
 *  NCCL group, one communicator per device), then the k-way merge on device 0.
 *  PEER: one kernel on device 0 reads every shard's top-k runs in place over
 *  NVLink (cudaDeviceEnablePeerAccess; copied with cudaMemcpyPeerAsync when
 *  peer access is unavailable) and merges them — exchange and merge fused.
 *  NCCL_SLICED: query-sliced all-to-all (grouped ncclSend/ncclRecv): device r
 *  receives only the runs of query slice r and merges it (received bytes per
 *  device ~ Q*k*8 instead of (G-1)*Q*k*8).
 *  With num_gpus = 1, exchange != AUTO still builds a one-shard handle that runs
 *  the chosen exchange (a one-rank NCCL communicator for the NCCL modes). */
typedef enum {
  GRIFFIN_EXCHANGE_AUTO = 0,
  GRIFFIN_EXCHANGE_NCCL_ALLGATHER = 1,
  GRIFFIN_EXCHANGE_PEER = 2,
  GRIFFIN_EXCHANGE_NCCL_SLICED = 3
} griffin_exchange;

typedef struct {
  uint32_t shard_index, num_shards;
  uint32_t doc_base, doc_end;     /* this shard owns docIDs [doc_base, doc_end) */
  uint32_t block_size, num_terms;
  uint64_t num_postings;          /* postings stored in this shard */
  uint64_t num_blocks;
  uint64_t payload_bytes;         /* EF low+high streams incl. 16-B block padding */
  uint64_t skip_bytes;            /* per-block first[] + meta[] */
  uint64_t tf_bytes;              /* packed tf streams */
  uint64_t device_bytes;          /* everything the index holds on the device */
} griffin_stats;

/* Intersection mode for griffin_debug_intersect / griffin_set_mode. */
typedef enum { GRIFFIN_MODE_AUTO = 0, GRIFFIN_MODE_MERGE = 1, GRIFFIN_MODE_GALLOP = 2 } griffin_mode;

/* Per-stage device timings and algorithmic counters accumulated while
 * profiling is on (griffin_set_profiling).  Times are CUDA-event milliseconds on
 * the launching stream. */
typedef struct {
  double ms_plan, ms_intersect, ms_compact, ms_topk, ms_merge;
  uint64_t launches_intersect, launches_total;
  uint64_t alg_bytes;        /* bytes the intersect kernels must read + write:
                                compressed payload + 8-B skip/meta per block read, 4 B per
                                decoded-arena posting, 8 B per intermediate entry, 32 B per
                                arena probe sector, per survivor one 32-B sector per tf
                                gather + 4-B norm + 8-B entry written */
  uint64_t payload_bytes;    /* compressed EF bytes of the blocks the method had to read */
  uint64_t decoded_postings; /* postings of those blocks */
  uint64_t survivors;        /* (docID, score) pairs emitted by intersection rounds */
  /* batch decode-once stage (griffin_set_reuse): EF-decode of hot lists into HBM */
  double ms_decode;
  uint64_t launches_decode;
  uint64_t dec_alg_bytes;    /* compressed bytes + skip entries read, decoded u32 written */
  uint64_t dec_payload_bytes;
  uint64_t dec_postings;
  /* SURVEY §8(d) algorithmic bytes: as alg_bytes, but postings read from the
   * decode-once arena are charged at their blocks' compressed size (payload +
   * 8-B skip/meta) instead of 4 B each; dec_c8d_bytes = the compressed bytes
   * the decode-once kernel reads (its arena writes are not algorithmic). */
  uint64_t c8d_bytes;
  uint64_t dec_c8d_bytes;
  uint64_t arena_postings;   /* decoded-arena postings read by the intersect kernels */
  /* unit shapes (counters mode): merge units and the elements they merged (R+S
   * inside their docID ranges), gallop units and their R elements */
  uint64_t merge_units, merge_elems, gallop_units, gallop_elems;
  /* bitvector units (griffin_set_bitmap) and their R elements looked up;
   * word-AND units (both lists of a round-1 pair are bitvectors) and their words */
  uint64_t bitmap_units, bitmap_elems, bitand_units, bitand_words;
} griffin_profile;

/* ---- index ------------------------------------------------------------------
 * griffin_index_build ("compression ... occurs once ... offline";
 * P:537-552 EF; P:609-610 fixed-length partitioned EF; Fig. 2 P:216-220 skip
 * pointers).  Validates the corpus on the host, computes global BM25 statistics
 * in double (rounded once to f32), keeps this shard's docID range, and
 * Elias-Fano encodes every list into blocks of B postings ON THE DEVICE
 * (size pass -> scan -> write pass).  On success *out owns all device memory. */
griffin_status griffin_index_build(const griffin_corpus *corpus, const griffin_build_opts *opts,
                                   griffin_index **out);
void griffin_index_destroy(griffin_index *ix);
griffin_status griffin_index_stats(const griffin_index *ix, griffin_stats *out);

/* ---- queries (host buffers; synchronous) --------------------------------------
 * A conjunctive query returns the docs containing every term (P:228-231,
 * P:269-271), BM25-scored, top k.  Duplicate terms are deduplicated; a term with
 * an empty list gives count 0.  Output arrays: out_docids[k], out_scores[k]
 * (GLOBAL docIDs; for a sharded index, this shard's top-k only). */
griffin_status griffin_query(griffin_index *ix, const uint32_t *terms, uint32_t nterms,
                             uint32_t k, uint32_t *out_docids, float *out_scores,
                             uint32_t *out_count);

/* Batch of nq queries: query q is terms[query_offsets[q] .. query_offsets[q+1]).
 * Outputs [nq*k] docIDs/scores (row q at q*k) and [nq] counts.  The whole batch
 * runs as one launch per SvS round on the device. */
griffin_status griffin_query_batch(griffin_index *ix, uint32_t nq, const uint32_t *query_offsets,
                                   const uint32_t *terms, uint32_t k, uint32_t *out_docids,
                                   float *out_scores, uint32_t *out_counts);

/* ---- queries (device buffers; asynchronous on `stream`) ------------------------
 * Same computation with every input and output in device memory.  max_terms is
 * a host-side bound on terms per query (<= GRIFFIN_MAX_TERMS).  Outputs are the
 * unique 64-bit keys (f32 score bits << 32) | (0xFFFFFFFF - global docID),
 * sorted descending ([nq*k], 0 past count) and counts [nq].  Workspace must be
 * reserved first (griffin_reserve); overflow or a bad term is reported by
 * griffin_sync_status. */
griffin_status griffin_reserve(griffin_index *ix, uint32_t nq, const uint32_t *query_offsets,
                               const uint32_t *terms, uint32_t k);
griffin_status griffin_query_batch_device(griffin_index *ix, uint32_t nq,
                                          const uint32_t *d_query_offsets, const uint32_t *d_terms,
                                          uint32_t max_terms, uint32_t k, uint64_t *d_out_keys,
                                          uint32_t *d_out_counts, void *stream);
/* Synchronise the index's work and return (then clear) any device-side error. */
griffin_status griffin_sync_status(griffin_index *ix);

/* Additional query workspaces, so several batches can be in flight on different
 * streams at once (a serving engine overlapping batch i+1's planning/decode
 * with batch i's intersection rounds).  A workspace owns the per-batch device
 * buffers (plans, intermediates, the decode-once arena, top-k candidates); the
 * index data is shared read-only.  One call at a time per workspace. */
typedef struct griffin_workspace griffin_workspace;
griffin_status griffin_workspace_create(griffin_index *ix, griffin_workspace **out);
void griffin_workspace_destroy(griffin_index *ix, griffin_workspace *ws);
griffin_status griffin_workspace_reserve(griffin_index *ix, griffin_workspace *ws, uint32_t nq,
                                         const uint32_t *query_offsets, const uint32_t *terms,
                                         uint32_t k);
griffin_status griffin_query_batch_device_ws(griffin_index *ix, griffin_workspace *ws, uint32_t nq,
                                             const uint32_t *d_query_offsets,
                                             const uint32_t *d_terms, uint32_t max_terms,
                                             uint32_t k, uint64_t *d_out_keys,
                                             uint32_t *d_out_counts, void *stream);
griffin_status griffin_workspace_sync_status(griffin_index *ix, griffin_workspace *ws);

/* griffin_query_batch (host buffers, same arguments, validation and results)
 * split into an enqueue and a wait on one workspace, so a caller holding several
 * workspaces keeps several batches — H2D of the queries, the whole path, D2H of
 * the results — in flight on different streams.  submit validates the batch on
 * the host, copies query_offsets/terms into the workspace's pinned staging
 * (the caller's arrays may be reused as soon as it returns) and enqueues
 * everything on `stream` (NULL: the index's stream); it fails with
 * GRIFFIN_ERR_INVALID_ARG if the workspace still holds an uncollected batch.
 * collect waits for that batch and writes [nq*k] docIDs, [nq*k] scores and
 * [nq] counts exactly as griffin_query_batch does; a device-detected error
 * (workspace overflow, bad term) is returned here.  ws = NULL: the index's own
 * workspace (while it holds an uncollected batch, griffin_query,
 * griffin_query_batch and griffin_query_batch_device fail with
 * GRIFFIN_ERR_INVALID_ARG). */
griffin_status griffin_query_batch_submit(griffin_index *ix, griffin_workspace *ws, uint32_t nq,
                                          const uint32_t *query_offsets, const uint32_t *terms,
                                          uint32_t k, void *stream);
griffin_status griffin_query_batch_collect(griffin_index *ix, griffin_workspace *ws,
                                           uint32_t *out_docids, float *out_scores,
                                           uint32_t *out_counts);
/* Zero-copy read of the last collected batch: collect with all three outputs
 * NULL waits and checks status without copying; then this returns read-only
 * host pointers to the [nq*k] docIDs, [nq*k] scores and [nq] counts in the
 * workspace's pinned staging, valid until the next submit on that workspace
 * (for ws = NULL also until the next griffin_query / griffin_query_batch).
 * GRIFFIN_ERR_INVALID_ARG while a batch is still uncollected. */
griffin_status griffin_query_batch_results(griffin_index *ix, griffin_workspace *ws,
                                           const uint32_t **docids, const float **scores,
                                           const uint32_t **counts);

/* Shard merge: given G per-shard sorted key runs
 * d_keys[g][nq*k] and counts d_counts[g][nq] (laid out contiguously, g-major, as
 * an all-gather produces them), write the global top-k keys and counts.  Exact:
 * keys are unique, so a global top-k key is in its shard's top-k. */
griffin_status griffin_merge_topk_device(griffin_index *ix, uint32_t num_runs, uint32_t nq,
                                         uint32_t k, const uint64_t *d_keys,
                                         const uint32_t *d_counts, uint64_t *d_out_keys,
                                         uint32_t *d_out_counts, void *stream);
/* keys -> (docID, score) rows, sentinel-filled past count. */
griffin_status griffin_keys_to_results_device(griffin_index *ix, uint32_t nq, uint32_t k,
                                              const uint64_t *d_keys, const uint32_t *d_counts,
                                              uint32_t *d_docids, float *d_scores, void *stream);

/* ---- configuration / instrumentation ---------------------------------------- */
griffin_status griffin_set_mode(griffin_index *ix, int mode); /* griffin_mode; default AUTO */
/* Intermediate-result capacity of workspaces reserved from now on, in
 * (docID, score) entries per buffer.  0 (default): the exact bound, the sum over
 * the batch's queries of min(df of its two shortest lists) — never overflows,
 * but tens of GB for a 10K-query batch of frequent terms (C5).  A budget caps
 * it: survivors are packed into the intermediates by actual count (a device scan
 * per round), so the budget only has to hold what a batch really produces; a
 * batch that exceeds it reports GRIFFIN_ERR_OOM (griffin_sync_status / the host
 * calls) and writes no partial results. */
griffin_status griffin_set_entry_budget(griffin_index *ix, uint64_t entries);
/* 0 off; 1 per-stage CUDA events + algorithmic-byte counters; 2 events only
 * (kernel durations without the counting work); 3 counters only. */
griffin_status griffin_set_profiling(griffin_index *ix, int on);
/* Batch list reuse: 0 = off (every round decodes its blocks, fused), 1 = on,
 * 2 = auto (default; on for batches of >= 8 queries).  When on, lists whose
 * estimated block demand in the batch is >= 1.5x their block count are
 * EF-decoded once per batch into an HBM arena (the paper's decompress-then-
 * intersect pipeline, Alg. 1 output `decmp_array`) and intersected from there. */
griffin_status griffin_set_reuse(griffin_index *ix, int mode);
/* Dense lists in the decode-once stage: a list selected for decode-once whose
 * density in the shard is >= 1/inv (df_local * inv >= shard docs) is decoded
 * into a docID bitvector with rank — per 32 docs one u64 word {bits, position
 * of the word's first posting} — instead of the docID arena (for density >=
 * 1/32 it is the smaller of the two).  An intersection round whose longer
 * list S has one then looks each R element up in O(1) (bit test; the rank
 * gives the posting position for S's tf) instead of merging or galloping
 * through S: the SvS result set and every score are unchanged,
 * only the work differs.  Default inv = 32; 0 turns the bitvectors off.
 * Forced merge / gallop modes (griffin_set_mode) never use them. */
griffin_status griffin_set_bitmap(griffin_index *ix, uint32_t inv);
/* Galloping into a compressed (not arena-decoded) list: 1 = EF NextGEQ (default;
 * select0 over the staged block's unary high stream finds the bucket of the
 * probe's high part, only that bucket's few elements are decoded — SURVEY
 * §8(f) NEXT-1), 0 = decode every touched block (Para-EF) and binary-search it.
 * Results are identical; only the work differs.  Invalid value -> INVALID_ARG. */
griffin_status griffin_set_nextgeq(griffin_index *ix, int on);
/* Probe pass (SvS rounds 2..m-1, one multi-list pass over the round-1
 * survivors): survivors per work unit, a multiple of 32 in [32, block_size];
 * 0 restores the default (block_size / 2, at least 32).  Smaller chunks give more, shorter
 * units (more parallelism when few survivors remain).  Results are identical.
 * Invalid value -> INVALID_ARG. */
griffin_status griffin_set_probe_chunk(griffin_index *ix, uint32_t chunk);
griffin_status griffin_get_profile(griffin_index *ix, griffin_profile *out); /* syncs */
griffin_status griffin_reset_profile(griffin_index *ix);
const char *griffin_last_error(void);

/* docID range owned by shard g of G over num_docs docs: [g*ceil(N/G), min(N,(g+1)*ceil(N/G))).
 * Pure host function (no device needed). */
griffin_status griffin_shard_range(uint32_t num_docs, uint32_t num_shards, uint32_t shard,
                                   uint32_t *doc_base, uint32_t *doc_end);

/* Merge-path split of the diagonal d over sorted arrays a[na], b[nb] (host
 * reference of the device search; Fig. 6, rule "advance in A iff
 * A[i] <= B[j]", P:690-691 / SURVEY A8) with the matched-pair fix-up of SURVEY
 * A9 applied when fixup != 0.  Pure host function. */
griffin_status griffin_merge_path_split(const uint32_t *a, uint32_t na, const uint32_t *b,
                                        uint32_t nb, uint32_t diag, int fixup, uint32_t *i_out,
                                        uint32_t *j_out);

/* ---- test-only parity hooks (same conventions) ---------------------------------
 * Logical EF streams of block `blk` of term t in this shard (low stream of
 * n*b bits, high stream of L bits, LSB-first u32 words). */
griffin_status griffin_debug_block_streams(griffin_index *ix, uint32_t term, uint64_t blk,
                                           uint32_t *first, uint32_t *n, uint32_t *b,
                                           uint32_t *low, uint64_t low_cap, uint64_t *low_bits,
                                           uint32_t *high, uint64_t high_cap, uint64_t *high_bits);
/* Warp-parallel decode (Alg. 1) of term t's whole list in this shard -> GLOBAL docIDs. */
griffin_status griffin_debug_decode_list(griffin_index *ix, uint32_t term, uint32_t *out,
                                         uint64_t cap, uint64_t *n);
/* Decode-only bandwidth kernel over every block of the shard (decode sweep):
 * returns the device time in ms and writes the XOR of all decoded docIDs (so the
 * work cannot be elided) to *checksum. */
griffin_status griffin_debug_decode_all(griffin_index *ix, int iters, double *ms,
                                        uint64_t *checksum, uint64_t *postings, uint64_t *bytes);
/* Full docID set of the conjunctive query (GLOBAL docIDs), mode = griffin_mode. */
griffin_status griffin_debug_intersect(griffin_index *ix, const uint32_t *terms, uint32_t nterms,
                                       int mode, uint32_t *out_docids, uint64_t cap,
                                       uint64_t *count);

/* ---- PforDelta comparator codec -------------------------
 * The paper's comparison scheme (§2.1.1; Fig. 3), for
 * bits/posting and decode-throughput comparisons with the EF index (Table 1,
 * Fig. 12).  Not on the query path.  Same block layout rules as the
 * EF index: blocks of block_size docIDs, per block an 8-B skip entry {first
 * docID, payload offset / 16 B + packed n/words/b} and a 16-B aligned stream:
 *   word 0: first exception position (n-1 if none) | n_exc << 10 | b << 20,
 *   then n-1 d-gap slots of b bits (LSB-first; an exception's slot holds the
 *   distance to the next exception minus one, the last 0), then the n_exc
 *   exception gaps as u32, last exception first.  b = bits of the largest of the
 *   ceil(0.9 (n-1)) smallest gaps; exceptions more than 2^b apart force one in
 *   between (readings P1-P3).
 * griffin_pfd_build validates like griffin_index_build (GRIFFIN_ERR_UNSORTED,
 * INVALID_ARG) and encodes on `device` (-1 = current); the handle owns its
 * device memory, freed by griffin_pfd_destroy.  Calls are synchronous. */
typedef struct griffin_pfd griffin_pfd;
typedef struct {
  uint32_t block_size;
  uint64_t num_blocks, num_postings;
  uint64_t payload_bytes;   /* streams incl. 16-B padding */
  uint64_t skip_bytes;      /* 8 B per block */
  uint64_t exceptions;      /* exception slots, forced ones included */
} griffin_pfd_stats_t;
griffin_status griffin_pfd_build(const griffin_corpus *c, uint32_t block_size, int device,
                                 griffin_pfd **out);
void griffin_pfd_destroy(griffin_pfd *p);
griffin_status griffin_pfd_stats(const griffin_pfd *p, griffin_pfd_stats_t *out);
/* Logical stream words of block `block` of term `term` (host buffer of cap words). */
griffin_status griffin_pfd_block_stream(griffin_pfd *p, uint32_t term, uint32_t block,
                                        uint32_t *first, uint32_t *n, uint32_t *words,
                                        uint32_t cap, uint32_t *nwords);
/* Warp-per-block decode of term's whole list (host buffer of cap docIDs). */
griffin_status griffin_pfd_decode_list(griffin_pfd *p, uint32_t term, uint32_t *out,
                                       uint64_t cap, uint64_t *n);
/* Decode-only sweep over every block (as griffin_debug_decode_all): mean device
 * ms of `iters` timed sweeps after one warm-up, postings, bytes read (streams +
 * skip entries) and the XOR of all decoded docIDs. */
griffin_status griffin_pfd_decode_all(griffin_pfd *p, uint32_t iters, double *ms,
                                      uint64_t *postings, uint64_t *bytes, uint64_t *checksum);

#ifdef __cplusplus
}
#endif
#endif /* GRIFFIN_H_ */
