// api.cu — the C ABI of include/griffin.h: host-side validation, global BM25
// statistics, docID-range sharding, workspace management and the synchronous
// host-buffer entry points.  Every step of the query path itself runs in the
// kernels of encode.cu / query.cu; nothing here computes query results.
#include <cstdlib>
#include <algorithm>
#include <cmath>
#include <cstring>
#include <string>
#include <thread>
#include <vector>

#include "internal.h"

namespace griffin {

static thread_local std::string g_err;
void set_error(const std::string &msg) { g_err = msg; }


void par_memcpy(void *dst, const void *src, size_t bytes) {
  constexpr size_t kSplit = 4u << 20;   // below this, one thread
  const unsigned hw = std::max(1u, std::thread::hardware_concurrency());
  const size_t nt = std::min<size_t>(std::min<size_t>(8, hw), bytes / kSplit);
  if (nt <= 1) {
    std::memcpy(dst, src, bytes);
    return;
  }
  const size_t per = (bytes / nt + 63) & ~size_t(63);
  std::vector<std::thread> th;
  for (size_t t = 1; t < nt; ++t) {
    const size_t a = t * per;
    if (a >= bytes) break;
    th.emplace_back([=] {
      std::memcpy(static_cast<uint8_t *>(dst) + a, static_cast<const uint8_t *>(src) + a,
                  std::min(per, bytes - a));
    });
  }
  std::memcpy(dst, src, std::min(per, bytes));
  for (auto &t : th) t.join();
}

static griffin_status invalid(const std::string &m) {
  set_error(m);
  return GRIFFIN_ERR_INVALID_ARG;
}

static griffin_status multi_unsupported() {
  set_error("not available on a multi-GPU handle (num_gpus > 1): use griffin_query / griffin_query_batch");
  return GRIFFIN_ERR_UNSUPPORTED;
}

griffin_status ensure_pinned_ws(Workspace &w, size_t bytes) {
  if (w.h_pinned_bytes >= bytes) return GRIFFIN_OK;
  if (w.h_pinned) w.old_pinned.push_back(w.h_pinned);   // freed with the workspace
  w.h_pinned = nullptr;
  w.h_pinned_bytes = 0;
  size_t nb = bytes + bytes / 4 + 4096;
  GRIFFIN_CUDA_TRY(cudaMallocHost(&w.h_pinned, nb));
  w.h_pinned_bytes = nb;
  return GRIFFIN_OK;
}
static griffin_status ensure_pinned(griffin_index *ix, size_t bytes) {
  return ensure_pinned_ws(ix->ws, bytes);
}

// Host validation of one batch's query terms + workspace reservation.
griffin_status reserve_for(griffin_index *ix, Workspace &w, uint32_t nq,
                           const uint32_t *qoffs, const uint32_t *terms, uint32_t k,
                           uint32_t *max_terms) {
  if (k == 0 || k > GRIFFIN_MAX_K) return invalid("k must be in [1, 4096]");
  uint64_t caps = 0, units = 0;
  uint32_t mt = 1;
  for (uint32_t q = 0; q < nq; ++q) {
    if (qoffs[q + 1] < qoffs[q]) return invalid("query_offsets must be non-decreasing");
    const uint32_t n = qoffs[q + 1] - qoffs[q];
    if (n == 0) return invalid("a query has no terms");
    // distinct terms without heap allocation (<= GRIFFIN_MAX_TERMS are valid)
    uint32_t ts[GRIFFIN_MAX_TERMS];
    uint32_t nd = 0;
    for (const uint32_t *p = terms + qoffs[q], *e = terms + qoffs[q + 1]; p < e; ++p) {
      const uint32_t t = *p;
      if (t >= ix->V) return invalid("query term >= num_terms");
      bool dup = false;
      for (uint32_t i = 0; i < nd; ++i) dup |= ts[i] == t;
      if (dup) continue;
      if (nd == GRIFFIN_MAX_TERMS) return invalid("more than GRIFFIN_MAX_TERMS distinct terms");
      ts[nd++] = t;
    }
    mt = std::max<uint32_t>(mt, nd);
    uint64_t c, u;
    host_query_bounds(ix, ts, nd, &c, &u);
    caps += c;
    units += u;
  }
  if (max_terms) *max_terms = mt;
  return reserve_ws(ix, w, nq, units, caps);
}

static griffin_status read_status(griffin_index *ix, Workspace &w, cudaStream_t st = nullptr) {
  if (!st) st = ix->stream;
  int status = 0;
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(&status, w.scal.as<unsigned long long>() + kScalStatus,
                                   sizeof(int), cudaMemcpyDeviceToHost, st));
  GRIFFIN_CUDA_TRY(cudaStreamSynchronize(st));
  if (status) {
    GRIFFIN_CUDA_TRY(cudaMemsetAsync(w.scal.as<unsigned long long>() + kScalStatus, 0, 8, st));
    GRIFFIN_CUDA_TRY(cudaStreamSynchronize(st));
    if (status & kStatusOverflow) {
      set_error("query workspace overflow (reserve more with griffin_reserve)");
      return GRIFFIN_ERR_OOM;
    }
    set_error("invalid query term(s) detected on the device");
    return GRIFFIN_ERR_INVALID_ARG;
  }
  return GRIFFIN_OK;
}

}  // namespace griffin

using namespace griffin;

extern "C" {

const char *griffin_last_error(void) { return g_err.c_str(); }

griffin_status griffin_shard_range(uint32_t num_docs, uint32_t num_shards, uint32_t shard,
                                   uint32_t *doc_base, uint32_t *doc_end) {
  if (num_shards == 0 || num_shards > GRIFFIN_MAX_SHARDS || shard >= num_shards || !doc_base ||
      !doc_end)
    return invalid("bad shard arguments");
  const uint64_t per = ((uint64_t)num_docs + num_shards - 1) / num_shards;
  *doc_base = (uint32_t)std::min<uint64_t>((uint64_t)shard * per, num_docs);
  *doc_end = (uint32_t)std::min<uint64_t>((uint64_t)(shard + 1) * per, num_docs);
  return GRIFFIN_OK;
}

griffin_status griffin_merge_path_split(const uint32_t *a, uint32_t na, const uint32_t *b,
                                        uint32_t nb, uint32_t diag, int fixup, uint32_t *i_out,
                                        uint32_t *j_out) {
  if ((!a && na) || (!b && nb) || diag > na + nb || !i_out || !j_out)
    return invalid("bad merge-path arguments");
  merge_path_split([&](uint32_t i) { return a[i]; }, na, [&](uint32_t j) { return b[j]; }, nb,
                   diag, fixup != 0, i_out, j_out);
  return GRIFFIN_OK;
}

// Host validation of a corpus (once per build, also for G shards).
static griffin_status validate_corpus(const griffin_corpus *c, uint64_t *sum_dl_out) {
  const uint32_t N = c->num_docs, V = c->num_terms;
  if (N == 0 || N >= 0xFFFFFFFFu) return invalid("num_docs must be in [1, 2^32-2]");
  if (!c->list_offsets || !c->doc_lengths) return invalid("null corpus arrays");
  if (c->list_offsets[0] != 0) return invalid("list_offsets[0] must be 0");
  for (uint32_t t = 0; t < V; ++t)
    if (c->list_offsets[t + 1] < c->list_offsets[t]) return invalid("list_offsets not monotone");
  const uint64_t P = c->list_offsets[V];
  if (P && (!c->docids || !c->tfs)) return invalid("null docids/tfs");
  for (uint32_t t = 0; t < V; ++t) {
    const uint64_t a = c->list_offsets[t], e = c->list_offsets[t + 1];
    if (e - a > 0xFFFFFFFFull) return invalid("list longer than 2^32-1");
    for (uint64_t p = a; p < e; ++p) {
      if (c->docids[p] >= N || (p > a && c->docids[p] <= c->docids[p - 1])) {
        set_error("list " + std::to_string(t) + " not strictly increasing or docID >= num_docs");
        return GRIFFIN_ERR_UNSORTED;
      }
      if (c->tfs[p] == 0) return invalid("tf must be >= 1");
    }
  }
  uint64_t sum_dl = 0;
  for (uint32_t d = 0; d < N; ++d) sum_dl += c->doc_lengths[d];
  if (sum_dl == 0) return invalid("sum of doc_lengths must be > 0");
  *sum_dl_out = sum_dl;
  return GRIFFIN_OK;
}

static griffin_status check_device(int dev) {
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    set_error("no CUDA device");
    return GRIFFIN_ERR_UNSUPPORTED;
  }
  if (dev < 0 || dev >= ndev) return invalid("device ordinal out of range");
  cudaDeviceProp prop;
  GRIFFIN_CUDA_TRY(cudaGetDeviceProperties(&prop, dev));
  if (prop.major != 10 || prop.minor != 0) {
    set_error("this build targets sm_100a (B200); device is sm_" + std::to_string(prop.major) +
              std::to_string(prop.minor));
    return GRIFFIN_ERR_UNSUPPORTED;
  }
  return GRIFFIN_OK;
}

// One docID-range shard (g of G) of a validated corpus on device `dev`.
static griffin_status build_shard(const griffin_corpus *c, const griffin_build_opts &opts,
                                  uint64_t sum_dl, uint32_t G, uint32_t g, int dev,
                                  griffin_index **out) {
  const uint32_t B = opts.block_size ? opts.block_size : 128;
  const double k1 = opts.bm25_k1 > 0 ? opts.bm25_k1 : 1.2;
  const double bb = opts.bm25_b >= 0 ? opts.bm25_b : 0.75;
  const uint32_t N = c->num_docs, V = c->num_terms;
  DeviceGuard guard(dev);
  griffin_index *ix = new griffin_index();
  ix->device = dev;
  ix->B = B;
  // B200 crossover measured at batch scale (tools/bench_configs.py c3, profiles/r01_c3_crossover.jsonl):
  // galloping already wins from lambda ~ 16 for B = 128, fused or arena; the paper's 128 (= B) was the
  // K20-vs-CPU crossover
  ix->T = opts.gallop_ratio ? opts.gallop_ratio : std::max<uint32_t>(4, B / 8);
  ix->Tdec = opts.gallop_ratio_decoded ? opts.gallop_ratio_decoded : std::max<uint32_t>(4, B / 8);
  ix->D = std::max<uint32_t>(2, 1024 / B);
  if (const char *e = std::getenv("GRIFFIN_TUNE_D")) ix->D = std::max<uint32_t>(2, (uint32_t)std::atoi(e));  // A/B probes
  if (const char *e = std::getenv("GRIFFIN_TOPK_FILTER")) ix->topk_filter = std::atoi(e);  // A/B
  if (const char *e = std::getenv("GRIFFIN_TDEC")) ix->Tdec = std::max(1, std::atoi(e));  // A/B
  if (const char *e = std::getenv("GRIFFIN_T")) ix->T = std::max(1, std::atoi(e));        // A/B
  if (const char *e = std::getenv("GRIFFIN_TAU_MIN_QUERIES")) ix->tau_min_queries = (uint32_t)std::atoi(e);  // tests / A/B
  if (const char *e = std::getenv("GRIFFIN_SORDER")) {   // A/B probes: 0 = off, else 1 + shift
    const int v = std::atoi(e);
    ix->sorder = v > 0;
    if (v > 0) ix->sorder_shift = (uint32_t)(v - 1);
  }
  ix->k1 = k1;
  ix->bm25_b = bb;
  ix->N = N;
  ix->V = V;
  ix->shard = g;
  ix->nshards = G;
  griffin_shard_range(N, G, g, &ix->doc_base, &ix->doc_end);
  ix->k1p1 = (float)(k1 + 1.0);
  if (cudaStreamCreateWithFlags(&ix->stream, cudaStreamNonBlocking) != cudaSuccess) {
    delete ix;
    set_error("cudaStreamCreate failed");
    return GRIFFIN_ERR_CUDA;
  }
  // global statistics (double, rounded once)
  const double avgdl = (double)sum_dl / (double)N;
  ix->h_terms.assign(V, TermInfo{});
  for (uint32_t t = 0; t < V; ++t) {
    const double df = (double)(c->list_offsets[t + 1] - c->list_offsets[t]);
    ix->h_terms[t].df_global = (uint32_t)(c->list_offsets[t + 1] - c->list_offsets[t]);
    ix->h_terms[t].idf = (float)std::log1p(((double)N - df + 0.5) / (df + 0.5));
  }
  const uint32_t nd = ix->doc_end - ix->doc_base;
  std::vector<float> norm(std::max<uint32_t>(nd, 1));
  for (uint32_t d = 0; d < nd; ++d)
    norm[d] = (float)(k1 * ((1.0 - bb) + bb * ((double)c->doc_lengths[ix->doc_base + d] / avgdl)));
  // this shard's slice of every list, local docIDs
  std::vector<uint64_t> post_off(V + 1, 0);
  std::vector<uint64_t> lo(V), hi(V);
  for (uint32_t t = 0; t < V; ++t) {
    const uint32_t *a = c->docids + c->list_offsets[t], *e = c->docids + c->list_offsets[t + 1];
    lo[t] = (G == 1) ? c->list_offsets[t] : (std::lower_bound(a, e, ix->doc_base) - c->docids);
    hi[t] = (G == 1) ? c->list_offsets[t + 1] : (std::lower_bound(a, e, ix->doc_end) - c->docids);
    post_off[t + 1] = post_off[t] + (hi[t] - lo[t]);
  }
  const uint64_t Ps = post_off[V];
  std::vector<uint32_t> ldoc(std::max<uint64_t>(Ps, 1)), ltf(std::max<uint64_t>(Ps, 1));
  for (uint32_t t = 0; t < V; ++t) {
    uint64_t o = post_off[t];
    for (uint64_t p = lo[t]; p < hi[t]; ++p, ++o) {
      ldoc[o] = c->docids[p] - ix->doc_base;
      ltf[o] = c->tfs[p];   // lossless: packed at bits(max tf - 1) <= 32
    }
  }
  griffin_status s = encode_index(ix, ldoc.data(), ltf.data(), post_off);
  if (s == GRIFFIN_OK) {
    cudaError_t e = cudaMalloc(&ix->d_norm, norm.size() * 4);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(ix->d_norm, norm.data(), norm.size() * 4, cudaMemcpyHostToDevice,
                          ix->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(ix->stream);
    if (e != cudaSuccess) {
      set_error(std::string("norm upload: ") + cudaGetErrorString(e));
      s = GRIFFIN_ERR_CUDA;
    }
  }
  if (s != GRIFFIN_OK) {
    griffin_index_destroy(ix);
    return s;
  }
  *out = ix;
  return GRIFFIN_OK;
}

griffin_status griffin_index_build(const griffin_corpus *c, const griffin_build_opts *o,
                                   griffin_index **out) {
  if (!c || !out) return invalid("null corpus/out");
  *out = nullptr;
  griffin_build_opts opts{};
  if (o) {
    opts = *o;
  } else {   // NULL: every documented default (b = 0.75, the current device)
    opts.bm25_b = -1.0;
    opts.device = -1;
  }
  const uint32_t B = opts.block_size ? opts.block_size : 128;
  if (B < 64 || B > 512 || (B % 32)) return invalid("block_size must be 64..512 and a multiple of 32");
  const uint32_t NG = opts.num_gpus ? opts.num_gpus : 1;
  if (NG > GRIFFIN_MAX_SHARDS) return invalid("num_gpus must be in [1, 8]");
  if (opts.exchange < 0 || opts.exchange > 3) return invalid("exchange must be 0..3");
  const uint32_t G = opts.num_shards ? opts.num_shards : 1;
  if (G > GRIFFIN_MAX_SHARDS || opts.shard_index >= G) return invalid("bad shard index / count");
  const bool multi = NG > 1 || opts.exchange != 0;
  if (multi && G > 1) return invalid("num_gpus > 1 builds every shard itself (num_shards must be 0/1)");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    set_error("no CUDA device");
    return GRIFFIN_ERR_UNSUPPORTED;
  }
  std::vector<int> devs(NG);
  for (uint32_t g = 0; g < NG; ++g) {
    int d = opts.devices ? opts.devices[g] : (NG > 1 ? (int)g : opts.device);
    if (d < 0) cudaGetDevice(&d);
    if (d >= ndev) return invalid(NG > 1 ? "num_gpus > visible devices (or a device ordinal out of range)"
                                         : "device ordinal out of range");
    griffin_status s = check_device(d);
    if (s) return s;
    devs[g] = d;
  }
  uint64_t sum_dl = 0;
  griffin_status s = validate_corpus(c, &sum_dl);
  if (s) return s;
  if (!multi) return build_shard(c, opts, sum_dl, G, opts.shard_index, devs[0], out);
  // num_gpus > 1: one handle over NG docID-range shards
  griffin_index *cx = new griffin_index();
  cx->device = devs[0];
  cx->B = B;
  cx->N = c->num_docs;
  cx->V = c->num_terms;
  cx->nshards = NG;
  cx->doc_base = 0;
  cx->doc_end = c->num_docs;
  for (uint32_t g = 0; g < NG; ++g) {
    griffin_index *sh = nullptr;
    if ((s = build_shard(c, opts, sum_dl, NG, g, devs[g], &sh))) {
      griffin_index_destroy(cx);
      return s;
    }
    cx->shards.push_back(sh);
  }
  if ((s = cluster_init(cx, opts.exchange))) {
    griffin_index_destroy(cx);
    return s;
  }
  *out = cx;
  return GRIFFIN_OK;
}

static void free_workspace(Workspace &w);

void griffin_index_destroy(griffin_index *ix) {
  if (!ix) return;
  if (ix->cl || !ix->shards.empty()) {   // multi-GPU handle
    cluster_destroy(ix);
    for (griffin_index *sh : ix->shards) griffin_index_destroy(sh);
    delete ix;
    return;
  }
  {
    DeviceGuard guard(ix->device);
    if (ix->stream) cudaStreamSynchronize(ix->stream);
    cudaFree(ix->d_terms);
    cudaFree(ix->d_first);
    cudaFree(ix->d_meta);
    cudaFree(ix->d_payload);
    cudaFree(ix->d_tfw);
    cudaFree(ix->d_norm);
    cudaFree(ix->d_bm_slot);
    cudaFree(ix->d_bm_term);
    for (Workspace *xw : ix->extra_ws) {
      free_workspace(*xw);
      delete xw;
    }
    ix->extra_ws.clear();
    free_workspace(ix->ws);
    free_workspace(ix->qws);
    for (cudaEvent_t e : ix->ev_pool) cudaEventDestroy(e);
    for (auto &g : ix->graphs) cudaGraphExecDestroy(g.exec);
    if (ix->stream) cudaStreamDestroy(ix->stream);
  }
  delete ix;
}

griffin_status griffin_index_stats(const griffin_index *ix, griffin_stats *out) {
  if (!ix || !out) return invalid("null argument");
  std::memset(out, 0, sizeof(*out));
  if (ix->cl) {   // multi-GPU handle: totals over its shards
    for (const griffin_index *sh : ix->shards) {
      griffin_stats t;
      griffin_index_stats(sh, &t);
      out->num_postings += t.num_postings;
      out->num_blocks += t.num_blocks;
      out->payload_bytes += t.payload_bytes;
      out->skip_bytes += t.skip_bytes;
      out->tf_bytes += t.tf_bytes;
      out->device_bytes += t.device_bytes;
    }
    out->shard_index = 0;
    out->num_shards = (uint32_t)ix->shards.size();
    out->doc_base = 0;
    out->doc_end = ix->N;
    out->block_size = ix->B;
    out->num_terms = ix->V;
    return GRIFFIN_OK;
  }
  out->shard_index = ix->shard;
  out->num_shards = ix->nshards;
  out->doc_base = ix->doc_base;
  out->doc_end = ix->doc_end;
  out->block_size = ix->B;
  out->num_terms = ix->V;
  out->num_postings = ix->postings;
  out->num_blocks = ix->nblocks;
  out->payload_bytes = ix->payload16 * 16;
  out->skip_bytes = ix->nblocks * 12;
  out->tf_bytes = ix->tf_words * 4;
  out->device_bytes = out->payload_bytes + out->skip_bytes + out->tf_bytes +
                      (uint64_t)ix->V * sizeof(TermInfo) + (uint64_t)(ix->doc_end - ix->doc_base) * 4;
  return GRIFFIN_OK;
}

griffin_status griffin_query_batch(griffin_index *ix, uint32_t nq, const uint32_t *qoffs,
                                   const uint32_t *terms, uint32_t k, uint32_t *out_docids,
                                   float *out_scores, uint32_t *out_counts) {
  if (!ix) return invalid("null index");
  if (nq == 0) return GRIFFIN_OK;
  if (!qoffs || !terms || !out_docids || !out_scores || !out_counts) return invalid("null argument");
  if (ix->cl) return cluster_query_batch(ix, nq, qoffs, terms, k, out_docids, out_scores, out_counts);
  std::lock_guard<std::mutex> lk(ix->mu);
  if (ix->ws.pending) return invalid("the index's workspace holds a submitted batch not yet collected");
  ix->ws.results_valid = false;
  DeviceGuard guard(ix->device);
  uint32_t max_terms = 1;
  griffin_status s = reserve_for(ix, ix->ws, nq, qoffs, terms, k, &max_terms);
  if (s) return s;
  Workspace &w = ix->ws;
  const uint64_t nt = qoffs[nq];
  const size_t nk = (size_t)nq * k;
  GRIFFIN_CUDA_TRY(w.qoffs.reserve(((size_t)nq + 1) * 4));
  GRIFFIN_CUDA_TRY(w.qterms.reserve(std::max<uint64_t>(nt, 1) * 4));
  GRIFFIN_CUDA_TRY(w.keys.reserve(nk * 8));
  GRIFFIN_CUDA_TRY(w.counts.reserve((size_t)nq * 4));
  GRIFFIN_CUDA_TRY(w.docids.reserve(nk * 4));
  GRIFFIN_CUDA_TRY(w.scores.reserve(nk * 4));
  // pinned staging: [qoffs | terms | docids | scores | counts]
  const size_t b_in = ((size_t)nq + 1 + nt) * 4, b_out = nk * 8 + (size_t)nq * 4;
  if ((s = ensure_pinned(ix, b_in + b_out))) return s;
  uint8_t *hp = static_cast<uint8_t *>(w.h_pinned);
  std::memcpy(hp, qoffs, ((size_t)nq + 1) * 4);
  std::memcpy(hp + ((size_t)nq + 1) * 4, terms, nt * 4);
  cudaStream_t st = ix->stream;
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(w.qoffs.p, hp, ((size_t)nq + 1) * 4, cudaMemcpyHostToDevice, st));
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(w.qterms.p, hp + ((size_t)nq + 1) * 4, nt * 4,
                                   cudaMemcpyHostToDevice, st));
  s = run_batch(ix, ix->ws, nq, w.qoffs.as<uint32_t>(), w.qterms.as<uint32_t>(), max_terms, k,
                w.keys.as<uint64_t>(), w.counts.as<uint32_t>(), st, true, ix->mode);
  if (s) return s;
  if ((s = launch_keys_to_results(ix, nq, k, w.keys.as<uint64_t>(), w.counts.as<uint32_t>(),
                                  w.docids.as<uint32_t>(), w.scores.as<float>(), st)))
    return s;
  uint8_t *ho = hp + b_in;
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(ho, w.docids.p, nk * 4, cudaMemcpyDeviceToHost, st));
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(ho + nk * 4, w.scores.p, nk * 4, cudaMemcpyDeviceToHost, st));
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(ho + nk * 8, w.counts.p, (size_t)nq * 4, cudaMemcpyDeviceToHost, st));
  if ((s = read_status(ix, ix->ws))) return s;  // synchronises
  par_memcpy(out_docids, ho, nk * 4);
  par_memcpy(out_scores, ho + nk * 4, nk * 4);
  std::memcpy(out_counts, ho + nk * 8, (size_t)nq * 4);
  return GRIFFIN_OK;
}

// identity of the workspace buffers a captured graph points into
static uint64_t ws_identity(const Workspace &w) {
  uint64_t h = 1469598103934665603ull;
  for (const DevBuf *b : {&w.plan_terms, &w.plan_m, &w.cap, &w.cap_off, &w.rcount, &w.rsel,
                          &w.qmode, &w.unit_base, &w.unit_off, &w.unit_cnt, &w.unit_dst, &w.urec, &w.uperm,
                          &w.rbuf0, &w.rbuf1, &w.bump, &w.cand, &w.tkstate, &w.scal, &w.keys,
                          &w.counts, &w.docids, &w.scores, &w.qoffs, &w.qterms, &w.demand,
                          &w.tdec, &w.runs, &w.run_base, &w.vtmp, &w.run_term, &w.arena, &w.bmap, &w.qtau})
    h = (h ^ (uint64_t)(uintptr_t)b->p) * 1099511628211ull;
  // capacities are baked into a captured graph's kernel arguments too
  for (const uint64_t v : {(uint64_t)w.nq_cap, (uint64_t)w.unit_cap, (uint64_t)w.entry_cap,
                           (uint64_t)w.bump.bytes})
    h = (h ^ v) * 1099511628211ull;
  return h ^ (uint64_t)(uintptr_t)w.h_pinned;
}

// Single query through a cached CUDA graph: H2D of the terms, every kernel of
// the path, D2H of the results and status, one graph launch (removes per-launch
// CPU overhead from the latency path).  Workspace is pre-sized once for the
// largest possible single query so captured addresses stay valid.
static griffin_status query_graph(griffin_index *ix, const uint32_t *terms, uint32_t nterms,
                                  uint32_t k, uint32_t *out_docids, float *out_scores,
                                  uint32_t *out_count) {
  Workspace &w = ix->qws;   // own workspace: batch reservations never move its graphs
  const uint32_t offs[2] = {0, nterms};
  uint32_t mt = 1;
  // validation + bounds (same rules as the batch path)
  griffin_status s = reserve_for(ix, w, 1, offs, terms, k, &mt);
  if (s) return s;
  if (!ix->single_ws) {
    uint64_t mx = 0, mb = 0;
    for (const TermInfo &t : ix->h_terms) {
      mx = std::max<uint64_t>(mx, t.df_local);
      mb = std::max<uint64_t>(mb, t.nblocks);
    }
    // units of any one query: blocks of t0 + max(blocks of a later list, probe
    // units of >= 32 survivors each)
    if ((s = reserve_ws(ix, w, 1, 2 * mb + mx / 32 + 2, mx + 1))) return s;
    if ((s = reserve_topk(ix, w, 1, GRIFFIN_MAX_K))) return s;
    if ((s = reserve_topk(ix, w, 1, 2048))) return s;   // the k with the most selection levels
    GRIFFIN_CUDA_TRY(w.qoffs.reserve(8));
    GRIFFIN_CUDA_TRY(w.qterms.reserve(GRIFFIN_MAX_TERMS * 4 * 4));
    GRIFFIN_CUDA_TRY(w.keys.reserve(GRIFFIN_MAX_K * 8));
    GRIFFIN_CUDA_TRY(w.counts.reserve(8));
    GRIFFIN_CUDA_TRY(w.docids.reserve(GRIFFIN_MAX_K * 4));
    GRIFFIN_CUDA_TRY(w.scores.reserve(GRIFFIN_MAX_K * 4));
    if ((s = ensure_pinned_ws(w, 64 * 4 + GRIFFIN_MAX_K * 8 + 64))) return s;
    ix->single_ws = true;
  }
  if (nterms > GRIFFIN_MAX_TERMS * 4) return GRIFFIN_ERR_UNSUPPORTED;  // caller falls back
  // pinned layout: [qoffs 2][terms 64][status 2] then results
  uint32_t *hp = static_cast<uint32_t *>(w.h_pinned);
  uint32_t *h_off = hp, *h_terms = hp + 2, *h_status = hp + 66;
  uint8_t *h_res = reinterpret_cast<uint8_t *>(hp + 68);
  const uint64_t id = ws_identity(w);
  cudaGraphExec_t exec = nullptr;
  for (auto &g : ix->graphs)
    if (g.mt == mt && g.k == k && g.mode == ix->mode && g.ws_id == id) exec = g.exec;
  cudaStream_t st = ix->stream;
  if (!exec) {
    if (ix->graphs.size() >= 64) {
      for (auto &g : ix->graphs) cudaGraphExecDestroy(g.exec);
      ix->graphs.clear();
    }
    cudaGraph_t graph = nullptr;
    GRIFFIN_CUDA_TRY(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
    cudaMemcpyAsync(w.qoffs.p, h_off, 8, cudaMemcpyHostToDevice, st);
    cudaMemcpyAsync(w.qterms.p, h_terms, GRIFFIN_MAX_TERMS * 4 * 4, cudaMemcpyHostToDevice, st);
    griffin_status rs = run_batch(ix, w, 1, w.qoffs.as<uint32_t>(), w.qterms.as<uint32_t>(), mt, k,
                                  w.keys.as<uint64_t>(), w.counts.as<uint32_t>(), st, true,
                                  ix->mode);
    if (!rs)
      rs = launch_keys_to_results(ix, 1, k, w.keys.as<uint64_t>(), w.counts.as<uint32_t>(),
                                  w.docids.as<uint32_t>(), w.scores.as<float>(), st);
    cudaMemcpyAsync(h_res, w.docids.p, (size_t)k * 4, cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(h_res + (size_t)k * 4, w.scores.p, (size_t)k * 4, cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(h_res + (size_t)k * 8, w.counts.p, 4, cudaMemcpyDeviceToHost, st);
    cudaMemcpyAsync(h_status, w.scal.as<unsigned long long>() + kScalStatus, 4,
                    cudaMemcpyDeviceToHost, st);
    cudaError_t e = cudaStreamEndCapture(st, &graph);
    if (rs || e != cudaSuccess) {
      if (graph) cudaGraphDestroy(graph);
      cudaGetLastError();
      return GRIFFIN_ERR_UNSUPPORTED;  // caller falls back to the plain launches
    }
    e = cudaGraphInstantiate(&exec, graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return GRIFFIN_ERR_UNSUPPORTED;
    }
    ix->graphs.push_back({mt, k, ix->mode, id, exec});
  }
  h_off[0] = 0;
  h_off[1] = nterms;
  std::memcpy(h_terms, terms, (size_t)nterms * 4);
  GRIFFIN_CUDA_TRY(cudaGraphLaunch(exec, st));
  GRIFFIN_CUDA_TRY(cudaStreamSynchronize(st));
  if (*h_status) {
    if ((s = read_status(ix, w))) return s;   // clears the device flag
  }
  std::memcpy(out_docids, h_res, (size_t)k * 4);
  std::memcpy(out_scores, h_res + (size_t)k * 4, (size_t)k * 4);
  std::memcpy(out_count, h_res + (size_t)k * 8, 4);
  return GRIFFIN_OK;
}

griffin_status griffin_query(griffin_index *ix, const uint32_t *terms, uint32_t nterms, uint32_t k,
                             uint32_t *out_docids, float *out_scores, uint32_t *out_count) {
  if (nterms == 0) return invalid("nterms must be > 0");
  if (!ix || !terms || !out_docids || !out_scores || !out_count) return invalid("null argument");
  if (ix->use_graphs && !ix->profiling && !ix->cl) {
    std::lock_guard<std::mutex> lk(ix->mu);
    if (ix->ws.pending) return invalid("the index's workspace holds a submitted batch not yet collected");
    ix->ws.results_valid = false;
    DeviceGuard guard(ix->device);
    griffin_status s = query_graph(ix, terms, nterms, k, out_docids, out_scores, out_count);
    if (s != GRIFFIN_ERR_UNSUPPORTED) return s;
  }
  const uint32_t offs[2] = {0, nterms};
  return griffin_query_batch(ix, 1, offs, terms, k, out_docids, out_scores, out_count);
}

griffin_status griffin_reserve(griffin_index *ix, uint32_t nq, const uint32_t *qoffs,
                               const uint32_t *terms, uint32_t k) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix || (nq && (!qoffs || !terms))) return invalid("null argument");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  return reserve_for(ix, ix->ws, nq, qoffs, terms, k, nullptr);
}

griffin_status griffin_query_batch_device(griffin_index *ix, uint32_t nq, const uint32_t *d_qoffs,
                                          const uint32_t *d_terms, uint32_t max_terms, uint32_t k,
                                          uint64_t *d_out_keys, uint32_t *d_out_counts,
                                          void *stream) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix) return invalid("null index");
  if (k == 0 || k > GRIFFIN_MAX_K) return invalid("k must be in [1, 4096]");
  if (max_terms == 0 || max_terms > GRIFFIN_MAX_TERMS) return invalid("max_terms out of range");
  if (nq == 0) return GRIFFIN_OK;
  std::lock_guard<std::mutex> lk(ix->mu);
  if (ix->ws.pending) return invalid("the index's workspace holds a submitted batch not yet collected");
  ix->ws.results_valid = false;
  DeviceGuard guard(ix->device);
  return run_batch(ix, ix->ws, nq, d_qoffs, d_terms, max_terms, k, d_out_keys, d_out_counts,
                   static_cast<cudaStream_t>(stream), true, ix->mode);
}

griffin_status griffin_sync_status(griffin_index *ix) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix) return invalid("null index");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  GRIFFIN_CUDA_TRY(cudaDeviceSynchronize());
  if (!ix->ws.scal.p) return GRIFFIN_OK;
  return read_status(ix, ix->ws);
}

griffin_status griffin_workspace_create(griffin_index *ix, griffin_workspace **out) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix || !out) return invalid("null argument");
  std::lock_guard<std::mutex> lk(ix->mu);
  Workspace *w = new Workspace();
  ix->extra_ws.push_back(w);
  *out = reinterpret_cast<griffin_workspace *>(w);
  return GRIFFIN_OK;
}

static void free_workspace(Workspace &w) {
  for (DevBuf *b : {&w.plan_terms, &w.plan_m, &w.cap, &w.cap_off, &w.rcount, &w.rsel, &w.qmode,
                    &w.unit_base, &w.unit_off, &w.unit_cnt, &w.unit_dst, &w.urec, &w.uperm, &w.rbuf0,
                    &w.rbuf1, &w.bump, &w.cand, &w.tkstate, &w.scal, &w.keys, &w.counts,
                    &w.docids, &w.scores, &w.qoffs, &w.qterms, &w.demand, &w.tdec, &w.runs,
                    &w.run_base, &w.vtmp, &w.run_term, &w.arena, &w.bmap, &w.qtau, &w.sbkt_cnt, &w.sbkt_pos,
                    &w.sbkt_tmp, &w.flt, &w.fstate})
    b->release();
  if (w.h_pinned) cudaFreeHost(w.h_pinned);
  for (void *p : w.old_pinned) cudaFreeHost(p);
  w.old_pinned.clear();
  w.h_pinned = nullptr;
  w.h_pinned_bytes = 0;
  if (w.done) cudaEventDestroy(w.done);
  w.done = nullptr;
  w.pending = false;
}

void griffin_workspace_destroy(griffin_index *ix, griffin_workspace *ws) {
  if (!ix || !ws) return;
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  Workspace *w = reinterpret_cast<Workspace *>(ws);
  cudaDeviceSynchronize();
  free_workspace(*w);
  for (size_t i = 0; i < ix->extra_ws.size(); ++i)
    if (ix->extra_ws[i] == w) ix->extra_ws.erase(ix->extra_ws.begin() + i);
  delete w;
}

griffin_status griffin_workspace_reserve(griffin_index *ix, griffin_workspace *ws, uint32_t nq,
                                         const uint32_t *qoffs, const uint32_t *terms,
                                         uint32_t k) {
  if (!ix || !ws || (nq && (!qoffs || !terms))) return invalid("null argument");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  return reserve_for(ix, *reinterpret_cast<Workspace *>(ws), nq, qoffs, terms, k, nullptr);
}

griffin_status griffin_query_batch_device_ws(griffin_index *ix, griffin_workspace *ws, uint32_t nq,
                                             const uint32_t *d_qoffs, const uint32_t *d_terms,
                                             uint32_t max_terms, uint32_t k, uint64_t *d_out_keys,
                                             uint32_t *d_out_counts, void *stream) {
  if (!ix || !ws) return invalid("null argument");
  if (k == 0 || k > GRIFFIN_MAX_K) return invalid("k must be in [1, 4096]");
  if (max_terms == 0 || max_terms > GRIFFIN_MAX_TERMS) return invalid("max_terms out of range");
  if (nq == 0) return GRIFFIN_OK;
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  return run_batch(ix, *reinterpret_cast<Workspace *>(ws), nq, d_qoffs, d_terms, max_terms, k,
                   d_out_keys, d_out_counts, static_cast<cudaStream_t>(stream), true, ix->mode);
}

griffin_status griffin_workspace_sync_status(griffin_index *ix, griffin_workspace *ws) {
  if (!ix || !ws) return invalid("null argument");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  GRIFFIN_CUDA_TRY(cudaDeviceSynchronize());
  Workspace &w = *reinterpret_cast<Workspace *>(ws);
  if (!w.scal.p) return GRIFFIN_OK;
  return read_status(ix, w);
}

// Host-buffer batch split into an enqueue and a wait, so a caller with several
// workspaces keeps several batches (H2D of the queries, the path, D2H of the
// results) in flight: the same staging as griffin_query_batch, but into the
// workspace's own pinned buffer, plus the status word, then an event.
griffin_status griffin_query_batch_submit(griffin_index *ix, griffin_workspace *ws, uint32_t nq,
                                          const uint32_t *qoffs, const uint32_t *terms,
                                          uint32_t k, void *stream) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix) return invalid("null index");
  if (nq && (!qoffs || !terms)) return invalid("null argument");
  Workspace &w = ws ? *reinterpret_cast<Workspace *>(ws) : ix->ws;
  std::lock_guard<std::mutex> lk(ix->mu);
  if (w.pending) return invalid("workspace has a submitted batch not yet collected");
  w.results_valid = false;
  DeviceGuard guard(ix->device);
  cudaStream_t st = stream ? static_cast<cudaStream_t>(stream) : ix->stream;
  uint32_t max_terms = 1;
  griffin_status s = GRIFFIN_OK;
  if (nq && (s = reserve_for(ix, w, nq, qoffs, terms, k, &max_terms))) return s;
  if (!nq && (k == 0 || k > GRIFFIN_MAX_K)) return invalid("k must be in [1, 4096]");
  const uint64_t nt = nq ? qoffs[nq] : 0;
  const size_t nk = (size_t)nq * k;
  // pinned staging: [qoffs | terms | docids | scores | counts | status]
  const size_t b_in = nq ? ((size_t)nq + 1 + nt) * 4 : 0;
  const size_t b_out = nk * 8 + (size_t)nq * 4;
  if ((s = ensure_pinned_ws(w, b_in + b_out + 8))) return s;
  if (!w.done) GRIFFIN_CUDA_TRY(cudaEventCreateWithFlags(&w.done, cudaEventDisableTiming));
  uint8_t *hp = static_cast<uint8_t *>(w.h_pinned);
  int *h_status = reinterpret_cast<int *>(hp + b_in + b_out);
  *h_status = 0;
  if (nq) {
    GRIFFIN_CUDA_TRY(w.qoffs.reserve(((size_t)nq + 1) * 4));
    GRIFFIN_CUDA_TRY(w.qterms.reserve(std::max<uint64_t>(nt, 1) * 4));
    GRIFFIN_CUDA_TRY(w.keys.reserve(nk * 8));
    GRIFFIN_CUDA_TRY(w.counts.reserve((size_t)nq * 4));
    GRIFFIN_CUDA_TRY(w.docids.reserve(nk * 4));
    GRIFFIN_CUDA_TRY(w.scores.reserve(nk * 4));
    std::memcpy(hp, qoffs, ((size_t)nq + 1) * 4);
    std::memcpy(hp + ((size_t)nq + 1) * 4, terms, nt * 4);
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(w.qoffs.p, hp, ((size_t)nq + 1) * 4, cudaMemcpyHostToDevice, st));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(w.qterms.p, hp + ((size_t)nq + 1) * 4, nt * 4,
                                     cudaMemcpyHostToDevice, st));
    if ((s = run_batch(ix, w, nq, w.qoffs.as<uint32_t>(), w.qterms.as<uint32_t>(), max_terms, k,
                       w.keys.as<uint64_t>(), w.counts.as<uint32_t>(), st, true, ix->mode)))
      return s;
    if ((s = launch_keys_to_results(ix, nq, k, w.keys.as<uint64_t>(), w.counts.as<uint32_t>(),
                                    w.docids.as<uint32_t>(), w.scores.as<float>(), st)))
      return s;
    uint8_t *ho = hp + b_in;
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(ho, w.docids.p, nk * 4, cudaMemcpyDeviceToHost, st));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(ho + nk * 4, w.scores.p, nk * 4, cudaMemcpyDeviceToHost, st));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(ho + nk * 8, w.counts.p, (size_t)nq * 4,
                                     cudaMemcpyDeviceToHost, st));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h_status, w.scal.as<unsigned long long>() + kScalStatus,
                                     sizeof(int), cudaMemcpyDeviceToHost, st));
  }
  GRIFFIN_CUDA_TRY(cudaEventRecord(w.done, st));
  w.pend_stream = st;
  w.pend_nq = nq;
  w.pend_k = k;
  w.pend_out = b_in;
  w.pending = true;
  return GRIFFIN_OK;
}

griffin_status griffin_query_batch_results(griffin_index *ix, griffin_workspace *ws,
                                           const uint32_t **docids, const float **scores,
                                           const uint32_t **counts) {
  if (!ix || !docids || !scores || !counts) return invalid("null argument");
  Workspace &w = ws ? *reinterpret_cast<Workspace *>(ws) : ix->ws;
  if (w.pending || !w.results_valid || !w.h_pinned)
    return invalid("no successfully collected batch on this workspace");
  const size_t nk = (size_t)w.pend_nq * w.pend_k;
  const uint8_t *ho = static_cast<const uint8_t *>(w.h_pinned) + w.pend_out;
  *docids = reinterpret_cast<const uint32_t *>(ho);
  *scores = reinterpret_cast<const float *>(ho + nk * 4);
  *counts = reinterpret_cast<const uint32_t *>(ho + nk * 8);
  return GRIFFIN_OK;
}

griffin_status griffin_query_batch_collect(griffin_index *ix, griffin_workspace *ws,
                                           uint32_t *out_docids, float *out_scores,
                                           uint32_t *out_counts) {
  if (!ix) return invalid("null index");
  Workspace &w = ws ? *reinterpret_cast<Workspace *>(ws) : ix->ws;
  if (!w.pending) return invalid("no submitted batch on this workspace");
  const size_t nk = (size_t)w.pend_nq * w.pend_k;
  const bool copy = out_docids || out_scores || out_counts;
  if (w.pend_nq && copy && (!out_docids || !out_scores || !out_counts))
    return invalid("null argument");
  {
    DeviceGuard guard(ix->device);
    cudaError_t e = cudaEventSynchronize(w.done);   // without the index lock: others submit
    if (e != cudaSuccess) {
      w.results_valid = false;
      w.pending = false;
      set_error(std::string("cudaEventSynchronize: ") + cudaGetErrorString(e));
      return GRIFFIN_ERR_CUDA;
    }
  }
  const uint8_t *ho = static_cast<const uint8_t *>(w.h_pinned) + w.pend_out;
  if (*reinterpret_cast<const int *>(ho + nk * 8 + (size_t)w.pend_nq * 4)) {
    std::lock_guard<std::mutex> lk(ix->mu);
    DeviceGuard guard(ix->device);
    griffin_status s = read_status(ix, w, w.pend_stream);   // clears the device flag
    if (s) {
      w.results_valid = false;
      w.pending = false;
      return s;
    }
  }
  if (w.pend_nq && copy) {
    par_memcpy(out_docids, ho, nk * 4);
    par_memcpy(out_scores, ho + nk * 4, nk * 4);
    std::memcpy(out_counts, ho + nk * 8, (size_t)w.pend_nq * 4);
  }
  // only now may a synchronous call on this workspace reuse the staging
  w.results_valid = true;
  w.pending = false;
  return GRIFFIN_OK;
}

griffin_status griffin_merge_topk_device(griffin_index *ix, uint32_t num_runs, uint32_t nq,
                                         uint32_t k, const uint64_t *d_keys,
                                         const uint32_t *d_counts, uint64_t *d_out_keys,
                                         uint32_t *d_out_counts, void *stream) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix) return invalid("null index");
  if (num_runs == 0 || num_runs > 32) return invalid("num_runs must be in [1, 32]");
  if (k == 0 || k > GRIFFIN_MAX_K) return invalid("k must be in [1, 4096]");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  return launch_merge_topk(ix, num_runs, nq, k, d_keys, d_counts, d_out_keys, d_out_counts,
                           static_cast<cudaStream_t>(stream));
}

griffin_status griffin_keys_to_results_device(griffin_index *ix, uint32_t nq, uint32_t k,
                                              const uint64_t *d_keys, const uint32_t *d_counts,
                                              uint32_t *d_docids, float *d_scores, void *stream) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix) return invalid("null index");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  return launch_keys_to_results(ix, nq, k, d_keys, d_counts, d_docids, d_scores,
                                static_cast<cudaStream_t>(stream));
}

griffin_status griffin_set_mode(griffin_index *ix, int mode) {
  if (ix && ix->cl) {   // multi-GPU handle: every shard
    for (griffin_index *sh : ix->shards) {
      griffin_status s = griffin_set_mode(sh, mode);
      if (s) return s;
    }
    return GRIFFIN_OK;
  }
  if (!ix || mode < 0 || mode > 2) return invalid("mode must be 0 (auto), 1 (merge) or 2 (gallop)");
  std::lock_guard<std::mutex> lk(ix->mu);
  ix->mode = mode;
  return GRIFFIN_OK;
}

griffin_status griffin_set_reuse(griffin_index *ix, int mode) {
  if (ix && ix->cl) {   // multi-GPU handle: every shard
    for (griffin_index *sh : ix->shards) {
      griffin_status s = griffin_set_reuse(sh, mode);
      if (s) return s;
    }
    return GRIFFIN_OK;
  }
  if (!ix || mode < 0 || mode > 2) return invalid("reuse must be 0 (off), 1 (on) or 2 (auto)");
  std::lock_guard<std::mutex> lk(ix->mu);
  ix->reuse = mode;
  return GRIFFIN_OK;
}

griffin_status griffin_set_bitmap(griffin_index *ix, uint32_t inv) {
  if (ix && ix->cl) {   // multi-GPU handle: every shard
    for (griffin_index *sh : ix->shards) {
      griffin_status s = griffin_set_bitmap(sh, inv);
      if (s) return s;
    }
    return GRIFFIN_OK;
  }
  if (!ix) return invalid("null index");
  std::lock_guard<std::mutex> lk(ix->mu);
  ix->bm_inv = inv;
  return GRIFFIN_OK;
}

griffin_status griffin_set_nextgeq(griffin_index *ix, int on) {
  if (ix && ix->cl) {   // multi-GPU handle: every shard
    for (griffin_index *sh : ix->shards) {
      griffin_status s = griffin_set_nextgeq(sh, on);
      if (s) return s;
    }
    return GRIFFIN_OK;
  }
  if (!ix || on < 0 || on > 1) return invalid("nextgeq must be 0 or 1");
  std::lock_guard<std::mutex> lk(ix->mu);
  if (ix->nextgeq != on) {   // captured single-query graphs bake the option in
    for (auto &g : ix->graphs) cudaGraphExecDestroy(g.exec);
    ix->graphs.clear();
  }
  ix->nextgeq = on;
  return GRIFFIN_OK;
}

griffin_status griffin_set_probe_chunk(griffin_index *ix, uint32_t chunk) {
  if (ix && ix->cl) {   // multi-GPU handle: every shard
    for (griffin_index *sh : ix->shards) {
      griffin_status s = griffin_set_probe_chunk(sh, chunk);
      if (s) return s;
    }
    return GRIFFIN_OK;
  }
  if (!ix) return invalid("null index");
  if (chunk != 0 && (chunk < 32 || chunk > ix->B || chunk % 32 != 0))
    return invalid("probe chunk must be 0 or a multiple of 32 in [32, block_size]");
  std::lock_guard<std::mutex> lk(ix->mu);
  if (ix->P != chunk) {   // captured single-query graphs bake the option in
    for (auto &g : ix->graphs) cudaGraphExecDestroy(g.exec);
    ix->graphs.clear();
  }
  ix->P = chunk;
  return GRIFFIN_OK;
}

griffin_status griffin_set_entry_budget(griffin_index *ix, uint64_t entries) {
  if (!ix) return invalid("null index");
  if (ix->cl) {
    for (griffin_index *sh : ix->shards) sh->entry_budget = entries;
    return GRIFFIN_OK;
  }
  std::lock_guard<std::mutex> lk(ix->mu);
  ix->entry_budget = entries;
  return GRIFFIN_OK;
}

griffin_status griffin_set_profiling(griffin_index *ix, int on) {
  if (ix && ix->cl) {   // multi-GPU handle: every shard
    for (griffin_index *sh : ix->shards) {
      griffin_status s = griffin_set_profiling(sh, on);
      if (s) return s;
    }
    return GRIFFIN_OK;
  }
  if (!ix) return invalid("null index");
  std::lock_guard<std::mutex> lk(ix->mu);
  if (on < 0 || on > 3) return invalid("profiling must be 0 (off), 1 (events + counters), 2 (events) or 3 (counters)");
  ix->profiling = on == 1 ? 3 : on == 2 ? 1 : on == 3 ? 2 : 0;
  return GRIFFIN_OK;
}

griffin_status griffin_reset_profile(griffin_index *ix) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix) return invalid("null index");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  GRIFFIN_CUDA_TRY(cudaDeviceSynchronize());
  ix->prof = griffin_profile{};
  ix->pending.clear();
  ix->ev_next = 0;
  ix->launch_count = 0;
  std::vector<Workspace *> all(ix->extra_ws);
  all.push_back(&ix->ws);
  all.push_back(&ix->qws);
  for (Workspace *w : all)
    if (w->scal.p) {
      GRIFFIN_CUDA_TRY(cudaMemset(w->scal.p, 0, 4 * 8));
      GRIFFIN_CUDA_TRY(cudaMemset(w->scal.as<unsigned long long>() + kScalDec, 0, 3 * 8));
      GRIFFIN_CUDA_TRY(cudaMemset(w->scal.as<unsigned long long>() + kScalArena, 0, 3 * 8));
      GRIFFIN_CUDA_TRY(cudaMemset(w->scal.as<unsigned long long>() + kScalDiag, 0, 4 * 8));
      GRIFFIN_CUDA_TRY(cudaMemset(w->scal.as<unsigned long long>() + kScalDiag2, 0, 4 * 8));
    }
  return GRIFFIN_OK;
}

griffin_status griffin_get_profile(griffin_index *ix, griffin_profile *out) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix || !out) return invalid("null argument");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  GRIFFIN_CUDA_TRY(cudaDeviceSynchronize());
  for (auto &p : ix->pending) {
    float ms = 0.f;
    GRIFFIN_CUDA_TRY(cudaEventElapsedTime(&ms, p.second.first, p.second.second));
    double *slot[6] = {&ix->prof.ms_plan, &ix->prof.ms_intersect, &ix->prof.ms_compact,
                       &ix->prof.ms_topk, &ix->prof.ms_merge, &ix->prof.ms_decode};
    *slot[p.first] += ms;
    if (p.first == 1) ix->prof.launches_intersect += 1;
    if (p.first == 5) ix->prof.launches_decode += 1;
  }
  ix->pending.clear();
  ix->ev_next = 0;
  *out = ix->prof;
  out->launches_total = ix->launch_count;
  std::vector<Workspace *> all(ix->extra_ws);
  all.push_back(&ix->ws);
  all.push_back(&ix->qws);
  out->alg_bytes = out->payload_bytes = out->decoded_postings = out->survivors = 0;
  out->dec_alg_bytes = out->dec_payload_bytes = out->dec_postings = 0;
  out->c8d_bytes = out->dec_c8d_bytes = out->arena_postings = 0;
  out->merge_units = out->merge_elems = out->gallop_units = out->gallop_elems = 0;
  out->bitmap_units = out->bitmap_elems = out->bitand_units = out->bitand_words = 0;
  for (Workspace *w : all) {
    if (!w->scal.p) continue;
    unsigned long long c[kScalCount];
    GRIFFIN_CUDA_TRY(cudaMemcpy(c, w->scal.p, sizeof(c), cudaMemcpyDeviceToHost));
    out->alg_bytes += c[0];
    out->payload_bytes += c[1];
    out->decoded_postings += c[2];
    out->survivors += c[3];
    out->dec_alg_bytes += c[kScalDec + 0];
    out->dec_payload_bytes += c[kScalDec + 1];
    out->dec_postings += c[kScalDec + 2];
    out->arena_postings += c[kScalArena];
    out->c8d_bytes += c[0] - 4ull * c[kScalArena] + c[kScalArena + 1];
    out->dec_c8d_bytes += c[kScalDecC8d];
    out->merge_units += c[kScalDiag];
    out->merge_elems += c[kScalDiag + 1];
    out->gallop_units += c[kScalDiag + 2];
    out->gallop_elems += c[kScalDiag + 3];
    out->bitmap_units += c[kScalDiag2];
    out->bitmap_elems += c[kScalDiag2 + 1];
    out->bitand_units += c[kScalDiag2 + 2];
    out->bitand_words += c[kScalDiag2 + 3];
  }
  return GRIFFIN_OK;
}

// ---- debug hooks ------------------------------------------------------------------

griffin_status griffin_debug_block_streams(griffin_index *ix, uint32_t term, uint64_t blk,
                                           uint32_t *first, uint32_t *n, uint32_t *b,
                                           uint32_t *low, uint64_t low_cap, uint64_t *low_bits,
                                           uint32_t *high, uint64_t high_cap, uint64_t *high_bits) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix || term >= ix->V) return invalid("bad term");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  const TermInfo &t = ix->h_terms[term];
  if (blk >= t.nblocks) return invalid("bad block");
  const uint64_t gb = (uint64_t)t.block0 + blk;
  uint2 m;
  uint32_t f;
  GRIFFIN_CUDA_TRY(cudaMemcpy(&m, ix->d_meta + gb, 8, cudaMemcpyDeviceToHost));
  GRIFFIN_CUDA_TRY(cudaMemcpy(&f, ix->d_first + gb, 4, cudaMemcpyDeviceToHost));
  const uint32_t bb = meta_b(m.y), nn = meta_n(m.y), hw = meta_hw(m.y);
  const uint32_t lw = low_words(nn, bb);
  std::vector<uint32_t> words((size_t)(lw + hw + 3) / 4 * 4);
  GRIFFIN_CUDA_TRY(cudaMemcpy(words.data(), ix->d_payload + m.x, words.size() * 4,
                              cudaMemcpyDeviceToHost));
  // logical high-stream length: position of the n-th one + 1
  uint64_t L = 0, ones = 0;
  for (uint64_t p = 0; p < (uint64_t)hw * 32 && ones < nn; ++p)
    if ((words[lw + p / 32] >> (p % 32)) & 1u) {
      ++ones;
      L = p + 1;
    }
  const uint64_t lb = (uint64_t)nn * bb;
  if ((lb + 31) / 32 > low_cap || (L + 31) / 32 > high_cap) return invalid("capacity too small");
  *first = f + ix->doc_base;
  *n = nn;
  *b = bb;
  *low_bits = lb;
  *high_bits = L;
  for (uint64_t i = 0; i < (lb + 31) / 32; ++i) {
    uint32_t v = words[i];
    if (i == lb / 32 && (lb % 32)) v &= (1u << (lb % 32)) - 1u;
    low[i] = v;
  }
  for (uint64_t i = 0; i < (L + 31) / 32; ++i) {
    uint32_t v = words[lw + i];
    if (i == L / 32 && (L % 32)) v &= (1u << (L % 32)) - 1u;
    high[i] = v;
  }
  return GRIFFIN_OK;
}

griffin_status griffin_debug_decode_list(griffin_index *ix, uint32_t term, uint32_t *out,
                                         uint64_t cap, uint64_t *n) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix || term >= ix->V || !n) return invalid("bad arguments");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  const TermInfo &t = ix->h_terms[term];
  *n = t.df_local;
  if (t.df_local > cap) return invalid("capacity too small");
  if (!t.df_local) return GRIFFIN_OK;
  uint32_t *d = nullptr;
  GRIFFIN_CUDA_TRY(cudaMalloc(&d, (size_t)t.nblocks * ix->B * 4));
  griffin_status s = launch_decode_list(ix, term, d, ix->stream);
  if (!s) {
    cudaError_t e = cudaMemcpyAsync(out, d, (size_t)t.df_local * 4, cudaMemcpyDeviceToHost, ix->stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(ix->stream);
    if (e != cudaSuccess) {
      set_error(cudaGetErrorString(e));
      s = GRIFFIN_ERR_CUDA;
    }
  }
  cudaFree(d);
  return s;
}

griffin_status griffin_debug_decode_all(griffin_index *ix, int iters, double *ms,
                                        uint64_t *checksum, uint64_t *postings, uint64_t *bytes) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix || iters <= 0) return invalid("bad arguments");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  unsigned long long *acc = nullptr;
  GRIFFIN_CUDA_TRY(cudaMalloc(&acc, 3 * 8));
  GRIFFIN_CUDA_TRY(cudaMemsetAsync(acc, 0, 24, ix->stream));
  griffin_status s = launch_decode_all(ix, acc, ix->stream);  // warm-up; its XOR is the checksum
  unsigned long long h0[3] = {0, 0, 0};
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h0, acc, 24, cudaMemcpyDeviceToHost, ix->stream));
  GRIFFIN_CUDA_TRY(cudaStreamSynchronize(ix->stream));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  GRIFFIN_CUDA_TRY(cudaMemsetAsync(acc, 0, 24, ix->stream));
  cudaEventRecord(a, ix->stream);
  for (int i = 0; i < iters && !s; ++i) s = launch_decode_all(ix, acc, ix->stream);
  cudaEventRecord(b, ix->stream);
  unsigned long long h[3] = {0, 0, 0};
  cudaMemcpyAsync(h, acc, 24, cudaMemcpyDeviceToHost, ix->stream);
  cudaError_t e = cudaStreamSynchronize(ix->stream);
  float t = 0;
  cudaEventElapsedTime(&t, a, b);
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(acc);
  if (e != cudaSuccess) {
    set_error(cudaGetErrorString(e));
    return GRIFFIN_ERR_CUDA;
  }
  if (s) return s;
  if (ms) *ms = t / iters;
  if (checksum) *checksum = h0[0];
  if (postings) *postings = h[1] / iters;
  if (bytes) *bytes = h[2] / iters;
  return GRIFFIN_OK;
}

griffin_status griffin_debug_intersect(griffin_index *ix, const uint32_t *terms, uint32_t nterms,
                                       int mode, uint32_t *out_docids, uint64_t cap,
                                       uint64_t *count) {
  if (ix && ix->cl) return multi_unsupported();
  if (!ix || !terms || nterms == 0 || !count) return invalid("bad arguments");
  if (mode < 0 || mode > 2) return invalid("bad mode");
  std::lock_guard<std::mutex> lk(ix->mu);
  DeviceGuard guard(ix->device);
  const uint32_t offs[2] = {0, nterms};
  if (ix->ws.pending) return invalid("the index's workspace holds a submitted batch not yet collected");
  ix->ws.results_valid = false;
  uint32_t max_terms = 1;
  griffin_status s = reserve_for(ix, ix->ws, 1, offs, terms, 1, &max_terms);
  if (s) return s;
  Workspace &w = ix->ws;
  GRIFFIN_CUDA_TRY(w.qoffs.reserve(8));
  GRIFFIN_CUDA_TRY(w.qterms.reserve((size_t)nterms * 4));
  cudaStream_t st = ix->stream;
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(w.qoffs.p, offs, 8, cudaMemcpyHostToDevice, st));
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(w.qterms.p, terms, (size_t)nterms * 4, cudaMemcpyHostToDevice, st));
  s = run_batch(ix, ix->ws, 1, w.qoffs.as<uint32_t>(), w.qterms.as<uint32_t>(), max_terms, 1, nullptr,
                nullptr, st, false, mode);
  if (s) return s;
  if ((s = read_status(ix, ix->ws))) return s;
  return copy_final_docids(ix, out_docids, cap, count);
}

}  // extern "C"
