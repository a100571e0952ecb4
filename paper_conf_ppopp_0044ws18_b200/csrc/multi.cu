// multi.cu — one griffin_index handle over G docID-range shards on G GPUs
// (SURVEY.md §8(b) num_gpus, §8(e) partitioning + collective, §8(f) NEXT-2).
//
// Every shard runs the whole single-GPU path (a1-a7) on its device and stream
// — the launches of all shards are issued back to back, so the devices work
// concurrently — and produces its top-k as unique u64 keys built from GLOBAL
// docIDs.  The exchange step (a8) then brings the G runs of every query
// together and the library's k-way merge keeps the global top-k:
//   NCCL_ALLGATHER  ncclAllGather of keys and counts in one NCCL group (one
//                   communicator per device, ncclCommInitAll), merge on device 0
//   PEER            merge_topk_peer_kernel on device 0 reads every shard's runs
//                   in place over NVLink (peer access) — exchange fused into
//                   the merge; cudaMemcpyPeerAsync staging if P2P is unavailable
//   NCCL_SLICED     query-sliced all-to-all with grouped ncclSend/ncclRecv:
//                   device r receives only the runs of query slice r, merges it
//                   and returns that slice of the results
// Exactness of merging per-shard top-k: keys are unique and totally ordered; a
// global top-k key has < k larger keys globally, hence in its own shard, so it
// is in that shard's top-k.
//
// NCCL is loaded at run time (dlopen of $GRIFFIN_NCCL_LIBRARY, else
// libnccl.so.2): the library has no link-time NCCL dependency, and a missing
// NCCL is reported as GRIFFIN_ERR_NCCL when an NCCL exchange is requested.
#include <dlfcn.h>
#include <nccl.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "internal.h"

namespace griffin {

struct NcclApi {
  bool ok = false;
  ncclResult_t (*commInitAll)(ncclComm_t *, int, const int *) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*allGather)(const void *, void *, size_t, ncclDataType_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  ncclResult_t (*send)(const void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*recv)(void *, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*groupStart)() = nullptr;
  ncclResult_t (*groupEnd)() = nullptr;
  const char *(*errStr)(ncclResult_t) = nullptr;
};

static NcclApi &nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    // GRIFFIN_NCCL_LIBRARY first: the process may later load another NCCL user
    // (PyTorch needs its own, newer libnccl.so.2; once a libnccl.so.2 is loaded
    // every later user binds to it), so the binding points it at that copy
    void *h = nullptr;
    if (const char *p = std::getenv("GRIFFIN_NCCL_LIBRARY")) h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
#define GRIFFIN_NCCL_SYM(f, n)                                  \
  api.f = reinterpret_cast<decltype(api.f)>(dlsym(h, n));      \
  if (!api.f) return;
    GRIFFIN_NCCL_SYM(commInitAll, "ncclCommInitAll")
    GRIFFIN_NCCL_SYM(commDestroy, "ncclCommDestroy")
    GRIFFIN_NCCL_SYM(allGather, "ncclAllGather")
    GRIFFIN_NCCL_SYM(send, "ncclSend")
    GRIFFIN_NCCL_SYM(recv, "ncclRecv")
    GRIFFIN_NCCL_SYM(groupStart, "ncclGroupStart")
    GRIFFIN_NCCL_SYM(groupEnd, "ncclGroupEnd")
    GRIFFIN_NCCL_SYM(errStr, "ncclGetErrorString")
#undef GRIFFIN_NCCL_SYM
    api.ok = true;
  });
  return api;
}

#define GRIFFIN_NCCL_TRY(expr)                                                      \
  do {                                                                              \
    ncclResult_t _r = (expr);                                                       \
    if (_r != ncclSuccess) {                                                        \
      ::griffin::set_error(std::string(#expr) + ": " + nccl().errStr(_r));          \
      return GRIFFIN_ERR_NCCL;                                                      \
    }                                                                               \
  } while (0)

struct Cluster {
  int exchange = GRIFFIN_EXCHANGE_PEER;   // resolved mode
  std::vector<int> devs;
  bool distinct = true;   // one shard per device
  bool p2p = true;        // device 0 can load every other shard's memory directly
  std::vector<ncclComm_t> comms;
  std::vector<DevBuf> gkeys, gcnts;                 // per device: exchanged runs
  std::vector<DevBuf> okeys, ocnts, odoc, oscore;   // per device: merged results
  std::vector<cudaEvent_t> done;                    // per shard: its batch finished
  void *h_res = nullptr;                            // pinned [docids | scores | counts | status G]
  size_t h_bytes = 0;
  std::mutex mu;
};

griffin_status cluster_init(griffin_index *cx, int exchange) {
  Cluster *cl = new Cluster();
  cx->cl = cl;
  const uint32_t G = (uint32_t)cx->shards.size();
  for (griffin_index *sh : cx->shards) cl->devs.push_back(sh->device);
  for (uint32_t a = 0; a < G; ++a)
    for (uint32_t b = a + 1; b < G; ++b) cl->distinct &= cl->devs[a] != cl->devs[b];
  cl->exchange = exchange == GRIFFIN_EXCHANGE_AUTO ? GRIFFIN_EXCHANGE_PEER : exchange;
  cl->gkeys.resize(G);
  cl->gcnts.resize(G);
  cl->okeys.resize(G);
  cl->ocnts.resize(G);
  cl->odoc.resize(G);
  cl->oscore.resize(G);
  cl->done.assign(G, nullptr);
  for (uint32_t g = 0; g < G; ++g) {
    DeviceGuard dg(cl->devs[g]);
    GRIFFIN_CUDA_TRY(cudaEventCreateWithFlags(&cl->done[g], cudaEventDisableTiming));
  }
  if (cl->exchange == GRIFFIN_EXCHANGE_PEER) {
    DeviceGuard dg(cl->devs[0]);
    for (uint32_t g = 1; g < G; ++g) {
      if (cl->devs[g] == cl->devs[0]) continue;
      int can = 0;
      cudaDeviceCanAccessPeer(&can, cl->devs[0], cl->devs[g]);
      if (!can) {
        cl->p2p = false;
        continue;
      }
      const cudaError_t e = cudaDeviceEnablePeerAccess(cl->devs[g], 0);
      if (e == cudaErrorPeerAccessAlreadyEnabled) {
        cudaGetLastError();
      } else if (e != cudaSuccess) {
        cudaGetLastError();
        cl->p2p = false;
      }
    }
  } else {   // NCCL exchanges
    if (!nccl().ok) {
      set_error("NCCL exchange requested but libnccl.so.2 could not be loaded");
      return GRIFFIN_ERR_NCCL;
    }
    if (!cl->distinct) {
      set_error("NCCL exchanges need one shard per device (use GRIFFIN_EXCHANGE_PEER)");
      return GRIFFIN_ERR_INVALID_ARG;
    }
    cl->comms.assign(G, nullptr);
    GRIFFIN_NCCL_TRY(nccl().commInitAll(cl->comms.data(), (int)G, cl->devs.data()));
  }
  return GRIFFIN_OK;
}

void cluster_destroy(griffin_index *cx) {
  Cluster *cl = cx->cl;
  if (!cl) return;
  for (size_t g = 0; g < cl->devs.size(); ++g) {
    DeviceGuard dg(cl->devs[g]);
    cudaDeviceSynchronize();
    for (auto *v : {&cl->gkeys, &cl->gcnts, &cl->okeys, &cl->ocnts, &cl->odoc, &cl->oscore})
      if (g < v->size()) (*v)[g].release();
    if (g < cl->done.size() && cl->done[g]) cudaEventDestroy(cl->done[g]);
  }
  for (ncclComm_t c : cl->comms)
    if (c) nccl().commDestroy(c);
  if (cl->h_res) cudaFreeHost(cl->h_res);
  delete cl;
  cx->cl = nullptr;
}

// Query slice owned by device r in the sliced exchange: [r*ceil(nq/G), ...).
static inline void slice_of(uint32_t nq, uint32_t G, uint32_t r, uint32_t *lo, uint32_t *hi) {
  const uint32_t step = (nq + G - 1) / G;
  *lo = std::min(nq, r * step);
  *hi = std::min(nq, (r + 1) * step);
}

griffin_status cluster_query_batch(griffin_index *cx, uint32_t nq, const uint32_t *qoffs,
                                   const uint32_t *terms, uint32_t k, uint32_t *out_docids,
                                   float *out_scores, uint32_t *out_counts) {
  Cluster *cl = cx->cl;
  if (k == 0 || k > GRIFFIN_MAX_K) {
    set_error("k must be in [1, 4096]");
    return GRIFFIN_ERR_INVALID_ARG;
  }
  if (nq == 0) return GRIFFIN_OK;
  std::lock_guard<std::mutex> lk(cl->mu);
  const uint32_t G = (uint32_t)cx->shards.size();
  const uint64_t nt = qoffs[nq];
  const size_t nk = (size_t)nq * k;
  // pinned results on the host: [docids nk | scores nk | counts nq | status G]
  const size_t hb = nk * 8 + (size_t)nq * 4 + (size_t)G * 4 + 64;
  if (cl->h_bytes < hb) {
    if (cl->h_res) cudaFreeHost(cl->h_res);
    cl->h_res = nullptr;
    cl->h_bytes = 0;
    GRIFFIN_CUDA_TRY(cudaMallocHost(&cl->h_res, hb + hb / 4));
    cl->h_bytes = hb + hb / 4;
  }
  uint8_t *hr = static_cast<uint8_t *>(cl->h_res);
  uint32_t *h_doc = reinterpret_cast<uint32_t *>(hr);
  float *h_sc = reinterpret_cast<float *>(hr + nk * 4);
  uint32_t *h_cnt = reinterpret_cast<uint32_t *>(hr + nk * 8);
  int *h_status = reinterpret_cast<int *>(hr + nk * 8 + (size_t)nq * 4);
  // ---- a1-a7 on every shard (asynchronous; the devices run concurrently).
  // Each shard's ~50 launches are issued by its own host thread, so no device
  // waits for the host to finish issuing the other shards' work.
  auto launch_shard = [&](uint32_t g) -> griffin_status {
    griffin_index *sh = cx->shards[g];
    DeviceGuard dg(sh->device);
    Workspace &w = sh->ws;
    uint32_t mt = 1;
    griffin_status s = reserve_for(sh, w, nq, qoffs, terms, k, &mt);
    if (s) return s;
    GRIFFIN_CUDA_TRY(w.qoffs.reserve(((size_t)nq + 1) * 4));
    GRIFFIN_CUDA_TRY(w.qterms.reserve(std::max<uint64_t>(nt, 1) * 4));
    GRIFFIN_CUDA_TRY(w.keys.reserve(nk * 8));
    GRIFFIN_CUDA_TRY(w.counts.reserve((size_t)nq * 4));
    const size_t b_in = ((size_t)nq + 1 + nt) * 4;
    if ((s = ensure_pinned_ws(w, b_in))) return s;
    uint8_t *hp = static_cast<uint8_t *>(w.h_pinned);
    std::memcpy(hp, qoffs, ((size_t)nq + 1) * 4);
    std::memcpy(hp + ((size_t)nq + 1) * 4, terms, nt * 4);
    cudaStream_t st = sh->stream;
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(w.qoffs.p, hp, ((size_t)nq + 1) * 4, cudaMemcpyHostToDevice, st));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(w.qterms.p, hp + ((size_t)nq + 1) * 4, nt * 4,
                                     cudaMemcpyHostToDevice, st));
    if ((s = run_batch(sh, w, nq, w.qoffs.as<uint32_t>(), w.qterms.as<uint32_t>(), mt, k,
                       w.keys.as<uint64_t>(), w.counts.as<uint32_t>(), st, true, sh->mode)))
      return s;
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h_status + g, w.scal.as<unsigned long long>() + kScalStatus,
                                     sizeof(int), cudaMemcpyDeviceToHost, st));
    GRIFFIN_CUDA_TRY(cudaEventRecord(cl->done[g], st));
    return GRIFFIN_OK;
  };
  {
    std::vector<griffin_status> st_g(G, GRIFFIN_OK);
    std::vector<std::string> err_g(G);
    std::vector<std::thread> th;
    for (uint32_t g = 1; g < G; ++g)
      th.emplace_back([&, g] {
        st_g[g] = launch_shard(g);
        if (st_g[g]) err_g[g] = griffin_last_error();   // thread-local message
      });
    st_g[0] = launch_shard(0);
    if (st_g[0]) err_g[0] = griffin_last_error();
    for (auto &t : th) t.join();
    for (uint32_t g = 0; g < G; ++g)
      if (st_g[g]) {
        set_error("shard " + std::to_string(g) + ": " + err_g[g]);
        return st_g[g];
      }
  }
  // ---- a8: exchange the per-shard top-k runs and merge them ----
  griffin_index *s0 = cx->shards[0];
  const int d0 = cl->devs[0];
  cudaStream_t st0 = s0->stream;
  auto reserve_out = [&](uint32_t r, size_t m) -> griffin_status {
    DeviceGuard dg(cl->devs[r]);
    GRIFFIN_CUDA_TRY(cl->okeys[r].reserve(std::max<size_t>(m * k, 1) * 8));
    GRIFFIN_CUDA_TRY(cl->ocnts[r].reserve(std::max<size_t>(m, 1) * 4));
    GRIFFIN_CUDA_TRY(cl->odoc[r].reserve(std::max<size_t>(m * k, 1) * 4));
    GRIFFIN_CUDA_TRY(cl->oscore[r].reserve(std::max<size_t>(m * k, 1) * 4));
    return GRIFFIN_OK;
  };
  griffin_status s = GRIFFIN_OK;
  if (cl->exchange == GRIFFIN_EXCHANGE_NCCL_SLICED) {
    std::vector<uint32_t> lo(G), hi(G);
    for (uint32_t r = 0; r < G; ++r) {
      slice_of(nq, G, r, &lo[r], &hi[r]);
      const size_t m = hi[r] - lo[r];
      if ((s = reserve_out(r, m))) return s;
      DeviceGuard dg(cl->devs[r]);
      GRIFFIN_CUDA_TRY(cl->gkeys[r].reserve(std::max<size_t>((size_t)G * m * k, 1) * 8));
      GRIFFIN_CUDA_TRY(cl->gcnts[r].reserve(std::max<size_t>((size_t)G * m, 1) * 4));
    }
    GRIFFIN_NCCL_TRY(nccl().groupStart());
    for (uint32_t g = 0; g < G; ++g) {
      griffin_index *sh = cx->shards[g];
      for (uint32_t r = 0; r < G; ++r) {
        const size_t m = hi[r] - lo[r];
        if (!m) continue;
        GRIFFIN_NCCL_TRY(nccl().send(sh->ws.keys.as<uint64_t>() + (size_t)lo[r] * k, m * k,
                                     ncclUint64, (int)r, cl->comms[g], sh->stream));
        GRIFFIN_NCCL_TRY(nccl().send(sh->ws.counts.as<uint32_t>() + lo[r], m, ncclUint32, (int)r,
                                     cl->comms[g], sh->stream));
        GRIFFIN_NCCL_TRY(nccl().recv(cl->gkeys[r].as<uint64_t>() + (size_t)g * m * k, m * k,
                                     ncclUint64, (int)g, cl->comms[r], cx->shards[r]->stream));
        GRIFFIN_NCCL_TRY(nccl().recv(cl->gcnts[r].as<uint32_t>() + (size_t)g * m, m, ncclUint32,
                                     (int)g, cl->comms[r], cx->shards[r]->stream));
      }
    }
    GRIFFIN_NCCL_TRY(nccl().groupEnd());
    for (uint32_t r = 0; r < G; ++r) {
      const size_t m = hi[r] - lo[r];
      if (!m) continue;
      griffin_index *sh = cx->shards[r];
      DeviceGuard dg(sh->device);
      if ((s = launch_merge_topk(sh, G, (uint32_t)m, k, cl->gkeys[r].as<uint64_t>(),
                                 cl->gcnts[r].as<uint32_t>(), cl->okeys[r].as<uint64_t>(),
                                 cl->ocnts[r].as<uint32_t>(), sh->stream)))
        return s;
      if ((s = launch_keys_to_results(sh, (uint32_t)m, k, cl->okeys[r].as<uint64_t>(),
                                      cl->ocnts[r].as<uint32_t>(), cl->odoc[r].as<uint32_t>(),
                                      cl->oscore[r].as<float>(), sh->stream)))
        return s;
      GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h_doc + (size_t)lo[r] * k, cl->odoc[r].p, m * k * 4,
                                       cudaMemcpyDeviceToHost, sh->stream));
      GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h_sc + (size_t)lo[r] * k, cl->oscore[r].p, m * k * 4,
                                       cudaMemcpyDeviceToHost, sh->stream));
      GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h_cnt + lo[r], cl->ocnts[r].p, m * 4,
                                       cudaMemcpyDeviceToHost, sh->stream));
    }
  } else {
    if ((s = reserve_out(0, nq))) return s;
    if (cl->exchange == GRIFFIN_EXCHANGE_NCCL_ALLGATHER) {
      for (uint32_t g = 0; g < G; ++g) {
        DeviceGuard dg(cl->devs[g]);
        GRIFFIN_CUDA_TRY(cl->gkeys[g].reserve((size_t)G * nk * 8));
        GRIFFIN_CUDA_TRY(cl->gcnts[g].reserve((size_t)G * nq * 4));
      }
      GRIFFIN_NCCL_TRY(nccl().groupStart());
      for (uint32_t g = 0; g < G; ++g) {
        griffin_index *sh = cx->shards[g];
        GRIFFIN_NCCL_TRY(nccl().allGather(sh->ws.keys.p, cl->gkeys[g].p, nk, ncclUint64,
                                          cl->comms[g], sh->stream));
        GRIFFIN_NCCL_TRY(nccl().allGather(sh->ws.counts.p, cl->gcnts[g].p, nq, ncclUint32,
                                          cl->comms[g], sh->stream));
      }
      GRIFFIN_NCCL_TRY(nccl().groupEnd());
      DeviceGuard dg(d0);
      if ((s = launch_merge_topk(s0, G, nq, k, cl->gkeys[0].as<uint64_t>(),
                                 cl->gcnts[0].as<uint32_t>(), cl->okeys[0].as<uint64_t>(),
                                 cl->ocnts[0].as<uint32_t>(), st0)))
        return s;
    } else {   // PEER: merge on device 0 straight from every shard's buffers
      DeviceGuard dg(d0);
      std::vector<const uint64_t *> kp(G);
      std::vector<const uint32_t *> cp(G);
      if (!cl->p2p) {
        GRIFFIN_CUDA_TRY(cl->gkeys[0].reserve((size_t)G * nk * 8));
        GRIFFIN_CUDA_TRY(cl->gcnts[0].reserve((size_t)G * nq * 4));
      }
      for (uint32_t g = 0; g < G; ++g) {
        griffin_index *sh = cx->shards[g];
        GRIFFIN_CUDA_TRY(cudaStreamWaitEvent(st0, cl->done[g], 0));
        kp[g] = sh->ws.keys.as<uint64_t>();
        cp[g] = sh->ws.counts.as<uint32_t>();
        if (!cl->p2p && cl->devs[g] != d0) {   // no P2P path: stage the runs on device 0
          uint64_t *dk = cl->gkeys[0].as<uint64_t>() + (size_t)g * nk;
          uint32_t *dc = cl->gcnts[0].as<uint32_t>() + (size_t)g * nq;
          GRIFFIN_CUDA_TRY(cudaMemcpyPeerAsync(dk, d0, kp[g], cl->devs[g], nk * 8, st0));
          GRIFFIN_CUDA_TRY(cudaMemcpyPeerAsync(dc, d0, cp[g], cl->devs[g], (size_t)nq * 4, st0));
          kp[g] = dk;
          cp[g] = dc;
        }
      }
      if ((s = launch_merge_topk_peer(s0, G, nq, k, kp.data(), cp.data(),
                                      cl->okeys[0].as<uint64_t>(), cl->ocnts[0].as<uint32_t>(),
                                      st0)))
        return s;
    }
    DeviceGuard dg(d0);
    if ((s = launch_keys_to_results(s0, nq, k, cl->okeys[0].as<uint64_t>(),
                                    cl->ocnts[0].as<uint32_t>(), cl->odoc[0].as<uint32_t>(),
                                    cl->oscore[0].as<float>(), st0)))
      return s;
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h_doc, cl->odoc[0].p, nk * 4, cudaMemcpyDeviceToHost, st0));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h_sc, cl->oscore[0].p, nk * 4, cudaMemcpyDeviceToHost, st0));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(h_cnt, cl->ocnts[0].p, (size_t)nq * 4, cudaMemcpyDeviceToHost, st0));
  }
  // ---- wait for every device; device-side errors of any shard ----
  for (uint32_t g = 0; g < G; ++g) {
    DeviceGuard dg(cl->devs[g]);
    GRIFFIN_CUDA_TRY(cudaStreamSynchronize(cx->shards[g]->stream));
  }
  int bad = 0;
  for (uint32_t g = 0; g < G; ++g) {
    if (!h_status[g]) continue;
    bad |= h_status[g];
    griffin_index *sh = cx->shards[g];
    DeviceGuard dg(sh->device);
    GRIFFIN_CUDA_TRY(cudaMemsetAsync(sh->ws.scal.as<unsigned long long>() + kScalStatus, 0, 8,
                                     sh->stream));
    GRIFFIN_CUDA_TRY(cudaStreamSynchronize(sh->stream));
  }
  if (bad & kStatusOverflow) {
    set_error("query workspace overflow (reserve more with griffin_reserve)");
    return GRIFFIN_ERR_OOM;
  }
  if (bad) {
    set_error("invalid query term(s) detected on the device");
    return GRIFFIN_ERR_INVALID_ARG;
  }
  par_memcpy(out_docids, h_doc, nk * 4);
  par_memcpy(out_scores, h_sc, nk * 4);
  std::memcpy(out_counts, h_cnt, (size_t)nq * 4);
  return GRIFFIN_OK;
}

}  // namespace griffin
