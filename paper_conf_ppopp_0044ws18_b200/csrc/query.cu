// query.cu — batched conjunctive query evaluation on one shard (sm_100a).
//
// Per batch:
//   plan_queries   dedupe terms, SvS order by (global df asc, termID asc)
//                  (P:232-240), region bounds            [thread/query]
//   for each SvS round r = 1..m-1 ("repeats until all the lists have
//   been incorporated or the list of matching docIDs is empty"):
//     plan_round   merge-vs-gallop per query: gallop iff |S| > T*|R|
//                  (P:620-625), unit counts                [thread/query]
//     scan         unit offsets
//     intersect    persistent warps over units:
//                    merge  — coarse merge path over the block heads (skip
//                             pointers, Fig. 2) of R and S gives each unit a docID
//                             range; its blocks are EF-decoded by the warp
//                             (Alg. 1) into smem, and a fine merge path splits the
//                             two tiles across the 32 lanes (Figs. 5-6,
//                             P:634-722); each lane merges its partition serially
//                    gallop — each R element finds its S block by binary
//                             search over the skip pointers; only the distinct
//                             touched blocks are decoded (Fig. 9)
//                  survivors get their BM25 partial score fused in
//     compact      per query, units' survivors -> the next sorted intermediate
//   topk           per query: bitonic sort (<= 4096) or radix select on unique
//                  keys (score_bits << 32 | ~docID) (§3.1.3)
#include <algorithm>
#include <cstdio>

#include "internal.h"
#include "scan.cuh"

namespace griffin {

constexpr int kIntersectThreads = 256;
constexpr int kWarpsPerCta = kIntersectThreads / 32;
constexpr uint32_t kTopkSmem = 4096;
constexpr int kTopkThreads = 512;

// ------------------------------------------------------------------- planning

__global__ void plan_queries_kernel(DevIndex ix, uint32_t nq, const uint32_t *__restrict__ qoffs,
                                    const uint32_t *__restrict__ qterms, uint32_t *plan_terms,
                                    uint32_t *plan_m, uint32_t *cap, uint32_t *rcount,
                                    uint8_t *rsel, unsigned long long *scal) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q == 0) {
    scal[kScalTotals] = 0;
    scal[kScalTotals + 1] = 0;
  }
  // (totals are accumulated by plan_totals_kernel, launched after this one)
  if (q >= nq) return;
  const uint32_t a = qoffs[q], e = qoffs[q + 1];
  uint32_t ts[kMaxTerms];
  uint32_t m = 0;
  int bad = (e <= a) ? kStatusBadTerm : 0;
  for (uint32_t i = a; i < e && !bad; ++i) {
    const uint32_t t = qterms[i];
    if (t >= ix.num_terms) {
      bad = kStatusBadTerm;
      break;
    }
    bool dup = false;
    for (uint32_t j = 0; j < m; ++j) dup |= (ts[j] == t);
    if (dup) continue;
    if (m == (uint32_t)kMaxTerms) {
      bad = kStatusTooManyTerms;
      break;
    }
    ts[m++] = t;
  }
  if (bad) {
    atomicOr(reinterpret_cast<int *>(scal + kScalStatus), bad);
    m = 0;
  }
  // insertion sort by (global df asc, termID asc)
  uint64_t key[kMaxTerms];
  for (uint32_t i = 0; i < m; ++i) key[i] = ((uint64_t)ix.terms[ts[i]].df_global << 32) | ts[i];
  for (uint32_t i = 1; i < m; ++i) {
    uint64_t kx = key[i];
    uint32_t j = i;
    while (j > 0 && key[j - 1] > kx) {
      key[j] = key[j - 1];
      --j;
    }
    key[j] = kx;
  }
  uint32_t c = 0;
  if (m) {
    bool empty = false;
    for (uint32_t i = 0; i < m; ++i) empty |= ix.terms[(uint32_t)key[i]].df_local == 0;
    const uint32_t d0 = ix.terms[(uint32_t)key[0]].df_local;
    c = empty ? 0u : (m == 1 ? d0 : min(d0, ix.terms[(uint32_t)key[1]].df_local));
  }
  for (uint32_t i = 0; i < m; ++i) plan_terms[q * kMaxTerms + i] = (uint32_t)key[i];
  plan_m[q] = m;
  cap[q] = c;
  rcount[q] = 0;
  rsel[q] = 0;
}

// Σ cap and Σ unit bounds (bound = nblocks(t0) + max_r nblocks(t_r)), checked
// against the reserved workspace before any round runs.
__global__ void plan_totals_kernel(DevIndex ix, uint32_t nq, const uint32_t *plan_terms,
                                   const uint32_t *plan_m, const uint32_t *cap,
                                   unsigned long long *scal) {
  unsigned long long c = 0, u = 0;
  for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < nq; q += gridDim.x * blockDim.x) {
    const uint32_t m = plan_m[q];
    if (!m || !cap[q]) continue;
    c += cap[q];
    uint32_t mx = 0;
    for (uint32_t i = 1; i < m; ++i) mx = max(mx, ix.terms[plan_terms[q * kMaxTerms + i]].nblocks);
    u += (unsigned long long)ix.terms[plan_terms[q * kMaxTerms]].nblocks + mx;
  }
  for (int d = 16; d; d >>= 1) {
    c += __shfl_xor_sync(0xffffffffu, c, d);
    u += __shfl_xor_sync(0xffffffffu, u, d);
  }
  if ((threadIdx.x & 31) == 0) {
    if (c) atomicAdd(scal + kScalTotals, c);
    if (u) atomicAdd(scal + kScalTotals + 1, u);
  }
}

__global__ void plan_round_kernel(DevIndex ix, RoundArgs a, uint32_t *qunits) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  const bool overflow = a.scal[kScalTotals] > a.entry_cap || a.scal[kScalTotals + 1] > a.unit_cap;
  if (q == 0) {
    a.scal[kScalBump] = 0;
    a.scal[kScalUnitCtr] = 0;
    if (overflow) atomicOr(reinterpret_cast<int *>(a.scal + kScalStatus), kStatusOverflow);
  }
  if (q >= a.nq) return;
  uint32_t mode = kModeNone, units = 0;
  const uint32_t m = a.plan_m[q];
  if (!overflow && a.cap[q] > 0) {
    const TermInfo t0 = ix.terms[a.plan_terms[q * kMaxTerms]];
    uint64_t nR = 0;
    uint32_t nbR = 0;
    bool pair = false;
    if (a.round == 1) {
      if (m == 1) {
        mode = kModeAll;
        units = t0.nblocks;
      } else {
        nR = t0.df_local;
        nbR = t0.nblocks;
        pair = true;
      }
    } else if (m > a.round && a.rcount[q] > 0) {
      nR = a.rcount[q];
      nbR = (uint32_t)((nR + ix.B - 1) / ix.B);
      pair = true;
    }
    if (pair) {
      const TermInfo tS = ix.terms[a.plan_terms[q * kMaxTerms + a.round]];
      const bool gallop = a.forced_mode == 2 ||
                          (a.forced_mode == 0 && (uint64_t)tS.df_local > (uint64_t)a.T * nR);
      mode = gallop ? kModeGallop : kModeMerge;
      units = gallop ? nbR : (nbR + tS.nblocks + a.D - 1) / a.D;
    }
  }
  a.qmode[q] = mode;
  qunits[q] = units;
}

// ------------------------------------------------------------------- intersect

struct Acc {
  unsigned long long alg = 0, pay = 0, post = 0, surv = 0;
};

struct WarpSmem {
  uint32_t *scratch;  // EF payload staging (16-B aligned)
  uint32_t *tile;     // decoded values, (D+2)*B
  uint32_t *match;    // per R-tile element: S posting position or kNone, (D+1)*B
};

__host__ __device__ inline uint32_t scratch_words(uint32_t B) {
  return ((B * 34u) / 32u + 24u + 3u) & ~3u;
}
__host__ __device__ inline uint32_t warp_smem_words(uint32_t B, uint32_t D) {
  return scratch_words(B) + (((D + 2) * B + (D + 1) * B + 3u) & ~3u);
}

// Load R "block" k into dst.  Compressed R: EF decode; intermediate R: copy the
// docIDs of chunk k (B entries).  Returns the element count.
template <bool RC>
__device__ __forceinline__ uint32_t load_r_block(const DevIndex &ix, const TermInfo &tR,
                                                 const uint2 *Rq, uint32_t nR, uint32_t k,
                                                 uint32_t *dst, uint32_t *scratch,
                                                 uint32_t *pay = nullptr) {
  if (RC) return warp_decode_block(ix, (uint64_t)tR.block0 + k, dst, scratch, pay);
  const uint32_t lane = lane_id();
  const uint32_t s = k * ix.B;
  const uint32_t n = min(ix.B, nR - s);
  for (uint32_t i = lane; i < n; i += 32) dst[i] = Rq[s + i].x;
  __syncwarp();
  if (pay) *pay = n * 8u;
  return n;
}

// Ordered emission of the matched R-tile elements [ia, ib) (two passes: count,
// then write at a bump-allocated offset).  KIND 0: round 1 (s = w_R + w_S);
// KIND 1: later round (s = s_prev + w_S); KIND 2: single-term (s = w_R).
template <int KIND>
__device__ void emit_unit(const DevIndex &ix, const RoundArgs &a, uint32_t u, const TermInfo &tR,
                          const TermInfo &tS, const uint2 *Rq, const uint32_t *tile,
                          const uint32_t *match, uint32_t ia, uint32_t ib, uint32_t posR0,
                          Acc &acc) {
  const uint32_t lane = lane_id(), lt = lanemask_lt();
  uint32_t cnt = 0;
  if (KIND == 2) {
    cnt = ib - ia;
  } else {
    for (uint32_t c0 = ia; c0 < ib; c0 += 32) {
      const uint32_t i = c0 + lane;
      cnt += __popc(__ballot_sync(0xffffffffu, i < ib && match[i] != kNone));
    }
  }
  unsigned long long off = 0;
  if (lane == 0 && cnt) off = atomicAdd(a.scal + kScalBump, (unsigned long long)cnt);
  off = __shfl_sync(0xffffffffu, off, 0);
  if (off + cnt > a.entry_cap) {
    if (lane == 0) atomicOr(reinterpret_cast<int *>(a.scal + kScalStatus), kStatusOverflow);
    cnt = 0;
  }
  if (cnt) {
    uint32_t run = 0;
    for (uint32_t c0 = ia; c0 < ib; c0 += 32) {
      const uint32_t i = c0 + lane;
      const bool p = i < ib && (KIND == 2 || match[i] != kNone);
      const uint32_t bal = __ballot_sync(0xffffffffu, p);
      if (p) {
        const uint32_t doc = tile[i];
        const float nrm = __ldg(ix.norm + doc);
        float s;
        if (KIND == 2) {
          s = bm25_w(tR.idf, tf_lookup(ix, tR, posR0 + i), nrm, ix.k1p1);
        } else {
          const float wS = bm25_w(tS.idf, tf_lookup(ix, tS, match[i]), nrm, ix.k1p1);
          if (KIND == 0) {
            s = bm25_w(tR.idf, tf_lookup(ix, tR, posR0 + i), nrm, ix.k1p1);  // first term: s = w
            s = __fadd_rn(s, wS);
          } else {
            s = __fadd_rn(__uint_as_float(Rq[posR0 + i].y), wS);
          }
        }
        a.bump[off + run + __popc(bal & lt)] = make_uint2(doc, __float_as_uint(s));
      }
      run += __popc(bal);
    }
  }
  if (lane == 0) {
    a.unit_off[u] = off;
    a.unit_cnt[u] = cnt;
    acc.surv += cnt;
    acc.alg += (unsigned long long)cnt * (KIND == 0 ? 20u : 16u);
  }
}

template <bool RC>
__global__ void __launch_bounds__(kIntersectThreads) intersect_kernel(DevIndex ix, RoundArgs a) {
  extern __shared__ uint4 smem4[];
  const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
  const uint32_t B = ix.B, D = a.D;
  uint32_t *wbase = reinterpret_cast<uint32_t *>(smem4) + wid * warp_smem_words(B, D);
  WarpSmem sm;
  sm.scratch = wbase;
  sm.tile = wbase + scratch_words(B);
  sm.match = sm.tile + (D + 2) * B;
  const uint64_t *ubase = a.unit_base;
  const uint64_t total = ubase[a.nq];
  Acc acc;
  for (;;) {
    unsigned long long u = 0;
    if (lane == 0) u = atomicAdd(a.scal + kScalUnitCtr, 1ull);
    u = __shfl_sync(0xffffffffu, u, 0);
    if (u >= total) break;
    // query of this unit: last q with ubase[q] <= u
    uint32_t lo = 0, hi = a.nq;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (ubase[mid] <= u) lo = mid; else hi = mid;
    }
    const uint32_t q = lo;
    const uint32_t lu = (uint32_t)(u - ubase[q]);
    const uint32_t mode = a.qmode[q];
    const uint32_t *pt = a.plan_terms + (size_t)q * kMaxTerms;
    const TermInfo tR = ix.terms[pt[0]];
    const uint2 *Rq = RC ? nullptr : a.rprev + a.cap_off[q];
    const uint32_t nR = RC ? tR.df_local : a.rcount[q];
    const uint32_t nbR = RC ? tR.nblocks : (nR + B - 1) / B;

    if (RC && mode == kModeAll) {  // single-term query: the whole list is the result
      uint32_t pay = 0;
      const uint32_t n = warp_decode_block(ix, (uint64_t)tR.block0 + lu, sm.tile, sm.scratch, &pay);
      if (lane == 0) {
        acc.pay += pay;
        acc.post += n;
        acc.alg += pay + 8u;
      }
      emit_unit<2>(ix, a, (uint32_t)u, tR, tR, nullptr, sm.tile, nullptr, 0, n, lu * B, acc);
      continue;
    }
    const TermInfo tS = ix.terms[pt[a.round]];
    const uint32_t *fS = ix.first + tS.block0;
    const uint32_t nbS = tS.nblocks;

    if (mode == kModeMerge) {
      // ---- coarse merge path over the block heads (no decode) ----
      auto hR = [&](uint32_t i) -> uint32_t {
        return RC ? __ldg(ix.first + tR.block0 + i) : Rq[i * B].x;
      };
      auto hS = [&](uint32_t j) -> uint32_t { return __ldg(fS + j); };
      const uint32_t tot = nbR + nbS;
      const uint32_t d0 = lu * D, d1 = min(d0 + D, tot);
      uint32_t si = 0, sj = 0;
      if (lane < 2) merge_path_split(hR, nbR, hS, nbS, lane ? d1 : d0, false, &si, &sj);
      const uint32_t i0 = __shfl_sync(0xffffffffu, si, 0), j0 = __shfl_sync(0xffffffffu, sj, 0);
      const uint32_t i1 = __shfl_sync(0xffffffffu, si, 1), j1 = __shfl_sync(0xffffffffu, sj, 1);
      const uint64_t INF = 1ull << 32;
      uint64_t lo_v = 0, hi_v = INF;
      if (lane == 0 && d0 > 0)
        lo_v = min(i0 < nbR ? (uint64_t)hR(i0) : INF, j0 < nbS ? (uint64_t)hS(j0) : INF);
      if (lane == 1 && d1 < tot)
        hi_v = min(i1 < nbR ? (uint64_t)hR(i1) : INF, j1 < nbS ? (uint64_t)hS(j1) : INF);
      lo_v = __shfl_sync(0xffffffffu, lo_v, 0);
      hi_v = __shfl_sync(0xffffffffu, hi_v, 1);
      const uint32_t rb0 = i0 ? i0 - 1 : 0, rb1 = i1;
      const uint32_t sb0 = j0 ? j0 - 1 : 0, sb1 = j1;
      // accounting: blocks whose head lies in this unit
      if (lane == 0) {
        for (uint32_t k = i0; k < i1; ++k) {
          uint32_t pay;
          if (RC) {
            const uint2 m = ix.meta[(uint64_t)tR.block0 + k];
            pay = ((low_words(meta_n(m.y), meta_b(m.y)) + meta_hw(m.y) + 3u) >> 2) * 16u;
            acc.post += meta_n(m.y);
            acc.pay += pay;
            acc.alg += pay + 8u;
          } else {
            acc.alg += (unsigned long long)min(B, nR - k * B) * 8u;
          }
        }
        for (uint32_t k = j0; k < j1; ++k) {
          const uint2 m = ix.meta[(uint64_t)tS.block0 + k];
          const uint32_t pay = ((low_words(meta_n(m.y), meta_b(m.y)) + meta_hw(m.y) + 3u) >> 2) * 16u;
          acc.post += meta_n(m.y);
          acc.pay += pay;
          acc.alg += pay + 8u;
        }
      }
      if (rb1 <= rb0 || sb1 <= sb0 || lo_v >= hi_v) {
        if (lane == 0) {
          a.unit_off[u] = 0;
          a.unit_cnt[u] = 0;
        }
        continue;
      }
      // ---- decode the unit's blocks into the smem tiles ----
      uint32_t nRt = 0;
      for (uint32_t k = rb0; k < rb1; ++k)
        nRt += load_r_block<RC>(ix, tR, Rq, nR, k, sm.tile + nRt, sm.scratch);
      uint32_t *tileS = sm.tile + nRt;
      uint32_t nSt = 0;
      for (uint32_t k = sb0; k < sb1; ++k)
        nSt += warp_decode_block(ix, (uint64_t)tS.block0 + k, tileS + nSt, sm.scratch);
      // ranges inside [lo, hi)
      uint32_t r_lo = 0;
      if (lane == 0) r_lo = lower_bound_s(sm.tile, 0, nRt, lo_v);
      if (lane == 1) r_lo = lower_bound_s(sm.tile, 0, nRt, hi_v);
      if (lane == 2) r_lo = lower_bound_s(tileS, 0, nSt, lo_v);
      if (lane == 3) r_lo = lower_bound_s(tileS, 0, nSt, hi_v);
      const uint32_t ra = __shfl_sync(0xffffffffu, r_lo, 0), rb = __shfl_sync(0xffffffffu, r_lo, 1);
      const uint32_t sa = __shfl_sync(0xffffffffu, r_lo, 2), sb = __shfl_sync(0xffffffffu, r_lo, 3);
      for (uint32_t i = ra + lane; i < rb; i += 32) sm.match[i] = kNone;
      __syncwarp();
      const uint32_t nr = rb - ra, ns = sb - sa;
      if (nr && ns) {
        // ---- fine merge path: lane l owns diagonals [l*L, (l+1)*L) ----
        const uint32_t *A = sm.tile + ra, *Bv = tileS + sa;
        auto gA = [&](uint32_t i) -> uint32_t { return A[i]; };
        auto gB = [&](uint32_t j) -> uint32_t { return Bv[j]; };
        const uint32_t tot2 = nr + ns, L = (tot2 + 31) >> 5;
        const uint32_t ds = min(lane * L, tot2), de = min(ds + L, tot2);
        uint32_t is, js, ie, je;
        merge_path_split(gA, nr, gB, ns, ds, true, &is, &js);
        merge_path_split(gA, nr, gB, ns, de, true, &ie, &je);
        const uint32_t posS0 = sb0 * B + sa;
        while (is < ie && js < je) {
          const uint32_t x = A[is], y = Bv[js];
          if (x == y) {
            sm.match[ra + is] = posS0 + js;
            ++is;
            ++js;
          } else if (x < y) {
            ++is;
          } else {
            ++js;
          }
        }
      }
      __syncwarp();
      if (RC)
        emit_unit<0>(ix, a, (uint32_t)u, tR, tS, Rq, sm.tile, sm.match, ra, rb, rb0 * B, acc);
      else
        emit_unit<1>(ix, a, (uint32_t)u, tR, tS, Rq, sm.tile, sm.match, ra, rb, rb0 * B, acc);
      __syncwarp();
    } else {
      // ---- gallop: R chunk lu, skip-pointer search into S ----
      uint32_t *tileR = sm.tile, *tileS = sm.tile + B;
      int *kidx = reinterpret_cast<int *>(sm.tile + 2 * B);
      uint32_t payR = 0;
      const uint32_t n = load_r_block<RC>(ix, tR, Rq, nR, lu, tileR, sm.scratch, &payR);
      if (lane == 0) {
        acc.alg += payR + (RC ? 8u : 0u);
        if (RC) {
          acc.pay += payR;
          acc.post += n;
        }
      }
      uint32_t kk = 0;
      if (lane == 0) kk = upper_bound_g(fS, 0, nbS, tileR[0]);
      if (lane == 1) kk = upper_bound_g(fS, 0, nbS, tileR[n - 1]);
      const uint32_t k_lo = __shfl_sync(0xffffffffu, kk, 0), k_hi = __shfl_sync(0xffffffffu, kk, 1);
      for (uint32_t e = lane; e < n; e += 32) {
        kidx[e] = (int)upper_bound_g(fS, k_lo, k_hi, tileR[e]) - 1;
        sm.match[e] = kNone;
      }
      __syncwarp();
      const int k_first = kidx[0];
      // skip R elements below S's first docID (no block)
      uint32_t e0 = 0;
      while (e0 < n) {
        const uint32_t e = e0 + lane;
        const uint32_t bal = __ballot_sync(0xffffffffu, e < n && kidx[e] < 0);
        if (bal == 0xffffffffu) {
          e0 += 32;
          continue;
        }
        e0 += __popc(bal);
        break;
      }
      while (e0 < n) {
        const int kb = kidx[e0];
        uint32_t pay = 0;
        const uint32_t ns = warp_decode_block(ix, (uint64_t)tS.block0 + kb, tileS, sm.scratch, &pay);
        if (lane == 0 && !(lu > 0 && kb == k_first)) {
          acc.pay += pay;
          acc.post += ns;
          acc.alg += pay + 8u;
        }
        uint32_t e = e0;
        for (;;) {
          const uint32_t ee = e + lane;
          const bool in = ee < n && kidx[ee] == kb;
          if (in) {
            const uint32_t x = tileR[ee];
            const uint32_t p = lower_bound_s(tileS, 0, ns, x);
            if (p < ns && tileS[p] == x) sm.match[ee] = (uint32_t)kb * B + p;
          }
          const uint32_t bal = __ballot_sync(0xffffffffu, in);
          if (bal == 0xffffffffu) {
            e += 32;
            continue;
          }
          e += __popc(bal);
          break;
        }
        e0 = e;
        __syncwarp();
      }
      __syncwarp();
      if (RC)
        emit_unit<0>(ix, a, (uint32_t)u, tR, tS, Rq, tileR, sm.match, 0, n, lu * B, acc);
      else
        emit_unit<1>(ix, a, (uint32_t)u, tR, tS, Rq, tileR, sm.match, 0, n, lu * B, acc);
      __syncwarp();
    }
  }
  if (lane == 0) {
    if (acc.alg) atomicAdd(a.scal + kScalCounters + 0, acc.alg);
    if (acc.pay) atomicAdd(a.scal + kScalCounters + 1, acc.pay);
    if (acc.post) atomicAdd(a.scal + kScalCounters + 2, acc.post);
    if (acc.surv) atomicAdd(a.scal + kScalCounters + 3, acc.surv);
  }
}

// ------------------------------------------------------------------- compaction

__global__ void compact_kernel(RoundArgs a) {
  const uint32_t lane = lane_id();
  const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
  const uint64_t *ubase = a.unit_base;
  for (uint32_t q = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); q < a.nq; q += nwarps) {
    if (a.qmode[q] == kModeNone) {
      // inactive this round: a query that ran out of terms keeps its result; one
      // whose plan was empty keeps count 0
      continue;
    }
    const uint64_t u0 = ubase[q], u1 = ubase[q + 1];
    uint2 *dst = a.rnext + a.cap_off[q];
    uint32_t run = 0;
    for (uint64_t c0 = u0; c0 < u1; c0 += 32) {
      const uint64_t uu = c0 + lane;
      const uint32_t cnt = uu < u1 ? a.unit_cnt[uu] : 0u;
      const uint64_t off = uu < u1 ? a.unit_off[uu] : 0ull;
      const uint32_t incl = warp_incl_scan(cnt);
      const uint32_t excl = incl - cnt;
      const uint32_t nu = (uint32_t)((u1 - c0) < 32 ? (u1 - c0) : 32);
      for (uint32_t j = 0; j < nu; ++j) {
        const uint32_t cj = __shfl_sync(0xffffffffu, cnt, j);
        const uint64_t oj = __shfl_sync(0xffffffffu, off, j);
        const uint32_t ej = __shfl_sync(0xffffffffu, excl, j);
        for (uint32_t i = lane; i < cj; i += 32) dst[run + ej + i] = a.bump[oj + i];
      }
      run += __shfl_sync(0xffffffffu, incl, 31);
    }
    if (lane == 0) {
      a.rcount[q] = run;
      a.rsel[q] = (uint8_t)(a.round & 1u);
    }
  }
}

// ------------------------------------------------------------------- top-k

__device__ __forceinline__ uint64_t make_key(uint2 e, uint32_t doc_base) {
  return ((uint64_t)e.y << 32) | (uint64_t)(0xFFFFFFFFu - (doc_base + e.x));
}

// in-smem bitonic sort, descending, n a power of two
__device__ void bitonic_desc(uint64_t *s, uint32_t n) {
  for (uint32_t size = 2; size <= n; size <<= 1) {
    for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
      for (uint32_t t = threadIdx.x; t < (n >> 1); t += blockDim.x) {
        const uint32_t lo = 2 * stride * (t / stride) + (t % stride);
        const uint32_t hi = lo + stride;
        const bool desc = (lo & size) == 0;
        const uint64_t x = s[lo], y = s[hi];
        if ((x < y) == desc) {
          s[lo] = y;
          s[hi] = x;
        }
      }
      __syncthreads();
    }
  }
}

__global__ void __launch_bounds__(kTopkThreads) topk_kernel(DevIndex ix, uint32_t nq, uint32_t k,
                                                            const uint32_t *rcount,
                                                            const uint8_t *rsel,
                                                            const uint64_t *cap_off,
                                                            const uint2 *rb0, const uint2 *rb1,
                                                            uint64_t *out_keys,
                                                            uint32_t *out_counts) {
  __shared__ uint64_t sk[kTopkSmem];
  __shared__ uint32_t hist[256];
  __shared__ uint64_t s_prefix;
  __shared__ uint32_t s_need, s_cnt;
  for (uint32_t q = blockIdx.x; q < nq; q += gridDim.x) {
    const uint32_t c = rcount[q];
    const uint2 *R = (rsel[q] ? rb1 : rb0) + cap_off[q];
    const uint32_t kk = min(k, c);
    uint32_t nsort;
    if (c <= kTopkSmem) {
      nsort = 1;
      while (nsort < c) nsort <<= 1;
      for (uint32_t i = threadIdx.x; i < nsort; i += blockDim.x)
        sk[i] = i < c ? make_key(R[i], ix.doc_base) : 0ull;
      __syncthreads();
    } else {
      // exact radix select of the k-th largest unique key, 8 bits per pass
      if (threadIdx.x == 0) {
        s_prefix = 0;
        s_need = kk;
        s_cnt = 0;
      }
      uint64_t mask = 0;
      for (int shift = 56; shift >= 0; shift -= 8) {
        for (uint32_t i = threadIdx.x; i < 256; i += blockDim.x) hist[i] = 0;
        __syncthreads();
        const uint64_t prefix = s_prefix;
        for (uint32_t i = threadIdx.x; i < c; i += blockDim.x) {
          const uint64_t key = make_key(R[i], ix.doc_base);
          if ((key & mask) == prefix) atomicAdd(&hist[(key >> shift) & 255u], 1u);
        }
        __syncthreads();
        if (threadIdx.x == 0) {
          uint32_t cum = 0, need = s_need;
          for (int d = 255; d >= 0; --d) {
            if (cum + hist[d] >= need) {
              s_prefix = prefix | ((uint64_t)d << shift);
              s_need = need - cum;
              break;
            }
            cum += hist[d];
          }
        }
        mask |= 0xFFull << shift;
        __syncthreads();
      }
      const uint64_t thr = s_prefix;
      for (uint32_t i = threadIdx.x; i < c; i += blockDim.x) {
        const uint64_t key = make_key(R[i], ix.doc_base);
        if (key >= thr) sk[atomicAdd(&s_cnt, 1u)] = key;
      }
      __syncthreads();
      nsort = 1;
      while (nsort < kk) nsort <<= 1;
      for (uint32_t i = kk + threadIdx.x; i < nsort; i += blockDim.x) sk[i] = 0ull;
      __syncthreads();
    }
    bitonic_desc(sk, nsort);
    for (uint32_t i = threadIdx.x; i < k; i += blockDim.x)
      out_keys[(size_t)q * k + i] = i < kk ? sk[i] : 0ull;
    if (threadIdx.x == 0) out_counts[q] = kk;
    __syncthreads();
  }
}

// ------------------------------------------------------------------- shard merge

// G-way merge of per-shard sorted key runs (warp per query; lane g holds run g's head).
__global__ void merge_topk_kernel(uint32_t G, uint32_t nq, uint32_t k, const uint64_t *keys,
                                  const uint32_t *counts, uint64_t *out, uint32_t *out_counts) {
  const uint32_t lane = lane_id();
  const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
  for (uint32_t q = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); q < nq; q += nwarps) {
    const uint32_t cnt = lane < G ? min(counts[(size_t)lane * nq + q], k) : 0u;
    const uint64_t *run = keys + ((size_t)lane * nq + q) * k;
    uint32_t p = 0;
    uint64_t head = p < cnt ? run[0] : 0ull;
    uint32_t i = 0;
    for (; i < k; ++i) {
      uint64_t best = head;
      for (int d = 16; d; d >>= 1) best = max(best, __shfl_xor_sync(0xffffffffu, best, d));
      if (best == 0ull) break;
      if (lane == 0) out[(size_t)q * k + i] = best;
      if (head == best) {  // keys are unique: exactly one lane advances
        ++p;
        head = p < cnt ? run[p] : 0ull;
      }
    }
    for (uint32_t j = i + lane; j < k; j += 32) out[(size_t)q * k + j] = 0ull;
    if (lane == 0) out_counts[q] = i;
  }
}

__global__ void keys_to_results_kernel(uint32_t nq, uint32_t k, const uint64_t *keys,
                                       const uint32_t *counts, uint32_t *docids, float *scores) {
  const uint64_t n = (uint64_t)nq * k;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t q = (uint32_t)(i / k), r = (uint32_t)(i % k);
    if (r < counts[q]) {
      const uint64_t key = keys[i];
      docids[i] = 0xFFFFFFFFu - (uint32_t)(key & 0xFFFFFFFFu);
      scores[i] = __uint_as_float((uint32_t)(key >> 32));
    } else {
      docids[i] = 0xFFFFFFFFu;
      scores[i] = __uint_as_float(0xFF800000u);
    }
  }
}

// ------------------------------------------------------------------- debug decode

__global__ void __launch_bounds__(256) decode_list_kernel(DevIndex ix, uint32_t block0,
                                                          uint32_t nblocks, uint32_t *out) {
  extern __shared__ uint4 smem4[];
  const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
  uint32_t *w = reinterpret_cast<uint32_t *>(smem4) + wid * (scratch_words(ix.B) + ix.B);
  const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
  for (uint32_t k = blockIdx.x * (blockDim.x >> 5) + wid; k < nblocks; k += nwarps) {
    const uint32_t n = warp_decode_block(ix, (uint64_t)block0 + k, w + scratch_words(ix.B), w);
    for (uint32_t i = lane; i < n; i += 32) out[(size_t)k * ix.B + i] = w[scratch_words(ix.B) + i] + ix.doc_base;
    __syncwarp();
  }
}

__global__ void __launch_bounds__(256) decode_all_kernel(DevIndex ix, uint64_t nblocks,
                                                         unsigned long long *acc) {
  extern __shared__ uint4 smem4[];
  const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
  uint32_t *w = reinterpret_cast<uint32_t *>(smem4) + wid * (scratch_words(ix.B) + ix.B);
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  uint32_t x = 0;
  unsigned long long post = 0, pay = 0;
  for (uint64_t k = blockIdx.x * (uint64_t)(blockDim.x >> 5) + wid; k < nblocks; k += nwarps) {
    uint32_t p = 0;
    const uint32_t n = warp_decode_block(ix, k, w + scratch_words(ix.B), w, &p);
    for (uint32_t i = lane; i < n; i += 32) x ^= w[scratch_words(ix.B) + i];
    __syncwarp();
    post += n;
    pay += p + 8u;
  }
  for (int d = 16; d; d >>= 1) x ^= __shfl_xor_sync(0xffffffffu, x, d);
  if (lane == 0) {
    atomicXor(acc + 0, (unsigned long long)x);
    atomicAdd(acc + 1, post);
    atomicAdd(acc + 2, pay);
  }
}

// ------------------------------------------------------------------- host side

static int num_sms(int dev) {
  static int cache[64] = {0};
  if (dev < 0 || dev >= 64) return 148;
  if (!cache[dev]) {
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    cache[dev] = v > 0 ? v : 148;
  }
  return cache[dev];
}

griffin_status reserve_ws(griffin_index *ix, uint32_t nq, uint64_t units, uint64_t entries) {
  Workspace &w = ix->ws;
  const size_t q = (size_t)nq + 1;
  GRIFFIN_CUDA_TRY(w.plan_terms.reserve(q * kMaxTerms * 4));
  GRIFFIN_CUDA_TRY(w.plan_m.reserve(q * 4));
  GRIFFIN_CUDA_TRY(w.cap.reserve(q * 4));
  GRIFFIN_CUDA_TRY(w.cap_off.reserve(q * 8 + 8));
  GRIFFIN_CUDA_TRY(w.rcount.reserve(q * 4));
  GRIFFIN_CUDA_TRY(w.rsel.reserve(q));
  GRIFFIN_CUDA_TRY(w.qmode.reserve(q * 4 + q * 4));  // qmode | qunits
  GRIFFIN_CUDA_TRY(w.unit_base.reserve(q * 8 + 8 + (q / kScanTile + 8) * 8));
  GRIFFIN_CUDA_TRY(w.unit_off.reserve((units + 1) * 8));
  GRIFFIN_CUDA_TRY(w.unit_cnt.reserve((units + 1) * 4));
  GRIFFIN_CUDA_TRY(w.rbuf0.reserve((entries + 1) * 8));
  GRIFFIN_CUDA_TRY(w.rbuf1.reserve((entries + 1) * 8));
  GRIFFIN_CUDA_TRY(w.bump.reserve((entries + 1) * 8));
  if (!w.scal.p) {
    GRIFFIN_CUDA_TRY(w.scal.reserve(kScalCount * 8));
    GRIFFIN_CUDA_TRY(cudaMemset(w.scal.p, 0, w.scal.bytes));
  }
  w.nq_cap = std::max<size_t>(w.nq_cap, nq);
  w.unit_cap = std::max<size_t>(w.unit_cap, units);
  w.entry_cap = std::max<size_t>(w.entry_cap, entries);
  // derive the real capacities from the buffers (reserve over-allocates)
  w.nq_cap = std::min(w.plan_m.bytes / 4 - 1, w.cap_off.bytes / 8 - 2);
  w.unit_cap = std::min(w.unit_off.bytes / 8 - 1, w.unit_cnt.bytes / 4 - 1);
  w.entry_cap = std::min(std::min(w.rbuf0.bytes, w.rbuf1.bytes), w.bump.bytes) / 8 - 1;
  return GRIFFIN_OK;
}

struct StageTimer {
  griffin_index *ix;
  cudaStream_t st;
  int stage;
  cudaEvent_t a = nullptr, b = nullptr;
  StageTimer(griffin_index *ix_, cudaStream_t st_, int stage_) : ix(ix_), st(st_), stage(stage_) {
    if (!ix->profiling) return;
    if (ix->ev_next + 2 > ix->ev_pool.size()) {
      for (int i = 0; i < 64; ++i) {
        cudaEvent_t e;
        cudaEventCreate(&e);
        ix->ev_pool.push_back(e);
      }
    }
    a = ix->ev_pool[ix->ev_next++];
    b = ix->ev_pool[ix->ev_next++];
    cudaEventRecord(a, st);
  }
  ~StageTimer() {
    if (!a) return;
    cudaEventRecord(b, st);
    ix->pending.push_back({stage, {a, b}});
  }
};

template <bool RC>
static cudaError_t launch_intersect(griffin_index *ix, const RoundArgs &ra, cudaStream_t st) {
  const size_t smem = (size_t)warp_smem_words(ix->B, ix->D) * 4 * kWarpsPerCta;
  static thread_local int configured_dev[2] = {-1, -1};
  static thread_local size_t configured_smem[2] = {0, 0};
  if (configured_dev[RC] != ix->device || configured_smem[RC] < smem) {
    cudaError_t e = cudaFuncSetAttribute(intersect_kernel<RC>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    configured_dev[RC] = ix->device;
    configured_smem[RC] = smem;
  }
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, intersect_kernel<RC>, kIntersectThreads,
                                                smem);
  per_sm = std::max(1, per_sm);
  const int grid = num_sms(ix->device) * per_sm;
  intersect_kernel<RC><<<grid, kIntersectThreads, smem, st>>>(ix->dev(), ra);
  return cudaGetLastError();
}

griffin_status run_batch(griffin_index *ix, uint32_t nq, const uint32_t *d_qoffs,
                         const uint32_t *d_terms, uint32_t max_terms, uint32_t k, uint64_t *d_keys,
                         uint32_t *d_counts, cudaStream_t st, bool final_topk, int forced_mode) {
  Workspace &w = ix->ws;
  if (nq == 0) return GRIFFIN_OK;
  if (nq > w.nq_cap || !w.scal.p) {
    set_error("workspace not reserved for this batch (call griffin_reserve)");
    return GRIFFIN_ERR_INVALID_ARG;
  }
  const DevIndex di = ix->dev();
  unsigned long long *scal = w.scal.as<unsigned long long>();
  uint32_t *qunits = w.qmode.as<uint32_t>() + (nq + 1);
  uint64_t *scan_tmp = w.unit_base.as<uint64_t>() + (nq + 2);
  RoundArgs ra{};
  ra.nq = nq;
  ra.D = ix->D;
  ra.T = ix->T;
  ra.forced_mode = forced_mode;
  ra.plan_terms = w.plan_terms.as<uint32_t>();
  ra.plan_m = w.plan_m.as<uint32_t>();
  ra.cap = w.cap.as<uint32_t>();
  ra.cap_off = w.cap_off.as<uint64_t>();
  ra.rcount = w.rcount.as<uint32_t>();
  ra.rsel = w.rsel.as<uint8_t>();
  ra.qmode = w.qmode.as<uint32_t>();
  ra.unit_base = w.unit_base.as<uint64_t>();
  ra.unit_off = w.unit_off.as<uint64_t>();
  ra.unit_cnt = w.unit_cnt.as<uint32_t>();
  ra.unit_cap = w.unit_cap;
  ra.bump = w.bump.as<uint2>();
  ra.entry_cap = w.entry_cap;
  ra.scal = scal;
  const unsigned qblocks = (nq + 255) / 256;
  {
    StageTimer t(ix, st, 0);
    ix->launch_count += 2;
    plan_queries_kernel<<<qblocks, 256, 0, st>>>(di, nq, d_qoffs, d_terms, w.plan_terms.as<uint32_t>(),
                                                 w.plan_m.as<uint32_t>(), w.cap.as<uint32_t>(),
                                                 w.rcount.as<uint32_t>(), w.rsel.as<uint8_t>(), scal);
    GRIFFIN_CUDA_TRY(cudaGetLastError());
    plan_totals_kernel<<<std::min<unsigned>(qblocks, 1024), 256, 0, st>>>(
        di, nq, w.plan_terms.as<uint32_t>(), w.plan_m.as<uint32_t>(), w.cap.as<uint32_t>(), scal);
    GRIFFIN_CUDA_TRY(cudaGetLastError());
    GRIFFIN_CUDA_TRY(exclusive_scan<uint32_t>(w.cap.as<uint32_t>(), w.cap_off.as<uint64_t>(), nq,
                                              scan_tmp, st, &ix->launch_count));
  }
  const uint32_t rounds = std::max<uint32_t>(1, max_terms > 0 ? max_terms - 1 : 1);
  for (uint32_t r = 1; r <= rounds; ++r) {
    ra.round = r;
    ra.rprev = (r & 1) ? w.rbuf0.as<uint2>() : w.rbuf1.as<uint2>();
    ra.rnext = (r & 1) ? w.rbuf1.as<uint2>() : w.rbuf0.as<uint2>();
    {
      StageTimer t(ix, st, 0);
      plan_round_kernel<<<qblocks, 256, 0, st>>>(di, ra, qunits);
      GRIFFIN_CUDA_TRY(cudaGetLastError());
      GRIFFIN_CUDA_TRY(exclusive_scan<uint32_t>(qunits, w.unit_base.as<uint64_t>(), nq, scan_tmp, st,
                                                &ix->launch_count));
      ix->launch_count += 3;  // plan_round + intersect + compact
    }
    {
      StageTimer t(ix, st, 1);
      if (r == 1) GRIFFIN_CUDA_TRY(launch_intersect<true>(ix, ra, st));
      else GRIFFIN_CUDA_TRY(launch_intersect<false>(ix, ra, st));
    }
    {
      StageTimer t(ix, st, 2);
      compact_kernel<<<std::min<unsigned>((nq + 7) / 8, 148 * 8), 256, 0, st>>>(ra);
      GRIFFIN_CUDA_TRY(cudaGetLastError());
    }
  }
  if (final_topk) {
    StageTimer t(ix, st, 3);
    ix->launch_count += 1;
    topk_kernel<<<std::min<uint32_t>(nq, 148 * 4), kTopkThreads, 0, st>>>(
        di, nq, k, w.rcount.as<uint32_t>(), w.rsel.as<uint8_t>(), w.cap_off.as<uint64_t>(),
        w.rbuf0.as<uint2>(), w.rbuf1.as<uint2>(), d_keys, d_counts);
    GRIFFIN_CUDA_TRY(cudaGetLastError());
  }
  return GRIFFIN_OK;
}

griffin_status launch_merge_topk(griffin_index *ix, uint32_t G, uint32_t nq, uint32_t k,
                                 const uint64_t *d_keys, const uint32_t *d_counts,
                                 uint64_t *d_out_keys, uint32_t *d_out_counts, cudaStream_t st) {
  if (nq == 0) return GRIFFIN_OK;
  StageTimer t(ix, st, 4);
  ix->launch_count += 1;
  merge_topk_kernel<<<std::min<uint32_t>((nq + 7) / 8, 148 * 16), 256, 0, st>>>(
      G, nq, k, d_keys, d_counts, d_out_keys, d_out_counts);
  GRIFFIN_CUDA_TRY(cudaGetLastError());
  return GRIFFIN_OK;
}

griffin_status launch_keys_to_results(griffin_index *ix, uint32_t nq, uint32_t k,
                                      const uint64_t *d_keys, const uint32_t *d_counts,
                                      uint32_t *d_docids, float *d_scores, cudaStream_t st) {
  const uint64_t n = (uint64_t)nq * k;
  if (!n) return GRIFFIN_OK;
  ix->launch_count += 1;
  keys_to_results_kernel<<<(unsigned)std::min<uint64_t>((n + 255) / 256, 148 * 32), 256, 0, st>>>(
      nq, k, d_keys, d_counts, d_docids, d_scores);
  GRIFFIN_CUDA_TRY(cudaGetLastError());
  return GRIFFIN_OK;
}

griffin_status launch_decode_list(griffin_index *ix, uint32_t term, uint32_t *d_out,
                                  cudaStream_t st) {
  const TermInfo &t = ix->h_terms[term];
  if (!t.nblocks) return GRIFFIN_OK;
  const size_t smem = (size_t)(scratch_words(ix->B) + ix->B) * 4 * 8;
  GRIFFIN_CUDA_TRY(cudaFuncSetAttribute(decode_list_kernel,
                                        cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  decode_list_kernel<<<std::min<uint32_t>((t.nblocks + 7) / 8, 148 * 8), 256, smem, st>>>(
      ix->dev(), t.block0, t.nblocks, d_out);
  GRIFFIN_CUDA_TRY(cudaGetLastError());
  return GRIFFIN_OK;
}

griffin_status launch_decode_all(griffin_index *ix, unsigned long long *d_acc, cudaStream_t st) {
  if (!ix->nblocks) return GRIFFIN_OK;
  const size_t smem = (size_t)(scratch_words(ix->B) + ix->B) * 4 * 8;
  GRIFFIN_CUDA_TRY(cudaFuncSetAttribute(decode_all_kernel,
                                        cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, decode_all_kernel, 256, smem);
  decode_all_kernel<<<num_sms(ix->device) * std::max(1, per_sm), 256, smem, st>>>(
      ix->dev(), ix->nblocks, d_acc);
  GRIFFIN_CUDA_TRY(cudaGetLastError());
  return GRIFFIN_OK;
}

griffin_status copy_final_docids(griffin_index *ix, uint32_t *h_out, uint64_t cap, uint64_t *count) {
  Workspace &w = ix->ws;
  uint32_t c = 0;
  uint8_t sel = 0;
  uint64_t off = 0;
  cudaStream_t st = ix->stream;
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(&c, w.rcount.p, 4, cudaMemcpyDeviceToHost, st));
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(&sel, w.rsel.p, 1, cudaMemcpyDeviceToHost, st));
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(&off, w.cap_off.p, 8, cudaMemcpyDeviceToHost, st));
  GRIFFIN_CUDA_TRY(cudaStreamSynchronize(st));
  *count = c;
  if (c > cap) {
    set_error("output capacity too small");
    return GRIFFIN_ERR_INVALID_ARG;
  }
  std::vector<uint2> tmp(c);
  const uint2 *src = (sel ? w.rbuf1.as<uint2>() : w.rbuf0.as<uint2>()) + off;
  if (c) GRIFFIN_CUDA_TRY(cudaMemcpyAsync(tmp.data(), src, (size_t)c * 8, cudaMemcpyDeviceToHost, st));
  GRIFFIN_CUDA_TRY(cudaStreamSynchronize(st));
  for (uint32_t i = 0; i < c; ++i) h_out[i] = tmp[i].x + ix->doc_base;
  return GRIFFIN_OK;
}

void host_query_bounds(const griffin_index *ix, const uint32_t *terms, uint32_t nterms,
                       uint64_t *cap, uint64_t *units) {
  std::vector<uint32_t> ts(terms, terms + nterms);
  std::sort(ts.begin(), ts.end());
  ts.erase(std::unique(ts.begin(), ts.end()), ts.end());
  *cap = 0;
  *units = 0;
  for (uint32_t t : ts)
    if (t >= ix->V) return;
  if (ts.empty() || ts.size() > (size_t)kMaxTerms) return;
  std::sort(ts.begin(), ts.end(), [&](uint32_t a, uint32_t b) {
    const uint32_t da = ix->h_terms[a].df_global, db = ix->h_terms[b].df_global;
    return da != db ? da < db : a < b;
  });
  for (uint32_t t : ts)
    if (ix->h_terms[t].df_local == 0) return;
  const TermInfo &t0 = ix->h_terms[ts[0]];
  if (ts.size() == 1) {
    *cap = t0.df_local;
    *units = t0.nblocks;
    return;
  }
  *cap = std::min(t0.df_local, ix->h_terms[ts[1]].df_local);
  uint32_t mx = 0;
  for (size_t i = 1; i < ts.size(); ++i) mx = std::max(mx, ix->h_terms[ts[i]].nblocks);
  *units = (uint64_t)t0.nblocks + mx;
}

}  // namespace griffin
