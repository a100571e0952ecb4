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
#include <atomic>
#include <map>
#include <mutex>
#include <tuple>

#include <nvtx3/nvToolsExt.h>

#include "internal.h"
#include "scan.cuh"

namespace griffin {

constexpr int kIntersectThreads = 256;
constexpr int kWarpsPerCta = kIntersectThreads / 32;
constexpr uint32_t kTopkSmem = 4096;
#ifndef GRIFFIN_EMIT_DEPTH
#define GRIFFIN_EMIT_DEPTH 1
#endif
#ifndef GRIFFIN_SKIP_DEPTH
#define GRIFFIN_SKIP_DEPTH 2
#endif
// Work per lane kept in flight by the intersect kernel's inner loops.  The
// kernel runs 3 CTAs x 8 warps per SM at the 80-register cap; deeper loops
// spilled (C2 round-1+2 intersect, ms: emission depth 4 / 2 / 1 = 0.653 /
// 0.626 / 0.607; arena probes 4 / 2 = 0.697 / 0.655; skip searches 4 / 2 =
// 0.605 / 0.603 — profiles/r01_configs.jsonl, session 3).
constexpr int kEmitDepth = GRIFFIN_EMIT_DEPTH;
#ifndef GRIFFIN_UNIT_EMIT_DEPTH
#define GRIFFIN_UNIT_EMIT_DEPTH 1
#endif   // survivors per lane per emission pass (gathers in flight)
constexpr int kSkipDepth = GRIFFIN_SKIP_DEPTH;   // interleaved skip-pointer searches per lane
#ifndef GRIFFIN_MERGE_UNROLL
#define GRIFFIN_MERGE_UNROLL 4
#endif
constexpr int kMergeUnroll = GRIFFIN_MERGE_UNROLL;
#ifndef GRIFFIN_IK_PAIR
#define GRIFFIN_IK_PAIR 1
#endif
constexpr bool kIkPair = GRIFFIN_IK_PAIR;   // intersect kernel: two-blocks-per-warp decoder at B = 128
constexpr int kTopkThreads = 512;
constexpr uint32_t kTileSlackC = 64;   // = kTileSlack (read slack after a tile), needed early

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

// Σ cap and Σ unit bounds (bound = nblocks(t0) + max(max_r nblocks(t_r),
// ceil(cap / P))), checked against the reserved workspace before any round runs.
__global__ void plan_totals_kernel(DevIndex ix, uint32_t nq, const uint32_t *plan_terms,
                                   const uint32_t *plan_m, const uint32_t *cap, uint32_t P,
                                   unsigned long long *scal) {
  unsigned long long c = 0, u = 0;
  for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < nq; q += gridDim.x * blockDim.x) {
    const uint32_t m = plan_m[q];
    if (!m || !cap[q]) continue;
    c += cap[q];
    uint32_t mx = 0;
    for (uint32_t i = 1; i < m; ++i) mx = max(mx, ix.terms[plan_terms[q * kMaxTerms + i]].nblocks);
    if (m >= 3) mx = max(mx, (cap[q] + P - 1) / P);   // probe pass
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

// R blocks (or B-entry intermediate chunks) per bitvector unit, U, and where
// its three U*B-word arrays live: the R tile at the start of the tile region,
// the compacted R indices at the start of the staging area (free after
// decoding), the compacted S positions after the R tile when the tile holds
// both, else after the indices in the staging area.  Bitvector units run in
// the round-1 gallop kernel (ROLE 2 layout, whose staging area is sized for
// 2*Umax*B words) and, for later SvS rounds without the probe pass, in the
// all-kinds kernel (ROLE 0 layout); U must fit both.  Fewer, larger units
// amortise the per-unit work (ticket, records, a TMA round trip, the output
// allocation) over up to U*B lookups.
#ifndef GRIFFIN_BM_UNIT_ELEMS
#define GRIFFIN_BM_UNIT_ELEMS 384
#endif
// most R elements per unit: Umax(B) = clamp(GRIFFIN_BM_UNIT_ELEMS / B, 1, 4)
__host__ __device__ inline uint32_t bm_unit_max(uint32_t B) {
  const uint32_t u = GRIFFIN_BM_UNIT_ELEMS / B;
  return u < 1u ? 1u : (u > 4u ? 4u : u);
}
__host__ __device__ inline uint32_t stage_words(uint32_t B, uint32_t D);
__host__ __device__ inline uint32_t other_tile_words(uint32_t B, uint32_t D, bool nextgeq);
__host__ __device__ inline uint32_t other_stage_words(uint32_t B, uint32_t D) {
  const uint32_t s = stage_words(B, D), w = 2u * bm_unit_max(B) * B;
  return s > w ? s : w;
}
// tile / staging words of the layout bitvector units run in (role2: ROLE 2)
__host__ __device__ inline void bm_layout(uint32_t B, uint32_t D, bool nextgeq, bool role2,
                                          uint32_t *tile, uint32_t *stg) {
  *tile = (role2 ? other_tile_words(B, D, nextgeq) : (D + 2u) * B + kTileSlackC) - kTileSlackC;
  *stg = role2 ? other_stage_words(B, D) : stage_words(B, D);
}
__host__ __device__ inline bool bm_spos_in_tile(uint32_t B, uint32_t D, bool nextgeq, bool role2,
                                                uint32_t U) {
  uint32_t tile, stg;
  bm_layout(B, D, nextgeq, role2, &tile, &stg);
  return 2u * U * B <= tile;
}
__host__ __device__ inline uint32_t bm_unit_blocks(uint32_t B, uint32_t D, bool nextgeq) {
  for (uint32_t U = bm_unit_max(B); U > 1u; --U) {
    bool ok = true;
    for (int r = 0; r < 2; ++r) {
      uint32_t tile, stg;
      bm_layout(B, D, nextgeq, r == 1, &tile, &stg);
      ok = ok && U * B <= tile && (2u * U * B <= tile || 2u * U * B <= stg);
    }
    if (ok) return U;
  }
  return 1u;
}

__global__ void plan_round_kernel(DevIndex ix, RoundArgs a, uint32_t *qunits) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  // units must fit their arrays; intermediates are checked at compaction time
  // against the entries actually produced (the workspace may hold fewer entries
  // than the sum of the per-query bounds, griffin_set_entry_budget)
  const bool overflow = a.scal[kScalTotals + 1] > a.unit_cap;
  if (q == 0) {
    a.scal[kScalBump] = 0;
    a.scal[kScalUnitCtr] = 0;
    a.scal[kScalUnitCtr2] = 0;
    a.scal[kScalPerm] = 0;
    a.scal[kScalPerm + 1] = 0;
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
      if (a.probe) {   // rounds 2..m-1 as one multi-list probe pass
        mode = kModeProbe;
        units = (uint32_t)((nR + a.pchunk - 1) / a.pchunk);
      } else {
        pair = true;
      }
    }
    if (pair) {
      const uint32_t sid = a.plan_terms[q * kMaxTerms + a.round];
      const TermInfo tS = ix.terms[sid];
      // crossover: T for compressed S (gallop decodes one block per
      // touched block), Tdec when S sits decoded in the batch arena
      const uint8_t kd = a.tdec ? a.tdec[sid] : kDecNone;
      const uint64_t T = kd == kDecArena ? a.Tdec : a.T;
      const bool gallop = a.forced_mode == 2 ||
                          (a.forced_mode == 0 && (uint64_t)tS.df_local > T * nR);
      // S decoded into a bitvector this batch: every R element is looked up in
      // O(1) (no merge or gallop through S), one unit per R chunk of B
      const bool bitmap = a.forced_mode == 0 && kd == kDecBitmap;
      // ... and so is R (round 1): AND the two bitvectors word by word over
      // R's docID range, kAndWords words per unit (no R decode, no lookups)
#ifdef GRIFFIN_NO_BITAND   // A/B builds
      const bool band = false;
#else
      const bool band = bitmap && a.round == 1 && a.tdec[a.plan_terms[q * kMaxTerms]] == kDecBitmap;
#endif
      mode = band ? kModeBitAnd : (bitmap ? kModeBitmap : (gallop ? kModeGallop : kModeMerge));
      const uint32_t U = bm_unit_blocks(ix.B, a.D, a.nextgeq != 0);
      if (band) {
        const uint32_t w0 = __ldg(ix.first + t0.block0) >> 5;
        units = (a.bm_words - w0 + kAndWords - 1) / kAndWords;
      } else {
        units = bitmap ? (nbR + U - 1) / U : (gallop ? nbR : (nbR + tS.nblocks + a.D - 1) / a.D);
      }
    }
  }
  a.qmode[q] = mode;
  qunits[q] = units;
}

// ------------------------------------------------------------------- intersect

// SURVEY §8(d) per-survivor algorithmic bytes: each tf gather is one 32-B
// sector, plus the doc's norm (4 B) and the (docID, score) entry written (8 B);
// round 1 gathers two tfs (R and S), later rounds one (the previous partial
// score comes with the intermediate entry, counted at 8 B per R element).
constexpr uint32_t kTfSector = 32, kSurvBytes = kTfSector + 4 + 8,
                   kSurvBytesR1 = 2 * kTfSector + 4 + 8;
// Per-warp counters live in the warp's shared memory (lane 0 updates them),
// not in registers: the kernel runs at the 80-register cap.
enum : int { kCAlg = 0, kCPay, kCPost, kCSurv, kCApost, kCAcomp, kCNum };
struct Acc {
  // alg bytes, payload bytes, decoded postings, survivors, decoded-arena postings
  // read, their compressed bytes
  unsigned long long *ctr = nullptr;
  // this warp's bump chunk in warp smem: {next free entry (u64), entries left (u32)}
  unsigned long long *boff = nullptr;
  uint32_t *bleft = nullptr;
};

// Output space for a unit's survivors (lane 0): carved from a per-warp chunk of
// the bump area, so the global counter sees one atomic per kBumpChunk entries
// instead of one per unit (same-address atomics serialise in L2).  Unit outputs
// are located by unit_off/unit_cnt, so chunk order and gaps do not matter.
__device__ __forceinline__ unsigned long long bump_alloc(const RoundArgs &a, Acc &acc,
                                                         uint32_t cnt) {
  // a unit bigger than a quarter chunk gets its own exact allocation (so a
  // refill never throws away more than a quarter chunk of the previous one)
  if (cnt > kBumpChunk / 4u) return atomicAdd(a.scal + kScalBump, (unsigned long long)cnt);
  unsigned long long off = *acc.boff;
  uint32_t left = *acc.bleft;
  if (cnt > left) {
    left = kBumpChunk;
    off = atomicAdd(a.scal + kScalBump, (unsigned long long)left);
  }
  *acc.boff = off + cnt;
  *acc.bleft = left - cnt;
  return off;
}

// Per-warp shared memory carve-up (u32 words):
//   [mbar+bump state 8][cnt 64][aux B+32][stg SW][tile (D+2)*B]
// stg holds TMA-staged EF payloads; after decoding, the merge path reuses it for
// the per-R-element match array.  The gallop path carves tile into
// tileR | kidx | match | tileS[G blocks].
__host__ __device__ inline uint32_t stage_words(uint32_t B, uint32_t D) {
  // ~2 B per posting of compressed payload for a unit's D+2 blocks (larger units
  // are staged in capacity-sized batches); also holds the merge's per-lane match
  // lists (<= 32*((D+2)*B/64+1) words) and always >= one worst-case block.
  return ((D + 2) * B / 2 + 64 + 3) & ~3u;
}
// read slack after the tile: the uniform-trip merge loop may read up to L =
// ceil((D+2)*B/32) words past a lane's segment (D <= 8 at B = 128 -> 40)
constexpr uint32_t kTileSlack = kTileSlackC;
// read slack after the staging area: decoders read a word or two past a block's
// high stream (look-ahead windows), also when it ends the staging area
constexpr uint32_t kStgSlack = kRunSlack;   // >= the run decoder's over-read
// per-warp header words: mbarrier (0-1), bump left (2), bump offset (4-5),
// counters (8-19)
constexpr uint32_t kWarpHdr = 24;
// with_tile = false: no decode tile (kernels that decode straight to HBM)
__host__ __device__ inline uint32_t warp_smem_words(uint32_t B, uint32_t D, bool with_tile = true) {
  return kWarpHdr + 64 + (B + 32) + stage_words(B, D) + kStgSlack +
         (with_tile ? (D + 2) * B + kTileSlack : 0u);
}
constexpr uint32_t kLutBytes = 2048;
// Run length (D + 2 blocks) of the decode-only kernels (sweep, decode-once):
// 2048 postings, i.e. two full passes of the run decoder (32/Lb = 1024/B
// blocks per pass), so its lane groups are never idle inside a run.
__host__ __device__ inline uint32_t sweep_D(uint32_t B) {
  const uint32_t r = 2048u / B;
  return r > 4u ? r - 2u : 2u;
}

struct WarpSmem {
  uint64_t *mbar;
  uint32_t *cnt, *aux, *stg, *tile;
  const uint8_t *lut;
  uint32_t phase;
};

// Probe-pass kernel layout: the probe unit's tile region holds its survivor
// chunk (tileR, scores, norms, block ids, matches: 5B words) plus, only when
// galloping into compressed lists decodes blocks (NextGEQ off), G = D-3 decoded
// S blocks.
__host__ __device__ inline uint32_t probe_tile_words(uint32_t B, uint32_t D, bool nextgeq) {
  return 5u * B + (nextgeq ? 0u : (D - 3u) * B) + kTileSlack;
}
__host__ __device__ inline uint32_t probe_warp_smem_words(uint32_t B, uint32_t D, bool nextgeq) {
  return kWarpHdr + 64 + (B + 32) + stage_words(B, D) + kStgSlack + probe_tile_words(B, D, nextgeq);
}

__device__ __forceinline__ WarpSmem carve_warp_smem(uint4 *smem4, uint32_t B, uint32_t D,
                                                    bool with_tile = true) {
  uint8_t *base = reinterpret_cast<uint8_t *>(smem4);
  WarpSmem w;
  w.lut = base;
  uint32_t *wb = reinterpret_cast<uint32_t *>(base + kLutBytes) +
                 (threadIdx.x >> 5) * warp_smem_words(B, D, with_tile);
  w.mbar = reinterpret_cast<uint64_t *>(wb);   // words 0-1; 2: bump left; 4-5: bump offset
  w.cnt = wb + kWarpHdr;
  w.aux = w.cnt + 64;
  w.stg = w.aux + B + 32;
  w.tile = with_tile ? w.stg + stage_words(B, D) + kStgSlack : nullptr;
  w.phase = 0;
  return w;
}

// CTA prologue: LUT + one mbarrier per warp.
__device__ __forceinline__ void cta_smem_init(uint4 *smem4, const WarpSmem &w) {
  build_select_lut(reinterpret_cast<uint8_t *>(smem4));
  if (lane_id() == 0) {
    mbar_init(w.mbar, 1);
    fence_mbar_init();
  }
  __syncthreads();
}

// Stage the payloads of the blocks whose (meta, staging offset in 16-B units)
// are held by lanes [0, nb) as one or more TMA bulk copies, then wait.
// `contig` = the blocks are consecutive in the payload (one copy suffices).
__device__ __forceinline__ void stage_blocks(const DevIndex &ix, WarpSmem &w, uint32_t nb,
                                             uint2 m, uint32_t soff16, uint32_t sz16,
                                             bool contig) {
  const uint32_t lane = lane_id();
  const uint32_t tot16 = __reduce_add_sync(0xffffffffu, lane < nb ? sz16 : 0u);
  if (tot16 == 0) return;
  const uint32_t m0x = __shfl_sync(0xffffffffu, m.x, 0);
  if (lane == 0) {
    fence_proxy_async();
    mbar_expect_tx(w.mbar, tot16 * 16u);
  }
  if (contig) {
    if (lane == 0) bulk_g2s(w.stg, ix.payload + m0x, tot16 * 16u, w.mbar);
  } else if (lane < nb && sz16) {
    fence_proxy_async();
    bulk_g2s(w.stg + soff16 * 4u, ix.payload + m.x, sz16 * 16u, w.mbar);
  }
  mbar_wait(w.mbar, w.phase);
  w.phase ^= 1u;
}

// Decode the staged blocks whose (meta word y, first docID f, staged offset so in
// 16-B units) sit in lanes [l0, l0+nb) into dst + i*B: two blocks per warp
// instruction stream when B = 128 (warp_decode_pair_staged), else one.
template <class Sink, bool PAIR = true>
__device__ __forceinline__ void decode_staged_lanes(const WarpSmem &w, uint32_t B, uint32_t l0,
                                                    uint32_t nb, uint32_t y, uint32_t f,
                                                    uint32_t so, uint32_t *dst, Sink &sink) {
  if (run_decoder_ok(B)) {   // power-of-two B: several blocks per warp pass
    warp_decode_runs(w.stg, l0, nb, y, f, so, dst, B, w.cnt, w.lut, sink);
    return;
  }
  uint32_t i0 = 0;
  if (PAIR && B == 128u) {   // pairs; an odd last block takes the single-block decoder
    const uint32_t npair = nb & ~1u;
    for (uint32_t i = 0; i < npair; i += 2) {
      const uint32_t la = l0 + i, lb = (l0 + i + 1) & 31u;
      const uint32_t ya = __shfl_sync(0xffffffffu, y, la), yb = __shfl_sync(0xffffffffu, y, lb);
      const uint32_t fa = __shfl_sync(0xffffffffu, f, la), fb = __shfl_sync(0xffffffffu, f, lb);
      const uint32_t sa = __shfl_sync(0xffffffffu, so, la), sb = __shfl_sync(0xffffffffu, so, lb);
      warp_decode_pair_staged(w.stg + sa * 4u, fa, ya, dst + i * B, w.stg + sb * 4u, fb, yb,
                              dst + (i + 1) * B, true, w.cnt, w.lut, sink);
    }
    i0 = npair;
  }
  {
    for (uint32_t i = i0; i < nb; ++i) {
      const uint32_t yi = __shfl_sync(0xffffffffu, y, l0 + i);
      const uint32_t fi = __shfl_sync(0xffffffffu, f, l0 + i);
      const uint32_t si = __shfl_sync(0xffffffffu, so, l0 + i);
      warp_decode_staged(w.stg + si * 4u, fi, yi, dst + i * B, w.cnt, w.lut, sink);
    }
  }
}
template <bool PAIR = true>
__device__ __forceinline__ void decode_staged_lanes(const WarpSmem &w, uint32_t B, uint32_t l0,
                                                    uint32_t nb, uint32_t y, uint32_t f,
                                                    uint32_t so, uint32_t *dst) {
  StoreSink s;
  decode_staged_lanes<StoreSink, PAIR>(w, B, l0, nb, y, f, so, dst, s);
}

// EF-decode the consecutive blocks held by lanes [l0, l0+nb) (meta m, first f,
// payload size sz in 16-B units; contiguous in the payload) into dst + i*B,
// staging them with TMA bulk copies in batches that fit the staging area.
template <class Sink, bool PAIR = true>
__device__ __forceinline__ void stage_decode_lanes(const DevIndex &ix, WarpSmem &w, uint32_t cap16,
                                                   uint32_t l0, uint32_t nb, uint2 m, uint32_t f,
                                                   uint32_t sz, uint32_t *dst, Sink &sink) {
  const uint32_t lane = lane_id();
  const uint32_t incl = warp_incl_scan(lane >= l0 && lane < l0 + nb ? sz : 0u);
  uint32_t i = 0;
  while (i < nb) {
    const uint32_t li = l0 + i;
    const uint32_t base = __shfl_sync(0xffffffffu, incl - sz, li);   // exclusive prefix at li
    const uint32_t fits = __ballot_sync(0xffffffffu, lane >= li && lane < l0 + nb &&
                                                         incl - base <= cap16);
    uint32_t nbat = __popc(fits);
    if (nbat == 0) nbat = 1;   // cannot happen (one block always fits); keep progress
    const uint32_t bytes = (__shfl_sync(0xffffffffu, incl, li + nbat - 1) - base) * 16u;
    const uint32_t m0 = __shfl_sync(0xffffffffu, m.x, li);
    if (lane == 0) {
      fence_proxy_async();
      mbar_expect_tx(w.mbar, bytes);
      bulk_g2s(w.stg, ix.payload + m0, bytes, w.mbar);
    }
    mbar_wait(w.mbar, w.phase);
    w.phase ^= 1u;
    decode_staged_lanes<Sink, PAIR>(w, ix.B, li, nbat, m.y, f, m.x - m0, dst + i * ix.B, sink);
    i += nbat;
  }
}
template <bool PAIR = true>
__device__ __forceinline__ void stage_decode_lanes(const DevIndex &ix, WarpSmem &w, uint32_t cap16,
                                                   uint32_t l0, uint32_t nb, uint2 m, uint32_t f,
                                                   uint32_t sz, uint32_t *dst) {
  StoreSink s;
  stage_decode_lanes<StoreSink, PAIR>(ix, w, cap16, l0, nb, m, f, sz, dst, s);
}

// Load R "block" k of an intermediate (chunk of B entries) into dst.
__device__ __forceinline__ uint32_t load_r_chunk(const uint2 *Rq, uint32_t nR, uint32_t B,
                                                 uint32_t k, uint32_t *dst) {
  const uint32_t lane = lane_id();
  const uint32_t s = k * B;
  const uint32_t n = min(B, nR - s);
  for (uint32_t i = lane; i < n; i += 32) dst[i] = Rq[s + i].x;
  __syncwarp();
  return n;
}

// Emission of a unit's survivors, already compacted in R order: survivor j is
// R tile element idx[j] (list position posR0 + idx[j]), found at S position
// spos[j].  KIND 0: round 1 (s = w_R + w_S); KIND 1: later round (s = s_prev +
// w_S); KIND 2: single-term (s = w_R; survivor j is tile element j, no idx).
// Every lane scores a survivor (gathers: norm, tf of S, tf of R or the previous
// partial score) and the unit's entries are written contiguously.
// rtf (KIND 0, optional): R's packed tf words from bit rtf_bit0 on, staged in
// shared memory, so R's tf is read there instead of gathered.
template <int KIND>
__device__ __forceinline__ void emit_compact(const DevIndex &ix, const RoundArgs &a, uint32_t u,
                                             const TermInfo &tR, const TermInfo &tS,
                                             const uint2 *Rq, const uint32_t *tile,
                                             const uint32_t *idx, const uint32_t *spos,
                                             uint32_t cnt, uint32_t posR0, Acc &acc,
                                             const uint32_t *rtf = nullptr,
                                             uint64_t rtf_bit0 = 0) {
  const uint32_t lane = lane_id();
  unsigned long long off = 0;
  if (lane == 0 && cnt) off = bump_alloc(a, acc, cnt);
  off = __shfl_sync(0xffffffffu, off, 0);
  if (off + cnt > a.bump_cap) {
    if (lane == 0) atomicOr(reinterpret_cast<int *>(a.scal + kScalStatus), kStatusOverflow);
    cnt = 0;
  }
  for (uint32_t j = lane; j < cnt; j += 32u) {
    const uint32_t i = KIND == 2 ? j : idx[j];
    const uint32_t doc = tile[i];
    const float nrm = __ldg(ix.norm + doc);
    float s;
    if (KIND == 2) {
      s = bm25_w(tR.idf, tf_lookup(ix, tR, posR0 + i), nrm, ix.k1p1);
    } else {
      const uint32_t t1 = tf_lookup(ix, tS, spos[j]);
      uint32_t t2;
      if (KIND == 0 && rtf) {
        const uint32_t bit = (uint32_t)((uint64_t)(posR0 + i) * tR.tf_w - rtf_bit0);
        t2 = (__funnelshift_r(rtf[bit >> 5], rtf[(bit >> 5) + 1], bit) &
              (0xFFFFFFFFu >> (32u - tR.tf_w))) + 1u;
      } else {
        t2 = KIND == 0 ? tf_lookup(ix, tR, posR0 + i) : Rq[posR0 + i].y;
      }
      const float wS = bm25_w(tS.idf, t1, nrm, ix.k1p1);
      if (KIND == 0) {
        s = bm25_w(tR.idf, t2, nrm, ix.k1p1);  // first term: s = w
        s = __fadd_rn(s, wS);
      } else {
        s = __fadd_rn(__uint_as_float(t2), wS);
      }
    }
    a.bump[off + j] = make_uint2(doc, __float_as_uint(s));
  }
  __syncwarp();
  if (lane == 0) {
    a.unit_off[u] = off;
    a.unit_cnt[u] = cnt;
    acc.ctr[kCSurv] += cnt;
    acc.ctr[kCAlg] += (unsigned long long)cnt * (KIND == 0 ? kSurvBytesR1 : kSurvBytes);
  }
}

// Emission of the matched R-tile elements [0, n) (match[i] = S position or
// kNone): compact the matches first (R tile index -> idx[], S position ->
// match[] in place, in R order), so the scoring loop runs every lane on a
// survivor instead of one lane in ~three.  idx: >= n words of scratch.
template <int KIND>
__device__ __forceinline__ void emit_unit(const DevIndex &ix, const RoundArgs &a, uint32_t u,
                                          const TermInfo &tR, const TermInfo &tS, const uint2 *Rq,
                                          const uint32_t *tile, uint32_t *match, uint32_t *idx,
                                          uint32_t n, uint32_t posR0, Acc &acc) {
  const uint32_t lane = lane_id(), lt = lanemask_lt();
  uint32_t cnt = 0;
  if (KIND == 2) {
    cnt = n;
  } else {
    for (uint32_t c0 = 0; c0 < n; c0 += 32) {
      const uint32_t i = c0 + lane;
      const uint32_t mv = i < n ? match[i] : kNone;
      const bool p = mv != kNone;
      const uint32_t bal = __ballot_sync(0xffffffffu, p);
      __syncwarp();   // every lane has read its match[i] before any compacted write
      if (p) {
        const uint32_t o = cnt + __popc(bal & lt);   // o <= i: in place is safe
        idx[o] = i;
        match[o] = mv;
      }
      cnt += __popc(bal);
    }
    __syncwarp();
  }
  emit_compact<KIND>(ix, a, u, tR, tS, Rq, tile, idx, match, cnt, posR0, acc);
}

// Ordered emission of per-lane match lists (merge units): lane l found c
// matches, packed (R tile index | S tile index << 16) at ml0[l*cap ..+c); lanes
// are in merge-path order, so the warp's j-th match overall is match
// j - excl[s] of the lane s whose inclusive count first exceeds j.  The matches
// are spread evenly over the lanes (4 per lane per pass, gathers issued
// together so their latencies overlap) and written coalesced.
// Round 1 (RC): s = w_R + w_S; later rounds: s = s_prev + w_S.
template <bool RC>
__device__ void emit_lanes(const DevIndex &ix, const RoundArgs &a, uint32_t u, const TermInfo &tR,
                           const TermInfo &tS, const uint2 *Rq, const uint32_t *tile,
                           const uint32_t *ml0, uint32_t cap, uint32_t c, uint32_t *scr,
                           uint32_t posR0, uint32_t posS0, uint32_t abase, uint32_t bbase,
                           Acc &acc) {
  const uint32_t lane = lane_id();
  const uint32_t incl = warp_incl_scan(c);
  uint32_t cnt = __shfl_sync(0xffffffffu, incl, 31);
  unsigned long long off = 0;
  if (lane == 0 && cnt) off = bump_alloc(a, acc, cnt);
  off = __shfl_sync(0xffffffffu, off, 0);
  if (off + cnt > a.bump_cap) {
    if (lane == 0) atomicOr(reinterpret_cast<int *>(a.scal + kScalStatus), kStatusOverflow);
    cnt = 0;
  }
  if (cnt) {
    scr[lane] = incl;
    __syncwarp();
    uint2 *dst = a.bump + off;
    for (uint32_t j0 = 0; j0 < cnt; j0 += 32u * kEmitDepth) {
      uint32_t doc[kEmitDepth], tS_[kEmitDepth], tR_[kEmitDepth], prev[kEmitDepth];
      float nrm[kEmitDepth];
#pragma unroll
      for (int t = 0; t < kEmitDepth; ++t) {
        const uint32_t j = j0 + 32u * t + lane;
        if (j < cnt) {
          uint32_t o = 0;   // owner lane: number of lanes with incl <= j
#pragma unroll
          for (uint32_t step = 16; step; step >>= 1)
            if (scr[o + step - 1] <= j) o += step;
          const uint32_t ex = o ? scr[o - 1] : 0u;
          const uint32_t e = ml0[o * cap + (j - ex)];
          const uint32_t i = ((e - abase) & 0xFFFFu) >> 2;            // R tile index
          const uint32_t js = (((e >> 16) - bbase) & 0xFFFFu) >> 2;   // S index from Bv
          doc[t] = tile[i];
          nrm[t] = __ldg(ix.norm + doc[t]);
          tS_[t] = tf_lookup(ix, tS, posS0 + js);
          if (RC) tR_[t] = tf_lookup(ix, tR, posR0 + i);
          else prev[t] = Rq[posR0 + i].y;
        }
      }
#pragma unroll
      for (int t = 0; t < kEmitDepth; ++t) {
        const uint32_t j = j0 + 32u * t + lane;
        if (j < cnt) {
          const float wS = bm25_w(tS.idf, tS_[t], nrm[t], ix.k1p1);
          float s;
          if (RC) {
            s = bm25_w(tR.idf, tR_[t], nrm[t], ix.k1p1);  // first term: s = w
            s = __fadd_rn(s, wS);
          } else {
            s = __fadd_rn(__uint_as_float(prev[t]), wS);
          }
          dst[j] = make_uint2(doc[t], __float_as_uint(s));
        }
      }
    }
    __syncwarp();
  }
  if (lane == 0) {
    a.unit_off[u] = off;
    a.unit_cnt[u] = cnt;
    acc.ctr[kCSurv] += cnt;
    acc.ctr[kCAlg] += (unsigned long long)cnt * (RC ? kSurvBytesR1 : kSurvBytes);
  }
}

// Coarse merge path over the block heads: lanes 0-15 find the crossing of
// diagonal d0, lanes 16-31 of d1, with a 16-ary search (each step probes 16
// points of the diagonal and narrows the range to one interval).
template <class HR, class HS>
__device__ __forceinline__ void warp_mp_search2(HR hR, uint32_t nbR, HS hS, uint32_t nbS,
                                                uint32_t d0, uint32_t d1, uint32_t *i0,
                                                uint32_t *i1) {
  const uint32_t lane = lane_id(), half = lane >> 4, hl = lane & 15u;
  const uint32_t d = half ? d1 : d0;
  // answer: smallest i in [lo, hi] with pred(i) = hR(i) > hS(d-i-1); pred(hi) := true
  uint32_t lo = d > nbS ? d - nbS : 0u;
  uint32_t hi = d < nbR ? d : nbR;
  for (;;) {
    const bool done = lo >= hi;
    if (__all_sync(0xffffffffu, done)) break;
    const uint32_t span = hi - lo;
    // probes cand(p) = lo + ceil((p+1)*span/16) - 1, p = 0..15; cand(15) = hi-1
    auto cand = [&](uint32_t p) -> uint32_t {
      return lo + (uint32_t)(((uint64_t)(p + 1) * span + 15u) / 16u) - 1u;
    };
    bool pred = true;
    if (!done) {
      const uint32_t c = cand(hl);
      pred = hR(c) > hS(d - c - 1);
    }
    const uint32_t hb = (__ballot_sync(0xffffffffu, pred) >> (half * 16u)) & 0xFFFFu;
    if (!done) {
      if (hb == 0) {
        lo = hi;
      } else {
        const uint32_t ps = __ffs(hb) - 1u;
        const uint32_t nhi = cand(ps);
        const uint32_t nlo = ps ? cand(ps - 1) + 1u : lo;
        hi = nhi;
        lo = nlo;
      }
    }
  }
  *i0 = __shfl_sync(0xffffffffu, lo, 0);
  *i1 = __shfl_sync(0xffffffffu, lo, 16);
}

// Partitioning stage ("Partitioning and Merging"): one thread per
// unit locates the unit's query and, for merge units, the crossing of the merge
// path with the unit's first diagonal over the two lists' block heads
// and the unit's first docID.  The merging stage reads {q, i0, j0, lo} of unit u
// and of unit u+1 (its end), so no warp ever searches on the critical path.
template <bool RC>
__device__ __forceinline__ void unit_record(const DevIndex &ix, const RoundArgs &a, uint64_t u);

// bucket of merge unit u for the S-locality order: global S block of its start
__device__ __forceinline__ uint32_t merge_unit_bucket(const DevIndex &ix, const RoundArgs &a,
                                                      uint64_t u) {
  const uint4 rec = a.urec[u];
  const uint32_t sid = a.plan_terms[(size_t)rec.x * kMaxTerms + a.round];
  return (ix.terms[sid].block0 + rec.z) >> a.sbkt_shift;
}

// Processing-order entry of unit u of query q: {u, q | mode << 29, R term,
// this round's S term}, so a kernel's unit head needs one dependent load (this
// entry) before it can fetch the unit record and both TermInfos in parallel.
__device__ __forceinline__ uint4 uperm_entry(const RoundArgs &a, uint64_t u, uint32_t q) {
  const uint32_t *pt = a.plan_terms + (size_t)q * kMaxTerms;
  return make_uint4((uint32_t)u, q | (a.qmode[q] << 29), pt[0], pt[a.round % kMaxTerms]);
}

// Units handed out in bitvector order (after the merge buckets): bitvector
// units, and probe-pass units whose first remaining list is a bitvector.
__device__ __forceinline__ bool bm_bucketed(const RoundArgs &a, uint32_t q) {
  const uint32_t md = a.qmode[q];
  return a.sbkt_nbb && (md == kModeBitmap || md == kModeBitAnd ||
                        (md == kModeProbe && a.tdec &&
                         a.tdec[a.plan_terms[(size_t)q * kMaxTerms + a.round]] == kDecBitmap));
}
// its bucket: the bitvector's slot and the unit's first R docID
template <bool RC>
__device__ __forceinline__ uint64_t bitmap_unit_bucket(const DevIndex &ix, const RoundArgs &a,
                                                       uint64_t u) {
  const uint4 rec = a.urec[u];
  const uint32_t q = rec.x, lu = rec.y;
  const uint32_t *pt = a.plan_terms + (size_t)q * kMaxTerms;
  uint32_t x0;
  if (a.qmode[q] == kModeProbe) {
    x0 = a.rprev[a.roff_prev[q] + (size_t)lu * a.pchunk].x;
  } else if (a.qmode[q] == kModeBitAnd) {
    x0 = (((__ldg(ix.first + ix.terms[pt[0]].block0) >> 5) + lu * kAndWords) << 5);
  } else {
    const uint32_t b0 = lu * bm_unit_blocks(ix.B, a.D, a.nextgeq != 0);
    x0 = RC ? __ldg(ix.first + ix.terms[pt[0]].block0 + b0)
            : a.rprev[a.roff_prev[q] + (size_t)b0 * ix.B].x;
  }
  return a.sbkt_nm + (uint64_t)a.bm_slot[pt[a.round]] * a.sbkt_nbb + (x0 >> kBmBucketShift);
}

template <bool RC>
__global__ void partition_kernel(DevIndex ix, RoundArgs a) {
  const uint64_t total = a.unit_base[a.nq];
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t u = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; u <= total; u += stride) {
    if (u == total) {
      a.urec[u] = make_uint4(kNone, 0, 0, 0);
      continue;
    }
    unit_record<RC>(ix, a, u);
  }
  // Processing order: merge units first, then gallop/probe/single-term units,
  // so that at any time the warps mostly run one unit kind's code (the kernel
  // is instruction-cache bound).  Output placement depends only on unit ids,
  // so the (atomic, unordered) list does not affect results.
  for (uint64_t base = blockIdx.x * (uint64_t)blockDim.x; base < total; base += stride) {
    const uint64_t u = base + threadIdx.x;
    const bool valid = u < total;
    uint32_t q = 0;
    if (valid) q = a.urec[u].x;
    const bool mg = valid && a.qmode[q] == kModeMerge;
    // bitvector units are bucketed too when the order is on (after the merge units)
    const bool bu = valid && a.sbkt_cnt && bm_bucketed(a, q);
    const uint32_t bm = __ballot_sync(0xffffffffu, mg),
                   bo = __ballot_sync(0xffffffffu, valid && !mg && !bu);
    const uint32_t lane = threadIdx.x & 31u, lt = (1u << lane) - 1u;
    unsigned long long hm = 0, ho = 0;
    if (lane == 0) {
      if (bm) hm = atomicAdd(a.scal + kScalPerm, (unsigned long long)__popc(bm));
      if (bo) ho = atomicAdd(a.scal + kScalPerm + 1, (unsigned long long)__popc(bo));
    }
    hm = __shfl_sync(0xffffffffu, hm, 0);
    ho = __shfl_sync(0xffffffffu, ho, 0);
    if (mg) {
      if (a.sbkt_cnt) atomicAdd(a.sbkt_cnt + merge_unit_bucket(ix, a, u), 1u);
      else a.uperm[hm + __popc(bm & lt)] = uperm_entry(a, u, q);
    } else if (bu) {
      atomicAdd(a.sbkt_cnt + bitmap_unit_bucket<RC>(ix, a, u), 1u);
    } else if (valid) {
      a.uperm[total - 1 - (ho + __popc(bo & lt))] = uperm_entry(a, u, q);
    }
  }
}

// S-locality order (after partition_kernel and a scan of the bucket counts):
// used for batches of >= kSorderMinQueries queries (C5, 10K queries: intersect
// 15.41 -> 14.76 ms; at C2's 1000 queries the extra scan + scatter cost more
// than the reuse gains: 0.703 -> 0.722 ms, profiles/r01_configs.jsonl).
// merge units are placed by the global S block their range starts at, so the
// units of different queries that merge against the same S range are handed
// out together and their S tiles come from L2 (a C2 batch merges 92M S
// postings of 39M distinct ones, C5 2.66 B of 455M).  Order inside a bucket is
// arbitrary; results do not depend on processing order.
#ifndef GRIFFIN_SORDER_MIN_QUERIES
#define GRIFFIN_SORDER_MIN_QUERIES 4096
#endif
constexpr uint32_t kSorderMinQueries = GRIFFIN_SORDER_MIN_QUERIES;
template <bool RC>
__global__ void sorder_scatter_kernel(DevIndex ix, RoundArgs a) {
  const uint64_t total = a.unit_base[a.nq];
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t u = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; u < total; u += stride) {
    const uint32_t q = a.urec[u].x;
    const uint32_t md = a.qmode[q];
    if (md != kModeMerge && !bm_bucketed(a, q)) continue;
    const uint64_t bk = md == kModeMerge ? merge_unit_bucket(ix, a, u) : bitmap_unit_bucket<RC>(ix, a, u);
    const unsigned long long slot = atomicAdd(a.sbkt_pos + bk, 1ull);
    a.uperm[slot] = uperm_entry(a, u, q);
  }
}

// Partition-stage record of unit u (see partition_kernel).
template <bool RC>
__device__ __forceinline__ void unit_record(const DevIndex &ix, const RoundArgs &a, uint64_t u) {
  {
    uint32_t lo = 0, hi = a.nq;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (a.unit_base[mid] <= u) lo = mid; else hi = mid;
    }
    const uint32_t q = lo;
    const uint32_t lu = (uint32_t)(u - a.unit_base[q]);
    uint4 rec = make_uint4(q, lu, 0, 0);
    if (a.qmode[q] == kModeGallop) {
      // skip-pointer range the R chunk can touch: [upper_bound(first elem) - 1,
      // upper_bound(last elem)); for a compressed R block the next block's head
      // bounds its last element
      const uint32_t *pt = a.plan_terms + (size_t)q * kMaxTerms;
      const TermInfo tR = ix.terms[pt[0]];
      const TermInfo tS = ix.terms[pt[a.round]];
      uint32_t x0, x1;
      if (RC) {
        x0 = __ldg(ix.first + tR.block0 + lu);
        x1 = lu + 1 < tR.nblocks ? __ldg(ix.first + tR.block0 + lu + 1) - 1u : 0xFFFFFFFFu;
      } else {
        const uint2 *Rq = a.rprev + a.roff_prev[q];
        const uint32_t s0 = lu * ix.B, s1 = min(s0 + ix.B, a.rcount[q]);
        x0 = Rq[s0].x;
        x1 = Rq[s1 - 1].x;
      }
      rec.z = upper_bound_g(ix.first + tS.block0, 0, tS.nblocks, x0);
      rec.w = upper_bound_g(ix.first + tS.block0, rec.z, tS.nblocks, x1);
    }
    if (a.qmode[q] == kModeMerge) {
      const uint32_t *pt = a.plan_terms + (size_t)q * kMaxTerms;
      const TermInfo tR = ix.terms[pt[0]];
      const TermInfo tS = ix.terms[pt[a.round]];
      const uint2 *Rq = RC ? nullptr : a.rprev + a.roff_prev[q];
      const uint32_t nbR = RC ? tR.nblocks : (a.rcount[q] + ix.B - 1) / ix.B;
      const uint32_t nbS = tS.nblocks;
      auto hR = [&](uint32_t i) -> uint32_t {
        return RC ? __ldg(ix.first + tR.block0 + i) : Rq[(size_t)i * ix.B].x;
      };
      auto hS = [&](uint32_t j) -> uint32_t { return __ldg(ix.first + tS.block0 + j); };
      const uint32_t d0 = lu * a.D;
      uint32_t i0, j0;
      merge_path_split(hR, nbR, hS, nbS, d0, false, &i0, &j0);
      uint32_t lov = 0;
      if (d0 > 0) {
        const uint64_t INF = 1ull << 32;
        lov = (uint32_t)min(i0 < nbR ? (uint64_t)hR(i0) : INF, j0 < nbS ? (uint64_t)hS(j0) : INF);
      }
      rec = make_uint4(q, i0, j0, lov);
    }
    a.urec[u] = rec;
  }
}

// Warp-cooperative upper_bound over a[0..n) (global): lanes 0-15 search x0,
// lanes 16-31 search x1, 16 probes per step (log16 steps instead of log2).
__device__ __forceinline__ void warp_upper_bound2(const uint32_t *__restrict__ a, uint32_t n,
                                                  uint32_t x0, uint32_t x1, uint32_t *r0,
                                                  uint32_t *r1) {
  const uint32_t lane = lane_id(), half = lane >> 4, hl = lane & 15u;
  const uint32_t x = half ? x1 : x0;
  uint32_t lo = 0, hi = n;   // answer: smallest i in [lo, hi] with a[i] > x (a[n] := inf)
  for (;;) {
    const bool done = lo >= hi;
    if (__all_sync(0xffffffffu, done)) break;
    const uint32_t span = hi - lo;
    auto cand = [&](uint32_t p) -> uint32_t {
      return lo + (uint32_t)(((uint64_t)(p + 1) * span + 15u) / 16u) - 1u;
    };
    bool pred = true;
    if (!done) pred = __ldg(a + cand(hl)) > x;
    const uint32_t hb = (__ballot_sync(0xffffffffu, pred) >> (half * 16u)) & 0xFFFFu;
    if (!done) {
      if (hb == 0) {
        lo = hi;
      } else {
        const uint32_t ps = __ffs(hb) - 1u;
        const uint32_t nhi = cand(ps);
        const uint32_t nlo = ps ? cand(ps - 1) + 1u : lo;
        hi = nhi;
        lo = nlo;
      }
    }
  }
  *r0 = __shfl_sync(0xffffffffu, lo, 0);
  *r1 = __shfl_sync(0xffffffffu, lo, 16);
}

// Skip-pointer block of each R element x (upper_bound(fS, x) - 1, kNone when x
// precedes the list), for element lists whose range spans many skip pointers:
// every `stride`-th skip pointer of [k_lo, k_hi) is sampled into shared memory
// in one coalesced pass, each element binary-searches the sample there, and only
// the last log2(stride) steps touch global memory, as interleaved independent
// chains (kSkipDepth elements per lane).  Also resets match[].
__device__ __forceinline__ void skip_blocks_sampled(const uint32_t *__restrict__ fS, uint32_t k_lo,
                                                    uint32_t k_hi, const uint32_t *tileR,
                                                    uint32_t n, uint32_t *kidx, uint32_t *match,
                                                    uint32_t *samp, uint32_t cap) {
  const uint32_t lane = lane_id();
  const uint32_t span = k_hi - k_lo;
  uint32_t stride = 1;
  while ((span + stride - 1) / stride > cap) stride <<= 1;
  const uint32_t ns = (span + stride - 1) / stride;
  for (uint32_t i = lane; i < ns; i += 32) samp[i] = __ldg(fS + k_lo + i * stride);
  __syncwarp();
  for (uint32_t base = 0; base < n; base += 32u * kSkipDepth) {
    uint32_t lo[kSkipDepth], hi[kSkipDepth], xv[kSkipDepth];
#pragma unroll
    for (int j = 0; j < kSkipDepth; ++j) {
      const uint32_t e = base + lane + 32u * j;
      xv[j] = e < n ? tileR[e] : 0u;
      // sample interval: t = #samples <= x; the answer lies in (k_lo+(t-1)*stride, k_lo+t*stride]
      uint32_t a = 0, b = ns;
      while (a < b) {
        const uint32_t mid = (a + b) >> 1;
        if (samp[mid] <= xv[j]) a = mid + 1; else b = mid;
      }
      lo[j] = a ? k_lo + (a - 1) * stride + 1 : k_lo;
      hi[j] = (e < n && a) ? min(k_lo + a * stride, k_hi) : lo[j];
    }
    for (;;) {
      bool any = false;
#pragma unroll
      for (int j = 0; j < kSkipDepth; ++j) {
        if (lo[j] < hi[j]) {
          const uint32_t mid = (lo[j] + hi[j]) >> 1;
          if (__ldg(fS + mid) <= xv[j]) lo[j] = mid + 1; else hi[j] = mid;
          any = true;
        }
      }
      if (!__any_sync(0xffffffffu, any)) break;
    }
#pragma unroll
    for (int j = 0; j < kSkipDepth; ++j) {
      const uint32_t e = base + lane + 32u * j;
      if (e < n) {
        kidx[e] = lo[j] - 1u;   // kNone (0 - 1) when x < fS[k_lo] and k_lo == 0
        match[e] = kNone;
      }
    }
  }
  __syncwarp();
}

// Arena probe (gallop / probe pass into a list decoded in the batch arena): each
// R element x knows its S block kb (skip search: first[kb] <= x < first[kb+1]).
// Docs are spread evenly enough inside a block that interpolation on the skip
// range [first[kb], first[kb+1]) lands in or next to the right 8-key chunk (one
// 32-B sector, 32-B aligned): load it, step one chunk left/right until x is
// bracketed, then compare.  ~1-2 dependent sector loads per probe instead of
// log2(B) for a binary search.  kArenaEpl independent probes per lane run in
// lockstep so their loads overlap.  Writes match[e] = kb*B + pos on a hit and
// returns the number of chunks loaded.
#ifndef GRIFFIN_ARENA_EPL
#define GRIFFIN_ARENA_EPL 2
#endif
constexpr int kArenaEpl = GRIFFIN_ARENA_EPL;
__device__ __forceinline__ uint32_t arena_probe_slice(const uint32_t *__restrict__ decS,
                                                      const uint32_t *__restrict__ fS,
                                                      uint32_t nblocksS, uint32_t dfS, uint32_t B,
                                                      const uint32_t *tileR, const uint32_t *kidx,
                                                      uint32_t *match, uint32_t base, uint32_t n) {
  const uint32_t lane = lane_id();
  uint32_t xv[kArenaEpl], kb[kArenaEpl], nb[kArenaEpl], c[kArenaEpl], dir[kArenaEpl];
  bool act[kArenaEpl];
  uint32_t chunks = 0;
#pragma unroll
  for (int j = 0; j < kArenaEpl; ++j) {
    const uint32_t e = base + lane + 32u * j;
    act[j] = false;
    kb[j] = kNone;
    xv[j] = 0;
    nb[j] = 0;
    c[j] = 0;
    dir[j] = 0;
    if (e < n) {
      kb[j] = kidx[e];
      if (kb[j] != kNone) {
        act[j] = true;
        xv[j] = tileR[e];
        nb[j] = min(B, dfS - kb[j] * B);
      }
    }
  }
  // interpolation estimate (the last block's upper end is its last element + 1)
  uint32_t f0[kArenaEpl], f1[kArenaEpl];
#pragma unroll
  for (int j = 0; j < kArenaEpl; ++j) {
    f0[j] = f1[j] = 0;
    if (act[j]) {
      f0[j] = __ldg(fS + kb[j]);
      f1[j] = kb[j] + 1 < nblocksS ? __ldg(fS + kb[j] + 1)
                                   : __ldg(decS + (size_t)kb[j] * B + nb[j] - 1) + 1u;
    }
  }
#pragma unroll
  for (int j = 0; j < kArenaEpl; ++j) {
    if (act[j]) {
      // a starting chunk only (the walk below finds x from any start): float
      // arithmetic instead of a 64-bit integer division
      const uint32_t span = f1[j] > f0[j] ? f1[j] - f0[j] : 1u;
      const float fe = __fmul_rz((float)(xv[j] - f0[j]), __fdividef((float)nb[j], (float)span));
      const uint32_t est = min(__float2uint_rz(fe), nb[j] - 1u);
      c[j] = est & ~7u;
    }
  }
  for (;;) {
    bool any = false;
#pragma unroll
    for (int j = 0; j < kArenaEpl; ++j) {
      if (!act[j]) continue;
      any = true;
      ++chunks;
      const uint4 *p = reinterpret_cast<const uint4 *>(decS + (size_t)kb[j] * B + c[j]);
      const uint4 lo4 = __ldg(p), hi4 = __ldg(p + 1);
      uint32_t v[8] = {lo4.x, lo4.y, lo4.z, lo4.w, hi4.x, hi4.y, hi4.z, hi4.w};
      const uint32_t valid = min(8u, nb[j] - c[j]);
      if (valid < 8u) {   // a block's tail: slots past its end hold no docIDs
#pragma unroll
        for (uint32_t i = 0; i < 8; ++i) v[i] = i < valid ? v[i] : kNone;
      }
      // less = #{v[i] < x} by a branch-free 3-step search of the sorted chunk,
      // eq = (v[less] == x)
      const uint32_t x = xv[j];
      const bool b4 = v[3] < x;
      const uint32_t a0 = b4 ? v[4] : v[0], a1 = b4 ? v[5] : v[1], a2 = b4 ? v[6] : v[2],
                     a3 = b4 ? v[7] : v[3];
      const bool b2 = a1 < x;
      const uint32_t e0 = b2 ? a2 : a0, e1 = b2 ? a3 : a1;
      const bool b1 = e0 < x;
      const uint32_t d0 = b1 ? e1 : e0;
      const bool b0 = d0 < x;
      const uint32_t less = (b4 ? 4u : 0u) + (b2 ? 2u : 0u) + (b1 ? 1u : 0u) + (b0 ? 1u : 0u);
      const uint32_t eq = (!b0 && d0 == x) ? 1u : 0u;
      // step toward x, never reversing: a reversal means x falls between two
      // adjacent chunks, i.e. it is absent
      if (less == 0 && !eq && c[j] > 0 && dir[j] != 2u) {
        c[j] -= 8;                       // x lies before this chunk
        dir[j] = 1u;
      } else if (less == valid && c[j] + 8u < nb[j] && dir[j] != 1u) {
        c[j] += 8;                       // x lies after this chunk
        dir[j] = 2u;
      } else {
        if (eq) match[base + lane + 32u * j] = kb[j] * B + c[j] + less;
        act[j] = false;
      }
    }
    if (!__any_sync(0xffffffffu, any)) break;
  }
  return chunks;
}

// Bitvector lookups of the elements x = tileR[0..n): match[e] = x's position
// in S, or kNone (4 independent 8-B loads in flight per lane).  Counting pass:
// one 32-B sector per distinct sector the warp reads in list order (SURVEY
// §8(d) charges gathers by sector).
__device__ __forceinline__ void bitvec_probe(const uint2 *__restrict__ bm,
                                             const uint32_t *tileR, uint32_t *match, uint32_t n,
                                             int count, Acc &acc) {
  const uint32_t lane = lane_id();
  uint32_t sectors = 0;
  for (uint32_t base = 0; base < n; base += 128u) {
    uint32_t x[4];
    uint2 wv[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const uint32_t e = base + lane + 32u * j;
      x[j] = e < n ? tileR[e] : 0u;
      wv[j] = e < n ? __ldg(bm + (x[j] >> 5)) : make_uint2(0, 0);
    }
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const uint32_t e = base + lane + 32u * j;
      if (e < n) {
        match[e] = bitvec_pos(wv[j], x[j]);
        if (count) sectors += (e == 0 || (tileR[e - 1] >> 7) != (x[j] >> 7)) ? 1u : 0u;
      }
    }
  }
  if (count) {
    const uint32_t sp = __reduce_add_sync(0xffffffffu, sectors);
    if (lane == 0) acc.ctr[kCAlg] += sp * 32ull;
  }
  __syncwarp();
}

// Bitvector lookups of the elements x = tileR[0..n), compacted in R order:
// the j-th hit is tile element idx[j] at S position spos[j]; returns the
// number of hits.  4 independent 8-B loads in flight per lane.
// 128 elements from base (4 per lane, independent loads in flight); FULL: no
// bounds checks (every element < n)
template <bool FULL>
__device__ __forceinline__ void bitvec_chunk(const uint2 *__restrict__ bm, const uint32_t *tileR,
                                             uint32_t base, uint32_t n, uint32_t *idx,
                                             uint32_t *spos, uint32_t &cnt) {
  const uint32_t lane = lane_id(), lt = lanemask_lt();
  uint32_t x[4];
  uint2 wv[4];
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint32_t e = base + lane + 32u * j;
    const bool in = FULL || e < n;
    x[j] = in ? tileR[e] : 0u;
    wv[j] = in ? __ldg(bm + (x[j] >> 5)) : make_uint2(0, 0);
  }
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint32_t bit = x[j] & 31u;
    const bool hit = (wv[j].x >> bit) & 1u;   // (0 for out-of-range lanes: word 0 loaded as zero)
    const uint32_t bal = __ballot_sync(0xffffffffu, hit);
    if (hit) {
      const uint32_t o = cnt + __popc(bal & lt);
      idx[o] = base + lane + 32u * j;
      spos[o] = ~wv[j].y + __popc(wv[j].x & ((1u << bit) - 1u));
    }
    cnt += __popc(bal);
  }
}

// Bitvector lookups of the elements x = tileR[0..n), compacted in R order:
// the j-th hit is tile element idx[j] at S position spos[j]; returns the
// number of hits.  Counting pass: one 32-B sector per distinct sector the
// warp reads in list order (SURVEY §8(d) charges gathers by sector).
__device__ __forceinline__ uint32_t bitvec_probe_compact(const uint2 *__restrict__ bm,
                                                         const uint32_t *tileR, uint32_t n,
                                                         uint32_t *idx, uint32_t *spos, int count,
                                                         Acc &acc) {
  const uint32_t lane = lane_id();
  uint32_t cnt = 0, base = 0;
  for (; base + 128u <= n; base += 128u) bitvec_chunk<true>(bm, tileR, base, n, idx, spos, cnt);
  if (base < n) bitvec_chunk<false>(bm, tileR, base, n, idx, spos, cnt);
  if (count) {
    uint32_t sectors = 0;
    for (uint32_t e = lane; e < n; e += 32u)
      sectors += (e == 0 || (tileR[e - 1] >> 7) != (tileR[e] >> 7)) ? 1u : 0u;
    const uint32_t sp = __reduce_add_sync(0xffffffffu, sectors);
    if (lane == 0) acc.ctr[kCAlg] += sp * 32ull;
  }
  __syncwarp();
  return cnt;
}

// Multi-list probe (SvS rounds 2..m-1 in one pass): every round-1 survivor is
// looked up in each remaining list in canonical order — skip-pointer search,
// then an in-place binary search of the decoded-arena block or a staged EF
// decode of the touched compressed blocks — its BM25 contribution added
// (s = s + w_t, SURVEY O6 order), and dropped at the first list that misses it.
// The surviving set equals SvS's; only the loop order differs.
__device__ void probe_unit(const DevIndex &ix, const RoundArgs &a, WarpSmem &sm, uint64_t u,
                           uint32_t q, uint32_t lu, Acc &acc) {
  const uint32_t lane = lane_id(), lt = lanemask_lt();
  const uint32_t B = ix.B, D = a.D;
  const uint32_t G = min(D - 3u, 31u);
  const uint32_t *pt = a.plan_terms + (size_t)q * kMaxTerms;
  const uint32_t m = a.plan_m[q];
  const uint2 *Rq = a.rprev + a.roff_prev[q];
  const uint32_t nR = a.rcount[q];
  uint32_t *tileR = sm.tile, *sc = sm.tile + B, *nrm = sm.tile + 2 * B, *kidx = sm.tile + 3 * B;
  uint32_t *match = sm.tile + 4 * B, *tileS = sm.tile + 5 * B;
  uint32_t *dblk = sm.aux, *sn = sm.aux + B;
  const uint32_t s0 = lu * a.pchunk;
  uint32_t n = min(a.pchunk, nR - s0);
  for (uint32_t e = lane; e < n; e += 32) {
    const uint2 v = Rq[s0 + e];
    tileR[e] = v.x;
    sc[e] = v.y;
    nrm[e] = 0xFFFFFFFFu;   // gathered when the survivor first passes a list (most are dropped)
  }
  __syncwarp();
  if (lane == 0) acc.ctr[kCAlg] += n * 8u;
  for (uint32_t r = 2; r < m && n > 0; ++r) {
    const uint32_t sid = pt[r];
    const TermInfo tS = ix.terms[sid];
    const uint32_t *fS = ix.first + tS.block0;
    const uint8_t kd = a.tdec ? a.tdec[sid] : kDecNone;
    const bool sdec = kd == kDecArena;
    const uint32_t *decS = sdec ? a.dec + (size_t)tS.block0 * B : nullptr;
    if (kd == kDecBitmap) {
      // ---- S decoded into a bitvector: O(1) lookups, then the shared drop/score step ----
      bitvec_probe(a.bm + (size_t)a.bm_slot[sid] * a.bm_words, tileR, match, n, a.count, acc);
    } else {
    // skip pointers this chunk can touch: [ub(first survivor) - 1, ub(last)),
    // found by a warp-cooperative 16-ary search; a chunk usually spans few
    // enough of them to be searched from one coalesced smem window
    uint32_t k0, k1;
    warp_upper_bound2(fS, tS.nblocks, tileR[0], tileR[n - 1], &k0, &k1);
    skip_blocks_sampled(fS, k0 ? k0 - 1u : 0u, k1, tileR, n, kidx, match, sm.stg,
                        stage_words(B, D));
    if (sdec) {
      // ---- decoded arena: interpolation probes of the touched block ----
      uint32_t probes = 0;
      for (uint32_t base = 0; base < n; base += 32u * kArenaEpl)
        probes += arena_probe_slice(decS, fS, tS.nblocks, tS.df_local, B, tileR, kidx, match,
                                    base, n);
      const uint32_t sp = __reduce_add_sync(0xffffffffu, probes);
      if (lane == 0) acc.ctr[kCAlg] += sp * 32ull;
    } else {
      // ---- compressed: distinct touched blocks, staged + decoded in groups ----
      uint32_t nd = 0, prev = kNone, e_first = n;
      for (uint32_t c0 = 0; c0 < n; c0 += 32) {
        const uint32_t e = c0 + lane;
        const uint32_t kv = e < n ? kidx[e] : kNone;
        uint32_t kp = __shfl_up_sync(0xffffffffu, kv, 1);
        if (lane == 0) kp = prev;
        const bool newb = e < n && kv != kNone && kv != kp;
        const uint32_t bal = __ballot_sync(0xffffffffu, newb);
        if (newb) dblk[nd + __popc(bal & lt)] = kv;
        const uint32_t gi = nd + __popc(bal & (lt | (1u << lane))) - 1u;
        if (e < n) kidx[e] = kv == kNone ? kNone : gi;
        const uint32_t valid = __ballot_sync(0xffffffffu, e < n && kv != kNone);
        if (e_first == n && valid) e_first = c0 + __ffs(valid) - 1u;
        nd += __popc(bal);
        prev = __shfl_sync(0xffffffffu, kv, 31);
      }
      __syncwarp();
      uint32_t ep = e_first;
      const uint32_t cap16 = stage_words(B, D) / 4u;
      for (uint32_t g0 = 0; g0 < nd;) {
        uint32_t ng = min(G, nd - g0);
        uint2 mm = make_uint2(0, 0);
        uint32_t f = 0, sz = 0, blk = 0, nn = 0;
        if (lane < ng) {
          blk = dblk[g0 + lane];
          nn = min(B, tS.df_local - blk * B);
          mm = ix.meta[(uint64_t)tS.block0 + blk];
          f = ix.first[(uint64_t)tS.block0 + blk];
          sz = block_size16(mm.y);
        }
        const uint32_t inc = warp_incl_scan(sz);
        const uint32_t nfit = __popc(__ballot_sync(0xffffffffu, lane < ng && inc <= cap16));
        ng = nfit ? nfit : 1u;
        if (lane >= ng) sz = 0;
        if (lane < ng) sn[lane] = nn;
        const uint32_t pay = __reduce_add_sync(0xffffffffu, lane < ng ? sz * 16u : 0u);
        const uint32_t pst = __reduce_add_sync(0xffffffffu, lane < ng && !a.nextgeq ? nn : 0u);
        if (lane == 0) {
          acc.ctr[kCPay] += pay;
          acc.ctr[kCPost] += pst;
          acc.ctr[kCAlg] += pay + 8u * ng;
        }
        const uint32_t soff = warp_incl_scan(sz) - sz;
        stage_blocks(ix, sm, ng, mm, soff, sz, false);
        if (!a.nextgeq) {
          for (uint32_t i = 0; i < ng; ++i) {
            const uint32_t y = __shfl_sync(0xffffffffu, mm.y, i);
            const uint32_t fi = __shfl_sync(0xffffffffu, f, i);
            const uint32_t so = __shfl_sync(0xffffffffu, soff, i);
            warp_decode_staged(sm.stg + so * 4u, fi, y, tileS + i * B, sm.cnt, sm.lut);
          }
        }
        __syncwarp();
        for (;;) {
          const uint32_t e = ep + lane;
          const uint32_t gi = e < n ? kidx[e] : kNone;
          const bool in = gi != kNone && gi < g0 + ng;
          if (a.nextgeq) {
            const uint32_t src = in ? gi - g0 : 0u;
            const uint32_t y = __shfl_sync(0xffffffffu, mm.y, src);
            const uint32_t fi = __shfl_sync(0xffffffffu, f, src);
            const uint32_t so = __shfl_sync(0xffffffffu, soff, src);
            if (in) {
              const uint32_t x = tileR[e];
              uint32_t v;
              const uint32_t p = ef_next_geq_staged(sm.stg + so * 4u, fi, y, x, sm.lut, v);
              if (p < meta_n(y) && v == x) match[e] = dblk[gi] * B + p;
            }
          } else if (in) {
            const uint32_t x = tileR[e];
            const uint32_t *seg = tileS + (gi - g0) * B;
            const uint32_t p = lower_bound_s(seg, 0, sn[gi - g0], x);
            if (p < sn[gi - g0] && seg[p] == x) match[e] = dblk[gi] * B + p;
          }
          const uint32_t bal = __ballot_sync(0xffffffffu, in);
          ep += __popc(bal);
          if (bal != 0xffffffffu) break;
        }
        __syncwarp();
        g0 += ng;
      }
    }
    }   // compressed / arena S
    __syncwarp();
    // ---- add w_t to the members, drop the rest (stable in-place compaction) ----
    uint32_t nn2 = 0;
    for (uint32_t c0 = 0; c0 < n; c0 += 32) {
      const uint32_t e = c0 + lane;
      const bool in = e < n;
      const uint32_t x = in ? tileR[e] : 0u, mt = in ? match[e] : kNone;
      uint32_t nm = in ? nrm[e] : 0u;
      float s = in ? __uint_as_float(sc[e]) : 0.f;
      const bool keep = in && mt != kNone;
      const bool gather = keep && nm == 0xFFFFFFFFu;
      if (gather) nm = __float_as_uint(__ldg(ix.norm + x));   // (norms are finite)
      if (a.count) {
        const uint32_t ng = __popc(__ballot_sync(0xffffffffu, gather));
        if (lane == 0) acc.ctr[kCAlg] += ng * 4u;   // the doc's norm, once
      }
      if (keep) s = __fadd_rn(s, bm25_w(tS.idf, tf_lookup(ix, tS, mt), __uint_as_float(nm), ix.k1p1));
      const uint32_t bal = __ballot_sync(0xffffffffu, keep);
      __syncwarp();
      if (keep) {
        const uint32_t pos = nn2 + __popc(bal & lt);
        tileR[pos] = x;
        sc[pos] = __float_as_uint(s);
        nrm[pos] = nm;
      }
      nn2 += __popc(bal);
      __syncwarp();
    }
    n = nn2;
    if (lane == 0) acc.ctr[kCAlg] += n * kTfSector;   // the kept survivors' tf gathers
  }
  // ---- emit the survivors ----
  unsigned long long off = 0;
  uint32_t cnt = n;
  if (lane == 0 && cnt) off = bump_alloc(a, acc, cnt);
  off = __shfl_sync(0xffffffffu, off, 0);
  if (off + cnt > a.bump_cap) {
    if (lane == 0) atomicOr(reinterpret_cast<int *>(a.scal + kScalStatus), kStatusOverflow);
    cnt = 0;
  }
  for (uint32_t e = lane; e < cnt; e += 32) a.bump[off + e] = make_uint2(tileR[e], sc[e]);
  if (lane == 0) {
    a.unit_off[u] = off;
    a.unit_cnt[u] = cnt;
    acc.ctr[kCSurv] += cnt;
    acc.ctr[kCAlg] += cnt * 8ull;
  }
  __syncwarp();
}


// Word-AND unit (round 1, both lists decoded into bitvectors this batch):
// words [w0, w1) of R's docID range.  Pass 1 counts the unit's survivors
// (popc of the ANDed words) for its output allocation; pass 2 walks 32 words
// per step (one per lane): each set bit of R.bits & S.bits is a survivor, its
// positions in R and S are the words' ranks + popc of the bits below it.  The
// survivors are buffered in shared memory (docID, R position, S position; at
// most C = cap of them, in docID order) and scored with every lane busy — w_R
// + w_S, SURVEY O6 — when the buffer fills; a 32-word step with more than C
// survivors is scored straight from the lanes.
__device__ __forceinline__ uint64_t make_key(uint2 e, uint32_t doc_base);
__device__ __forceinline__ void bitand_unit(const DevIndex &ix, const RoundArgs &a, uint32_t u,
                                            uint32_t q, uint32_t lu, uint32_t t0, uint32_t tSid,
                                            const TermInfo &tR, const TermInfo &tS,
                                            uint32_t *sdoc, uint32_t *srp, uint32_t *ssp,
                                            uint32_t cap, Acc &acc) {
  const uint32_t lane = lane_id(), lt = lanemask_lt();
  const uint2 *bR = a.bm + (size_t)a.bm_slot[t0] * a.bm_words;
  const uint2 *bS = a.bm + (size_t)a.bm_slot[tSid] * a.bm_words;
  const uint32_t w0 = (__ldg(ix.first + tR.block0) >> 5) + lu * kAndWords;
  const uint32_t w1 = min(w0 + kAndWords, a.bm_words);
  // a 2-term query's keys below its subset threshold cannot reach its top-k
  // (bitand_tau_kernel): they are scored but not written
  const uint64_t tau = a.qtau ? a.qtau[q] : 0ull;
  uint32_t c = 0;
  for (uint32_t w = w0 + lane; w < w1; w += 32u) c += __popc(__ldg(&bR[w].x) & __ldg(&bS[w].x));
  uint32_t cnt = __reduce_add_sync(0xffffffffu, c);
  unsigned long long off = 0;
  if (lane == 0 && cnt) off = bump_alloc(a, acc, cnt);
  off = __shfl_sync(0xffffffffu, off, 0);
  if (off + cnt > a.bump_cap) {
    if (lane == 0) atomicOr(reinterpret_cast<int *>(a.scal + kScalStatus), kStatusOverflow);
    cnt = 0;
  }
  uint32_t kept = 0;   // survivors written (all of them when tau = 0)
  uint32_t gsmall = 1;   // largest power of two <= min(8, cap / 32) (cap >= 32 in every layout)
  while (gsmall < 8u && 64u * gsmall <= cap) gsmall <<= 1;
  if (cnt) {
    uint32_t fb = 0;       // buffered survivors
    auto flush = [&]() {
      __syncwarp();
      for (uint32_t j0 = 0; j0 < fb; j0 += 32u) {
        const uint32_t j = j0 + lane;
        uint2 e = make_uint2(0, 0);
        bool keep = false;
        if (j < fb) {
          const uint32_t doc = sdoc[j];
          const float nrm = __ldg(ix.norm + doc);
          const float wS = bm25_w(tS.idf, tf_lookup(ix, tS, ssp[j]), nrm, ix.k1p1);
          const float wR = bm25_w(tR.idf, tf_lookup(ix, tR, srp[j]), nrm, ix.k1p1);   // first term: s = w
          e = make_uint2(doc, __float_as_uint(__fadd_rn(wR, wS)));
          keep = make_key(e, ix.doc_base) >= tau;
        }
        const uint32_t bal = __ballot_sync(0xffffffffu, keep);
        if (keep) a.bump[off + kept + __popc(bal & lt)] = e;
        kept += __popc(bal);
      }
      fb = 0;
      __syncwarp();
    };
    for (uint32_t wb = w0; wb < w1; wb += 32u) {
      const uint32_t w = wb + lane;
      const uint2 ra = w < w1 ? __ldg(bR + w) : make_uint2(0, 0);
      const uint2 sa = w < w1 ? __ldg(bS + w) : make_uint2(0, 0);
      const uint32_t mm = ra.x & sa.x;
      const uint32_t k = __popc(mm);
      const uint32_t incl = warp_incl_scan(k), excl = incl - k;
      const uint32_t T = __shfl_sync(0xffffffffu, incl, 31);
      if (T == 0) continue;
      // buffered in groups of lanes that fit the buffer: the whole warp, or
      // gsmall lanes (<= 32 docs each, <= cap in all) when one step holds
      // more survivors than `cap`
      const uint32_t gl = T <= cap ? 32u : gsmall;
      for (uint32_t g = 0; g < 32u; g += gl) {
        const uint32_t gb = __shfl_sync(0xffffffffu, excl, g);
        const uint32_t gT = __shfl_sync(0xffffffffu, incl, g + gl - 1u) - gb;
        if (gT == 0) continue;
        if (fb + gT > cap) flush();
        if (lane >= g && lane < g + gl) {
          uint32_t m = mm, o = fb + excl - gb;
          while (m) {
            const uint32_t bit = __ffs(m) - 1u;
            m &= m - 1u;
            const uint32_t below = (1u << bit) - 1u;
            sdoc[o] = (w << 5) | bit;
            srp[o] = ~ra.y + __popc(ra.x & below);
            ssp[o] = ~sa.y + __popc(sa.x & below);
            ++o;
          }
        }
        fb += gT;
      }
    }
    flush();
  }
  __syncwarp();
  if (lane == 0) {
    const uint32_t nw = w1 > w0 ? w1 - w0 : 0u;
    a.unit_off[u] = off;
    a.unit_cnt[u] = kept;
    acc.ctr[kCSurv] += kept;
    // 16 B per word pair; per scored survivor two tf sectors + the norm, per kept one the entry
    acc.ctr[kCAlg] += (unsigned long long)cnt * (2u * kTfSector + 4u) + 8ull * kept + 16ull * nw;
    if (a.count) {
      atomicAdd(a.scal + kScalDiag2 + 2, 1ull);
      atomicAdd(a.scal + kScalDiag2 + 3, (unsigned long long)nw);
    }
  }
}


// Round-1 unit kinds run as two kernels, back to back (ROLE): 1 = the merge
// units (the processing order puts them first: tickets [0, #merge)), 2 = the
// gallop, bitvector, word-AND and single-term units (tickets [#merge, total))
// with a smaller shared layout (no merge tiles).  It ran at 4 CTAs/SM (64
// registers) while it held only gallop units; with the bitvector kinds it
// spilled there, and 3 CTAs/SM without spills is faster (C5 intersect 7.58 ->
// 7.27 ms).  ROLE 0 = every unit kind in one kernel (the SvS rounds without
// the probe pass).
#ifndef GRIFFIN_IK2_MINB
#define GRIFFIN_IK2_MINB 3
#endif
#ifndef GRIFFIN_INTERSECT_MINB
#define GRIFFIN_INTERSECT_MINB 3
#endif
__host__ __device__ inline uint32_t other_tile_words(uint32_t B, uint32_t D, bool nextgeq) {
  const uint32_t G = (D - 1u) < 31u ? D - 1u : 31u;
  return 3u * B + (nextgeq ? 0u : G * B) + kTileSlack;
}
__host__ __device__ inline uint32_t other_warp_smem_words(uint32_t B, uint32_t D, bool nextgeq) {
  return kWarpHdr + 64 + (B + 32) + other_stage_words(B, D) + kStgSlack + other_tile_words(B, D, nextgeq);
}
template <int ROLE>
struct IkMinBlocks { static constexpr int v = ROLE == 2 ? GRIFFIN_IK2_MINB : GRIFFIN_INTERSECT_MINB; };

template <bool RC, int ROLE>
__global__ void __launch_bounds__(kIntersectThreads, IkMinBlocks<ROLE>::v) intersect_kernel(DevIndex ix, RoundArgs a) {
  extern __shared__ uint4 smem4[];
  const uint32_t lane = lane_id();
  const uint32_t B = ix.B, D = a.D;
  WarpSmem sm;
  if (ROLE == 2) {
    uint8_t *base = reinterpret_cast<uint8_t *>(smem4);
    sm.lut = base;
    uint32_t *wb = reinterpret_cast<uint32_t *>(base + kLutBytes) +
                   (threadIdx.x >> 5) * other_warp_smem_words(B, D, a.nextgeq != 0);
    sm.mbar = reinterpret_cast<uint64_t *>(wb);
    sm.cnt = wb + kWarpHdr;
    sm.aux = sm.cnt + 64;
    sm.stg = sm.aux + B + 32;
    sm.tile = sm.stg + other_stage_words(B, D) + kStgSlack;
    sm.phase = 0;
  } else {
    sm = carve_warp_smem(smem4, B, D);
  }
  cta_smem_init(smem4, sm);
  const uint64_t nmerge = a.scal[kScalPerm];   // merge units: tickets [0, nmerge)
  const uint64_t total = ROLE == 1 ? nmerge : a.unit_base[a.nq];
  const uint32_t G = min(D - 1u, 31u);   // gallop: S blocks staged per group
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  Acc acc;
  acc.bleft = reinterpret_cast<uint32_t *>(sm.mbar) + 2;
  acc.boff = reinterpret_cast<unsigned long long *>(sm.mbar) + 2;
  acc.ctr = reinterpret_cast<unsigned long long *>(sm.mbar) + 4;
  if (lane == 0) {
    *acc.bleft = 0;
    *acc.boff = 0;
#pragma unroll
    for (int c = 0; c < kCNum; ++c) acc.ctr[c] = 0;
  }
  // dynamic unit tickets (balances long gallop/probe units); the next ticket is
  // requested at the start of a unit so its latency overlaps the unit's work
  unsigned long long ticket = 0;
  unsigned long long *ctr = a.scal + (ROLE == 2 ? kScalUnitCtr2 : kScalUnitCtr);
  const uint64_t tk0 = ROLE == 2 ? nmerge : 0ull;
  if (lane == 0) ticket = tk0 + atomicAdd(ctr, 1ull);
  (void)nwarps;
  for (;;) {
    const uint64_t tk = __shfl_sync(0xffffffffu, ticket, 0);
    if (tk >= total) break;
    if (lane == 0) ticket = tk0 + atomicAdd(ctr, 1ull);
    const uint4 pe = a.uperm[tk];   // merge units first (see partition_kernel)
    const uint64_t u = pe.x;
    const uint32_t q = pe.y & 0x1FFFFFFFu, mode = pe.y >> 29, t0 = pe.z, tSid = pe.w;
    const uint4 rec = a.urec[u];
    const uint4 nxt = a.urec[u + 1];
    const uint32_t lu = rec.y;   // gallop/all: unit index within the query
    const TermInfo tR = ix.terms[t0];
    const uint2 *Rq = RC ? nullptr : a.rprev + a.roff_prev[q];
    const uint32_t nR = RC ? tR.df_local : a.rcount[q];
    const uint32_t nbR = RC ? tR.nblocks : (nR + B - 1) / B;
    // R source: compressed EF, the batch's decoded arena, or the intermediate
    const bool rdec = RC && a.tdec && a.tdec[t0] == kDecArena;
    const uint32_t *decR = rdec ? a.dec + (size_t)tR.block0 * B : nullptr;

    if (ROLE != 1 && RC && mode == kModeAll) {  // single-term query: the whole list is the result
      const uint32_t n = min(B, nR - lu * B);
      if (rdec) {
        if (lane == 0) {
          fence_proxy_async();
          mbar_expect_tx(sm.mbar, ((n + 3u) & ~3u) * 4u);
          bulk_g2s(sm.tile, decR + (size_t)lu * B, ((n + 3u) & ~3u) * 4u, sm.mbar);
        }
        mbar_wait(sm.mbar, sm.phase);
        sm.phase ^= 1u;
        if (lane == 0) {
          acc.ctr[kCAlg] += n * 4u;
          acc.ctr[kCApost] += n;
          acc.ctr[kCAcomp] += block_size16(ix.meta[(uint64_t)tR.block0 + lu].y) * 16u + 8u;
        }
      } else {
        const uint64_t gb = (uint64_t)tR.block0 + lu;
        const uint2 m = ix.meta[gb];
        const uint32_t f = ix.first[gb];
        const uint32_t sz = block_size16(m.y);
        stage_blocks(ix, sm, 1, m, 0, sz, true);
        warp_decode_staged(sm.stg, f, m.y, sm.tile, sm.cnt, sm.lut);
        if (lane == 0) {
          acc.ctr[kCPay] += sz * 16u;
          acc.ctr[kCPost] += n;
          acc.ctr[kCAlg] += sz * 16u + 8u;
        }
      }
      emit_unit<2>(ix, a, (uint32_t)u, tR, tR, nullptr, sm.tile, nullptr, nullptr, n, lu * B, acc);
      continue;
    }
    if (ROLE == 0 && !RC && mode == kModeProbe) {
      probe_unit(ix, a, sm, u, q, lu, acc);
      continue;
    }
    const TermInfo tS = ix.terms[tSid];
    const uint32_t *fS = ix.first + tS.block0;
    const uint32_t nbS = tS.nblocks;
    const bool sdec = a.tdec && a.tdec[tSid] == kDecArena;
    const uint32_t *decS = sdec ? a.dec + (size_t)tS.block0 * B : nullptr;

    if (ROLE != 2 && (ROLE == 1 || mode == kModeMerge)) {
      // ---- the unit's docID range [lo, hi) and block ranges, from the partition
      // stage's merge-path crossings (unit u and unit u+1) ----
      const uint32_t i0 = rec.y, j0 = rec.z;
      const bool last = nxt.x != q;
      const uint32_t i1 = last ? nbR : nxt.y, j1 = last ? nbS : nxt.z;
      const uint64_t lo_v = rec.w, hi_v = last ? (1ull << 32) : (uint64_t)nxt.w;
      const uint32_t rb0 = i0 ? i0 - 1 : 0, rb1 = i1;
      const uint32_t sb0 = j0 ? j0 - 1 : 0, sb1 = j1;
      const uint32_t nRb = rb1 > rb0 ? rb1 - rb0 : 0, nSb = sb1 > sb0 ? sb1 - sb0 : 0;
      if (nRb == 0 || nSb == 0 || lo_v >= hi_v) {
        if (lane == 0) {
          a.unit_off[u] = 0;
          a.unit_cnt[u] = 0;
        }
        continue;
      }
      const uint32_t nRt = min(rb1 * B, nR) - rb0 * B;
      const uint32_t nSt = min(sb1 * B, tS.df_local) - sb0 * B;
      uint32_t *tileS = sm.tile + nRb * B;
      // ---- metas of the compressed lists: lanes [0,nRb) R, [nRb, nRb+nSb) S ----
      const bool rcomp = RC && !rdec;
      const bool isR = lane < nRb, isS = lane >= nRb && lane < nRb + nSb;
      const bool lm = (rcomp && isR) || (!sdec && isS);
      uint2 m = make_uint2(0, 0);
      uint32_t f = 0;
      if (lm) {
        const uint64_t gb = isR ? (uint64_t)tR.block0 + rb0 + lane
                                : (uint64_t)tS.block0 + sb0 + (lane - nRb);
        m = ix.meta[gb];
        f = ix.first[gb];
      }
      const uint32_t sz = lm ? block_size16(m.y) : 0u;
      const uint32_t mR0 = __shfl_sync(0xffffffffu, m.x, 0);
      const uint32_t mS0 = __shfl_sync(0xffffffffu, m.x, nRb);
      const uint32_t totR16 = __reduce_add_sync(0xffffffffu, (lm && isR) ? sz : 0u);
      const uint32_t totS16 = __reduce_add_sync(0xffffffffu, (lm && isS) ? sz : 0u);
      const uint32_t soff = isR ? m.x - mR0 : (isS ? totR16 + (m.x - mS0) : 0u);
      // ---- accounting: blocks whose head lies in this unit (profiling) ----
      if (a.count) {
        const bool own = (isR && rb0 + lane >= i0) || (isS && sb0 + (lane - nRb) >= j0);
        const uint32_t nn = isR ? min(B, nR - (rb0 + lane) * B)
                                : (isS ? min(B, tS.df_local - (sb0 + lane - nRb) * B) : 0u);
        uint32_t pay = 0, post = 0, alg = 0, ap = 0, ac = 0;
        if (own) {
          if (lm) {
            pay = sz * 16u;
            post = nn;
            alg = pay + 8u;
          } else {
            alg = nn * (isR && !RC ? 8u : 4u);  // intermediate (docID+score) or decoded arena
            if (!(isR && !RC)) {   // arena block: its compressed size for the §8(d) count
              ap = nn;
              const uint64_t gb = isR ? (uint64_t)tR.block0 + rb0 + lane
                                      : (uint64_t)tS.block0 + sb0 + (lane - nRb);
              ac = block_size16(ix.meta[gb].y) * 16u + 8u;
            }
          }
        }
        const uint32_t sp = __reduce_add_sync(0xffffffffu, pay);
        const uint32_t sn = __reduce_add_sync(0xffffffffu, post);
        const uint32_t sa = __reduce_add_sync(0xffffffffu, alg);
        const uint32_t sap = __reduce_add_sync(0xffffffffu, ap);
        const uint32_t sac = __reduce_add_sync(0xffffffffu, ac);
        if (lane == 0) {
          acc.ctr[kCPay] += sp;
          acc.ctr[kCPost] += sn;
          acc.ctr[kCAlg] += sa;
          acc.ctr[kCApost] += sap;
          acc.ctr[kCAcomp] += sac;
        }
      }
      // ---- TMA: decoded-arena ranges -> tiles; compressed payloads -> stg (one
      // round trip when they fit the staging area, else capacity-sized batches) ----
      const uint32_t cap16 = stage_words(B, D) / 4u;
      const bool fit = totR16 + totS16 <= cap16;
      {
        const uint32_t bRd = rdec ? ((nRt + 3u) & ~3u) * 4u : 0u;
        const uint32_t bSd = sdec ? ((nSt + 3u) & ~3u) * 4u : 0u;
        const uint32_t bRc = (rcomp && fit) ? totR16 * 16u : 0u;
        const uint32_t bSc = (!sdec && fit) ? totS16 * 16u : 0u;
        const uint32_t tx = bRd + bSd + bRc + bSc;
        if (lane == 0 && tx) {
          fence_proxy_async();
          mbar_expect_tx(sm.mbar, tx);
          if (bRd) bulk_g2s(sm.tile, decR + (size_t)rb0 * B, bRd, sm.mbar);
          if (bSd) bulk_g2s(tileS, decS + (size_t)sb0 * B, bSd, sm.mbar);
          if (bRc) bulk_g2s(sm.stg, ix.payload + mR0, bRc, sm.mbar);
          if (bSc) bulk_g2s(sm.stg + totR16 * 4u, ix.payload + mS0, bSc, sm.mbar);
        }
        if (!RC) {  // intermediate R: docIDs out of the (docID, score) entries
          const uint32_t s0 = rb0 * B;
          for (uint32_t i = lane; i < nRt; i += 32) sm.tile[i] = Rq[s0 + i].x;
        }
        if (tx) {
          mbar_wait(sm.mbar, sm.phase);
          sm.phase ^= 1u;
        }
      }
      // ---- EF-decode the compressed blocks into the smem tiles ----
      // (one call site per decoder path: every inlined copy of the decoders
      // costs ~5 KB of SASS, and the kernel is instruction-cache bound)
      if (fit) {
        // R and S tiles are contiguous: one pass over every compressed block
        const uint32_t l0 = rcomp ? 0u : nRb;
        const uint32_t nbd = (rcomp ? nRb : 0u) + (sdec ? 0u : nSb);
        if (nbd) decode_staged_lanes<kIkPair>(sm, B, l0, nbd, m.y, f, soff, rcomp ? sm.tile : tileS);
      } else {
#pragma unroll 1
        for (uint32_t jb = 0; jb < 2; ++jb) {
          if (jb == 0 ? rcomp : !sdec)
            stage_decode_lanes<kIkPair>(ix, sm, cap16, jb ? nRb : 0u, jb ? nSb : nRb, m, f, sz,
                               jb ? tileS : sm.tile);
        }
      }
      __syncwarp();
      // sentinel after the S tile's valid elements: the uniform-trip merge loop
      // below may step B past them (a lane whose A elements outlast B), and
      // stale shared memory there (e.g. another unit's R tile) could equal an
      // in-segment A element and count as a false match
      if (lane == 0) tileS[nSt] = kNone;
      __syncwarp();
      // ranges inside [lo, hi): four lower_bounds — (R, lo), (R, hi), (S, lo),
      // (S, hi) — each by an 8-lane group doing an 8-ary search (7 probes per
      // step, ballot + popc), ~log8 dependent smem loads instead of log2
      uint32_t r_lo;
      {
        const uint32_t g = lane >> 3, sub = lane & 7u;
        const uint32_t *arr = g < 2 ? sm.tile : tileS;
        const uint64_t key = (g & 1) ? hi_v : lo_v;
        const uint32_t gmask = 0xFFu << (g * 8u);
        uint32_t lo = 0, hi = g < 2 ? nRt : nSt;   // answer in [lo, hi]
        while (__any_sync(0xffffffffu, lo < hi)) {
          const uint32_t step = (hi - lo + 8u) >> 3;   // 8 steps cover the hi-lo+1 candidates
          const uint32_t qp = lo + (sub + 1u) * step - 1u;
          const bool pr = lo < hi && sub < 7u && qp < hi && (uint64_t)arr[qp] < key;
          const uint32_t c = __popc(__ballot_sync(0xffffffffu, pr) & gmask);
          if (lo < hi) {
            const uint32_t nlo = lo + c * step;
            hi = min(hi, lo + (c + 1u) * step - 1u);
            lo = nlo;
          }
        }
        r_lo = lo;
      }
      const uint32_t ra = __shfl_sync(0xffffffffu, r_lo, 0), rb = __shfl_sync(0xffffffffu, r_lo, 8);
      const uint32_t sa = __shfl_sync(0xffffffffu, r_lo, 16), sb = __shfl_sync(0xffffffffu, r_lo, 24);
      const uint32_t nr = rb - ra, ns = sb - sa;
      const uint32_t tot2 = nr + ns, L = (tot2 + 31) >> 5;
      if (a.count && lane == 0) {   // unit-shape diagnostics (counting pass only)
        atomicAdd(a.scal + kScalDiag, 1ull);
        atomicAdd(a.scal + kScalDiag + 1, (unsigned long long)tot2);
      }
      const uint32_t cap = (L >> 1) + 2;           // matches per lane <= ceil(L/2), +1 slack write
      uint32_t *ml = sm.stg + lane * cap;          // staging is free after decode
      uint32_t c = 0;
      if (nr && ns) {
        // ---- fine merge path: lane l owns diagonals [l*L, (l+1)*L); its end is
        // the next lane's start, matched pairs never split (A9) ----
        const uint32_t *A = sm.tile + ra, *Bv = tileS + sa;
        auto gA = [&](uint32_t i) -> uint32_t { return A[i]; };
        auto gB = [&](uint32_t j) -> uint32_t { return Bv[j]; };
        const uint32_t ds = min(lane * L, tot2);
        uint32_t is, js;
        merge_path_split(gA, nr, gB, ns, ds, true, &is, &js);
        uint32_t ie = __shfl_down_sync(0xffffffffu, is, 1);
        uint32_t je = __shfl_down_sync(0xffffffffu, js, 1);
        if (lane == 31) {
          ie = nr;
          je = ns;
        }
        // branch-free serial merge with a warp-uniform trip count: every lane
        // runs exactly L steps (its segment holds <= L merged elements and each
        // step consumes >= 1, so the segment is covered).  Steps past the
        // segment's end read the next lane's (still sorted) elements; a match
        // counts only while the A index is inside the segment (pa < paE), and no
        // in-segment element can equal an out-of-segment one (merge-path order +
        // the A9 fix-up).  Every step writes the candidate pair and keeps it only
        // on a match, so the loop has no divergent branch at all.
        // match key = low 16 bits of both smem addresses (one PRMT per step
        // instead of maintaining a packed index pair; the tiles span < 64 KB,
        // emit_lanes turns the halves back into tile indices)
        uint32_t pa = smem_u32(A + is), pb = smem_u32(Bv + js);
        const uint32_t paE = smem_u32(A + ie);
        const uint32_t pm0 = smem_u32(ml);
        uint32_t pm = pm0;
#pragma unroll kMergeUnroll
        for (uint32_t t = 0; t < L; ++t) {
          uint32_t x, y;
          asm volatile("ld.shared.u32 %0, [%1];" : "=r"(x) : "r"(pa));
          asm volatile("ld.shared.u32 %0, [%1];" : "=r"(y) : "r"(pb));
          asm volatile("st.shared.u32 [%0], %1;" ::"r"(pm), "r"(__byte_perm(pa, pb, 0x5410)));
          pm += (x == y && pa < paE) ? 4u : 0u;
          pa += (x <= y) ? 4u : 0u;
          pb += (y <= x) ? 4u : 0u;
        }
        c = (pm - pm0) >> 2;
      }
      __syncwarp();
      if (RC)
        emit_lanes<true>(ix, a, (uint32_t)u, tR, tS, Rq, sm.tile, sm.stg, cap, c, sm.cnt, rb0 * B,
                         sb0 * B + sa, smem_u32(sm.tile) & 0xFFFFu,
                         smem_u32(tileS + sa) & 0xFFFFu, acc);
      else
        emit_lanes<false>(ix, a, (uint32_t)u, tR, tS, Rq, sm.tile, sm.stg, cap, c, sm.cnt, rb0 * B,
                          sb0 * B + sa, smem_u32(sm.tile) & 0xFFFFu,
                          smem_u32(tileS + sa) & 0xFFFFu, acc);
      __syncwarp();
    } else if (ROLE != 1 && mode == kModeBitAnd) {
      // survivor buffer: docIDs in the tile, R / S positions in the staging area
      uint32_t tw, sw;
      bm_layout(B, D, a.nextgeq != 0, ROLE == 2, &tw, &sw);
      const uint32_t cap = min(tw, sw / 2u);
      bitand_unit(ix, a, (uint32_t)u, q, lu, t0, tSid, tR, tS, sm.tile, sm.stg, sm.stg + cap, cap, acc);
    } else if (ROLE != 1 && mode == kModeBitmap) {
      // ---- S decoded into a bitvector this batch: R blocks [b0, b0+nb) (or
      // intermediate chunks) looked up in O(1), hits compacted, then scored ----
      const uint32_t U = bm_unit_blocks(B, D, a.nextgeq != 0);
      const uint32_t b0 = lu * U, nb = min(U, nbR - b0), s0 = b0 * B;
      const uint32_t n = min(U * B, nR - s0);
      uint32_t *tileR = sm.tile, *idx = sm.stg;   // idx: the staging area, free after decode
      uint32_t *spos = bm_spos_in_tile(B, D, a.nextgeq != 0, ROLE == 2, U) ? sm.tile + U * B
                                                                             : sm.stg + U * B;
      if (RC && rdec) {
        const uint32_t by = ((n + 3u) & ~3u) * 4u;
        if (lane == 0) {
          fence_proxy_async();
          mbar_expect_tx(sm.mbar, by);
          bulk_g2s(tileR, decR + s0, by, sm.mbar);
        }
        mbar_wait(sm.mbar, sm.phase);
        sm.phase ^= 1u;
        if (a.count) {
          const uint32_t c = lane < nb ? block_size16(ix.meta[(uint64_t)tR.block0 + b0 + lane].y) * 16u + 8u : 0u;
          const uint32_t sc = __reduce_add_sync(0xffffffffu, c);
          if (lane == 0) {
            acc.ctr[kCAlg] += n * 4u;
            acc.ctr[kCApost] += n;
            acc.ctr[kCAcomp] += sc;
          }
        }
      } else if (RC) {
        uint2 m = make_uint2(0, 0);
        uint32_t f = 0, sz = 0;
        if (lane < nb) {
          const uint64_t gb = (uint64_t)tR.block0 + b0 + lane;
          m = ix.meta[gb];
          f = ix.first[gb];
          sz = block_size16(m.y);
        }
        stage_decode_lanes<kIkPair>(ix, sm, stage_words(B, D) / 4u, 0, nb, m, f, sz, tileR);
        if (a.count) {
          const uint32_t sp = __reduce_add_sync(0xffffffffu, sz) * 16u;
          if (lane == 0) {
            acc.ctr[kCPay] += sp;
            acc.ctr[kCPost] += n;
            acc.ctr[kCAlg] += sp + 8u * nb;
          }
        }
      } else {
        for (uint32_t i = lane; i < n; i += 32) tileR[i] = Rq[s0 + i].x;
        if (a.count && lane == 0) acc.ctr[kCAlg] += n * 8u;
      }
      __syncwarp();
      if (a.count && lane == 0) {
        atomicAdd(a.scal + kScalDiag2, 1ull);
        atomicAdd(a.scal + kScalDiag2 + 1, (unsigned long long)n);
      }
      // round 1: R's tf words for positions [s0, s0+n) staged (coalesced) in
      // the aux area when they fit — survivors read R's tf there
      const uint32_t *rtf = nullptr;
      uint64_t rtf_bit0 = 0;
      if (RC && tR.tf_w) {
        const uint64_t b0w = ((uint64_t)s0 * tR.tf_w) >> 5;
        const uint64_t b1w = ((uint64_t)(s0 + n) * tR.tf_w + 31u) >> 5;
        const uint32_t nw = (uint32_t)(b1w - b0w) + 1u;   // + the funnel's look-ahead word
        if (nw <= B + 32u) {
          for (uint32_t i = lane; i < nw; i += 32u) sm.aux[i] = __ldg(ix.tfw + tR.tf_off + b0w + i);
          rtf = sm.aux;
          rtf_bit0 = b0w * 32u;
        }
      }
      const uint32_t cnt = bitvec_probe_compact(a.bm + (size_t)a.bm_slot[tSid] * a.bm_words, tileR,
                                                n, idx, spos, a.count, acc);
      if (RC)
        emit_compact<0>(ix, a, (uint32_t)u, tR, tS, Rq, tileR, idx, spos, cnt, s0, acc, rtf,
                        rtf_bit0);
      else
        emit_compact<1>(ix, a, (uint32_t)u, tR, tS, Rq, tileR, idx, spos, cnt, s0, acc);
      __syncwarp();
    } else if (ROLE != 1) {
      // ---- gallop: R chunk lu, skip-pointer search into S (Fig. 9) ----
      uint32_t *tileR = sm.tile, *kidx = sm.tile + B, *match = sm.tile + 2 * B;
      uint32_t *tileS = sm.tile + 3 * B;
      uint32_t *dblk = sm.aux, *sn = sm.aux + B;
      const uint32_t n = min(B, nR - lu * B);
      if (RC && rdec) {
        const uint32_t by = ((n + 3u) & ~3u) * 4u;
        if (lane == 0) {
          fence_proxy_async();
          mbar_expect_tx(sm.mbar, by);
          bulk_g2s(tileR, decR + (size_t)lu * B, by, sm.mbar);
        }
        mbar_wait(sm.mbar, sm.phase);
        sm.phase ^= 1u;
        if (lane == 0) {
          acc.ctr[kCAlg] += n * 4u;
          acc.ctr[kCApost] += n;
          acc.ctr[kCAcomp] += block_size16(ix.meta[(uint64_t)tR.block0 + lu].y) * 16u + 8u;
        }
      } else if (RC) {
        const uint64_t gb = (uint64_t)tR.block0 + lu;
        const uint2 m = ix.meta[gb];
        const uint32_t f = ix.first[gb];
        const uint32_t sz = block_size16(m.y);
        stage_blocks(ix, sm, 1, m, 0, sz, true);
        warp_decode_staged(sm.stg, f, m.y, tileR, sm.cnt, sm.lut);
        if (lane == 0) {
          acc.ctr[kCPay] += sz * 16u;
          acc.ctr[kCPost] += n;
          acc.ctr[kCAlg] += sz * 16u + 8u;
        }
      } else {
        load_r_chunk(Rq, nR, B, lu, tileR);
        if (lane == 0) acc.ctr[kCAlg] += n * 8u;
      }
      __syncwarp();
      const uint32_t k_lo = rec.z, k_hi = rec.w;   // from the partition stage
      if (a.count && lane == 0) {
        atomicAdd(a.scal + kScalDiag + 2, 1ull);
        atomicAdd(a.scal + kScalDiag + 3, (unsigned long long)n);
      }
      // skip pointers the chunk can touch: [k_lo-1, k_hi); stage them in smem when
      // they fit (one round trip), else search them in global memory
      const uint32_t w0 = k_lo ? k_lo - 1u : 0u, span = k_hi - w0;
      if (span <= stage_words(B, D)) {
        uint32_t *win = sm.stg;
        for (uint32_t i = lane; i < span; i += 32) win[i] = __ldg(fS + w0 + i);
        __syncwarp();
        for (uint32_t e = lane; e < n; e += 32) {
          // upper_bound in the window, shifted back to block indices
          uint32_t lo2 = 0, hi2 = span;
          const uint32_t x = tileR[e];
          while (lo2 < hi2) {
            const uint32_t mid = (lo2 + hi2) >> 1;
            if (win[mid] <= x) lo2 = mid + 1; else hi2 = mid;
          }
          kidx[e] = w0 + lo2 - 1u;   // kNone: below S's first docID
          match[e] = kNone;
        }
      } else {
        // wide range: sampled skip pointers in smem, then short global searches
        skip_blocks_sampled(fS, k_lo ? k_lo - 1u : 0u, k_hi, tileR, n, kidx, match, sm.stg,
                            stage_words(B, D));
      }
      __syncwarp();
      if (sdec) {
        // S decoded in the arena: interpolation probes of the touched block in
        // place (no staging), kArenaEpl independent probes per lane in flight
        uint32_t probes = 0;
        for (uint32_t base = 0; base < n; base += 32u * kArenaEpl)
          probes += arena_probe_slice(decS, fS, tS.nblocks, tS.df_local, B, tileR, kidx, match,
                                      base, n);
        const uint32_t sp = __reduce_add_sync(0xffffffffu, probes);
        if (lane == 0) acc.ctr[kCAlg] += sp * 32ull;
        __syncwarp();
        if (RC)
          emit_unit<0>(ix, a, (uint32_t)u, tR, tS, Rq, tileR, match, kidx, n, lu * B, acc);
        else
          emit_unit<1>(ix, a, (uint32_t)u, tR, tS, Rq, tileR, match, kidx, n, lu * B, acc);
        __syncwarp();
        continue;
      }
      const uint32_t k_first = kidx[0];
      // distinct touched blocks (kidx is non-decreasing): dblk[], and kidx[e] :=
      // index of e's block in dblk (kNone if none)
      uint32_t nd = 0, prev = kNone, e_first = n;
      for (uint32_t c0 = 0; c0 < n; c0 += 32) {
        const uint32_t e = c0 + lane;
        const uint32_t kv = e < n ? kidx[e] : kNone;
        uint32_t kp = __shfl_up_sync(0xffffffffu, kv, 1);
        if (lane == 0) kp = prev;
        const bool newb = e < n && kv != kNone && kv != kp;
        const uint32_t bal = __ballot_sync(0xffffffffu, newb);
        const uint32_t rank = __popc(bal & lanemask_lt());
        if (newb) dblk[nd + rank] = kv;
        const uint32_t gi = nd + __popc(bal & (lanemask_lt() | (1u << lane))) - 1u;
        if (e < n) kidx[e] = kv == kNone ? kNone : gi;
        const uint32_t valid = __ballot_sync(0xffffffffu, e < n && kv != kNone);
        if (e_first == n && valid) e_first = c0 + __ffs(valid) - 1u;
        nd += __popc(bal);
        prev = __shfl_sync(0xffffffffu, kv, 31);
      }
      __syncwarp();
      uint32_t ep = e_first;
      const uint32_t cap16 = stage_words(B, D) / 4u;
      for (uint32_t g0 = 0; g0 < nd;) {
        uint32_t ng = min(G, nd - g0);
        uint2 m = make_uint2(0, 0);
        uint32_t f = 0, sz = 0, blk = 0, nn = 0;
        if (lane < ng) {
          blk = dblk[g0 + lane];
          nn = min(B, tS.df_local - blk * B);
          if (!sdec) {
            m = ix.meta[(uint64_t)tS.block0 + blk];
            f = ix.first[(uint64_t)tS.block0 + blk];
            sz = block_size16(m.y);
          }
        }
        if (!sdec) {  // as many touched blocks as the staging area holds
          const uint32_t inc = warp_incl_scan(sz);
          const uint32_t nfit = __popc(__ballot_sync(0xffffffffu, lane < ng && inc <= cap16));
          ng = nfit ? nfit : 1u;
          if (lane >= ng) sz = 0;
        }
        if (lane < ng) sn[lane] = nn;
        __syncwarp();
        {
          const bool own = lane < ng && !(lu > 0 && blk == k_first);
          const uint32_t sp = __reduce_add_sync(0xffffffffu, (own && !sdec) ? sz * 16u : 0u);
          const uint32_t spn =
              __reduce_add_sync(0xffffffffu, (own && !sdec && !a.nextgeq) ? nn : 0u);
          const uint32_t sa = __reduce_add_sync(
              0xffffffffu, own ? (sdec ? nn * 4u : sz * 16u + 8u) : 0u);
          if (lane == 0) {
            acc.ctr[kCPay] += sp;
            acc.ctr[kCPost] += spn;
            acc.ctr[kCAlg] += sa;
          }
        }
        uint32_t soff = 0;
        if (sdec) {
          // decoded arena: each touched block straight into its tileS slot
          const uint32_t by = lane < ng ? ((nn + 3u) & ~3u) * 4u : 0u;
          const uint32_t tot = __reduce_add_sync(0xffffffffu, by);
          if (lane == 0) {
            fence_proxy_async();
            mbar_expect_tx(sm.mbar, tot);
          }
          __syncwarp();
          if (lane < ng) bulk_g2s(tileS + lane * B, decS + (size_t)blk * B, by, sm.mbar);
          mbar_wait(sm.mbar, sm.phase);
          sm.phase ^= 1u;
        } else {
          soff = warp_incl_scan(sz) - sz;
          stage_blocks(ix, sm, ng, m, soff, sz, false);
          if (!a.nextgeq) {
            for (uint32_t i = 0; i < ng; ++i) {
              const uint32_t y = __shfl_sync(0xffffffffu, m.y, i);
              const uint32_t fi = __shfl_sync(0xffffffffu, f, i);
              const uint32_t so = __shfl_sync(0xffffffffu, soff, i);
              warp_decode_staged(sm.stg + so * 4u, fi, y, tileS + i * B, sm.cnt, sm.lut);
            }
          }
        }
        __syncwarp();
        // elements mapping to this group: contiguous from ep
        const bool ngeq = !sdec && a.nextgeq;
        for (;;) {
          const uint32_t e = ep + lane;
          const uint32_t gi = e < n ? kidx[e] : kNone;
          const bool in = gi != kNone && gi < g0 + ng;
          if (ngeq) {
            // NextGEQ on the staged payload: no block decode (NEXT-1)
            const uint32_t src = in ? gi - g0 : 0u;
            const uint32_t y = __shfl_sync(0xffffffffu, m.y, src);
            const uint32_t fi = __shfl_sync(0xffffffffu, f, src);
            const uint32_t so = __shfl_sync(0xffffffffu, soff, src);
            if (in) {
              const uint32_t x = tileR[e];
              uint32_t v;
              const uint32_t p = ef_next_geq_staged(sm.stg + so * 4u, fi, y, x, sm.lut, v);
              if (p < meta_n(y) && v == x) match[e] = dblk[gi] * B + p;
            }
          } else if (in) {
            const uint32_t x = tileR[e];
            const uint32_t *seg = tileS + (gi - g0) * B;
            const uint32_t p = lower_bound_s(seg, 0, sn[gi - g0], x);
            if (p < sn[gi - g0] && seg[p] == x) match[e] = dblk[gi] * B + p;
          }
          const uint32_t bal = __ballot_sync(0xffffffffu, in);
          ep += __popc(bal);
          if (bal != 0xffffffffu) break;
        }
        __syncwarp();
        g0 += ng;
      }
      if (RC)
        emit_unit<0>(ix, a, (uint32_t)u, tR, tS, Rq, tileR, match, kidx, n, lu * B, acc);
      else
        emit_unit<1>(ix, a, (uint32_t)u, tR, tS, Rq, tileR, match, kidx, n, lu * B, acc);
      __syncwarp();
    }
  }
  if (lane == 0) {
    const int slot[kCNum] = {kScalCounters, kScalCounters + 1, kScalCounters + 2,
                             kScalCounters + 3, kScalArena, kScalArena + 1};
#pragma unroll
    for (int c = 0; c < kCNum; ++c)
      if (acc.ctr[c]) atomicAdd(a.scal + slot[c], acc.ctr[c]);
  }
}

// SvS rounds 2..m-1 as one multi-list probe pass: its own kernel,
// so it carries only the probe unit's code and shared memory (no merge tiles)
// at GRIFFIN_PROBE_MINB CTAs of 8 warps per SM.  The pass is global-latency
// bound (skip-pointer searches, arena probes, bitvector lookups); 4 CTAs (64
// registers) hid more of it until the bitvector lookups and lazy norm gathers
// made 3 CTAs with 80 registers faster (C5 intersect 7.26 -> 7.11 ms).
#ifndef GRIFFIN_PROBE_MINB
#define GRIFFIN_PROBE_MINB 3
#endif
__global__ void __launch_bounds__(kIntersectThreads, GRIFFIN_PROBE_MINB) probe_kernel(DevIndex ix, RoundArgs a) {
  extern __shared__ uint4 smem4[];
  const uint32_t lane = lane_id();
  const uint32_t B = ix.B, D = a.D;
  uint8_t *base = reinterpret_cast<uint8_t *>(smem4);
  WarpSmem sm;
  sm.lut = base;
  uint32_t *wb = reinterpret_cast<uint32_t *>(base + kLutBytes) +
                 (threadIdx.x >> 5) * probe_warp_smem_words(B, D, a.nextgeq != 0);
  sm.mbar = reinterpret_cast<uint64_t *>(wb);
  sm.cnt = wb + kWarpHdr;
  sm.aux = sm.cnt + 64;
  sm.stg = sm.aux + B + 32;
  sm.tile = sm.stg + stage_words(B, D) + kStgSlack;
  sm.phase = 0;
  cta_smem_init(smem4, sm);
  const uint64_t total = a.unit_base[a.nq];
  Acc acc;
  acc.bleft = reinterpret_cast<uint32_t *>(sm.mbar) + 2;
  acc.boff = reinterpret_cast<unsigned long long *>(sm.mbar) + 2;
  acc.ctr = reinterpret_cast<unsigned long long *>(sm.mbar) + 4;
  if (lane == 0) {
    *acc.bleft = 0;
    *acc.boff = 0;
#pragma unroll
    for (int c = 0; c < kCNum; ++c) acc.ctr[c] = 0;
  }
  unsigned long long ticket = 0;
  if (lane == 0) ticket = atomicAdd(a.scal + kScalUnitCtr, 1ull);
  for (;;) {
    const uint64_t tk = __shfl_sync(0xffffffffu, ticket, 0);
    if (tk >= total) break;
    if (lane == 0) ticket = atomicAdd(a.scal + kScalUnitCtr, 1ull);
    const uint64_t u = a.uperm[tk].x;
    const uint4 rec = a.urec[u];
    probe_unit(ix, a, sm, u, rec.x, rec.y, acc);   // every unit of the pass is a probe unit
  }
  if (lane == 0) {
    const int slot[kCNum] = {kScalCounters, kScalCounters + 1, kScalCounters + 2,
                             kScalCounters + 3, kScalArena, kScalArena + 1};
#pragma unroll
    for (int c = 0; c < kCNum; ++c)
      if (acc.ctr[c]) atomicAdd(a.scal + slot[c], acc.ctr[c]);
  }
}

// ------------------------------------------------------------------- compaction

// Global exclusive scan of the per-unit survivor counts (n = total units, read
// on the device; CTAs past n exit).  Units of one query are contiguous, so a
// query's output offset of unit u is udst[u] - udst[first unit of q].
// (grid-stride over the `ntiles` tiles of the reserved unit capacity: the
// grid is sized for the device, not for the capacity, and tiles past the
// round's unit count only write a zero sum)
__global__ void __launch_bounds__(kScanThreads) unit_scan_sums(const uint32_t *cnt,
                                                               const uint64_t *n_dev,
                                                               uint64_t *tsum, uint32_t ntiles) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t tot;
  const uint64_t n = *n_dev;
  for (uint32_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const uint64_t t0 = (uint64_t)tile * kScanTile;
    if (t0 >= n) {
      if (threadIdx.x == 0) tsum[tile] = 0;
      continue;
    }
    uint64_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
      const uint64_t idx = t0 + (uint64_t)threadIdx.x * kScanItems + i;
      if (idx < n) s += cnt[idx];
    }
    block_excl_scan<uint64_t>(s, ws, &tot);
    if (threadIdx.x == 0) tsum[tile] = tot;
  }
}
__global__ void __launch_bounds__(kScanThreads) unit_scan_apply(const uint32_t *cnt,
                                                                const uint64_t *n_dev,
                                                                const uint64_t *toff,
                                                                uint64_t *out, uint32_t ntiles) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t tot;
  const uint64_t n = *n_dev;
  for (uint32_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    const uint64_t t0 = (uint64_t)tile * kScanTile;
    if (t0 >= n) break;   // tiles are visited in increasing order per block
    uint64_t loc[kScanItems];
    uint64_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
      const uint64_t idx = t0 + (uint64_t)threadIdx.x * kScanItems + i;
      loc[i] = idx < n ? cnt[idx] : 0;
      s += loc[i];
    }
    uint64_t run = toff[tile] + block_excl_scan<uint64_t>(s, ws, &tot);
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
      const uint64_t idx = t0 + (uint64_t)threadIdx.x * kScanItems + i;
      if (idx < n) out[idx] = run;
      run += loc[i];
    }
  }
}

// Warp per unit: copy its survivors from the bump area to the next
// intermediate, in unit (= docID) order.  Rounds 1 and 2 write their buffers
// (rbuf1, rbuf0) for the first time: survivors are packed by actual count, unit
// u at the exclusive scan of unit counts, so a buffer only has to hold what the
// round produces (a round that does not fit flags an overflow and writes
// nothing).  Later rounds (the SvS loop without the probe pass) write each
// query in place over its own region of round r-2 in the same buffer, which it
// fits (SvS survivor sets only shrink) and which no finished query uses.  The
// warp holding a query's last unit publishes its new |R| and region offset.
__global__ void __launch_bounds__(256) compact_copy_kernel(RoundArgs a, const uint64_t *udst) {
  const uint32_t lane = lane_id();
  const uint64_t *ubase = a.unit_base;
  const uint64_t total = ubase[a.nq];
  const bool packed = a.round <= 2;
  if (packed && a.scal[kScalRoundTot] > a.entry_cap) {
    if (blockIdx.x == 0 && threadIdx.x == 0)
      atomicOr(reinterpret_cast<int *>(a.scal + kScalStatus), kStatusOverflow);
    return;
  }
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t u = blockIdx.x * (uint64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); u < total;
       u += nwarps) {
    const uint64_t my = udst[u];
    const uint32_t cnt = a.unit_cnt[u];
    const uint2 *src = a.bump + a.unit_off[u];
    uint2 *dst;
    if (packed) {   // rounds 1-2: the packed offset (per-query bookkeeping: compact_queries_kernel)
      dst = a.rnext + my;
    } else {
      const uint32_t q = a.urec[u].x;   // the partition stage's record
      const uint64_t base = udst[ubase[q]];
      dst = a.rnext + a.roff_next[q] + (my - base);
      if (lane == 0 && u + 1 == ubase[q + 1]) {
        a.rcount[q] = (uint32_t)(my + cnt - base);
        a.rsel[q] = (uint8_t)(a.round & 1u);
      }
    }
    // four entries per lane in flight
    for (uint32_t i0 = 0; i0 < cnt; i0 += 128u) {
      uint2 v[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t i = i0 + 32u * j + lane;
        if (i < cnt) v[j] = src[i];
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t i = i0 + 32u * j + lane;
        if (i < cnt) dst[i] = v[j];
      }
    }
  }
}

// Packed rounds: per query, its survivors' count, buffer and packed offset
// (the exclusive scan of its units' counts; rtot = the round's total).
__global__ void compact_queries_kernel(RoundArgs a, const uint64_t *udst) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= a.nq || a.scal[kScalRoundTot] > a.entry_cap) return;
  const uint64_t total = a.unit_base[a.nq], rtot = a.scal[kScalRoundTot];
  const uint64_t u0 = a.unit_base[q], u1 = a.unit_base[q + 1];
  if (u0 == u1) return;   // no units this round: the query's count stays as planned (0)
  const uint64_t b0 = udst[u0], b1 = u1 < total ? udst[u1] : rtot;
  a.rcount[q] = (uint32_t)(b1 - b0);
  a.rsel[q] = (uint8_t)(a.round & 1u);
  a.roff_next[q] = b0;
}

// Query q's final intermediate: buffer rsel[q] at q's offset in that buffer
// (roff holds one per-query offset array per buffer: [0, nq] rbuf0, then rbuf1).
__device__ __forceinline__ const uint2 *final_region(const uint8_t *rsel, const uint64_t *roff,
                                                     uint32_t nq, const uint2 *rb0,
                                                     const uint2 *rb1, uint32_t q) {
  return rsel[q] ? rb1 + roff[(size_t)nq + 1 + q] : rb0 + roff[q];
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
        // stride is a power of two: 2*stride*(t/stride) + t%stride without division
        const uint32_t lo = ((t & ~(stride - 1u)) << 1) | (t & (stride - 1u));
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

struct SelectSmem {
  uint32_t hist[256];
  uint64_t prefix;
  uint32_t need, digit, bcount, cnt;
};

// Warp 0 finds, scanning the 256 digit bins from the top, the bin holding the
// need-th largest key; updates prefix/need.  Caller synchronises.
__device__ __forceinline__ void select_digit(SelectSmem &ss, int shift) {
  if (threadIdx.x < 32) {
    const uint32_t lane = threadIdx.x;
    const uint32_t need = ss.need;   // read by every lane before any lane updates it
    uint32_t loc[8], s = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) {  // lane l owns bins 255-8l .. 248-8l (descending)
      loc[i] = ss.hist[255 - 8 * lane - i];
      s += loc[i];
    }
    const uint32_t incl = warp_incl_scan(s);
    __syncwarp();
    const uint32_t excl = incl - s;
    if (excl < need && need <= incl) {
      uint32_t cum = excl;
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        if (cum < need && need <= cum + loc[i]) {
          const uint32_t d = 255 - 8 * lane - i;
          ss.prefix |= (uint64_t)d << shift;
          ss.need = need - cum;
          ss.bcount = loc[i];
        }
        cum += loc[i];
      }
    }
  }
}

// Exact CTA radix select on unique keys: returns thr such that exactly kk of the
// keys produced by key(i), i < n, are >= thr (8-bit digits, MSB first; stops
// when the selected bin holds a single key).
template <class KeyF>
__device__ uint64_t cta_radix_select(KeyF key, uint32_t n, uint32_t kk, SelectSmem &ss) {
  if (threadIdx.x == 0) {
    ss.prefix = 0;
    ss.need = kk;
  }
  uint64_t mask = 0;
  for (int shift = 56; shift >= 0; shift -= 8) {
    for (uint32_t i = threadIdx.x; i < 256; i += blockDim.x) ss.hist[i] = 0;
    __syncthreads();
    const uint64_t prefix = ss.prefix;
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
      const uint64_t x = key(i);
      if ((x & mask) == prefix) atomicAdd(&ss.hist[(x >> shift) & 255u], 1u);
    }
    __syncthreads();
    select_digit(ss, shift);
    __syncthreads();
    mask |= 0xFFull << shift;
    if (ss.bcount == 1 && ss.need == 1) {
      // the single key in the bin is the threshold
      const uint64_t p = ss.prefix;
      __syncthreads();
      for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
        const uint64_t x = key(i);
        if ((x & mask) == p) ss.prefix = x;
      }
      __syncthreads();
      return ss.prefix;
    }
  }
  return ss.prefix;
}

// Top-k threshold of a 2-term word-AND query (round 1 is its last round): the
// k-th largest key among a SUBSET of its survivors — strided 32-word steps of
// the AND over R's docID range, up to kTauKeys keys — is at most its k-th
// largest key overall (the subset's k largest are survivors), so every key of
// its top-k is >= it and bitand_unit may drop the survivors below it (exact;
// keys are unique).  tau = 0 (no dropping) when the subset holds
// fewer than k keys, for other queries, and when k > kTauKeys / 2.
#ifndef GRIFFIN_TAU_KEYS
#define GRIFFIN_TAU_KEYS 8192
#endif
constexpr uint32_t kTauKeys = GRIFFIN_TAU_KEYS;
__host__ __device__ inline size_t tau_smem_bytes() { return (size_t)kTauKeys * 8; }
__global__ void __launch_bounds__(1024) bitand_tau_kernel(DevIndex ix, RoundArgs a, uint32_t k,
                                                         uint64_t *tau) {
  extern __shared__ uint64_t tkeys[];
  __shared__ SelectSmem ss;
  __shared__ uint32_t nk;
  const uint32_t lane = lane_id(), warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
  for (uint32_t q = blockIdx.x; q < a.nq; q += gridDim.x) {
    const uint32_t *pt = a.plan_terms + (size_t)q * kMaxTerms;
    if (a.qmode[q] != kModeBitAnd || a.plan_m[q] != 2 || k == 0 || k > kTauKeys / 2) {
      if (threadIdx.x == 0) tau[q] = 0;
      continue;
    }
    const TermInfo tR = ix.terms[pt[0]], tS = ix.terms[pt[1]];
    const uint2 *bR = a.bm + (size_t)a.bm_slot[pt[0]] * a.bm_words;
    const uint2 *bS = a.bm + (size_t)a.bm_slot[pt[1]] * a.bm_words;
    const uint32_t w0 = __ldg(ix.first + tR.block0) >> 5;
    const uint32_t nch = (a.bm_words - w0 + 31u) / 32u;
    // stride over 32-word steps so the sample holds about kTauKeys keys
    // (an estimate: a subset of any size is exact, a larger one is tighter)
    const double est = (double)tR.df_local * (double)tS.df_local / (double)max(1u, ix.n_docs);
    const uint32_t stride = max(1u, (uint32_t)(est / kTauKeys));
    if (threadIdx.x == 0) nk = 0;
    __syncthreads();
    // four 32-word steps per warp in flight
    for (uint32_t c0 = warp * stride * 4u; c0 < nch; c0 += nwarps * stride * 4u) {
      if (*(volatile uint32_t *)&nk >= kTauKeys) break;
      uint2 ra[4], sa[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t c = c0 + (uint32_t)j * stride;
        const uint32_t w = w0 + c * 32u + lane;
        const bool in = c < nch && w < a.bm_words;
        ra[j] = in ? __ldg(bR + w) : make_uint2(0, 0);
        sa[j] = in ? __ldg(bS + w) : make_uint2(0, 0);
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t w = w0 + (c0 + (uint32_t)j * stride) * 32u + lane;
        uint32_t m = ra[j].x & sa[j].x;
        while (m) {
          const uint32_t bit = __ffs(m) - 1u;
          m &= m - 1u;
          const uint32_t below = (1u << bit) - 1u, doc = (w << 5) | bit;
          const float nrm = __ldg(ix.norm + doc);
          const float wS = bm25_w(tS.idf, tf_lookup(ix, tS, ~sa[j].y + __popc(sa[j].x & below)), nrm, ix.k1p1);
          const float wR = bm25_w(tR.idf, tf_lookup(ix, tR, ~ra[j].y + __popc(ra[j].x & below)), nrm, ix.k1p1);
          const uint32_t slot = atomicAdd(&nk, 1u);
          if (slot < kTauKeys)
            tkeys[slot] = make_key(make_uint2(doc, __float_as_uint(__fadd_rn(wR, wS))), ix.doc_base);
        }
      }
    }
    __syncthreads();
    const uint32_t n = min(nk, kTauKeys);
    uint64_t thr = 0;
    if (n >= k) thr = cta_radix_select([&](uint32_t i) { return tkeys[i]; }, n, k, ss);
    if (threadIdx.x == 0) tau[q] = thr;
    __syncthreads();
  }
}

constexpr int kTopkMaxLevels = 5;
struct CandBufs {
  uint64_t *lv[kTopkMaxLevels + 1];   // lv[L] = candidates produced by level L (L >= 1)
};

// Per query, where its current top-k candidates live: qlev 0 = the survivor
// entries of the final intersection round, qlev L >= 1 = cand level L at qoff.
struct TopkState {
  uint8_t *qlev;
  uint64_t *qoff;
  uint32_t *qn;
  // sampled-threshold pre-filter (queries with > kFiltMin candidates)
  uint64_t *flt;     // slot s holds keys at flt[s * kFiltCap ..]
  uint64_t *ftau;    // per query: threshold key
  uint32_t *fslot;   // per query: slot or kNone
  uint32_t *fcnt;    // per slot: keys >= threshold seen
  uint32_t *fctr;    // slots handed out
  uint32_t fmax;     // slots available (0 = pre-filter off)
};
constexpr uint8_t kLevFilt = 7;            // qlev: candidates are the query's filter slot
constexpr uint32_t kFiltMin = 65536;       // pre-filter queries with more candidates than this
constexpr uint32_t kFiltCap = 65536;       // keys kept per filtered query (else fall back)
constexpr uint32_t kFiltSample = kTopkSmem;
constexpr size_t kFiltSlots = 256;
constexpr uint64_t kFiltBatchMin = 64ull << 20;   // see topk_filter_on         // filtered queries per batch (the rest: no filter)

__device__ __forceinline__ const uint64_t *cand_keys(const CandBufs &cb, const TopkState &ts,
                                                     uint32_t lev, uint32_t q) {
  return lev == kLevFilt ? ts.flt + ts.qoff[q] : cb.lv[lev] + ts.qoff[q];
}

__global__ void topk_init_kernel(uint32_t nq, const uint32_t *rcount, TopkState ts) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q < nq) {
    ts.qlev[q] = 0;
    ts.qoff[q] = 0;
    ts.qn[q] = rcount[q];
    if (ts.fmax) ts.fslot[q] = kNone;
  }
  if (q == 0 && ts.fmax) *ts.fctr = 0;
}

// Pre-filter, step 1 (one CTA per query with n > kFiltMin candidates): a
// systematic sample of kFiltSample keys; its r-th largest key becomes the
// query's threshold tau, with r = mu + 4 sqrt(mu) + 2 for mu = k*s/n the
// expected number of sampled keys among the true top k, so that with high
// probability >= k keys are >= tau while only ~r*n/s survive the filter.
// Exactness never depends on the sample: a query whose filtered count is < k
// (or overflows kFiltCap) keeps its unfiltered candidates (topk_filter_update).
__global__ void __launch_bounds__(kTopkThreads) topk_sample_kernel(
    DevIndex ix, uint32_t nq, uint32_t k, const uint8_t *rsel, const uint64_t *cap_off,
    const uint2 *rb0, const uint2 *rb1, TopkState ts) {
  __shared__ uint64_t sk[kFiltSample];
  __shared__ SelectSmem ss;
  __shared__ uint32_t slot;
  for (uint32_t q = blockIdx.x; q < nq; q += gridDim.x) {
    const uint32_t n = ts.qn[q];
    if (n <= kFiltMin) continue;   // block-uniform
    const float mu = (float)k * (float)kFiltSample / (float)n;
    const uint32_t r = (uint32_t)ceilf(mu + 4.f * sqrtf(mu) + 2.f);
    if (r > kFiltSample / 8) continue;
    const uint2 *R = final_region(rsel, cap_off, nq, rb0, rb1, q);
    for (uint32_t j = threadIdx.x; j < kFiltSample; j += blockDim.x)
      sk[j] = make_key(R[(uint32_t)(((uint64_t)j * n) / kFiltSample)], ix.doc_base);
    __syncthreads();
    const uint64_t tau = cta_radix_select([&](uint32_t i) { return sk[i]; }, kFiltSample, r, ss);
    if (threadIdx.x == 0) {
      slot = atomicAdd(ts.fctr, 1u);
      if (slot < ts.fmax) {
        ts.ftau[q] = tau;
        ts.fcnt[slot] = 0;
        ts.fslot[q] = slot;
      }
    }
    __syncthreads();
  }
}

__global__ void topk_filter_plan_kernel(uint32_t nq, TopkState ts, uint32_t *nch) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q < nq) nch[q] = ts.fslot[q] != kNone ? (ts.qn[q] + kTopkSmem - 1) / kTopkSmem : 0u;
}

// Pre-filter, step 2: stream every candidate of the filtered queries (CTA per
// chunk of kTopkSmem) and append the keys >= tau to the query's slot
// (warp-aggregated atomics; order inside the slot is irrelevant).
__global__ void __launch_bounds__(256) topk_filter_kernel(
    DevIndex ix, uint32_t nq, const uint8_t *rsel, const uint64_t *cap_off, const uint2 *rb0,
    const uint2 *rb1, TopkState ts, const uint64_t *cbase) {
  const uint64_t total = cbase[nq];
  const uint32_t lane = lane_id();
  for (uint64_t c = blockIdx.x; c < total; c += gridDim.x) {
    uint32_t lo = 0, hi = nq;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (cbase[mid] <= c) lo = mid; else hi = mid;
    }
    const uint32_t q = lo;
    const uint32_t ci = (uint32_t)(c - cbase[q]);
    const uint32_t len = min(kTopkSmem, ts.qn[q] - ci * kTopkSmem);
    const uint2 *R = final_region(rsel, cap_off, nq, rb0, rb1, q) + (size_t)ci * kTopkSmem;
    const uint64_t tau = ts.ftau[q];
    const uint32_t slot = ts.fslot[q];
    uint64_t *out = ts.flt + (size_t)slot * kFiltCap;
    // four entries per lane in flight; one output reservation per 128 entries
    for (uint32_t i0 = (threadIdx.x - lane) * 4u; i0 < len; i0 += blockDim.x * 4u) {
      uint64_t x[4];
      bool keep[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const uint32_t i = i0 + 32u * j + lane;
        x[j] = i < len ? make_key(R[i], ix.doc_base) : 0ull;
        keep[j] = i < len && x[j] >= tau;
      }
      uint32_t bal[4], tot = 0;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        bal[j] = __ballot_sync(0xffffffffu, keep[j]);
        tot += __popc(bal[j]);
      }
      if (tot) {
        uint32_t base = 0;
        if (lane == 0) base = atomicAdd(ts.fcnt + slot, tot);
        base = __shfl_sync(0xffffffffu, base, 0);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const uint32_t pos = base + __popc(bal[j] & lanemask_lt());
          if (keep[j] && pos < kFiltCap) out[pos] = x[j];
          base += __popc(bal[j]);
        }
      }
    }
  }
}

// Pre-filter, step 3: a query whose slot holds >= min(k, n) keys (and did not
// overflow) continues from its slot; otherwise from all its candidates.
__global__ void topk_filter_update_kernel(uint32_t nq, uint32_t k, TopkState ts) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= nq) return;
  const uint32_t slot = ts.fslot[q];
  if (slot == kNone) return;
  const uint32_t f = ts.fcnt[slot];
  if (f >= min(k, ts.qn[q]) && f <= kFiltCap) {
    ts.qlev[q] = kLevFilt;
    ts.qoff[q] = (uint64_t)slot * kFiltCap;
    ts.qn[q] = f;
  }
}

__global__ void topk_plan_kernel(uint32_t nq, TopkState ts, uint32_t *nch) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q < nq) {
    const uint32_t c = ts.qn[q];
    nch[q] = c > kTopkSmem ? (c + kTopkSmem - 1) / kTopkSmem : 0u;
  }
}

__global__ void topk_update_kernel(uint32_t nq, uint32_t k, uint32_t level, TopkState ts,
                                   const uint32_t *nch, const uint64_t *cbase) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q < nq && nch[q]) {
    ts.qlev[q] = (uint8_t)level;
    ts.qoff[q] = cbase[q] * k;
    ts.qn[q] = nch[q] * k;
  }
}

// One selection level: every query with more than kTopkSmem candidates is cut
// into chunks of kTopkSmem; each chunk (one CTA, keys staged in smem) keeps its
// top min(k, len) keys at out[(cbase[q] + ci) * k ...] (zero-padded).  Levels
// repeat until every query's candidates fit one CTA's shared memory.
__global__ void __launch_bounds__(kTopkThreads) topk_chunk_kernel(
    DevIndex ix, uint32_t nq, uint32_t k, const uint8_t *rsel, const uint64_t *cap_off,
    const uint2 *rb0, const uint2 *rb1, TopkState ts, CandBufs cb, const uint64_t *cbase,
    uint64_t *out_lv) {
  __shared__ uint64_t sk[kTopkSmem];
  __shared__ SelectSmem ss;
  const uint64_t total = cbase[nq];
  for (uint64_t c = blockIdx.x; c < total; c += gridDim.x) {
    uint32_t lo = 0, hi = nq;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (cbase[mid] <= c) lo = mid; else hi = mid;
    }
    const uint32_t q = lo;
    const uint32_t ci = (uint32_t)(c - cbase[q]);
    const uint32_t lev = ts.qlev[q];
    const uint32_t len = min(kTopkSmem, ts.qn[q] - ci * kTopkSmem);
    if (lev == 0) {
      const uint2 *R = final_region(rsel, cap_off, nq, rb0, rb1, q) + (size_t)ci * kTopkSmem;
      for (uint32_t i = threadIdx.x; i < len; i += blockDim.x) sk[i] = make_key(R[i], ix.doc_base);
    } else {
      const uint64_t *K = cand_keys(cb, ts, lev, q) + (size_t)ci * kTopkSmem;
      for (uint32_t i = threadIdx.x; i < len; i += blockDim.x) sk[i] = K[i];
    }
    __syncthreads();
    uint64_t *out = out_lv + c * k;
    const uint32_t kk = min(k, len);
    if (kk == len) {
      for (uint32_t i = threadIdx.x; i < k; i += blockDim.x) out[i] = i < len ? sk[i] : 0ull;
    } else {
      // inputs of levels >= 2 carry zero padding (below every real key; not
      // unique): keep the nonzero keys >= thr — exactly kk when thr > 0, all of
      // them (< kk) when thr == 0 — and zero-fill the rest of the k slots
      const uint64_t thr = cta_radix_select([&](uint32_t i) { return sk[i]; }, len, kk, ss);
      if (threadIdx.x == 0) ss.cnt = 0;
      __syncthreads();
      for (uint32_t i = threadIdx.x; i < len; i += blockDim.x)
        if (sk[i] >= thr && sk[i] != 0ull) out[atomicAdd(&ss.cnt, 1u)] = sk[i];
      __syncthreads();
      for (uint32_t i = ss.cnt + threadIdx.x; i < k; i += blockDim.x) out[i] = 0ull;
    }
    __syncthreads();
  }
}

// Final, per query: select the top kk of its current candidates in smem (or by
// global radix passes when they still do not fit), bitonic-sort, write keys +
// count.  Zero keys (chunk padding) are below every real key.
__global__ void __launch_bounds__(kTopkThreads) topk_final_kernel(
    DevIndex ix, uint32_t nq, uint32_t k, const uint32_t *rcount, const uint8_t *rsel,
    const uint64_t *cap_off, const uint2 *rb0, const uint2 *rb1, TopkState ts, CandBufs cb,
    uint64_t *out_keys, uint32_t *out_counts) {
  __shared__ uint64_t sk[kTopkSmem];
  __shared__ SelectSmem ss;
  for (uint32_t q = blockIdx.x; q < nq; q += gridDim.x) {
    const uint32_t c = rcount[q];
    const uint32_t kk = min(k, c);
    const uint2 *R = final_region(rsel, cap_off, nq, rb0, rb1, q);
    const uint32_t lev = ts.qlev[q];
    const uint64_t *C = lev ? cand_keys(cb, ts, lev, q) : nullptr;
    const uint32_t n = ts.qn[q];
    auto key = [&](uint32_t i) -> uint64_t { return lev ? C[i] : make_key(R[i], ix.doc_base); };
    uint32_t nsel;
    if (n <= kTopkSmem) {
      for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) sk[i] = key(i);
      __syncthreads();
      if (kk < n) {
        const uint64_t thr = cta_radix_select([&](uint32_t i) { return sk[i]; }, n, kk, ss);
        if (threadIdx.x == 0) ss.cnt = 0;
        __syncthreads();
        uint64_t mine[kTopkSmem / kTopkThreads];
        uint32_t nm = 0;
        for (uint32_t i = threadIdx.x; i < n; i += blockDim.x)
          if (sk[i] >= thr) mine[nm++] = sk[i];
        __syncthreads();
        for (uint32_t j = 0; j < nm; ++j) sk[atomicAdd(&ss.cnt, 1u)] = mine[j];
        __syncthreads();
      }
      nsel = kk;
    } else {
      const uint64_t thr = cta_radix_select(key, n, kk, ss);
      if (threadIdx.x == 0) ss.cnt = 0;
      __syncthreads();
      for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
        const uint64_t x = key(i);
        if (x >= thr) sk[atomicAdd(&ss.cnt, 1u)] = x;
      }
      __syncthreads();
      nsel = kk;
    }
    uint32_t nsort = 1;
    while (nsort < nsel) nsort <<= 1;
    for (uint32_t i = nsel + threadIdx.x; i < nsort; i += blockDim.x) sk[i] = 0ull;
    __syncthreads();
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

// The same G-way merge reading each shard's runs where they live (NEXT-2, fused
// exchange + merge): run g is keys[g][q*k ..], counts[g][q] — device pointers
// that may be on peer GPUs (loads go over NVLink once peer access is enabled).
struct PeerRuns {
  const uint64_t *keys[GRIFFIN_MAX_SHARDS];
  const uint32_t *counts[GRIFFIN_MAX_SHARDS];
};
__global__ void merge_topk_peer_kernel(uint32_t G, uint32_t nq, uint32_t k, PeerRuns r,
                                       uint64_t *out, uint32_t *out_counts) {
  const uint32_t lane = lane_id();
  const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
  for (uint32_t q = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); q < nq; q += nwarps) {
    const uint32_t cnt = lane < G ? min(r.counts[lane][q], k) : 0u;
    const uint64_t *run = lane < G ? r.keys[lane] + (size_t)q * k : nullptr;
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

// Warp decodes the consecutive blocks [k0, k0+nb) (nb <= D+2) of the shard into
// w.tile via one TMA bulk copy; returns total postings and payload bytes.
template <class Sink = StoreSink>
__device__ __forceinline__ uint32_t decode_run(const DevIndex &ix, WarpSmem &w, uint32_t D,
                                               uint64_t k0, uint32_t nb, uint32_t *pay_bytes,
                                               uint32_t *my_n = nullptr, uint32_t *dst = nullptr,
                                               Sink *sink = nullptr) {
  const uint32_t lane = lane_id();
  uint2 m = make_uint2(0, 0);
  uint32_t f = 0, sz = 0;
  if (lane < nb) {
    m = ix.meta[k0 + lane];
    f = ix.first[k0 + lane];
    sz = block_size16(m.y);
  }
  if (sink) stage_decode_lanes(ix, w, stage_words(ix.B, D) / 4u, 0, nb, m, f, sz, dst ? dst : w.tile, *sink);
  else stage_decode_lanes(ix, w, stage_words(ix.B, D) / 4u, 0, nb, m, f, sz, dst ? dst : w.tile);
  const uint32_t tot = __reduce_add_sync(0xffffffffu, lane < nb ? meta_n(m.y) : 0u);
  *pay_bytes = __reduce_add_sync(0xffffffffu, sz) * 16u;
  if (my_n) *my_n = lane < nb ? meta_n(m.y) : 0u;
  return tot;
}

__global__ void __launch_bounds__(256) decode_list_kernel(DevIndex ix, uint32_t D, uint32_t block0,
                                                          uint32_t nblocks, uint32_t *out) {
  extern __shared__ uint4 smem4[];
  const uint32_t lane = lane_id();
  WarpSmem w = carve_warp_smem(smem4, ix.B, D);
  cta_smem_init(smem4, w);
  const uint32_t run = D + 2;
  const uint32_t nruns = (nblocks + run - 1) / run;
  const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
  for (uint32_t r = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); r < nruns; r += nwarps) {
    const uint32_t k = r * run, nb = min(run, nblocks - k);
    uint32_t pay;
    const uint32_t n = decode_run(ix, w, D, (uint64_t)block0 + k, nb, &pay);
    for (uint32_t i = lane; i < n; i += 32) out[(size_t)k * ix.B + i] = w.tile[i] + ix.doc_base;
    __syncwarp();
  }
}

// Decode sweep: every block of the shard once (runs of D+2 blocks per warp).
__global__ void __launch_bounds__(256) decode_all_kernel(DevIndex ix, uint32_t D, uint64_t nblocks,
                                                         unsigned long long *acc) {
  // D = sweep_D(B): the launcher sizes shared memory for it
  extern __shared__ uint4 smem4[];
  const uint32_t lane = lane_id();
  WarpSmem w = carve_warp_smem(smem4, ix.B, D, false);   // no tile: XorSink
  cta_smem_init(smem4, w);
  const uint32_t run = D + 2;
  const uint64_t nruns = (nblocks + run - 1) / run;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  uint32_t x = 0;
  unsigned long long post = 0, pay = 0;
  for (uint64_t r = blockIdx.x * (uint64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); r < nruns;
       r += nwarps) {
    const uint64_t k = r * run;
    const uint32_t nb = (uint32_t)((nblocks - k) < run ? (nblocks - k) : run);
    uint32_t p;
    // decoded docIDs are folded into a register checksum by the decoder itself
    // (XorSink): the sweep measures decoding, not a tile write + re-read
    XorSink xs;
    const uint32_t n = decode_run(ix, w, D, k, nb, &p, nullptr, nullptr, &xs);
    x ^= xs.x;
    post += n;
    pay += p + 8u * nb;
  }
  for (int d = 16; d; d >>= 1) x ^= __shfl_xor_sync(0xffffffffu, x, d);
  if (lane == 0) {
    atomicXor(acc + 0, (unsigned long long)x);
    atomicAdd(acc + 1, post);
    atomicAdd(acc + 2, pay);
  }
}

// ------------------------------------------------------------------- batch reuse

// Estimated block demand of every term in the batch: round 1 reads all blocks
// of t0; each later term is merged (all its blocks) or galloped (<= |R| blocks),
// with |R| bounded by the query's region cap after round 1.
__global__ void demand_kernel(DevIndex ix, RoundArgs a, uint32_t *demand) {
  const uint32_t q = blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= a.nq) return;
  const uint32_t m = a.plan_m[q];
  if (!m || !a.cap[q]) return;
  const uint32_t *pt = a.plan_terms + (size_t)q * kMaxTerms;
  const TermInfo t0 = ix.terms[pt[0]];
  atomicAdd(&demand[pt[0]], t0.nblocks);
  uint64_t r_est = t0.df_local;
  for (uint32_t r = 1; r < m; ++r) {
    const TermInfo tS = ix.terms[pt[r]];
    const bool gallop = a.forced_mode == 2 ||
                        (a.forced_mode == 0 && (uint64_t)tS.df_local > (uint64_t)a.T * r_est);
    const uint32_t add = gallop ? (uint32_t)(r_est < tS.nblocks ? r_est : tS.nblocks) : tS.nblocks;
    atomicAdd(&demand[pt[r]], add);
    if (r == 1) r_est = a.cap[q];
  }
}

// bm_slot (or null: bitvectors off): a selected term with a bitvector slot is
// decoded into it (kDecBitmap), any other selected term into the arena.
__global__ void select_kernel(DevIndex ix, const uint32_t *demand, const uint32_t *bm_slot,
                              uint8_t *tdec, uint32_t *runs, uint32_t run_len) {
  const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= ix.num_terms) return;
  const uint32_t nb = ix.terms[t].nblocks;
  // decode once if the batch would otherwise decode >= 1.5x the list's blocks
  const bool sel = nb > 0 && 2ull * demand[t] >= 3ull * nb;
  tdec[t] = sel ? ((bm_slot && bm_slot[t] != kNone) ? kDecBitmap : kDecArena) : kDecNone;
  runs[t] = sel ? (nb + run_len - 1) / run_len : 0u;
}

// Zero the bitvector slots of this batch's kDecBitmap terms (slot-major grid).
__global__ void bm_zero_kernel(const uint8_t *tdec, const uint32_t *bm_term, uint32_t nslots,
                               uint32_t words, uint4 *bm) {
  const uint32_t per = (words + 1u) / 2u;   // uint4 = two words
  for (uint32_t s = blockIdx.y; s < nslots; s += gridDim.y) {
    if (tdec[bm_term[s]] != kDecBitmap) continue;
    uint4 *p = bm + (size_t)s * per;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < per; i += gridDim.x * blockDim.x)
      p[i] = make_uint4(0, 0, 0, 0);
  }
}

#ifndef GRIFFIN_DECODE_ONCE_MINB
#define GRIFFIN_DECODE_ONCE_MINB 3
#endif
// Para-EF decode of every block of the selected terms into the arena
// (slot = global block * B + i): warp per run of <= D+2 consecutive blocks,
// TMA-staged payloads, decoded tile written back with 128-bit stores.
// run -> term map for decode_once (replaces a per-run binary search over run_base)
__global__ void run_map_kernel(uint32_t V, const uint32_t *runs, const uint64_t *run_base,
                               uint32_t *run_term) {
  const uint32_t t = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;   // warp per term
  if (t >= V) return;
  const uint32_t nr = runs[t];
  const uint64_t b = run_base[t];
  for (uint32_t i = lane_id(); i < nr; i += 32) run_term[b + i] = t;
}

__global__ void __launch_bounds__(256, GRIFFIN_DECODE_ONCE_MINB) decode_once_kernel(DevIndex ix, uint32_t D,
                                                          const uint64_t *run_base,
                                                          const uint32_t *run_term, uint32_t *arena,
                                                          const uint8_t *tdec, uint2 *bm,
                                                          const uint32_t *bm_slot, uint32_t bm_words,
                                                          unsigned long long *scal) {
  extern __shared__ uint4 smem4[];
  const uint32_t lane = lane_id();
  WarpSmem w = carve_warp_smem(smem4, ix.B, D, false);
  cta_smem_init(smem4, w);
  const uint32_t V = ix.num_terms, run = D + 2, B = ix.B;
  const uint64_t total = run_base[V];
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  unsigned long long alg = 0, pay = 0, post = 0, c8d = 0;
  for (uint64_t r = blockIdx.x * (uint64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); r < total;
       r += nwarps) {
    const uint32_t lo = run_term[r];
    const TermInfo t = ix.terms[lo];
    const uint32_t ri = (uint32_t)(r - run_base[lo]);
    const uint32_t k0 = ri * run, nb = min(run, t.nblocks - k0);
    const uint64_t gb = (uint64_t)t.block0 + k0;
    uint32_t p, n;
    if (tdec[lo] == kDecBitmap) {
      // dense list: into its bitvector + rank (arena + gb * B only names positions)
      BitSink bs;
      bs.bm = bm + (size_t)bm_slot[lo] * bm_words;
      bs.tile = arena + gb * B;
      bs.pos0 = k0 * B;
      n = decode_run(ix, w, D, gb, nb, &p, nullptr, arena + gb * B, &bs);
      bs.finish();
      if (lane == 0) alg += p + 8ull * nb + (uint64_t)bm_words * 8ull * nb / t.nblocks;
    } else {
      // decoded straight into the arena (128-bit stores, coalesced per half-warp)
      n = decode_run(ix, w, D, gb, nb, &p, nullptr, arena + gb * B);
      if (lane == 0) alg += p + 8ull * nb + 4ull * n;
    }
    if (lane == 0) {
      pay += p;
      post += n;
      c8d += p + 8ull * nb;
    }
  }
  if (lane == 0) {
    if (alg) atomicAdd(scal + kScalDec + 0, alg);
    if (pay) atomicAdd(scal + kScalDec + 1, pay);
    if (post) atomicAdd(scal + kScalDec + 2, post);
    if (c8d) atomicAdd(scal + kScalDecC8d, c8d);
  }
}

// ------------------------------------------------------------------- host side

int num_sms(int dev) {
  static std::atomic<int> cache[64];   // zero-initialised; written by any launching thread
  int v = 0;
  if (dev < 0 || dev >= 64) {
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev < 0 ? 0 : dev);
    return v > 0 ? v : 1;
  }
  if (!(v = cache[dev].load(std::memory_order_relaxed))) {
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    v = v > 0 ? v : 1;
    cache[dev].store(v, std::memory_order_relaxed);
  }
  return v;
}

static griffin_status ensure_bm_slots(griffin_index *ix);
// S-locality buckets: merge units by S block, then bitvector units by (S slot, R docID)
static uint64_t sorder_merge_buckets(const griffin_index *ix) {
  return (ix->nblocks >> ix->sorder_shift) + 1;
}
static uint32_t sorder_bm_per_slot(const griffin_index *ix) {
  return ((ix->doc_end - ix->doc_base) >> kBmBucketShift) + 1;
}
static uint64_t sorder_buckets(const griffin_index *ix) {
  return sorder_merge_buckets(ix) + (uint64_t)ix->bm_nslots * sorder_bm_per_slot(ix);
}

griffin_status reserve_ws(griffin_index *ix, Workspace &w, uint32_t nq, uint64_t units,
                          uint64_t entries) {
  // `entries` is the exact per-batch bound (sum over queries of min(df0, df1));
  // a budget caps it: the intermediates are packed by actual survivors, and a
  // batch whose survivors exceed it reports GRIFFIN_ERR_OOM (overflow)
  if (ix->entry_budget && entries > ix->entry_budget) entries = ix->entry_budget;
  const size_t q = (size_t)nq + 1;
  GRIFFIN_CUDA_TRY(w.plan_terms.reserve(q * kMaxTerms * 4));
  GRIFFIN_CUDA_TRY(w.plan_m.reserve(q * 4));
  GRIFFIN_CUDA_TRY(w.cap.reserve(q * 4));
  GRIFFIN_CUDA_TRY(w.cap_off.reserve(2 * q * 8 + 8));   // per-query region offsets, per buffer
  GRIFFIN_CUDA_TRY(w.rcount.reserve(q * 4));
  GRIFFIN_CUDA_TRY(w.rsel.reserve(q));
  GRIFFIN_CUDA_TRY(w.qmode.reserve(q * 4 + q * 4));  // qmode | qunits
  GRIFFIN_CUDA_TRY(w.unit_base.reserve(q * 8 + 8 + (q / kScanTile + 8) * 8));
  GRIFFIN_CUDA_TRY(w.unit_off.reserve((units + 1) * 8));
  GRIFFIN_CUDA_TRY(w.unit_cnt.reserve((units + 1) * 4));
  GRIFFIN_CUDA_TRY(w.urec.reserve((units + 2) * 16));
  GRIFFIN_CUDA_TRY(w.uperm.reserve((units + 2) * 16));
  GRIFFIN_CUDA_TRY(w.unit_dst.reserve((units + 2) * 8 + (units / kScanTile + 2) * 8));
  if (ix->sorder && nq >= kSorderMinQueries) {   // S-locality buckets (no allocation in run_batch)
    griffin_status bs = ensure_bm_slots(ix);
    if (bs) return bs;
    const size_t nbkt = sorder_buckets(ix);
    GRIFFIN_CUDA_TRY(w.sbkt_cnt.reserve(nbkt * 4));
    GRIFFIN_CUDA_TRY(w.sbkt_pos.reserve((nbkt + 1) * 8));
    GRIFFIN_CUDA_TRY(w.sbkt_tmp.reserve((nbkt / kScanTile + 4) * 8));
  }
  GRIFFIN_CUDA_TRY(w.rbuf0.reserve((entries + 1) * 8));
  GRIFFIN_CUDA_TRY(w.rbuf1.reserve((entries + 1) * 8));
  // per-warp bump chunks: at most one partly used chunk per resident warp
  const size_t bump_slack = (size_t)num_sms(ix->device) * 64 * kBumpChunk;
  GRIFFIN_CUDA_TRY(w.bump.reserve((entries + bump_slack + 1) * 8));
  if (!w.scal.p) {
    GRIFFIN_CUDA_TRY(w.scal.reserve(kScalCount * 8));
    GRIFFIN_CUDA_TRY(cudaMemset(w.scal.p, 0, w.scal.bytes));
  }
  // every buffer above was reserved for at least these sizes (grow-only)
  w.nq_cap = std::max<size_t>(w.nq_cap, nq);
  w.unit_cap = std::max<size_t>(w.unit_cap, units);
  w.entry_cap = std::max<size_t>(w.entry_cap, entries);
  return GRIFFIN_OK;
}

// Per-stage instrumentation: an NVTX range around the stage's host-side
// launches (always; a no-op without an attached tool such as nsys/ncu
// --nvtx), and, while profiling is on, CUDA events on the launching stream.
static const char *const kStageNames[6] = {"griffin/plan", "griffin/intersect", "griffin/compact",
                                           "griffin/topk", "griffin/merge", "griffin/decode_once"};
struct StageTimer {
  griffin_index *ix;
  cudaStream_t st;
  int stage;
  cudaEvent_t a = nullptr, b = nullptr;
  StageTimer(griffin_index *ix_, cudaStream_t st_, int stage_) : ix(ix_), st(st_), stage(stage_) {
    nvtxRangePushA(kStageNames[stage]);
    if (!(ix->profiling & 1)) return;
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
    nvtxRangePop();
    if (!a) return;
    cudaEventRecord(b, st);
    ix->pending.push_back({stage, {a, b}});
  }
};

// Process-wide launch configuration of a kernel on a device: the dynamic
// shared-memory attribute only ever grows (several host threads — the multi-GPU
// handle's per-shard launchers — configure the same kernel for different block
// sizes; a per-thread cache could shrink it under another thread's launch), and
// the occupancy query runs once per (kernel, device, smem), not per launch.
cudaError_t launch_config(const void *fn, int dev, size_t smem, int threads, int *per_sm) {
  static std::mutex mu;
  static std::map<std::pair<const void *, int>, size_t> attr;
  static std::map<std::tuple<const void *, int, size_t>, int> occ;
  std::lock_guard<std::mutex> lk(mu);
  size_t &cur = attr[{fn, dev}];
  if (cur < smem) {
    const cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                               (int)smem);
    if (e != cudaSuccess) return e;
    cur = smem;
  }
  const auto key = std::make_tuple(fn, dev, smem);
  auto it = occ.find(key);
  if (it == occ.end()) {
    int p = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&p, fn, threads, smem);
    it = occ.emplace(key, std::max(1, p)).first;
  }
  if (per_sm) *per_sm = it->second;
  return cudaSuccess;
}

template <bool RC, int ROLE>
static cudaError_t launch_intersect(griffin_index *ix, const RoundArgs &ra, cudaStream_t st) {
  const size_t words = ROLE == 2 ? other_warp_smem_words(ix->B, ix->D, ra.nextgeq != 0)
                                 : warp_smem_words(ix->B, ix->D);
  const size_t smem = kLutBytes + words * 4 * kWarpsPerCta;
  int per_sm = 1;
  const cudaError_t e = launch_config((const void *)intersect_kernel<RC, ROLE>, ix->device, smem,
                                      kIntersectThreads, &per_sm);
  if (e != cudaSuccess) return e;
  const int grid = num_sms(ix->device) * per_sm;
  intersect_kernel<RC, ROLE><<<grid, kIntersectThreads, smem, st>>>(ix->dev(), ra);
  return cudaGetLastError();
}

static cudaError_t launch_probe(griffin_index *ix, const RoundArgs &ra, cudaStream_t st) {
  const size_t smem = kLutBytes + (size_t)probe_warp_smem_words(ix->B, ix->D, ra.nextgeq != 0) *
                                      4 * kWarpsPerCta;
  int per_sm = 1;
  const cudaError_t e = launch_config((const void *)probe_kernel, ix->device, smem,
                                      kIntersectThreads, &per_sm);
  if (e != cudaSuccess) return e;
  probe_kernel<<<num_sms(ix->device) * per_sm, kIntersectThreads, smem, st>>>(ix->dev(), ra);
  return cudaGetLastError();
}

// Top-k candidate buffers for a batch of nq queries with this k (grow-only;
// called before a CUDA-graph capture so no allocation happens inside it).
// Pre-filter policy: always for k > 64 (one chunk level keeps k of kTopkSmem
// keys, so a large k needs up to 4 levels over sets shrinking only ~4x); for
// k <= 64 only when the batch may hold > kFiltBatchMin candidates (C4/C5-size
// batches: one level over 10^8 keys costs more than sample + filter, while at
// C2 the extra launches cost 0.03 ms).  topk_filter: 0 off, 1 auto, 2 always.
static bool topk_filter_on(const griffin_index *ix, const Workspace &w, uint32_t k) {
  if (ix->topk_filter == 2) return true;
  return ix->topk_filter == 1 && (k > 64 || w.entry_cap > kFiltBatchMin);
}

griffin_status reserve_topk(griffin_index *ix, Workspace &w, uint32_t nq, uint32_t k) {
  const uint64_t cand_cap = (w.entry_cap / kTopkSmem + nq + 1) * (uint64_t)k;
  const int levels = k <= 64 ? 1 : (k <= 1024 ? 4 : (k <= 2048 ? kTopkMaxLevels : 0));
  GRIFFIN_CUDA_TRY(w.cand.reserve(cand_cap * 8 * std::max(levels, 1)));
  GRIFFIN_CUDA_TRY(w.tkstate.reserve(((size_t)nq + 1) * (1 + 8 + 4) + 64));
  if (topk_filter_on(ix, w, k) && w.entry_cap > kFiltMin && nq >= 2) {   // a query may exceed kFiltMin
    const size_t slots = std::min<size_t>(nq, kFiltSlots);
    GRIFFIN_CUDA_TRY(w.flt.reserve(slots * kFiltCap * 8));
    GRIFFIN_CUDA_TRY(w.fstate.reserve(((size_t)nq + 1) * 12 + slots * 4 + 64));
  }
  return GRIFFIN_OK;
}

// Bitvector slots of the terms eligible for kDecBitmap (griffin_set_bitmap):
// df_local * bm_inv >= shard docs; recomputed when the knob changes.
static griffin_status ensure_bm_slots(griffin_index *ix) {
  if (ix->bm_slots_inv == ix->bm_inv && (ix->d_bm_slot || !ix->bm_inv)) return GRIFFIN_OK;
  cudaFree(ix->d_bm_slot);
  cudaFree(ix->d_bm_term);
  ix->d_bm_slot = ix->d_bm_term = nullptr;
  ix->bm_nslots = 0;
  ix->bm_slots_inv = ix->bm_inv;
  if (!ix->bm_inv) return GRIFFIN_OK;
  const uint64_t nd = ix->doc_end - ix->doc_base;
  std::vector<uint32_t> slot(ix->V, kNone), term;
  for (uint32_t t = 0; t < ix->V; ++t) {
    const uint64_t df = ix->h_terms[t].df_local;
    if (df > 0 && df * ix->bm_inv >= nd) {
      slot[t] = (uint32_t)term.size();
      term.push_back(t);
    }
  }
  ix->bm_nslots = (uint32_t)term.size();
  GRIFFIN_CUDA_TRY(cudaMalloc(&ix->d_bm_slot, (size_t)ix->V * 4 + 4));
  GRIFFIN_CUDA_TRY(cudaMalloc(&ix->d_bm_term, term.size() * 4 + 4));
  GRIFFIN_CUDA_TRY(cudaMemcpy(ix->d_bm_slot, slot.data(), (size_t)ix->V * 4, cudaMemcpyHostToDevice));
  if (!term.empty())
    GRIFFIN_CUDA_TRY(cudaMemcpy(ix->d_bm_term, term.data(), term.size() * 4, cudaMemcpyHostToDevice));
  return GRIFFIN_OK;
}

griffin_status run_batch(griffin_index *ix, Workspace &w, uint32_t nq, const uint32_t *d_qoffs,
                         const uint32_t *d_terms, uint32_t max_terms, uint32_t k, uint64_t *d_keys,
                         uint32_t *d_counts, cudaStream_t st, bool final_topk, int forced_mode) {
  if (nq == 0) return GRIFFIN_OK;
  if (nq >= (1u << 29)) {   // unit order entries pack the query index in 29 bits
    set_error("a batch holds at most 2^29 - 1 queries");
    return GRIFFIN_ERR_INVALID_ARG;
  }
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
  ra.Tdec = ix->Tdec;
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
  ra.urec = w.urec.as<uint4>();
  ra.uperm = w.uperm.as<uint4>();
  ra.unit_cap = w.unit_cap;
  ra.bump = w.bump.as<uint2>();
  ra.entry_cap = w.entry_cap;
  ra.bump_cap = w.bump.bytes / 8 - 1;
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
        di, nq, w.plan_terms.as<uint32_t>(), w.plan_m.as<uint32_t>(), w.cap.as<uint32_t>(),
        probe_chunk(ix), scal);
    GRIFFIN_CUDA_TRY(cudaGetLastError());
  }
  // batch reuse: decode hot lists once into the arena (decompress-then-intersect)
  const bool reuse = ix->reuse == 1 || (ix->reuse == 2 && nq >= 8);
  ra.dec = nullptr;
  ra.tdec = nullptr;
  if (reuse && ix->V) {
    StageTimer t(ix, st, 5);
    const uint32_t V = ix->V;
    GRIFFIN_CUDA_TRY(w.demand.reserve((size_t)V * 4));
    GRIFFIN_CUDA_TRY(w.tdec.reserve(V));
    GRIFFIN_CUDA_TRY(w.runs.reserve((size_t)V * 4));
    GRIFFIN_CUDA_TRY(w.run_base.reserve(((size_t)V + 2) * 8));
    GRIFFIN_CUDA_TRY(w.vtmp.reserve(((size_t)V / kScanTile + 4) * 8));
    const uint32_t Dsw = sweep_D(ix->B);
    GRIFFIN_CUDA_TRY(w.run_term.reserve((ix->nblocks / (Dsw + 2) + (size_t)V + 2) * 4));
    GRIFFIN_CUDA_TRY(w.arena.reserve((ix->nblocks * ix->B + 64) * 4));
    // dense lists: bitvector slots (forced modes never read them)
    const bool bitmaps = ix->bm_inv && forced_mode == 0 && ix->h_terms.size() == V;
    const uint32_t bm_words = (ix->doc_end - ix->doc_base + 31u) / 32u;
    if (bitmaps) {
      griffin_status bs = ensure_bm_slots(ix);
      if (bs) return bs;
      GRIFFIN_CUDA_TRY(w.bmap.reserve((size_t)ix->bm_nslots * ((bm_words + 1u) & ~1u) * 8 + 16));
    }
    const bool use_bm = bitmaps && ix->bm_nslots > 0;
    GRIFFIN_CUDA_TRY(cudaMemsetAsync(w.demand.p, 0, (size_t)V * 4, st));
    ra.T = ix->T;
    demand_kernel<<<qblocks, 256, 0, st>>>(di, ra, w.demand.as<uint32_t>());
    select_kernel<<<(V + 255) / 256, 256, 0, st>>>(di, w.demand.as<uint32_t>(),
                                                   use_bm ? ix->d_bm_slot : nullptr,
                                                   w.tdec.as<uint8_t>(), w.runs.as<uint32_t>(),
                                                   Dsw + 2);
    if (use_bm) {
      // slots are padded to an even word count (uint4 zeroing)
      const uint32_t words = (bm_words + 1u) & ~1u;
      dim3 zg(std::max(1u, std::min(64u, (words / 2 + 255) / 256)), std::min(ix->bm_nslots, 1024u));
      bm_zero_kernel<<<zg, 256, 0, st>>>(w.tdec.as<uint8_t>(), ix->d_bm_term, ix->bm_nslots, words,
                                         w.bmap.as<uint4>());
      ix->launch_count += 1;
    }
    ra.bm = use_bm ? w.bmap.as<uint2>() : nullptr;
    ra.bm_slot = use_bm ? ix->d_bm_slot : nullptr;
    ra.bm_words = (bm_words + 1u) & ~1u;
    GRIFFIN_CUDA_TRY(exclusive_scan<uint32_t>(w.runs.as<uint32_t>(), w.run_base.as<uint64_t>(), V,
                                              w.vtmp.as<uint64_t>(), st, &ix->launch_count));
    run_map_kernel<<<(uint32_t)(((uint64_t)V * 32 + 255) / 256), 256, 0, st>>>(V, w.runs.as<uint32_t>(),
                                                    w.run_base.as<uint64_t>(),
                                                    w.run_term.as<uint32_t>());
    const size_t smem = kLutBytes + (size_t)warp_smem_words(ix->B, Dsw, false) * 4 * 8;
    int per_sm = 1;
    GRIFFIN_CUDA_TRY(launch_config((const void *)decode_once_kernel, ix->device, smem, 256, &per_sm));
    decode_once_kernel<<<num_sms(ix->device) * std::max(1, per_sm), 256, smem, st>>>(
        di, Dsw, w.run_base.as<uint64_t>(), w.run_term.as<uint32_t>(), w.arena.as<uint32_t>(),
        w.tdec.as<uint8_t>(), const_cast<uint2 *>(ra.bm), ra.bm_slot, ra.bm_words, scal);
    GRIFFIN_CUDA_TRY(cudaGetLastError());
    ix->launch_count += 4;
    ra.dec = w.arena.as<uint32_t>();
    ra.tdec = w.tdec.as<uint8_t>();
  }
  // multi-list probe replaces SvS rounds 2..m-1 (auto mode, B small enough for its smem)
  ra.probe = forced_mode == 0 && ix->probe && ix->D >= 5;
  ra.nextgeq = ix->nextgeq;
  ra.count = (ix->profiling & 2) ? 1 : 0;
  ra.pchunk = probe_chunk(ix);
  uint32_t rounds = std::max<uint32_t>(1, max_terms > 0 ? max_terms - 1 : 1);
  if (ra.probe) rounds = std::min<uint32_t>(rounds, 2);
  for (uint32_t r = 1; r <= rounds; ++r) {
    ra.round = r;
    ra.rprev = (r & 1) ? w.rbuf0.as<uint2>() : w.rbuf1.as<uint2>();
    ra.rnext = (r & 1) ? w.rbuf1.as<uint2>() : w.rbuf0.as<uint2>();
    ra.roff_prev = ra.cap_off + ((r - 1) & 1u) * ((size_t)nq + 1);
    ra.roff_next = ra.cap_off + (r & 1u) * ((size_t)nq + 1);
    {
      StageTimer t(ix, st, 0);
      plan_round_kernel<<<qblocks, 256, 0, st>>>(di, ra, qunits);
      GRIFFIN_CUDA_TRY(cudaGetLastError());
      GRIFFIN_CUDA_TRY(exclusive_scan<uint32_t>(qunits, w.unit_base.as<uint64_t>(), nq, scan_tmp, st,
                                                &ix->launch_count));
      ix->launch_count += 1;  // plan_round (the scan counts itself)
    }
    ra.qtau = nullptr;
    if (r == 1 && final_topk && ra.bm && k <= kTauKeys / 2 && nq >= std::max(8u, ix->tau_min_queries)) {
      // 2-term word-AND queries: their top-k key threshold from a subset of
      // their survivors (a top-k selection step: timed with the top-k stage;
      // large batches only — at C2's 1000 queries its launch costs more than
      // it saves: top-k 0.09 -> 0.20 ms, compaction 0.093 -> 0.082 ms)
      StageTimer tt(ix, st, 3);
      GRIFFIN_CUDA_TRY(w.qtau.reserve(((size_t)nq + 1) * 8));
      GRIFFIN_CUDA_TRY(launch_config((const void *)bitand_tau_kernel, ix->device, tau_smem_bytes(),
                                     1024, nullptr));
      bitand_tau_kernel<<<std::min<uint32_t>(nq, num_sms(ix->device) * 2), 1024, tau_smem_bytes(),
                          st>>>(di, ra, k, w.qtau.as<uint64_t>());
      GRIFFIN_CUDA_TRY(cudaGetLastError());
      ix->launch_count += 1;
      ra.qtau = w.qtau.as<uint64_t>();
    }
    {
      StageTimer t(ix, st, 1);
      const unsigned pgrid = num_sms(ix->device) * 8;
      ra.sbkt_cnt = nullptr;
      ra.sbkt_pos = nullptr;
      uint64_t nbkt = 0;
      // (the probe pass has no merge units; it orders its units by their first
      // remaining list's bitvector when that list has one)
      if (ix->sorder && nq >= kSorderMinQueries && (r == 1 || !ra.probe || ra.bm) && w.sbkt_cnt.p) {
        ra.sbkt_shift = ix->sorder_shift;
        ra.sbkt_nm = sorder_merge_buckets(ix);
        ra.sbkt_nbb = sorder_bm_per_slot(ix);
        // bitvector buckets only when this batch uses bitvectors and the buffers
        // (sized in reserve_ws) hold them; else those units join the tail
        const bool bmb = ra.bm && sorder_buckets(ix) * 4 <= w.sbkt_cnt.bytes &&
                         (sorder_buckets(ix) + 1) * 8 <= w.sbkt_pos.bytes;
        if (!bmb) ra.sbkt_nbb = 0;
        nbkt = bmb ? sorder_buckets(ix) : ra.sbkt_nm;
        GRIFFIN_CUDA_TRY(cudaMemsetAsync(w.sbkt_cnt.p, 0, nbkt * 4, st));
        ra.sbkt_cnt = w.sbkt_cnt.as<uint32_t>();
        ra.sbkt_pos = w.sbkt_pos.as<unsigned long long>();
      }
      if (r == 1) partition_kernel<true><<<pgrid, 256, 0, st>>>(di, ra);
      else partition_kernel<false><<<pgrid, 256, 0, st>>>(di, ra);
      if (ra.sbkt_cnt) {
        GRIFFIN_CUDA_TRY(exclusive_scan<uint32_t>(ra.sbkt_cnt, w.sbkt_pos.as<uint64_t>(), nbkt,
                                                  w.sbkt_tmp.as<uint64_t>(), st,
                                                  &ix->launch_count));
        if (r == 1) sorder_scatter_kernel<true><<<pgrid, 256, 0, st>>>(di, ra);
        else sorder_scatter_kernel<false><<<pgrid, 256, 0, st>>>(di, ra);
        ix->launch_count += 1;
      }
      if (r == 1) {   // merge units, then gallop / single-term units
        GRIFFIN_CUDA_TRY((launch_intersect<true, 1>(ix, ra, st)));
        GRIFFIN_CUDA_TRY((launch_intersect<true, 2>(ix, ra, st)));
        ix->launch_count += 1;
      } else if (ra.probe) {
        GRIFFIN_CUDA_TRY(launch_probe(ix, ra, st));   // all units are probe units
      } else {
        GRIFFIN_CUDA_TRY((launch_intersect<false, 0>(ix, ra, st)));
      }
      ix->launch_count += 2;  // partition + intersect
    }
    {
      StageTimer t(ix, st, 2);
      const uint64_t *n_dev = w.unit_base.as<uint64_t>() + nq;
      const unsigned tiles = (unsigned)(w.unit_cap / kScanTile + 1);
      uint64_t *tsum = w.unit_dst.as<uint64_t>() + (w.unit_cap + 2);
      const unsigned sgrid = std::min<unsigned>(tiles, num_sms(ix->device) * 2);
      unit_scan_sums<<<sgrid, kScanThreads, 0, st>>>(ra.unit_cnt, n_dev, tsum, tiles);
      scan_single_kernel<uint64_t><<<1, kScanThreads, 0, st>>>(tsum, tsum, tiles,
                                                               reinterpret_cast<uint64_t *>(scal + kScalRoundTot));
      unit_scan_apply<<<sgrid, kScanThreads, 0, st>>>(ra.unit_cnt, n_dev, tsum,
                                                      w.unit_dst.as<uint64_t>(), tiles);
      compact_copy_kernel<<<num_sms(ix->device) * 8, 256, 0, st>>>(ra, w.unit_dst.as<uint64_t>());
      if (r <= 2) {
        compact_queries_kernel<<<qblocks, 256, 0, st>>>(ra, w.unit_dst.as<uint64_t>());
        ix->launch_count += 1;
      }
      GRIFFIN_CUDA_TRY(cudaGetLastError());
      ix->launch_count += 4;  // sums, single, apply, copy
    }
  }
  if (final_topk) {
    StageTimer t(ix, st, 3);
    uint32_t *nch = qunits;  // reuse the per-query unit-count scratch
    uint64_t *cbase = w.unit_base.as<uint64_t>();
    // candidates per level <= (entries / kTopkSmem + nq + 1) * k (each level shrinks them
    // by kTopkSmem / k; small k needs 2 levels, large k up to kTopkMaxLevels)
    const uint64_t cand_cap = (w.entry_cap / kTopkSmem + nq + 1) * (uint64_t)k;
    const int levels = k <= 64 ? 1 : (k <= 1024 ? 4 : (k <= 2048 ? kTopkMaxLevels : 0));
    griffin_status rs_ = reserve_topk(ix, w, nq, k);
    if (rs_) return rs_;
    CandBufs cb{};
    for (int L = 1; L <= levels; ++L) cb.lv[L] = w.cand.as<uint64_t>() + (size_t)(L - 1) * cand_cap;
    TopkState ts;
    ts.qoff = w.tkstate.as<uint64_t>();
    ts.qn = reinterpret_cast<uint32_t *>(ts.qoff + nq + 1);
    ts.qlev = reinterpret_cast<uint8_t *>(ts.qn + nq + 1);
    ts.fmax = 0;
    // for k > 64 (one chunk level keeps k of kTopkSmem keys, so large k needs
    // up to 4 levels over shrinking-by-4x sets; C5 top-1000: 3.12 -> 1.29 ms);
    // for k <= 64 one level already shrinks 64x and the extra launches cost more
    if (topk_filter_on(ix, w, k) && w.flt.p && w.fstate.p && nq >= 2) {
      ts.fmax = (uint32_t)std::min<size_t>(w.flt.bytes / (kFiltCap * 8), kFiltSlots);
      ts.flt = w.flt.as<uint64_t>();
      ts.ftau = w.fstate.as<uint64_t>();
      ts.fslot = reinterpret_cast<uint32_t *>(ts.ftau + nq + 1);
      ts.fctr = ts.fslot + nq + 1;
      ts.fcnt = ts.fctr + 1;
      if ((size_t)(nq + 1) * 12 + 8 + (size_t)ts.fmax * 4 > w.fstate.bytes) ts.fmax = 0;
    }
    const uint32_t *rc = w.rcount.as<uint32_t>();
    const uint8_t *rs = w.rsel.as<uint8_t>();
    topk_init_kernel<<<qblocks, 256, 0, st>>>(nq, rc, ts);
    ix->launch_count += 1;
    if (ts.fmax) {
      topk_sample_kernel<<<std::min<uint32_t>(nq, num_sms(ix->device) * 4), kTopkThreads, 0, st>>>(
          di, nq, k, rs, w.cap_off.as<uint64_t>(), w.rbuf0.as<uint2>(), w.rbuf1.as<uint2>(), ts);
      topk_filter_plan_kernel<<<qblocks, 256, 0, st>>>(nq, ts, nch);
      GRIFFIN_CUDA_TRY(exclusive_scan<uint32_t>(nch, cbase, nq, scan_tmp, st, &ix->launch_count));
      topk_filter_kernel<<<num_sms(ix->device) * 8, 256, 0, st>>>(
          di, nq, rs, w.cap_off.as<uint64_t>(), w.rbuf0.as<uint2>(), w.rbuf1.as<uint2>(), ts, cbase);
      topk_filter_update_kernel<<<qblocks, 256, 0, st>>>(nq, k, ts);
      GRIFFIN_CUDA_TRY(cudaGetLastError());
      ix->launch_count += 4;
    }
    for (int L = 1; L <= levels; ++L) {
      topk_plan_kernel<<<qblocks, 256, 0, st>>>(nq, ts, nch);
      GRIFFIN_CUDA_TRY(exclusive_scan<uint32_t>(nch, cbase, nq, scan_tmp, st, &ix->launch_count));
      topk_chunk_kernel<<<num_sms(ix->device) * 4, kTopkThreads, 0, st>>>(
          di, nq, k, rs, w.cap_off.as<uint64_t>(), w.rbuf0.as<uint2>(), w.rbuf1.as<uint2>(), ts,
          cb, cbase, cb.lv[L]);
      topk_update_kernel<<<qblocks, 256, 0, st>>>(nq, k, L, ts, nch, cbase);
      ix->launch_count += 3;
    }
    topk_final_kernel<<<std::min<uint32_t>(nq, num_sms(ix->device) * 4), kTopkThreads, 0, st>>>(
        di, nq, k, rc, rs, w.cap_off.as<uint64_t>(), w.rbuf0.as<uint2>(), w.rbuf1.as<uint2>(), ts,
        cb, d_keys, d_counts);
    GRIFFIN_CUDA_TRY(cudaGetLastError());
    ix->launch_count += 1;
  }
  return GRIFFIN_OK;
}

griffin_status launch_merge_topk(griffin_index *ix, uint32_t G, uint32_t nq, uint32_t k,
                                 const uint64_t *d_keys, const uint32_t *d_counts,
                                 uint64_t *d_out_keys, uint32_t *d_out_counts, cudaStream_t st) {
  if (nq == 0) return GRIFFIN_OK;
  StageTimer t(ix, st, 4);
  ix->launch_count += 1;
  merge_topk_kernel<<<std::min<uint32_t>((nq + 7) / 8, num_sms(ix->device) * 16), 256, 0, st>>>(
      G, nq, k, d_keys, d_counts, d_out_keys, d_out_counts);
  GRIFFIN_CUDA_TRY(cudaGetLastError());
  return GRIFFIN_OK;
}

griffin_status launch_merge_topk_peer(griffin_index *ix, uint32_t G, uint32_t nq, uint32_t k,
                                      const uint64_t *const *keys, const uint32_t *const *counts,
                                      uint64_t *d_out_keys, uint32_t *d_out_counts,
                                      cudaStream_t st) {
  if (nq == 0) return GRIFFIN_OK;
  if (G == 0 || G > GRIFFIN_MAX_SHARDS) {
    set_error("peer merge: 1..8 runs");
    return GRIFFIN_ERR_INVALID_ARG;
  }
  PeerRuns r{};
  for (uint32_t g = 0; g < G; ++g) {
    r.keys[g] = keys[g];
    r.counts[g] = counts[g];
  }
  ix->launch_count += 1;
  merge_topk_peer_kernel<<<std::min<uint32_t>((nq + 7) / 8, num_sms(ix->device) * 16), 256, 0, st>>>(
      G, nq, k, r, d_out_keys, d_out_counts);
  GRIFFIN_CUDA_TRY(cudaGetLastError());
  return GRIFFIN_OK;
}

griffin_status launch_keys_to_results(griffin_index *ix, uint32_t nq, uint32_t k,
                                      const uint64_t *d_keys, const uint32_t *d_counts,
                                      uint32_t *d_docids, float *d_scores, cudaStream_t st) {
  const uint64_t n = (uint64_t)nq * k;
  if (!n) return GRIFFIN_OK;
  ix->launch_count += 1;
  keys_to_results_kernel<<<(unsigned)std::min<uint64_t>((n + 255) / 256, (uint64_t)num_sms(ix->device) * 32), 256, 0, st>>>(
      nq, k, d_keys, d_counts, d_docids, d_scores);
  GRIFFIN_CUDA_TRY(cudaGetLastError());
  return GRIFFIN_OK;
}

griffin_status launch_decode_list(griffin_index *ix, uint32_t term, uint32_t *d_out,
                                  cudaStream_t st) {
  const TermInfo &t = ix->h_terms[term];
  if (!t.nblocks) return GRIFFIN_OK;
  const size_t smem = kLutBytes + (size_t)warp_smem_words(ix->B, ix->D) * 4 * 8;
  GRIFFIN_CUDA_TRY(launch_config((const void *)decode_list_kernel, ix->device, smem, 256, nullptr));
  const uint32_t runs = (t.nblocks + ix->D + 1) / (ix->D + 2);
  decode_list_kernel<<<std::min<uint32_t>((runs + 7) / 8, num_sms(ix->device) * 8), 256, smem, st>>>(
      ix->dev(), ix->D, t.block0, t.nblocks, d_out);
  GRIFFIN_CUDA_TRY(cudaGetLastError());
  return GRIFFIN_OK;
}

griffin_status launch_decode_all(griffin_index *ix, unsigned long long *d_acc, cudaStream_t st) {
  if (!ix->nblocks) return GRIFFIN_OK;
  const uint32_t Dsw = sweep_D(ix->B);
  const size_t smem = kLutBytes + (size_t)warp_smem_words(ix->B, Dsw, false) * 4 * 8;
  int per_sm = 1;
  GRIFFIN_CUDA_TRY(launch_config((const void *)decode_all_kernel, ix->device, smem, 256, &per_sm));
  ix->launch_count += 1;
  decode_all_kernel<<<num_sms(ix->device) * std::max(1, per_sm), 256, smem, st>>>(
      ix->dev(), Dsw, ix->nblocks, d_acc);
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
  GRIFFIN_CUDA_TRY(cudaStreamSynchronize(st));   // sel picks the offset array
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(&off, w.cap_off.as<uint64_t>() + (sel ? 2 : 0), 8,
                                   cudaMemcpyDeviceToHost, st));
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

// Workspace bounds of one query (host): cap = entries of its round-1 region,
// units = an upper bound of its units in any round.  `ts` = its distinct terms
// (any order, all < V, 1..kMaxTerms of them); sorted here into SvS order.
void host_query_bounds(const griffin_index *ix, uint32_t *ts, uint32_t n, uint64_t *cap,
                       uint64_t *units) {
  *cap = 0;
  *units = 0;
  auto less = [&](uint32_t a, uint32_t b) {
    const uint32_t da = ix->h_terms[a].df_global, db = ix->h_terms[b].df_global;
    return da != db ? da < db : a < b;
  };
  for (uint32_t i = 1; i < n; ++i) {   // insertion sort: n <= kMaxTerms
    const uint32_t x = ts[i];
    uint32_t j = i;
    for (; j > 0 && less(x, ts[j - 1]); --j) ts[j] = ts[j - 1];
    ts[j] = x;
  }
  for (uint32_t i = 0; i < n; ++i)
    if (ix->h_terms[ts[i]].df_local == 0) return;
  const TermInfo &t0 = ix->h_terms[ts[0]];
  if (n == 1) {
    *cap = t0.df_local;
    *units = t0.nblocks;
    return;
  }
  *cap = std::min(t0.df_local, ix->h_terms[ts[1]].df_local);
  uint32_t mx = 0;
  for (uint32_t i = 1; i < n; ++i) mx = std::max(mx, ix->h_terms[ts[i]].nblocks);
  const uint32_t P = probe_chunk(ix);   // probe-pass units: ceil(|R| / P), |R| <= cap
  if (n >= 3) mx = std::max<uint32_t>(mx, (uint32_t)((*cap + P - 1) / P));
  *units = (uint64_t)t0.nblocks + mx;
}

}  // namespace griffin
