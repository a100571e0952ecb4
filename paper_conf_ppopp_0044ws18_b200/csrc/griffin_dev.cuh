// griffin_dev.cuh — device-side data layout and warp-level building blocks of
// the Griffin-GPU path on sm_100a.  Product code: shares nothing with oracle/.
//
// HBM layout of one shard:
//   terms[V]      TermInfo (32 B): first block, #blocks, local/global df, idf, tf stream
//   first[nb]     u32   first (local) docID of each block      — skip pointers, Fig. 2
//   meta[nb]      uint2 {payload offset /16 B, b | (n-1)<<5 | hw<<15}
//   payload       per block: low stream (n*b bits) then high stream (hw words),
//                 LSB-first u32 words, each block padded to 16 B
//   tfw           per term, tf-1 packed at width w_t
//   norm[n_docs]  f32 k1*((1-b)+b*dl/avgdl), host-computed in double (A14)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace griffin {

constexpr uint32_t kNone = 0xFFFFFFFFu;
constexpr int kWarp = 32;
constexpr int kMaxTerms = 16;

struct TermInfo {
  uint32_t block0;     // global block index of the term's first block in this shard
  uint32_t nblocks;
  uint32_t df_local;   // postings in this shard
  uint32_t df_global;  // postings in the whole corpus (SvS order + idf)
  float idf;
  uint32_t tf_w;       // tf bit width
  uint64_t tf_off;     // first u32 word of the term's packed tf stream
};
static_assert(sizeof(TermInfo) == 32, "TermInfo is one 32-B sector");

struct DevIndex {
  const TermInfo *terms;
  const uint32_t *first;
  const uint2 *meta;
  const uint4 *payload;
  const uint32_t *tfw;
  const float *norm;
  uint32_t num_terms;
  uint32_t doc_base;
  uint32_t n_docs;      // docs in this shard
  uint32_t B;           // block size
  uint32_t log2B;
  float k1p1;
};

// ---- meta packing -------------------------------------------------------------
__host__ __device__ inline uint32_t meta_b(uint32_t y) { return y & 31u; }
__host__ __device__ inline uint32_t meta_n(uint32_t y) { return ((y >> 5) & 1023u) + 1u; }
__host__ __device__ inline uint32_t meta_hw(uint32_t y) { return (y >> 15) & 255u; }
__host__ __device__ inline uint32_t meta_pack(uint32_t b, uint32_t n, uint32_t hw) {
  return b | ((n - 1u) << 5) | (hw << 15);
}
__host__ __device__ inline uint32_t low_words(uint32_t n, uint32_t b) { return (n * b + 31u) >> 5; }

// ---- lane helpers -------------------------------------------------------------
__device__ __forceinline__ uint32_t lane_id() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%laneid;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint4 ldg_nc_v4(const uint4 *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

// Warp inclusive scan (shuffle, Kogge-Stone) — the prefix sum of Alg. 1 l.3.
__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t v) {
  const uint32_t lane = lane_id();
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t t = __shfl_up_sync(0xffffffffu, v, d);
    if (lane >= (uint32_t)d) v += t;
  }
  return v;
}

// ---- shared memory / async-proxy primitives (sm_90+; TMA bulk copies) -----------
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
// order this thread's earlier generic-proxy smem accesses before later async-proxy writes
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
// 1-D TMA bulk copy global -> shared (16-B aligned, size multiple of 16)
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
          "r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t phase) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tWAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}

// ---- select-in-word (the shared-memory look-up table of) --------------
// lut[v*8 + r] = bit position of the r-th one of byte v.  Built once per CTA.
__device__ __forceinline__ void build_select_lut(uint8_t *lut) {
  for (uint32_t v = threadIdx.x; v < 256; v += blockDim.x) {
    uint32_t r = 0;
    for (uint32_t bit = 0; bit < 8; ++bit)
      if ((v >> bit) & 1u) lut[v * 8 + r++] = (uint8_t)bit;
    for (; r < 8; ++r) lut[v * 8 + r] = 0;
  }
}
// position of the r-th (0-based) one of x; requires r < popc(x)
__device__ __forceinline__ uint32_t select_in_word(uint32_t x, uint32_t r, const uint8_t *lut) {
  const uint32_t c1 = __popc(x & 0xFFu), c2 = __popc(x & 0xFFFFu), c3 = __popc(x & 0xFFFFFFu);
  uint32_t sh = 0, base = 0;
  if (r >= c1) { sh = 8; base = c1; }
  if (r >= c2) { sh = 16; base = c2; }
  if (r >= c3) { sh = 24; base = c3; }
  return sh + lut[((x >> sh) & 0xFFu) * 8u + (r - base)];
}

// ---- decoder output sinks -------------------------------------------------------
// StoreSink writes decoded docIDs (smem tile or HBM arena); XorSink folds them
// into a register checksum (the decode-only sweep: nothing is written back).
struct StoreSink {
  __device__ __forceinline__ void put4(uint32_t *p, uint4 v) { *reinterpret_cast<uint4 *>(p) = v; }
  __device__ __forceinline__ void put(uint32_t *p, uint32_t v) { *p = v; }
};
struct XorSink {
  uint32_t x = 0;
  __device__ __forceinline__ void put4(uint32_t *, uint4 v) { x ^= v.x ^ v.y ^ v.z ^ v.w; }
  __device__ __forceinline__ void put(uint32_t *, uint32_t v) { x ^= v; }
};
// BitSink writes a list's decoded docIDs into its bitvector with rank: word
// w = {bits of docs [32w, 32w+32), ~(list position of the word's first
// posting)} (the rank is only read where a bit is set).  The decoder hands
// each lane its elements in list order; a lane ORs a run of elements that
// share a word into a register and writes the word once.  A run whose
// neighbours on both sides were decoded by this lane, in other words, owns
// the word outright (plain 64-bit store); any other run may share its word
// with another lane: atomicOr for the bits, atomicMax of ~position (= the
// smallest position) for the rank — the area is zeroed first.  Positions come
// from the output pointer: the decoder writes element i of the run at tile + i.
struct BitSink {
  uint2 *bm;              // the list's bitvector
  const uint32_t *tile;   // decoder destination base
  uint32_t pos0;          // list position of tile[0]
  uint32_t cw = 0xFFFFFFFFu, bits = 0, fpos = 0, lpos = 0xFFFFFFFEu;
  bool cf = false;        // the run's predecessor was seen here (in another word)
  // flush the current run if `fl`; cl = its successor was seen here.  Written
  // as predicated code: lanes break runs at different elements, so a branch
  // would serialise the flush for almost every element of a warp.
  __device__ __forceinline__ void flush_if(bool fl, bool cl) {
    const bool own = fl && cf && cl;
    if (own) bm[cw] = make_uint2(bits, ~fpos);
    if (fl && !own) {
      atomicOr(&bm[cw].x, bits);
      atomicMax(&bm[cw].y, ~fpos);
    }
  }
  // element v at list position pos; contig = pos follows the previous element
  __device__ __forceinline__ void add(uint32_t pos, uint32_t v, bool contig) {
    const uint32_t w = v >> 5;
    const bool brk = w != cw || !contig;
    flush_if(brk && cw != 0xFFFFFFFFu, contig);
    cf = brk ? contig : cf;
    fpos = brk ? pos : fpos;
    bits = (brk ? 0u : bits) | (1u << (v & 31u));
    cw = w;
  }
  __device__ __forceinline__ void put4(uint32_t *p, uint4 v) {
    const uint32_t pos = pos0 + (uint32_t)(p - tile);
    const bool c0 = pos == lpos + 1u;   // the four are consecutive positions
    add(pos, v.x, c0);
    add(pos + 1u, v.y, true);
    add(pos + 2u, v.z, true);
    add(pos + 3u, v.w, true);
    lpos = pos + 3u;
  }
  __device__ __forceinline__ void put(uint32_t *p, uint32_t v) {
    const uint32_t pos = pos0 + (uint32_t)(p - tile);
    add(pos, v, pos == lpos + 1u);
    lpos = pos;
  }
  // end of this lane's elements: its last run may share its word
  __device__ __forceinline__ void finish() {
    flush_if(cw != 0xFFFFFFFFu, false);
    cw = 0xFFFFFFFFu;
    lpos = 0xFFFFFFFEu;   // the next element never continues this run
  }
};
// Bitvector lookup of docID x: its list position, or kNone if absent.
__device__ __forceinline__ uint32_t bitvec_pos(uint2 w, uint32_t x) {
  const uint32_t bit = x & 31u;
  return ((w.x >> bit) & 1u) ? ~w.y + __popc(w.x & ((1u << bit) - 1u)) : 0xFFFFFFFFu;
}

// ---- eight consecutive elements of a staged block (one lane) ----------------------
// Elements k .. k+ne-1 (ne <= 8) given p = the high-stream position of element
// k's one and `win` = the 32 high-stream bits after it.  The ones of elements
// k+1..k+4 come from `win`; a fresh window read right after element k+4's one
// gives k+5..k+7, so a run of zeros inside one 32-bit window (likely when the
// high stream is sparse, u/2^b ~ 2n) does not force the slow path.  Low bits by
// funnel shifts of the staged low stream (one window covers all eight when
// b <= 4, two when b <= 8).  Falls back to a serial walk when a window lacks
// ones (only near the end of a partial block).  Returns the position of the
// last decoded element's one (valid when ne == 8 and the fast path ran).
template <class Sink>
__device__ __forceinline__ uint32_t decode8(const uint32_t *__restrict__ stg,
                                            const uint32_t *__restrict__ hs, uint32_t first,
                                            uint32_t b, uint32_t mask, uint32_t k, uint32_t ne,
                                            uint32_t p, uint32_t win, uint32_t *dst, Sink &sink) {
  uint32_t w1 = win;
  const uint32_t t1 = __ffs(w1);
  w1 &= w1 - 1u;
  const uint32_t t2 = __ffs(w1);
  w1 &= w1 - 1u;
  const uint32_t t3 = __ffs(w1);
  w1 &= w1 - 1u;
  const uint32_t t4 = __ffs(w1);
  const uint32_t p4 = p + t4;   // element k+4's one
  const uint32_t wb = p4 + 1u;
  const uint32_t win2 = __funnelshift_r(hs[wb >> 5], hs[(wb >> 5) + 1], wb);
  uint32_t w2 = win2;
  const uint32_t s1 = __ffs(w2);
  w2 &= w2 - 1u;
  const uint32_t s2 = __ffs(w2);
  w2 &= w2 - 1u;
  const uint32_t s3 = __ffs(w2);
  const bool ok = (ne <= 1u || __popc(win) >= min(ne - 1u, 4u)) &&
                  (ne <= 5u || __popc(win2) >= ne - 5u);
  if (ok) {
    uint32_t hv[8];
    hv[0] = p - k;
    hv[1] = p + t1 - (k + 1u);
    hv[2] = p + t2 - (k + 2u);
    hv[3] = p + t3 - (k + 3u);
    hv[4] = p4 - (k + 4u);
    hv[5] = p4 + s1 - (k + 5u);
    hv[6] = p4 + s2 - (k + 6u);
    hv[7] = p4 + s3 - (k + 7u);
    uint32_t lv[8];
    const uint32_t bp = k * b;
    if (b <= 4u) {
      const uint32_t lw32 = __funnelshift_r(stg[bp >> 5], stg[(bp >> 5) + 1], bp);
#pragma unroll
      for (uint32_t j = 0; j < 8; ++j) lv[j] = (lw32 >> (j * b)) & mask;
    } else if (b <= 8u) {
      const uint32_t q = bp + 4u * b;
      const uint32_t x1 = __funnelshift_r(stg[bp >> 5], stg[(bp >> 5) + 1], bp);
      const uint32_t x2 = __funnelshift_r(stg[q >> 5], stg[(q >> 5) + 1], q);
#pragma unroll
      for (uint32_t j = 0; j < 4; ++j) {
        lv[j] = (x1 >> (j * b)) & mask;
        lv[j + 4] = (x2 >> (j * b)) & mask;
      }
    } else if (b <= 16u) {
      // two low fields per 32-bit window (most postings of the C2/C5 indexes
      // have b in 9..16): half the shared loads and address math of one
      // window per element
#pragma unroll
      for (uint32_t j = 0; j < 8; j += 2) {
        const uint32_t q = bp + j * b;
        const uint32_t x = __funnelshift_r(stg[q >> 5], stg[(q >> 5) + 1], q);
        lv[j] = x & mask;
        lv[j + 1] = (x >> b) & mask;
      }
    } else {
#pragma unroll
      for (uint32_t j = 0; j < 8; ++j) {
        const uint32_t q = bp + j * b;
        lv[j] = __funnelshift_r(stg[q >> 5], stg[(q >> 5) + 1], q) & mask;
      }
    }
    uint32_t v[8];
#pragma unroll
    for (uint32_t j = 0; j < 8; ++j) v[j] = first + ((hv[j] << b) | lv[j]);
    if (ne == 8u) {
      sink.put4(dst + k, make_uint4(v[0], v[1], v[2], v[3]));
      sink.put4(dst + k + 4, make_uint4(v[4], v[5], v[6], v[7]));
    } else {
#pragma unroll
      for (uint32_t j = 0; j < 8; ++j)
        if (j < ne) sink.put(dst + k + j, v[j]);
    }
    return p4 + s3;
  }
  // serial walk with a refilled 32-bit window
  uint32_t wbb = p + 1u, ww = win, pp = p, bp = k * b;
  for (uint32_t j = 0; j < ne; ++j) {
    if (j) {
      while (ww == 0u) {
        wbb += 32u;
        ww = __funnelshift_r(hs[wbb >> 5], hs[(wbb >> 5) + 1], wbb);
      }
      pp = wbb + (__ffs(ww) - 1u);
      ww &= ww - 1u;
    }
    const uint32_t lo_bits = __funnelshift_r(stg[bp >> 5], stg[(bp >> 5) + 1], bp) & mask;
    sink.put(dst + k + j, first + (((pp - (k + j)) << b) | lo_bits));
    bp += b;
  }
  return pp;
}

// ---- Elias-Fano block decode (Para-EF, §3.1.1 / Alg. 1) -------------
// One warp decodes one block of n <= B postings, already staged in shared memory
// (low stream: lw words, then high stream: hw words), into dst[0..n) as absolute
// local docIDs x_k = first + ((h_k << b) | low_k).
//  * Alg. 1 l.2-3: lane w popcounts high word w; a warp shuffle scan gives the
//    inclusive prefix counts (the "synchronization point").
//  * Alg. 1 l.4-8 (scheduling): instead of scattering word ids element by
//    element, lane l owns the E = ceil(n/32) consecutive elements k0 = l*E ...;
//    it binary-searches the prefix counts for the word holding element k0 and
//    selects the bit with the byte LUT.
//  * Alg. 1 l.9-10: the following E-1 ones are the next set bits (clear-lowest +
//    find-first-set); h_k = p_k - k (the zeros before the k-th one);
//    the b low bits are funnel-shifted out of the staged low stream.
// `cnt` is per-warp smem scratch of >= 64 u32.
template <class Sink>
__device__ __forceinline__ void warp_decode_staged(const uint32_t *__restrict__ stg, uint32_t first,
                                                   uint32_t y, uint32_t *__restrict__ dst,
                                                   uint32_t *__restrict__ cnt,
                                                   const uint8_t *__restrict__ lut, Sink &sink) {
  const uint32_t lane = lane_id();
  const uint32_t b = meta_b(y), n = meta_n(y), hw = meta_hw(y);
  const uint32_t lw = low_words(n, b);
  const uint32_t *hs = stg + lw;
  const uint32_t w0 = lane < hw ? hs[lane] : 0u;
  const uint32_t c0 = __popc(w0);
  const uint32_t i0 = warp_incl_scan(c0);
  const uint32_t E = (n + 31u) >> 5;
  const uint32_t k0 = lane * E;
  uint32_t w, x, ex, nx;
  if (hw <= 32 && (E & (E - 1u)) == 0) {
    // Owner of element k0 without a search: word w holds elements
    // [excl_w, incl_w), i.e. the targets of lanes [ceil(excl_w/E), ceil(incl_w/E)).
    // Mark each such range's first lane with w+1, then an inclusive max-scan
    // hands every lane its owner word.
    const uint32_t lgE = __ffs(E) - 1u;
    const uint32_t ex0 = i0 - c0;
    const uint32_t a = (ex0 + E - 1u) >> lgE, bnd = (i0 + E - 1u) >> lgE;
    cnt[lane] = 0u;
    __syncwarp();
    if (lane < hw && a < bnd && a < 32u) cnt[a] = lane + 1u;
    __syncwarp();
    uint32_t v = cnt[lane];
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, v, d);
      if (lane >= (uint32_t)d) v = max(v, t);
    }
    w = v ? v - 1u : 0u;
    x = __shfl_sync(0xffffffffu, w0, w);
    ex = __shfl_sync(0xffffffffu, ex0, w);
    nx = __shfl_sync(0xffffffffu, w0, (w + 1u) & 31u);
    if (w + 1u >= hw) nx = 0u;
  } else {
    cnt[lane] = i0;
    if (hw > 32) {
      const uint32_t w1 = lane + 32 < hw ? hs[lane + 32] : 0u;
      cnt[lane + 32] = __shfl_sync(0xffffffffu, i0, 31) + warp_incl_scan(__popc(w1));
    }
    __syncwarp();
    // word holding element k0: smallest w with cnt[w] > k0
    uint32_t lo = 0, hi = hw - 1;
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      if (cnt[mid] > k0) hi = mid; else lo = mid + 1;
    }
    w = lo;
    x = hs[w];
    ex = w ? cnt[w - 1] : 0u;
    nx = hs[w + 1];
  }
  if (k0 < n) {
    const uint32_t ne = min(E, n - k0);
    const uint32_t pos = select_in_word(x, k0 - ex, lut);
    const uint32_t p0 = (w << 5) + pos;
    // the 32 bits following element k0's one (clamped funnel: pos+1 may be 32)
    uint32_t win = __funnelshift_rc(x, nx, pos + 1u);
    const uint32_t mask = b ? (0xFFFFFFFFu >> (32u - b)) : 0u;
    if (E == 8 || E == 16) {   // B = 256 / 512: runs of eight (decode8)
      const uint32_t p7 = decode8(stg, hs, first, b, mask, k0, min(8u, ne), p0, win, dst, sink);
      if (ne > 8u) {   // second run: element k0+8's one is the next one after p7
        uint32_t wb = p7 + 1u;
        uint32_t w8 = __funnelshift_r(hs[wb >> 5], hs[(wb >> 5) + 1], wb);
        while (w8 == 0u) {
          wb += 32u;
          w8 = __funnelshift_r(hs[wb >> 5], hs[(wb >> 5) + 1], wb);
        }
        const uint32_t p8 = wb + (__ffs(w8) - 1u);
        decode8(stg, hs, first, b, mask, k0 + 8u, ne - 8u, p8,
                __funnelshift_r(hs[(p8 + 1u) >> 5], hs[((p8 + 1u) >> 5) + 1], p8 + 1u), dst, sink);
      }
    } else if (E == 4 && ne == 4 && __popc(win) >= 3u) {
      // fast path (B = 128): the next three ones are inside the window
      const uint32_t t1 = __ffs(win);
      win &= win - 1u;
      const uint32_t t2 = __ffs(win);
      win &= win - 1u;
      const uint32_t t3 = __ffs(win);
      const uint32_t h0 = p0 - k0, h1 = p0 + t1 - (k0 + 1), h2 = p0 + t2 - (k0 + 2),
                     h3 = p0 + t3 - (k0 + 3);
      uint32_t l0, l1, l2, l3;
      const uint32_t bp = k0 * b;
      if (b <= 8) {  // all four low fields inside one 32-bit window
        const uint32_t lw32 = __funnelshift_r(stg[bp >> 5], stg[(bp >> 5) + 1], bp);
        l0 = lw32 & mask;
        l1 = (lw32 >> b) & mask;
        l2 = (lw32 >> (2 * b)) & mask;
        l3 = (lw32 >> (3 * b)) & mask;
      } else {
        uint32_t q = bp;
        l0 = __funnelshift_r(stg[q >> 5], stg[(q >> 5) + 1], q) & mask;
        q += b;
        l1 = __funnelshift_r(stg[q >> 5], stg[(q >> 5) + 1], q) & mask;
        q += b;
        l2 = __funnelshift_r(stg[q >> 5], stg[(q >> 5) + 1], q) & mask;
        q += b;
        l3 = __funnelshift_r(stg[q >> 5], stg[(q >> 5) + 1], q) & mask;
      }
      sink.put4(dst + k0, make_uint4(first + ((h0 << b) | l0), first + ((h1 << b) | l1),
                                     first + ((h2 << b) | l2), first + ((h3 << b) | l3)));
    } else {
      // generic path: walk the ones with a 32-bit window, refilling when empty
      uint32_t wb = p0 + 1u;  // absolute bit position of win's bit 0
      uint32_t p = p0;
      uint32_t bp = k0 * b;
      for (uint32_t j = 0; j < ne; ++j) {
        if (j) {
          while (win == 0u) {
            wb += 32u;
            win = __funnelshift_r(hs[wb >> 5], hs[(wb >> 5) + 1], wb);
          }
          p = wb + (__ffs(win) - 1u);
          win &= win - 1u;
        }
        const uint32_t lo_bits = __funnelshift_r(stg[bp >> 5], stg[(bp >> 5) + 1], bp) & mask;
        sink.put(dst + k0 + j, first + (((p - (k0 + j)) << b) | lo_bits));
        bp += b;
      }
    }
  }
  __syncwarp();
}

// ---- two blocks per warp (B = 128) ----------------------------------------------
// The per-block fixed work of warp_decode_staged (prefix scan of the high words,
// owner search, select) costs as much as its per-element work at B = 128; here
// each half-warp runs the same algorithm on its own block with 16 lanes x 8
// consecutive elements (width-16 shuffles), so one instruction stream decodes
// two blocks.  Requires n <= 128 (hence hw <= 12 <= 16 high words) for both.
// Block B is skipped when has_b is false.  dst pointers 16-B aligned.
template <class Sink>
__device__ __forceinline__ void warp_decode_pair_staged(
    const uint32_t *stg_a, uint32_t first_a, uint32_t y_a, uint32_t *dst_a,
    const uint32_t *stg_b, uint32_t first_b, uint32_t y_b, uint32_t *dst_b, bool has_b,
    uint32_t *__restrict__ cnt, const uint8_t *__restrict__ lut, Sink &sink) {
  const uint32_t lane = lane_id(), hf = lane >> 4, l = lane & 15u;
  const bool act = hf == 0 || has_b;
  const uint32_t *stg = hf ? stg_b : stg_a;
  const uint32_t first = hf ? first_b : first_a;
  const uint32_t y = hf ? y_b : y_a;
  uint32_t *dst = hf ? dst_b : dst_a;
  const uint32_t b = meta_b(y), n = act ? meta_n(y) : 0u, hw = act ? meta_hw(y) : 0u;
  const uint32_t *hs = stg + low_words(n, b);
  const uint32_t w0 = l < hw ? hs[l] : 0u;
  const uint32_t c0 = __popc(w0);
  uint32_t i0 = c0;
#pragma unroll
  for (int d = 1; d < 16; d <<= 1) {
    const uint32_t t = __shfl_up_sync(0xffffffffu, i0, d, 16);
    if (l >= (uint32_t)d) i0 += t;
  }
  // owner word of element k0 = 8l: mark + inclusive max-scan (as the E = 4 path)
  const uint32_t ex0 = i0 - c0;
  const uint32_t a = (ex0 + 7u) >> 3, bnd = (i0 + 7u) >> 3;
  cnt[lane] = 0u;
  __syncwarp();
  if (l < hw && a < bnd && a < 16u) cnt[(hf << 4) + a] = l + 1u;
  __syncwarp();
  uint32_t v = cnt[lane];
#pragma unroll
  for (int d = 1; d < 16; d <<= 1) {
    const uint32_t t = __shfl_up_sync(0xffffffffu, v, d, 16);
    if (l >= (uint32_t)d) v = max(v, t);
  }
  const uint32_t w = v ? v - 1u : 0u;
  const uint32_t src = (hf << 4) | (w & 15u);
  const uint32_t x = __shfl_sync(0xffffffffu, w0, src);
  const uint32_t ex = __shfl_sync(0xffffffffu, ex0, src);
  uint32_t nx = __shfl_sync(0xffffffffu, w0, (src + 1u) & 31u);
  if (w + 1u >= hw) nx = 0u;
  const uint32_t k0 = l << 3;
  if (k0 < n) {
    const uint32_t pos = select_in_word(x, k0 - ex, lut);
    const uint32_t mask = b ? (0xFFFFFFFFu >> (32u - b)) : 0u;
    decode8(stg, hs, first, b, mask, k0, min(8u, n - k0), (w << 5) + pos,
            __funnelshift_rc(x, nx, pos + 1u), dst, sink);
  }
  __syncwarp();
}

__device__ __forceinline__ void warp_decode_staged(const uint32_t *__restrict__ stg, uint32_t first,
                                                   uint32_t y, uint32_t *__restrict__ dst,
                                                   uint32_t *__restrict__ cnt,
                                                   const uint8_t *__restrict__ lut) {
  StoreSink s;
  warp_decode_staged(stg, first, y, dst, cnt, lut, s);
}

// ---- run decoder: several blocks per warp, 32 consecutive elements per lane -----
// (B = 64/128/256/512.)  Alg. 1 re-cut for instruction count rather than for
// the paper's thread-per-element mapping: a group of Lb = B/32 lanes decodes one
// block, so one warp pass decodes 32/Lb blocks (16 at B = 64, 8 at B = 128)
// and every per-block and per-lane step is paid once per 32 postings:
//  * Alg. 1 l.2-3 (prefix sum): lane l of the group popcounts high words l,
//    l+Lb and l+2Lb (a block's unary stream has L < 3n <= 3*32*Lb bits); one
//    packed shuffle scan of width Lb gives all three inclusive prefixes.
//  * l.4-8 (scheduling): element k0 = 32t, where lane t starts, lies in the
//    word whose [exclusive, inclusive) prefix interval contains 32t; an
//    interval of <= 32 ones holds at most one multiple of 32, so every word
//    lane writes (word, exclusive prefix) straight into its target's record (no
//    search), and the target selects the bit with the byte LUT.
//  * l.9-10: the next ones come from a 96-bit stream of the high bits after the
//    current one, bit-reversed into three registers: FLO finds the next one
//    (i = its reversed index; 31 - i zeros precede it, so h += 31 - i), and a
//    funnel shift by 32 - i drops it and refills from the lower registers.  The
//    stream is re-seeded from shared memory after 16 elements (the position of
//    element 15's one is k0 + 15 + h), so no select is needed for the second
//    half.  x = first + (h << b) + low, low fields funnel-shifted out of the
//    staged low stream (a lane's 32 fields start word-aligned at word l*b).
//  * A lane that meets 32 zeros in a row inside its stream (~1e-4 of lanes at
//    the 1/3 .. 1/2 densities EF gives) takes the serial window walk.
// Inputs in lanes [l0, l0+nb): the block's meta word y, first docID f and its
// staged offset so (16-B units from stg).  Block i goes to dst + i*B.  `rec` is
// 32 words of per-warp scratch; stg needs kRunSlack words of read slack.
constexpr uint32_t kRunSlack = 40;   // a partial block's last lane reads <= 32 + 4 words past it
__host__ __device__ inline bool run_decoder_ok(uint32_t B) {
  return B == 64 || B == 128 || B == 256 || B == 512;
}

// Serial fallback (rare): elements [kfrom, kto) of the block, element kfrom's
// one being the first one at or after high-stream bit c; refilled 32-bit window.
template <class Sink>
__device__ __forceinline__ void lane_walk(const uint32_t *__restrict__ blk, const uint32_t *__restrict__ hs,
                                       uint32_t first, uint32_t b, uint32_t mask, uint32_t kfrom,
                                       uint32_t kto, uint32_t c, uint32_t *dst, Sink &sink) {
  uint32_t wb = c;
  uint32_t win = __funnelshift_r(hs[wb >> 5], hs[(wb >> 5) + 1], wb);
  for (uint32_t k = kfrom; k < kto; ++k) {
    while (win == 0u) {
      wb += 32u;
      win = __funnelshift_r(hs[wb >> 5], hs[(wb >> 5) + 1], wb);
    }
    const uint32_t p = wb + (__ffs(win) - 1u);
    win &= win - 1u;
    const uint32_t bp = k * b;
    const uint32_t lo = __funnelshift_r(blk[bp >> 5], blk[(bp >> 5) + 1], bp) & mask;
    sink.put(dst + k, first + (((p - k) << b) | lo));
  }
}

// FLO: bit index of the highest set bit (0xFFFFFFFF for 0)
__device__ __forceinline__ uint32_t flo_u32(uint32_t x) {
  uint32_t r;
  asm("bfind.u32 %0, %1;" : "=r"(r) : "r"(x));
  return r;
}
// x << s for s in [0, 32] (32 -> 0)
__device__ __forceinline__ uint32_t shl_c(uint32_t x, uint32_t s) {
  uint32_t r;
  asm("shl.b32 %0, %1, %2;" : "=r"(r) : "r"(x), "r"(s));
  return r;
}

// 96 high-stream bits starting at bit c, bit-reversed (bit c -> bit 31 of s0)
__device__ __forceinline__ void seed_stream(const uint32_t *__restrict__ hs, uint32_t c,
                                            uint32_t &s0, uint32_t &s1, uint32_t &s2) {
  const uint32_t cw = c >> 5;
  const uint32_t a0 = hs[cw], a1 = hs[cw + 1], a2 = hs[cw + 2], a3 = hs[cw + 3];
  s0 = __brev(__funnelshift_r(a0, a1, c));
  s1 = __brev(__funnelshift_r(a1, a2, c));
  s2 = __brev(__funnelshift_r(a2, a3, c));
}

// next one of the stream: returns its reversed index i (h grows by 31 - i);
// bad collects i (its top bit is set iff the stream's first word was empty)
__device__ __forceinline__ uint32_t stream_next(uint32_t &s0, uint32_t &s1, uint32_t &s2,
                                                uint32_t &bad) {
  const uint32_t i = flo_u32(s0);
  bad |= i;
  const uint32_t sh = 32u - i;   // drop the one and the zeros before it
  s0 = __funnelshift_lc(s1, s0, sh);
  s1 = __funnelshift_lc(s2, s1, sh);
  s2 = shl_c(s2, sh);
  return i;
}

template <uint32_t LG, class Sink>
__device__ __forceinline__ void warp_decode_runs_t(const uint32_t *__restrict__ stg, uint32_t l0,
                                                   uint32_t nb, uint32_t y_l, uint32_t f_l,
                                                   uint32_t so_l, uint32_t *dst,
                                                   uint32_t *__restrict__ rec,
                                                   const uint8_t *__restrict__ lut, Sink &sink) {
  constexpr uint32_t Lb = 1u << LG, bpw = 32u >> LG, B = Lb * 32u;
  const uint32_t lane = lane_id();
  const uint32_t g = lane >> LG, l = lane & (Lb - 1u);
  uint32_t *r = rec + (g << LG);
  for (uint32_t i = 0; i < nb; i += bpw) {
    const uint32_t bi = i + g;
    const bool act = bi < nb;
    const uint32_t src = (l0 + (act ? bi : nb - 1u)) & 31u;
    const uint32_t y = __shfl_sync(0xffffffffu, y_l, src);
    const uint32_t first = __shfl_sync(0xffffffffu, f_l, src);
    const uint32_t so = __shfl_sync(0xffffffffu, so_l, src);
    const uint32_t b = meta_b(y), n = act ? meta_n(y) : 0u, hw = act ? meta_hw(y) : 0u;
    const uint32_t *blk = stg + so * 4u;
    const uint32_t *hs = blk + low_words(n, b);
    const uint32_t wa = l < hw ? hs[l] : 0u;
    const uint32_t wb = l + Lb < hw ? hs[l + Lb] : 0u;
    const uint32_t wc = l + 2u * Lb < hw ? hs[l + 2u * Lb] : 0u;
    const uint32_t ca = __popc(wa), cb = __popc(wb), cc = __popc(wc);
    uint32_t c = ca | (cb << 10) | (cc << 20);   // three 10-bit counters (<= 512 each)
#pragma unroll
    for (uint32_t d = 1; d < Lb; d <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, c, d, Lb);
      if (l >= d) c += t;
    }
    const uint32_t tot = __shfl_sync(0xffffffffu, c, Lb - 1u, Lb);
    const uint32_t ta = tot & 0x3FFu, tb = (tot >> 10) & 0x3FFu;
    {  // exclusive prefixes of words l, l+Lb, l+2Lb; record the target (if any) of each
      const uint32_t ea = (c & 0x3FFu) - ca;
      const uint32_t eb = ta + ((c >> 10) & 0x3FFu) - cb;
      const uint32_t ec = ta + tb + (c >> 20) - cc;
      const uint32_t xa = (ea + 31u) >> 5, xb = (eb + 31u) >> 5, xc = (ec + 31u) >> 5;
      if ((xa << 5) < ea + ca) r[xa] = l | (ea << 8);
      if ((xb << 5) < eb + cb) r[xb] = (l + Lb) | (eb << 8);
      if ((xc << 5) < ec + cc) r[xc] = (l + 2u * Lb) | (ec << 8);
    }
    __syncwarp();
    const uint32_t k0 = l << 5;
    if (k0 < n) {
      const uint32_t rv = r[l];
      const uint32_t w = rv & 0xFFu, ex = rv >> 8;
      const uint32_t p0 = (w << 5) + select_in_word(hs[w], k0 - ex, lut);
      const uint32_t ne = min(32u, n - k0);
      const uint32_t mask = b ? (0xFFFFFFFFu >> (32u - b)) : 0u;
      // low fields: element k0 + j at bit j*b of the lane's run (word l*b)
      const uint32_t *lw = blk + l * b;
      uint32_t s0, s1, s2, bad = 0u;
      uint32_t h = p0 - k0;   // high part of the current element
      uint32_t *out = dst + bi * B;
      // (a lane of a list's partial last block decodes all 32 slots from the
      // staged bytes after its block — the staging area's read slack covers
      // them — and stores only its ne elements)
      seed_stream(hs, p0 + 1u, s0, s1, s2);
#pragma unroll
      for (uint32_t half = 0; half < 2; ++half) {
        // half 1 re-seeds after element 15's one, at bit k0 + 15 + h + 1
        if (half) seed_stream(hs, k0 + 16u + h, s0, s1, s2);
        const uint32_t c_half = k0 + half * 16u + h;   // search start for the walk
        uint32_t lo[16], v[16];
        if (b <= 16u) {   // two fields per 32-bit window
#pragma unroll
          for (uint32_t j = 0; j < 16; j += 2) {
            const uint32_t o = (half * 16u + j) * b;
            const uint32_t wv = __funnelshift_r(lw[o >> 5], lw[(o >> 5) + 1], o);
            lo[j] = wv & mask;
            lo[j + 1] = (wv >> b) & mask;
          }
        } else {
#pragma unroll
          for (uint32_t j = 0; j < 16; ++j) {
            const uint32_t o = (half * 16u + j) * b;
            lo[j] = __funnelshift_r(lw[o >> 5], lw[(o >> 5) + 1], o) & mask;
          }
        }
#pragma unroll
        for (uint32_t j = 0; j < 16; ++j) {
          if (half || j) h += 31u - stream_next(s0, s1, s2, bad);
          v[j] = first + (h << b) + lo[j];
        }
        if (ne == 32u && !(bad >> 31)) {
#pragma unroll
          for (uint32_t j = 0; j < 16; j += 4)
            sink.put4(out + k0 + half * 16u + j, make_uint4(v[j], v[j + 1], v[j + 2], v[j + 3]));
        } else if (!(bad >> 31)) {   // partial block: this lane's first ne elements
#pragma unroll
          for (uint32_t j = 0; j < 16; ++j)
            if (half * 16u + j < ne) sink.put(out + k0 + half * 16u + j, v[j]);
        } else {   // a run of >= 32 zeros inside the stream: walk this half (and the next)
          lane_walk(blk, hs, first, b, mask, k0 + half * 16u, k0 + ne,
                    half ? c_half : p0, out, sink);
          break;
        }
        if (half * 16u + 16u >= ne) break;
      }
    }
    __syncwarp();
  }
}

template <class Sink>
__device__ __forceinline__ void warp_decode_runs(const uint32_t *__restrict__ stg, uint32_t l0,
                                                 uint32_t nb, uint32_t y_l, uint32_t f_l,
                                                 uint32_t so_l, uint32_t *dst, uint32_t B,
                                                 uint32_t *__restrict__ rec,
                                                 const uint8_t *__restrict__ lut, Sink &sink) {
  switch (B) {   // uniform per index: only one instantiation ever runs
    case 64: warp_decode_runs_t<1>(stg, l0, nb, y_l, f_l, so_l, dst, rec, lut, sink); break;
    case 128: warp_decode_runs_t<2>(stg, l0, nb, y_l, f_l, so_l, dst, rec, lut, sink); break;
    case 256: warp_decode_runs_t<3>(stg, l0, nb, y_l, f_l, so_l, dst, rec, lut, sink); break;
    default: warp_decode_runs_t<4>(stg, l0, nb, y_l, f_l, so_l, dst, rec, lut, sink); break;
  }
}

// ---- EF NextGEQ inside one staged block -------------------
// Index of the first element >= x of the block staged at stg (n if none) and
// its value in `val`, without decoding the block: the elements whose high part
// is >= h = (x - first) >> b start right after the h-th zero of the unary high
// stream (each zero closes one high bucket), so a select0 over the
// high words (popc per word, byte LUT in the word) gives their index
// i0 = pos - h; only the few elements of bucket h (about u/n / 2^b <= 2 on
// average) are then decoded and compared.  One lane per query element.
__device__ __forceinline__ uint32_t ef_next_geq_staged(const uint32_t *__restrict__ stg,
                                                       uint32_t first, uint32_t y, uint32_t x,
                                                       const uint8_t *__restrict__ lut,
                                                       uint32_t &val) {
  const uint32_t b = meta_b(y), n = meta_n(y), hw = meta_hw(y);
  const uint32_t *hs = stg + low_words(n, b);
  val = first;
  if (x <= first) return 0u;
  const uint32_t h = (x - first) >> b;
  uint32_t pos = 0;   // first bit of the one-scan
  uint32_t w = 0, cur = 0;
  if (h) {
    uint32_t need = h;
    for (;;) {
      if (w >= hw) return n;   // fewer than h zeros: every high part is < h
      cur = hs[w];
      const uint32_t z = 32u - __popc(cur);
      if (z >= need) break;
      need -= z;
      ++w;
    }
    pos = (w << 5) + select_in_word(~cur, need - 1u, lut) + 1u;
  }
  uint32_t i = pos - h;   // ones before pos = pos - (zeros before pos = h)
  const uint32_t mask = b ? (0xFFFFFFFFu >> (32u - b)) : 0u;
  w = pos >> 5;
  cur = w < hw ? hs[w] & (0xFFFFFFFFu << (pos & 31u)) : 0u;
  while (i < n) {
    while (cur == 0u) {
      if (++w >= hw) return n;
      cur = hs[w];
    }
    const uint32_t p = (w << 5) + (__ffs(cur) - 1u);
    cur &= cur - 1u;
    const uint32_t bp = i * b;
    const uint32_t lo = __funnelshift_r(stg[bp >> 5], stg[(bp >> 5) + 1], bp) & mask;
    const uint32_t xv = first + (((p - i) << b) | lo);
    if (xv >= x) {
      val = xv;
      return i;
    }
    ++i;
  }
  return n;
}

// payload size of a block in 16-B units
__host__ __device__ inline uint32_t block_size16(uint32_t y) {
  return (low_words(meta_n(y), meta_b(y)) + meta_hw(y) + 3u) >> 2;
}
// staging words per block (upper bound for any b <= 31, plus read slack)
__host__ __device__ inline uint32_t stage_words_per_block(uint32_t B) {
  return ((B * 34u) / 32u + 8u + 3u) & ~3u;
}

// ---- tf and BM25 ---------------------------------------------------------------
__device__ __forceinline__ uint32_t tf_lookup(const DevIndex &ix, const TermInfo &t, uint32_t pos) {
  if (t.tf_w == 0) return 1u;
  const uint64_t bit = (uint64_t)pos * t.tf_w;
  const uint32_t *w = ix.tfw + t.tf_off + (bit >> 5);
  const uint32_t v = __funnelshift_r(__ldg(w), __ldg(w + 1), (uint32_t)(bit & 31u));
  return (v & (0xFFFFFFFFu >> (32u - t.tf_w))) + 1u;
}

// w_{t,d} = idf_t * ((tf*(k1+1)) / (tf + norm_d)) — one IEEE f32 op each, no FMA
// contraction (explicit _rn intrinsics), order fixed by SURVEY O6.
__device__ __forceinline__ float bm25_w(float idf, uint32_t tf, float norm, float k1p1) {
  const float tf_f = __uint2float_rn(tf);
  const float num = __fmul_rn(tf_f, k1p1);
  const float den = __fadd_rn(tf_f, norm);
  return __fmul_rn(idf, __fdiv_rn(num, den));
}

// ---- searches ------------------------------------------------------------------
// number of elements of a[0..n) that are <= x (upper_bound), global memory
__device__ __forceinline__ uint32_t upper_bound_g(const uint32_t *__restrict__ a, uint32_t lo,
                                                  uint32_t hi, uint32_t x) {
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(a + mid) <= x) lo = mid + 1; else hi = mid;
  }
  return lo;
}
__device__ __forceinline__ uint32_t lower_bound_s(const uint32_t *a, uint32_t lo, uint32_t hi,
                                                  uint64_t x) {
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;
    if ((uint64_t)a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// Merge-path diagonal search (Fig. 6): on diagonal d of the |A|x|B|
// grid find the crossing (i, d-i) of the path built by "advance in A iff
// A[i] <= B[j]".  With fixup, a matched pair A[i-1]==B[j]
// is never split.  Getter-based so it works on smem, global or
// strided (chunk-head) arrays.
template <class GA, class GB>
__host__ __device__ inline void merge_path_split(GA A, uint32_t na, GB B, uint32_t nb, uint32_t d,
                                                 bool fixup, uint32_t *ri, uint32_t *rj) {
  uint32_t lo = d > nb ? d - nb : 0u;
  uint32_t hi = d < na ? d : na;
  while (lo < hi) {
    const uint32_t mid = (lo + hi) >> 1;   // take `mid` from A and d-mid from B
    if (A(mid) <= B(d - mid - 1)) lo = mid + 1; else hi = mid;
  }
  uint32_t i = lo, j = d - lo;
  if (fixup && i > 0 && j < nb && A(i - 1) == B(j)) ++j;
  *ri = i;
  *rj = j;
}

}  // namespace griffin
