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

// ---- Elias-Fano block decode (Para-EF, §3.1.1 / Alg. 1) -------------
// One warp decodes one block of n <= B postings into dst[0..n) (shared memory),
// as absolute local docIDs x_i = first + ((h_i << b) | low_i).
//  * scheduling phase (Alg. 1 l.2-8): the high stream is consumed one 32-bit
//    word per warp step; lane l owns bit l of the word, its rank among the word's
//    ones is popc(word & lanemask_lt) and the running count of ones before the
//    word is the warp-uniform prefix `base` (the prefix sum of l.3).  A lane whose
//    bit is set is element k = base + rank and writes its high part h_k = p - k
//    (the number of zeros before the k-th one).
//  * decompress phase (l.9-10): lane-strided elements funnel-shift their b low
//    bits out of the staged low stream and OR them in.
// `scratch` is per-warp shared memory of >= payload words + 4 u32, 16-B aligned.
__device__ __forceinline__ uint32_t warp_decode_block(const DevIndex &ix, uint64_t blk,
                                                      uint32_t *__restrict__ dst,
                                                      uint32_t *__restrict__ scratch,
                                                      uint32_t *payload_bytes = nullptr) {
  const uint32_t lane = lane_id();
  const uint2 m = ix.meta[blk];
  const uint32_t first = ix.first[blk];
  const uint32_t b = meta_b(m.y), n = meta_n(m.y), hw = meta_hw(m.y);
  const uint32_t lw = low_words(n, b);
  const uint32_t n16 = (lw + hw + 3u) >> 2;
  const uint4 *src = ix.payload + m.x;
  uint4 *s4 = reinterpret_cast<uint4 *>(scratch);
  for (uint32_t i = lane; i < n16; i += 32) s4[i] = ldg_nc_v4(src + i);
  if (lane == 0) s4[n16] = make_uint4(0, 0, 0, 0);
  __syncwarp();
  // scheduling phase: scatter high parts
  const uint32_t *hs = scratch + lw;
  const uint32_t lt = lanemask_lt();
  uint32_t base = 0;
  for (uint32_t w = 0; base < n; ++w) {
    const uint32_t word = hs[w];
    const uint32_t k = base + __popc(word & lt);
    if ((word >> lane) & 1u) dst[k] = (w << 5) + lane - k;
    base += __popc(word);
  }
  __syncwarp();
  // decompress phase: low bits
  const uint32_t mask = b ? (0xFFFFFFFFu >> (32u - b)) : 0u;
  for (uint32_t e = lane; e < n; e += 32) {
    const uint32_t bit = e * b;
    const uint32_t wi = bit >> 5;
    const uint32_t lo = __funnelshift_r(scratch[wi], scratch[wi + 1], bit & 31u) & mask;
    dst[e] = first + ((dst[e] << b) | lo);
  }
  __syncwarp();
  if (payload_bytes) *payload_bytes = n16 * 16u;
  return n;
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
