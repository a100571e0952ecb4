// pfd.cu — GPU PforDelta block codec: the paper's comparison scheme (§2.1.1,
// P:285-311, Fig. 3), built as the NEXT-3 comparator of SURVEY.md §8(f): the
// same lists in the same block layout as the EF index, so bits/posting and
// decode throughput can be set side by side (Table 1 / Fig. 12 shape).
//
// Block of n <= B docIDs: x_0 is the skip entry (first[]), the m = n-1 d-gaps
// g_i = x_i - x_{i-1} are coded (stream layout as oracle/pfd.cpp, which this
// file does not share code with):
//   word 0   first exception position (m if none) | n_exc << 10 | b << 20
//   slots    m x b bits LSB-first: the gap, or for an exception the distance to
//            the next exception minus one (last: 0)
//   values   n_exc u32 exception gaps, last exception first
// b = bits of the largest of the ceil(0.9 m) smallest gaps; two
// consecutive exceptions more than 2^b apart force the gap 2^b after the first
// to be an exception, so every link fits in b bits (reading P3).
// Encode: size pass (thread per block) -> scan -> write pass (thread per
// block).  Decode: warp per block — lanes unpack four slots each, lane 0 walks
// the exception list in shared memory (the scheme's inherently serial patch
// step), then a warp prefix sum turns gaps into docIDs.
#include <algorithm>
#include <vector>

#include "internal.h"
#include "scan.cuh"

struct griffin_pfd {
  int device = 0;
  cudaStream_t stream = nullptr;
  uint32_t B = 128, V = 0;
  uint32_t *d_first = nullptr;
  uint2 *d_meta = nullptr;      // {payload offset / 16 B, (n-1) | words << 10 | b << 20}
  uint4 *d_payload = nullptr;
  uint64_t nblocks = 0, payload16 = 0, postings = 0, exceptions = 0;
  std::vector<uint64_t> term_block0;   // [V+1]
};

namespace griffin {

__host__ __device__ inline uint32_t pfd_n(uint32_t y) { return (y & 1023u) + 1u; }
__host__ __device__ inline uint32_t pfd_words(uint32_t y) { return (y >> 10) & 1023u; }
__host__ __device__ inline uint32_t pfd_b(uint32_t y) { return (y >> 20) & 63u; }

__device__ __forceinline__ uint32_t bit_width(uint32_t v) { return 32u - __clz(v); }

// b by the 90% rule, and the exception count including forced exceptions.
__device__ void pfd_plan(const uint32_t *__restrict__ x, uint32_t n, uint32_t *b_out,
                         uint32_t *nexc_out) {
  const uint32_t m = n - 1;
  uint32_t cnt[33];
  for (int w = 0; w <= 32; ++w) cnt[w] = 0;
  for (uint32_t i = 1; i < n; ++i) ++cnt[bit_width(x[i] - x[i - 1])];
  uint32_t b = 0;
  if (m) {
    const uint32_t need = (9u * m + 9u) / 10u;
    uint32_t acc = 0;
    for (uint32_t w = 1; w <= 32; ++w) {
      acc += cnt[w];
      if (acc >= need) {
        b = w;
        break;
      }
    }
  }
  uint32_t nexc = 0;
  if (b < 32) {
    const int64_t maxd = 1ll << b;
    int64_t prev = -1;
    for (uint32_t i = 0; i < m; ++i) {
      if (x[i + 1] - x[i] < (1u << b)) continue;
      while (prev >= 0 && (int64_t)i - prev > maxd) {
        prev += maxd;
        ++nexc;
      }
      ++nexc;
      prev = i;
    }
  }
  *b_out = b;
  *nexc_out = nexc;
}

__global__ void pfd_size_kernel(const uint32_t *__restrict__ doc, const uint64_t *__restrict__ bs,
                                const uint32_t *__restrict__ bn, uint64_t nb,
                                uint32_t *__restrict__ first, uint2 *__restrict__ meta,
                                uint32_t *__restrict__ size16) {
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < nb;
       k += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t *x = doc + bs[k];
    const uint32_t n = bn[k];
    uint32_t b, nexc;
    pfd_plan(x, n, &b, &nexc);
    const uint32_t words = 1u + (uint32_t)(((uint64_t)(n - 1) * b + 31u) >> 5) + nexc;
    first[k] = x[0];
    meta[k] = make_uint2(0u, (n - 1u) | (words << 10) | (b << 20));
    size16[k] = (words + 3u) >> 2;
  }
}

// Set the b-bit slot at bit position `bit` to v (the block's words are owned by
// this thread and pre-zeroed).
__device__ __forceinline__ void set_bits(uint32_t *w, uint64_t bit, uint32_t v, uint32_t b) {
  if (!b) return;
  const uint32_t sh = (uint32_t)(bit & 31u), idx = (uint32_t)(bit >> 5);
  const uint32_t mask = b >= 32 ? 0xFFFFFFFFu : ((1u << b) - 1u);
  w[idx] = (w[idx] & ~(mask << sh)) | (v << sh);
  if (sh + b > 32u) {
    const uint32_t hm = mask >> (32u - sh);
    w[idx + 1] = (w[idx + 1] & ~hm) | (v >> (32u - sh));
  }
}

__global__ void pfd_write_kernel(const uint32_t *__restrict__ doc, const uint64_t *__restrict__ bs,
                                 const uint64_t *__restrict__ off16, uint64_t nb,
                                 uint2 *__restrict__ meta, uint32_t *__restrict__ payload,
                                 unsigned long long *nexc_total) {
  unsigned long long my_exc = 0;
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < nb;
       k += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t *x = doc + bs[k];
    uint2 mm = meta[k];
    const uint32_t n = pfd_n(mm.y), m = n - 1, b = pfd_b(mm.y), words = pfd_words(mm.y);
    const uint32_t slot_words = (uint32_t)(((uint64_t)m * b + 31u) >> 5);
    const uint32_t nexc = words - 1u - slot_words;
    uint32_t *w = payload + off16[k] * 4;
    const bool any_exc = b < 32;
    // pass 1: every gap that fits into its slot
    for (uint32_t i = 0; i < m; ++i) {
      const uint32_t g = x[i + 1] - x[i];
      if (!(any_exc && g >= (1u << b))) set_bits(w + 1, (uint64_t)i * b, g, b);
    }
    // pass 2: the exception list (natural + forced), links and values
    const int64_t maxd = any_exc ? (1ll << b) : 0;
    int64_t prev = -1;
    uint32_t e = 0, fe = m;
    auto mark = [&](uint32_t p) {   // position p becomes exception number e
      set_bits(w + 1, (uint64_t)p * b, 0u, b);
      if (prev >= 0) set_bits(w + 1, (uint64_t)prev * b, (uint32_t)(p - prev - 1), b);
      else fe = p;
      w[1 + slot_words + (nexc - 1u - e)] = x[p + 1] - x[p];
      ++e;
      prev = p;
    };
    if (any_exc) {
      for (uint32_t i = 0; i < m; ++i) {
        if (x[i + 1] - x[i] < (1u << b)) continue;
        while (prev >= 0 && (int64_t)i - prev > maxd) mark((uint32_t)(prev + maxd));
        mark(i);
      }
    }
    w[0] = fe | (nexc << 10) | (b << 20);
    mm.x = (uint32_t)off16[k];
    meta[k] = mm;
    my_exc += e;
  }
  if (my_exc) atomicAdd(nexc_total, my_exc);
}

// Warp decodes one block whose stream is in shared memory `s` into dst[0..n).
// `g` is per-warp scratch of >= B words.
__device__ __forceinline__ void pfd_warp_decode(const uint32_t *__restrict__ s, uint32_t first,
                                                uint32_t n, uint32_t *__restrict__ g,
                                                uint32_t *__restrict__ dst) {
  const uint32_t lane = lane_id();
  const uint32_t m = n - 1;
  const uint32_t hdr = s[0];
  const uint32_t fe = hdr & 1023u, nexc = (hdr >> 10) & 1023u, b = (hdr >> 20) & 63u;
  const uint32_t slot_words = (uint32_t)(((uint64_t)m * b + 31u) >> 5);
  const uint32_t mask = b >= 32 ? 0xFFFFFFFFu : ((1u << b) - 1u);
  const uint32_t E = (n + 31u) >> 5;   // elements per lane: x_{lane*E ...}
  // slots: lane l unpacks gaps g[p] for p in [l*E, l*E+E) (gap p = x_{p+1} - x_p)
  for (uint32_t j = 0; j < E; ++j) {
    const uint32_t p = lane * E + j;
    if (p < m) {
      const uint64_t bit = (uint64_t)p * b;
      const uint32_t lo = s[1 + (bit >> 5)], hi = s[2 + (bit >> 5)];
      g[p] = b ? (__funnelshift_r(lo, hi, (uint32_t)(bit & 31u)) & mask) : 0u;
    }
  }
  __syncwarp();
  if (lane == 0) {   // the exception list: serial by construction (linked list)
    uint32_t p = fe;
    for (uint32_t e = 0; e < nexc; ++e) {
      const uint32_t link = g[p];
      g[p] = s[1 + slot_words + (nexc - 1u - e)];
      p += link + 1u;
    }
  }
  __syncwarp();
  // x_i = first + sum_{p < i} g[p]: lane l owns x_{lE .. lE+E-1}
  uint32_t loc[16];
  uint32_t run = 0;
#pragma unroll
  for (uint32_t j = 0; j < 16; ++j) {
    if (j < E) {
      const uint32_t i = lane * E + j;
      run += (i >= 1 && i < n) ? g[i - 1] : 0u;
      loc[j] = run;
    }
  }
  const uint32_t incl = warp_incl_scan(run);
  const uint32_t base = first + (incl - run);
#pragma unroll
  for (uint32_t j = 0; j < 16; ++j) {
    if (j < E) {
      const uint32_t i = lane * E + j;
      if (i < n) dst[i] = base + loc[j];
    }
  }
  __syncwarp();
}

constexpr uint32_t kPfdWarps = 8;

// Warp per block, grid-stride: stage the stream (coalesced u32 loads), decode,
// fold into a checksum (decode-only sweep, like decode_all_kernel for EF) or
// write out[] (debug list decode, global positions).
__global__ void __launch_bounds__(256) pfd_decode_kernel(const uint32_t *__restrict__ first,
                                                         const uint2 *__restrict__ meta,
                                                         const uint32_t *__restrict__ payload,
                                                         uint64_t b0, uint64_t nb, uint32_t B,
                                                         uint32_t *out,
                                                         unsigned long long *acc) {
  extern __shared__ uint32_t pfd_smem[];
  const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
  // per warp: stream (<= 2B+8 words) | gaps (B) | tile (B)
  const uint32_t per = 2 * B + 8 + 2 * B;
  uint32_t *s = pfd_smem + wid * per, *g = s + 2 * B + 8, *tile = g + B;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  uint32_t x = 0;
  unsigned long long post = 0, bytes = 0;
  for (uint64_t k = blockIdx.x * (uint64_t)(blockDim.x >> 5) + wid; k < nb; k += nwarps) {
    const uint2 mm = meta[b0 + k];
    const uint32_t n = pfd_n(mm.y), words = pfd_words(mm.y);
    const uint32_t *src = payload + (uint64_t)mm.x * 4;
    for (uint32_t i = lane; i < words + 2; i += 32) s[i] = i < words ? __ldg(src + i) : 0u;
    __syncwarp();
    pfd_warp_decode(s, __ldg(first + b0 + k), n, g, tile);
    if (out) {
      for (uint32_t i = lane; i < n; i += 32) out[k * B + i] = tile[i];
    } else {
      for (uint32_t i = lane; i < n; i += 32) x ^= tile[i];
    }
    __syncwarp();
    post += n;
    bytes += ((words + 3u) >> 2) * 16u + 8u;
  }
  if (acc) {
    for (int d = 16; d; d >>= 1) x ^= __shfl_xor_sync(0xffffffffu, x, d);
    if (lane == 0) {
      atomicXor(acc + 0, (unsigned long long)x);
      atomicAdd(acc + 1, post);
      atomicAdd(acc + 2, bytes);
    }
  }
}

static griffin_status pfd_fail(const char *m, griffin_status s = GRIFFIN_ERR_INVALID_ARG) {
  set_error(m);
  return s;
}

}  // namespace griffin

using namespace griffin;

extern "C" {

griffin_status griffin_pfd_build(const griffin_corpus *c, uint32_t block_size, int device,
                                 griffin_pfd **out) {
  if (!c || !out) return pfd_fail("null corpus/out");
  *out = nullptr;
  const uint32_t B = block_size ? block_size : 128;
  if (B < 64 || B > 512 || (B % 32)) return pfd_fail("block_size must be 64..512, multiple of 32");
  const uint32_t V = c->num_terms, N = c->num_docs;
  if (!c->list_offsets || (c->list_offsets[V] && !c->docids)) return pfd_fail("null corpus arrays");
  for (uint32_t t = 0; t < V; ++t) {
    const uint64_t a = c->list_offsets[t], e = c->list_offsets[t + 1];
    if (e < a) return pfd_fail("list_offsets not monotone");
    for (uint64_t p = a; p < e; ++p)
      if (c->docids[p] >= N || (p > a && c->docids[p] <= c->docids[p - 1]))
        return pfd_fail("list not strictly increasing or docID >= num_docs", GRIFFIN_ERR_UNSORTED);
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
    return pfd_fail("no CUDA device", GRIFFIN_ERR_UNSUPPORTED);
  int dev = device;
  if (dev < 0) cudaGetDevice(&dev);
  if (dev >= ndev) return pfd_fail("device ordinal out of range");
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(dev);
  griffin_pfd *p = new griffin_pfd();
  p->device = dev;
  p->B = B;
  p->V = V;
  auto fail = [&](griffin_status s) {
    griffin_pfd_destroy(p);
    cudaSetDevice(prev);
    return s;
  };
#define PFD_TRY(x)                                            \
  do {                                                        \
    cudaError_t e_ = (x);                                     \
    if (e_ != cudaSuccess) {                                  \
      set_error(std::string("CUDA: ") + cudaGetErrorString(e_)); \
      return fail(GRIFFIN_ERR_CUDA);                          \
    }                                                         \
  } while (0)
  PFD_TRY(cudaStreamCreateWithFlags(&p->stream, cudaStreamNonBlocking));
  std::vector<uint64_t> bs;
  std::vector<uint32_t> bn;
  p->term_block0.resize(V + 1);
  for (uint32_t t = 0; t < V; ++t) {
    p->term_block0[t] = bs.size();
    for (uint64_t s = c->list_offsets[t]; s < c->list_offsets[t + 1]; s += B) {
      bs.push_back(s);
      bn.push_back((uint32_t)std::min<uint64_t>(B, c->list_offsets[t + 1] - s));
    }
  }
  p->term_block0[V] = bs.size();
  const uint64_t nb = bs.size(), P = c->list_offsets[V];
  p->nblocks = nb;
  p->postings = P;
  cudaStream_t st = p->stream;
  DevBuf d_doc, d_bs, d_bn, d_size, d_off, d_tmp, d_cnt;
  PFD_TRY(d_doc.reserve(std::max<uint64_t>(P, 1) * 4));
  PFD_TRY(d_bs.reserve((nb + 1) * 8));
  PFD_TRY(d_bn.reserve((nb + 1) * 4));
  PFD_TRY(d_size.reserve((nb + 1) * 4));
  PFD_TRY(d_off.reserve((nb + 1) * 8));
  PFD_TRY(d_tmp.reserve((nb / kScanTile + 8) * 8));
  PFD_TRY(d_cnt.reserve(8));
  PFD_TRY(cudaMemsetAsync(d_cnt.p, 0, 8, st));
  if (P) PFD_TRY(cudaMemcpyAsync(d_doc.p, c->docids, P * 4, cudaMemcpyHostToDevice, st));
  if (nb) {
    PFD_TRY(cudaMemcpyAsync(d_bs.p, bs.data(), nb * 8, cudaMemcpyHostToDevice, st));
    PFD_TRY(cudaMemcpyAsync(d_bn.p, bn.data(), nb * 4, cudaMemcpyHostToDevice, st));
  }
  PFD_TRY(cudaMalloc(&p->d_first, (nb + 1) * 4));
  PFD_TRY(cudaMalloc(&p->d_meta, (nb + 1) * 8));
  uint64_t total16 = 0;
  if (nb) {
    pfd_size_kernel<<<(unsigned)std::min<uint64_t>((nb + 127) / 128, (uint64_t)num_sms(p->device) * 64), 128, 0, st>>>(
        d_doc.as<uint32_t>(), d_bs.as<uint64_t>(), d_bn.as<uint32_t>(), nb, p->d_first,
        p->d_meta, d_size.as<uint32_t>());
    PFD_TRY(cudaGetLastError());
    PFD_TRY(exclusive_scan<uint32_t>(d_size.as<uint32_t>(), d_off.as<uint64_t>(), nb,
                                     d_tmp.as<uint64_t>(), st));
    PFD_TRY(cudaMemcpyAsync(&total16, d_off.as<uint64_t>() + nb, 8, cudaMemcpyDeviceToHost, st));
    PFD_TRY(cudaStreamSynchronize(st));
  }
  p->payload16 = total16;
  PFD_TRY(cudaMalloc(&p->d_payload, (total16 + 64) * 16));
  PFD_TRY(cudaMemsetAsync(p->d_payload, 0, (total16 + 64) * 16, st));
  if (nb) {
    pfd_write_kernel<<<(unsigned)std::min<uint64_t>((nb + 127) / 128, (uint64_t)num_sms(p->device) * 64), 128, 0, st>>>(
        d_doc.as<uint32_t>(), d_bs.as<uint64_t>(), d_off.as<uint64_t>(), nb, p->d_meta,
        reinterpret_cast<uint32_t *>(p->d_payload), d_cnt.as<unsigned long long>());
    PFD_TRY(cudaGetLastError());
  }
  unsigned long long ne = 0;
  PFD_TRY(cudaMemcpyAsync(&ne, d_cnt.p, 8, cudaMemcpyDeviceToHost, st));
  PFD_TRY(cudaStreamSynchronize(st));
  p->exceptions = ne;
#undef PFD_TRY
  cudaSetDevice(prev);
  *out = p;
  return GRIFFIN_OK;
}

void griffin_pfd_destroy(griffin_pfd *p) {
  if (!p) return;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(p->device);
  if (p->stream) cudaStreamSynchronize(p->stream);
  cudaFree(p->d_first);
  cudaFree(p->d_meta);
  cudaFree(p->d_payload);
  if (p->stream) cudaStreamDestroy(p->stream);
  cudaSetDevice(prev);
  delete p;
}

griffin_status griffin_pfd_stats(const griffin_pfd *p, griffin_pfd_stats_t *out) {
  if (!p || !out) return pfd_fail("null argument");
  out->block_size = p->B;
  out->num_blocks = p->nblocks;
  out->num_postings = p->postings;
  out->payload_bytes = p->payload16 * 16;
  out->skip_bytes = p->nblocks * 8;
  out->exceptions = p->exceptions;
  return GRIFFIN_OK;
}

griffin_status griffin_pfd_block_stream(griffin_pfd *p, uint32_t term, uint32_t block,
                                        uint32_t *first, uint32_t *n, uint32_t *words,
                                        uint32_t cap, uint32_t *nwords) {
  if (!p || !first || !n || !nwords || term >= p->V) return pfd_fail("bad arguments");
  const uint64_t b0 = p->term_block0[term], nb = p->term_block0[term + 1] - b0;
  if (block >= nb) return pfd_fail("block out of range");
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(p->device);
  uint2 mm;
  griffin_status rc = GRIFFIN_OK;
  if (cudaMemcpy(&mm, p->d_meta + b0 + block, 8, cudaMemcpyDeviceToHost) != cudaSuccess ||
      cudaMemcpy(first, p->d_first + b0 + block, 4, cudaMemcpyDeviceToHost) != cudaSuccess) {
    rc = pfd_fail("CUDA copy failed", GRIFFIN_ERR_CUDA);
  } else {
    *n = pfd_n(mm.y);
    *nwords = pfd_words(mm.y);
    if (*nwords > cap) {
      rc = pfd_fail("capacity too small");
    } else if (*nwords && cudaMemcpy(words, reinterpret_cast<const uint32_t *>(p->d_payload) +
                                                (uint64_t)mm.x * 4,
                                            *nwords * 4, cudaMemcpyDeviceToHost) != cudaSuccess) {
      rc = pfd_fail("CUDA copy failed", GRIFFIN_ERR_CUDA);
    }
  }
  cudaSetDevice(prev);
  return rc;
}

griffin_status griffin_pfd_decode_list(griffin_pfd *p, uint32_t term, uint32_t *out,
                                       uint64_t cap, uint64_t *n_out) {
  if (!p || !n_out || term >= p->V) return pfd_fail("bad arguments");
  const uint64_t b0 = p->term_block0[term], nb = p->term_block0[term + 1] - b0;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(p->device);
  griffin_status rc = GRIFFIN_OK;
  uint64_t n = 0;
  if (nb) {
    uint2 last;
    cudaMemcpy(&last, p->d_meta + b0 + nb - 1, 8, cudaMemcpyDeviceToHost);
    n = (nb - 1) * p->B + pfd_n(last.y);
  }
  *n_out = n;
  if (n > cap) {
    rc = pfd_fail("capacity too small");
  } else if (n) {
    uint32_t *d = nullptr;
    const size_t smem = (size_t)(4 * p->B + 8) * 4 * kPfdWarps;
    if (cudaMalloc(&d, nb * p->B * 4) != cudaSuccess) {
      rc = pfd_fail("out of device memory", GRIFFIN_ERR_OOM);
    } else {
      launch_config((const void *)pfd_decode_kernel, p->device, smem, 256, nullptr);
      pfd_decode_kernel<<<(unsigned)std::min<uint64_t>((nb + 7) / 8, (uint64_t)num_sms(p->device) * 4), 256, smem,
                          p->stream>>>(p->d_first, p->d_meta,
                                       reinterpret_cast<const uint32_t *>(p->d_payload), b0, nb,
                                       p->B, d, nullptr);
      if (cudaGetLastError() != cudaSuccess || cudaStreamSynchronize(p->stream) != cudaSuccess ||
          cudaMemcpy(out, d, n * 4, cudaMemcpyDeviceToHost) != cudaSuccess)
        rc = pfd_fail("decode failed", GRIFFIN_ERR_CUDA);
      cudaFree(d);
    }
  }
  cudaSetDevice(prev);
  return rc;
}

griffin_status griffin_pfd_decode_all(griffin_pfd *p, uint32_t iters, double *ms,
                                      uint64_t *postings, uint64_t *bytes, uint64_t *checksum) {
  if (!p || !ms || !postings || !bytes || !checksum || iters == 0) return pfd_fail("bad arguments");
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(p->device);
  griffin_status rc = GRIFFIN_OK;
  unsigned long long *acc = nullptr;
  cudaEvent_t a = nullptr, b = nullptr;
  const size_t smem = (size_t)(4 * p->B + 8) * 4 * kPfdWarps;
  int per_sm = 1, nsm = 1;
  launch_config((const void *)pfd_decode_kernel, p->device, smem, 256, &per_sm);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, p->device);
  const unsigned grid = (unsigned)std::max(1, nsm * std::max(1, per_sm));
  if (cudaMalloc(&acc, 3 * 8) != cudaSuccess) {
    cudaSetDevice(prev);
    return pfd_fail("out of device memory", GRIFFIN_ERR_OOM);
  }
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  unsigned long long h[3] = {0, 0, 0}, first_ck = 0;
  for (uint32_t it = 0; it <= iters; ++it) {   // iteration 0: warm-up, gives the checksum
    cudaMemsetAsync(acc, 0, 24, p->stream);
    if (it == 1) cudaEventRecord(a, p->stream);
    if (p->nblocks)
      pfd_decode_kernel<<<grid, 256, smem, p->stream>>>(
          p->d_first, p->d_meta, reinterpret_cast<const uint32_t *>(p->d_payload), 0, p->nblocks,
          p->B, nullptr, acc);
    if (it == 0) {
      cudaMemcpyAsync(h, acc, 24, cudaMemcpyDeviceToHost, p->stream);
      cudaStreamSynchronize(p->stream);
      first_ck = h[0];
    }
  }
  cudaEventRecord(b, p->stream);
  if (cudaStreamSynchronize(p->stream) != cudaSuccess || cudaGetLastError() != cudaSuccess) {
    rc = pfd_fail("decode sweep failed", GRIFFIN_ERR_CUDA);
  } else {
    float t = 0.f;
    cudaEventElapsedTime(&t, a, b);
    *ms = (double)t / iters;
    *postings = h[1];
    *bytes = h[2];
    *checksum = first_ck;
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(acc);
  cudaSetDevice(prev);
  return rc;
}

}  // extern "C"
