// encode.cu — Elias-Fano block encoding of the index on the device
// (§2.1.1, §3.1.1, Fig. 4
// P:485-495, "fixed-length partitioned EF" P:609-610, skip pointers Fig. 2).
//
// Per block of n <= B postings x_0 < ... < x_{n-1} (local docIDs):
//   first = x_0, v_i = x_i - first, u = v_{n-1} + 1, b = floor(log2(u / n)) (A1, A2)
//   low stream  : bits [i*b, (i+1)*b) = v_i mod 2^b            (lw = ceil(n*b/32) words)
//   high stream : bit (v_i >> b) + i set, L = n + (v_{n-1} >> b) (hw = ceil(L/32) words)
//   payload     : low words then high words, padded to 16 B
// Three device passes: size (thread per block) -> exclusive scan of the 16-B
// sizes -> write (warp per block, streams assembled in shared memory).
#include <algorithm>
#include <vector>

#include "internal.h"
#include "scan.cuh"

namespace griffin {

__device__ __forceinline__ uint32_t floor_log2_nz(uint32_t q) { return 31u - __clz(q); }

__global__ void encode_size_kernel(const uint32_t *__restrict__ doc,
                                   const uint64_t *__restrict__ blk_start,
                                   const uint32_t *__restrict__ blk_n, uint64_t nb,
                                   uint32_t *__restrict__ first, uint2 *__restrict__ meta,
                                   uint32_t *__restrict__ size16) {
  for (uint64_t k = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; k < nb;
       k += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t s = blk_start[k];
    const uint32_t n = blk_n[k];
    const uint32_t x0 = doc[s], xl = doc[s + n - 1];
    const uint32_t vmax = xl - x0;
    // u / n with u = vmax + 1 may need 33 bits only if vmax == 2^32-1, impossible (< N < 2^32-1)
    const uint32_t q = (uint32_t)(((uint64_t)vmax + 1u) / n);
    const uint32_t b = floor_log2_nz(q);
    const uint32_t L = n + (vmax >> b);
    const uint32_t hw = (L + 31u) >> 5;
    const uint32_t lw = low_words(n, b);
    first[k] = x0;
    meta[k] = make_uint2(0u, meta_pack(b, n, hw));
    size16[k] = (lw + hw + 3u) >> 2;
  }
}

// Warp per block.  `stage` = per-warp smem words (>= max payload words, 16-B aligned).
__global__ void __launch_bounds__(256) encode_write_kernel(
    const uint32_t *__restrict__ doc, const uint64_t *__restrict__ blk_start,
    const uint64_t *__restrict__ off16, uint64_t nb, uint32_t stage_words, uint2 *__restrict__ meta,
    uint4 *__restrict__ payload) {
  extern __shared__ uint4 enc_smem[];
  const uint32_t lane = lane_id(), wid = threadIdx.x >> 5;
  uint32_t *stage = reinterpret_cast<uint32_t *>(enc_smem) + wid * stage_words;
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t k = blockIdx.x * (uint64_t)(blockDim.x >> 5) + wid; k < nb; k += nwarps) {
    const uint2 m = meta[k];
    const uint32_t b = meta_b(m.y), n = meta_n(m.y), hw = meta_hw(m.y);
    const uint32_t lw = low_words(n, b);
    const uint32_t n16 = (lw + hw + 3u) >> 2;
    for (uint32_t i = lane; i < n16 * 4; i += 32) stage[i] = 0u;
    __syncwarp();
    const uint64_t s = blk_start[k];
    const uint32_t x0 = doc[s];
    for (uint32_t i = lane; i < n; i += 32) {
      const uint32_t v = doc[s + i] - x0;
      if (b) {
        const uint32_t lo = v & (0xFFFFFFFFu >> (32u - b));
        const uint32_t bit = i * b;
        atomicOr(&stage[bit >> 5], lo << (bit & 31u));
        if ((bit & 31u) + b > 32u) atomicOr(&stage[(bit >> 5) + 1], lo >> (32u - (bit & 31u)));
      }
      const uint32_t hb = (v >> b) + i;
      atomicOr(&stage[lw + (hb >> 5)], 1u << (hb & 31u));
    }
    __syncwarp();
    const uint64_t o = off16[k];
    const uint4 *s4 = reinterpret_cast<const uint4 *>(stage);
    for (uint32_t i = lane; i < n16; i += 32) payload[o + i] = s4[i];
    if (lane == 0) meta[k].x = (uint32_t)o;
    __syncwarp();
  }
}

// tf packing: tf-1 at width w_t, LSB-first, per-term word stream.
__global__ void tf_pack_kernel(const uint32_t *__restrict__ tfs, const uint64_t *__restrict__ blk_start,
                               const uint32_t *__restrict__ blk_n,
                               const uint32_t *__restrict__ blk_term, const TermInfo *__restrict__ terms,
                               const uint64_t *__restrict__ term_post0, uint64_t nb,
                               uint32_t *__restrict__ tfw) {
  const uint32_t lane = lane_id();
  const uint64_t nwarps = (uint64_t)gridDim.x * (blockDim.x >> 5);
  for (uint64_t k = blockIdx.x * (uint64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); k < nb;
       k += nwarps) {
    const TermInfo t = terms[blk_term[k]];
    if (t.tf_w == 0) continue;
    const uint64_t s = blk_start[k];
    const uint64_t p0 = s - term_post0[blk_term[k]];
    const uint32_t n = blk_n[k];
    for (uint32_t i = lane; i < n; i += 32) {
      const uint32_t v = tfs[s + i] - 1u;
      const uint64_t bit = (p0 + i) * t.tf_w;
      uint32_t *w = tfw + t.tf_off + (bit >> 5);
      const uint32_t sh = (uint32_t)(bit & 31u);
      atomicOr(w, v << sh);
      if (sh + t.tf_w > 32u) atomicOr(w + 1, v >> (32u - sh));
    }
  }
}

static uint32_t bits_needed(uint32_t x) {  // smallest w with x < 2^w
  uint32_t w = 0;
  while (w < 32 && (x >> w) != 0) ++w;
  return w;
}

griffin_status encode_index(griffin_index *ix, const uint32_t *h_doc, const uint32_t *h_tfs,
                            const std::vector<uint64_t> &post_off) {
  const uint32_t V = ix->V, B = ix->B;
  const uint64_t P = post_off[V];
  // block table + term info (host)
  std::vector<uint64_t> blk_start;
  std::vector<uint32_t> blk_n, blk_term;
  uint64_t tf_words = 0;
  for (uint32_t t = 0; t < V; ++t) {
    TermInfo &ti = ix->h_terms[t];
    const uint64_t a = post_off[t], e = post_off[t + 1];
    ti.block0 = (uint32_t)blk_start.size();
    ti.df_local = (uint32_t)(e - a);
    ti.nblocks = (uint32_t)((e - a + B - 1) / B);
    uint32_t mx = 1;
    for (uint64_t p = a; p < e; ++p) mx = std::max(mx, h_tfs[p]);
    ti.tf_w = bits_needed(mx - 1u);
    ti.tf_off = tf_words;
    tf_words += ((e - a) * ti.tf_w + 31) / 32;
    for (uint64_t s = a; s < e; s += B) {
      blk_start.push_back(s);
      blk_n.push_back((uint32_t)std::min<uint64_t>(B, e - s));
      blk_term.push_back(t);
    }
  }
  tf_words += 2;  // tf_lookup reads one word past the end
  const uint64_t nb = blk_start.size();
  if (nb >= 0xFFFFFFFFull) {
    set_error("too many blocks for one shard");
    return GRIFFIN_ERR_INVALID_ARG;
  }
  ix->nblocks = nb;
  ix->postings = P;
  ix->tf_words = tf_words;
  cudaStream_t st = ix->stream;
  // staging
  DevBuf d_doc, d_tf, d_bs, d_bn, d_bt, d_size, d_off, d_tmp, d_p0;
  GRIFFIN_CUDA_TRY(d_doc.reserve(std::max<uint64_t>(P, 1) * 4));
  GRIFFIN_CUDA_TRY(d_tf.reserve(std::max<uint64_t>(P, 1) * 4));
  GRIFFIN_CUDA_TRY(d_bs.reserve((nb + 1) * 8));
  GRIFFIN_CUDA_TRY(d_bn.reserve((nb + 1) * 4));
  GRIFFIN_CUDA_TRY(d_bt.reserve((nb + 1) * 4));
  GRIFFIN_CUDA_TRY(d_size.reserve((nb + 1) * 4));
  GRIFFIN_CUDA_TRY(d_off.reserve((nb + 1) * 8));
  GRIFFIN_CUDA_TRY(d_tmp.reserve((nb / kScanTile + 8) * 8));
  GRIFFIN_CUDA_TRY(d_p0.reserve((V + 1) * 8));
  if (P) {
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(d_doc.p, h_doc, P * 4, cudaMemcpyHostToDevice, st));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(d_tf.p, h_tfs, P * 4, cudaMemcpyHostToDevice, st));
  }
  if (nb) {
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(d_bs.p, blk_start.data(), nb * 8, cudaMemcpyHostToDevice, st));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(d_bn.p, blk_n.data(), nb * 4, cudaMemcpyHostToDevice, st));
    GRIFFIN_CUDA_TRY(cudaMemcpyAsync(d_bt.p, blk_term.data(), nb * 4, cudaMemcpyHostToDevice, st));
  }
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(d_p0.p, post_off.data(), (V + 1) * 8, cudaMemcpyHostToDevice, st));
  // index arrays
  GRIFFIN_CUDA_TRY(cudaMalloc(&ix->d_first, (nb + 1) * 4));
  GRIFFIN_CUDA_TRY(cudaMalloc(&ix->d_meta, (nb + 1) * 8));
  GRIFFIN_CUDA_TRY(cudaMalloc(&ix->d_terms, std::max<uint32_t>(V, 1) * sizeof(TermInfo)));
  GRIFFIN_CUDA_TRY(cudaMalloc(&ix->d_tfw, tf_words * 4));
  GRIFFIN_CUDA_TRY(cudaMemsetAsync(ix->d_tfw, 0, tf_words * 4, st));
  GRIFFIN_CUDA_TRY(cudaMemsetAsync(ix->d_first, 0, (nb + 1) * 4, st));
  GRIFFIN_CUDA_TRY(cudaMemsetAsync(ix->d_meta, 0, (nb + 1) * 8, st));
  if (nb) {
    encode_size_kernel<<<(unsigned)std::min<uint64_t>((nb + 255) / 256, (uint64_t)num_sms(ix->device) * 64), 256, 0, st>>>(
        d_doc.as<uint32_t>(), d_bs.as<uint64_t>(), d_bn.as<uint32_t>(), nb, ix->d_first,
        ix->d_meta, d_size.as<uint32_t>());
    GRIFFIN_CUDA_TRY(cudaGetLastError());
    GRIFFIN_CUDA_TRY(exclusive_scan<uint32_t>(d_size.as<uint32_t>(), d_off.as<uint64_t>(), nb,
                                              d_tmp.as<uint64_t>(), st));
  } else {
    GRIFFIN_CUDA_TRY(cudaMemsetAsync(d_off.p, 0, 8, st));
  }
  uint64_t total16 = 0;
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(&total16, d_off.as<uint64_t>() + nb, 8, cudaMemcpyDeviceToHost, st));
  GRIFFIN_CUDA_TRY(cudaStreamSynchronize(st));
  if (total16 >= 0xFFFFFFFFull) {
    set_error("payload exceeds 64 GB per shard");
    return GRIFFIN_ERR_INVALID_ARG;
  }
  ix->payload16 = total16;
  GRIFFIN_CUDA_TRY(cudaMalloc(&ix->d_payload, (total16 + 64) * 16));  // slack for over-reads
  GRIFFIN_CUDA_TRY(cudaMemsetAsync(ix->d_payload, 0, (total16 + 64) * 16, st));
  GRIFFIN_CUDA_TRY(cudaMemcpyAsync(ix->d_terms, ix->h_terms.data(), V * sizeof(TermInfo),
                                   cudaMemcpyHostToDevice, st));
  if (nb) {
    const uint32_t stage_words = ((B * 34u) / 32u + 16u + 3u) & ~3u;
    const size_t smem = (size_t)stage_words * 4 * 8;
    encode_write_kernel<<<(unsigned)std::min<uint64_t>((nb + 7) / 8, (uint64_t)num_sms(ix->device) * 16), 256, smem, st>>>(
        d_doc.as<uint32_t>(), d_bs.as<uint64_t>(), d_off.as<uint64_t>(), nb, stage_words,
        ix->d_meta, ix->d_payload);
    GRIFFIN_CUDA_TRY(cudaGetLastError());
    tf_pack_kernel<<<(unsigned)std::min<uint64_t>((nb + 7) / 8, (uint64_t)num_sms(ix->device) * 16), 256, 0, st>>>(
        d_tf.as<uint32_t>(), d_bs.as<uint64_t>(), d_bn.as<uint32_t>(), d_bt.as<uint32_t>(),
        ix->d_terms, d_p0.as<uint64_t>(), nb, ix->d_tfw);
    GRIFFIN_CUDA_TRY(cudaGetLastError());
  }
  GRIFFIN_CUDA_TRY(cudaStreamSynchronize(st));
  d_doc.release();
  d_tf.release();
  d_bs.release();
  d_bn.release();
  d_bt.release();
  d_size.release();
  d_off.release();
  d_tmp.release();
  d_p0.release();
  return GRIFFIN_OK;
}

}  // namespace griffin
