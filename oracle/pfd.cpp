// ORACLE — test infrastructure only (see oracle.cpp's header for the rules).
//
// PforDelta block codec, the paper's comparison scheme (§2.1.1, P:285-311;
// Fig. 3), written out step by step for the NEXT-3 comparator
// (SURVEY.md §8(f)).  Plain sequential C++; shares nothing with the CUDA path.
//
// One block holds n docIDs x_0 < ... < x_{n-1}; x_0 is the block's skip entry
// (stored next to the block, like the Elias-Fano block's first docID) and the
// m = n-1 d-gaps g_i = x_i - x_{i-1} (i = 1..n-1; Fig. 3: 9 docIDs, 8 gaps) are
// coded:
//   b      given, or (reading P2) the number of bits of the largest "regular"
//          value, the regular values being the ceil(0.9 m) smallest gaps
//          ("a majority of elements (e.g., 90%) ... b is determined by the
//          smallest number of bits to represent the largest regular value",
//          P:297-300).
//   slots  m slots of b bits: a regular gap is its value; an exception (gap >=
//          2^b) holds the distance to the next exception minus one ("uses b
//          bits to store the position of the next exception (in a linked list
//          manner)"; Fig. 3: "next 3", "next 1"); the last one holds
//          0.  Reading P3: when two consecutive exceptions are more than 2^b
//          apart, the gap 2^b after the earlier one is made a (forced)
//          exception so every link fits in b bits.
//   values the exceptions' gaps, uncompressed u32, "at the end of the whole
//          compressed sequence", last exception first (Fig. 3
//          prints 47 68 42 for exceptions 42, 68, 47).
// Stream (u32 words, LSB-first bit packing as the EF streams, reading A3):
//   word 0: first exception position (m if none) | n_exc << 10 | b << 20
//   then ceil(m*b/32) words of slots, then n_exc exception words.

#include <algorithm>
#include <cstdint>
#include <vector>

namespace {

uint32_t bits_of(uint32_t v) {   // bits needed to represent v (v >= 1)
  uint32_t r = 0;
  while (v) {
    ++r;
    v /= 2;
  }
  return r;
}

uint32_t choose_b(const std::vector<uint32_t> &gaps) {
  const uint32_t m = (uint32_t)gaps.size();
  if (m == 0) return 0;
  std::vector<uint32_t> s = gaps;
  std::sort(s.begin(), s.end());
  const uint32_t regular = (9 * m + 9) / 10;   // ceil(0.9 m)
  return bits_of(s[regular - 1]);
}

}  // namespace

extern "C" {

// Encode one block.  b_in < 0: choose b by the 90% rule.  Returns the number of
// words written (0 on bad input / capacity); b and the exception count out.
uint32_t oracle_pfd_encode(const uint32_t *x, uint32_t n, int b_in, uint32_t *out, uint32_t cap,
                           uint32_t *b_out, uint32_t *nexc_out) {
  if (n == 0 || n > 1024) return 0;
  std::vector<uint32_t> gaps;
  for (uint32_t i = 1; i < n; ++i) {
    if (x[i] <= x[i - 1]) return 0;
    gaps.push_back(x[i] - x[i - 1]);
  }
  const uint32_t m = (uint32_t)gaps.size();
  const uint32_t b = b_in >= 0 ? (uint32_t)b_in : choose_b(gaps);
  if (m > 0 && (b < 1 || b > 32)) return 0;
  // exceptions: gaps that do not fit in b bits
  std::vector<bool> is_exc(m, false);
  for (uint32_t i = 0; i < m; ++i)
    if (b < 32 && gaps[i] >= (1u << b)) is_exc[i] = true;
  // forced exceptions: consecutive exceptions at most 2^b apart (reading P3)
  if (b < 32) {
    const uint64_t maxd = 1ull << b;
    int64_t prev = -1;
    for (uint32_t i = 0; i < m; ++i) {
      if (!is_exc[i]) continue;
      while (prev >= 0 && (uint64_t)(i - prev) > maxd) {
        prev = prev + (int64_t)maxd;
        is_exc[(uint32_t)prev] = true;
      }
      prev = i;
    }
  }
  std::vector<uint32_t> pos;
  for (uint32_t i = 0; i < m; ++i)
    if (is_exc[i]) pos.push_back(i);
  const uint32_t nexc = (uint32_t)pos.size();
  std::vector<uint32_t> slot(m);
  for (uint32_t i = 0; i < m; ++i) slot[i] = gaps[i];
  for (uint32_t e = 0; e < nexc; ++e) slot[pos[e]] = e + 1 < nexc ? pos[e + 1] - pos[e] - 1 : 0u;
  const uint32_t slot_words = (uint32_t)(((uint64_t)m * b + 31) / 32);
  const uint32_t words = 1 + slot_words + nexc;
  if (words > cap) return 0;
  for (uint32_t w = 0; w < words; ++w) out[w] = 0;
  out[0] = (nexc ? pos[0] : m) | (nexc << 10) | (b << 20);
  for (uint32_t i = 0; i < m; ++i)
    for (uint32_t k = 0; k < b; ++k) {
      const uint64_t bit = (uint64_t)i * b + k;
      if ((slot[i] >> k) & 1u) out[1 + bit / 32] |= 1u << (bit % 32);
    }
  for (uint32_t e = 0; e < nexc; ++e) out[1 + slot_words + e] = gaps[pos[nexc - 1 - e]];
  if (b_out) *b_out = b;
  if (nexc_out) *nexc_out = nexc;
  return words;
}

// Decode one block: n docIDs from the stream and the skip entry x_0.
int oracle_pfd_decode(const uint32_t *in, uint32_t first, uint32_t n, uint32_t *x) {
  if (n == 0) return -1;
  const uint32_t m = n - 1;
  const uint32_t fe = in[0] & 1023u, nexc = (in[0] >> 10) & 1023u, b = (in[0] >> 20) & 63u;
  const uint32_t slot_words = (uint32_t)(((uint64_t)m * b + 31) / 32);
  std::vector<uint32_t> g(m, 0);
  for (uint32_t i = 0; i < m; ++i) {
    uint32_t v = 0;
    for (uint32_t k = 0; k < b; ++k) {
      const uint64_t bit = (uint64_t)i * b + k;
      v |= ((in[1 + bit / 32] >> (bit % 32)) & 1u) << k;
    }
    g[i] = v;
  }
  // walk the exception list, patching each slot with its stored value
  uint32_t p = fe;
  for (uint32_t e = 0; e < nexc; ++e) {
    if (p >= m) return -1;
    const uint32_t link = g[p];
    g[p] = in[1 + slot_words + (nexc - 1 - e)];
    p = p + link + 1;
  }
  x[0] = first;
  for (uint32_t i = 1; i < n; ++i) x[i] = x[i - 1] + g[i - 1];
  return 0;
}

}  // extern "C"
