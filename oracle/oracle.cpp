// ORACLE — test infrastructure only.
//
// A plain, slow, obviously-correct CPU implementation of the Griffin-GPU
// conjunctive query path (Liu, Wang, Swanson, PPoPP'18; /root/reference/PAPER.md,
// cited as P:<line>).  Only tests/, __graft_entry__.smoke() and bench.py's
// cpu_baseline / --impl reference legs may load this library.  It shares no code,
// header, table or constant generator with the CUDA path
// (paper_conf_ppopp_0044ws18_b200/csrc) and neither side includes the other.
//
// Build: g++ -O2 -std=c++17 -ffp-contract=off -fPIC -shared (no -ffast-math), see
// oracle/__init__.py.  Every float operation in scoring is one IEEE-754 binary32
// operation, round-to-nearest-even, with no FMA contraction.
//
// Steps:
//   O1 global BM25 statistics (readings A12-A14)
//   O2 fixed-size blocks
//   O3 Elias-Fano encode per block (Fig. 4, reading A1-A3, A6)
//   O4 sequential EF decode
//   O5 SvS intersection with std::set_intersection
//   O6 BM25 score in canonical (df asc, termID asc) order (A12-A15)
//   O7 top-k by a full std::sort of unique keys ("brute-force" sort, A16)
//
// Parity pins: see tests/test_oracle.py.  "parity unpinned": the BM25 constants
// k1=1.2, b=0.75 and the IDF variant (paper silent) — pinned only
// against the textbook closed form, not against any number printed in the paper.

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <thread>
#include <vector>

namespace {

// floor(log2(q)) for q >= 1, by repeated halving (no bit tricks).
uint32_t floor_log2_u64(uint64_t q) {
  uint32_t r = 0;
  while (q >= 2) {
    q /= 2;
    ++r;
  }
  return r;
}

void put_bit(std::vector<uint32_t> &words, uint64_t pos) {
  uint64_t w = pos / 32;
  if (words.size() <= w) words.resize(w + 1, 0u);
  words[w] |= (1u << (pos % 32));
}

uint32_t get_bit(const uint32_t *words, uint64_t pos) {
  return (words[pos / 32] >> (pos % 32)) & 1u;
}

// O3: EF-encode values v[0..n) (non-decreasing, v[n-1] < U) with
// b = floor(log2(U / n)) (integer division, reading A1).  Low stream: bits
// [i*b, (i+1)*b) hold v_i mod 2^b.  High stream: the unary-coded d-gaps of the
// high parts h_i = v_i >> b (Fig. 4 caption): for each i, (h_i - h_{i-1})
// zeros followed by a one — i.e. bit h_i + i is set.  Both streams LSB-first in
// little-endian 32-bit words (reading A3).
struct EFSeq {
  uint32_t b = 0;
  uint64_t low_bits = 0, high_bits = 0;
  std::vector<uint32_t> low, high;
};

EFSeq ef_encode_seq(const uint32_t *v, uint32_t n, uint64_t U) {
  EFSeq e;
  e.b = floor_log2_u64(U / n);
  e.low_bits = (uint64_t)n * e.b;
  e.low.assign((e.low_bits + 31) / 32, 0u);
  for (uint32_t i = 0; i < n; ++i)
    for (uint32_t j = 0; j < e.b; ++j)
      if ((v[i] >> j) & 1u) put_bit(e.low, (uint64_t)i * e.b + j);
  // unary d-gaps, written literally as "0^gap 1"
  uint64_t pos = 0;
  uint64_t prev_high = 0;
  for (uint32_t i = 0; i < n; ++i) {
    uint64_t h = (uint64_t)(v[i] >> e.b);
    uint64_t gap = h - prev_high;
    pos += gap;                        // `gap` zeros
    put_bit(e.high, pos);              // the terminating one
    pos += 1;
    prev_high = h;
  }
  e.high_bits = pos;                   // = n + h_{n-1}
  e.high.resize((e.high_bits + 31) / 32, 0u);
  return e;
}

// O4: sequential decode.  Scan the high stream; the k-th one at position p means
// the accumulated number of zeros is p - k, i.e. h_k = p - k.
void ef_decode_seq(const uint32_t *low, const uint32_t *high, uint32_t n, uint32_t b,
                   uint32_t *out) {
  uint64_t p = 0;
  for (uint32_t k = 0; k < n; ++k) {
    while (get_bit(high, p) == 0) ++p;
    uint64_t h = p - k;
    uint32_t lo = 0;
    for (uint32_t j = 0; j < b; ++j)
      lo |= get_bit(low, (uint64_t)k * b + j) << j;
    out[k] = (uint32_t)((h << b) | lo);
    ++p;
  }
}

struct Block {
  uint32_t first, n, b;
  uint64_t low_off, high_off;     // word offsets into Index::words
  uint64_t low_bits, high_bits;
};

struct Index {
  uint32_t N = 0, V = 0, B = 128;
  std::vector<uint64_t> list_off;          // CSR copy of the postings' positions
  std::vector<uint32_t> tfs;               // raw tf per posting (CSR order)
  std::vector<uint64_t> term_block0;       // [V+1] first block of each term
  std::vector<Block> blocks;
  std::vector<uint32_t> words;
  std::vector<float> idf, norm;
  float k1p1 = 0.f;
};

}  // namespace

extern "C" {

// ---- sequence-level codec (Fig. 4 reproduction; explicit U) -----------------
// Returns 0 on success, -1 if a capacity is too small or the input is invalid.
int oracle_ef_encode(const uint32_t *v, uint32_t n, uint64_t U, uint32_t *b_out,
                     uint32_t *low, uint64_t low_cap, uint64_t *low_bits,
                     uint32_t *high, uint64_t high_cap, uint64_t *high_bits) {
  if (n == 0 || U < n) return -1;
  for (uint32_t i = 0; i < n; ++i)
    if ((uint64_t)v[i] >= U || (i && v[i] < v[i - 1])) return -1;
  EFSeq e = ef_encode_seq(v, n, U);
  if (e.low.size() > low_cap || e.high.size() > high_cap) return -1;
  *b_out = e.b;
  *low_bits = e.low_bits;
  *high_bits = e.high_bits;
  std::copy(e.low.begin(), e.low.end(), low);
  std::copy(e.high.begin(), e.high.end(), high);
  return 0;
}

int oracle_ef_decode(const uint32_t *low, const uint32_t *high, uint32_t n, uint32_t b,
                     uint32_t *out) {
  ef_decode_seq(low, high, n, b, out);
  return 0;
}

// ---- index (O1-O3) -------------------------------------------------------------
void *oracle_index_build(uint32_t num_docs, uint32_t num_terms, const uint64_t *offsets,
                         const uint32_t *docids, const uint32_t *tfs,
                         const uint32_t *doc_lengths, uint32_t block_size, double k1,
                         double bm25_b) {
  if (num_docs == 0 || block_size == 0) return nullptr;
  Index *ix = new Index();
  ix->N = num_docs;
  ix->V = num_terms;
  ix->B = block_size;
  ix->list_off.assign(offsets, offsets + num_terms + 1);
  uint64_t total = offsets[num_terms];
  ix->tfs.assign(tfs, tfs + total);
  // O1: global statistics in double, rounded once to float (A13, A14)
  uint64_t sum_dl = 0;
  for (uint32_t d = 0; d < num_docs; ++d) sum_dl += doc_lengths[d];
  double avgdl = (double)sum_dl / (double)num_docs;
  double K1 = (double)k1, Bb = (double)bm25_b;
  ix->norm.resize(num_docs);
  for (uint32_t d = 0; d < num_docs; ++d)
    ix->norm[d] = (float)(K1 * ((1.0 - Bb) + Bb * ((double)doc_lengths[d] / avgdl)));
  ix->idf.resize(num_terms);
  for (uint32_t t = 0; t < num_terms; ++t) {
    double df = (double)(offsets[t + 1] - offsets[t]);
    ix->idf[t] = (float)std::log1p(((double)num_docs - df + 0.5) / (df + 0.5));
  }
  ix->k1p1 = (float)(K1 + 1.0);
  // O2 + O3: blocks of B postings, EF per block on v_i = x_i - first, U = v_{n-1}+1
  ix->term_block0.assign(num_terms + 1, 0);
  std::vector<uint32_t> v;
  for (uint32_t t = 0; t < num_terms; ++t) {
    ix->term_block0[t] = ix->blocks.size();
    uint64_t a = offsets[t], e = offsets[t + 1];
    for (uint64_t s = a; s < e; s += block_size) {
      uint32_t n = (uint32_t)std::min<uint64_t>(block_size, e - s);
      uint32_t first = docids[s];
      v.resize(n);
      for (uint32_t i = 0; i < n; ++i) v[i] = docids[s + i] - first;
      EFSeq q = ef_encode_seq(v.data(), n, (uint64_t)v[n - 1] + 1);
      Block bl;
      bl.first = first;
      bl.n = n;
      bl.b = q.b;
      bl.low_off = ix->words.size();
      bl.low_bits = q.low_bits;
      ix->words.insert(ix->words.end(), q.low.begin(), q.low.end());
      bl.high_off = ix->words.size();
      bl.high_bits = q.high_bits;
      ix->words.insert(ix->words.end(), q.high.begin(), q.high.end());
      ix->blocks.push_back(bl);
    }
  }
  ix->term_block0[num_terms] = ix->blocks.size();
  return ix;
}

void oracle_index_free(void *h) { delete static_cast<Index *>(h); }

uint64_t oracle_num_blocks(void *h, uint32_t t) {
  Index *ix = static_cast<Index *>(h);
  return ix->term_block0[t + 1] - ix->term_block0[t];
}

// Logical streams of block `blk` of term `t` (for encoder parity).
int oracle_block_streams(void *h, uint32_t t, uint64_t blk, uint32_t *first, uint32_t *n,
                         uint32_t *b, uint32_t *low, uint64_t low_cap, uint64_t *low_bits,
                         uint32_t *high, uint64_t high_cap, uint64_t *high_bits) {
  Index *ix = static_cast<Index *>(h);
  if (t >= ix->V) return -1;
  uint64_t gb = ix->term_block0[t] + blk;
  if (gb >= ix->term_block0[t + 1]) return -1;
  const Block &bl = ix->blocks[gb];
  uint64_t lw = (bl.low_bits + 31) / 32, hw = (bl.high_bits + 31) / 32;
  if (lw > low_cap || hw > high_cap) return -1;
  *first = bl.first;
  *n = bl.n;
  *b = bl.b;
  *low_bits = bl.low_bits;
  *high_bits = bl.high_bits;
  std::copy(ix->words.begin() + bl.low_off, ix->words.begin() + bl.low_off + lw, low);
  std::copy(ix->words.begin() + bl.high_off, ix->words.begin() + bl.high_off + hw, high);
  return 0;
}

}  // extern "C"

namespace {

// O4 over a whole list.
std::vector<uint32_t> decode_list(const Index &ix, uint32_t t) {
  std::vector<uint32_t> out;
  out.reserve(ix.list_off[t + 1] - ix.list_off[t]);
  std::vector<uint32_t> tmp;
  for (uint64_t gb = ix.term_block0[t]; gb < ix.term_block0[t + 1]; ++gb) {
    const Block &bl = ix.blocks[gb];
    tmp.resize(bl.n);
    ef_decode_seq(&ix.words[bl.low_off], &ix.words[bl.high_off], bl.n, bl.b, tmp.data());
    for (uint32_t i = 0; i < bl.n; ++i) out.push_back(bl.first + tmp[i]);
  }
  return out;
}

// O5 term order: distinct terms by (df asc, termID asc).
std::vector<uint32_t> svs_order(const Index &ix, const uint32_t *terms, uint32_t nterms) {
  std::vector<uint32_t> ts(terms, terms + nterms);
  std::sort(ts.begin(), ts.end());
  ts.erase(std::unique(ts.begin(), ts.end()), ts.end());
  std::sort(ts.begin(), ts.end(), [&](uint32_t a, uint32_t b) {
    uint64_t da = ix.list_off[a + 1] - ix.list_off[a];
    uint64_t db = ix.list_off[b + 1] - ix.list_off[b];
    return da != db ? da < db : a < b;
  });
  return ts;
}

// O5: SvS with std::set_intersection; stop when all lists are used or R is empty
// (P:234-240).  Returns the decoded lists too (for tf lookup).
std::vector<uint32_t> svs(const Index &ix, const std::vector<uint32_t> &order,
                          std::vector<std::vector<uint32_t>> *lists) {
  std::vector<uint32_t> R;
  for (size_t j = 0; j < order.size(); ++j) {
    lists->push_back(decode_list(ix, order[j]));
    if (j == 0) {
      R = lists->back();
    } else {
      std::vector<uint32_t> out;
      std::set_intersection(R.begin(), R.end(), lists->back().begin(),
                            lists->back().end(), std::back_inserter(out));
      R.swap(out);
    }
    if (R.empty()) break;
  }
  return R;
}

uint32_t f32_bits(float f) {
  uint32_t u;
  std::memcpy(&u, &f, 4);
  return u;
}

// O6 + O7 for one query.
int run_query(const Index &ix, const uint32_t *terms, uint32_t nterms, uint32_t k,
              uint32_t *out_docids, float *out_scores, uint32_t *out_count) {
  if (nterms == 0 || k == 0) return -1;
  for (uint32_t i = 0; i < nterms; ++i)
    if (terms[i] >= ix.V) return -1;
  std::vector<uint32_t> order = svs_order(ix, terms, nterms);
  std::vector<std::vector<uint32_t>> lists;
  std::vector<uint32_t> R = svs(ix, order, &lists);
  if (lists.size() < order.size()) R.clear();  // stopped early on an empty R
  std::vector<uint64_t> keys;
  keys.reserve(R.size());
  for (uint32_t d : R) {
    float s = 0.0f;
    for (size_t j = 0; j < order.size(); ++j) {
      uint32_t t = order[j];
      const std::vector<uint32_t> &L = lists[j];
      size_t pos = std::lower_bound(L.begin(), L.end(), d) - L.begin();
      float tf_f = (float)ix.tfs[ix.list_off[t] + pos];
      float num = tf_f * ix.k1p1;
      float den = tf_f + ix.norm[d];
      float w = ix.idf[t] * (num / den);
      s = (j == 0) ? w : s + w;
    }
    keys.push_back(((uint64_t)f32_bits(s) << 32) | (uint64_t)(0xFFFFFFFFu - d));
  }
  std::sort(keys.begin(), keys.end(), [](uint64_t a, uint64_t b) { return a > b; });
  uint32_t c = (uint32_t)std::min<size_t>(k, keys.size());
  for (uint32_t i = 0; i < k; ++i) {
    if (i < c) {
      uint32_t sb = (uint32_t)(keys[i] >> 32);
      float s;
      std::memcpy(&s, &sb, 4);
      out_docids[i] = 0xFFFFFFFFu - (uint32_t)(keys[i] & 0xFFFFFFFFu);
      out_scores[i] = s;
    } else {
      out_docids[i] = 0xFFFFFFFFu;
      out_scores[i] = -INFINITY;
    }
  }
  *out_count = c;
  return 0;
}

}  // namespace

extern "C" {

int oracle_decode_list(void *h, uint32_t t, uint32_t *out, uint64_t cap, uint64_t *n) {
  Index *ix = static_cast<Index *>(h);
  if (t >= ix->V) return -1;
  std::vector<uint32_t> L = decode_list(*ix, t);
  *n = L.size();
  if (L.size() > cap) return -1;
  std::copy(L.begin(), L.end(), out);
  return 0;
}

// O5 only: the docID set of the conjunctive query.
int oracle_intersect(void *h, const uint32_t *terms, uint32_t nterms, uint32_t *out,
                     uint64_t cap, uint64_t *count) {
  Index *ix = static_cast<Index *>(h);
  if (nterms == 0) return -1;
  for (uint32_t i = 0; i < nterms; ++i)
    if (terms[i] >= ix->V) return -1;
  std::vector<uint32_t> order = svs_order(*ix, terms, nterms);
  std::vector<std::vector<uint32_t>> lists;
  std::vector<uint32_t> R = svs(*ix, order, &lists);
  if (lists.size() < order.size()) R.clear();
  *count = R.size();
  if (R.size() > cap) return -1;
  std::copy(R.begin(), R.end(), out);
  return 0;
}

int oracle_query(void *h, const uint32_t *terms, uint32_t nterms, uint32_t k,
                 uint32_t *out_docids, float *out_scores, uint32_t *out_count) {
  return run_query(*static_cast<Index *>(h), terms, nterms, k, out_docids, out_scores,
                   out_count);
}

// Queries split round-robin over `nthreads` std::threads (the baseline's
// all-cores mode); each query is still the plain single-threaded run_query.
int oracle_query_batch(void *h, uint32_t nq, const uint32_t *qoff, const uint32_t *terms,
                       uint32_t k, uint32_t *out_docids, float *out_scores,
                       uint32_t *out_counts, uint32_t nthreads) {
  const Index &ix = *static_cast<Index *>(h);
  if (nthreads == 0) nthreads = 1;
  std::atomic<int> err{0};
  auto work = [&](uint32_t tid) {
    for (uint32_t q = tid; q < nq; q += nthreads) {
      int rc = run_query(ix, terms + qoff[q], qoff[q + 1] - qoff[q], k,
                         out_docids + (uint64_t)q * k, out_scores + (uint64_t)q * k,
                         out_counts + q);
      if (rc) err = rc;
    }
  };
  std::vector<std::thread> th;
  for (uint32_t i = 1; i < nthreads; ++i) th.emplace_back(work, i);
  work(0);
  for (auto &t : th) t.join();
  return err.load();
}

float oracle_idf(void *h, uint32_t t) { return static_cast<Index *>(h)->idf[t]; }
float oracle_norm(void *h, uint32_t d) { return static_cast<Index *>(h)->norm[d]; }
float oracle_k1p1(void *h) { return static_cast<Index *>(h)->k1p1; }
uint64_t oracle_index_bytes(void *h) {
  Index *ix = static_cast<Index *>(h);
  return ix->words.size() * 4ull + ix->blocks.size() * 8ull;
}

}  // extern "C"
