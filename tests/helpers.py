"""Test-side input builders (no method arithmetic)."""
import numpy as np

from synth import Corpus, QueryLog


def corpus_from_lists(num_docs, lists, tfs=None, doc_lengths=None):
    offs = np.zeros(len(lists) + 1, np.uint64)
    offs[1:] = np.cumsum([len(l) for l in lists])
    docids = np.concatenate([np.asarray(l, np.uint32) for l in lists]) if lists else np.zeros(0, np.uint32)
    if tfs is None:
        tf = np.ones(len(docids), np.uint32)
    else:
        tf = np.concatenate([np.asarray(t, np.uint32) for t in tfs])
    if doc_lengths is None:
        dl = np.full(num_docs, 100, np.uint32)
    else:
        dl = np.asarray(doc_lengths, np.uint32)
    return Corpus(num_docs=num_docs, offsets=offs, docids=docids.astype(np.uint32),
                  tfs=tf.astype(np.uint32), doc_lengths=dl)


def random_corpus(rng, num_docs, num_terms, max_df, max_tf=20):
    lists, tfs = [], []
    for _ in range(num_terms):
        df = int(rng.integers(0, max_df + 1))
        df = min(df, num_docs)
        lst = np.sort(rng.choice(num_docs, size=df, replace=False)).astype(np.uint32)
        lists.append(lst)
        tfs.append(rng.integers(1, max_tf + 1, size=df).astype(np.uint32))
    dl = rng.integers(1, 2000, size=num_docs).astype(np.uint32)
    return corpus_from_lists(num_docs, lists, tfs, dl)


def random_queries(rng, num_terms, nq, max_terms=5):
    offs = [0]
    terms = []
    for _ in range(nq):
        k = int(rng.integers(1, max_terms + 1))
        terms.extend(int(t) for t in rng.integers(0, num_terms, size=k))
        offs.append(len(terms))
    return QueryLog(offsets=np.array(offs, np.uint32), terms=np.array(terms, np.uint32))


def bits_lsb_first(words, nbits):
    """Stream-order bit string of an LSB-first little-endian u32 word array."""
    return "".join(str((int(words[i // 32]) >> (i % 32)) & 1) for i in range(nbits))


def f32_from_hex(h):
    return np.frombuffer(np.uint32(int(h, 16)).tobytes(), np.float32)[0]


def f32_bits(x):
    return int(np.frombuffer(np.float32(x).tobytes(), np.uint32)[0])
