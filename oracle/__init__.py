"""ORACLE — test infrastructure only (see oracle/oracle.cpp header).

Thin ctypes wrapper around liboracle.so, the plain C++ CPU implementation of the
path.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product package never
imports it, and this package never imports the product package.

Pinned functions: EF encode/decode (Fig. 4, round trip, size bound), SvS
intersection (§2.1.2 example, brute force), BM25 (closed form, hand example),
top-k (definition).  "parity unpinned": the BM25 constants / IDF variant
(paper silent) beyond the textbook closed form.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.cpp")
_SRCS = [_SRC, os.path.join(_HERE, "pfd.cpp")]
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

_u32p = ctypes.POINTER(ctypes.c_uint32)
_u64p = ctypes.POINTER(ctypes.c_uint64)
_f32p = ctypes.POINTER(ctypes.c_float)


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain g++, -ffp-contract=off, no fast-math)."""
    if force or not os.path.exists(_LIB) or any(os.path.getmtime(_LIB) < os.path.getmtime(f)
                                                 for f in _SRCS):
        cmd = ["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
               "-shared", "-pthread", *_SRCS, "-o", _LIB + ".tmp"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_ef_encode.argtypes = [_u32p, ctypes.c_uint32, ctypes.c_uint64, _u32p, _u32p,
                                         ctypes.c_uint64, _u64p, _u32p, ctypes.c_uint64, _u64p]
        lib.oracle_ef_decode.argtypes = [_u32p, _u32p, ctypes.c_uint32, ctypes.c_uint32, _u32p]
        lib.oracle_index_build.restype = ctypes.c_void_p
        lib.oracle_index_build.argtypes = [ctypes.c_uint32, ctypes.c_uint32, _u64p, _u32p, _u32p,
                                           _u32p, ctypes.c_uint32, ctypes.c_double, ctypes.c_double]
        lib.oracle_index_free.argtypes = [ctypes.c_void_p]
        lib.oracle_num_blocks.restype = ctypes.c_uint64
        lib.oracle_num_blocks.argtypes = [ctypes.c_void_p, ctypes.c_uint32]
        lib.oracle_block_streams.argtypes = [ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64,
                                             _u32p, _u32p, _u32p, _u32p, ctypes.c_uint64, _u64p,
                                             _u32p, ctypes.c_uint64, _u64p]
        lib.oracle_decode_list.argtypes = [ctypes.c_void_p, ctypes.c_uint32, _u32p,
                                           ctypes.c_uint64, _u64p]
        lib.oracle_intersect.argtypes = [ctypes.c_void_p, _u32p, ctypes.c_uint32, _u32p,
                                         ctypes.c_uint64, _u64p]
        lib.oracle_query.argtypes = [ctypes.c_void_p, _u32p, ctypes.c_uint32, ctypes.c_uint32,
                                     _u32p, _f32p, _u32p]
        lib.oracle_query_batch.argtypes = [ctypes.c_void_p, ctypes.c_uint32, _u32p, _u32p,
                                           ctypes.c_uint32, _u32p, _f32p, _u32p, ctypes.c_uint32]
        for fn in ("oracle_idf", "oracle_norm"):
            getattr(lib, fn).restype = ctypes.c_float
            getattr(lib, fn).argtypes = [ctypes.c_void_p, ctypes.c_uint32]
        lib.oracle_k1p1.restype = ctypes.c_float
        lib.oracle_k1p1.argtypes = [ctypes.c_void_p]
        lib.oracle_pfd_encode.restype = ctypes.c_uint32
        lib.oracle_pfd_encode.argtypes = [_u32p, ctypes.c_uint32, ctypes.c_int, _u32p,
                                          ctypes.c_uint32, _u32p, _u32p]
        lib.oracle_pfd_decode.argtypes = [_u32p, ctypes.c_uint32, ctypes.c_uint32, _u32p]
        lib.oracle_index_bytes.restype = ctypes.c_uint64
        lib.oracle_index_bytes.argtypes = [ctypes.c_void_p]
        _lib = lib
    return _lib


def _p(a: np.ndarray, ty):
    return a.ctypes.data_as(ty)


def ef_encode(values, U: int):
    """Sequence-level EF encode with explicit universe U (Fig. 4).
    Returns (b, low_words, low_bits, high_words, high_bits)."""
    lib = _load()
    v = np.ascontiguousarray(values, dtype=np.uint32)
    n = len(v)
    cap = n + 64 + (n * 32) // 32 + 4
    low = np.zeros(cap * 2, np.uint32)
    high = np.zeros(cap * 2, np.uint32)
    b = ctypes.c_uint32()
    lb = ctypes.c_uint64()
    hb = ctypes.c_uint64()
    rc = lib.oracle_ef_encode(_p(v, _u32p), n, U, ctypes.byref(b), _p(low, _u32p), len(low),
                              ctypes.byref(lb), _p(high, _u32p), len(high), ctypes.byref(hb))
    if rc:
        raise ValueError("oracle_ef_encode rejected the input")
    return (b.value, low[:(lb.value + 31) // 32].copy(), lb.value,
            high[:(hb.value + 31) // 32].copy(), hb.value)


def ef_decode(low, high, n: int, b: int) -> np.ndarray:
    lib = _load()
    low = np.ascontiguousarray(np.concatenate([np.asarray(low, np.uint32), np.zeros(2, np.uint32)]))
    high = np.ascontiguousarray(np.concatenate([np.asarray(high, np.uint32), np.zeros(2, np.uint32)]))
    out = np.zeros(n, np.uint32)
    lib.oracle_ef_decode(_p(low, _u32p), _p(high, _u32p), n, b, _p(out, _u32p))
    return out


def pfd_encode(x, b: Optional[int] = None):
    """PforDelta block encode (pfd.cpp): returns (words, b, n_exceptions).  The
    block's first docID x[0] is its skip entry and is not in the stream."""
    lib = _load()
    v = np.ascontiguousarray(x, dtype=np.uint32)
    cap = 2 + 2 * len(v) + 8
    out = np.zeros(cap, np.uint32)
    bo, ne = ctypes.c_uint32(), ctypes.c_uint32()
    nw = lib.oracle_pfd_encode(_p(v, _u32p), len(v), -1 if b is None else int(b), _p(out, _u32p),
                               cap, ctypes.byref(bo), ctypes.byref(ne))
    if nw == 0:
        raise ValueError("oracle_pfd_encode rejected the input")
    return out[:nw].copy(), bo.value, ne.value


def pfd_decode(words, first: int, n: int) -> np.ndarray:
    lib = _load()
    w = np.ascontiguousarray(np.concatenate([np.asarray(words, np.uint32), np.zeros(2, np.uint32)]))
    out = np.zeros(n, np.uint32)
    if lib.oracle_pfd_decode(_p(w, _u32p), first, n, _p(out, _u32p)):
        raise ValueError("oracle_pfd_decode: malformed stream")
    return out


def pfd_list_bytes(docids, block_size: int = 128) -> int:
    """PforDelta size of one list in the same block layout as the EF index: per
    block the stream (16-B padded) + an 8-B skip entry (first docID + offset)."""
    x = np.asarray(docids, np.uint32)
    tot = 0
    for s in range(0, len(x), block_size):
        w, _, _ = pfd_encode(x[s:s + block_size])
        tot += ((len(w) * 4 + 15) // 16) * 16 + 8
    return tot


class OracleIndex:
    """The oracle's own index over a CSR corpus (O1-O3)."""

    def __init__(self, corpus, block_size: int = 128, k1: float = 1.2, b: float = 0.75):
        lib = _load()
        self._c = corpus
        self._keep = [np.ascontiguousarray(corpus.offsets, np.uint64),
                      np.ascontiguousarray(corpus.docids, np.uint32),
                      np.ascontiguousarray(corpus.tfs, np.uint32),
                      np.ascontiguousarray(corpus.doc_lengths, np.uint32)]
        off, doc, tf, dl = self._keep
        self.h = lib.oracle_index_build(corpus.num_docs, corpus.num_terms, _p(off, _u64p),
                                        _p(doc, _u32p), _p(tf, _u32p), _p(dl, _u32p),
                                        block_size, k1, b)
        if not self.h:
            raise ValueError("oracle_index_build failed")
        self._keep = None
        self.block_size = block_size

    def __del__(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.oracle_index_free(self.h)
            self.h = None

    def num_blocks(self, t: int) -> int:
        return int(_load().oracle_num_blocks(self.h, t))

    def block_streams(self, t: int, blk: int):
        """(first, n, b, low_words, low_bits, high_words, high_bits) of one block."""
        lib = _load()
        cap = 4096
        low = np.zeros(cap, np.uint32)
        high = np.zeros(cap, np.uint32)
        first, n, b = ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint32()
        lb, hb = ctypes.c_uint64(), ctypes.c_uint64()
        rc = lib.oracle_block_streams(self.h, t, blk, ctypes.byref(first), ctypes.byref(n),
                                      ctypes.byref(b), _p(low, _u32p), cap, ctypes.byref(lb),
                                      _p(high, _u32p), cap, ctypes.byref(hb))
        if rc:
            raise IndexError((t, blk))
        return (first.value, n.value, b.value, low[:(lb.value + 31) // 32].copy(), lb.value,
                high[:(hb.value + 31) // 32].copy(), hb.value)

    def decode_list(self, t: int) -> np.ndarray:
        n = int(self._c.offsets[t + 1] - self._c.offsets[t])
        out = np.zeros(max(n, 1), np.uint32)
        cnt = ctypes.c_uint64()
        rc = _load().oracle_decode_list(self.h, t, _p(out, _u32p), len(out), ctypes.byref(cnt))
        if rc:
            raise ValueError("decode_list")
        return out[:cnt.value]

    def intersect(self, terms) -> np.ndarray:
        t = np.ascontiguousarray(terms, np.uint32)
        cap = int(min(self._c.df()[t].min(), 1 << 31)) + 1
        out = np.zeros(cap, np.uint32)
        cnt = ctypes.c_uint64()
        rc = _load().oracle_intersect(self.h, _p(t, _u32p), len(t), _p(out, _u32p), cap,
                                      ctypes.byref(cnt))
        if rc:
            raise ValueError("intersect")
        return out[:cnt.value]

    def query(self, terms, k: int) -> Tuple[np.ndarray, np.ndarray, int]:
        t = np.ascontiguousarray(terms, np.uint32)
        d = np.zeros(k, np.uint32)
        s = np.zeros(k, np.float32)
        c = ctypes.c_uint32()
        rc = _load().oracle_query(self.h, _p(t, _u32p), len(t), k, _p(d, _u32p), _p(s, _f32p),
                                  ctypes.byref(c))
        if rc:
            raise ValueError("query")
        return d, s, c.value

    def query_batch(self, qlog, k: int, nthreads: int = 1):
        nq = qlog.num_queries
        off = np.ascontiguousarray(qlog.offsets, np.uint32)
        terms = np.ascontiguousarray(qlog.terms, np.uint32)
        d = np.zeros(nq * k, np.uint32)
        s = np.zeros(nq * k, np.float32)
        c = np.zeros(nq, np.uint32)
        rc = _load().oracle_query_batch(self.h, nq, _p(off, _u32p), _p(terms, _u32p), k,
                                        _p(d, _u32p), _p(s, _f32p), _p(c, _u32p), nthreads)
        if rc:
            raise ValueError("query_batch")
        return d.reshape(nq, k), s.reshape(nq, k), c

    def idf(self, t: int) -> float:
        return float(_load().oracle_idf(self.h, t))

    def norm(self, d: int) -> float:
        return float(_load().oracle_norm(self.h, d))

    def k1p1(self) -> float:
        return float(_load().oracle_k1p1(self.h))

    def nbytes(self) -> int:
        return int(_load().oracle_index_bytes(self.h))
