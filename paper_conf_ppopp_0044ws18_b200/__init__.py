"""B200-native Griffin-GPU conjunctive query path — thin Python binding.

Argument marshalling only: every step of the path (EF encode, EF decode,
merge-path / galloping intersection, BM25, top-k, shard merge) runs in the CUDA
kernels of ``libgriffin.so`` behind the C ABI of ``include/griffin.h``; the
functions here carry the same names as the C entry points.  PyTorch is used only
for device memory, streams and ``torch.distributed`` (see ``sharded.py``).

There is no CPU fallback: importing this package without a built
``libgriffin.so`` raises, and building an index without a B200 returns
GRIFFIN_ERR_UNSUPPORTED.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Tuple

import numpy as np

from . import _build

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = _build.LIB

STATUS = {0: "GRIFFIN_OK", 1: "GRIFFIN_ERR_INVALID_ARG", 2: "GRIFFIN_ERR_UNSORTED",
          3: "GRIFFIN_ERR_OOM", 4: "GRIFFIN_ERR_CUDA", 5: "GRIFFIN_ERR_NCCL",
          6: "GRIFFIN_ERR_UNSUPPORTED"}
MODE_AUTO, MODE_MERGE, MODE_GALLOP = 0, 1, 2
EXCHANGE_AUTO, EXCHANGE_NCCL_ALLGATHER, EXCHANGE_PEER, EXCHANGE_NCCL_SLICED = 0, 1, 2, 3
MAX_TERMS, MAX_K = 16, 4096


class GriffinError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class _Corpus(ctypes.Structure):
    _fields_ = [("num_docs", ctypes.c_uint32), ("num_terms", ctypes.c_uint32),
                ("list_offsets", ctypes.c_void_p), ("docids", ctypes.c_void_p),
                ("tfs", ctypes.c_void_p), ("doc_lengths", ctypes.c_void_p)]


class _Opts(ctypes.Structure):
    _fields_ = [("block_size", ctypes.c_uint32), ("bm25_k1", ctypes.c_double),
                ("bm25_b", ctypes.c_double), ("gallop_ratio", ctypes.c_uint32),
                ("device", ctypes.c_int32), ("shard_index", ctypes.c_uint32),
                ("num_shards", ctypes.c_uint32), ("gallop_ratio_decoded", ctypes.c_uint32),
                ("num_gpus", ctypes.c_uint32), ("devices", ctypes.c_void_p),
                ("exchange", ctypes.c_int32)]


class Stats(ctypes.Structure):
    _fields_ = [("shard_index", ctypes.c_uint32), ("num_shards", ctypes.c_uint32),
                ("doc_base", ctypes.c_uint32), ("doc_end", ctypes.c_uint32),
                ("block_size", ctypes.c_uint32), ("num_terms", ctypes.c_uint32),
                ("num_postings", ctypes.c_uint64), ("num_blocks", ctypes.c_uint64),
                ("payload_bytes", ctypes.c_uint64), ("skip_bytes", ctypes.c_uint64),
                ("tf_bytes", ctypes.c_uint64), ("device_bytes", ctypes.c_uint64)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class Profile(ctypes.Structure):
    _fields_ = [("ms_plan", ctypes.c_double), ("ms_intersect", ctypes.c_double),
                ("ms_compact", ctypes.c_double), ("ms_topk", ctypes.c_double),
                ("ms_merge", ctypes.c_double), ("launches_intersect", ctypes.c_uint64),
                ("launches_total", ctypes.c_uint64), ("alg_bytes", ctypes.c_uint64),
                ("payload_bytes", ctypes.c_uint64), ("decoded_postings", ctypes.c_uint64),
                ("survivors", ctypes.c_uint64), ("ms_decode", ctypes.c_double),
                ("launches_decode", ctypes.c_uint64), ("dec_alg_bytes", ctypes.c_uint64),
                ("dec_payload_bytes", ctypes.c_uint64), ("dec_postings", ctypes.c_uint64),
                ("c8d_bytes", ctypes.c_uint64), ("dec_c8d_bytes", ctypes.c_uint64),
                ("arena_postings", ctypes.c_uint64), ("merge_units", ctypes.c_uint64),
                ("merge_elems", ctypes.c_uint64), ("gallop_units", ctypes.c_uint64),
                ("gallop_elems", ctypes.c_uint64),
                ("bitmap_units", ctypes.c_uint64), ("bitmap_elems", ctypes.c_uint64),
                ("bitand_units", ctypes.c_uint64), ("bitand_words", ctypes.c_uint64)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


_lib = None
_vp, _u32, _u64, _i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32
_SIGS = {
    "griffin_index_build": [ctypes.POINTER(_Corpus), ctypes.POINTER(_Opts), ctypes.POINTER(_vp)],
    "griffin_index_destroy": [_vp],
    "griffin_index_stats": [_vp, ctypes.POINTER(Stats)],
    "griffin_query": [_vp, _vp, _u32, _u32, _vp, _vp, _vp],
    "griffin_query_batch": [_vp, _u32, _vp, _vp, _u32, _vp, _vp, _vp],
    "griffin_reserve": [_vp, _u32, _vp, _vp, _u32],
    "griffin_query_batch_device": [_vp, _u32, _vp, _vp, _u32, _u32, _vp, _vp, _vp],
    "griffin_sync_status": [_vp],
    "griffin_workspace_create": [_vp, ctypes.POINTER(_vp)],
    "griffin_workspace_destroy": [_vp, _vp],
    "griffin_workspace_reserve": [_vp, _vp, _u32, _vp, _vp, _u32],
    "griffin_query_batch_device_ws": [_vp, _vp, _u32, _vp, _vp, _u32, _u32, _vp, _vp, _vp],
    "griffin_workspace_sync_status": [_vp, _vp],
    "griffin_query_batch_submit": [_vp, _vp, _u32, _vp, _vp, _u32, _vp],
    "griffin_query_batch_collect": [_vp, _vp, _vp, _vp, _vp],
    "griffin_query_batch_results": [_vp, _vp, ctypes.POINTER(_vp), ctypes.POINTER(_vp),
                                    ctypes.POINTER(_vp)],
    "griffin_merge_topk_device": [_vp, _u32, _u32, _u32, _vp, _vp, _vp, _vp, _vp],
    "griffin_keys_to_results_device": [_vp, _u32, _u32, _vp, _vp, _vp, _vp, _vp],
    "griffin_set_mode": [_vp, ctypes.c_int],
    "griffin_set_profiling": [_vp, ctypes.c_int],
    "griffin_set_reuse": [_vp, ctypes.c_int],
    "griffin_set_nextgeq": [_vp, ctypes.c_int],
    "griffin_set_bitmap": [_vp, _u32],
    "griffin_set_probe_chunk": [_vp, _u32],
    "griffin_set_entry_budget": [_vp, _u64],
    "griffin_pfd_build": [_vp, _u32, ctypes.c_int, _vp],
    "griffin_pfd_stats": [_vp, _vp],
    "griffin_pfd_block_stream": [_vp, _u32, _u32, _vp, _vp, _vp, _u32, _vp],
    "griffin_pfd_decode_list": [_vp, _u32, _vp, _u64, _vp],
    "griffin_pfd_decode_all": [_vp, _u32, _vp, _vp, _vp, _vp],
    "griffin_get_profile": [_vp, ctypes.POINTER(Profile)],
    "griffin_reset_profile": [_vp],
    "griffin_shard_range": [_u32, _u32, _u32, ctypes.POINTER(_u32), ctypes.POINTER(_u32)],
    "griffin_merge_path_split": [_vp, _u32, _vp, _u32, _u32, ctypes.c_int, ctypes.POINTER(_u32),
                                 ctypes.POINTER(_u32)],
    "griffin_debug_block_streams": [_vp, _u32, _u64, ctypes.POINTER(_u32), ctypes.POINTER(_u32),
                                    ctypes.POINTER(_u32), _vp, _u64, ctypes.POINTER(_u64), _vp,
                                    _u64, ctypes.POINTER(_u64)],
    "griffin_debug_decode_list": [_vp, _u32, _vp, _u64, ctypes.POINTER(_u64)],
    "griffin_debug_decode_all": [_vp, ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                                 ctypes.POINTER(_u64), ctypes.POINTER(_u64), ctypes.POINTER(_u64)],
    "griffin_debug_intersect": [_vp, _vp, _u32, ctypes.c_int, _vp, _u64, ctypes.POINTER(_u64)],
}


def _nccl_hint():
    """Point the library's run-time NCCL load (NCCL exchanges only) at the copy
    PyTorch uses (the nvidia-nccl wheel) when present: the first libnccl.so.2
    loaded into a process is the one every later user binds to."""
    if os.environ.get("GRIFFIN_NCCL_LIBRARY"):
        return
    try:
        import importlib.util
        spec = importlib.util.find_spec("nvidia.nccl")
        for d in (spec.submodule_search_locations or []) if spec else []:
            p = os.path.join(d, "lib", "libnccl.so.2")
            if os.path.exists(p):
                os.environ["GRIFFIN_NCCL_LIBRARY"] = p
                return
    except (ImportError, ValueError):
        pass


def load_library():
    """Load libgriffin.so (building it in-tree with nvcc if it is missing or stale)."""
    global _lib
    if _lib is None:
        _nccl_hint()
        alt = os.environ.get("GRIFFIN_LIBRARY")   # A/B runs: another build of the same ABI
        if alt:
            lib = ctypes.CDLL(alt)
        else:
            if not os.path.exists(LIB_PATH) or _build._stale():
                _build.build()
            lib = ctypes.CDLL(LIB_PATH)
        for name, args in _SIGS.items():
            fn = getattr(lib, name, None)
            if fn is None and alt:   # an older A/B build may predate some entry points
                continue
            if fn is None:
                raise GriffinError(f"libgriffin.so lacks {name}")
            fn.argtypes = args
            fn.restype = ctypes.c_int
        lib.griffin_index_destroy.restype = None
        lib.griffin_workspace_destroy.restype = None
        if hasattr(lib, "griffin_pfd_destroy"):
            lib.griffin_pfd_destroy.restype = None
            lib.griffin_pfd_destroy.argtypes = [_vp]
        lib.griffin_last_error.restype = ctypes.c_char_p
        lib.griffin_last_error.argtypes = []
        _lib = lib
    return _lib


def griffin_last_error() -> str:
    return load_library().griffin_last_error().decode()


def _check(status: int):
    if status != 0:
        raise GriffinError(status, griffin_last_error())


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def _submit(ih, wh, offsets, terms, k, stream):
    off = np.ascontiguousarray(offsets, np.uint32)
    t = np.ascontiguousarray(terms, np.uint32)
    st = ctypes.c_void_p(stream.cuda_stream if stream is not None else 0)
    _check(load_library().griffin_query_batch_submit(ih, wh, len(off) - 1, _ptr(off), _ptr(t), k,
                                                     st))
    return (len(off) - 1, k)


class _ViewKeeper:
    """Base object of zero-copy result views: keeps the owning workspace (or
    index) alive and defers its close() until the last view is gone, so a view
    never points into freed pinned memory.  Its contents are only meaningful
    until the next submit on that workspace (the library keeps superseded
    staging buffers allocated until the workspace is freed)."""

    def __init__(self, owner):
        # a workspace's views also pin its index (destroying the index frees
        # every workspace of it)
        self.owners = [owner] + ([owner.index] if hasattr(owner, "index") else [])
        for o in self.owners:
            o._live_views += 1

    def __del__(self):
        for o in self.owners:
            o._live_views -= 1
            if o._live_views == 0 and o._close_deferred:
                o._close_deferred = False
                o.close()


def _collect(ih, wh, pend, out=None, owner=None):
    """out: optional (docids u32 >= nq*k, scores f32 >= nq*k, counts u32 >= nq)
    arrays to fill (a serving loop reuses them instead of faulting in fresh
    pages every batch), or "view": no copy — read-only numpy views of the
    workspace's pinned staging (griffin_query_batch_results), valid until the
    next submit on that workspace; the views keep `owner` alive."""
    nq, k = pend
    if isinstance(out, str) and out == "view":
        lib = load_library()
        _check(lib.griffin_query_batch_collect(ih, wh, None, None, None))
        pd, ps, pc = _vp(), _vp(), _vp()
        _check(lib.griffin_query_batch_results(ih, wh, ctypes.byref(pd), ctypes.byref(ps),
                                               ctypes.byref(pc)))
        keeper = _ViewKeeper(owner) if owner is not None else None

        def view(p, n, ct, dt):
            if n == 0:
                return np.zeros(0, dt)
            buf = (ct * n).from_address(p.value)
            buf._keeper = keeper   # numpy holds buf as the array's base
            a = np.frombuffer(buf, dtype=dt)
            a.flags.writeable = False
            return a
        return (view(pd, nq * k, ctypes.c_uint32, np.uint32).reshape(nq, k),
                view(ps, nq * k, ctypes.c_float, np.float32).reshape(nq, k),
                view(pc, nq, ctypes.c_uint32, np.uint32))
    if out is None:
        d = np.zeros(max(nq * k, 1), np.uint32)
        s = np.zeros(max(nq * k, 1), np.float32)
        c = np.zeros(max(nq, 1), np.uint32)
    else:
        d, s, c = out
        if (d.dtype != np.uint32 or s.dtype != np.float32 or c.dtype != np.uint32
                or d.size < nq * k or s.size < nq * k or c.size < nq
                or not (d.flags.c_contiguous and s.flags.c_contiguous and c.flags.c_contiguous)):
            raise ValueError("out arrays: contiguous u32[nq*k], f32[nq*k], u32[nq] required")
        d, s, c = d.reshape(-1), s.reshape(-1), c.reshape(-1)
    _check(load_library().griffin_query_batch_collect(ih, wh, _ptr(d), _ptr(s), _ptr(c)))
    return d[:nq * k].reshape(nq, k), s[:nq * k].reshape(nq, k), c[:nq]


def _dptr(t) -> ctypes.c_void_p:
    """device pointer of a torch tensor (plumbing only)"""
    return ctypes.c_void_p(t.data_ptr())


def griffin_shard_range(num_docs: int, num_shards: int, shard: int) -> Tuple[int, int]:
    a, b = _u32(), _u32()
    _check(load_library().griffin_shard_range(num_docs, num_shards, shard, ctypes.byref(a),
                                               ctypes.byref(b)))
    return a.value, b.value


def griffin_merge_path_split(a, b, diag: int, fixup: bool = True) -> Tuple[int, int]:
    a = np.ascontiguousarray(a, np.uint32)
    b = np.ascontiguousarray(b, np.uint32)
    i, j = _u32(), _u32()
    _check(load_library().griffin_merge_path_split(_ptr(a), len(a), _ptr(b), len(b), diag,
                                                    int(fixup), ctypes.byref(i), ctypes.byref(j)))
    return i.value, j.value


class GriffinIndex:
    """Owns one `griffin_index`: one docID-range shard on one device, or with
    num_gpus > 1 (or an explicit exchange) a handle over num_gpus shards on
    `devices` whose queries return the global top-k (include/griffin.h)."""

    def __init__(self, corpus, block_size: int = 128, k1: float = 1.2, b: float = 0.75,
                 gallop_ratio: int = 0, device: int = -1, shard_index: int = 0,
                 num_shards: int = 1, gallop_ratio_decoded: int = 0, num_gpus: int = 1,
                 devices=None, exchange: int = EXCHANGE_AUTO):
        lib = load_library()
        self._arrays = [np.ascontiguousarray(corpus.offsets, np.uint64),
                        np.ascontiguousarray(corpus.docids, np.uint32),
                        np.ascontiguousarray(corpus.tfs, np.uint32),
                        np.ascontiguousarray(corpus.doc_lengths, np.uint32)]
        off, doc, tf, dl = self._arrays
        c = _Corpus(corpus.num_docs, len(off) - 1, off.ctypes.data, doc.ctypes.data,
                    tf.ctypes.data, dl.ctypes.data)
        devs = None if devices is None else np.ascontiguousarray(devices, np.int32)
        o = _Opts(block_size, k1, b, gallop_ratio, device, shard_index, num_shards,
                  gallop_ratio_decoded, num_gpus, devs.ctypes.data if devs is not None else None,
                  exchange)
        h = ctypes.c_void_p()
        status = lib.griffin_index_build(ctypes.byref(c), ctypes.byref(o), ctypes.byref(h))
        self._arrays = None
        _check(status)
        self.h = h
        self.num_docs = corpus.num_docs
        self.num_terms = len(off) - 1
        self.block_size = block_size

    _live_views = 0
    _close_deferred = False

    def close(self):
        if self._live_views:   # zero-copy result views still point into its staging
            self._close_deferred = True
            return
        if getattr(self, "h", None) and _lib is not None:
            _lib.griffin_index_destroy(self.h)
            self.h = None

    def __del__(self):
        self.close()

    # -- host-buffer API
    def griffin_index_stats(self) -> dict:
        s = Stats()
        _check(load_library().griffin_index_stats(self.h, ctypes.byref(s)))
        return s.as_dict()

    def griffin_query(self, terms, k: int):
        t = np.ascontiguousarray(terms, np.uint32)
        d = np.zeros(k, np.uint32)
        s = np.zeros(k, np.float32)
        c = np.zeros(1, np.uint32)
        _check(load_library().griffin_query(self.h, _ptr(t), len(t), k, _ptr(d), _ptr(s), _ptr(c)))
        return d, s, int(c[0])

    def griffin_query_batch(self, offsets, terms, k: int, out=None):
        """out: optional (docids u32 >= nq*k, scores f32 >= nq*k, counts u32 >= nq)
        arrays to fill, reused across calls (no fresh pages per batch)."""
        off = np.ascontiguousarray(offsets, np.uint32)
        t = np.ascontiguousarray(terms, np.uint32)
        nq = len(off) - 1
        if out is None:
            d = np.zeros(nq * k, np.uint32)
            s = np.zeros(nq * k, np.float32)
            c = np.zeros(max(nq, 1), np.uint32)
        else:
            d, s, c = (x.reshape(-1) for x in out)
            if (d.dtype != np.uint32 or s.dtype != np.float32 or c.dtype != np.uint32
                    or d.size < nq * k or s.size < nq * k or c.size < nq):
                raise ValueError("out arrays: u32[nq*k], f32[nq*k], u32[nq] required")
        _check(load_library().griffin_query_batch(self.h, nq, _ptr(off), _ptr(t), k, _ptr(d),
                                                  _ptr(s), _ptr(c)))
        return d[:nq * k].reshape(nq, k), s[:nq * k].reshape(nq, k), c[:nq]

    # -- device-buffer API (torch tensors carry the device memory)
    def griffin_reserve(self, offsets, terms, k: int):
        off = np.ascontiguousarray(offsets, np.uint32)
        t = np.ascontiguousarray(terms, np.uint32)
        _check(load_library().griffin_reserve(self.h, len(off) - 1, _ptr(off), _ptr(t), k))

    def griffin_query_batch_device(self, d_offsets, d_terms, max_terms: int, k: int, d_out_keys,
                                   d_out_counts, stream=None):
        nq = d_offsets.numel() - 1
        st = ctypes.c_void_p(stream.cuda_stream if stream is not None else 0)
        _check(load_library().griffin_query_batch_device(
            self.h, nq, _dptr(d_offsets), _dptr(d_terms), max_terms, k, _dptr(d_out_keys),
            _dptr(d_out_counts), st))

    def griffin_sync_status(self):
        _check(load_library().griffin_sync_status(self.h))

    def griffin_workspace_create(self) -> "GriffinWorkspace":
        return GriffinWorkspace(self)

    # -- pipelined host-buffer batch on the index's own workspace (ws = NULL)
    def griffin_query_batch_submit(self, offsets, terms, k: int, stream=None):
        self._pend = _submit(self.h, None, offsets, terms, k, stream)

    def griffin_query_batch_collect(self, out=None):
        out = _collect(self.h, None, getattr(self, "_pend", (0, 1)), out, owner=self)
        self._pend = (0, 1)
        return out

    def griffin_merge_topk_device(self, num_runs: int, nq: int, k: int, d_keys, d_counts,
                                  d_out_keys, d_out_counts, stream=None):
        st = ctypes.c_void_p(stream.cuda_stream if stream is not None else 0)
        _check(load_library().griffin_merge_topk_device(self.h, num_runs, nq, k, _dptr(d_keys),
                                                        _dptr(d_counts), _dptr(d_out_keys),
                                                        _dptr(d_out_counts), st))

    def griffin_keys_to_results_device(self, nq: int, k: int, d_keys, d_counts, d_docids,
                                       d_scores, stream=None):
        st = ctypes.c_void_p(stream.cuda_stream if stream is not None else 0)
        _check(load_library().griffin_keys_to_results_device(self.h, nq, k, _dptr(d_keys),
                                                             _dptr(d_counts), _dptr(d_docids),
                                                             _dptr(d_scores), st))

    # -- configuration / instrumentation
    def griffin_set_mode(self, mode: int):
        _check(load_library().griffin_set_mode(self.h, mode))

    def griffin_set_reuse(self, mode: int):
        """0 off (fused decode every round), 1 on (decode hot lists once per batch), 2 auto."""
        _check(load_library().griffin_set_reuse(self.h, mode))

    def griffin_set_bitmap(self, inv: int):
        """Dense lists (density >= 1/inv) decoded once per batch into a bitvector
        + rank instead of the docID arena; 0 off, default 32."""
        _check(load_library().griffin_set_bitmap(self.h, inv))

    def griffin_set_nextgeq(self, on: bool):
        """Gallop into compressed lists by EF NextGEQ (True, default) or block decode."""
        _check(load_library().griffin_set_nextgeq(self.h, int(on)))

    def griffin_set_probe_chunk(self, chunk: int):
        """Probe-pass survivors per unit (multiple of 32 in [32, B]; 0 = B)."""
        _check(load_library().griffin_set_probe_chunk(self.h, chunk))

    def griffin_set_entry_budget(self, entries: int):
        """Intermediate entries per workspace buffer (0 = exact per-batch bound)."""
        _check(load_library().griffin_set_entry_budget(self.h, entries))

    def griffin_set_profiling(self, on):
        """False/0 off, True/1 events + counters, 2 events only, 3 counters only."""
        _check(load_library().griffin_set_profiling(self.h, int(on)))

    def griffin_get_profile(self) -> dict:
        p = Profile()
        _check(load_library().griffin_get_profile(self.h, ctypes.byref(p)))
        return p.as_dict()

    def griffin_reset_profile(self):
        _check(load_library().griffin_reset_profile(self.h))

    # -- parity hooks
    def griffin_debug_block_streams(self, term: int, blk: int):
        cap = 4096
        low = np.zeros(cap, np.uint32)
        high = np.zeros(cap, np.uint32)
        f, n, b = _u32(), _u32(), _u32()
        lb, hb = _u64(), _u64()
        _check(load_library().griffin_debug_block_streams(
            self.h, term, blk, ctypes.byref(f), ctypes.byref(n), ctypes.byref(b), _ptr(low), cap,
            ctypes.byref(lb), _ptr(high), cap, ctypes.byref(hb)))
        return (f.value, n.value, b.value, low[:(lb.value + 31) // 32].copy(), lb.value,
                high[:(hb.value + 31) // 32].copy(), hb.value)

    def griffin_debug_decode_list(self, term: int) -> np.ndarray:
        cap = self.griffin_index_stats()["num_postings"] + 1
        out = np.zeros(cap, np.uint32)
        n = _u64()
        _check(load_library().griffin_debug_decode_list(self.h, term, _ptr(out), cap,
                                                         ctypes.byref(n)))
        return out[:n.value]

    def griffin_debug_decode_all(self, iters: int = 3):
        ms, cs, post, by = ctypes.c_double(), _u64(), _u64(), _u64()
        _check(load_library().griffin_debug_decode_all(self.h, iters, ctypes.byref(ms),
                                                        ctypes.byref(cs), ctypes.byref(post),
                                                        ctypes.byref(by)))
        return dict(ms=ms.value, checksum=cs.value, postings=post.value, bytes=by.value)

    def griffin_debug_intersect(self, terms, mode: int = MODE_AUTO,
                                cap: Optional[int] = None) -> np.ndarray:
        t = np.ascontiguousarray(terms, np.uint32)
        if cap is None:
            cap = self.griffin_index_stats()["num_postings"] + 1
        out = np.zeros(max(cap, 1), np.uint32)
        n = _u64()
        _check(load_library().griffin_debug_intersect(self.h, _ptr(t), len(t), mode, _ptr(out),
                                                       cap, ctypes.byref(n)))
        return out[:n.value]


class GriffinWorkspace:
    """An extra query workspace of an index (griffin_workspace): lets several
    batches be in flight on different streams."""

    def __init__(self, index: GriffinIndex):
        self.index = index
        h = ctypes.c_void_p()
        _check(load_library().griffin_workspace_create(index.h, ctypes.byref(h)))
        self.h = h

    _live_views = 0
    _close_deferred = False

    def close(self):
        if self._live_views:   # zero-copy result views still point into its staging
            self._close_deferred = True
            return
        if getattr(self, "h", None) and _lib is not None and getattr(self.index, "h", None):
            _lib.griffin_workspace_destroy(self.index.h, self.h)
        self.h = None

    def __del__(self):
        self.close()

    def griffin_workspace_reserve(self, offsets, terms, k: int):
        off = np.ascontiguousarray(offsets, np.uint32)
        t = np.ascontiguousarray(terms, np.uint32)
        _check(load_library().griffin_workspace_reserve(self.index.h, self.h, len(off) - 1,
                                                        _ptr(off), _ptr(t), k))

    def griffin_query_batch_device_ws(self, d_offsets, d_terms, max_terms: int, k: int,
                                      d_out_keys, d_out_counts, stream=None):
        nq = d_offsets.numel() - 1
        st = ctypes.c_void_p(stream.cuda_stream if stream is not None else 0)
        _check(load_library().griffin_query_batch_device_ws(
            self.index.h, self.h, nq, _dptr(d_offsets), _dptr(d_terms), max_terms, k,
            _dptr(d_out_keys), _dptr(d_out_counts), st))

    def griffin_workspace_sync_status(self):
        _check(load_library().griffin_workspace_sync_status(self.index.h, self.h))

    # -- pipelined host-buffer batch (griffin_query_batch_submit / _collect)
    def griffin_query_batch_submit(self, offsets, terms, k: int, stream=None):
        self._pend = _submit(self.index.h, self.h, offsets, terms, k, stream)

    def griffin_query_batch_collect(self, out=None):
        out = _collect(self.index.h, self.h, getattr(self, "_pend", (0, 1)), out, owner=self)
        self._pend = (0, 1)
        return out


class PfdStats(ctypes.Structure):
    _fields_ = [("block_size", ctypes.c_uint32), ("num_blocks", ctypes.c_uint64),
                ("num_postings", ctypes.c_uint64), ("payload_bytes", ctypes.c_uint64),
                ("skip_bytes", ctypes.c_uint64), ("exceptions", ctypes.c_uint64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class GriffinPfd:
    """PforDelta-coded copy of a corpus' docID lists on the device (griffin_pfd_*,
    the NEXT-3 comparator codec; not on the query path)."""

    def __init__(self, corpus, block_size: int = 128, device: int = -1):
        lib = load_library()
        arrs = [np.ascontiguousarray(corpus.offsets, np.uint64),
                np.ascontiguousarray(corpus.docids, np.uint32),
                np.ascontiguousarray(corpus.tfs, np.uint32),
                np.ascontiguousarray(corpus.doc_lengths, np.uint32)]
        off, doc, tf, dl = arrs
        c = _Corpus(corpus.num_docs, len(off) - 1, off.ctypes.data, doc.ctypes.data,
                    tf.ctypes.data, dl.ctypes.data)
        h = ctypes.c_void_p()
        _check(lib.griffin_pfd_build(ctypes.byref(c), block_size, device, ctypes.byref(h)))
        self.h = h
        self.block_size = block_size

    def close(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.griffin_pfd_destroy(self.h)
            self.h = None

    def __del__(self):
        self.close()

    def griffin_pfd_stats(self) -> dict:
        s = PfdStats()
        _check(load_library().griffin_pfd_stats(self.h, ctypes.byref(s)))
        return s.as_dict()

    def griffin_pfd_block_stream(self, term: int, block: int):
        """(first, n, stream words) of one block."""
        cap = 4 * self.block_size + 16
        w = np.zeros(cap, np.uint32)
        f, n, nw = ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint32()
        _check(load_library().griffin_pfd_block_stream(self.h, term, block, ctypes.byref(f),
                                                       ctypes.byref(n), _ptr(w), cap,
                                                       ctypes.byref(nw)))
        return f.value, n.value, w[:nw.value].copy()

    def griffin_pfd_decode_list(self, term: int, cap: int) -> np.ndarray:
        out = np.zeros(max(cap, 1), np.uint32)
        n = _u64()
        _check(load_library().griffin_pfd_decode_list(self.h, term, _ptr(out), len(out),
                                                      ctypes.byref(n)))
        return out[:n.value]

    def griffin_pfd_decode_all(self, iters: int = 3) -> dict:
        ms = ctypes.c_double()
        p, b, ck = _u64(), _u64(), _u64()
        _check(load_library().griffin_pfd_decode_all(self.h, iters, ctypes.byref(ms),
                                                     ctypes.byref(p), ctypes.byref(b),
                                                     ctypes.byref(ck)))
        return {"ms": ms.value, "postings": p.value, "bytes": b.value, "checksum": ck.value}


__all__ = ["GriffinIndex", "GriffinWorkspace", "GriffinPfd", "GriffinError", "load_library", "griffin_last_error",
           "griffin_shard_range", "griffin_merge_path_split", "MODE_AUTO", "MODE_MERGE",
           "MODE_GALLOP", "EXCHANGE_AUTO", "EXCHANGE_NCCL_ALLGATHER", "EXCHANGE_PEER",
           "EXCHANGE_NCCL_SLICED", "LIB_PATH"]
