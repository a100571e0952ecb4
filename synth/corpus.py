"""Deterministic synthetic corpora and query logs shaped like the paper's workloads.

Rules ("Generator"):
  G0  every random stream is keyed by (config seed, stream kind, entity id), so the
      output never depends on thread count or generation order.
  G1  doc lengths  dl_d = clamp(round(exp(ln 300 + 0.7 Z)), 1, 65535).
  G2  Zipf list sizes df_r = max(df_min, floor(df_max * r^-alpha)), termID = r-1
      (shape of PAPER.md Fig. 10: most lists 1K..1M, long tail to 26M).
  G3  each list is a uniform random subset of [0, N) drawn by geometric gaps with
      p = df_r / N, plus the planted documents of G5.
  G4  tf = 1 + min(floor(Exp(mean 1.5)), 65534)   (the per-posting "document
      frequency" of P:357-361 / P:1009-1010, read as term frequency).
  G5  query log: term count 2/3/4/5 with weights 27/33/24/10 (Fig. 11, P:1019-1021;
      the 5-term share is assumed), terms drawn without replacement with
      P(r) ~ r^-beta; each query plants m_q = floor(10^U[1,3.5]) documents into all
      of its terms' lists so result sizes reach "several thousands".
  G6  ratio pairs (C3): |S| ~ U[1M, 2M], |R| = |S| / lambda, |R n S| = 10% of |R|
      (the 7 ratio groups of P:858-859 plus lambda = 1000).

Nothing here computes any part of the method (no coding, intersection, scoring).
"""
from __future__ import annotations

import dataclasses
import hashlib
import json
import math
import os
from typing import Dict, List, Optional, Sequence

import numpy as np

SEED_BASE = 0x4752494646494E00  # "GRIFFIN\0" (G0)

# stream kinds (G0)
_K_DL, _K_LIST, _K_TF, _K_QCOUNT, _K_QTERMS, _K_PLANT, _K_PAIR = range(7)


@dataclasses.dataclass
class Corpus:
    """CSR corpus exactly as `griffin_corpus` (include/griffin.h) takes it."""
    num_docs: int
    offsets: np.ndarray      # uint64 [V+1]
    docids: np.ndarray       # uint32, strictly increasing within each list
    tfs: np.ndarray          # uint32, >= 1
    doc_lengths: np.ndarray  # uint32 [N]

    @property
    def num_terms(self) -> int:
        return int(self.offsets.shape[0] - 1)

    @property
    def num_postings(self) -> int:
        return int(self.offsets[-1])

    def df(self) -> np.ndarray:
        return np.diff(self.offsets).astype(np.int64)

    def list(self, t: int) -> np.ndarray:
        return self.docids[self.offsets[t]:self.offsets[t + 1]]

    def tf_list(self, t: int) -> np.ndarray:
        return self.tfs[self.offsets[t]:self.offsets[t + 1]]


@dataclasses.dataclass
class QueryLog:
    offsets: np.ndarray  # uint32 [nq+1]
    terms: np.ndarray    # uint32

    @property
    def num_queries(self) -> int:
        return int(self.offsets.shape[0] - 1)

    def query(self, q: int) -> np.ndarray:
        return self.terms[self.offsets[q]:self.offsets[q + 1]]

    def slice(self, q0: int, q1: int) -> "QueryLog":
        off = self.offsets[q0:q1 + 1].astype(np.int64)
        return QueryLog(offsets=(off - off[0]).astype(np.uint32),
                        terms=self.terms[off[0]:off[-1]].copy())


def _rng(seed: int, kind: int, entity: int) -> np.random.Generator:
    return np.random.default_rng(
        np.random.SeedSequence([seed & 0xFFFFFFFF, (seed >> 32) & 0xFFFFFFFF, kind,
                                entity & 0xFFFFFFFF, entity >> 32]))


def zipf_dfs(alpha: float, df_max: int, df_min: int, num_terms: Optional[int] = None) -> np.ndarray:
    """G2 target list sizes; V defaults to the largest r with df_max*r^-alpha >= df_min."""
    if num_terms is None:
        num_terms = int(math.floor((df_max / df_min) ** (1.0 / alpha)))
    r = np.arange(1, num_terms + 1, dtype=np.float64)
    return np.maximum(df_min, np.floor(df_max * r ** (-alpha))).astype(np.int64)


def _doc_lengths(n: int, seed: int) -> np.ndarray:
    out = np.empty(n, dtype=np.uint32)
    chunk = 1 << 22
    for c0 in range(0, n, chunk):
        c1 = min(n, c0 + chunk)
        z = _rng(seed, _K_DL, c0 // chunk).standard_normal(c1 - c0)
        dl = np.rint(np.exp(math.log(300.0) + 0.7 * z))
        out[c0:c1] = np.clip(dl, 1, 65535).astype(np.uint32)
    return out


def _random_list(n_docs: int, df: int, rng: np.random.Generator) -> np.ndarray:
    """G3: uniform random subset via geometric gaps, p = df/N."""
    if df <= 0:
        return np.empty(0, dtype=np.uint32)
    if df >= n_docs:
        return np.arange(n_docs, dtype=np.uint32)
    p = df / n_docs
    m = int(df + 6 * math.sqrt(df) + 16)
    pos = np.cumsum(rng.geometric(p, size=m).astype(np.int64)) - 1
    while pos[-1] < n_docs - 1:
        more = np.cumsum(rng.geometric(p, size=m).astype(np.int64)) + pos[-1]
        pos = np.concatenate([pos, more])
    return pos[pos < n_docs].astype(np.uint32)


def _tfs(n: int, rng: np.random.Generator) -> np.ndarray:
    """G4."""
    e = np.floor(rng.exponential(1.5, size=n))
    return (1 + np.minimum(e, 65534)).astype(np.uint32)


def make_queries(num_queries: int, num_terms: int, seed: int, beta: float = 0.9,
                 count_weights: Dict[int, float] = None) -> QueryLog:
    """G5 term sets (planting is done by make_corpus)."""
    if count_weights is None:
        count_weights = {2: 27.0, 3: 33.0, 4: 24.0, 5: 10.0}
    ks = np.array(sorted(count_weights), dtype=np.int64)
    w = np.array([count_weights[k] for k in ks], dtype=np.float64)
    w /= w.sum()
    cdf_terms = np.cumsum(np.arange(1, num_terms + 1, dtype=np.float64) ** (-beta))
    cdf_terms /= cdf_terms[-1]
    offs = [0]
    terms: List[int] = []
    for q in range(num_queries):
        rng = _rng(seed, _K_QTERMS, q)
        k = int(ks[np.searchsorted(np.cumsum(w), rng.random(), side="right").clip(0, len(ks) - 1)])
        k = min(k, num_terms)
        chosen: List[int] = []
        while len(chosen) < k:
            t = int(np.searchsorted(cdf_terms, rng.random(), side="right"))
            t = min(t, num_terms - 1)
            if t not in chosen:
                chosen.append(t)
        terms.extend(chosen)
        offs.append(len(terms))
    return QueryLog(offsets=np.array(offs, dtype=np.uint32), terms=np.array(terms, dtype=np.uint32))


def _planted_lists(num_docs: int, seed: int, queries: Optional[QueryLog],
                   plant_log10: Sequence[float], plant_fixed: Optional[int]) -> Dict[int, np.ndarray]:
    """G5 planting: term -> sorted unique docIDs planted into its list."""
    planted: Dict[int, List[np.ndarray]] = {}
    if queries is not None:
        for q in range(queries.num_queries):
            rng = _rng(seed, _K_PLANT, q)
            if plant_fixed is not None:
                m = plant_fixed
            else:
                m = int(math.floor(10 ** rng.uniform(plant_log10[0], plant_log10[1])))
            m = min(m, num_docs)
            if m <= 0:
                continue
            docs = np.unique(rng.integers(0, num_docs, size=m, dtype=np.int64)).astype(np.uint32)
            for t in queries.query(q):
                planted.setdefault(int(t), []).append(docs)
    return {t: np.unique(np.concatenate(v)).astype(np.uint32) for t, v in planted.items()}


def _term_list(t: int, num_docs: int, dfs: np.ndarray, seed: int,
               planted: Dict[int, np.ndarray], extra_lists) -> np.ndarray:
    """G3 (+ G5 planting) for term t; depends only on (seed, t)."""
    if t < len(dfs):
        lst = _random_list(num_docs, int(dfs[t]), _rng(seed, _K_LIST, t))
    else:
        lst = np.asarray(extra_lists[t - len(dfs)], dtype=np.uint32)
    if t in planted:
        lst = np.union1d(lst, planted[t]).astype(np.uint32)
    return lst


# ---- parallel generation (spawned workers; each term's streams depend only
# on (seed, term), so the result is identical to the sequential loop) --------
_PAR = {}


def _par_init(params):
    _PAR.update(params)


def _par_phase1(args):
    wid, terms, tmpdir = args
    g = _PAR
    lens = []
    with open(os.path.join(tmpdir, f"d{wid}.bin"), "wb") as fd, \
            open(os.path.join(tmpdir, f"t{wid}.bin"), "wb") as ft:
        for t in terms:
            lst = _term_list(t, g["num_docs"], g["dfs"], g["seed"], g["planted"], g["extra"])
            fd.write(lst.tobytes())
            ft.write(_tfs(len(lst), _rng(g["seed"], _K_TF, t)).tobytes())
            lens.append(len(lst))
    return wid, lens


def _par_phase2(args):
    wid, terms, tmpdir, offsets, dpath, tpath = args
    src_d = np.fromfile(os.path.join(tmpdir, f"d{wid}.bin"), dtype=np.uint32)
    src_t = np.fromfile(os.path.join(tmpdir, f"t{wid}.bin"), dtype=np.uint32)
    dd = np.load(dpath, mmap_mode="r+")
    tt = np.load(tpath, mmap_mode="r+")
    pos = 0
    for t in terms:
        a, b = int(offsets[t]), int(offsets[t + 1])
        dd[a:b] = src_d[pos:pos + b - a]
        tt[a:b] = src_t[pos:pos + b - a]
        pos += b - a
    dd.flush()
    tt.flush()
    os.remove(os.path.join(tmpdir, f"d{wid}.bin"))
    os.remove(os.path.join(tmpdir, f"t{wid}.bin"))
    return wid


def _make_corpus_parallel(num_docs, dfs, seed, planted, extra_lists, num_terms, outdir, workers):
    import multiprocessing as mp
    # longest-processing-time assignment of terms to workers (size ~ target df)
    size = np.array([int(dfs[t]) if t < len(dfs) else len(extra_lists[t - len(dfs)])
                     for t in range(num_terms)], dtype=np.int64)
    for t, v in planted.items():
        size[t] += len(v)
    order = np.argsort(-size, kind="stable")
    load = np.zeros(workers, np.int64)
    assign: List[List[int]] = [[] for _ in range(workers)]
    for t in order:
        w = int(np.argmin(load))
        assign[w].append(int(t))
        load[w] += size[t] + 64
    for a in assign:
        a.sort()
    params = dict(num_docs=num_docs, dfs=dfs, seed=seed, planted=planted, extra=extra_lists)
    tmpdir = os.path.join(outdir, "tmp")
    os.makedirs(tmpdir, exist_ok=True)
    # fork: make_workload runs this in a fresh single-threaded interpreter
    # (see _generate_into), so forking is safe; a dead worker raises
    # BrokenProcessPool instead of hanging
    from concurrent.futures import ProcessPoolExecutor
    ctx = mp.get_context("fork")
    lens = np.zeros(num_terms, np.uint64)
    with ProcessPoolExecutor(workers, mp_context=ctx, initializer=_par_init,
                             initargs=(params,)) as pool:
        for wid, ls in pool.map(_par_phase1, [(w, assign[w], tmpdir) for w in range(workers)]):
            lens[assign[wid]] = np.array(ls, np.uint64)
        offsets = np.zeros(num_terms + 1, dtype=np.uint64)
        np.cumsum(lens, out=offsets[1:])
        P = int(offsets[-1])
        dpath, tpath = os.path.join(outdir, "docids.npy"), os.path.join(outdir, "tfs.npy")
        np.lib.format.open_memmap(dpath, mode="w+", dtype=np.uint32, shape=(P,)).flush()
        np.lib.format.open_memmap(tpath, mode="w+", dtype=np.uint32, shape=(P,)).flush()
        list(pool.map(_par_phase2, [(w, assign[w], tmpdir, offsets, dpath, tpath)
                                    for w in range(workers)]))
    os.rmdir(tmpdir)
    return offsets


def make_corpus(num_docs: int, dfs: np.ndarray, seed: int,
                queries: Optional[QueryLog] = None,
                plant_log10: Sequence[float] = (1.0, 3.5),
                plant_fixed: Optional[int] = None,
                extra_lists: Optional[List[np.ndarray]] = None,
                outdir: Optional[str] = None, workers: int = 1) -> Corpus:
    """Build the CSR corpus (G1-G5).  `extra_lists` appends explicit docID lists
    (used by the ratio-pair workload G6) as additional terms.  With `outdir`
    and workers > 1 the lists are generated by forked workers straight into
    .npy files there (returned memory-mapped); the content is identical."""
    num_terms = int(len(dfs)) + (len(extra_lists) if extra_lists else 0)
    planted = _planted_lists(num_docs, seed, queries, plant_log10, plant_fixed)
    dl = _doc_lengths(num_docs, seed)
    if outdir is not None and workers > 1:
        offsets = _make_corpus_parallel(num_docs, dfs, seed, planted, extra_lists, num_terms,
                                        outdir, workers)
        np.save(os.path.join(outdir, "offsets.npy"), offsets)
        np.save(os.path.join(outdir, "doc_lengths.npy"), dl)
        return _load_corpus(outdir, num_docs)
    lists: List[np.ndarray] = [_term_list(t, num_docs, dfs, seed, planted, extra_lists)
                               for t in range(num_terms)]
    lens = np.array([len(l) for l in lists], dtype=np.uint64)
    offsets = np.zeros(num_terms + 1, dtype=np.uint64)
    np.cumsum(lens, out=offsets[1:])
    docids = np.empty(int(offsets[-1]), dtype=np.uint32)
    tfs = np.empty(int(offsets[-1]), dtype=np.uint32)
    for t, lst in enumerate(lists):
        a, b = int(offsets[t]), int(offsets[t + 1])
        docids[a:b] = lst
        tfs[a:b] = _tfs(b - a, _rng(seed, _K_TF, t))
    lists.clear()
    return Corpus(num_docs=num_docs, offsets=offsets, docids=docids, tfs=tfs, doc_lengths=dl)


def _load_corpus(d: str, num_docs: int) -> Corpus:
    return Corpus(num_docs=num_docs, offsets=np.load(os.path.join(d, "offsets.npy")),
                  docids=np.load(os.path.join(d, "docids.npy"), mmap_mode="r"),
                  tfs=np.load(os.path.join(d, "tfs.npy"), mmap_mode="r"),
                  doc_lengths=np.load(os.path.join(d, "doc_lengths.npy")))


# Named configurations (BASELINE.json "configs", concretised in SURVEY.md §8(d)).
# `batches`: the query log holds this many consecutive batches of `num_queries`
# (all planted, G5); a benchmark step is one batch and the timed loop rotates
# through them instead of replaying one batch.
CONFIGS = {
    # C1: single 2-term AND query, 100K docs, lists ~10K and ~1K, top-10.
    "c1": dict(num_docs=100_000, alpha=1.0, df_max=50_000, df_min=10,
               num_queries=1, fixed_query=(4, 49), plant_fixed=50, k=10, block=128),
    # C2: 10M docs, 1K-query 2-5 term log, top-10.
    "c2": dict(num_docs=10_000_000, alpha=0.8, df_max=5_000_000, df_min=1_000,
               num_queries=1_000, batches=3, k=10, block=128),
    # C3: 25M docs, GOV2-shaped.
    "c3": dict(num_docs=25_000_000, alpha=0.8, df_max=10_000_000, df_min=1_000,
               num_queries=1_000, k=10, block=128),
    # C4: 50M docs ClueWeb-shaped, sharded over 2/4/8 GPUs.
    "c4": dict(num_docs=50_000_000, alpha=0.8, df_max=30_000_000, df_min=1_000,
               num_queries=10_000, batches=3, k=10, block=128),
    # C5: C4 index, 10K concurrent queries, top-1000, block sweep.
    "c5": dict(num_docs=50_000_000, alpha=0.8, df_max=30_000_000, df_min=1_000,
               num_queries=10_000, batches=3, k=1000, block=128),
    # small CPU/GPU test shapes (several blocks, ragged tails)
    "tiny": dict(num_docs=20_000, alpha=0.8, df_max=8_000, df_min=40,
                 num_queries=64, k=10, block=128),
    "small": dict(num_docs=1_000_000, alpha=0.8, df_max=500_000, df_min=200,
                  num_queries=200, k=10, block=128),
}
# C4 and C5 share one corpus (the same index at top-10 and top-1000)
_CORPUS_OF = {"c4": "c5"}
GENERATOR_VERSION = "g2"   # bump when any rule above changes (invalidates caches)
_CACHE_MIN_POSTINGS = 50_000_000


def cache_dir() -> Optional[str]:
    """On-disk corpus cache (GRIFFIN_SYNTH_CACHE; default /tmp/griffin_synth;
    "" disables).  Large corpora are generated once into .npy files there and
    memory-mapped, so several processes (e.g. one per GPU) share one copy."""
    d = os.environ.get("GRIFFIN_SYNTH_CACHE", "/tmp/griffin_synth")
    return d or None


def make_workload(name: str, seed: Optional[int] = None, num_queries: Optional[int] = None,
                  workers: Optional[int] = None, **overrides):
    """Return (Corpus, QueryLog, cfg) for a named config (C1..C5, tiny, small).
    The log holds cfg["batches"] (default 1) batches of cfg["num_queries"]."""
    cfg = dict(CONFIGS[name])
    cfg.update(overrides)
    if num_queries is not None:
        cfg["num_queries"] = num_queries
    cfg.setdefault("batches", 1)
    base = _CORPUS_OF.get(name, name)
    if seed is None:
        seed = SEED_BASE + (int(base[1]) if base[0] == "c" and base[1:].isdigit() else 99)
    dfs = zipf_dfs(cfg["alpha"], cfg["df_max"], cfg["df_min"], cfg.get("num_terms"))
    if "fixed_query" in cfg:
        qterms = np.array(cfg["fixed_query"], dtype=np.uint32)
        ql = QueryLog(offsets=np.array([0, len(qterms)], dtype=np.uint32), terms=qterms)
    else:
        ql = make_queries(cfg["num_queries"] * cfg["batches"], len(dfs), seed,
                          beta=cfg.get("beta", 0.9))
    cfg["seed"] = seed
    corpus = None
    cdir = cache_dir()
    big = int(dfs.sum()) >= _CACHE_MIN_POSTINGS
    if cdir and big:
        key = json.dumps({k: cfg[k] for k in sorted(cfg) if k not in ("k", "block")},
                         sort_keys=True) + GENERATOR_VERSION
        d = os.path.join(cdir, f"{base}-{hashlib.sha1(key.encode()).hexdigest()[:16]}")
        done = os.path.join(d, "DONE")
        try:
            import fcntl
            os.makedirs(cdir, exist_ok=True)
            with open(os.path.join(cdir, ".lock"), "w") as lk:
                fcntl.flock(lk, fcntl.LOCK_EX)   # one generator per cache; others wait, then mmap
                if not os.path.exists(done):
                    os.makedirs(d, exist_ok=True)
                    nw = workers or min(32, os.cpu_count() or 1)
                    _generate_into(d, name, seed, num_queries, overrides, max(2, nw))
                    open(done, "w").close()
            corpus = _load_corpus(d, cfg["num_docs"])
        except OSError:
            corpus = None   # no usable cache: generate in memory
    if corpus is None:
        corpus = make_corpus(cfg["num_docs"], dfs, seed, queries=ql,
                             plant_fixed=cfg.get("plant_fixed"))
    return corpus, ql, cfg


def sub_corpus(c: Corpus, terms) -> Corpus:
    """The corpus with every list outside `terms` emptied: N, doc lengths (so
    avgdl and every norm) and the kept lists (so their df and idf) are
    unchanged, hence any query over `terms` has the same answer on it.  Lets a
    checker index only the lists a sample of queries touches."""
    keep = sorted(set(int(t) for t in terms))
    df = np.zeros(c.num_terms, np.uint64)
    df[keep] = np.diff(c.offsets)[keep]
    off = np.zeros(c.num_terms + 1, np.uint64)
    np.cumsum(df, out=off[1:])
    docs = np.concatenate([np.asarray(c.list(t)) for t in keep] or [np.zeros(0, np.uint32)])
    tfs = np.concatenate([np.asarray(c.tf_list(t)) for t in keep] or [np.zeros(0, np.uint32)])
    return Corpus(num_docs=c.num_docs, offsets=off, docids=docs.astype(np.uint32),
                  tfs=tfs.astype(np.uint32), doc_lengths=c.doc_lengths)


def _generate_into(d, name, seed, num_queries, overrides, workers):
    """Generate a workload's corpus into cache dir d in a fresh interpreter (the
    caller may hold CUDA contexts and threads, which forked workers must not
    inherit)."""
    import subprocess
    import sys
    arg = json.dumps({"d": d, "name": name, "seed": seed, "num_queries": num_queries,
                      "overrides": overrides, "workers": workers})
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    subprocess.run([sys.executable, "-c", "import sys, json; sys.path.insert(0, sys.argv[2]); "
                    "from synth.corpus import _generate_main; _generate_main(json.loads(sys.argv[1]))",
                    arg, root], check=True)


def _generate_main(a):
    cfg = dict(CONFIGS[a["name"]])
    cfg.update(a["overrides"])
    if a["num_queries"] is not None:
        cfg["num_queries"] = a["num_queries"]
    cfg.setdefault("batches", 1)
    dfs = zipf_dfs(cfg["alpha"], cfg["df_max"], cfg["df_min"], cfg.get("num_terms"))
    ql = make_queries(cfg["num_queries"] * cfg["batches"], len(dfs), a["seed"],
                      beta=cfg.get("beta", 0.9))
    make_corpus(cfg["num_docs"], dfs, a["seed"], queries=ql, plant_fixed=cfg.get("plant_fixed"),
                outdir=a["d"], workers=a["workers"])


def batch_of(ql: QueryLog, cfg, i: int) -> QueryLog:
    """Batch i (mod cfg["batches"]) of a workload's query log."""
    n = cfg["num_queries"]
    i %= cfg.get("batches", 1)
    return ql.slice(i * n, (i + 1) * n)


def make_pair_workload(num_docs: int, s_len: int, ratios: Sequence[float], seed: int,
                       overlap: float = 0.10):
    """G6: one (R, S) pair per ratio; corpus holds only the pair lists.
    Returns (Corpus, QueryLog) with query i = (2i, 2i+1)."""
    lists: List[np.ndarray] = []
    for i, lam in enumerate(ratios):
        rng = _rng(seed, _K_PAIR, i)
        s = _random_list(num_docs, s_len, rng)
        r_len = max(1, int(round(len(s) / lam)))
        n_common = int(round(overlap * r_len))
        common = rng.choice(s, size=min(n_common, len(s)), replace=False) if n_common else np.empty(0, np.uint32)
        rest = _random_list(num_docs, max(1, r_len - len(common)), rng)
        r = np.union1d(common, rest).astype(np.uint32)
        lists.extend([r, s])
    dfs = np.zeros(0, dtype=np.int64)
    corpus = make_corpus(num_docs, dfs, seed, queries=None, extra_lists=lists)
    nq = len(ratios)
    ql = QueryLog(offsets=np.arange(0, 2 * nq + 1, 2, dtype=np.uint32),
                  terms=np.arange(2 * nq, dtype=np.uint32))
    return corpus, ql


def make_ratio_groups(num_docs: int, s_len: int, groups, pairs_per_group: int, seed: int,
                      overlap: float = 0.10):
    """G6 at batch scale: per ratio group one long list S (|S| = s_len) and
    `pairs_per_group` short lists R with |R| = |S|/lambda, lambda log-uniform in
    the group, |R n S| = overlap*|R|.  Returns (Corpus, QueryLog, group_of_query)."""
    lists: List[np.ndarray] = []
    qterms: List[int] = []
    gid: List[int] = []
    for gi, (lo, hi) in enumerate(groups):
        rng = _rng(seed, _K_PAIR, 1_000_000 + gi)
        s = _random_list(num_docs, s_len, rng)
        s_id = len(lists)
        lists.append(s)
        for p in range(pairs_per_group):
            rng = _rng(seed, _K_PAIR, gi * 100_000 + p)
            lam = float(np.exp(rng.uniform(np.log(lo), np.log(hi))))
            r_len = max(1, int(round(len(s) / lam)))
            n_common = int(round(overlap * r_len))
            common = rng.choice(s, size=min(n_common, len(s)), replace=False) if n_common else np.empty(0, np.uint32)
            rest = _random_list(num_docs, max(1, r_len - len(common)), rng)
            lists.append(np.union1d(common, rest).astype(np.uint32))
            qterms.extend([len(lists) - 1, s_id])
            gid.append(gi)
    corpus = make_corpus(num_docs, np.zeros(0, dtype=np.int64), seed, queries=None, extra_lists=lists)
    nq = len(gid)
    ql = QueryLog(offsets=np.arange(0, 2 * nq + 1, 2, dtype=np.uint32),
                  terms=np.array(qterms, dtype=np.uint32))
    return corpus, ql, np.array(gid)
