"""Seeded synthetic workload generator (SURVEY.md §8(d) rules G0-G6).

This module is shared INPUT infrastructure: it produces the corpora and query
logs that both the CUDA path and the CPU oracle consume.  It holds none of the
method's arithmetic (no Elias-Fano coding, no intersection, no BM25, no top-k)
and imports neither ``oracle`` nor the product package.
"""
from .corpus import (Corpus, QueryLog, CONFIGS, make_corpus, make_queries,
                     make_workload, make_pair_workload, make_ratio_groups, zipf_dfs,
                     batch_of, cache_dir, sub_corpus)

__all__ = ["Corpus", "QueryLog", "CONFIGS", "make_corpus", "make_queries",
           "make_workload", "make_pair_workload", "make_ratio_groups", "zipf_dfs",
           "batch_of", "cache_dir", "sub_corpus"]
