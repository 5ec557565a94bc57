"""oracle -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation (numpy, float64) of what the hot path
computes: batched IVF_FLAT / IVF_SQ8 k-NN search (L2 and inner product) with an exclusion
bitset and per-query top-k including k > 1024, plus brute-force exact k-NN and the shard
merge.  It follows PAPER.md (Milvus, SIGMOD'21) step by step; every function cites the
passage it follows.  Readings of passages the paper leaves silent or garbled are listed in
DESIGN.md §2 and marked "reading" here.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with the CUDA path
(``paper_conf_sigmod_wangygjxlwglxyy21_b200``) and neither imports the other.

Parity status of each function (DESIGN.md §2 lists the pins):
  exact_knn, assign, sq8_train/encode/decode, probe, IvfIndex.search, topk_rounds,
  merge_topk, recall -- all pinned by tests/test_oracle_*.py.
  multi.py: range_bitset, partition_plan, partition_search (strategy E),
  multivector_scores / multivector_topk (§4.2) -- pinned by tests/test_oracle_multi.py.
  kmeans.py: lloyd_step, kmeans, sse -- pinned by tests/test_oracle_kmeans.py.
  pq.py: pq_encode, pq_decode, IvfPqIndex -- pinned by tests/test_oracle_pq.py.
"""
from .ivf import (  # noqa: F401
    FLAT, IP, L2, SQ8, IvfIndex, assign, bit_is_set, distances, exact_knn, merge_topk, pad_value, probe,
    recall_at_k, select_topk, sq8_decode, sq8_encode, sq8_train, topk_rounds,
)
from .multi import (  # noqa: F401,E402
    multivector_scores, multivector_topk, partition_plan, partition_search, range_bitset,
)
from . import kmeans as km  # noqa: F401,E402
from .pq import IvfPqIndex, pq_decode, pq_encode  # noqa: F401,E402
