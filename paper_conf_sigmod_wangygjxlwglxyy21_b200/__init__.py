"""B200-native batched IVF k-NN (IVF_FLAT / IVF_SQ8, L2 / IP) -- the data-parallel query hot
path of Milvus (Wang et al., SIGMOD'21), behind the C ABI of include/mv.h.

    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
    ix = Index(d=128, metric="l2", kind="flat", nlist=4096)
    ix.set_centroids(C); ix.add(X, ids)
    D, I = ix.search(Q, k=10, nprobe=16, bitset=None)

There is no CPU fallback: importing the binding loads libmv.so and fails loudly without it.
"""
from ._lib import MV_IP, MV_IVF_FLAT, MV_IVF_PQ, MV_IVF_SQ8, MV_L2, MvError, load  # noqa: F401
from .index import Index, kmeans, merge_topk  # noqa: F401

__all__ = ["Index", "kmeans", "merge_topk", "MvError", "MV_L2", "MV_IP", "MV_IVF_FLAT", "MV_IVF_SQ8"]
