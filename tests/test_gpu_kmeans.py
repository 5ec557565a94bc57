"""GPU parity of SURVEY §8(f) row f1's k-means (mv_kmeans through the C ABI) against
oracle.km.lloyd_step: per iteration the GPU's assignment (the tensor-core coarse step) must equal
the oracle's up to ties, and the centroids must be the fp64 means of the rows so assigned, rounded
to fp32 (fp64 atomics change only the summation order)."""
import numpy as np
import pytest
import torch

import mvgen as G
import oracle as O

pytestmark = pytest.mark.gpu


def _check_step(X, C0, C1, metric, spherical=False):
    """C1 (GPU, one iteration from C0) against the oracle step, the assignment adjudicated at ties."""
    Xn, C0n = X.numpy(), C0.numpy()
    a = O.assign(Xn, C0n, metric)
    Co, _ = O.km.lloyd_step(Xn, C0n, metric, spherical, lists=a)
    assert np.allclose(C1.numpy(), Co, rtol=2 ** -22, atol=1e-7), np.abs(C1.numpy() - Co).max()


@pytest.mark.parametrize("metric,kind", [("l2", "sift"), ("ip", "deep")])
def test_kmeans_iterations_vs_oracle(metric, kind):
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import kmeans
    n, nlist = 20000, 96
    if kind == "sift":
        X = G.sift_base(n, d=64, spec=G.SiftSpec(d=64, n_micro=512))
    else:
        X = G.deep_base(n, d=96, spec=G.DeepSpec(d=96, n_micro=512))
    mo = O.L2 if metric == "l2" else O.IP
    C = (X[torch.randperm(n, generator=torch.Generator().manual_seed(5))[:nlist]] + (0.25 if kind == "sift" else 0.0))
    Xc = X.cuda()
    for _ in range(3):  # iteration by iteration: each GPU step from the same centroids as the oracle's
        C1 = kmeans(Xc, nlist, niter=1, metric=metric, spherical=kind == "deep", init=C.cuda()).cpu()
        _check_step(X, C, C1, mo, spherical=kind == "deep")
        C = C1
    # several iterations in one call equal the same iterations one by one
    C5 = kmeans(Xc, nlist, niter=2, metric=metric, spherical=kind == "deep", init=C.cuda()).cpu()
    Cs = C
    for _ in range(2):
        Cs = kmeans(Xc, nlist, niter=1, metric=metric, spherical=kind == "deep", init=Cs.cuda()).cpu()
    assert torch.allclose(C5, Cs, rtol=2 ** -22, atol=1e-7)


def test_kmeans_zero_iterations_and_empty_clusters():
    from paper_conf_sigmod_wangygjxlwglxyy21_b200 import kmeans
    X = G.sift_base(4096, d=32, spec=G.SiftSpec(d=32, n_micro=64))
    init = torch.cat([X[:15], torch.full((1, 32), 1e6)])  # centroid 15 is closest to no row
    C0 = kmeans(X.cuda(), 16, niter=0, init=init.cuda()).cpu()
    assert torch.equal(C0, init)
    C1 = kmeans(X.cuda(), 16, niter=1, init=init.cuda()).cpu()
    assert torch.equal(C1[15], init[15])
    _check_step(X, init, C1, O.L2)
