import os, sys, torch, numpy as np
sys.path.insert(0, '.')
import mvgen as G, oracle as O
from mvgen.kmeans import kmeans
from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
spec = G.SiftSpec(d=128, n_micro=512)
X = G.sift_base(12000, spec=spec); Q = G.sift_queries(300, spec=spec)
ids = G.permuted_ids(12000, seed=11)
C = kmeans(X, 64, iters=4)
ix = Index(128, "l2", "sq8", 64); ix.set_centroids(C.cuda()); ix.train_sq8(X.cuda()); ix.add(X.cuda(), ids.cuda())
for k in (10, 64):
    os.environ.pop("MV_FORCE_SIMT", None)
    D1, I1 = ix.search(Q.cuda(), k, 6)
    os.environ["MV_FORCE_SIMT"] = "1"
    D2, I2 = ix.search(Q.cuda(), k, 6)
    os.environ.pop("MV_FORCE_SIMT", None)
    d = (D1 - D2).abs(); r = d / D2.abs().clamp_min(1e-9)
    bad = ~torch.isclose(D1, D2, rtol=1e-5, atol=1e-3)
    print(k, "maxabs", d.max().item(), "maxrel", r.max().item(), "nbad", bad.sum().item(), "idagree", (I1 == I2).float().mean().item())
    if bad.any():
        q, j = torch.nonzero(bad)[0].tolist()
        print(" q", q, "j", j, "tc", D1[q, :].tolist()[:12], "\n simt", D2[q, :].tolist()[:12])
        print(" tc ids", I1[q].tolist()[:12], "\n simt ids", I2[q].tolist()[:12])
