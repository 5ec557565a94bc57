import sys, torch
sys.path.insert(0, '.')
import mvgen as G
from mvgen.kmeans import kmeans
from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
spec = G.SiftSpec(d=128, n_micro=512)
X = G.sift_base(5000, spec=spec); Q = G.sift_queries(64, spec=spec)
C = kmeans(X, 16, iters=3)
k = int(sys.argv[1]) if len(sys.argv) > 1 else 10
ix = Index(128, "l2", "flat", 16); ix.set_centroids(C.cuda()); ix.add(X.cuda(), torch.arange(5000).cuda())
D, I = ix.search(Q.cuda(), k, 4); torch.cuda.synchronize()
print("ok", ix.describe()["last_scan"], I[0, :5].tolist())
