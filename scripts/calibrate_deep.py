"""Calibrate the Deep-shaped generator (c3): recall@10 of IVF_SQ8 IP at nprobe 32, nlist 16384 on
10M x 96 for a grid of (s1, s2).  Data preparation only; prints one line per setting."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import mvgen as G
from mvgen.kmeans import kmeans
import bench
from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index

n = int(os.environ.get("CAL_N", 10_000_000))
dev = torch.device("cuda", 0)
for s1, s2 in [tuple(map(float, a.split(","))) for a in sys.argv[1:]]:
    t0 = time.time()
    spec = G.DeepSpec(s1=s1, s2=s2)
    X = G.deep_base(n, spec=spec, device=dev)
    Q = G.deep_queries(10_000, spec=spec, device=dev)
    C = kmeans(X, 16384, iters=10, spherical=True)
    ix = Index(96, "ip", "sq8", 16384, device=0)
    ix.set_centroids(C)
    xs = X[torch.randperm(n, device=dev)[:64 * 16384]]
    vmin = xs.min(0).values.contiguous()
    ix.set_sq8(vmin, (xs.max(0).values - vmin).contiguous())
    ix.add(X, torch.arange(n, device=dev))
    gt = bench.ground_truth(X, Q, 10, "ip")
    out = []
    for npb in (16, 32, 64):
        D, I = ix.search(Q, 10, npb)
        out.append((npb, round(bench.recall_at(gt, I, 10), 4)))
    print(f"s1={s1} s2={s2} recall@10 {out} ({time.time() - t0:.0f}s)", flush=True)
    del X, ix
    torch.cuda.empty_cache()
