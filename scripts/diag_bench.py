import os, sys, time, torch
sys.path.insert(0, os.getcwd())
import bench
from paper_conf_sigmod_wangygjxlwglxyy21_b200 import Index
cfg = dict(bench.CONFIGS["c2"]); dev = torch.device("cuda", 0)
X, Q, C, bs = bench.make_data(cfg, dev)
ix = Index(128, "l2", "flat", 4096, device=0); ix.set_centroids(C); ix.add(X, torch.arange(cfg["n"], device=dev))
def run(tag, clocks=False, prof=True):
    for _ in range(5): ix.search(Q, 10, 16)
    torch.cuda.synchronize()
    ix.profile_read(reset=True); ix.profile(prof)
    clk = bench.Clocks(0)
    if clocks: clk.start(); time.sleep(0.3)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    hs = []
    e0.record()
    for _ in range(20):
        t = time.perf_counter(); D, I = ix.search(Q, 10, 16); hs.append((time.perf_counter() - t) * 1e3)
    e1.record(); torch.cuda.synchronize()
    if clocks: clk.stop()
    ix.profile(False); st = ix.profile_read(reset=True)
    print(tag, f"gpu {e0.elapsed_time(e1)/20:.3f} ms/step host {[round(h,2) for h in hs[:6]]} max {max(hs):.2f}", st[0], flush=True)
run("plain")
run("clocks", clocks=True)
run("plain-noprof", prof=False)
run("clocks-noprof", clocks=True, prof=False)
