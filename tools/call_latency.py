"""Breakdown of one config-1 ad_score_poses call (256 poses, gradients): device time of
the kernel alone, the call (kernel + error read-back), and H2D + call + D2H, plus the
host wall clock per call.  python tools/call_latency.py"""
import os
import statistics
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth  # noqa: E402

w = synth.make_config(1)
ctx = ad.Context(0)
ctx.upload_grid(w.grid)
lid = ctx.upload_ligand(w.ligands[0], w.ff)
hg = torch.from_numpy(np.ascontiguousarray(w.genes)).pin_memory()
g = hg.cuda()
n, s = hg.shape
out = torch.empty(n * (1 + s), device="cuda")
E, G = out[:n], out[n:].view(n, s)
hout = torch.empty(n * (1 + s)).pin_memory()
st = torch.cuda.current_stream()


def run(mode, reps=300):
    host, dev = [], []
    for k in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        a.record(st)
        if mode == "e2e":
            g.copy_(hg, non_blocking=True)
        ad.ad_score_poses(ctx.h, lid, None, g, E, G)
        if mode == "e2e":
            hout.copy_(out, non_blocking=True)
        b.record(st)
        b.synchronize()
        t1 = time.perf_counter()
        if k >= 50:
            host.append((t1 - t0) * 1e6)
            dev.append(a.elapsed_time(b) * 1e3)
    print(f"{mode:5s} host {statistics.median(host):7.1f} us   device {statistics.median(dev):7.1f} us")


run("call")
run("e2e")

# host-side split: Python marshalling vs the C entry point (launch enqueue only)
import ctypes as C  # noqa: E402
L = ad.lib()
args = (ctx.h, lid, None, n, C.c_void_p(g.data_ptr()), s, C.c_void_p(E.data_ptr()), C.c_void_p(G.data_ptr()), None,
        C.c_void_p(st.cuda_stream))
for name, fn in (("python ad_score_poses (enqueue)", lambda: ad.ad_score_poses(ctx.h, lid, None, g, E, G)),
                 ("raw C ad_score_poses (enqueue)", lambda: L.ad_score_poses(*args)),
                 ("torch.cuda.current_stream()", lambda: torch.cuda.current_stream()),
                 ("cudaEventRecord via torch", lambda: torch.cuda.Event().record(st))):
    ts = []
    for k in range(400):
        t0 = time.perf_counter()
        fn()
        ts.append((time.perf_counter() - t0) * 1e6)
        if k % 50 == 0:
            torch.cuda.synchronize()
    print(f"{name:36s} {statistics.median(ts[50:]):7.2f} us")
