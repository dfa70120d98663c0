"""Config 4: the reduction microbenchmark of Eq 1-5.
For every engine x P partials x C components: 148 x 8 blocks per launch, `reps`
timed launches (CUDA events, after warm-up); reports ns per block-reduction,
block-reductions/s, and the max abs error / sum|x| against math.fsum with the O-7
bound (ceil(log2 P) + 2) 2^-24 (FP16 no-EC: its own (4 + P/32) 2^-11 bound).
usage: python tools/bench_reduce.py [out.json] [reps]"""
import json
import math
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_solis_vasquezts25_b200 import ad, synth  # noqa: E402

ENGINES = ("simt", "tc", "paper", "tc_fp16")


def main():
    out_path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/reduce_config4.json"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 100
    ctx = ad.Context(0)
    nb = 148 * 8
    rows = []
    for dist in ("uniform", "logmag"):
        for P in (128, 256, 512, 1024):
            for C in (8, 16, 24, 32, 40):
                x = synth.make_reduction_partials(10 * P + C + (0 if dist == "uniform" else 1), nb, P, C, dist)
                xd = torch.from_numpy(x).cuda()
                x64 = x.astype(np.float64)
                ex = np.array([[math.fsum(x64[b, :, c]) for c in range(C)] for b in range(64)])
                sabs = np.abs(x64[:64]).sum(axis=1)
                for eng in ENGINES:
                    o = torch.empty(nb, C, device="cuda")
                    for _ in range(3):
                        ad.ad_reduce_blocks(ctx.h, ad.ENGINES[eng], xd, o)
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    torch.cuda.synchronize()
                    a.record()
                    for _ in range(reps):
                        ad.ad_reduce_blocks(ctx.h, ad.ENGINES[eng], xd, o)
                    b.record()
                    torch.cuda.synchronize()
                    ms = a.elapsed_time(b) / reps
                    got = o[:64].cpu().numpy().astype(np.float64)
                    with np.errstate(invalid="ignore"):
                        rel = np.abs(got - ex) / np.maximum(sabs, 1e-30)
                    bound = (4 + P / 32) * 2.0 ** -11 if eng == "tc_fp16" else (math.ceil(math.log2(P)) + 2) * 2.0 ** -24
                    fin = np.isfinite(rel)
                    rows.append({"dist": dist, "P": P, "C": C, "engine": eng, "ms_per_launch": ms,
                                 "ns_per_block_reduction": ms * 1e6 / nb,
                                 "block_reductions_per_s": nb / (ms * 1e-3),
                                 "max_err_over_sumabs": float(rel[fin].max()) if fin.any() else None,
                                 "bound": bound, "within_bound": bool(fin.all() and (rel <= bound).all()),
                                 "non_finite": int((~fin).sum())})
    ctx.close()
    summ = {}
    for eng in ENGINES:
        r = [q for q in rows if q["engine"] == eng and q["dist"] == "uniform"]
        summ[eng] = {"mean_ns_per_block_reduction": float(np.mean([q["ns_per_block_reduction"] for q in r])),
                     "all_within_bound_uniform": all(q["within_bound"] for q in r),
                     "all_within_bound_logmag": all(q["within_bound"] for q in rows
                                                    if q["engine"] == eng and q["dist"] == "logmag")}
    res = {"config": "config 4: 1184 blocks (148 x 8) per launch", "reps": reps, "summary": summ, "rows": rows}
    os.makedirs(os.path.dirname(out_path) or ".", exist_ok=True)
    with open(out_path, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(summ, indent=1))


if __name__ == "__main__":
    main()
