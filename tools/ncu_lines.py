"""Per-CUDA-line stall samples / instructions from an ncu source export
(ncu -i X.ncu-rep --page source --csv --print-source cuda,sass > f.csv):
python tools/ncu_lines.py f.csv [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hdr = None
out = []
fname = ""
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 8 or not r[0] or r[2] != "-":
        continue
    d = dict(zip(hdr[2:], r[2:]))
    try:
        samp = int(d["Warp Stall Sampling (All Samples)"])
        inst = int(d["Instructions Executed"])
    except (KeyError, ValueError):
        continue
    out.append((samp, inst, fname, int(r[0]), r[1].strip()[:90]))
tot = sum(o[0] for o in out)
tinst = sum(o[1] for o in out)
print(f"total samples {tot}, warp instructions {tinst:.4g}")
for s, i, f, ln, src in sorted(out, reverse=True)[:top]:
    print(f"{100*s/tot:5.1f}% {100*i/tinst:5.1f}%i {f}:{ln:<5} {src}")


def phases(out, ranges):
    """Bucket (samples, inst) by line ranges: ranges = [(name, lo, hi), ...] on ad_kernels.cuh."""
    acc = {}
    for s, i, f, ln, _ in out:
        name = "other:" + f
        if f == "ad_kernels.cuh":
            for nm, lo, hi in ranges:
                if lo <= ln <= hi:
                    name = nm
                    break
        a = acc.setdefault(name, [0, 0])
        a[0] += s
        a[1] += i
    return acc


if len(sys.argv) > 3:
    rng = []
    for spec in sys.argv[3].split(","):
        nm, lo, hi = spec.split(":")
        rng.append((nm, int(lo), int(hi)))
    for nm, (s, i) in sorted(phases(out, rng).items(), key=lambda kv: -kv[1][0]):
        print(f"{nm:28s} samples {100*s/tot:5.1f}%  inst {100*i/tinst:5.1f}%  ({i/1:.4g})")
