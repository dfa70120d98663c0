"""Shared-memory wavefronts (total / ideal) per source line and per phase from an ncu
source export (ncu -i X.ncu-rep --page source --csv --print-source cuda,sass > f.csv):
python tools/ncu_wavefronts.py f.csv n_evals [name:lo:hi,...]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1], errors="replace")))
n_evals = float(sys.argv[2])
hdr, fname, out = None, "", []
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
        wf = float(d.get("L1 Wavefronts Shared") or 0)
        ideal = float(d.get("L1 Wavefronts Shared Ideal") or 0)
        inst = float(d.get("Instructions Executed") or 0)
    except ValueError:
        continue
    out.append((wf, ideal, inst, fname, int(r[0]), r[1].strip()[:80]))
tot = sum(o[0] for o in out)
print(f"shared wavefronts per eval {tot / n_evals:.1f} (ideal {sum(o[1] for o in out) / n_evals:.1f})")
for wf, ideal, inst, f, ln, src in sorted(out, reverse=True)[:30]:
    if wf:
        print(f"{wf / n_evals:7.1f} ideal {ideal / n_evals:7.1f}  {f}:{ln:<5} {src}")
if len(sys.argv) > 3:
    acc = {}
    for wf, ideal, inst, f, ln, _ in out:
        name = "other:" + f
        if f == "ad_kernels.cuh":
            for spec in sys.argv[3].split(","):
                nm, lo, hi = spec.split(":")
                if int(lo) <= ln <= int(hi):
                    name = nm
                    break
        a = acc.setdefault(name, [0.0, 0.0, 0.0])
        a[0] += wf
        a[1] += ideal
        a[2] += inst
    for nm, (wf, ideal, inst) in sorted(acc.items(), key=lambda kv: -kv[1][0]):
        print(f"{nm:24s} wavefronts/eval {wf / n_evals:7.1f} (ideal {ideal / n_evals:7.1f})  inst/eval {inst / n_evals:7.1f}")
