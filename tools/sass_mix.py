"""Dynamic SASS opcode mix (and stall samples) per evaluation from an ncu SASS
source export: ncu -i X.ncu-rep --page source --csv --print-source sass > f.csv
python tools/sass_mix.py f.csv EVALS [top]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
evals = float(sys.argv[2])
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
hdr = rows[1]
ix, isamp = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
cnt, samp = collections.Counter(), collections.Counter()
tot = ts = 0
for r in rows[2:]:
    if len(r) != len(hdr):
        continue
    src = r[1].strip().split()
    if not src:
        continue
    op = src[1] if src[0].startswith("@") and len(src) > 1 else src[0]
    op = op.split(".")[0]
    n, s = int(r[ix] or 0), int(r[isamp] or 0)
    cnt[op] += n
    samp[op] += s
    tot += n
    ts += s
print(f"warp instructions per eval {tot / evals:.1f}")
for op, n in cnt.most_common(top):
    print(f"{op:10s} {n / evals:8.1f}  {100 * n / tot:5.1f}% inst  {100 * samp[op] / ts:5.1f}% samples")
