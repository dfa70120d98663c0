"""List the innermost loops (backward branches) of a kernel's SASS with op counts.
python tools/sass_loops.py LIB.so MANGLED_NAME [min_mufu]"""
import collections
import re
import subprocess
import sys

lib, fn = sys.argv[1], sys.argv[2]
min_mufu = int(sys.argv[3]) if len(sys.argv) > 3 else 1
txt = subprocess.run(["cuobjdump", "-sass", "-fun", fn, lib], capture_output=True, text=True).stdout
ins = []
for line in txt.splitlines():
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);", line)
    if m:
        ins.append((int(m.group(1), 16), m.group(2).strip()))
addr_idx = {a: k for k, (a, _) in enumerate(ins)}
loops = []
for k, (a, t) in enumerate(ins):
    m = re.search(r"\bBRA\b.*?(0x[0-9a-f]+)", t)
    if m:
        tgt = int(m.group(1), 16)
        if tgt <= a and tgt in addr_idx:
            loops.append((addr_idx[tgt], k))
for lo, hi in loops:
    body = ins[lo:hi + 1]
    ops = collections.Counter(re.sub(r"^@!?U?P\w+\s+", "", t).split()[0] for _, t in body)
    mufu = sum(v for o, v in ops.items() if o.startswith("MUFU"))
    if mufu < min_mufu:
        continue
    sm = sum(v for o, v in ops.items() if o.startswith(("LDS", "STS")))
    print(f"loop {body[0][0]:#06x}-{body[-1][0]:#06x}: {len(body)} instr, MUFU {mufu}, LDS/STS {sm}, "
          f"LDL/STL {ops['LDL'] + ops['STL']}, LDG {sum(v for o, v in ops.items() if o.startswith('LDG'))}")
    if "-v" in sys.argv:
        print("   ", ops.most_common(25))
