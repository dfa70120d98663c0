"""Condense a compute-sanitizer racecheck log (stdin) into counts per
(severity, hazard, kernel-side source lines, case): python tools/racecheck_summary.py < log"""
import collections
import re
import sys

cnt = collections.Counter()
case = "?"
cur = None
for line in sys.stdin:
    if line.startswith("=== case"):
        case = line.split(None, 2)[2].strip()
        continue
    m = re.match(r"=+ (Error|Warning): (.*?) hazard detected", line)
    if m:
        cur = [m.group(1), m.group(2).replace("(Warp Level Programming) Potential ", "warp:"), [], case]
        continue
    if cur is not None:
        m = re.search(r"(Read|Write) Thread.*? at (.*?)\+0x[0-9a-f]+ in (\S+)", line)
        if m:
            fn = re.sub(r"\(.*", "", m.group(2)).split("::")[-1]
            cur[2].append(f"{m.group(1)}@{fn}:{m.group(3)}")
            if len(cur[2]) == 2:
                cnt[(cur[0], cur[1], " / ".join(cur[2]), cur[3])] += 1
                cur = None
        elif "RACECHECK SUMMARY" in line:
            print(line.strip())
for (sev, kind, where, c), n in sorted(cnt.items(), key=lambda kv: -kv[1]):
    print(f"{n:8d} {sev:7s} {kind:28s} {where}   [{c}]")
