"""Registers / spills / stack of every libad kernel from ptxas -v (compiles to a
temporary .so; the in-tree library is untouched): python tools/ptxas_report.py [filter]"""
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_solis_vasquezts25_b200 import build as B  # noqa: E402

flt = sys.argv[1] if len(sys.argv) > 1 else "k_warp_engine"
out = os.path.join(tempfile.mkdtemp(), "libad_v.so")
cmd = ["nvcc", *B.NVCC_FLAGS, "-Xptxas", "-v", "-I", os.path.join(ROOT, "include"), "-o", out,
       os.path.join(B.SRC, "ad_api.cu")]
txt = subprocess.run(cmd, capture_output=True, text=True).stderr
fn = None
for line in txt.splitlines():
    m = re.search(r"Compiling entry function '(\S+)'", line)
    if m:
        fn = m.group(1)
        continue
    m = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m and fn:
        stack, st, ld = m.groups()
        continue
    m = re.search(r"Used (\d+) registers", line)
    if m and fn and flt in fn:
        dem = subprocess.run(["c++filt", fn], capture_output=True, text=True).stdout.strip()
        print(f"regs {m.group(1):>3} stack {stack:>4} spill st {st:>4} ld {ld:>4}  {dem[:110]}")
        fn = None
