"""Write profiles/ summaries from ncu reports in gpurun_out/ (run here, no GPU needed).

usage: python tools/make_profile_summary.py ROUND key=path.ncu-rep [key=path ...] [launches=path.csv]
Writes profiles/ncu_<ROUND>.md (human summary) and merges dram bytes per launch into
profiles/ncu_summary.json (read by bench.py for roofline.traffic).
"""
import csv
import json
import os
import sys
from collections import defaultdict

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import summary  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    agg = defaultdict(list)
    for r in rows[hdr + 1:]:
        if len(r) > vi:
            agg[r[ki]].append(float(r[vi].replace(",", "")))
    tot = sum(sum(v) for v in agg.values())
    return [(k, len(v), sum(v), sum(v) / tot) for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1]))]


def main():
    rnd = sys.argv[1]
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    js_path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    js = json.load(open(js_path)) if os.path.exists(js_path) else {"ls_kernel": {}}
    lines = [f"# ncu summaries, round {rnd}", "",
             "Captured with `ncu --set full --clock-control none --import-source on -k regex:<kernel> -s 1 -c 1` "
             "on `python tools/prof_ls.py <config> <engine> 2` (one LS launch: config 2 = 3000 poses x 300 "
             "iterations), B200, under gpurun.  ncu replays serialise and run cold, so durations are not bench "
             "numbers; compare shares and per-launch counters.", ""]
    for arg in sys.argv[2:]:
        key, path = arg.split("=", 1)
        if key == "launches":
            lines += ["## Launch list (ncu --metrics gpu__time_duration.sum, bench.py --steps 2 --warmup 1)", "",
                      "| kernel | launches | total ns | share |", "|---|---|---|---|"]
            for k, n, t, s in launches(path):
                lines.append(f"| `{k[:80]}` | {n} | {t:.0f} | {s:.3f} |")
            lines.append("")
            continue
        s = summary(path)
        lines += [f"## {key}  (`{os.path.basename(path)}`)", ""]
        for k, v in s.items():
            lines.append(f"- `{k}`: {v}")
        lines.append("")
        try:
            dr = float(s["dram__bytes_read.sum"][0]) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[
                s["dram__bytes_read.sum"][1]]
            dw = float(s["dram__bytes_write.sum"][0]) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[
                s["dram__bytes_write.sum"][1]]
            js["ls_kernel"][key] = {"dram_bytes_per_launch": dr + dw, "round": rnd, "report": os.path.basename(path)}
            # the measured co-bounds of the kernel (bench.py roofline.co_bounds)
            for name, metric in (("issue_active_pct", "smsp__issue_active.avg.pct_of_peak_sustained_active"),
                                 ("l1tex_throughput_pct", "l1tex__throughput.avg.pct_of_peak_sustained_active"),
                                 ("warp_instructions", "smsp__inst_executed.sum"),
                                 ("shared_wavefronts", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
                                 ("tensor_pipe_pct", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active")):
                if metric in s:
                    js["ls_kernel"][key][name] = float(s[metric][0])
        except (KeyError, ValueError):
            pass
    open(os.path.join(ROOT, "profiles", f"ncu_{rnd}.md"), "w").write("\n".join(lines) + "\n")
    json.dump(js, open(js_path, "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
