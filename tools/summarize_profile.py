"""Summaries for profiles/: (1) a launch list (ncu --metrics gpu__time_duration.sum CSV) -> per-kernel
share of the step; (2) a `ncu --set full` report -> the key pipe / DRAM metrics of the match kernel,
and profiles/match_traffic.json (bench.py's roofline `traffic`).
usage: python tools/summarize_profile.py TAG [config=c4]"""
import csv
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1]
cfg = sys.argv[2] if len(sys.argv) > 2 else "c4"
out_dir = os.path.join(ROOT, "profiles")
g = os.path.join(ROOT, "gpurun_out")

# (1) launch list
rows = [r for r in csv.reader(open(os.path.join(g, f"{tag}_launches.csv"))) if len(r) > 14 and r[0] != "ID"]
tot = defaultdict(float)
cnt = defaultdict(int)
for r in rows:
    if r[12] == "gpu__time_duration.sum":
        name = r[4].split("(")[0]
        v = float(r[14].replace(",", ""))
        tot[name] += v * (1e-6 if r[13] == "ns" else 1e-3 if r[13] == "us" else 1.0 if r[13] == "ms" else 1e3)
        cnt[name] += 1
S = sum(tot.values())
lines = [f"# {tag} launch list: ncu --metrics gpu__time_duration.sum --clock-control none "
         f"(bench.py --steps 2 --warmup 3 --no-cpu-baseline, {cfg})",
         "# cold-cache, serialised per-launch times: compare SHARES of the step, not absolutes",
         f"{'kernel':56s} {'launches':>8s} {'total ms':>11s} {'mean ms':>10s} {'share':>7s}"]
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    lines.append(f"{k[:56]:56s} {cnt[k]:8d} {v:11.3f} {v / cnt[k]:10.3f} {100 * v / S:6.2f}%")
open(os.path.join(out_dir, f"{tag}_launches_summary.txt"), "w").write("\n".join(lines) + "\n")
print("\n".join(lines))

# (2) full capture
rep = os.path.join(g, f"{tag}_match.ncu-rep")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines()))
h, u, v = r[0], r[1], r[2]
keys = ["gpu__time_duration.sum", "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
        "launch__shared_mem_per_block_dynamic", "sm__cycles_elapsed.avg.per_second",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_subpipe_imma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed"]
out = [f"# {tag}: ncu --set full --clock-control none of one match_kernel launch at the bench configuration ({cfg})"]
vals = {}
for k in keys:
    if k in h:
        i = h.index(k)
        out.append(f"{k:80s} {v[i]:>22s} {u[i]}")
        vals[k] = (v[i], u[i])
open(os.path.join(out_dir, f"{tag}_match_ncu_summary.txt"), "w").write("\n".join(out) + "\n")
print("\n".join(out))


def to_bytes(x):
    val, unit = float(x[0].replace(",", "")), x[1]
    return val * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


if "dram__bytes_read.sum" in vals:
    b = to_bytes(vals["dram__bytes_read.sum"]) + to_bytes(vals.get("dram__bytes_write.sum", ("0", "byte")))
    tf = os.path.join(out_dir, "match_traffic.json")
    d = json.load(open(tf)) if os.path.exists(tf) else {}
    d[cfg] = {"dram_bytes_per_launch": b, "source": f"profiles/{tag}_match_ncu_summary.txt (ncu --set full, one launch)"}
    json.dump(d, open(tf, "w"), indent=1)
    print("traffic", b)
