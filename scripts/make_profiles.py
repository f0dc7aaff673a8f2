"""Summarise gpurun_out/ ncu captures into profiles/ (tracked).  Usage: make_profiles.py <round tag>"""
import csv, json, os, subprocess, sys, shutil
from collections import defaultdict
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
G, P = "gpurun_out", "profiles"
os.makedirs(P, exist_ok=True)

def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    return dict(zip(rows[0], rows[2])) if len(rows) > 2 else {}

lines = []
# launch list
if os.path.exists(f"{G}/launches.csv"):
    shutil.copy(f"{G}/launches.csv", f"{P}/{tag}_launches.csv")
    rows = list(csv.reader(open(f"{G}/launches.csv")))
    i = [j for j, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr = rows[i]; ki = hdr.index("Kernel Name"); vi = hdr.index("Metric Value")
    d = defaultdict(list)
    for r in rows[i + 1:]:
        if len(r) > vi:
            d[r[ki].split("(")[0]].append(float(r[vi].replace(",", "")))
    hot = {k: v for k, v in d.items() if "cusfft::k_" in k and not any(s in k for s in ("cheb", "dc_window", "taps", "normalize", "ghat", "twiddles", "gauss"))}
    step = sum(sum(v) / len(v) for v in hot.values())
    lines.append(f"## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; cold-cache, serialised)\n")
    lines.append(f"Command: `ncu ... python bench.py --steps 2 --warmup 3 --no-cpu-baseline` (file `{tag}_launches.csv`).\n")
    lines.append("| kernel | launches | mean µs | share of hot-path sum |\n|---|---|---|---|")
    for k, v in sorted(hot.items(), key=lambda kv: -sum(kv[1]) / len(kv[1])):
        m = sum(v) / len(v) / 1e3
        lines.append(f"| `{k}` | {len(v)} | {m:.2f} | {m * 1e3 / step * 100:.1f}% |")
    other = {k: v for k, v in d.items() if k not in hot}
    lines.append("\nOther launches in the same command (plan-time filter construction, L2 flush, dense cuFFT context):\n")
    lines.append("| kernel | launches | mean µs |\n|---|---|---|")
    for k, v in sorted(other.items(), key=lambda kv: -sum(kv[1]) / len(kv[1])):
        lines.append(f"| `{k[:70]}` | {len(v)} | {sum(v) / len(v) / 1e3:.2f} |")
# full captures
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum", "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "smsp__inst_executed.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__grid_size", "launch__block_size"]
traffic = None
fold_parts = {}
for name, rep in [("k_stage (staged gather, phase 1)", f"{G}/prof_k_stage.ncu-rep"),
                  ("k_fold_fft1 (fold phase 2 + FFT pass 1)", f"{G}/prof_fold_full.ncu-rep"), ("k_fft (pass 2 + keys)", f"{G}/prof_k_fft.ncu-rep"),
                  ("k_select", f"{G}/prof_k_select.ncu-rep"), ("k_vote", f"{G}/prof_k_vote.ncu-rep"),
                  ("k_estimate", f"{G}/prof_k_estimate.ncu-rep"), ("k_output", f"{G}/prof_k_output.ncu-rep")]:
    if not os.path.exists(rep):
        continue
    m = raw(rep)
    lines.append(f"\n## {name} — `ncu --set full --clock-control none` (C3, `scripts/run_c3.py`)\n")
    lines.append("| metric | value |\n|---|---|")
    for w in want:
        if w in m:
            lines.append(f"| {w} | {m[w]} |")
    if ("fold" in name or "stage" in name) and "dram__bytes_read.sum" in m:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(out.splitlines()))
        unit = dict(zip(rows[0], rows[1]))
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
        rd = float(m["dram__bytes_read.sum"]) * scale[unit["dram__bytes_read.sum"]]
        wr = float(m["dram__bytes_write.sum"]) * scale[unit["dram__bytes_write.sum"]]
        fold_parts[name.split()[0]] = (rd, wr)
if fold_parts:
    rd = sum(v[0] for v in fold_parts.values())
    wr = sum(v[1] for v in fold_parts.values())
    traffic = {"kernel": " + ".join(sorted(fold_parts)), "config": "C3", "source": f"{tag}_ncu_summary.md (ncu --set full)",
               "parts": {k: {"dram_bytes_read": v[0], "dram_bytes_write": v[1]} for k, v in fold_parts.items()},
               "dram_bytes_read": rd, "dram_bytes_write": wr, "dram_bytes_per_launch": rd + wr}
if traffic:
    json.dump(traffic, open(f"{P}/fold_traffic_C3.json", "w"), indent=1)
open(f"{P}/{tag}_ncu_summary.md", "w").write("\n".join(lines) + "\n")
print("\n".join(lines[:40]))
