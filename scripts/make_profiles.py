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
    hot = {k: v for k, v in d.items() if "cusfft::k_" in k and not any(s in k for s in ("cheb", "dc_window", "taps", "normalize", "ghat", "ginv", "phase_table", "twiddles", "gauss"))}
    step = sum(sum(v) / len(v) for v in hot.values())
    lines.append(f"## Launch list (ncu --metrics gpu__time_duration.sum --clock-control none; cold-cache, serialised)\n")
    lines.append(f"Command: `ncu --metrics gpu__time_duration.sum --clock-control none ... python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cupti --no-default-line` (file `{tag}_launches.csv`).  Per-launch times are cold-cache and serialised; the SHARES are what compare with the bench's in-graph numbers.\n")
    lines.append("| kernel | launches | mean µs | share of hot-path sum |\n|---|---|---|---|")
    for k, v in sorted(hot.items(), key=lambda kv: -sum(kv[1]) / len(kv[1])):
        m = sum(v) / len(v) / 1e3
        lines.append(f"| `{k}` | {len(v)} | {m:.2f} | {m * 1e3 / step * 100:.1f}% |")
    other = {k: v for k, v in d.items() if k not in hot}
    lines.append("\nOther launches in the same command (plan-time filter construction, L2 flush, dense cuFFT context):\n")
    lines.append("| kernel | launches | mean µs |\n|---|---|---|")
    for k, v in sorted(other.items(), key=lambda kv: -sum(kv[1]) / len(kv[1])):
        lines.append(f"| `{k[:70]}` | {len(v)} | {sum(v) / len(v) / 1e3:.2f} |")
# full captures: ONE application-replay report of one whole execution
# (--cache-control none: phase 2 sees the staging buffer phase 1 left in L2,
# as in the timed step; x itself is cold because run_c3 flushes L2 first)
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum", "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "smsp__inst_executed.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__grid_size", "launch__block_size"]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
rep = f"{G}/prof_{tag}.ncu-rep" if os.path.exists(f"{G}/prof_{tag}.ncu-rep") else f"{G}/prof_all.ncu-rep"
traffic = None
fold_parts = {}
if os.path.exists(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], dict(zip(rows[0], rows[1]))
    lines.append("\n## Full captures of one C3 execution — `ncu --set full --cache-control none --replay-mode application "
                 "--clock-control none` (`scripts/run_c3.py`, L2 flushed before the execution)\n")
    names = [r[hdr.index("Kernel Name")].split("(")[0].replace("void ", "") for r in rows[2:]]
    lines.append("| metric | " + " | ".join(f"`{n}`" for n in names) + " |")
    lines.append("|---|" + "---|" * len(names))
    for w in want:
        if w in hdr:
            lines.append(f"| {w} ({units.get(w, '')}) | " + " | ".join(r[hdr.index(w)] for r in rows[2:]) + " |")
    for n, r in zip(names, rows[2:]):
        if "k_stage" in n or "k_fold" in n:
            rd = float(r[hdr.index("dram__bytes_read.sum")]) * scale[units["dram__bytes_read.sum"]]
            wr = float(r[hdr.index("dram__bytes_write.sum")]) * scale[units["dram__bytes_write.sum"]]
            a = fold_parts.get(n, (0.0, 0.0))  # several launches per execution (branched graph): summed
            fold_parts[n] = (a[0] + rd, a[1] + wr)
if fold_parts:
    rd = sum(v[0] for v in fold_parts.values())
    wr = sum(v[1] for v in fold_parts.values())
    info = json.load(open(f"{G}/plan_info.json")) if os.path.exists(f"{G}/plan_info.json") else {}
    sp = [v for k, v in fold_parts.items() if k.startswith("cusfft::k_stage_packed") or k.startswith("k_stage_packed")]
    traffic = {"kernel": " + ".join(sorted(fold_parts)), "config": "C3", "source": f"{tag}_ncu_summary.md (ncu --set full)",
               "sum_w": info.get("sum_w"), "plan": info,
               "k_stage_packed_dram_bytes_per_launch": (sp[0][0] + sp[0][1]) if sp else None,
               "parts": {k: {"dram_bytes_read": v[0], "dram_bytes_write": v[1], "dram_bytes_per_launch": v[0] + v[1]}
                         for k, v in fold_parts.items()},
               "dram_bytes_read": rd, "dram_bytes_write": wr, "dram_bytes_per_launch": rd + wr}
if traffic:
    json.dump(traffic, open(f"{P}/fold_traffic_C3.json", "w"), indent=1)
open(f"{P}/{tag}_ncu_summary.md", "w").write("\n".join(lines) + "\n")
print("\n".join(lines[:60]))
