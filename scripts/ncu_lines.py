"""Warp-stall samples per CUDA source line from an ncu report (cuda,sass source view).
Usage: ncu_lines.py REPORT [top]"""
import csv, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                     capture_output=True, text=True).stdout.splitlines()
fname, agg, src = "?", {}, {}
for r in csv.reader(out):
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] in ("Function Name", "Line No"):
        continue
    if len(r) > 4 and r[0].isdigit() and r[2] == "-":  # a CUDA source line with its aggregated samples
        try:
            v = float(r[4])
        except ValueError:
            continue
        key = (fname, int(r[0]))
        agg[key] = agg.get(key, 0) + v
        src[key] = r[1]
tot = sum(agg.values()) or 1
print(f"total samples {tot:.0f}")
for key, v in sorted(agg.items(), key=lambda kv: -kv[1])[:top]:
    print(f"{v / tot * 100:5.1f}%  {key[0]}:{key[1]:<5d} {src[key].strip()[:100]}")
