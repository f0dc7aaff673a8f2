"""Top SASS instructions by warp-stall samples from an ncu report (source page)."""
import csv, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 15
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=sass"],
                     capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(out[1:]))
hdr = rows[0]
ci = hdr.index("Warp Stall Sampling (All Samples)")
si = hdr.index("Source")
data = [r for r in rows[1:] if len(r) > ci and r[ci].replace('.', '').isdigit()]
tot = sum(float(r[ci]) for r in data) or 1
print(f"total samples {tot:.0f}")
for idx, r in sorted(enumerate(data), key=lambda t: -float(t[1][ci]))[:top]:
    print(f"{float(r[ci]) / tot * 100:5.1f}%  #{idx:4d}  {r[si].strip()[:90]}")
