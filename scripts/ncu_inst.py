"""Per-CUDA-source-line stall samples and executed instructions from an ncu report (needs -lineinfo)."""
import csv, subprocess, sys, os
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 20
out = subprocess.run(["ncu", "-i", rep] + (["-k", sys.argv[3]] if len(sys.argv) > 3 else []) + ["--page", "source", "--csv", "--print-source=cuda,sass"],
                     capture_output=True, text=True).stdout.splitlines()
fname = "?"; hdr = None; agg = []
for r in csv.reader(out):
    if not r: continue
    if r[0] == "File Path": fname = os.path.basename(r[1]); continue
    if r[0] == "Line No": hdr = r; continue
    if hdr and r[0] not in ("", "Function Name"):
        d = dict(zip(hdr, r))
        try:
            agg.append((float(d["Warp Stall Sampling (All Samples)"]), float(d["Instructions Executed"]), fname, r[0], r[1].strip()))
        except ValueError:
            pass
ts = sum(a[0] for a in agg) or 1; ti = sum(a[1] for a in agg) or 1
print(f"samples {ts:.0f}  warp-instructions {ti:.0f}")
print("-- by stall samples")
for s, i, f, ln, src in sorted(agg, key=lambda a: -a[0])[:top]:
    print(f"{s/ts*100:5.1f}% smp {i/ti*100:5.1f}% ins  {f}:{ln}  {src[:80]}")
print("-- by instructions")
for s, i, f, ln, src in sorted(agg, key=lambda a: -a[1])[:top // 2]:
    print(f"{s/ts*100:5.1f}% smp {i/ti*100:5.1f}% ins  {f}:{ln}  {src[:80]}")
