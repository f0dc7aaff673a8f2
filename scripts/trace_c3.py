"""In-graph per-kernel spans of the C3 pipeline (needs the -DCUSFFT_TRACE build:
CUSFFT_LIB=libcusfft_trace.so).  Usage: trace_c3.py [L] [tolerance] [reps]"""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import bench
from paper_conf_ipps_wangcc16_b200 import Plan, load_library
from paper_conf_ipps_wangcc16_b200.workload import planted_signal
n, k = 2**24, 1000
L = int(sys.argv[1]) if len(sys.argv) > 1 else 16
tol = float(sys.argv[2]) if len(sys.argv) > 2 else 1e-7
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 5
x, S, X = planted_signal(n, k, 1)
xd = torch.from_numpy(x).cuda()
prm = bench.plan_params("C3")
if len(sys.argv) > 2:
    prm["tolerance"] = tol
plan = Plan(n, k, L=L, seed=3, **prm)
if os.environ.get("TRACE_TIMING"):
    plan.set_timing(int(os.environ["TRACE_TIMING"]))
lib = load_library()
fl = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
fr = torch.ones(64 << 20, dtype=torch.int32, device="cuda")
names = {1: "k_stage_packed", 2: "k_fold_fft1*", 4: "k_fold", 5: "k_fft pass1", 6: "k_fft pass2",
         7: "k_keys", 8: "k_select*", 9: "k_tail / k_vote", 10: "k_estimate", 11: "k_output"}
acc = {}
for rep in range(reps):
    fl.zero_(); fr.sum()
    torch.cuda.synchronize()
    lib.cusfft_debug_trace_reset()
    plan.execute(xd)
    torch.cuda.synchronize()
    buf = (ctypes.c_ulonglong * 256)()
    lib.cusfft_debug_trace(buf, 256)
    t = np.array(list(buf), dtype=np.float64)
    spans = {i: (t[128 + 2 * i], t[129 + 2 * i]) for i in names if t[129 + 2 * i] > 0}
    t0 = min(s for s, e in spans.values())
    end = max(e for s, e in spans.values())
    if rep == 0:
        continue  # first run captures the graph
    if rep == reps - 1:
        phases = {i: (t[i] - t0) / 1e3 for i in range(96) if t[i] > 0}
        print("phase slots (us):", " ".join(f"{i}:{v:.2f}" for i, v in sorted(phases.items(), key=lambda kv: kv[1])))
        print("select candidates per loop:", [int(t[96 + i]) & 0xFFFFFFFF for i in range(16) if 0 < t[96 + i] < 2**40])
        print("fold_fft1: latest CTA start (us) loc/est", [(t[112 + q] - t0) / 1e3 for q in (0, 1) if t[112 + q] > 0],
              "cycles: first rows landed", int(t[114]), "slot compute", int(t[115]), "CTA", int(t[116]))
        print("fft2_select cycles (max over CTAs, from entry): loads", int(t[117]), "fft", int(t[118]),
              "keys", int(t[119]), "cl.wait", int(t[120]), "hist push", int(t[121]), "sync1", int(t[122]),
              "classify+push", int(t[123]), "sync2", int(t[124]), "resolve+scan", int(t[125]), "write", int(t[126]))
        cyc = {i: int(t[i]) for i in range(64, 96) if t[i] > 0}
        if cyc:
            print("tail cycles: vote(w0 max)", cyc.get(70), "vote(CTA max)", cyc.get(71), "estimate(CTA max)", cyc.get(72),
                  "first pass (warp max)", cyc.get(73), "+barrier", cyc.get(74), "loop_estimate loads", cyc.get(75))
            o = [cyc.get(i) for i in range(80, 87)]
            if all(o):
                print("output phases (cycles): load", o[1] - o[0], "pick", o[2] - o[1], "classify", o[3] - o[2],
                      "count+scan+scatter", o[4] - o[3], "insertion", o[5] - o[4], "write", o[6] - o[5], "total", o[6] - o[0])
    if rep == reps - 1 and hasattr(lib, "cusfft_debug_cta_trace"):
        cbuf = (ctypes.c_ulonglong * (3 * 16384))()
        m = lib.cusfft_debug_cta_trace(cbuf, 16384)
        rec = np.array(list(cbuf)[:3 * m], dtype=np.uint64).reshape(-1, 3) if m > 0 else np.zeros((0, 3), np.uint64)
        print(f"per-CTA records: {m}")
        for kid in sorted(set(int(r) & 0xFF for r in rec[:, 2])):
            sel_ = rec[(rec[:, 2] & np.uint64(0xFF)) == np.uint64(kid)]
            st = (sel_[:, 0].astype(np.float64) - t0) / 1e3
            en = (sel_[:, 1].astype(np.float64) - t0) / 1e3
            du = en - st
            q = lambda a: " ".join(f"{np.percentile(a, p):6.2f}" for p in (0, 10, 50, 90, 100))
            print(f"  {names.get(kid, kid)!s:16s} n={len(st):4d} start[0,10,50,90,100] {q(st)} | end {q(en)} | dur {q(du)}")
            lo, hi = int(np.floor(st.min())), int(np.ceil(en.max()))
            hist = [int(((st >= b) & (st < b + 1)).sum()) for b in range(lo, hi)]
            live = [int(((st < b + 1) & (en > b)).sum()) for b in range(lo, hi)]
            print(f"  {'':16s} starts/us from {lo}: {hist}")
            print(f"  {'':16s} live CTAs/us     : {live}")
    for i, (s, e) in spans.items():
        acc.setdefault(i, []).append(((s - t0) / 1e3, (e - t0) / 1e3))
    acc.setdefault(0, []).append((0.0, (end - t0) / 1e3))
print(f"C3 L={L} {prm} staged={plan.info()['staged']}")
print(f"{'kernel':16s} {'start us':>9s} {'end us':>9s} {'span us':>9s}")
for i, v in sorted(acc.items(), key=lambda kv: np.mean([a for a, b in kv[1]])):
    s = np.median([a for a, b in v]); e = np.median([b for a, b in v])
    print(f"{names.get(i, 'TOTAL'):16s} {s:9.2f} {e:9.2f} {e - s:9.2f}")
