"""SURVEY §8(f) N3 study (oracle only, CPU): separate location / estimation
filters at C3 (n = 2^24, k = 1000, B = 16384, L_loc = 8 location loops +
8 estimation-only loops, T = 5).

The paper separates the L location loops (Steps 1-5) from the
loops the estimation runs over (Alg. 5 loops over ``outer_loops``, L308;
one batched FFT over them, L232).  Here the location loops r < L_loc use
their own filter (delta_loc, lambda_loc) and the estimation-only loops
(delta_est, lambda_est); both groups share B.  Every loop still
estimates (Alg. 5 over all loops), each with its own filter response G^.

Each step is an oracle primitive (perm_filter, bucket_fft, cutoff,
location_recovery, estimate, select_output) called per group; only the
median over the concatenated per-loop estimates (L95, Alg. 5:
element of rank floor((L-1)/2), re and im separately) is written out here.

Usage: n3_study.py OUT.jsonl SEED0 NSEEDS NPROC
"""
import json
import os
import sys
from multiprocessing import Pool

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np

import oracle as O
from paper_conf_ipps_wangcc16_b200.workload import planted_signal

n, k, L_loc, L_est, T = 2 ** 24, 1000, 8, int(os.environ.get("N3_LEST", "8")), 5  # N3_LEST: estimation-only loops
B = int(os.environ.get("N3_B", "16384"))  # N3_B=8192: half the formula's buckets (Bcst = 1/2)
nb = n // B

# name: (delta_loc, lambda_loc * B, delta_est, num / k, lambda_est * B)
SETTINGS = {
    "base_d1e-7": (1e-7, 0.5, 1e-7, 1, 0.5),
    "loc_d1e-6": (1e-6, 0.5, 1e-7, 1, 0.5),
    "loc_d1e-5": (1e-5, 0.5, 1e-7, 1, 0.5),
    "loc_d1e-4": (1e-4, 0.5, 1e-7, 1, 0.5),
    "loc_d1e-6_est_d1e-8": (1e-6, 0.5, 1e-8, 1, 0.5),
    "loc_d1e-5_est_d1e-8": (1e-5, 0.5, 1e-8, 1, 0.5),
    "loc_d1e-6_lam0.75": (1e-6, 0.75, 1e-7, 1, 0.5),
    "loc_d1e-6_lam1.0": (1e-6, 1.0, 1e-7, 1, 0.5),
    "loc_d1e-6_lam1.0_num2k": (1e-6, 1.0, 1e-7, 2, 0.5),
    "loc_d1e-5_lam1.0": (1e-5, 1.0, 1e-7, 1, 0.5),
    "loc_d1e-4_lam1.0": (1e-4, 1.0, 1e-7, 1, 0.5),
    "loc_d1e-5_lam1.5": (1e-5, 1.5, 1e-7, 1, 0.5),
    "loc_d1e-6_lam2.0": (1e-6, 2.0, 1e-7, 1, 0.5),
    "loc_d1e-6_lam1.0_est_lam0.75": (1e-6, 1.0, 1e-7, 1, 0.75),
    "all_d1e-7_lam0.75": (1e-7, 0.75, 1e-7, 1, 0.75),
}
# second round (N3_SET=2): wider main lobes for all loops, and per-group combinations
SETTINGS2 = {
    "all_d1e-7_lam1.0": (1e-7, 1.0, 1e-7, 1, 1.0),
    "all_d1e-7_lam1.25": (1e-7, 1.25, 1e-7, 1, 1.25),
    "all_d1e-8_lam1.0": (1e-8, 1.0, 1e-8, 1, 1.0),
    "all_d1e-8_lam0.75": (1e-8, 0.75, 1e-8, 1, 0.75),
    "loc_d1e-6_lam1.5_est_lam0.75": (1e-6, 1.5, 1e-7, 1, 0.75),
    "loc_d1e-6_lam2.0_est_lam1.0": (1e-6, 2.0, 1e-7, 1, 1.0),
    "loc_d1e-6_lam1.0_est_lam1.0": (1e-6, 1.0, 1e-7, 1, 1.0),
}
# third round (N3_SET=3): the candidates over more seeds; num = 1.25 k gives the
# cutoff slack against buckets a wide main lobe lets a neighbour share
SETTINGS3 = {
    "all_d1e-7_lam0.75": (1e-7, 0.75, 1e-7, 1, 0.75),
    "all_d1e-7_lam1.0": (1e-7, 1.0, 1e-7, 1, 1.0),
    "all_d1e-7_lam1.0_num1.25k": (1e-7, 1.0, 1e-7, 1.25, 1.0),
    "loc_d1e-7_lam1.25_est_lam1.0_num1.25k": (1e-7, 1.25, 1e-7, 1.25, 1.0),
}
# fourth round (N3_SET=4): a looser location filter next to the lambda = 0.75/B estimation filter
SETTINGS4 = {
    "loc_d1e-6_lam0.75_est_d1e-7_lam0.75": (1e-6, 0.75, 1e-7, 1, 0.75),
    "loc_d1e-5_lam0.75_est_d1e-7_lam0.75": (1e-5, 0.75, 1e-7, 1, 0.75),
    "loc_d1e-5_lam0.875_est_d1e-7_lam0.75": (1e-5, 0.875, 1e-7, 1, 0.75),
}
# fifth round (N3_SET=5, with N3_B=8192): half the buckets, both main-lobe widths
SETTINGS5 = {
    "all_d1e-7_lam0.75": (1e-7, 0.75, 1e-7, 1, 0.75),
    "all_d1e-7_lam0.5": (1e-7, 0.5, 1e-7, 1, 0.5),
}
# sixth round (N3_SET=6, with N3_LEST=4 / 6): fewer estimation-only loops (L = 12 / 14) at the
# C3 bench filter
SETTINGS6 = {
    "all_d1e-7_lam0.75": (1e-7, 0.75, 1e-7, 1, 0.75),
    "all_d1e-7_lam0.5": (1e-7, 0.5, 1e-7, 1, 0.5),
}
if os.environ.get("N3_SET") == "6":
    SETTINGS = SETTINGS6
if os.environ.get("N3_SET") == "5":
    SETTINGS = SETTINGS5
if os.environ.get("N3_SET") == "4":
    SETTINGS = SETTINGS4
if os.environ.get("N3_SET") == "2":
    SETTINGS = SETTINGS2
if os.environ.get("N3_SET") == "3":
    SETTINGS = SETTINGS3

_taps = {}


def taps(delta, lam_b):
    key = (delta, lam_b)
    if key not in _taps:
        p = O.make_params(n, k, B=B, L=16, tolerance=delta, lobefrac=lam_b / B)
        g = O.filter_taps(p)
        _taps[key] = (g, O.filter_response(g, n, nb))
    return _taps[key]


def run_setting(x, S, X, seed, name):
    d_loc, lam_loc, d_est, numf, lam_est = SETTINGS[name]
    g_loc, G_loc = taps(d_loc, lam_loc)
    g_est, G_est = taps(d_est, lam_est)
    a, sigma, tau = O.draw_permutations(seed, n, L_loc + L_est)
    u = np.stack([O.perm_filter(x, g_loc if r < L_loc else g_est, int(sigma[r]), int(tau[r]), B)
                  for r in range(L_loc + L_est)])
    uhat = O.bucket_fft(u)
    J = [O.cutoff(uhat[r], int(numf * k)) for r in range(L_loc)]
    hits = np.sort(O.location_recovery(J, a[:L_loc], n, B, T))
    _, pl_loc = O.estimate(hits, uhat[:L_loc], sigma[:L_loc], tau[:L_loc], G_loc, n, B)
    _, pl_est = O.estimate(hits, uhat[L_loc:], sigma[L_loc:], tau[L_loc:], G_est, n, B)
    per_loop = np.concatenate([pl_loc, pl_est], axis=1)
    med = (per_loop.shape[1] - 1) // 2
    vals = np.sort(per_loop.real, axis=1)[:, med] + 1j * np.sort(per_loop.imag, axis=1)[:, med]
    locs, out = O.select_output(hits, vals, k)
    return {"setting": name, "B": B, "L": L_loc + L_est, "seed": seed, "delta_loc": d_loc, "lambda_loc_B": lam_loc, "delta_est": d_est,
            "lambda_est_B": lam_est, "num": int(numf * k), "w_loc": len(g_loc), "w_est": len(g_est),
            "sum_w": L_loc * len(g_loc) + L_est * len(g_est),
            "exact": bool(set(locs.tolist()) == set(S.tolist())),
            "l1": O.l1_error(locs, out, S, X, k), "hits": int(len(hits))}


def one_seed(s):
    x, S, X = planted_signal(n, k, 1000 + s)
    return [run_setting(x, S, X, 7 + s, name) for name in SETTINGS]


if __name__ == "__main__":
    out, s0, ns, npr = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
    with Pool(npr) as pool, open(out, "a") as f:
        for rows in pool.imap_unordered(one_seed, range(s0, s0 + ns)):
            for r in rows:
                f.write(json.dumps(r) + "\n")
            f.flush()
