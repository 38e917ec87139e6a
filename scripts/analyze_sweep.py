#!/usr/bin/env python3
"""Analysis of the B200 autotuning data set, following the
paper's method (Sec. IV): a random-forest regression of the
measured performance on the tuning parameters (R randomForest, 500 trees, in
regression mode) and each parameter's predictive power as
the increase in mean-squared error when that parameter's column is permuted
(Table I's "%IncMSE"), plus the predicted-vs-observed
correlation (Fig. 21).

    python scripts/analyze_sweep.py tuning/sweep_b200_r01*.jsonl > profiles/r01/sweep_analysis.md

The parameters are the B200 axes, mapped to the paper's where they exist:
n; variant (the paper's unrolling / looking / tile-size dimension: REG and
RTMA are fully unrolled with n_b = n, SMEM/PANEL/PTMEM stage a panel, TILE is
the paper's partially unrolled top-looking tile code); chunking (chunked vs
simple interleaved); chunk size; threads per block; panel/tile width; staging
(TMA bulk vs per-thread).
"""
import json
import sys

import numpy as np


def load(paths):
    rows = []
    for p in paths:
        for line in open(p):
            r = json.loads(line)
            if "gbs" in r:
                rows.append(r)
    return rows


def main():
    from sklearn.ensemble import RandomForestRegressor
    from sklearn.model_selection import train_test_split

    rows = load(sys.argv[1:])
    feats = ["n", "variant", "chunking", "chunk size", "threads/block", "panel or tile width", "staging",
             "L1/shared carveout"]
    # carveout: percent of max shared memory preferred (0 = driver default); points
    # without the field were measured at the default (round-1 sweep)
    X = np.array([[r["n"], r["variant"], int(r["chunk"] > 0), r["chunk"] if r["chunk"] > 0 else 0,
                   r["threads_per_block"], r["param"], r["staging"], r.get("carveout", 0)] for r in rows],
                 dtype=float)
    y = np.array([r["gflops"] for r in rows])
    Xtr, Xte, ytr, yte = train_test_split(X, y, test_size=0.25, random_state=2017)
    rf = RandomForestRegressor(n_estimators=500, random_state=2017, n_jobs=-1, oob_score=True)
    rf.fit(Xtr, ytr)
    base = np.mean((rf.predict(Xte) - yte) ** 2)
    rng = np.random.default_rng(2017)
    imp = []
    for j in range(X.shape[1]):
        incs = []
        for _ in range(5):
            Xp = Xte.copy()
            Xp[:, j] = rng.permutation(Xp[:, j])
            incs.append((np.mean((rf.predict(Xp) - yte) ** 2) - base) / base * 100)
        imp.append(np.mean(incs))
    pred = rf.predict(Xte)
    corr = np.corrcoef(pred, yte)[0, 1]
    depth = np.mean([e.get_depth() for e in rf.estimators_])
    print("# B200 autotuning data set: random-forest analysis (paper Sec. IV method)\n")
    print(f"{len(rows)} successful measurements (the paper: > 14,000 on a P100); target = Gflop/s "
          f"(n^3/3 per matrix) at batch 1M.  500 trees, mean depth {depth:.1f} (paper: 500 trees, "
          f"depth 11); out-of-bag R^2 = {rf.oob_score_:.3f}; held-out predicted-vs-observed "
          f"correlation r = {corr:.4f} (the paper's Fig. 21).\n")
    print("| Parameter | %IncMSE (permutation, held-out 25%) | Type |")
    print("|---|---|---|")
    types = ["integer", "categorical (14)", "binary", "integer", "integer", "integer", "categorical (3)",
             "integer (0 = default, 1..100 %)"]
    for f, v, t in sorted(zip(feats, imp, types), key=lambda x: -x[1]):
        print(f"| {f} | {v:.1f} | {t} |")
    print("\nPaper Table I (P100, for comparison): n 43.1; tile size 103.9; looking 99.9; "
          "chunking 157.4; chunk size 25.9; unrolling 85.7; L1/shared -18.6.")
    carve = [r for r in rows if r.get("carveout", 0) != 0]
    if carve:
        import collections
        by = collections.defaultdict(dict)
        for r in rows:
            if r.get("batch", 1 << 20) == 1 << 20:
                by[(r["n"], r["chunk"], r["variant"], r["threads_per_block"], r["param"], r["staging"])][
                    r.get("carveout", 0)] = r["gbs"]
        print("\n## Carveout axis (the tuning table's kernel at each n, 1M matrices)\n")
        print("GB/s at each preferred shared-memory carveout (percent of max shared memory; "
              "default = driver's choice).\n")
        print("| n | chunk | variant | default | 1% | 25% | 50% | 100% | best / default |")
        print("|---|---|---|---|---|---|---|---|---|")
        V = {1: "REG", 2: "SMEM", 3: "TILE", 4: "PANEL", 5: "PTMEM", 6: "RTMA", 7: "RTMAP", 8: "QTM",
             9: "REGX", 10: "RCW", 11: "REGV", 12: "RCW16", 13: "RCWD", 14: "RCWP"}
        for k, d in sorted(by.items()):
            if len(d) < 5:
                continue
            cells = " | ".join(f"{d.get(c, float('nan')):.0f}" for c in (0, 1, 25, 50, 100))
            print(f"| {k[0]} | {k[1]} | {V[k[2]]} | {cells} | {max(d.values()) / d[0]:.3f} |")


if __name__ == "__main__":
    main()
