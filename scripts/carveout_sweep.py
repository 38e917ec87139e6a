#!/usr/bin/env python3
"""Carveout axis of the autotuning sweep (Table I's "L1 or shared" parameter,
PAPER.md:216,407): for the tuning table's row of each n (and
chunk), time the same kernel at every preferred shared-memory carveout.

    python scripts/carveout_sweep.py --n 1-64 --chunks 32,0 --carveouts 0,1,25,50,100 --out sweep.jsonl

Delegates to scripts/autotune.py (--only = the table row, --carveouts)."""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", default="4,8,12,16,20,24,28,32,36,40,44,48,52,56,60,64")
    ap.add_argument("--chunks", default="32,0")
    ap.add_argument("--carveouts", default="0,1,25,50,100")
    ap.add_argument("--batch", type=int, default=1 << 20)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--out", required=True)
    a = ap.parse_args()
    import paper_conf_ipps_gatesklpd17_b200 as bsp
    ns = []
    for part in a.n.split(","):
        if "-" in part:
            lo, hi = part.split("-")
            ns += list(range(int(lo), int(hi) + 1))
        else:
            ns.append(int(part))
    for chunk in [int(c) for c in a.chunks.split(",")]:
        for n in ns:
            t = bsp.bspotrf_get_tuning(n, chunk).as_dict()
            only = [dict(t, n=n, chunk=chunk)]
            cmd = [sys.executable, os.path.join(ROOT, "scripts", "autotune.py"), "--n", str(n),
                   "--chunks", str(chunk), "--batch", str(a.batch), "--reps", str(a.reps),
                   "--variants", "1,2,3,4,5,6,7,8,9,10,11,12", "--carveouts", a.carveouts,
                   "--only", json.dumps(only), "--out", a.out]
            subprocess.run(cmd, check=True)
            print(f"n={n} chunk={chunk} done", flush=True)


if __name__ == "__main__":
    main()
