#!/usr/bin/env python3
"""Targeted table update: replace tuning/table.json rows (n, chunk) where a new
sweep's best point beats the row's current configuration by >= --min-gain.

    python scripts/update_table.py NEW.jsonl --n 49-64 --chunks 32,0,64,128,256,-1 \
        [--variants 14] [--min-gain 0.02] [--note "..."]

chunk -1 is the table's "any other chunk" row; it is judged on the chunk-256
measurements (as scripts/make_table.py does) and only takes runtime-stride
configurations (no TMA staging).  The current row's GB/s is looked up in the
new sweep first, then in every tuning/sweep_b200_*.jsonl (latest file wins);
a row whose configuration was never measured at that (n, chunk) is replaced
by the new best.  IEEE points only (fast-math REGX is never chosen)."""
import argparse
import glob
import json
import os
import statistics

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ("variant", "threads_per_block", "param", "staging", "carveout")


def parse_range(s):
    out = []
    for part in s.split(","):
        if "-" in part[1:]:
            a, b = part.split("-")
            out += list(range(int(a), int(b) + 1))
        else:
            out.append(int(part))
    return out


def cfg(r):
    return tuple(r.get(k, 0) for k in KEYS)


def load(path):
    rows = []
    for line in open(path):
        try:
            r = json.loads(line)
        except ValueError:
            continue
        if "gbs" in r and not (r["variant"] == 9 and r["staging"] == 1):
            rows.append(r)
    return rows


def measured(rows, n, chunk):
    """(config -> median GB/s) at (n, chunk)."""
    acc = {}
    for r in rows:
        if r["n"] == n and r["chunk"] == chunk:
            acc.setdefault(cfg(r), []).append(r["gbs"])
    return {k: statistics.median(v) for k, v in acc.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("sweep")
    ap.add_argument("--n", required=True)
    ap.add_argument("--chunks", default="32,0")
    ap.add_argument("--variants", default=None)
    ap.add_argument("--min-gain", type=float, default=0.02)
    ap.add_argument("--table", default=os.path.join(ROOT, "tuning", "table.json"))
    ap.add_argument("--note", default=None)
    ap.add_argument("--dry-run", action="store_true")
    a = ap.parse_args()
    new = load(a.sweep)
    if a.variants:
        vs = set(parse_range(a.variants))
        cand_rows = [r for r in new if r["variant"] in vs]
    else:
        cand_rows = new
    old_files = sorted(glob.glob(os.path.join(ROOT, "tuning", "sweep_b200_*.jsonl")), key=os.path.getmtime)
    table = json.load(open(a.table))
    entries = table["entries"]
    changed = []
    for n in parse_range(a.n):
        for chunk in parse_range(a.chunks):
            mc = 256 if chunk == -1 else chunk
            cands = measured(cand_rows, n, mc)
            if chunk == -1:
                cands = {k: v for k, v in cands.items() if not (k[3] == 1 and k[0] != 8)}
            if not cands:
                continue
            best_k = max(cands, key=cands.get)
            idx = next((i for i, e in enumerate(entries) if e["n"] == n and e["chunk"] == chunk), None)
            cur_k = cfg(entries[idx]) if idx is not None else None
            cur = None
            if cur_k is not None:
                cur = measured(new, n, mc).get(cur_k)
                for f in reversed(old_files):
                    if cur is not None:
                        break
                    cur = measured(load(f), n, mc).get(cur_k)
            gain = None if cur is None else cands[best_k] / cur - 1.0
            if cur_k == best_k or (gain is not None and gain < a.min_gain):
                print(f"n={n:2d} chunk={chunk:3d}: keep {cur_k} ({cur and round(cur)} GB/s; best new "
                      f"{best_k} {cands[best_k]:.0f})")
                continue
            row = dict(n=n, chunk=chunk, **dict(zip(KEYS, best_k)))
            if idx is None:
                entries.append(row)
            else:
                entries[idx] = row
            changed.append((n, chunk))
            print(f"n={n:2d} chunk={chunk:3d}: {cur_k} ({cur and round(cur)} GB/s) -> {best_k} "
                  f"({cands[best_k]:.0f} GB/s{'' if gain is None else f', +{100 * gain:.1f}%'})")
    if changed and not a.dry_run:
        rel = os.path.relpath(a.sweep, ROOT)
        table["source"] += "; " + (a.note or f"{len(changed)} rows from {rel} (>= {100 * a.min_gain:.0f}% better)")
        json.dump(table, open(a.table, "w"), indent=1)
        print(f"{len(changed)} rows updated -> {a.table}")


if __name__ == "__main__":
    main()
