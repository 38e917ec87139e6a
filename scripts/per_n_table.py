#!/usr/bin/env python3
"""Render the "vs n" blocks of a bench.py JSON line as markdown.

    python scripts/per_n_table.py BENCH.json > profiles/r02/per_n.md
"""
import json
import sys

V = {1: "REG", 2: "SMEM", 3: "TILE", 4: "PANEL", 5: "PTMEM", 6: "RTMA", 7: "RTMAP", 8: "QTM",
     9: "REGX", 10: "RCW", 11: "REGV", 12: "RCW16", 13: "RCWD", 14: "RCWP"}


def main():
    r = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    pn, pl = r.get("per_n") or {}, r.get("per_n_large_batch") or {}
    peak = pn.get("peak_gbs")
    print(f"# Batched SPOTRF vs n on one B200 (bench.py, {sys.argv[1]})\n")
    print(f"Factorization: the tuning table's kernel, {pn.get('batch')} matrices, chunk {pn.get('chunk')}, "
          f"dd generator; {pn.get('timing')}.  Fraction of the measured {peak} GB/s copy bandwidth "
          "(MEASURED_PEAKS.json).  Conversion: canonical <-> interleaved of the same batch "
          "(8 n^2 bytes per matrix per direction); canonical path = convert in + factor + convert out.\n")
    print("| n | kernel | GB/s | frac | Gflop/s | vs copy | convert in GB/s (frac) | convert out GB/s (frac) | "
          "canonical path Gflop/s | fused canonical Gflop/s (GB/s) |")
    print("|---|---|---|---|---|---|---|---|---|---|")
    for x in pn.get("rows", []):
        ci, co = x.get("convert_in_gbs"), x.get("convert_out_gbs")
        f = lambda v: f"{v:.0f} ({v / peak:.2f})" if v else "-"
        print(f"| {x['n']} | {V[x['variant']]} | {x['gbs']:.0f} | {x['frac']:.3f} | {x['gflops']:.0f} | "
              f"{x.get('vs_copy', '-')} | {f(ci)} | {f(co)} | {x.get('canonical_path_gflops', '-')} | "
              + (f"{x['canonical_fused_gflops']:.0f} ({x['canonical_fused_gbs']:.0f})" if "canonical_fused_gbs" in x else "-")
              + " |")
    if pl:
        print(f"\nn <= 4 at {pl.get('batch')} matrices (out of the launch-latency regime):\n")
        print("| n | kernel | GB/s | frac | vs copy | convert in GB/s (frac) | convert out GB/s (frac) |")
        print("|---|---|---|---|---|---|---|")
        for x in pl.get("rows", []):
            ci, co = x.get("convert_in_gbs"), x.get("convert_out_gbs")
            f = lambda v: f"{v:.0f} ({v / peak:.2f})" if v else "-"
            print(f"| {x['n']} | {V[x['variant']]} | {x['gbs']:.0f} | {x['frac']:.3f} | {x.get('vs_copy', '-')} | "
                  f"{f(ci)} | {f(co)} |")


if __name__ == "__main__":
    main()
