#!/usr/bin/env python3
"""Autotune sweep (JSONL) -> tuning/table.json (best point per (n, chunk)) and a
markdown summary.  Rows: exact chunk 0/32/64/128/256/512, plus chunk -1 ("any
other chunk": best among configurations valid for a runtime chunk stride,
measured at chunk 256)."""
import collections
import json
import sys

src = sys.argv[1]
out_table = sys.argv[2] if len(sys.argv) > 2 else "tuning/table.json"
out_md = sys.argv[3] if len(sys.argv) > 3 else None
rows = [json.loads(l) for l in open(src)]
# the default table is IEEE-only (bitwise reproducible): fast-math REGX points are reported, not chosen
ok = [r for r in rows if "ms" in r and not (r["variant"] == 9 and r["staging"] == 1)]
best = {}
for r in ok:
    k = (r["n"], r["chunk"])
    if k not in best or r["ms"] < best[k]["ms"]:
        best[k] = r
def key(r):
    return dict(variant=r["variant"], threads_per_block=r["threads_per_block"], param=r["param"],
                staging=r["staging"], carveout=r.get("carveout", 0))
entries = []
ns = sorted({r["n"] for r in ok})
for n in ns:
    for c in (0, 32, 64, 128, 256, 512):
        if (n, c) in best:
            entries.append(dict(n=n, chunk=c, **key(best[(n, c)])))
    # any other chunk: runtime-stride-capable best at 256 (else 32 w/o TMA)
    tma = lambda r: r["staging"] == 1 and r["variant"] != 8        # QTM staging 1 is not TMA
    cand = [r for r in ok if r["n"] == n and r["chunk"] in (256, 512) and not tma(r)]
    if not cand:
        cand = [r for r in ok if r["n"] == n and not tma(r)]
    if cand:
        b = min(cand, key=lambda r: r["ms"])
        entries.append(dict(n=n, chunk=-1, **key(b)))
json.dump({"source": f"B200 autotune sweep {src}", "entries": entries}, open(out_table, "w"), indent=1)
print(f"{len(entries)} rows -> {out_table}")
if out_md:
    V = {1: "REG", 2: "SMEM", 3: "TILE", 4: "PANEL", 5: "PTMEM", 6: "RTMA", 7: "RTMAP", 8: "QTM", 9: "REGX", 10: "RCW", 11: "REGV", 12: "RCW16", 13: "RCWD", 14: "RCWP"}
    with open(out_md, "w") as f:
        f.write("| n | best chunk | variant | tpb | param | staging | ms (1M) | GB/s | Gflop/s | "
                "best chunk=0 GB/s | 32 | 64 | 128 | 256 | 512 |\n|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|\n")
        for n in ns:
            bs = {c: best[(n, c)] for c in (0, 32, 64, 128, 256, 512) if (n, c) in best}
            b = min(bs.values(), key=lambda r: r["ms"])
            cells = " | ".join(f"{bs[c]['gbs']:.0f}" if c in bs else "-" for c in (0, 32, 64, 128, 256, 512))
            f.write(f"| {n} | {b['chunk']} | {V[b['variant']]} | {b['threads_per_block']} | {b['param']} | "
                    f"{b['staging']} | {b['ms']:.4f} | {b['gbs']:.0f} | {b['gflops']:.0f} | {cells} |\n")
    print(f"summary -> {out_md}")
