#!/usr/bin/env python3
"""Register / spill report of the kernels the tuning table selects, from the
LAST ptxas record of each function in build/ptxas.log (the build appends).

    python scripts/check_spills.py [--all] [--chunk 32]
"""
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
V = {1: "REG", 2: "SMEM", 3: "TILE", 4: "PANEL", 5: "PTMEM", 6: "RTMA", 7: "RTMAP", 8: "QTM",
     9: "REGX", 10: "RCW", 11: "REGV", 12: "RCW16", 13: "RCWD", 14: "RCWP"}
KNAME = {1: "potrf_reg_kernel", 2: "potrf_smem_kernel", 3: "potrf_tile_kernel", 4: "potrf_panel_kernel",
         5: "potrf_ptmem_kernel", 6: "potrf_regtma_kernel", 7: "potrf_rtmap_kernel", 8: "potrf_qtm_kernel",
         9: "potrf_regx_kernel", 10: "potrf_rcw_kernel", 11: "potrf_regv_kernel", 12: "potrf_rcw16_kernel",
         13: "potrf_rcwd_kernel", 14: "potrf_rcwp_kernel"}


def parse(path):
    last = {}
    cur = None
    for line in open(path, errors="ignore"):
        m = re.search(r"Function properties for (\S+)", line)
        if m:
            cur = m.group(1)
            continue
        m = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", line)
        if m and cur:
            last.setdefault(cur, {})["spill"] = (int(m.group(1)), int(m.group(2)))
            continue
        m = re.search(r"Used (\d+) registers", line)
        if m and cur:
            last.setdefault(cur, {})["regs"] = int(m.group(1))
            cur = None
    return last


def demangled_args(sym):
    """template args of _ZN3bsp<len><name>I<args>E... as a list of ints/bools."""
    m = re.match(r"_ZN3bsp\d+(\w+?)I(.*)EEvP", sym)
    if not m:
        return None, None
    name, args = m.group(1), m.group(2)
    vals = re.findall(r"L(i|b)(\d+)E", args)
    return name, [int(v) for _, v in vals]


def main():
    recs = parse(os.path.join(ROOT, "build", "ptxas.log"))
    table = json.load(open(os.path.join(ROOT, "tuning", "table.json")))["entries"]
    chunk = None
    if "--chunk" in sys.argv:
        chunk = int(sys.argv[sys.argv.index("--chunk") + 1])
    byname = {}
    for sym, r in recs.items():
        name, args = demangled_args(sym)
        if name:
            byname.setdefault(name, []).append((args, r, sym))
    bad = 0
    print("| n | chunk | variant | param | kernel template args | regs | spill st/ld |")
    print("|---|---|---|---|---|---|---|")
    for e in table:
        if chunk is not None and e["chunk"] != chunk:
            continue
        kn = KNAME[e["variant"]]
        v, n, c = e["variant"], e["n"], e["chunk"]
        tmpl = c in (32, 64, 128)
        want = None
        if v == 1:
            want = [n, c if tmpl else 0, e["param"]]
        elif v in (2, 4, 5):                      # <N, CT, S, TMA>
            tma = 1 if e["staging"] == 1 or (e["staging"] == 0 and (c == 32 if v == 5 else tmpl)) else 0
            ct = c if tma else (32 if c == 32 else 0)
            want = [n, ct, e["param"], tma] + ([0] if v == 5 else [])
            if v == 5 and e["staging"] == 3:          # TMA, fill batches of 12 (FILLT template arg)
                want = [n, 32, e["param"], 1, 0, 12]
        elif v in (10,):
            want = [n, 32 if c == 32 else 0, e["param"]]
        elif v in (12, 13):
            want = [n, 32 if c == 32 else 0]
        elif v == 14:                             # <N, CT, D1, TM, NC>: runtime chunks staged by 2-D TMA
            d1, nc = e["param"] & 1, 3 if e["param"] & 2 else 2
            want = [n, 32, d1, 0, nc] if c == 32 else [n, 0, d1, 1 if n <= 51 else 0, nc]
        elif v == 9:
            want = [n, e["param"], e["staging"]]
        elif v in (6, 7, 3):
            want = [n, e["param"]]
        elif v == 11:
            want = [n]
        cands = [(a, r) for a, r, _ in byname.get(kn, []) if a and a[:len(want)] == want] if want else []
        if not cands:
            print(f"| {n} | {c} | {V[v]} | {e['param']} | (no record for {want}) | - | - |")
        for a, r in cands[:1]:
            sp = r.get("spill", (0, 0))
            bad += sp != (0, 0)
            print(f"| {e['n']} | {e['chunk']} | {V[e['variant']]} | {e['param']} | {a} | {r.get('regs')} | "
                  f"{sp[0]}/{sp[1]} |")
    print(f"\nrows with spills: {bad}")


if __name__ == "__main__":
    main()
