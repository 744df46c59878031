"""Rank SASS instructions of one kernel from `ncu --page source --csv --print-source sass` by
warp-stall samples; also print the instruction-executed totals by opcode."""
import csv
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
I = {h: i for i, h in enumerate(hdr)}
data = [r for r in rows[2:] if len(r) == len(hdr) and r[0] != "Address"]
tot_s = sum(int(r[I["# Samples"]] or 0) for r in data)
tot_i = sum(int(r[I["Instructions Executed"]] or 0) for r in data)
print(f"samples {tot_s}, warp-instructions executed {tot_i}")
ops = Counter()
for r in data:
    op = r[I["Source"]].split()[0] if r[I["Source"]].split() else "?"
    if op.startswith("@"):
        op = r[I["Source"]].split()[1]
    ops[op.split(".")[0]] += int(r[I["Instructions Executed"]] or 0)
print("by opcode:", ", ".join(f"{k}:{v / tot_i:.1%}" for k, v in ops.most_common(14)))
top = sorted(data, key=lambda r: -int(r[I["# Samples"]] or 0))[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]
for r in top:
    st = {k: int(r[I[k]] or 0) for k in hdr if k.startswith("stall_") and "Not Issued" not in k}
    main = sorted(st.items(), key=lambda kv: -kv[1])[:2]
    print(f"{int(r[I['# Samples']]) / tot_s:6.1%}  {r[I['Source']].strip()[:60]:60s} {main}")


def stall_totals(path):
    rows = list(csv.reader(open(path)))
    hdr = rows[1]
    I = {h: i for i, h in enumerate(hdr)}
    data = [r for r in rows[2:] if len(r) == len(hdr) and r[0] != "Address"]
    tot = Counter()
    for r in data:
        for k in hdr:
            if k.startswith("stall_") and "Not Issued" not in k:
                tot[k] += int(r[I[k]] or 0)
    s = sum(tot.values()) or 1
    return ", ".join(f"{k[6:]}:{v / s:.0%}" for k, v in tot.most_common(8))
