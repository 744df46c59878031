"""Top stall sites of an `ncu --page source --csv` export (SASS view): instruction, samples, and
the column header of the stall breakdown. usage: python scripts/sass_hot.py file.csv.gz [N]"""
import csv
import gzip
import sys

rows = list(csv.reader(gzip.open(sys.argv[1], "rt")))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
hdr = rows[1]
iS, iA, iN = hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
body = [r for r in rows[2:] if len(r) == len(hdr)]
tot = sum(float(r[iA] or 0) for r in body)
print(f"total samples {tot:.0f}, {len(body)} instructions")
# stall-reason columns: those starting with 'stall' if present
stall_cols = [i for i, h in enumerate(hdr) if h.lower().startswith("stall_") or "(stall" in h.lower()]
for idx, r in sorted(enumerate(body), key=lambda t: -float(t[1][iA] or 0))[:n]:
    extra = ""
    if stall_cols:
        top = sorted(((float(r[i] or 0), hdr[i]) for i in stall_cols), reverse=True)[:2]
        extra = "  " + ", ".join(f"{h}={v:.0f}" for v, h in top if v)
    print(f"{float(r[iA] or 0) / tot:6.1%} {idx:5d} {r[iS].strip()[:70]:70s} exec={r[iN]}{extra}")
