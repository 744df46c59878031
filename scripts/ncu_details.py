"""Key metrics + rules of an `ncu --page details --csv` export (one or more kernels).
usage: python scripts/ncu_details.py details.csv [section-substring ...]"""
import csv
import sys

KEEP = ("Speed Of Light", "Memory Workload", "Occupancy", "Warp State", "Scheduler", "Launch Stat", "Compute Workload")


def main():
    rows = list(csv.reader(open(sys.argv[1])))
    h = rows[0]
    iK, iS, iM, iU, iV = (h.index(k) for k in ("Kernel Name", "Section Name", "Metric Name", "Metric Unit", "Metric Value"))
    iR = h.index("Rule Description")
    want = sys.argv[2:] or KEEP
    last = None
    for r in rows[1:]:
        r = r + [""] * (len(h) - len(r))
        k = r[iK].split("(")[0]
        if k != last:
            print("==", k)
            last = k
        if r[iM] and any(w in r[iS] for w in want):
            print(f"  {r[iS][:24]:24s} | {r[iM][:48]:48s} | {r[iV]} {r[iU]}")
        elif r[iR]:
            print("  RULE:", r[iR][:300])


if __name__ == "__main__":
    main()
