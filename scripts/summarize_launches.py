"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list: per-kernel count,
total and mean duration, and each kernel's share of the library's time per execute."""
import csv
import sys
from collections import OrderedDict


def load(path):
    rows = list(csv.reader(open(path)))
    hdr, out = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d.get("Metric Name", "gpu__time_duration.sum") != "gpu__time_duration.sum":
                continue
            name = d["Kernel Name"].split("(")[0].replace("void ", "")
            out.append((name, d["Grid Size"], d["Block Size"], float(d["Metric Value"])))
    return out


def summarize(path, only_prefix="fmmfft::"):
    ks = [k for k in load(path) if k[0].startswith(only_prefix)]
    agg = OrderedDict()
    for name, grid, blk, ns in ks:
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += ns
    tot = sum(v[1] for v in agg.values())
    lines = [f"{'kernel':40s} {'launches':>8s} {'total_us':>10s} {'mean_us':>9s} {'share':>6s}"]
    for name, (n, ns) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"{name:40s} {n:8d} {ns / 1e3:10.1f} {ns / n / 1e3:9.2f} {ns / tot:6.1%}")
    lines.append(f"{'total':40s} {sum(v[0] for v in agg.values()):8d} {tot / 1e3:10.1f}")
    return "\n".join(lines)


if __name__ == "__main__":
    print(summarize(sys.argv[1]))
