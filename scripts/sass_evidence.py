"""Per-kernel SASS evidence of the Blackwell-native instructions (B200_PROFILING.md table):
UTC*MMA (tcgen05.mma), LDTM/STTM (tcgen05.ld/st), UTMALDG/UTMASTG/UBLKCP (TMA / bulk copy),
UTCBAR (tcgen05.commit), HMMA (legacy mma.sync). usage: python scripts/sass_evidence.py LIB.so"""
import collections
import re
import subprocess
import sys

PAT = re.compile(r"\b(UTC[A-Z]*MMA|UTCBAR|LDTM|STTM|UTMALDG|UTMASTG|UBLKCP|HMMA|DMMA|FFMA2|FFMA|DFMA)\b")


def main():
    lib = sys.argv[1]
    sass = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True, check=True).stdout
    cur, counts = None, collections.OrderedDict()
    for line in sass.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            cur = m.group(1)
            continue
        if cur:
            for op in PAT.findall(line):
                counts.setdefault(cur, collections.Counter())[op] += 1
    for fn, c in counts.items():
        dem = subprocess.run(["c++filt", fn], capture_output=True, text=True).stdout.strip()
        if any(k.startswith(("UTC", "LDTM", "STTM", "UTMA", "UBLK")) for k in c) or "s2t" in dem:
            print(f"{dem[:90]:90s} " + " ".join(f"{k}={v}" for k, v in sorted(c.items())))


if __name__ == "__main__":
    main()
