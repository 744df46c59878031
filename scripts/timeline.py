"""Execution timeline of one FMM-FFT execute — the analogue of the paper's Figure 2 profile
(nvprof timelines of cuFFTXt and the FMM-FFT). nsys is not in this image; the
kernel activity records come from CUPTI through torch.profiler (kineto), which sees the library's
graph-launched kernels with their device start / end times and streams.

    python scripts/timeline.py [--workload cfg3] [--out profiles/r02_timeline]

Writes <out>_<workload>.txt: one line per kernel of ONE execute (start / end in us from the
first kernel, stream, share of the step), a per-stream busy summary and the overlap of the side
stream (S halo + S2T) with the main stream (the paper's "the FMM computation is parallelized via
CUDA streams and overlaps the FMM communication"); and <out>_<workload>.json, the
Chrome trace of that execute (chrome://tracing / Perfetto).
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import torch
    from torch.profiler import ProfilerActivity, profile

    import bench
    import synth_inputs as SI
    from paper_conf_sc_cecka17_b200 import FmmFFT, build

    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="cfg3")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02_timeline"))
    a = ap.parse_args()
    build.build()
    N, prec, Pf, B, Q, M_L, desc = bench.WORKLOADS[a.workload]
    G = bench.VIRTUAL.get(a.workload, 1)
    P = Pf(G)
    npdt = np.complex64 if prec == "c64" else np.complex128
    x = torch.from_numpy(SI.complex_uniform(0, N, dtype=npdt)).cuda()
    plan = FmmFFT(N=N, P=P, G=G, B=B, Q=Q, precision=prec, M_L=M_L, virtual=G > 1)
    y = torch.empty_like(x)
    for _ in range(5):
        plan(x, out=y)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(3):
            plan(x, out=y)
        torch.cuda.synchronize()
    trace = a.out + f"_{a.workload}.full.json"
    prof.export_chrome_trace(trace)
    with open(trace) as f:
        ev = json.load(f)["traceEvents"]
    os.remove(trace)
    k = [e for e in ev if e.get("cat") == "kernel" and "fmmfft" in e.get("name", "")]
    k.sort(key=lambda e: e["ts"])
    if not k:
        raise SystemExit("no fmmfft kernels recorded (CUPTI unavailable?)")
    # split into executes: the last execute = kernels after the last gap > 50 us... use count per execute
    per = len(k) // 3
    last = k[-per:]
    t0 = min(e["ts"] for e in last)
    t1 = max(e["ts"] + e["dur"] for e in last)
    span = t1 - t0
    streams = sorted({e["args"].get("stream", e.get("tid")) for e in last})
    lines = [f"# one execute of {a.workload} ({desc}; G = {G}{' virtual ranks' if G > 1 else ''}): "
             f"{len(last)} kernels, {span:.1f} us from the first kernel's start to the last kernel's end",
             "# CUPTI kernel records via torch.profiler; streams: " + ", ".join(str(s) for s in streams),
             f"{'start_us':>9} {'end_us':>9} {'dur_us':>8} {'stream':>7}  kernel"]
    for e in last:
        s = e["ts"] - t0
        lines.append(f"{s:9.1f} {s + e['dur']:9.1f} {e['dur']:8.1f} {str(e['args'].get('stream', e.get('tid'))):>7}  "
                     f"{e['name'].split('(')[0]}")
    busy = {}
    for e in last:
        st = e["args"].get("stream", e.get("tid"))
        busy.setdefault(st, []).append((e["ts"] - t0, e["ts"] - t0 + e["dur"]))

    def union(iv):
        iv = sorted(iv)
        out = []
        for s, t in iv:
            if out and s <= out[-1][1]:
                out[-1][1] = max(out[-1][1], t)
            else:
                out.append([s, t])
        return out

    lines.append("# per stream: busy us (union of its kernels) / share of the span")
    u = {st: union(iv) for st, iv in busy.items()}
    for st, iv in u.items():
        b = sum(t - s for s, t in iv)
        lines.append(f"#   stream {st}: {b:.1f} us ({100 * b / span:.0f} %)")
    if len(u) >= 2:
        (sa, ia), (sb, ib) = sorted(u.items(), key=lambda kv: -sum(t - s for s, t in kv[1]))[:2]
        ov = 0.0
        for s, t in ia:
            for s2, t2 in ib:
                ov += max(0.0, min(t, t2) - max(s, s2))
        lines.append(f"# overlap of stream {sb} with stream {sa}: {ov:.1f} us "
                     f"({100 * ov / max(1e-9, sum(t - s for s, t in ib)):.0f} % of stream {sb}'s busy time)")
    with open(a.out + f"_{a.workload}.txt", "w") as f:
        f.write("\n".join(lines) + "\n")
    keep = [e for e in ev if e in last]
    with open(a.out + f"_{a.workload}.json", "w") as f:
        json.dump({"traceEvents": keep}, f)
    print("\n".join(lines[:3] + lines[-6:]))


if __name__ == "__main__":
    main()
