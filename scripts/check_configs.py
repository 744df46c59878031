"""Run many (N, P, B, Q, precision, M_L) plans through the C ABI and compare each with the oracle's
radix-2 FFT. One child process walks the list; if a config kills the CUDA context, the parent
records it and restarts the child after it.

    python scripts/check_configs.py [N_LOG2 ...]
"""
import itertools
import json
import subprocess
import sys

CHILD = r'''
import sys, json, numpy as np, torch
sys.path.insert(0, ".")
import synth_inputs as SI
from oracle import fmmfft_oracle as O
from paper_conf_sc_cecka17_b200 import FmmFFT
cfgs = json.loads(sys.argv[1])
for k, (N, P, B, Q, prec, M_L) in enumerate(cfgs):
    print(json.dumps({"k": k, "start": True}), flush=True)
    x = SI.complex_uniform(0, N, dtype=np.complex64 if prec == "c64" else np.complex128)
    try:
        y = FmmFFT(N=N, P=P, B=B, Q=Q, precision=prec, M_L=M_L)(torch.from_numpy(x).cuda()).cpu().numpy()
        err = O.rel_l2(y.astype(np.complex128), O.fft_radix2(x))
    except Exception as e:
        print(json.dumps({"k": k, "exc": str(e)[:160]}), flush=True)
        if "CUDA" in str(e) or "illegal" in str(e):
            sys.exit(3)
        continue
    print(json.dumps({"k": k, "err": err}), flush=True)
'''


def main():
    lns = [int(a) for a in sys.argv[1:]] or [20]
    cfgs = []
    for ln, (prec, Qs) in itertools.product(lns, (("c64", (8, 16)), ("c128", (16, 24)))):
        for Q in Qs:
            for lp in range(1, 11):
                P = 1 << lp
                if prec == "c128" and P > 512:
                    continue
                for B in (2, 3, 4):
                    if ln - lp - 6 >= B:
                        cfgs.append([1 << ln, P, B, Q, prec, 64])
    res, start = {}, 0
    while start < len(cfgs):
        r = subprocess.run([sys.executable, "-c", CHILD, json.dumps(cfgs[start:])], capture_output=True, text=True, timeout=1500)
        last = None
        for line in r.stdout.splitlines():
            d = json.loads(line)
            k = start + d["k"]
            last = k
            if "err" in d or "exc" in d:
                res[k] = d
        if last is None:
            print("child failed:", r.stderr[-500:])
            break
        if last not in res:
            res[last] = {"exc": "process died: " + (r.stderr.strip().splitlines() or [""])[-1][:160]}
        start = last + 1
    bad = 0
    for k, cfg in enumerate(cfgs):
        d = res.get(k, {"exc": "not run"})
        tol = 1e-5 if cfg[4] == "c64" else 1e-11
        ok = "err" in d and d["err"] < tol
        bad += not ok
        if not ok:
            print("FAIL", cfg, d, flush=True)
    print(f"{len(cfgs)} configs, {bad} failing")


if __name__ == "__main__":
    main()
