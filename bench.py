"""Benchmark: 1D C2C FFT GFLOP/s = 5 N log2 N / t of the FMM-FFT (BASELINE.json "metric").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl fmmfft|reference] [--workload NAME]

Every N runs the same workload, configs[2] (cfg3: N = 2^26 complex64, P = 16 N, B = 4, Q = 16;
strong scaling — one global FFT of fixed size; at N = 1 its G = 1 shape, P = 16). At N = 1 the
line also carries configs[1] (cfg2: N = 2^20, P = 64, B = 2, Q = 16) as `configs_extra.cfg2`.
`--gpus N` with N > 1 outside torchrun re-launches itself under torch.distributed.run (one rank
per GPU over NCCL) and exits non-zero if fewer than N GPUs are visible.

A "step" is one fmmfft_execute of the whole hot path (Algorithm 1 + POST + the distributed 2D
FFT) on inputs resident in HBM. Between steps L2 is flushed (a 256 MiB write, outside the timed
events). Each step is timed with CUDA events on the launching stream; the K steps are bracketed
by barrier + synchronize; the per-rank median step time is reduced with MAX over ranks. Rank 0
prints ONE JSON line. --impl reference times the CPU float64 oracle (oracle/) on host cores.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import socket
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    # name: (N, precision, P(G), B, Q, M_L, description)
    "cfg1": (1 << 12, "c128", lambda G: 16, 2, 16, 64, "configs[0]: N=2^12 complex128, P=16, B=2, Q=16"),
    "cfg2": (1 << 20, "c64", lambda G: 64, 2, 16, 64, "configs[1]: N=2^20 complex64, P=64, G=1, B=2, Q=16"),
    "cfg3": (1 << 26, "c64", lambda G: 16 * G, 4, 16, 64, "configs[2]: N=2^26 complex64, P=16G, B=4, Q=16"),
    "cfg4": (1 << 28, "c128", lambda G: 64 * G, 2, 24, 64, "configs[3]: N=2^28 complex128, P=64G, B=2, Q=24"),
    # the G = 8 data flow of cfg3 as 8 virtual ranks on ONE GPU (per-rank kernels, halo / all-gather /
    # all-to-all as device copies): evidence for the multi-GPU kernel path, not a scaling number
    "cfg3v8": (1 << 26, "c64", lambda G: 128, 4, 16, 64, "configs[2] at G=8 as 8 virtual ranks on one GPU"),
}
VIRTUAL = {"cfg3v8": 8}
DEFAULT_WORKLOAD = "cfg3"
METRIC = "1D C2C FFT GFLOP/s (5N log2N/t)"
NVLINK_GBS = 770.0      # measured peer copy per direction per GPU (B200_PROFILING.md); 900 nominal

NVML_REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
                0x20: "sync_boost", 0x40: "sw_thermal_slowdown", 0x80: "hw_thermal_slowdown",
                0x100: "hw_power_brake_slowdown", 0x200: "display_clock_setting"}


def flops_fft(N: int) -> float:
    return 5.0 * N * math.log2(N)


class ClockSampler:
    """NVML SM clock + throttle reasons, sampled every 0.5 ms while `active` is set (the timed
    loop), with one sample taken the moment it is set so short loops are covered too."""

    def __init__(self, device_index: int, period_s: float = 0.0005):
        self.samples = []
        self.max_mhz = None
        self._stop = threading.Event()
        self._h = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            self._h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self._h = None
        self.period = period_s
        self.t = threading.Thread(target=self._run, daemon=True)
        self.active = threading.Event()

    def sample(self):
        try:
            mhz = self._nv.nvmlDeviceGetClockInfo(self._h, self._nv.NVML_CLOCK_SM)
            rs = self._nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
            self.samples.append((mhz, rs))
        except Exception:
            pass

    def _run(self):
        while not self._stop.is_set():
            if self.active.wait(timeout=0.05):
                self.sample()
                time.sleep(self.period)

    def __enter__(self):
        if self._h is not None:
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        self.active.set()
        if self._h is not None:
            self.t.join(timeout=2)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": [], "samples": 0}
        mask = 0
        for _, r in self.samples:
            mask |= r
        return {"sm_mhz": statistics.median(m for m, _ in self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": [n for b, n in NVML_REASONS.items() if mask & b and b != 0x1],
                "samples": len(self.samples)}


def load_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def load_traffic(workload: str, G: int, kernel: str):
    """Per-launch DRAM bytes (dram__bytes_read.sum + dram__bytes_write.sum) of one kernel from the
    committed `ncu --set full` summary (profiles/ncu_traffic.json), if it was captured."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        e = d.get(f"{workload}_G{G}", {}).get(kernel)
        return e and e.get("dram_bytes")
    except Exception:
        return None


def stage_rooflines(N, P, B, Q, M_L, G, L, prec, tree_fused, s2t_tc, mfft_kernel, top_L=0, s2t_fft=False,
                    s2m_w=False, s2m_m2m=False):
    """Algorithmic work per execute of each stage, per rank, restated from PAPER.md §5.1
    (P:1159-1174): W = flops (a complex-data x real-operator multiply-add is 2C = 4 real flops),
    D = algorithmic HBM bytes (each operand read once, each result written once). Returns
    {stage: (kernel, flops W, bytes D)}; tests/test_bench_counts.py pins W against the oracle's
    contractions."""
    C, nb = 2, 2 ** L / G
    fmm = P - 1
    esz = 8 if prec == "c64" else 16
    nl = N // G
    up = sum(2 ** l for l in range(B, L)) / G                      # parents formed by M2M
    dn = sum(2 ** l for l in range(B + 1, L + 1)) / G              # targets of M2L / L2L
    m2m = 2 * C * fmm * Q * Q * 2 * up
    down = 2 * C * fmm * Q * Q * 4 * dn
    base = 2 * C * fmm * Q * Q * 2 ** B * (2 ** B - 3) / G
    exp_b = Q * fmm * esz                                          # one box's expansions, all FMMs
    # S2T as the fast convolution (k_s2t_fft): per (box, p) a forward and an inverse 128-point FFT
    # (5 n log2 n each) and 3 complex products per frequency — the flops that kernel performs
    s2t = (("k_s2t_fft", (2 * 5 * 128 * 7 + 3 * 128 * 8) * nb * fmm, 2 * nl * esz) if s2t_fft else
           ("k_s2t_tc" if s2t_tc else "k_near_up", 6 * C * M_L * M_L * nb * fmm, 2 * nl * esz))
    out = {
        "s2m": ("k_s2m_w" if s2m_w else "k_s2m", 2 * C * M_L * nb * fmm * Q, nl * esz + nb * exp_b),
        "s2t": s2t,
        "post_pfft": ("k_post_pfft", 2 * C * M_L * Q * nb * fmm + 5 * nl * math.log2(P), 2 * nl * esz + nb * exp_b),
        "mfft": (mfft_kernel, 5 * nl * math.log2(N // P), 2 * nl * esz),
    }
    if tree_fused:
        out["top"] = ("k_tree_pc", m2m + down + base, 2 * nb * exp_b)
    elif top_L:
        # wide levels per level; levels B..top_L of each FMM in one cluster kernel (k_tree_pc)
        up_w = sum(2 ** l for l in range(top_L, L)) / G
        dn_w = sum(2 ** l for l in range(top_L + 1, L + 1)) / G
        m2m_w = 2 * C * fmm * Q * Q * 2 * up_w
        down_w = 2 * C * fmm * Q * Q * 4 * dn_w
        out["m2m"] = ("k_m2m_lvl", m2m_w, 3 * up_w * exp_b)
        out["top"] = ("k_tree_pc", (m2m - m2m_w) + (down - down_w) + base, 2 * 2 ** top_L / G * exp_b)
        out["down"] = ("k_m2l_lvl", down_w, 3 * dn_w * exp_b)
    else:
        out["m2m"] = ("k_m2m_lvl + k_up", m2m, 3 * up * exp_b)
        out["top"] = ("k_base", base, 2 * 2 ** B * exp_b)
        out["down"] = ("k_m2l_lvl + k_tree_down", down, 3 * dn * exp_b)
    if s2m_m2m and "m2m" in out:
        # the first upward level (parents at L-1) is computed inside k_s2m_w: its flops and its
        # parent write move from the M2M stage to the S2M stage (the M^L re-read disappears)
        par = 2 ** (L - 1) / G
        f1 = 2 * C * fmm * Q * Q * 2 * par
        k, W, D = out["m2m"]
        out["m2m"] = (k, W - f1, D - 3 * par * exp_b)
        k, W, D = out["s2m"]
        out["s2m"] = (k, W + f1, D + par * exp_b)
    return out


# ------------------------------------------------------------------------------ CPU oracle legs
def _oracle_threads(n):
    try:
        from threadpoolctl import threadpool_limits
        return threadpool_limits(n)
    except Exception:
        return None


def oracle_sample(workload: str, G: int, budget_s: float, threads: int = 1):
    """The CPU float64 oracle on a bounded sample of the workload: the full problem if one run
    fits in the budget, else the same (P, B, Q, M_L) at the largest N' that does."""
    import synth_inputs as SI
    from oracle import fmmfft_oracle as O
    N, prec, Pf, B, Q, M_L, _ = WORKLOADS[workload]
    P = Pf(G)
    Ns = P * M_L * (1 << B)                       # smallest legal N' for these parameters: L = B
    lim = _oracle_threads(threads)
    x = SI.complex_uniform(0, Ns)
    t0 = time.perf_counter()
    O.fmmfft(x, P, B, Q, M_L)
    t = time.perf_counter() - t0
    while Ns < N and t * 2.2 < budget_s:
        Ns *= 2
        x = SI.complex_uniform(0, Ns)
        t0 = time.perf_counter()
        O.fmmfft(x, P, B, Q, M_L)
        t = time.perf_counter() - t0
    del lim
    return Ns, P, B, Q, M_L, x


def cpu_baseline(workload: str, G: int, budget_s: float = 12.0):
    """The oracle as it stands timed on the host: 1 thread and all `nproc` threads (numpy's BLAS
    pool; the oracle's einsums are mostly single-threaded, so the two are close)."""
    from oracle import fmmfft_oracle as O
    nproc = os.cpu_count() or 1
    res = {}
    for threads in (1, nproc):
        Ns, P, B, Q, M_L, x = oracle_sample(workload, G, budget_s / 2, threads)
        lim = _oracle_threads(threads)
        times, t_start = [], time.perf_counter()
        while not times or time.perf_counter() - t_start < budget_s / 2:
            t0 = time.perf_counter()
            O.fmmfft(x, P, B, Q, M_L)
            times.append(time.perf_counter() - t0)
        del lim
        t = statistics.median(times)
        res[threads] = (flops_fft(Ns) / t / 1e9, Ns, P, B, Q, M_L, t, len(times))
    v1, vn = res[1], res[nproc]
    return {"value": v1[0], "unit": "GFLOP/s", "cores": 1, "kind": "oracle", "nproc": nproc,
            "sample": f"oracle.fmmfft (numpy float64) at N={v1[1]} with P={v1[2]}, B={v1[3]}, Q={v1[4]}, M_L={v1[5]}; "
                      f"median of {v1[7]} runs ({v1[6]:.3f} s each) on 1 thread",
            "all_cores": {"value": vn[0], "unit": "GFLOP/s", "cores": nproc, "N_sample": vn[1],
                          "sample": f"same, numpy BLAS pool at {nproc} threads, median of {vn[7]} runs ({vn[6]:.3f} s)"}}


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle as it stands, on host cores, rank 0 only."""
    if rank != 0:
        return
    workload = args.workload or DEFAULT_WORKLOAD
    N, prec, Pf, B, Q, M_L, desc = WORKLOADS[workload]
    per_step = max(0.05, 150.0 / (args.steps + args.warmup))
    Ns, P, B, Q, M_L, x = oracle_sample(workload, world, per_step)
    from oracle import fmmfft_oracle as O
    lim = _oracle_threads(1)
    for _ in range(args.warmup):
        O.fmmfft(x, P, B, Q, M_L)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        O.fmmfft(x, P, B, Q, M_L)
        times.append(time.perf_counter() - t0)
    del lim
    t = statistics.median(times)
    val = flops_fft(Ns) / t / 1e9
    sample = (f"oracle.fmmfft (numpy float64, 1 thread) at N={Ns} (of N={N}) with P={P}, B={B}, Q={Q}, "
              f"M_L={M_L}, one run per step, median")
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOP/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": workload, "desc": desc, "N_sample": Ns},
            "cpu_baseline": {"value": val, "unit": "GFLOP/s", "cores": 1, "kind": "oracle", "sample": sample,
                             "nproc": os.cpu_count()},
            "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------ GPU arm
def timed_steps(fn, flush, steps, stream):
    """Per-step ms of fn() by CUDA events on `stream`, L2 flushed before each step (outside)."""
    import torch
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    for a, b_ in ev:
        flush.zero_()
        a.record(stream)
        fn()
        b_.record(stream)
    torch.cuda.synchronize()
    return [a.elapsed_time(b_) for a, b_ in ev]


def roofline_table(stages, N, P, B, Q, M_L, G, info, prec, workload, virt):
    """Per-stage roofline in the paper's model (eq. 3): t_roof = max(W / gamma,
    D / beta); the stage's bound is the larger term, achieved = that work / measured time,
    frac = t_roof / t. Peaks: MEASURED_PEAKS.json HBM copy; FP32 / FP64 FMA from the guide's unit
    counts at the measured max clock; 3xTF32 = measured bf16 dense x 1/2 (tf32 : bf16) / 3."""
    peaks = load_peaks()
    sm_max = peaks.get("sm_max_mhz", 1965.0)
    hbm = peaks.get("hbm_gbs", 6536.4)
    alu = 148 * (128 if prec == "c64" else 64) * 2 * sm_max * 1e6 / 1e12
    tc = peaks.get("bf16_tflops", 1650.0) * 0.5 / 3
    v = info["variant"]
    mk = "k_fft_row" if v & 4 else "k_fft_col + k_fft_rowt" if v & 8 else "k_fft_pass"
    s2t_tc = bool(v & 2)
    rl = {}
    for name, (kname, W, D) in stage_rooflines(N, P, B, Q, M_L, G, info["L"], prec, bool(v & 1), s2t_tc, mk,
                                               info.get("top_level", 0) if v & 512 else 0, bool(v & 128),
                                               bool(v & 256), bool(v & 1024)).items():
        t = stages.get(name)
        if not t or t != t:
            continue
        gamma, gname = (tc, "tensor") if (name == "s2t" and s2t_tc) else (alu, "alu")
        t_w, t_d = W / (gamma * 1e12), D / (hbm * 1e9)
        if t_w >= t_d:
            e = {"bound": gname, "achieved": W / (t * 1e-3) / 1e12, "peak": gamma, "unit": "TFLOP/s",
                 "algorithmic_flops_per_launch": W}
        else:
            e = {"bound": "hbm", "achieved": D / (t * 1e-3) / 1e9, "peak": hbm, "unit": "GB/s",
                 "algorithmic_bytes_per_launch": D}
        e.update(kernel=kname, frac=max(t_w, t_d) / (t * 1e-3), avg_launch_ms=t, flops=W, bytes=D,
                 traffic=load_traffic(workload, G, kname.split(" ")[0]))
        rl[name] = e
    if G > 1 and not virt and stages.get("a2a"):
        D = (G - 1) / G * (N // G) * (8 if prec == "c64" else 16)
        t = stages["a2a"]
        rl["a2a"] = {"kernel": "ncclSend/Recv group", "bound": "nvlink", "achieved": D / (t * 1e-3) / 1e9,
                     "peak": NVLINK_GBS, "unit": "GB/s", "frac": D / (NVLINK_GBS * 1e9) / (t * 1e-3),
                     "avg_launch_ms": t, "algorithmic_bytes_per_launch": D}
    basis = {"alu": f"148 SMs x {'128 FP32' if prec == 'c64' else '64 FP64'} FMA/clk x 2 x {sm_max} MHz (guide unit counts)",
             "tensor": "MEASURED_PEAKS.json bf16 dense x 0.5 (tf32 nominal ratio) / 3 (3xTF32)",
             "hbm": "MEASURED_PEAKS.json HBM copy bandwidth",
             "nvlink": "measured peer copy 770 GB/s per direction (B200_PROFILING.md)"}
    return rl, basis


def measure(workload, world, rank, steps, warmup, flush, stream, barrier, sampler=None, profile=True):
    """Plan, warm up and time one workload; returns a dict of results (rank-local + max over ranks)."""
    import numpy as np
    import torch
    import torch.distributed as dist

    import synth_inputs as SI
    from paper_conf_sc_cecka17_b200 import FmmFFT
    N, prec, Pf, B, Q, M_L, desc = WORKLOADS[workload]
    vg = VIRTUAL.get(workload, 1) if world == 1 else 1
    P, G = Pf(world), world * vg
    npdt = np.complex64 if prec == "c64" else np.complex128
    esz = 8 if prec == "c64" else 16
    kw = dict(N=N, P=P, G=G, B=B, Q=Q, precision=prec, M_L=M_L, virtual=vg > 1)
    plan = FmmFFT(**kw)
    x_host = SI.shard(N, world, rank, dtype=npdt)
    x = torch.from_numpy(x_host).cuda()
    y = torch.empty_like(x)
    for _ in range(max(3, warmup)):
        flush.zero_()
        plan(x, y, stream)
    torch.cuda.synchronize()

    # ---- the timed region: K steps, CUDA events per step on the launching stream
    barrier()
    torch.cuda.synchronize()
    if sampler:
        sampler.active.set()
        sampler.sample()
    step_ms = timed_steps(lambda: plan(x, y, stream), flush, steps, stream)
    if sampler:
        sampler.sample()
        sampler.active.clear()
    barrier()
    info = plan.info
    t = torch.tensor([statistics.median(step_ms), sum(step_ms) / len(step_ms)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_med, ms_mean = float(t[0]), float(t[1])
    res = {"workload": workload, "desc": desc, "N": N, "P": P, "G": G, "B": B, "Q": Q, "M_L": M_L, "prec": prec,
           "vg": vg, "esz": esz, "info": info, "ms": ms_med, "ms_mean": ms_mean,
           "value": flops_fft(N) / (ms_med * 1e-3) / 1e9, "x": x, "y": y, "x_host": x_host, "plan": plan, "kw": kw}

    # ---- correctness of the timed output: Parseval over the whole job (any size)
    ny = torch.sum(torch.abs(y.to(torch.complex128)) ** 2)
    nx = torch.sum(torch.abs(x.to(torch.complex128)) ** 2)
    if world > 1:
        dist.all_reduce(ny)
        dist.all_reduce(nx)
    res["parseval_rel_dev"] = float(ny / (N * nx) - 1)

    # ---- per-stage breakdown: a separate profiled plan (events at every stage boundary, near field
    # serialised so every interval holds only its own kernels), K more steps
    if profile:
        plan_p = FmmFFT(profile=True, **kw)
        y2 = torch.empty_like(x)
        for _ in range(3):
            plan_p(x, y2, stream)
        stage_sum = {}
        barrier()
        for _ in range(steps):
            flush.zero_()
            plan_p(x, y2, stream)
            for n_, v in plan_p.stage_times().items():
                stage_sum.setdefault(n_, []).append(v)
        barrier()
        stages = {n_: statistics.median(v) for n_, v in stage_sum.items()}
        if world > 1:
            names = sorted(stages)
            tt = torch.tensor([stages[n_] for n_ in names], dtype=torch.float64, device="cuda")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            stages = dict(zip(names, tt.tolist()))
        plan_p.close()
        res["stages"] = stages
        res["rl"], res["basis"] = roofline_table(stages, N, P, B, Q, M_L, G, info, prec, workload, vg > 1)
        dom = max(res["rl"], key=lambda k: res["rl"][k]["avg_launch_ms"])
        res["roofline"] = dict(res["rl"][dom], stage=dom, peak_basis=res["basis"][res["rl"][dom]["bound"]])
    return res


def e2e_measure(res, world, steps, stream, barrier):
    """Same metric end to end through the C ABI with HOST buffers: every step copies its input
    from pinned host memory and its output back (fmmfft_execute_host), inside the events."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_cecka17_b200 import FmmFFT
    xh = torch.from_numpy(res["x_host"]).pin_memory()
    yh = torch.empty_like(xh).pin_memory()
    plan_e2e = FmmFFT(**res["kw"])
    for _ in range(2):
        plan_e2e.execute_host(xh, yh, stream)
    torch.cuda.synchronize()
    k = max(3, min(steps, 20))
    ee = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(k)]
    barrier()
    torch.cuda.synchronize()
    for a, b_ in ee:
        a.record(stream)
        plan_e2e.execute_host(xh, yh, stream)
        b_.record(stream)
    torch.cuda.synchronize()
    barrier()
    t = torch.tensor([statistics.median(a.elapsed_time(b_) for a, b_ in ee)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    plan_e2e.close()
    nb = xh.numel() * xh.element_size()
    return {"value": flops_fft(res["N"]) / (float(t) * 1e-3) / 1e9, "unit": "GFLOP/s",
            "h2d_bytes_per_step": nb, "d2h_bytes_per_step": nb, "ms_per_step": float(t),
            "api": "fmmfft_execute_host (pinned host buffers; H2D + execute + D2H per step)"}


def cufft_comparator(x, flush, steps):
    """cuFFT (torch.fft.fft, the library 1D FFT) on the same device, input, L2 flush and event
    timing: the single-GPU comparator of BASELINE.json's "speedup vs cuFFTXt" (context), plus the
    library's own four-step FFT of the whole vector without the FMM (FMMFFT_FLAG_DIRECT)."""
    import torch
    st = torch.cuda.current_stream()
    for _ in range(3):
        torch.fft.fft(x)
    torch.cuda.synchronize()
    ms = statistics.median(timed_steps(lambda: torch.fft.fft(x), flush, steps, st))
    out = {"lib": "cuFFT via torch.fft.fft (1 GPU)", "value": flops_fft(x.numel()) / (ms * 1e-3) / 1e9,
           "unit": "GFLOP/s", "ms_per_step": ms}
    try:
        from paper_conf_sc_cecka17_b200 import FmmFFT
        prec = "c64" if x.dtype == torch.complex64 else "c128"
        d = FmmFFT(N=x.numel(), P=1, precision=prec, direct=True)
        y = torch.empty_like(x)
        for _ in range(3):
            d(x, y, st)
        torch.cuda.synchronize()
        ms_d = statistics.median(timed_steps(lambda: d(x, y, st), flush, steps, st))
        out["inhouse_fourstep"] = {"value": flops_fft(x.numel()) / (ms_d * 1e-3) / 1e9, "unit": "GFLOP/s",
                                   "ms_per_step": ms_d, "kernels": "k_fft_col + k_fft_rowt (no FMM)"}
        d.close()
    except Exception as e:  # the comparator is context only
        out["inhouse_fourstep"] = {"error": str(e)[:200]}
    return out


def cufftxt_comparator(N, prec, ngpu, steps, y_block):
    """cuFFTXt on the same box: one process driving all N GPUs (cufftXtSetGPUs), same N, same
    seeded input; reported with the output left in cuFFT's multi-GPU order and with the
    device-to-device reorder to natural order. Runs in a child process of rank 0 (a library
    comparator must not be able to take the bench down), while the other ranks wait."""
    code = r'''
import ctypes, json, sys, numpy as np
sys.path.insert(0, sys.argv[1])
import synth_inputs as SI
N, ngpu, dbl, iters = int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), int(sys.argv[5])
lib = ctypes.CDLL(sys.argv[6])
x = SI.complex_uniform(0, N, dtype=np.complex128 if dbl else np.complex64)
y = np.empty_like(x)
ms = (ctypes.c_double * 2)()
err = ctypes.create_string_buffer(512)
rc = lib.cufftxt_bench(ctypes.c_longlong(N), ngpu, dbl, iters, x.ctypes.data_as(ctypes.c_void_p),
                       y.ctypes.data_as(ctypes.c_void_p), ms, err, 512)
n = N // ngpu
np.save(sys.argv[7], y[:n])
print(json.dumps({"rc": rc, "err": err.value.decode(), "ms": [ms[0], ms[1]]}))
'''
    import numpy as np
    from paper_conf_sc_cecka17_b200 import build as b
    lib = b.build_comparator()
    tmp = os.path.join("/tmp", f"cufftxt_y0_{os.getpid()}.npy")
    try:
        r = subprocess.run([sys.executable, "-c", code, ROOT, str(N), str(ngpu), "1" if prec == "c128" else "0",
                            str(max(5, min(steps, 20))), lib, tmp], capture_output=True, text=True, timeout=600)
        d = json.loads(r.stdout.strip().splitlines()[-1])
    except Exception as e:
        return {"lib": "cuFFTXt", "error": f"{type(e).__name__}: {str(e)[:200]}"}
    if d["rc"]:
        return {"lib": "cuFFTXt", "error": d["err"]}
    out = {"lib": f"cuFFTXt 1D C2C, cufftXtSetGPUs({ngpu}), single process", "unit": "GFLOP/s",
           "timing": "host wall clock around back-to-back executes, every device synchronised",
           "shuffled": {"ms_per_step": d["ms"][0], "value": flops_fft(N) / (d["ms"][0] * 1e-3) / 1e9,
                        "note": "output left in cuFFT's multi-GPU (shuffled) order"},
           "natural": {"ms_per_step": d["ms"][1], "value": flops_fft(N) / (d["ms"][1] * 1e-3) / 1e9,
                       "note": "+ cufftXtMemcpy device-to-device into natural order (our output's order)"}}
    try:
        y0 = np.load(tmp)
        out["rel_l2_vs_fmmfft_rank0"] = float(np.linalg.norm(y0 - y_block) / np.linalg.norm(y0))
        os.remove(tmp)
    except Exception:
        pass
    return out


def inhouse_3transpose(N, prec, world, x, flush, steps, stream, barrier):
    """The library's own distributed radix-P Cooley-Tukey FFT with THREE all-to-alls
    (FMMFFT_FLAG_DIRECT at G > 1): same N, same shards, same
    exchange code and M-FFT kernels as the FMM-FFT, so the ratio isolates the transposes saved."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_cecka17_b200 import FmmFFT
    d = FmmFFT(N=N, P=1, G=world, precision=prec, direct=True)
    y = torch.empty_like(x)
    for _ in range(3):
        d(x, y, stream)
    torch.cuda.synchronize()
    barrier()
    ms = statistics.median(timed_steps(lambda: d(x, y, stream), flush, steps, stream))
    barrier()
    t = torch.tensor([ms], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    d.close()
    return {"value": flops_fft(N) / (float(t) * 1e-3) / 1e9, "unit": "GFLOP/s", "ms_per_step": float(t),
            "kernels": "k_transpose_rc, k_fft_col + k_fft_rowt, k_twiddle_chunk, k_fft_col + 3 NCCL all-to-alls"}


def autotuned_pick(N, prec, flush, steps, x, stream):
    import torch
    from paper_conf_sc_cecka17_b200 import FmmFFT, autotune
    tol = 1e-5 if prec == "c64" else 1e-11
    t = autotune(N, 1, prec, tol, True)
    pa = FmmFFT(N=N, P=t["P"], G=1, B=t["B"], Q=t["Q"], precision=prec, M_L=t["M_L"])
    ya = torch.empty_like(x)
    for _ in range(3):
        pa(x, ya, stream)
    torch.cuda.synchronize()
    ms = statistics.median(timed_steps(lambda: pa(x, ya, stream), flush, steps, stream))
    pa.close()
    return {"P": t["P"], "B": t["B"], "Q": t["Q"], "M_L": t["M_L"], "tol": tol, "predicted_error": t["error"],
            "value": flops_fft(N) / (ms * 1e-3) / 1e9, "unit": "GFLOP/s", "ms_per_step": ms,
            "note": "fmmfft_autotune pick for the same N / precision / error bound; context, not the headline"}


def real_comparator(N, P, B, Q, prec, M_L, flush, steps):
    """Context: the real-input transform (FMMFFT_FLAG_REAL) of 2N reals, whose
    complex plan is this workload's (N, P, B, Q), against cuFFT's rfft (torch.fft.rfft) on the same
    seeded input, same L2 flush and event timing. GFLOP/s use the real-FFT convention 2.5 n log2 n."""
    import torch
    import synth_inputs as SI
    from paper_conf_sc_cecka17_b200 import FmmFFT
    n = 2 * N
    rdt = torch.float32 if prec == "c64" else torch.float64
    xr = torch.from_numpy(SI.real_uniform(0, n)).to(rdt).cuda()
    out = {"n_real": n, "flops_convention": "2.5 n log2 n"}
    plan = FmmFFT(N=n, P=P, B=B, Q=Q, precision=prec, M_L=M_L, real=True)
    y = torch.empty(N + 1, dtype=plan.dtype, device="cuda")
    st = torch.cuda.current_stream()
    for name, fn in (("fmmfft_r2c", lambda: plan(xr, y, st)), ("cufft_rfft", lambda: torch.fft.rfft(xr))):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        ms = statistics.median(timed_steps(fn, flush, steps, st))
        out[name] = {"value": 2.5 * n * math.log2(n) / (ms * 1e-3) / 1e9, "unit": "GFLOP/s", "ms_per_step": ms}
    plan.close()
    return out


def run_fmmfft(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_cecka17_b200 import init_comm
    from paper_conf_sc_cecka17_b200 import build as b

    if rank == 0:
        b.build()
    if world > 1:
        dist.barrier()
    torch.cuda.set_device(local_rank)
    if world > 1:
        init_comm()
    workload = args.workload or DEFAULT_WORKLOAD
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()

    sampler = ClockSampler(local_rank if "CUDA_VISIBLE_DEVICES" not in os.environ else torch.cuda.current_device())
    with sampler:
        res = measure(workload, world, rank, args.steps, args.warmup, flush, stream, barrier, sampler)
    e2e = e2e_measure(res, world, args.steps, stream, barrier)
    N, prec = res["N"], res["prec"]
    comp_steps = min(args.steps, 50)
    extras = {}
    if world == 1 and not args.no_extras:
        extras["comparator"] = cufft_comparator(res["x"], flush, comp_steps)
        try:
            extras["autotuned"] = autotuned_pick(N, prec, flush, comp_steps, res["x"], stream)
        except Exception as e:
            extras["autotuned"] = {"error": str(e)[:200]}
        if res["vg"] == 1:
            try:
                extras["real_input"] = real_comparator(N, res["P"], res["B"], res["Q"], prec, res["M_L"], flush, comp_steps)
            except Exception as e:  # context only
                extras["real_input"] = {"error": str(e)[:200]}
        if workload != "cfg2":
            c2 = measure("cfg2", 1, 0, args.steps, args.warmup, flush, stream, barrier)
            c2_cmp = cufft_comparator(c2["x"], flush, comp_steps)
            extras["configs_extra"] = {"cfg2": {
                "desc": c2["desc"], "value": c2["value"], "unit": "GFLOP/s", "ms_per_step": c2["ms"],
                "roofline": c2["roofline"], "stages_ms": c2["stages"],
                "comparator": {"cuFFT": c2_cmp["value"], "inhouse_fourstep": c2_cmp["inhouse_fourstep"].get("value")},
                "parseval_rel_dev": c2["parseval_rel_dev"], "kernels_per_execute": c2["info"]["kernels_per_execute"]}}
            c2["plan"].close()
    if world > 1 and not args.no_extras:
        try:
            extras["inhouse_3transpose"] = inhouse_3transpose(N, prec, world, res["x"], flush, comp_steps, stream, barrier)
        except Exception as e:  # context only
            extras["inhouse_3transpose"] = {"error": str(e)[:200]}
        yb = res["y"].cpu().numpy() if rank == 0 else None
        if rank == 0:
            extras["comparator"] = cufftxt_comparator(N, prec, world, comp_steps, yb)
        barrier()
    if rank != 0:
        res["plan"].close()
        return
    clocks = sampler.summary()
    info = res["info"]
    line = {
        "metric": METRIC, "value": res["value"], "unit": "GFLOP/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms"], "higher_is_better": True,
        "scaling": "strong" if res["vg"] == 1 else "n/a (virtual ranks on one GPU)", "vs_baseline": None,
        "dtype": "f32" if prec == "c64" else "f64", "data": "synthetic",
        "config": {"workload": workload, "desc": res["desc"], "N": N, "P": res["P"], "G": res["G"], "B": res["B"],
                   "Q": res["Q"], "M_L": res["M_L"], "L": info["L"], "precision": prec,
                   "l2": "flushed (256 MiB write between steps, outside events); inputs 512 MiB > L2",
                   "timing": "median of K per-step CUDA-event times, max over ranks",
                   "ms_mean": res["ms_mean"], "parseval_rel_dev": res["parseval_rel_dev"]},
        "roofline": res["roofline"],
        "stages_roofline": res["rl"],
        "stages_ms": res["stages"],
        "e2e": e2e,
        "gpu_launches": info["kernels_per_execute"] * args.steps,
        "clocks": {k: clocks[k] for k in ("sm_mhz", "sm_max_mhz", "reasons", "samples")},
    }
    if res["vg"] > 1:
        line["config"]["virtual_ranks"] = res["vg"]
    if "a2a" in res["rl"]:
        line["a2a"] = res["rl"]["a2a"]
    elif world == 1:
        line["a2a"] = {"note": "G = 1: the transpose is local (no NVLink traffic)"}
    line.update(extras)
    if world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline(workload, res["G"])
    res["plan"].close()
    print(json.dumps(line), flush=True)


def free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def self_launch(args) -> int:
    """--gpus N > 1 outside torchrun: one rank per GPU under torch.distributed.run."""
    import torch
    have = torch.cuda.device_count()
    if have < args.gpus:
        print(f"bench.py: --gpus {args.gpus} needs {args.gpus} visible GPUs, found {have}", file=sys.stderr)
        return 2
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.run(cmd).returncode


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="fmmfft", choices=["fmmfft", "reference"])
    ap.add_argument("--workload", default=None, choices=sorted(WORKLOADS))
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-extras", action="store_true",
                    help="skip the comparators and the autotuner pick (profiling runs: only the FMM-FFT's launches)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    in_torchrun = "WORLD_SIZE" in os.environ
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world if in_torchrun else args.gpus)
        return
    if not in_torchrun and args.gpus > 1:
        sys.exit(self_launch(args))
    if in_torchrun and world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}", file=sys.stderr)
        sys.exit(2)
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        run_fmmfft(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.barrier()
            from paper_conf_sc_cecka17_b200 import destroy_comm
            destroy_comm()
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
