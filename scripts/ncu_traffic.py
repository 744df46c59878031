"""Summarise an `ncu --set full` report: per kernel, duration, DRAM bytes (read + write), SM
throughput, issue activity, occupancy and registers; merge the DRAM bytes into
profiles/ncu_traffic.json under the workload key, and print a table for profiles/.

    python scripts/ncu_traffic.py REPORT.ncu-rep WORKLOAD_KEY [summary.txt]

ncu replays every kernel with caches flushed (--cache-control all), so dram__bytes_read is the
kernel's cold-cache read traffic; writes that stay resident in the 126 MB L2 at kernel end show
as 0 DRAM write bytes (they are written back later, outside the kernel)."""
import csv
import io
import json
import os
import subprocess
import sys

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
           "launch__block_size", "smsp__inst_executed.sum", "lts__t_bytes.sum",
           "smsp__sass_thread_inst_executed_op_ffma_pred_on.sum", "lts__t_sectors.sum",
           "dram__throughput.avg.pct_of_peak_sustained_elapsed",
           "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__pipe_tensor_subpipe_hmma_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
           "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
           "sm__inst_executed_pipe_tensor_subpipe_hmma.sum"]
# added to `--set full` on the capture command line (scripts/profile_r02.sh)
EXTRA = ",".join(METRICS[-6:])
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "us": 1, "ns": 1e-3, "ms": 1e3, "usecond": 1, "nsecond": 1e-3,
        "msecond": 1e3}


def load(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", ",".join(METRICS)],
                         capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        if len(r) != len(hdr):
            continue
        d = {"kernel": r[hdr.index("Kernel Name")].split("(")[0].replace("void ", "").replace("fmmfft::", "").strip()}
        for m in METRICS:
            if m not in hdr:
                continue
            i = hdr.index(m)
            try:
                v = float(r[i].replace(",", ""))
            except ValueError:
                continue
            d[m] = v * UNIT.get(units[i], 1)
        res.append(d)
    return res


def main():
    rep, key = sys.argv[1], sys.argv[2]
    ks = load(rep)
    lines = [f"# {os.path.basename(rep)} ({key}); ncu --set full --clock-control none, one launch per kernel",
             f"{'kernel':34s} {'us':>7s} {'dramR_MB':>9s} {'dramW_MB':>9s} {'L2_MB':>7s} {'SM%':>5s} {'issue%':>6s} "
             f"{'occ%':>5s} {'regs':>4s} {'grid':>6s} {'blk':>5s} {'Minst':>7s} {'dram%':>5s} {'fma%':>5s} {'tens%':>5s}"]
    traffic = {}
    for d in ks:
        name = d["kernel"].split("<")[0]
        dram = d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
        lines.append(f"{d['kernel'][:34]:34s} {d.get('gpu__time_duration.sum', 0):7.2f} "
                     f"{d.get('dram__bytes_read.sum', 0) / 1e6:9.3f} {d.get('dram__bytes_write.sum', 0) / 1e6:9.3f} "
                     f"{d.get('lts__t_bytes.sum', d.get('lts__t_sectors.sum', 0) * 32) / 1e6:7.2f} "
                     f"{d.get('sm__throughput.avg.pct_of_peak_sustained_elapsed', 0):5.1f} "
                     f"{d.get('smsp__issue_active.avg.pct_of_peak_sustained_active', 0):6.1f} "
                     f"{d.get('sm__warps_active.avg.pct_of_peak_sustained_active', 0):5.1f} "
                     f"{d.get('launch__registers_per_thread', 0):4.0f} {d.get('launch__grid_size', 0):6.0f} "
                     f"{d.get('launch__block_size', 0):5.0f} {d.get('smsp__inst_executed.sum', 0) / 1e6:7.3f} "
                     f"{d.get('dram__throughput.avg.pct_of_peak_sustained_elapsed', 0):5.1f} "
                     f"{d.get('sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active', 0):5.1f} "
                     f"{d.get('sm__pipe_tensor_subpipe_hmma_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed', d.get('sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed', 0)):5.1f}")
        if name not in traffic:
            traffic[name] = {"dram_bytes": dram, "tensor_pipe_pct": d.get(
                "sm__pipe_tensor_subpipe_hmma_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed"), "dram_read_bytes": d.get("dram__bytes_read.sum", 0),
                             "dram_write_bytes": d.get("dram__bytes_write.sum", 0), "duration_us": d.get("gpu__time_duration.sum"),
                             "report": os.path.basename(rep)}
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_traffic.json")
    allt = json.load(open(path)) if os.path.exists(path) else {}
    allt[key] = traffic
    json.dump(allt, open(path, "w"), indent=1, sort_keys=True)
    txt = "\n".join(lines) + "\n"
    print(txt)
    if len(sys.argv) > 3:
        open(sys.argv[3], "w").write(txt)


if __name__ == "__main__":
    main()
