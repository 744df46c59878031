"""Print the quick_perf results: bench value / stage times and the launch summaries."""
import glob
import json
import sys

tag = sys.argv[1]
for f in sorted(glob.glob(f"gpurun_out/q/{tag}_bench_*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "ERR", e, open(f.replace(".json", ".err")).read()[-800:])
        continue
    print(f, f"{d['value']:.0f} GFLOP/s  {d['ms_per_step']*1e3:.1f} us  launches/exec {d['gpu_launches']//d['steps']}")
    print("   stages(us):", {k: round(v * 1e3, 1) for k, v in d["stages_ms"].items()})
    r = d["roofline"]
    print("   roofline:", r["stage"], r["kernel"], r["bound"], f"frac {r['frac']:.3f}")
for f in sorted(glob.glob(f"gpurun_out/q/{tag}_launches_*.txt")):
    print(f)
    print(open(f).read())
for f in sorted(glob.glob(f"gpurun_out/q/{tag}_tests.log")):
    print(open(f).read()[-1500:])
