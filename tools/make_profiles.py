"""Turn one gpurun profiling round (gpurun_out/*_<tag>*) into committed summaries under profiles/."""
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
from ncu_summary import summarize  # noqa: E402

KEYMAP = {"nbody1m": "nbody_force_1m", "nbody1m_p8": "nbody_force_1m_p8", "nbody4096": "nbody_force_4096",
          "bs_map": "bs_map", "bs_fused": "bs_map_reduce", "mandel": "mandelbrot", "matmul": "matmul",
          "reduce": "reduce_sum_f32", "cp": "parboil_cp", "mriq": "parboil_mriq",
          "nbody64": "nbody_f64", "series": "jg_series_f32", "idea": "jg_crypt", "sim4096": "nbody_simulate_4096"}


def main(tag):
    out = os.path.join(ROOT, "gpurun_out")
    prof = os.environ.get("PROF_DIR") or os.path.join(ROOT, "profiles")   # PROF_DIR: summarise on the GPU box
    os.makedirs(prof, exist_ok=True)
    summary, traffic = {}, {}
    for k, name in KEYMAP.items():
        rep = os.path.join(out, f"prof_{k}_{tag}.ncu-rep")
        if not os.path.exists(rep):
            continue
        rows = summarize(rep)
        if not rows:
            continue
        summary[name] = rows[0]
        traffic[name] = rows[0].get("dram_read_bytes", 0) + rows[0].get("dram_write_bytes", 0)
    with open(os.path.join(prof, f"ncu_{tag}_summary.json"), "w") as f:
        json.dump(summary, f, indent=1)
    tp = os.path.join(prof, "ncu_traffic.json")
    old = json.load(open(tp)) if os.path.exists(tp) else {}
    old.update(traffic)
    rounds = old.get("_rounds", {})
    rounds.update({k: tag for k in traffic})
    old["_rounds"] = rounds
    old["_source"] = ("dram__bytes_read.sum + dram__bytes_write.sum per launch, ncu --set full; "
                      "latest round that profiled each kernel in _rounds")
    with open(tp, "w") as f:
        json.dump(old, f, indent=1)
    for fn in (f"launches_{tag}.csv", f"bench_{tag}.json"):
        src = os.path.join(out, fn)
        if os.path.exists(src):
            shutil.copy(src, os.path.join(prof, fn))
    # a readable launch-share table from the launch list
    lp = os.path.join(out, f"launches_{tag}.csv")
    if os.path.exists(lp):
        import csv
        tot = {}
        with open(lp) as f:
            lines = [l for l in f if l.startswith('"')]
        for r in csv.DictReader(lines):
            if r.get("Metric Name") != "gpu__time_duration.sum":
                continue
            nm = r["Kernel Name"].split("(")[0][:70]
            v = float(r["Metric Value"].replace(",", ""))
            c, s = tot.get(nm, (0, 0.0))
            tot[nm] = (c + 1, s + v)
        allns = sum(s for _, s in tot.values())
        with open(os.path.join(prof, f"launches_{tag}_shares.txt"), "w") as f:
            f.write(f"# ncu launch list of `python bench.py --steps 3 --warmup 3` (cold-cache, serialised)\n")
            f.write(f"# kernel, launches, total_ms, share\n")
            for nm, (c, s) in sorted(tot.items(), key=lambda kv: -kv[1][1]):
                f.write(f"{nm:72s} {c:5d} {s/1e6:10.3f} {s/allns:7.2%}\n")
    print(json.dumps({k: {kk: v.get(kk) for kk in ("duration_ns", "dram_pct_peak", "pipe_fma_pct", "pipe_tensor_pct", "pipe_xu_pct", "issue_active_pct", "sm_hz")} for k, v in summary.items()}, indent=1))


if __name__ == "__main__":
    main(sys.argv[1])
