"""Summarise the F1 staging-ablation ncu captures (tools/prof_ablation.sh) and timings
(tools/ablate_nbody.py) into one table: per variant and size, the counters that explain each bar
of the paper's Fig. 8 on B200. Usage: python tools/ablation_table.py gpurun_out/ablate OUT_PREFIX"""
import csv
import glob
import json
import os
import sys

NAMES = {"vsmall": "small-N production (in-CTA splits)", "v0": "tma_smem (production)", "v1": "global_scalar",
         "v2": "global_vec", "v3": "readonly_vec", "v4": "local_scalar", "v5": "local_vec", "v6": "constant_vec"}
COLS = [("gpu__time_duration.sum", "ns", 1), ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "gld_req", 1),
        ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "gld_sectors", 1), ("l1tex__t_sector_hit_rate.pct", "L1_hit_%", 0),
        ("lts__t_sectors_srcunit_tex_op_read.sum", "L2_read_sectors", 1), ("lts__t_sector_hit_rate.pct", "L2_hit_%", 0),
        ("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "lds_wavefronts", 1),
        ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", "bank_conflicts", 1),
        ("idc__requests.sum", "const_cache_req", 1),
        ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA_%", 0),
        ("sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "XU_%", 0),
        ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_%", 0),
        ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU_%", 0),
        ("smsp__average_warp_latency_issue_stalled_long_scoreboard.ratio", "stall_long_sb", 0),
        ("smsp__average_warp_latency_issue_stalled_short_scoreboard.ratio", "stall_short_sb", 0)]


def num(x, unit=""):
    try:
        v = float(x.replace(",", ""))
    except (ValueError, AttributeError):
        return None
    if v != v:                                # nan: a launch whose CTAs all exited (mass-uniform split)
        return None
    return v * {"ms": 1e6, "us": 1e3, "usecond": 1e3, "msecond": 1e6}.get(unit, 1.0)


def main(d, out):
    rows = []
    for f in sorted(glob.glob(os.path.join(d, "*.raw.csv"))):
        tag = os.path.basename(f)[:-len(".raw.csv")]
        case, v = tag.rsplit("_", 1)
        rs = [r for r in csv.reader(open(f)) if len(r) > 11]
        if len(rs) < 3:
            continue
        hdr, units, data = rs[0], rs[1], rs[2:]
        agg = {}
        for key, nm, summed in COLS:
            if key not in hdr:
                continue
            j, jt = hdr.index(key), hdr.index("gpu__time_duration.sum")
            pairs = [(num(r[j], units[j]), num(r[jt], units[jt]) or 0.0) for r in data]
            pairs = [(x, w) for x, w in pairs if x is not None]
            if not pairs:
                continue
            if summed:
                agg[nm] = sum(x for x, _ in pairs)
            else:                            # time-weighted mean over the call's kernels
                agg[nm] = sum(x * w for x, w in pairs) / max(sum(w for _, w in pairs), 1e-9)
        agg["kernels"] = sorted({r[hdr.index("Kernel Name")].split("(")[0] for r in data})
        agg["us"] = agg.pop("ns", 0.0) / 1e3
        rows.append({"case": case, "variant": NAMES.get(v, v), **agg})
    with open(out + ".json", "w") as f:
        json.dump(rows, f, indent=1)
    keys = ["us", "gld_sectors", "L1_hit_%", "L2_read_sectors", "lds_wavefronts", "bank_conflicts", "const_cache_req",
            "FMA_%", "XU_%", "issue_%", "LSU_%"]
    with open(out + ".md", "w") as f:
        for case in ("config1_n4096", "config5_p8"):
            f.write(f"\n### {case}\n\n| variant | " + " | ".join(keys) + " |\n|---|" + "---|" * len(keys) + "\n")
            for r in rows:
                if r["case"] != case:
                    continue
                cells = []
                for k in keys:
                    x = r.get(k)
                    cells.append("" if x is None else (f"{x:.3g}" if abs(x) < 1e4 else f"{x:.3e}"))
                f.write(f"| {r['variant']} | " + " | ".join(cells) + " |\n")
    print(open(out + ".md").read())


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
