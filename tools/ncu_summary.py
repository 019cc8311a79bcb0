"""Summarise ncu --set full reports (raw page) into a compact JSON per kernel."""
import csv
import io
import json
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration_ns",
    "dram__bytes_read.sum": "dram_read_bytes",
    "dram__bytes_write.sum": "dram_write_bytes",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct_peak",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_throughput_pct",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active": "pipe_fma_pct",
    "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active": "pipe_fmaheavy_pct",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active": "pipe_xu_pct",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active": "pipe_alu_pct",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active": "pipe_tensor_pct",
    "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active": "pipe_tc_pct",
    "sm__inst_executed.avg.per_cycle_active": "ipc_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "launch__registers_per_thread": "regs",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "sm__cycles_elapsed.avg.per_second": "sm_hz",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_throughput_pct",
    "lts__t_bytes.sum": "l2_bytes",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum": "smem_ld_bank_conflicts",
    "smsp__thread_inst_executed_per_inst_executed.ratio": "threads_per_inst",
    "lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum": "l2_hit_sectors",
}


def summarize(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return {}
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")][:80]}
        for k, nm in KEYS.items():
            if k in hdr:
                v = r[hdr.index(k)].replace(",", "")
                try:
                    v = float(v)
                except ValueError:
                    pass
                u = units[hdr.index(k)]
                scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
                         "ns": 1, "nsecond": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6,
                         "s": 1e9, "second": 1e9, "Ghz": 1e9, "Mhz": 1e6, "hz": 1}.get(u)
                if scale is not None and isinstance(v, float):
                    v *= scale
                d[nm] = v
        # stall reasons
        stalls = {}
        for i, h in enumerate(hdr):
            if h.startswith("smsp__average_warp_latency_issue_stalled_") or (h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("_not_issued")):
                try:
                    stalls[h.split("stalled_")[1]] = float(r[i].replace(",", ""))
                except ValueError:
                    pass
        top = sorted(stalls.items(), key=lambda kv: -kv[1])[:6]
        d["top_stalls"] = top
        res.append(d)
    return res


if __name__ == "__main__":
    allres = {}
    for rep in sys.argv[1:]:
        allres[rep.split("/")[-1].replace(".ncu-rep", "")] = summarize(rep)
    print(json.dumps(allres, indent=1))
