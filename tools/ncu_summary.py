"""Summarise ncu reports (.ncu-rep) into JSON: per kernel launch the duration, DRAM
bytes, achieved DRAM bandwidth, registers, occupancy, shared-memory wavefronts and bank
conflicts, global sectors per request and the issue-stall mix.  Reads the reports
with `ncu -i <rep> --page raw --csv` (works without a GPU).

    python tools/ncu_summary.py gpurun_out/prof21_*.ncu-rep > profiles/r01_ncu_summary.json
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct_of_peak",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum": "smem_ld_wavefronts",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum": "smem_st_wavefronts",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum": "smem_ld_conflicts",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum": "smem_st_conflicts",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum": "global_ld_sectors",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum": "global_ld_requests",
    "l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum": "global_st_sectors",
    "l1tex__t_requests_pipe_lsu_mem_global_op_st.sum": "global_st_requests",
    "smsp__inst_executed_op_shfl.sum": "shfl_instructions",
    "smsp__sass_inst_executed_op_shared_ld.sum": "smem_ld_instructions",
    "smsp__sass_inst_executed_op_shared_st.sum": "smem_st_instructions",
    "sm__cycles_elapsed.avg.per_second": "sm_clock_hz",
}


def _num(v):
    try:
        return float(v.replace(",", ""))
    except (ValueError, AttributeError):
        return v


def summarise(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    head, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"report": os.path.basename(rep), "kernel": r[head.index("Kernel Name")][:60]}
        for k, name in KEYS.items():
            if k in head:
                i = head.index(k)
                v = _num(r[i])
                u = units[i]
                if u == "nsecond" and isinstance(v, float):
                    v, u = v / 1e3, "usecond"
                if u == "msecond" and isinstance(v, float):
                    v, u = v * 1e3, "usecond"
                if u in ("Kbyte", "Mbyte", "Gbyte", "byte") and isinstance(v, float):
                    v = v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u]
                    u = "byte"
                d[name] = v
        if "duration" in d and "dram_read" in d:
            d["dram_GBps"] = round((d["dram_read"] + d["dram_write"]) / (d["duration"] * 1e-6) / 1e9, 1)
        res.append(d)
    return res


if __name__ == "__main__":
    allr = []
    for rep in sys.argv[1:]:
        allr += summarise(rep)
    print(json.dumps(allr, indent=1))
