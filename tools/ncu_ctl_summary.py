"""Summarise the smem-counter control captures (tools/jobs/r2s3c.sh) into one JSON:
per case, conflicts and wavefronts per shared-memory instruction from ncu's hardware
counters beside the SASS-attributed (address-derived) wavefronts."""
import csv
import glob
import json
import os
import re
import sys


def metrics(path):
    rows = [l for l in open(path) if l.startswith('"')]
    r = list(csv.reader(rows))
    if not r:
        return None
    h = r[0]
    i, v = h.index("Metric Name"), h.index("Metric Value")
    return {x[i]: float(x[v].replace(",", "")) for x in r[1:]}


def per_instr(m):
    ld_i = m.get("smsp__sass_inst_executed_op_shared_ld.sum") or 0
    st_i = m.get("smsp__sass_inst_executed_op_shared_st.sum") or 0
    f = lambda a, b: round(a / b, 4) if b else None
    return {
        "duration_us": round(m["gpu__time_duration.sum"] / 1e3, 1),
        "GBps_dram": round((m["dram__bytes_read.sum"] + m["dram__bytes_write.sum"]) / m["gpu__time_duration.sum"], 1),
        "registers": m.get("launch__registers_per_thread"),
        "warps_active_pct": m.get("sm__warps_active.avg.pct_of_peak_sustained_active"),
        "lds": ld_i, "sts": st_i,
        "ld_conflicts_per_instr": f(m["l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum"], ld_i),
        "st_conflicts_per_instr": f(m["l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum"], st_i),
        "ld_wavefronts_per_instr_hw": f(m["l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum"], ld_i),
        "st_wavefronts_per_instr_hw": f(m["l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum"], st_i),
        "ld_wavefronts_per_instr_sass": f(m.get("sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", 0), ld_i),
        "st_wavefronts_per_instr_sass": f(m.get("sm__sass_l1tex_data_pipe_lsu_wavefronts_mem_shared_op_st.sum", 0), st_i),
    }


def main(prefix):
    cases = []
    for p in sorted(glob.glob(f"gpurun_out/{prefix}_ncu_*.csv")):
        m = metrics(p)
        if not m:
            continue
        name = os.path.basename(p)[len(prefix) + 5:-4]
        d = {"case": name}
        g = re.match(r"ctl_m(\d)_v(\d+)_na(\d)_one(\d)", name)
        if g:
            d.update({"mode": ["stream", "smem only", "loads only"][int(g[1])], "vectors_per_thread": int(g[2]),
                      "load": "ld.global.nc.L1::no_allocate" if g[3] == "1" else "ld.global",
                      "grid": "one tile per CTA" if g[4] == "1" else "persistent"})
        d.update(per_instr(m))
        cases.append(d)
    return cases


if __name__ == "__main__":
    print(json.dumps(main(sys.argv[1] if len(sys.argv) > 1 else "r2s3c"), indent=1))
