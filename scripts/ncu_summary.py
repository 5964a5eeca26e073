#!/usr/bin/env python
"""Summarise an ncu --set full report (per kernel launch): duration, pipes, stalls,
smem conflicts, DRAM traffic.  Usage: ncu_summary.py report.ncu-rep [--json out]."""
import csv
import io
import json
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_throughput_pct",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active": "fma_pipe_inst_pct_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_elapsed": "fma_pipe_cycles_pct_elapsed",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed": "tensor_pipe_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "lts__t_bytes.sum": "l2_bytes",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_pct",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum": "smem_ld_conflicts",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum": "smem_st_conflicts",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum": "smem_ld_wavefronts",
    "launch__registers_per_thread": "regs",
    "launch__grid_size": "grid",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
}
STALLS = ["barrier", "dispatch_stall", "long_scoreboard", "math_pipe_throttle", "mio_throttle", "no_instruction",
          "not_selected", "selected", "short_scoreboard", "wait", "lg_throttle", "sleeping", "branch_resolving"]


def to_bytes(v, unit):
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(unit, 1)
    return float(v) * mult


def main(path, out=None):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        e = {"kernel": d.get("Kernel Name", "")[:90], "id": d.get("ID")}
        for k, name in KEYS.items():
            if k in d and d[k] not in ("", "n/a"):
                v = d[k].replace(",", "")
                try:
                    if name.startswith("dram_read") or name.startswith("dram_write") or name == "l2_bytes":
                        e[name] = to_bytes(v, u[k])
                    elif name == "duration":
                        e["duration_us"] = float(v) / (1e3 if u[k] == "nsecond" else 1.0) if u[k] in ("nsecond", "usecond") else float(v)
                        if u[k] == "usecond":
                            e["duration_us"] = float(v)
                        if u[k] == "msecond":
                            e["duration_us"] = float(v) * 1e3
                    else:
                        e[name] = float(v)
                except ValueError:
                    pass
        st = {}
        for s in STALLS:
            k = f"smsp__average_warps_issue_stalled_{s}_per_issue_active.ratio"
            if k in d and d[k]:
                st[s] = round(float(d[k]), 3)
        e["stalls_per_issue"] = st
        res.append(e)
    for e in res:
        print(json.dumps(e))
    if out:
        with open(out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[3] if len(sys.argv) > 3 and sys.argv[2] == "--json" else None)
