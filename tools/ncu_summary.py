#!/usr/bin/env python
"""Summarise an ncu --set full report (per launch) into JSON for profiles/.

usage: tools/ncu_summary.py REPORT.ncu-rep [--config medium] [--out profiles/x.json]
"""
import argparse
import csv
import io
import json
import subprocess

KEYS = {
    "duration_ns": "gpu__time_duration.sum",
    "sm_clock_hz": "sm__cycles_elapsed.avg.per_second",
    "issue_active_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "fma_pipe_cycles_pct": "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "fma_inst_pct": "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "alu_pipe_cycles_pct": "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "xu_inst_pct": "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "max_warps_pct": "sm__maximum_warps_per_active_cycle_pct",
    "registers": "launch__registers_per_thread",
    "waves_per_sm": "launch__waves_per_multiprocessor",
    "grid": "launch__grid_size",
    "block": "launch__block_size",
    "dram_read_bytes": "dram__bytes_read.sum",
    "dram_write_bytes": "dram__bytes_write.sum",
    "smem_bank_conflicts_ld": "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
    "inst_executed": "smsp__inst_executed.sum",
    "thread_inst_ffma": "smsp__sass_thread_inst_executed_op_ffma_pred_on.sum",
    "thread_inst_fmul": "smsp__sass_thread_inst_executed_op_fmul_pred_on.sum",
    "thread_inst_fadd": "smsp__sass_thread_inst_executed_op_fadd_pred_on.sum",
}
STALLS = ["barrier", "math_pipe_throttle", "wait", "short_scoreboard", "selected", "not_selected",
          "long_scoreboard", "dispatch_stall", "no_instruction", "mio_throttle", "lg_throttle", "branch_resolving",
          "membar", "sleeping", "drain", "imc_miss", "tex_throttle", "misc"]
SCALE = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1.0, "ns": 1.0, "us": 1e3, "ms": 1e6, "usecond": 1e3,
         "msecond": 1e6, "nsecond": 1.0, "Ghz": 1e9, "Mhz": 1e6, "hz": 1.0}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("report")
    ap.add_argument("--out")
    args = ap.parse_args()
    raw = subprocess.run(["ncu", "-i", args.report, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    col = {h: i for i, h in enumerate(hdr)}
    out = []
    for r in data:
        d = {"kernel": r[col["Kernel Name"]]}
        for k, m in KEYS.items():
            if m in col:
                v = r[col[m]].replace(",", "")
                try:
                    d[k] = float(v) * SCALE.get(units[col[m]], 1.0)
                except ValueError:
                    d[k] = v
        st = {}
        tot = 0.0
        for s in STALLS:
            m = f"smsp__pcsamp_warps_issue_stalled_{s}"
            if m in col:
                try:
                    st[s] = float(r[col[m]].replace(",", ""))
                    tot += st[s]
                except ValueError:
                    pass
        if tot:
            d["stall_share"] = {k: round(v / tot, 4) for k, v in sorted(st.items(), key=lambda x: -x[1]) if v}
        out.append(d)
    js = json.dumps(out, indent=1)
    if args.out:
        open(args.out, "w").write(js + "\n")
    print(js)


if __name__ == "__main__":
    main()
