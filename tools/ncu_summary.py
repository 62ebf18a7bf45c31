"""Summarise an ncu report: key throughput metrics + warp stall breakdown.  Usage: ncu_summary.py rep"""
import csv
import subprocess
import sys

rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h, units = rows[0], rows[1]
keys = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__block_size", "launch__grid_size",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "smsp__inst_executed.sum", "sm__cycles_elapsed.avg", "lts__t_sectors_srcunit_tex_op_read.sum",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed"]
for r in rows[2:]:
    d = dict(zip(h, r))
    print("=" * 80)
    for k in keys:
        if k in d:
            u = units[h.index(k)]
            print(f"{k:70s} {d[k]:>18s} {u}")
    st = {k: d[k] for k in h if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
    tot = sum(float(v.replace(",", "") or 0) for v in st.values())
    for k, v in sorted(st.items(), key=lambda kv: -float(kv[1].replace(",", "") or 0))[:8]:
        fv = float(v.replace(",", "") or 0)
        if fv:
            print(f"  stall {k[len('smsp__pcsamp_warps_issue_stalled_'):]:40s} {100 * fv / tot:5.1f}%")
