#!/usr/bin/env python
"""Fold one `ncu --set full` capture of the fused kernel into profiles/ncu_metrics.json, keyed by the
bench's config key, as per-input-byte figures that bench.py scales to its own input size:

  dram_bytes_per_input_byte   (dram__bytes_read.sum + dram__bytes_write.sum) / input bytes
  lds_util                    shared-memory load wavefronts / (SM cycles x SMs): vs 1 wavefront/clk/SM
  bank_conflicts_per_kib      shared-load bank-conflict replays per KiB of input
  alu_pipe_pct / fma_pipe_pct / issue_pct / warps_active_pct / dram_pct (ncu's own percentages)

Usage: ncu_metrics.py REPORT.ncu-rep CONFIG_KEY INPUT_BYTES [SOURCE_NOTE]
"""
import csv
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "profiles", "ncu_metrics.json")


def f(d, k):
    v = d.get(k, "")
    return float(v.replace(",", "")) if v not in ("", "n/a") else None


def main():
    rep, key, nbytes = sys.argv[1], sys.argv[2], float(sys.argv[3])
    note = sys.argv[4] if len(sys.argv) > 4 else os.path.basename(rep)
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, units = rows[0], rows[1]
    d = dict(zip(h, rows[2]))
    unit = {k: units[h.index(k)] for k in h}

    def bytes_of(k):
        v = f(d, k)
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit.get(k, "byte"), 1)
        return v * scale if v is not None else None

    rd, wr = bytes_of("dram__bytes_read.sum"), bytes_of("dram__bytes_write.sum")
    cyc, sms = f(d, "sm__cycles_elapsed.avg"), 148.0
    wav = f(d, "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum")
    bc = f(d, "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum")
    rec = {
        "kernel": d.get("Kernel Name"), "input_bytes": nbytes, "source": note,
        "duration_ms": f(d, "gpu__time_duration.sum") if unit.get("gpu__time_duration.sum") == "ms" else
        (f(d, "gpu__time_duration.sum") or 0) / (1e3 if unit.get("gpu__time_duration.sum") == "us" else 1e6),
        "dram_read_bytes": rd, "dram_write_bytes": wr,
        "dram_bytes_per_input_byte": round((rd + wr) / nbytes, 4) if rd is not None else None,
        "lds_util": round(wav / (cyc * sms), 4) if wav and cyc else None,
        "bank_conflicts": bc, "bank_conflicts_per_kib": round(bc / (nbytes / 1024), 3) if bc is not None else None,
        "alu_pipe_pct": f(d, "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active"),
        "fma_pipe_pct": f(d, "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active"),
        "issue_pct": f(d, "smsp__issue_active.avg.pct_of_peak_sustained_active"),
        "warps_active_pct": f(d, "sm__warps_active.avg.pct_of_peak_sustained_active"),
        "dram_pct": f(d, "dram__throughput.avg.pct_of_peak_sustained_elapsed"),
        "registers": f(d, "launch__registers_per_thread"), "block": f(d, "launch__block_size"),
    }
    db = json.load(open(OUT)) if os.path.exists(OUT) else {}
    db[key] = rec
    with open(OUT, "w") as fh:
        json.dump(db, fh, indent=1, sort_keys=True)
    print(json.dumps({key: rec}))


if __name__ == "__main__":
    main()
