"""Condense an ncu summary of the main sweep launch (tools/ncu_summary.py
output) into profiles/ncu_sweep_kernel_current.json, the fractions bench.py
reports under roofline.ncu: issue, ALU pipe, L1/shared LSU wavefronts, DRAM,
and the DRAM bytes per candidate (the roofline's `traffic`).
usage: ncu_current.py <summary.json> <candidates in the captured launch> <tag>"""
import json
import os
import sys

s = json.load(open(sys.argv[1]))[0]
n = float(sys.argv[2])


def v(k):
    x = s.get(k)
    return float(x[0]) if x and x[0] not in ("", None) else None


rd, wr = v("dram__bytes_read.sum"), v("dram__bytes_write.sum")
unit = s.get("dram__bytes_read.sum", [None, "Gbyte"])[1]
scale = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0}.get(unit, 1e9)
out = {
    "capture": sys.argv[3],
    "kernel": s.get("Kernel Name", [""])[0],
    "launch_ms_under_ncu": v("gpu__time_duration.sum"),
    "candidates": n,
    "issue_active_frac": (v("smsp__issue_active.avg.pct_of_peak_sustained_active") or 0) / 100,
    "alu_pipe_frac": (v("TPC.TriageCompute.sm__inst_executed_pipe_alu_realtime.avg.pct_of_peak_sustained_elapsed") or 0) / 100,
    "lsu_wavefronts_frac": (v("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed") or 0) / 100,
    "shared_wavefronts_frac": (v("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed") or 0) / 100,
    "dram_gbs": ((rd or 0) + (wr or 0)) * scale / ((v("gpu__time_duration.sum") or 1) / 1000) / 1e9,
    "dram_bytes_per_candidate": ((rd or 0) + (wr or 0)) * scale / n,
    "warp_instructions": v("smsp__inst_executed.sum"),
    "shared_bank_conflicts": v("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"),
    "registers_per_thread": v("launch__registers_per_thread"),
    "top_stalls_per_issue": s.get("top_stalls_per_issue"),
}
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
try:
    hbm = float(json.load(open(os.path.join(root, "MEASURED_PEAKS.json")))["hbm_gbs"])
except Exception:
    hbm = 6550.0
out["dram_frac"] = out["dram_gbs"] / hbm
out["dram_peak_gbs"] = hbm
fr = {k: out[k] for k in ("issue_active_frac", "alu_pipe_frac", "lsu_wavefronts_frac", "dram_frac")}
out["binding"] = max(fr, key=fr.get)
with open(os.path.join(root, "profiles", "ncu_sweep_kernel_current.json"), "w") as f:
    json.dump(out, f, indent=1)
print(json.dumps(out, indent=1))
