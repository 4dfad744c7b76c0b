"""Summarise an ncu report: key metrics, stall reasons, hottest SASS lines. python tools/ncu_summary.py rep [nlines]"""
import csv
import subprocess
import sys

rep = sys.argv[1]
nl = int(sys.argv[2]) if len(sys.argv) > 2 else 20
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines()))
h, v = r[0], r[2]
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "smsp__inst_executed.sum", "sm__cycles_elapsed.avg", "lts__t_bytes.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum"]
for k in KEYS:
    if k in h:
        print(f"{k:70s} {v[h.index(k)]}")
st = [(n.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""), float(v[i] or 0))
      for i, n in enumerate(h) if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("per_issue_active.ratio")]
print("stalls:", ", ".join(f"{n}={x:.2f}" for n, x in sorted(st, key=lambda t: -t[1]) if x > 0.05))
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(src.splitlines()))
hh = r[1]
rows = r[2:]
iS, iE = hh.index("Warp Stall Sampling (All Samples)"), hh.index("Instructions Executed")
rows = [x for x in rows if "EXIT" not in x[1]]
rows.sort(key=lambda x: -float(x[iS] or 0))
print("hot SASS (samples, executed, instr):")
for x in rows[:nl]:
    print(f"  {x[iS]:>6} {x[iE]:>9}  {x[1][:100]}")
