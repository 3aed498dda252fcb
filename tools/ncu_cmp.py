"""Compare key metrics across ncu reports: python tools/ncu_cmp.py a.ncu-rep b.ncu-rep ..."""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "smsp__inst_executed.sum", "sm__inst_issued.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active"]
STALLS = ["short_scoreboard", "long_scoreboard", "wait", "selected", "not_selected", "branch_resolving", "mio_throttle",
          "lg_throttle", "math_pipe_throttle", "dispatch_stall", "no_instruction", "barrier", "membar", "sleeping", "drain", "misc", "tex_throttle"]


def load(p):
    out = subprocess.run(["ncu", "-i", p, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return dict(zip(r[0], r[2]))


reps = [(p.split("/")[-1].replace(".ncu-rep", ""), load(p)) for p in sys.argv[1:]]
print(f"{'metric':70s}" + "".join(f"{n[:16]:>18s}" for n, _ in reps))
for k in KEYS:
    print(f"{k[:70]:70s}" + "".join(f"{d.get(k, '-')[:16]:>18s}" for _, d in reps))
for st in STALLS:
    k = f"smsp__average_warps_issue_stalled_{st}_per_issue_active.ratio"
    print(f"{'stall ' + st:70s}" + "".join(f"{d.get(k, '-')[:16]:>18s}" for _, d in reps))
