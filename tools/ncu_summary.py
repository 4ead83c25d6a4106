"""Compact summary of an ncu report (raw page): duration, pipe utilisation, memory throughput,
DRAM/L2 bytes and the top warp-stall reasons."""
import csv
import subprocess
import sys


def raw(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    units = dict(zip(rows[0], rows[1]))
    return [dict(((k, (v + " " + units.get(k, "")).strip()) for k, v in zip(rows[0], r))) for r in rows[2:]]


KEYS = ["Kernel Name", "gpu__time_duration.sum", "sm__cycles_elapsed.avg",
        "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active"]

if __name__ == "__main__":
    for path in sys.argv[1:]:
        for r in raw(path):
            print("==", path)
            for k in KEYS:
                if k in r:
                    print(f"  {k}: {r[k]}")
            st = {k: float(v) for k, v in r.items() if k.startswith("smsp__pcsamp_warps_issue_stalled_") and
                  not k.endswith("_not_issued") and v.replace('.', '', 1).isdigit()}
            tot = sum(st.values()) or 1
            for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:8]:
                print(f"  stall {k[len('smsp__pcsamp_warps_issue_stalled_'):]}: {100 * v / tot:.1f}%")
