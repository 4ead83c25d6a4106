"""Per-launch table of an ncu report (raw page, with units): duration, DRAM bytes read + written,
achieved DRAM GB/s and its fraction of the measured HBM peak (MEASURED_PEAKS.json), tensor-pipe and
FP64-pipe activity, top stall.  Usage: python tools/ncu_table.py report.ncu-rep [...]"""
import csv
import json
import os
import subprocess
import sys

SCALE = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
         "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3, "second": 1.0, "ns": 1e-9, "us": 1e-6, "ms": 1e-3,
         "s": 1.0}


def rows(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(out.splitlines()))
    head, units = r[0], r[1]
    return [{h: (v, u) for h, u, v in zip(head, units, row)} for row in r[2:]]


def val(d, k):
    v, u = d.get(k, ("", ""))
    try:
        return float(v.replace(",", "")) * SCALE.get(u, 1.0)
    except ValueError:
        return None


def main():
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    peak = json.load(open(os.path.join(root, "MEASURED_PEAKS.json")))["hbm_gbs"]
    print(f"HBM peak (MEASURED_PEAKS.json hbm_gbs): {peak:.0f} GB/s\n")
    print("| kernel | ms | DRAM read GB | DRAM write GB | GB/s | frac of HBM peak | tensor % | fp64 pipe % | top stall |")
    print("|---|---|---|---|---|---|---|---|---|")
    for path in sys.argv[1:]:
        for d in rows(path):
            name = d.get("Kernel Name", ("?", ""))[0].split("(")[0].replace("void ", "")
            t = val(d, "gpu__time_duration.sum")
            rd, wr = val(d, "dram__bytes_read.sum") or 0.0, val(d, "dram__bytes_write.sum") or 0.0
            bw = (rd + wr) / t / 1e9 if t else 0.0
            ten = d.get("TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
                        ("", ""))[0]
            f64 = d.get("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", ("", ""))[0]
            st = {k: val(d, k) for k in d if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("_not_issued")}
            st = {k: v for k, v in st.items() if v}
            top = max(st, key=st.get)[len("smsp__pcsamp_warps_issue_stalled_"):] if st else ""
            tot = sum(st.values()) or 1
            print(f"| {name} | {t * 1e3:.3f} | {rd / 1e9:.3f} | {wr / 1e9:.3f} | {bw:.0f} | {bw / peak:.2f} | {ten} | {f64} | "
                  f"{top} {100 * st.get('smsp__pcsamp_warps_issue_stalled_' + top, 0) / tot:.0f}% |")


if __name__ == "__main__":
    main()
