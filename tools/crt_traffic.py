"""DRAM traffic record of the dominant kernel for bench.py's `roofline.traffic` (profiles/r02/ncu_traffic_crt.json).

  python tools/crt_traffic.py <config> <skip> <ncu_summary.txt> <out.json>

The ncu capture (tools/ncu_session.sh crt: `-k regex:crt_gemm_kernel<(int)16 -s <skip> -c 1` of
tools/one_eval.py <config> 0) gives DRAM read/write bytes and the duration of ONE CRT-16 launch; this
script runs the same single evaluation WITHOUT ncu, with per-launch profiling of the FP64 class on
and MPGEO_TIMELINE set, and takes the FP64-equivalent flops of the (skip+1)-th FP64-class launch
(launches are recorded in host issue order, the order ncu counts them).  Writes bytes per flop."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


SCALE = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ms": 1.0, "us": 1e-3, "s": 1e3,
         "%": 1.0, "": 1.0}


def ncu_fields(path):
    """name -> value in bytes / ms (the summary prints 'value unit')."""
    d = {}
    for line in open(path):
        line = line.strip()
        if ":" in line:
            k, v = line.split(":", 1)
            f = v.split()
            try:
                d[k.strip()] = float(f[0]) * SCALE.get(f[1] if len(f) > 1 else "", 1.0)
            except (ValueError, IndexError):
                pass
    return d


def main():
    cfg_name, skip, summ, out = sys.argv[1], int(sys.argv[2]), sys.argv[3], sys.argv[4]
    tl = "/tmp/crt_traffic_timeline.txt"
    if os.path.exists(tl):
        os.remove(tl)
    os.environ["MPGEO_TIMELINE"] = tl
    import torch

    import paper_conf_cluster_caoalgkb23_b200 as mp
    import synth
    from bench import CONFIGS
    cfg = CONFIGS[cfg_name]
    n, nb = cfg["n"], cfg["nb"]
    x, y = synth.locations(n, seed=0)
    z = synth.normal_vector(n, seed=1)
    dx, dy, dz = (torch.from_numpy(v).cuda() for v in (x, y, z))
    ev = mp.Evaluator(n, nb)
    ev.handle.set_profiling(True, classes=[0])  # class 0: FP64-class update (CRT-16 GEMM/SYRK)
    ev.eval(dx, dy, dz, cfg["theta"], u_req=1e-9, mode=mp.MP_MAP_ADAPTIVE)
    ev.handle.profile()  # flushes the timeline
    recs = [ln.split() for ln in open(tl) if ln.strip() and ln.strip() != "--"]
    fp64 = [r for r in recs if int(r[0]) == 0]
    rec = fp64[skip]
    flops = float(rec[4])
    f = ncu_fields(summ)
    rd, wr, ms = f["dram__bytes_read.sum"], f["dram__bytes_write.sum"], f["gpu__time_duration.sum"]
    res = {
        "kernel": "crt_gemm_kernel<16> (FP64 class as 16 INT8 tcgen05 GEMMs, CRT)",
        "dram_bytes_per_flop": (rd + wr) / flops,
        "capture": {"launch": f"launch {skip + 1} of the FP64 class in one cold {cfg_name} evaluation",
                    "duration_ms": ms, "dram_read_bytes": rd, "dram_write_bytes": wr,
                    "fp64_equivalent_flops": flops, "tile_gemms": flops / (2.0 * nb ** 3),
                    "tensor_pipe_active_pct": f.get(
                        "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed"),
                    "lts_throughput_pct": f.get("lts__throughput.avg.pct_of_peak_sustained_elapsed")},
        "algorithmic_bytes": "SURVEY 8(d) FP64 tile GEMM: (8 + 8 + 16) B x nb^2 per tile-GEMM; the engine's own: 16 int8 "
                             "residue planes of A and of B + FP64 C read and written = 48 B x nb^2",
        "source": f"tools/ncu_session.sh crt (ncu --set full --clock-control none -k regex:crt_gemm_kernel<\\(int\\)16 "
                  f"-s {skip} -c 1 python tools/one_eval.py {cfg_name} 0) + tools/crt_traffic.py (flops of that launch "
                  f"from MPGEO_TIMELINE)",
    }
    json.dump(res, open(out, "w"), indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
