#!/usr/bin/env python
"""bench.py — Tflop/s and joules per Matérn log-likelihood evaluation (BASELINE.json metric).

One "step" = one whole evaluation l(theta) of Eq. (1): Matérn tile generation with tile
norms, the precision maps (Alg. 2), the mixed-precision tile Cholesky
(Alg. 1) and the log-determinant + forward solve — every row of SURVEY.md §8(a) — through the
C ABI (mp_eval).  Tflop/s = (n^3/3) / T_eval.

Default (N=1): config 3 of BASELINE.json, n = 160,000 (400 x 400 jittered grid, Morton order),
nb = 2048, theta = (1, 0.03, 0.5), adaptive FP64/FP32/FP16 map at u_req = 1e-9 — the largest
configuration that fits one B200 (config 4, n = 360k, needs 320 GB).  The matrix (~68 GB) is far
larger than L2, so no explicit flush is needed between steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--map adaptive]
  python bench.py --impl reference ...   # the CPU oracle on a bounded sample (the reference arm)

N > 1 (torchrun, one process per GPU): ONE evaluation distributed over a P x Q process grid (as
square as possible, P <= Q; 2 -> 1x2, 4 -> 2x2, 8 -> 2x4), 2D block-cyclic tiles, panel
tiles exchanged through peer memory in their communication precision; same
workload as N = 1 (strong scaling); time is the max over ranks.  `--replicas` instead runs one
independent evaluation per rank (weak scaling, no data-path exchange).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    "c1": dict(n=1600, nb=400, theta=(1.0, 0.1, 0.5), map="fp64"),
    "c2": dict(n=40000, nb=2048, theta=(1.0, 0.03, 0.5), map="band"),
    "c3": dict(n=160000, nb=2048, theta=(1.0, 0.03, 0.5), map="adaptive"),
    "c4": dict(n=360000, nb=2048, theta=(1.0, 0.03, 0.5), map="adaptive"),  # 8 GPUs (2x4)
    "c5": dict(n=250000, nb=2048, theta=(1.0, 0.03, 0.5), map="adaptive"),
}
METRIC = "Tflop/s & joules per MLE log-likelihood eval (n=360k) at 1/2/4/8 B200"
FP64_NOMINAL, BF16_NOMINAL, INT8_NOMINAL = 40.0, 2250.0, 4500.0  # dense TFLOP/s (TOP/s), B200 nominal
OZ_PRODUCTS = 36  # int8 GEMMs per FP64 GEMM in the Ozaki split with S = 8 slices (S (S+1) / 2)
CRT_PRODUCTS = 16  # int8 GEMMs per FP64 GEMM in the CRT (Ozaki scheme II) engine: one per modulus
# FP64-class engines (mp_handle_config "ozaki" % 100): products per FP64 GEMM, kernel, int8 planes per operand
ENGINES = {16: (CRT_PRODUCTS, "crt_gemm_kernel (FP64-class update as 16 INT8 tcgen05 GEMMs, CRT / Ozaki scheme II)",
                "crt-int8 (16 moduli)", 16),
           8: (OZ_PRODUCTS, "ozaki_gemm_kernel<8> (FP64-class update as 36 INT8 tcgen05 GEMMs)", "ozaki-int8 (S=8)", 8)}


def ncu_traffic(engine):
    """dram bytes per FP64-equivalent flop of the dominant kernel, from one `ncu --set full` capture of a
    launch inside a bench run (profiles/r01/ncu_traffic*.json record the capture and its command)."""
    name = {16: "ncu_traffic_crt.json", 8: "ncu_traffic.json"}.get(engine)
    p = os.path.join(ROOT, "profiles", "r01", name) if name else None
    return json.load(open(p)) if p and os.path.exists(p) else None


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            threading.Thread(target=self._read, daemon=True).start()
        except (OSError, FileNotFoundError):
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 9:
                self.rows.append(parts)

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[5 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def nvml_energy_mj(device: int):
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(device)
        return float(pynvml.nvmlDeviceGetTotalEnergyConsumption(h))
    except Exception:
        return None


def cublas_dgemm_tflops(seconds=1.5):
    """Context only: cuBLAS DGEMM 8192^3 back to back (not the roofline denominator)."""
    import torch
    a = torch.randn(8192, 8192, dtype=torch.float64, device="cuda")
    b = torch.randn(8192, 8192, dtype=torch.float64, device="cuda")
    torch.matmul(a, b)
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    it = 0
    s.record()
    t0 = time.time()
    while time.time() - t0 < seconds:
        torch.matmul(a, b)
        it += 1
    e.record()
    torch.cuda.synchronize()
    return 2 * 8192**3 * it / (s.elapsed_time(e) / 1e3) / 1e12


# --------------------------------------------------------------------------- oracle (CPU) leg
def oracle_sample_eval(n=10000, nb=512, theta=(1.0, 0.03, 0.5), u_req=1e-9, map_mode="adaptive"):
    """One oracle evaluation as it stands (generation + norms + maps + tile Cholesky + Eq. (1))."""
    import synth
    from oracle.loglik import loglik as oracle_loglik
    from oracle.precision import precision_maps
    from oracle.tiles import gen_lower_tiles, num_tiles, tile_sqnorms

    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    t0 = time.perf_counter()
    if map_mode == "fp64":
        oracle_loglik(x, y, z, theta, nb)
    else:
        s = tile_sqnorms(gen_lower_tiles(x, y, theta, nb), num_tiles(n, nb))
        oracle_loglik(x, y, z, theta, nb, maps=precision_maps(s, u_req))
    return time.perf_counter() - t0


def cpu_cores():
    try:
        from threadpoolctl import threadpool_info
        th = [i.get("num_threads", 0) for i in threadpool_info() if i.get("user_api") == "blas"]
        return max(th) if th else os.cpu_count()
    except Exception:
        return os.cpu_count()


def cpu_baseline(map_mode):
    n_s, nb_s = 10000, 512
    t = oracle_sample_eval(n_s, nb_s, map_mode=map_mode)
    return {"value": (n_s**3 / 3) / t / 1e12, "unit": "Tflop/s", "cores": cpu_cores(), "kind": "oracle",
            "sample": f"1 oracle evaluation at n={n_s} (100x100 grid), nb={nb_s}, {map_mode} map, same theta/recipe "
                      f"as the workload: NumPy/SciPy FP64 generation+norms+maps+tile Cholesky+Eq.(1); {t:.1f} s",
            "seconds": t}


def run_reference(args, cfg, world, rank):
    if rank != 0:
        return
    steps, times = args.steps, []
    for i in range(args.warmup + args.steps):
        t = oracle_sample_eval(map_mode=cfg["map"])
        if i >= args.warmup:
            times.append(t)
    n_s = 10000
    T = sum(times)
    val = steps * (n_s**3 / 3) / T / 1e12
    cores = cpu_cores()
    out = {"impl": "reference", "metric": METRIC, "value": val, "unit": "Tflop/s", "n_gpus": world, "steps": steps,
           "warmup": args.warmup, "ms_per_step": 1e3 * T / steps, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": f"{args.config} sample: n=10000 nb=512 (bounded oracle sample)",
                      "map": cfg["map"], "theta": list(cfg["theta"])},
           "cpu_baseline": {"value": val, "unit": "Tflop/s", "cores": cores, "kind": "oracle",
                            "sample": "each step = 1 oracle evaluation at n=10000, nb=512 (CPU, NumPy/SciPy FP64)"},
           "e2e": {"value": val, "unit": "Tflop/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# --------------------------------------------------------------------------- GPU leg
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c3", choices=sorted(CONFIGS))
    ap.add_argument("--map", default=None, choices=["adaptive", "fp64", "band", "extreme"])
    ap.add_argument("--policy", default="auto", choices=["auto", "ttc"])
    ap.add_argument("--u-req", type=float, default=1e-9)
    ap.add_argument("--theta", default=None, help="sigma2,beta,nu override (e.g. 1,0.03,0.8 for the Bessel path)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--replicas", action="store_true", help="N>1: independent evaluations per rank")
    args = ap.parse_args()
    cfg = dict(CONFIGS[args.config])
    if args.map:
        cfg["map"] = args.map
    if args.theta:
        cfg["theta"] = tuple(float(v) for v in args.theta.split(","))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, cfg, world, rank)
    if args.warmup < 3:
        print("note: --warmup raised to 3 (timing rules)", file=sys.stderr)
        args.warmup = 3

    import numpy as np
    import torch

    import paper_conf_cluster_caoalgkb23_b200 as mp
    import synth

    # one process per GPU; on a box with fewer GPUs than ranks the ranks share devices (the peer-memory
    # exchange then runs over same-device IPC) — used to validate the N > 1 path on one GPU
    local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        # the process group only carries timings and the 64-byte IPC handles (the data path is the
        # library's own peer-memory exchange), so gloo is enough
        dist.init_process_group("gloo")
    n, nb, theta = cfg["n"], cfg["nb"], cfg["theta"]
    mode = {"adaptive": mp.MP_MAP_ADAPTIVE, "fp64": mp.MP_MAP_FP64, "band": mp.MP_MAP_BAND,
            "extreme": mp.MP_MAP_EXTREME}[cfg["map"]]
    policy = mp.MP_COMM_AUTO if args.policy == "auto" else mp.MP_COMM_TTC
    distributed = world > 1 and not args.replicas
    seed = 0 if distributed or world == 1 else rank
    x, y = synth.locations(n, seed=seed)
    z = synth.normal_vector(n, seed=1 + seed)
    dx, dy, dz = (torch.from_numpy(a).cuda() for a in (x, y, z))
    hx, hy, hz = (torch.from_numpy(a).pin_memory() for a in (x, y, z))
    if distributed:
        P = int(math.isqrt(world))
        while world % P:
            P -= 1
        Q = world // P
        handle = mp.Handle(local, rank, world, P, Q)
        ev = mp.Evaluator(n, nb, handle=handle)
    else:
        P = Q = 1
        ev = mp.Evaluator(n, nb, device=local)
    h = ev.handle
    stream = h.stream

    def step(on_host=False):
        if on_host:
            return ev.eval(hx.numpy(), hy.numpy(), hz.numpy(), theta, u_req=args.u_req, mode=mode, policy=policy)
        return ev.eval(dx, dy, dz, theta, u_req=args.u_req, mode=mode, policy=policy)

    for _ in range(args.warmup):
        rep = step()
    torch.cuda.synchronize()

    def barrier():
        torch.cuda.synchronize()
        if dist:
            dist.barrier()

    # ---- timed region: K evaluations, inputs resident in HBM
    clocks = ClockSampler(local)
    barrier()
    e0_mj = nvml_energy_mj(local)
    clocks.start()
    h.set_profiling(True)
    l0 = h.launches
    ev_s, ev_e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev_s.record(stream)
    reps = []
    for _ in range(args.steps):
        reps.append(step())
    ev_e.record(stream)
    barrier()
    e1_mj = nvml_energy_mj(local)
    ck = clocks.stop()
    launches = h.launches - l0
    prof = h.profile()
    h.set_profiling(False)
    t_ms = ev_s.elapsed_time(ev_e)
    if dist:
        t = torch.tensor([t_ms], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        t_ms = float(t.item())
    joules = None if e0_mj is None or e1_mj is None else (e1_mj - e0_mj) / 1e3
    if joules is not None and rank >= torch.cuda.device_count():
        joules = 0.0  # ranks sharing a device (single-GPU validation): count each GPU once
    if dist and joules is not None:
        t = torch.tensor([joules], dtype=torch.float64)
        dist.all_reduce(t)
        joules = float(t.item())
    flops_eval = n**3 / 3.0
    evals_per_step = 1 if distributed else world
    value = evals_per_step * args.steps * flops_eval / (t_ms / 1e3) / 1e12

    # ---- e2e: same metric through mp_eval with pinned HOST inputs (H2D inside the call) and the
    # results (norms, info, partial sums, scalars) read back to the host every step
    e2e = None
    if not args.no_e2e:
        barrier()
        es, ee = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        es.record(stream)
        for _ in range(args.steps):
            step(on_host=True)
        ee.record(stream)
        barrier()
        te = es.elapsed_time(ee)
        if dist:
            t = torch.tensor([te], dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            te = float(t.item())
        nt = ev.nt
        chunks = (n + 4095) // 4096
        d2h = (nt * (nt + 1) // 2) * 8 if mode in (mp.MP_MAP_ADAPTIVE, mp.MP_MAP_BAND) else 0
        d2h += 4 + (nt + chunks) * 8
        e2e = {"value": evals_per_step * args.steps * flops_eval / (te / 1e3) / 1e12, "unit": "Tflop/s",
               "h2d_bytes_per_step": 3 * n * 8, "d2h_bytes_per_step": d2h, "ms_per_step": te / args.steps}

    if rank != 0:
        if dist:
            dist.destroy_process_group()
        return
    peaks, peak_src = measured_peaks()
    p = prof.as_dict()
    dom = p["upd_fp64"]
    engine = h.config()
    fp64_peak = peaks["bf16_tflops_sustained"] * FP64_NOMINAL / BF16_NOMINAL
    int8_peak = peaks["bf16_tflops_sustained"] * INT8_NOMINAL / BF16_NOMINAL
    fp64_eq = dom["flops"] / (dom["ms"] / 1e3) / 1e12 if dom["ms"] > 0 else 0.0
    flops_per_launch = dom["flops"] / max(1, dom["launches"])
    eng = ENGINES.get(engine["ozaki"] % 100)
    tr = ncu_traffic(engine["ozaki"] % 100)
    traffic = (tr["dram_bytes_per_flop"] * flops_per_launch) if tr and eng else None
    # algorithmic bytes of an FP64-class tile-GEMM on the INT8 path: the int8 planes of A and B (8 or 16
    # B/entry each) + the FP64 C tile read and written (16 B/entry)
    planes = eng[3] if eng else 8
    alg_bytes_per_launch = flops_per_launch / (2.0 * nb**3) * (planes + planes + 16) * nb * nb
    try:
        cub = cublas_dgemm_tflops()
    except Exception:
        cub = None
    last = reps[-1]
    upd = list(last.flops_update)
    fp64_class_peak = (int8_peak / eng[0]) if eng else fp64_peak
    # FP32-class engine: CRT-8 (8 INT8 GEMMs, ozaki >= 200), 4-slice split (10 INT8 GEMMs, >= 100), 3xFP16 (tc 2), 3xTF32
    fp32_class_peak = ((int8_peak / 8) if engine["ozaki"] >= 200 else (int8_peak / 10) if engine["ozaki"] >= 100
                       else peaks["bf16_tflops_sustained"] / 3 if engine["tc"] == 2  # 3xFP16 at the f16 rate
                       else peaks["bf16_tflops_sustained"] * 0.5 / 3)
    roof_time_s = (upd[0] / (fp64_class_peak * 1e12)
                   + upd[1] / (fp32_class_peak * 1e12)
                   + upd[2] / (peaks["bf16_tflops_sustained"] * 1e12))
    t_upd_s = (p["upd_fp64"]["ms"] + p["upd_fp32"]["ms"] + p["upd_fp16"]["ms"]) / 1e3 / args.steps
    out = {
        "metric": METRIC, "value": value, "unit": "Tflop/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": t_ms / args.steps, "higher_is_better": True,
        "scaling": "strong" if distributed else "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: n={n} ({int(math.isqrt(n))}^2 jittered grid, Morton order), nb={nb}, "
                               f"theta={list(theta)}, {cfg['map']} map u_req={args.u_req}, comm={args.policy}",
                   "n": n, "nb": nb, "map": cfg["map"], "policy": args.policy,
                   "fp64_engine": eng[2] if eng else "dmma",
                   "fp32_engine": ("crt-int8 (8 moduli, FP32 C)" if engine["ozaki"] >= 200 else
                                   "ozaki-int8 (S=4)" if engine["ozaki"] >= 100 else
                                   ("tcgen05 3xFP16 (row-scaled)" if engine["tc"] == 2 else
                                    "tcgen05 3xTF32" if engine["tc"] else "dmma-rounded")),
                   "fp16_engine": "tcgen05 f16" if engine["tc"] else "dmma-rounded", "lookahead": engine["lookahead"],
                   "parallelism": (f"2D block-cyclic {P}x{Q}, peer-memory panel exchange" if distributed
                                   else ("replicas" if world > 1 else "1 GPU")),
                   "l2": "matrix (~%.0f GB) >> 126 MB L2; no flush needed" % (n * n / 2 * 5 / 1e9)},
        "joules_per_eval": None if joules is None else joules / args.steps,
        "loglik": last.loglik, "tiles_fp64_fp32_fp16": list(last.tiles), "stc_tiles": last.stc_tiles,
        "flops_update_per_class": upd,
        "phase_ms": {"gen+map": last.t_gen_ms, "potrf": last.t_potrf_ms, "solve": last.t_solve_ms},
        "profile": {k: {"ms_per_step": v["ms"] / args.steps, "launches_per_step": v["launches"] / args.steps,
                        "tflops": (v["flops"] / (v["ms"] / 1e3) / 1e12) if v["ms"] > 0 and v["flops"] else None}
                    for k, v in p.items()},
        "update_roofline_fraction": roof_time_s / t_upd_s if t_upd_s > 0 else None,
        "roofline": (
            {"bound": "tensor", "kernel": eng[1],
             "achieved": eng[0] * fp64_eq, "peak": int8_peak, "unit": "TFLOP/s",
             "frac": eng[0] * fp64_eq / int8_peak, "traffic": traffic,
             "algorithmic_bytes_per_launch": alg_bytes_per_launch,
             "traffic_source": tr.get("source") if tr else None,
             "peak_source": f"{peak_src} bf16_tflops_sustained x {INT8_NOMINAL}/{BF16_NOMINAL} (INT8 nominal / bf16 nominal); "
                            "achieved = executed int8 multiply-add ops x 2 per second",
             "fp64_equivalent_tflops": fp64_eq, "cublas_dgemm_tflops_live": cub,
             "fp64_equivalent_vs_cublas_dgemm": (fp64_eq / cub) if cub else None}
            if eng else
            {"bound": "tensor", "kernel": "dgemm_nt_kernel (FP64 DMMA trailing update)",
             "achieved": fp64_eq, "peak": fp64_peak, "unit": "TFLOP/s",
             "frac": fp64_eq / fp64_peak if fp64_peak else None, "traffic": None,
             "peak_source": f"{peak_src} bf16_tflops_sustained x {FP64_NOMINAL}/{BF16_NOMINAL} (FP64 DMMA nominal / bf16 nominal)",
             "cublas_dgemm_tflops_live": cub, "frac_vs_cublas_dgemm": (fp64_eq / cub) if cub else None}),
        "gpu_launches": launches,
        "clocks": ck,
        "e2e": e2e,
    }
    if world == 1 and not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_baseline(cfg["map"])
    print(json.dumps(out), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
