#!/usr/bin/env python
#!/usr/bin/env python
"""bench.py — Tflop/s and joules per Matérn log-likelihood evaluation (BASELINE.json metric).

One "step" = one whole evaluation l(theta) of Eq. (1): Matérn tile generation with tile
norms, the precision maps (Alg. 2), the mixed-precision tile Cholesky
(Alg. 1) and the log-determinant + forward solve — every row of SURVEY.md §8(a) — through the
C ABI (mp_eval).  Tflop/s = (n^3/3) / T_eval.

Default (N=1): config 5 of BASELINE.json, n = 250,000 (500 x 500 jittered grid, Morton order),
nb = 2048, theta = (1, 0.03, 0.5), adaptive FP64/FP32/FP16 map at u_req = 1e-9 — the largest
configuration that fits one B200 (C5's first strong-scaling point; config 4, n = 360k, needs
320 GB of tiles).  The workspace is sized by the evaluation's storage map (~160 GB of tiles plus
one panel's operand caches).  The matrix is far larger than L2, so no flush is needed between steps.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c5] [--map adaptive]
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
    "c2a": dict(n=40000, nb=2048, theta=(1.0, 0.03, 0.5), map="adaptive"),  # C2 size, adaptive map (tools)
    "c0": dict(n=4096, nb=512, theta=(1.0, 0.03, 0.5), map="adaptive"),      # small case (sanitizers, tools)
    "c0q": dict(n=4096, nb=512, theta=(1.0, 0.03, 0.5), map="adaptive4"),    # the same, four-level map (tools)
}
METRIC = "Tflop/s & joules per MLE log-likelihood eval (n=360k) at 1/2/4/8 B200"
FP64_NOMINAL, BF16_NOMINAL, INT8_NOMINAL = 40.0, 2250.0, 4500.0  # dense TFLOP/s (TOP/s), B200 nominal
TF32_NOMINAL = 1100.0  # dense TF32 TFLOP/s, B200 nominal
CRT_PRODUCTS = 16  # int8 GEMMs per FP64 GEMM in the CRT (Ozaki scheme II) engine: one per modulus
FP64_ENGINES = {0: "crt-int8 (16 moduli, Ozaki scheme II; per-row normwise bound K 2^-57 max|a_i.| max|b_j.|)",
                1: "dmma-fp64 (native)"}
FP32_ENGINES = {0: "tcgen05 3xFP16 (row-scaled 11+11-bit split; per-row normwise bound)",
                1: "tcgen05 3xTF32", 2: "dmma (FP32-rounded operands, FP32 C)"}
DTYPE = {(0, 0, 1): "mixed f64(crt16-int8)/f32(3xf16)/f16(row-scaled)"}  # + "/fp16-storage" with fp16_storage


def ncu_traffic():
    """DRAM bytes per FP64-equivalent flop of the CRT-16 kernel from one `ncu --set full` capture of a
    launch inside an evaluation (the newest profiles/r0*/ncu_traffic_crt.json records the capture and
    its command)."""
    for rnd in ("r02", "r01"):
        p = os.path.join(ROOT, "profiles", rnd, "ncu_traffic_crt.json")
        if os.path.exists(p):
            return json.load(open(p))
    return None


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
ORACLE_SAMPLE = dict(n=10000, nb=512)  # 100 x 100 grid: ~15 s of oracle time on 16 cores


def oracle_sample_eval(n, nb, theta):
    """One oracle evaluation as it stands, the FP64 definition (generation + tile Cholesky, Alg. 1 +
    Eq. (1)); the maps are computed too (tile norms + Alg. 2), as the GPU path does."""
    import synth
    from oracle.loglik import loglik as oracle_loglik
    from oracle.precision import precision_maps
    from oracle.tiles import gen_lower_tiles, num_tiles, tile_sqnorms

    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    t0 = time.perf_counter()
    precision_maps(tile_sqnorms(gen_lower_tiles(x, y, theta, nb), num_tiles(n, nb)), 1e-9)
    oracle_loglik(x, y, z, theta, nb)
    return time.perf_counter() - t0


def cpu_cores():
    try:
        from threadpoolctl import threadpool_info
        th = [i.get("num_threads", 0) for i in threadpool_info() if i.get("user_api") == "blas"]
        return max(th) if th else os.cpu_count()
    except Exception:
        return os.cpu_count()


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_baseline(theta):
    n_s, nb_s = ORACLE_SAMPLE["n"], ORACLE_SAMPLE["nb"]
    t = oracle_sample_eval(n_s, nb_s, theta)
    return {"value": (n_s**3 / 3) / t / 1e12, "unit": "Tflop/s", "cores": cpu_cores(), "cpu": cpu_model(),
            "kind": "oracle",
            "sample": f"1 oracle evaluation at n={n_s} (100x100 grid, same recipe and theta as the workload), "
                      f"nb={nb_s}: NumPy/SciPy FP64 definition (generation, tile norms + maps, tile Cholesky, "
                      f"Eq. (1)); {t:.1f} s; rate = (n^3/3)/T at the sample size",
            "seconds": t}


def run_reference(args, cfg, world, rank):
    if rank != 0:
        return
    n_s, nb_s = ORACLE_SAMPLE["n"], ORACLE_SAMPLE["nb"]
    steps, times = args.steps, []
    for i in range(args.warmup + args.steps):
        t = oracle_sample_eval(n_s, nb_s, cfg["theta"])
        if i >= args.warmup:
            times.append(t)
    T = sum(times)
    val = steps * (n_s**3 / 3) / T / 1e12
    cores = cpu_cores()
    out = {"impl": "reference", "metric": METRIC, "value": val, "unit": "Tflop/s", "n_gpus": world, "steps": steps,
           "warmup": args.warmup, "ms_per_step": 1e3 * T / steps, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": f"{args.config} sample: n={n_s} nb={nb_s} (bounded oracle sample)",
                      "map": "fp64 definition (+ adaptive maps computed)", "theta": list(cfg["theta"])},
           "cpu_baseline": {"value": val, "unit": "Tflop/s", "cores": cores, "cpu": cpu_model(), "kind": "oracle",
                            "sample": f"each step = 1 oracle evaluation at n={n_s}, nb={nb_s} (CPU, NumPy/SciPy "
                                      "FP64 definition)"},
           "e2e": {"value": val, "unit": "Tflop/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


# --------------------------------------------------------------------------- GPU leg
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="c5", choices=sorted(CONFIGS))
    ap.add_argument("--map", default=None, choices=["adaptive", "adaptive4", "fp64", "band", "extreme"])
    ap.add_argument("--policy", default="auto", choices=["auto", "ttc"])
    ap.add_argument("--u-req", type=float, default=1e-9)
    ap.add_argument("--theta", default=None, help="sigma2,beta,nu override (e.g. 1,0.03,0.8 for the Bessel path)")
    ap.add_argument("--engine", default=None, help="mp_config overrides, e.g. fp64_engine=1,lookahead=0")
    ap.add_argument("--e2e-steps", type=int, default=3, help="evaluations in the end-to-end pass (<= steps)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-profile", action="store_true", help="skip the per-class breakdown evaluation")
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
    engine_cfg = {}
    if args.engine:
        for kv in args.engine.split(","):
            k, v = kv.split("=")
            engine_cfg[k.strip()] = int(v)

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
        # the process group carries timings, the communicator id and the 64-byte IPC handles (the data
        # path is the library's own peer-memory exchange), so gloo is enough
        dist.init_process_group("gloo")
    n, nb, theta = cfg["n"], cfg["nb"], cfg["theta"]
    mode = {"adaptive": mp.MP_MAP_ADAPTIVE, "adaptive4": mp.MP_MAP_ADAPTIVE4, "fp64": mp.MP_MAP_FP64,
            "band": mp.MP_MAP_BAND, "extreme": mp.MP_MAP_EXTREME}[cfg["map"]]
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
        handle = mp.Handle(local, rank, world, P, Q, uid=mp.shared_unique_id(), config=engine_cfg)
        ev = mp.Evaluator(n, nb, handle=handle)
    else:
        P = Q = 1
        ev = mp.Evaluator(n, nb, device=local, config=engine_cfg)
    h = ev.handle
    stream = h.stream
    eng = ev.M.engines()

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

    def max_over_ranks(v):
        if not dist:
            return v
        t = torch.tensor([v], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # ---- timed region: K evaluations, inputs resident in HBM.  Only the dominant class (the FP64-class
    # update) carries per-launch CUDA events (on the stream it is launched on), for the roofline line.
    dom_cls = "upd_fp64"
    clocks = ClockSampler(local)
    barrier()
    e0_mj = nvml_energy_mj(local)
    clocks.start()
    h.set_profiling(True, classes=[dom_cls])
    l0 = h.launches
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps + 1)]
    evs[0].record(stream)
    reps = []
    for i in range(args.steps):
        reps.append(step())
        evs[i + 1].record(stream)
    barrier()
    e1_mj = nvml_energy_mj(local)
    ck = clocks.stop()
    launches = h.launches - l0
    dom = h.profile().as_dict()[dom_cls]
    h.set_profiling(False)
    step_ms = [evs[i].elapsed_time(evs[i + 1]) for i in range(args.steps)]
    t_ms = max_over_ranks(evs[0].elapsed_time(evs[-1]))
    step_ms = [max_over_ranks(v) for v in step_ms]
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
    potrf_ms = statistics.median([r.t_potrf_ms for r in reps])

    # ---- e2e: the same metric through mp_eval with pinned HOST inputs (H2D inside the call) and the
    # results (norms, info, partial sums, scalars) read back to the host every step
    e2e = None
    if not args.no_e2e:
        ke = max(1, min(args.e2e_steps, args.steps))
        barrier()
        es, ee = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        es.record(stream)
        for _ in range(ke):
            step(on_host=True)
        ee.record(stream)
        barrier()
        te = max_over_ranks(es.elapsed_time(ee))
        nt = ev.nt
        chunks = (n + 4095) // 4096
        d2h = (nt * (nt + 1) // 2) * 8 if mode in (mp.MP_MAP_ADAPTIVE, mp.MP_MAP_ADAPTIVE4, mp.MP_MAP_BAND) else 0
        d2h += 4 + (nt + chunks) * 8
        e2e = {"value": evals_per_step * ke * flops_eval / (te / 1e3) / 1e12, "unit": "Tflop/s",
               "h2d_bytes_per_step": 3 * n * 8, "d2h_bytes_per_step": d2h, "ms_per_step": te / ke, "steps": ke}

    # ---- per-class breakdown: one more evaluation with events around every launch (outside the
    # timed region; its events would otherwise perturb the timing)
    prof = None
    if not args.no_profile:
        h.set_profiling(True)
        step()
        prof = h.profile().as_dict()
        h.set_profiling(False)

    # per-rank view (N > 1): own wall time of the timed steps and device-busy time per update class of the
    # profiled evaluation, gathered on rank 0 (the driver's max-over-ranks value stays the headline)
    mine = {"rank": rank, "device": local, "ms_per_step": evs[0].elapsed_time(evs[-1]) / args.steps,
            "busy_ms": None if prof is None else {k: round(v["ms"], 1) for k, v in prof.items()}}
    per_rank = [mine]
    if dist:
        per_rank = [None] * world
        dist.all_gather_object(per_rank, mine)
    if rank != 0:
        if dist:
            dist.destroy_process_group()
        return
    peaks, peak_src = measured_peaks()
    bf16_s = peaks["bf16_tflops_sustained"]
    fp64_peak = bf16_s * FP64_NOMINAL / BF16_NOMINAL      # DMMA FP64, derived from the measured bf16 rate
    int8_peak = bf16_s * INT8_NOMINAL / BF16_NOMINAL      # INT8 dense
    tf32_peak = bf16_s * TF32_NOMINAL / BF16_NOMINAL
    crt = eng["fp64"] == mp.MP_F64_CRT16
    try:
        cub = cublas_dgemm_tflops()
    except Exception:
        cub = None
    fp64_eq = dom["flops"] / (dom["ms"] / 1e3) / 1e12 if dom["ms"] > 0 else 0.0
    flops_per_launch = dom["flops"] / max(1, dom["launches"])
    alg_bytes_per_launch = flops_per_launch / (2.0 * nb**3) * (8 + 8 + 16) * nb * nb  # 8+8+16 B/entry
    engine_bytes_per_launch = flops_per_launch / (2.0 * nb**3) * (16 + 16 + 16) * nb * nb  # int8 planes + FP64 C
    tr = ncu_traffic() if crt else None
    traffic = (tr["dram_bytes_per_flop"] * flops_per_launch) if tr else None
    last = reps[-1]
    upd = list(last.flops_update)
    upd[2] += last.flops_update_fp16h  # four-level maps: the pure-FP16 class runs at the f16 rate too (class upd_fp16)
    # update time at the engines' peaks (FP64 class at INT8 peak / 16 with CRT, FP32 class at the f16 rate / 3
    # (3xFP16) or TF32 / 3, FP16 class at the f16 rate) and at the NATIVE peaks of the classes (FP64 DMMA, TF32
    # for the FP32 class as the survey's 3xTF32 plan counts it — 1 product —, FP16)
    fp64_class_peak = int8_peak / CRT_PRODUCTS if crt else fp64_peak
    fp32_class_peak = (bf16_s / 3 if eng["fp32"] == mp.MP_F32_3XFP16 else tf32_peak / 3 if eng["fp32"] == mp.MP_F32_3XTF32
                       else fp64_peak)
    roof_engine_s = upd[0] / (fp64_class_peak * 1e12) + upd[1] / (fp32_class_peak * 1e12) + upd[2] / (bf16_s * 1e12)
    # native FP64: the DMMA pipe demonstrably exceeds the bf16-derived figure, so the larger of it and the
    # live cuBLAS DGEMM rate (measured in this run) is the FP64 denominator of the native fraction
    fp64_native = max(fp64_peak, cub or 0.0)
    roof_native_s = upd[0] / (fp64_native * 1e12) + upd[1] / (tf32_peak * 1e12) + upd[2] / (bf16_s * 1e12)
    t_upd_s = None
    if prof:
        t_upd_s = (prof["upd_fp64"]["ms"] + prof["upd_fp32"]["ms"] + prof["upd_fp16"]["ms"]) / 1e3
    dt = DTYPE.get((eng["fp64"], eng["fp32"], eng["fp16_tensor"]),
                   f"mixed f64({'crt16-int8' if crt else 'dmma'})/f32({['3xf16', '3xtf32', 'dmma'][eng['fp32']]})/"
                   f"f16({'row-scaled' if eng['fp16_tensor'] else 'dmma'})")
    if h.config().get("fp16_storage"):
        dt += " fp16-storage"
    if cfg["map"] == "fp64":
        dt = "f64 (" + ("crt16-int8 emulation" if crt else "dmma") + ")"
    out = {
        "metric": METRIC, "value": value, "unit": "Tflop/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": t_ms / args.steps, "higher_is_better": True,
        "scaling": "strong" if distributed else "weak",
        "vs_baseline": None, "dtype": dt,
        "dtype_detail": {"fp64_class": FP64_ENGINES[eng["fp64"]], "fp32_class": FP32_ENGINES[eng["fp32"]],
                         "fp16_class": "tcgen05 f16 on row-scaled FP16 operands, FP32 accumulation" if eng["fp16_tensor"]
                         else "dmma on FP16-rounded operands",
                         "potrf_trsm_solve": "FP64 (DMMA); FP32/FP16-class TRSM as the CRT-8 product with L_kk^-1"
                         if eng["lowp_trsm_product"] else "FP64 (DMMA)"},
        "data": "synthetic",
        "config": {"workload": f"{args.config}: n={n} ({int(math.isqrt(n))}^2 jittered grid, Morton order), nb={nb}, "
                               f"theta={list(theta)}, {cfg['map']} map u_req={args.u_req}, comm={args.policy}",
                   "n": n, "nb": nb, "map": cfg["map"], "policy": args.policy, "engine_overrides": engine_cfg,
                   "parallelism": (f"2D block-cyclic {P}x{Q}, peer-memory panel exchange" if distributed
                                   else ("replicas" if world > 1 else "1 GPU")),
                   "workspace_gb": ev.M.nbytes / 1e9,
                   "l2": "matrix (~%.0f GB) >> 126 MB L2; no flush needed" % (ev.M.nbytes / 1e9)},
        "ms_per_step_median": statistics.median(step_ms), "ms_per_step_max": max(step_ms),
        "ms_per_step_all": step_ms,
        "factorization_tflops": flops_eval / (potrf_ms / 1e3) / 1e12 if potrf_ms > 0 else None,
        "joules_per_eval": None if joules is None else joules / args.steps,
        "loglik": last.loglik, "tiles_fp64_fp32_fp16": list(last.tiles), "stc_tiles": last.stc_tiles,
        **({"tiles_pure_fp16": last.tiles_fp16h, "flops_update_pure_fp16": last.flops_update_fp16h}
           if cfg["map"] == "adaptive4" else {}),
        "flops_update_per_class": upd,
        "phase_ms": {"gen+map": last.t_gen_ms, "potrf": last.t_potrf_ms, "solve": last.t_solve_ms},
        "profile": None if prof is None else {
            "note": "one extra evaluation after the timed region with CUDA events around every launch",
            **{k: {"ms": v["ms"], "launches": v["launches"],
                   "tflops": (v["flops"] / (v["ms"] / 1e3) / 1e12) if v["ms"] > 0 and v["flops"] else None}
               for k, v in prof.items()}},
        "update_roofline_fraction": roof_engine_s / t_upd_s if t_upd_s else None,
        "update_roofline_fraction_native": roof_native_s / t_upd_s if t_upd_s else None,
        "roofline_definitions": "update_roofline_fraction = update time at the ENGINES' peaks (FP64 class: INT8 peak/16 "
                                "with CRT; FP32 class: f16 peak/3 for 3xFP16; FP16: f16 peak) / measured update time; "
                                "..._native = the same at the classes' NATIVE peaks (FP64: max(bf16-derived, live cuBLAS "
                                "DGEMM), TF32, FP16) — above 1 because the FP64 class is emulated on INT8 faster than "
                                "native FP64",
        "roofline": (
            {"bound": "tensor", "kernel": "crt_gemm_kernel<16> (FP64-class GEMM/SYRK as 16 INT8 tcgen05 GEMMs, CRT)",
             "achieved": CRT_PRODUCTS * fp64_eq, "peak": int8_peak, "unit": "TFLOP/s",
             "frac": CRT_PRODUCTS * fp64_eq / int8_peak, "traffic": traffic,
             "algorithmic_bytes_per_launch": alg_bytes_per_launch,
             "engine_bytes_per_launch": engine_bytes_per_launch,
             "launches_timed": dom["launches"], "ms_timed": dom["ms"],
             "traffic_source": tr.get("source") if tr else None,
             "peak_source": f"{peak_src} bf16_tflops_sustained x {INT8_NOMINAL}/{BF16_NOMINAL} (INT8 nominal / bf16 "
                            "nominal); achieved = executed int8 multiply-add ops x 2 per second over the timed region",
             "fp64_equivalent_tflops": fp64_eq, "fp64_equivalent_vs_dmma_peak": fp64_eq / fp64_peak,
             "cublas_dgemm_tflops_live": cub, "fp64_equivalent_vs_cublas_dgemm": (fp64_eq / cub) if cub else None}
            if crt else
            {"bound": "tensor", "kernel": "dgemm_nt_kernel (FP64 DMMA trailing update)",
             "achieved": fp64_eq, "peak": fp64_peak, "unit": "TFLOP/s",
             "frac": fp64_eq / fp64_peak if fp64_peak else None, "traffic": None,
             "algorithmic_bytes_per_launch": alg_bytes_per_launch,
             "peak_source": f"{peak_src} bf16_tflops_sustained x {FP64_NOMINAL}/{BF16_NOMINAL} (FP64 DMMA nominal / bf16 nominal)",
             "cublas_dgemm_tflops_live": cub, "frac_vs_cublas_dgemm": (fp64_eq / cub) if cub else None}),
        "gpu_launches": launches,
        "clocks": ck,
        **({"grid": f"{P}x{Q}", "per_rank": per_rank} if world > 1 else {}),
        "e2e": e2e,
    }
    if world == 1 and not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_baseline(theta)
    print(json.dumps(out), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
