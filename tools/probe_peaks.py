"""Hardware probe (context only, not product code): cuBLAS DGEMM/SGEMM/TF32/FP16 rates and host info."""
import json, os, time, subprocess
import torch
def rate(dtype, n, iters=10, tf32=False):
    torch.backends.cuda.matmul.allow_tf32 = tf32
    a = torch.randn(n, n, device="cuda", dtype=dtype); b = torch.randn(n, n, device="cuda", dtype=dtype)
    for _ in range(3): torch.matmul(a, b)
    torch.cuda.synchronize()
    s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    best = 1e9
    for _ in range(iters):
        s.record(); torch.matmul(a, b); e.record(); torch.cuda.synchronize()
        best = min(best, s.elapsed_time(e) / 1e3)
    return 2 * n**3 / best / 1e12
out = {"gpu": torch.cuda.get_device_name(0), "sms": torch.cuda.get_device_properties(0).multi_processor_count}
out["dgemm_8192_tflops"] = rate(torch.float64, 8192)
out["dgemm_2048_tflops"] = rate(torch.float64, 2048, 50)
out["sgemm_8192_tflops"] = rate(torch.float32, 8192)
out["tf32_8192_tflops"] = rate(torch.float32, 8192, tf32=True)
out["hgemm_8192_tflops"] = rate(torch.float16, 8192)
out["cpu_count"] = os.cpu_count()
out["cpu_model"] = subprocess.run("grep -m1 'model name' /proc/cpuinfo", shell=True, capture_output=True, text=True).stdout.strip()
out["mem"] = subprocess.run("free -g | head -2", shell=True, capture_output=True, text=True).stdout
print(json.dumps(out, indent=1))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/probe_peaks.json", "w"), indent=1)
