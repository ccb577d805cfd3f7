"""Box facts probe: device props, torch TF32 and FP32 (cuBLAS) matmul rates.
Context numbers only (cuBLAS is the comparator, not the product)."""
import json, time, torch
p = torch.cuda.get_device_properties(0)
out = {"name": p.name, "sms": p.multi_processor_count, "cc": f"{p.major}.{p.minor}",
       "mem_gb": p.total_memory / 2**30, "l2_mb": getattr(p, "L2_cache_size", 0) / 2**20}
def rate(n, tf32, reps=10):
    torch.backends.cuda.matmul.allow_tf32 = tf32
    a = torch.randn(n, n, device="cuda"); b = torch.randn(n, n, device="cuda")
    for _ in range(3): c = a @ b
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    best = 1e9
    for _ in range(reps):
        e0.record(); c = a @ b; e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return 2 * n**3 / (best * 1e-3) / 1e12
out["cublas_tf32_tflops_8192"] = rate(8192, True)
out["cublas_fp32_tflops_8192"] = rate(8192, False)
print(json.dumps(out))
json.dump(out, open("gpurun_out/box_facts.json", "w"))
