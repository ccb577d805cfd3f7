"""Timeline of blas3_sgemm_streamed consuming A while it arrives (one GPU):
a comm stream writes A's 8 column panels (after a 0.5 ms delay, then one
panel at a time) and releases each panel's flag; the GEMM is launched at once
and its producer waits per k-block.  Prints the kernel/copy timeline and the
GEMM's duration against a plain SGEMM of the same shape.
python tools/streamed_demo.py [n]"""
import json
import os
import sys
import tempfile

import torch
from torch.profiler import ProfilerActivity, profile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402
from paper_conf_ipps_cuiwxyf11_b200 import dist as d3  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
src = b3.colmajor(n, n); src.uniform_(-1, 1)
A = b3.colmajor(n, n); B = b3.colmajor(n, n); B.uniform_(-1, 1); C = b3.colmajor(n, n); C.uniform_(-1, 1)
pan = d3.uniform_panels(n, 8)
flags = torch.zeros(len(pan), dtype=torch.int32, device="cuda")
nsm = torch.cuda.get_device_properties(0).multi_processor_count


def streamed(value):
    compute = torch.cuda.current_stream()
    comm = torch.cuda.Stream()
    comm.wait_stream(compute)
    with torch.cuda.stream(comm):
        torch.cuda._sleep(1_000_000)
        for i, (c0, c1) in enumerate(pan):
            A[:, c0:c1].copy_(src[:, c0:c1])
            b3.signal(flags, i, value)
    with b3.options(max_sms=nsm - 16):
        b3.sgemm_streamed("N", "N", 1.0, A, B, 0.0, C, flags, pan[0][1] - pan[0][0], value)
    compute.wait_stream(comm)


streamed(1); torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    streamed(2)
    torch.cuda.synchronize()
    with b3.options(max_sms=nsm - 16):
        b3.sgemm("N", "N", 1.0, A, B, 0.0, C)
    torch.cuda.synchronize()
tmp = os.path.join(tempfile.mkdtemp(), "t.json")
prof.export_chrome_trace(tmp)
evs = sorted((float(e["ts"]), float(e["dur"]), e["name"][:60], e.get("args", {}).get("stream", e.get("tid")))
             for e in json.load(open(tmp))["traceEvents"]
             if e.get("cat") in ("kernel", "gpu_memcpy", "gpu_memset"))
t0 = evs[0][0]
for ts, du, nm, st in evs:
    print(f"{ts - t0:9.1f} {ts - t0 + du:9.1f} {du:8.1f}  s{st}  {nm}")
