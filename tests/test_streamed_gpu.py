"""blas3_sgemm_streamed (row F1: device-side consumption of a panel-pipelined
broadcast) on one GPU.  A "comm" stream stands in for the NCCL broadcast: it
writes A's column panels into the operand buffer (after a delay, so the GEMM
really starts before its data) and releases each panel's flag with
blas3_signal; the GEMM is launched at once on the compute stream.  The result
must equal a plain SGEMM bit for bit (same kernel, same k order), whatever
order the panels arrive in (at the same SM count: the split-tail plan depends
on it).  Runs in a subprocess: a broken flag protocol
traps the kernel (4 s) and would poison the CUDA context of the test run."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r'''
import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
from paper_conf_ipps_cuiwxyf11_b200 import dist as d3
import blas3_inputs as gen
torch.cuda.set_device(0)
def dev(x): return b3.from_fortran(x)
def bits(t): return np.ascontiguousarray(t.cpu().numpy()).view(np.uint32)
ok = True
for (m, n, k, panels, tb, order) in [(1000, 1200, 2048, 8, "N", "fwd"), (512, 768, 1000, 4, "T", "rev"),
                                    (2304, 2048, 4096, 8, "N", "rev"), (300, 260, 96, 3, "N", "fwd")]:
    A = gen.uniform(m, k, "st-a"); B = gen.uniform(*((k, n) if tb == "N" else (n, k)), "st-b")
    C = gen.uniform(m, n, "st-c")
    dA_src, dB = dev(A), dev(B)
    want = dev(C)
    with b3.options(max_sms=132):                         # the same launch shape (split tail) as below
        b3.sgemm("N", tb, 1.5, dA_src, dB, 0.5, want)
    pan = d3.uniform_panels(k, panels)
    flags = torch.zeros(len(pan), dtype=torch.int32, device="cuda")
    for value in (1, 2):                                  # two calls on the same flags
        dA = torch.full_like(dA_src, float("nan"))        # nothing of A is there yet
        got = dev(C)
        compute = torch.cuda.current_stream()
        comm = torch.cuda.Stream()
        comm.wait_stream(compute)
        with torch.cuda.stream(comm):
            torch.cuda._sleep(2_000_000)                  # the GEMM is running before any panel lands
            for i in (range(len(pan)) if order == "fwd" else reversed(range(len(pan)))):
                c0, c1 = pan[i]
                dA[:, c0:c1].copy_(dA_src[:, c0:c1])
                b3.signal(flags, i, value)
        with b3.options(max_sms=132):                     # leave SMs to the comm stream's kernels
            b3.sgemm_streamed("N", tb, 1.5, dA, dB, 0.5, got, flags, pan[0][1] - pan[0][0], value)
        compute.wait_stream(comm)
        torch.cuda.synchronize()
        same = np.array_equal(bits(got), bits(want))
        print(m, n, k, panels, tb, order, value, "bit-identical" if same else "DIFFERENT", flush=True)
        ok &= same
# the dist executor's device-side path at world size 1 (flags only, no broadcast)
A = gen.uniform(1024, 2048, "sd-a"); B = gen.uniform(2048, 512, "sd-b"); C = gen.uniform(1024, 512, "sd-c")
want = dev(C)
with b3.options(max_sms=torch.cuda.get_device_properties(0).multi_processor_count - 16):
    b3.sgemm("N", "N", 1.5, dev(A), dev(B), 0.5, want)
got = dev(C); d3.sgemm("N", "N", 1.5, dev(A), dev(B), 0.5, got, panels=8, pipeline=True, device_side=True)
torch.cuda.synchronize()
same = np.array_equal(bits(got), bits(want))
print("dist device_side", "bit-identical" if same else "DIFFERENT")
ok &= same
print("ALL_OK" if ok else "FAILED")
'''


def test_streamed_gemm_matches_sgemm_bitwise():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import __graft_entry__
    __graft_entry__.build()
    r = subprocess.run([sys.executable, "-c", CHILD], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "ALL_OK" in r.stdout, r.stdout[-3000:] + r.stderr[-3000:]
