"""Tall-skinny SSYRK / SSYR2K (configs[3] shape: N = 16384, K = 512), for ncu captures:
python tools/ts_call.py ssyrk|ssyr2k [reps]"""
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402

r = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
n, k = 16384, 512
A = b3.colmajor(n, k); B = b3.colmajor(n, k); C = b3.colmajor(n, n)
for t in (A, B, C):
    t.uniform_(-1, 1)
for _ in range(reps):
    if r == "ssyrk":
        b3.ssyrk("L", "N", 1.5, A, 0.5, C)
    else:
        b3.ssyr2k("L", "N", 1.5, A, B, 0.5, C)
torch.cuda.synchronize()
print("done", r)
