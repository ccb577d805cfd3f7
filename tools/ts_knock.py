"""Where tall-skinny SSYRK (N = 16384, K = 512) spends its time: the same call
with beta = 0 (no C loads) and under the BLAS3_DEBUG_TC knock-outs given in
argv (run once per setting as separate processes; results are wrong by design).
python tools/ts_knock.py"""
import os
import subprocess
import sys

code = r'''
import sys, torch, numpy as np
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
n, k = 16384, 512
A = b3.colmajor(n, k); A.uniform_(-1, 1); C = b3.colmajor(n, n); C.uniform_(-1, 1)
G = b3.colmajor(8192, 8192); G.uniform_(-1, 1); H = b3.colmajor(8192, 8192); H.uniform_(-1, 1)
def t(fn, reps=10):
    fn(); torch.cuda.synchronize()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    ts = []
    for _ in range(5):
        e0.record()
        for _ in range(reps): fn()
        e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1) / reps)
    return float(np.median(ts))
f = 1.0 * k * n * (n + 1)
b1 = t(lambda: b3.ssyrk("L", "N", 1.5, A, 0.5, C))
b0 = t(lambda: b3.ssyrk("L", "N", 1.5, A, 0.0, C))
sg = t(lambda: b3.sgemm("N", "N", 1.5, G, H, 0.5, G), 3)
print(f"{sys.argv[1]:>8s}: beta=0.5 {b1*1e3:7.1f} us {f/b1/1e9:6.1f} TF/s | beta=0 {b0*1e3:7.1f} us {f/b0/1e9:6.1f} TF/s | sgemm8192 {2*8192**3/sg/1e9:6.1f} TF/s", flush=True)
'''
for dbg in ["0"] + sys.argv[1:]:
    env = dict(os.environ, BLAS3_DEBUG_TC=dbg)
    subprocess.run([sys.executable, "-c", code, dbg], env=env)
