"""Size-stability sweep (the paper's Fig. 13 range): every routine family at
N = 512..8192.  Each measurement is `reps` calls back to back between two CUDA
events (the GPU never waits for the host, as in any stream of calls), rounds
interleaved, medians; % of this library's SGEMM NN at the same N.
python tools/size_sweep.py [sizes] [rounds]"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3  # noqa: E402

sizes = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "512,1024,1536,2048,3072,4096,8192").split(",")]
rounds = int(sys.argv[2]) if len(sys.argv) > 2 else 5


def mk(m, n):
    t = b3.colmajor(m, n)
    t.uniform_(-1, 1)
    return t


print("| N | routine | variant | us | TF/s | % SGEMM |\n|---|---|---|---|---|---|")
for n in sizes:
    A, B, C, X = mk(n, n), mk(n, n), mk(n, n), mk(n, n)
    T = mk(n, n); T.mul_(1.0 / n); T.diagonal().fill_(1.0)
    cases = [("sgemm", "NN", 2.0 * n ** 3, lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C), None),
             ("ssymm", "LL", 2.0 * n ** 3, lambda: b3.ssymm("L", "L", 1.5, A, B, 0.5, C), None),
             ("ssymm", "RL", 2.0 * n ** 3, lambda: b3.ssymm("R", "L", 1.5, A, B, 0.5, C), None),
             ("ssyrk", "LN", 1.0 * n * n * (n + 1), lambda: b3.ssyrk("L", "N", 1.5, A, 0.5, C), None),
             ("ssyr2k", "LN", 2.0 * n ** 3 + n, lambda: b3.ssyr2k("L", "N", 1.5, A, B, 0.5, C), None),
             ("strmm", "LLNN", 1.0 * n ** 3, lambda: b3.strmm("L", "L", "N", "N", 1.0, T, X), lambda: X.copy_(B)),
             ("strsm", "LLNN", 1.0 * n ** 3, lambda: b3.strsm("L", "L", "N", "N", 1.0, T, X), lambda: X.copy_(B))]
    reps = max(3, int(3e10 / (2.0 * n ** 3)))
    res = {i: [] for i in range(len(cases))}
    for rnd in range(rounds):
        for i, (_, _, fl, fn, pre) in enumerate(cases):
            if pre:
                pre()
            fn()
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
            e0.record()
            for _ in range(reps):
                fn()
            e1.record(); torch.cuda.synchronize()
            res[i].append(e0.elapsed_time(e1) / reps)
    sg = None
    for i, (r, v, fl, _, _) in enumerate(cases):
        ms = float(np.median(res[i]))
        tf = fl / ms / 1e9
        sg = tf if r == "sgemm" else sg
        print(f"| {n} | {r} | {v} | {ms * 1e3:.1f} | {tf:.1f} | {100 * tf / sg:.0f} |", flush=True)
    del A, B, C, X, T
    torch.cuda.empty_cache()
