"""Latency of small tcgen05 launches (the TRSM inversion-doubling regime).
`dev` = device time only: a sleep kernel is queued first so the host has
finished enqueuing before the GPU reaches the timed region; `host` = host
enqueue time per call."""
import sys, time, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3

def dev_time(fn, reps=20):
    for _ in range(3): fn()
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(True); e1 = torch.cuda.Event(True)
    torch.cuda._sleep(50_000_000)          # ~25 ms of GPU busy time
    e0.record()
    t0 = time.perf_counter()
    for _ in range(reps): fn()
    t1 = time.perf_counter()
    e1.record(); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3, (t1 - t0) / reps * 1e6

for (m, n, k) in [(128, 128, 32), (128, 128, 128), (256, 256, 256), (1024, 1024, 128),
                  (4096, 128, 128), (1024, 1024, 1024), (2048, 2048, 1024)]:
    A = b3.colmajor(m, k); B = b3.colmajor(k, n); C = b3.colmajor(m, n)
    for x in (A, B, C): x.uniform_(-1, 1)
    d, h = dev_time(lambda: b3.sgemm("N", "N", 1.0, A, B, 0.0, C))
    print(f"m={m:5d} n={n:5d} k={k:5d}: sgemm dev {d:7.1f} us  host {h:6.1f} us", flush=True)
for (n, nrhs) in [(128, 128), (2048, 128), (2048, 2048), (4096, 4096)]:
    T = b3.colmajor(n, n); T.uniform_(-1, 1); T.diagonal().add_(n / 2.0)
    Bm = b3.colmajor(n, nrhs); Bm.uniform_(-1, 1)
    d, h = dev_time(lambda: b3.strsm('L', 'L', 'N', 'N', 1.0, T, Bm), reps=5)
    print(f"strsm n={n} nrhs={nrhs}: dev {d:.1f} us  host {h:.1f} us  ({n*n*nrhs/d/1e6:.1f} TF/s)", flush=True)
