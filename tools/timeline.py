"""Kernel timeline of one library call (CUPTI via torch.profiler), for finding
gaps, tails and stream overlap inside multi-launch routines (STRSM).

python tools/timeline.py strsm [n] [cols]   -> prints one line per kernel:
    start_us end_us dur_us stream grid name   (relative to the first kernel)
and a summary (busy time = union of kernel intervals, sum of durations).
"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from torch.profiler import profile, ProfilerActivity
import paper_conf_ipps_cuiwxyf11_b200 as b3

which = sys.argv[1] if len(sys.argv) > 1 else "strsm"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 8192
cols = int(sys.argv[3]) if len(sys.argv) > 3 else n
A = b3.colmajor(n, n); A.uniform_(-1, 1)
T = b3.colmajor(n, n); T.uniform_(-1, 1); T.diagonal().add_(n / 2.0)
B = b3.colmajor(n, cols); B.uniform_(-1, 1)
C = b3.colmajor(n, cols); C.uniform_(-1, 1)
calls = {
    "strsm": lambda: b3.strsm("L", "L", "N", "N", 1.5, T, B),
    "strmm": lambda: b3.strmm("L", "L", "N", "N", 1.5, T, B),
    "sgemm": lambda: b3.sgemm("N", "N", 1.5, A, B, 0.5, C),
}
X = b3.colmajor(n, cols)


def chain():
    b3.sgemm("N", "N", 1.5, A, B, 0.5, C)
    b3.ssymm("L", "L", 1.5, A, B, 0.5, C)
    b3.ssyrk("L", "N", 1.5, A, 0.5, C)
    b3.ssyr2k("L", "N", 1.5, A, B, 0.5, C)
    X.copy_(B)
    b3.strmm("L", "L", "N", "N", 1.5, T, X)
    b3.strsm("L", "L", "N", "N", 1.5, T, X)


calls["chain"] = chain
fn = calls[which]
for k, v in json.loads(os.environ.get("TL_OPTS", "{}")).items():   # tuning options
    b3.set_option(k, v)
for _ in range(3):
    fn()
torch.cuda.synchronize()
reps = int(os.environ.get("TL_REPS", "1"))      # profile reps back to back, print the last
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
import tempfile
tmp = os.path.join(tempfile.mkdtemp(), "trace.json")
prof.export_chrome_trace(tmp)
tr = json.load(open(tmp))
evs = []
for e in tr.get("traceEvents", []):
    if e.get("cat") == "kernel" or (e.get("cat") == "gpu_memset") or (e.get("cat") == "gpu_memcpy"):
        a = e.get("args", {})
        evs.append((float(e["ts"]), float(e["ts"]) + float(e["dur"]), e["name"], a.get("stream", e.get("tid")),
                    a.get("grid", "")))
evs.sort()
if reps > 1:
    evs = evs[-int(os.environ.get("TL_LAST", "60")):]
t0 = evs[0][0]
busy, cur_s, cur_e = 0.0, None, None
for s_, e_, *_ in evs:
    if cur_e is None or s_ > cur_e:
        if cur_e is not None:
            busy += cur_e - cur_s
        cur_s, cur_e = s_, e_
    else:
        cur_e = max(cur_e, e_)
busy += cur_e - cur_s
span = max(e_ for _, e_, *_ in evs) - t0
for s_, e_, nm, st, gr in evs:
    print(f"{s_ - t0:9.1f} {e_ - t0:9.1f} {e_ - s_:8.1f}  s{st}  {str(gr):14s} {nm[:50]}")
print(json.dumps({"which": which, "n": n, "cols": cols, "kernels": len(evs), "span_us": round(span, 1),
                  "busy_us": round(busy, 1), "sum_us": round(sum(e_ - s_ for s_, e_, *_ in evs), 1)}))
