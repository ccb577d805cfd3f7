"""Kernel timeline of one DTRSM call (CUPTI via torch.profiler): per-kernel
durations summed by name, for the fp64 triangular solve's launch structure.
python tools/dtrsm_timeline.py [n]"""
import collections, json, os, sys, tempfile
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from torch.profiler import profile, ProfilerActivity
import paper_conf_ipps_cuiwxyf11_b200 as b3
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
T = b3.colmajor(n, n, dtype=torch.float64); T.uniform_(-1, 1); T.mul_(1.0 / n); T.diagonal().fill_(1.0)
B = b3.colmajor(n, n, dtype=torch.float64); B.uniform_(-1, 1)
for _ in range(2):
    b3.dtrsm("L", "L", "N", "N", 1.0, T, B)
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    b3.dtrsm("L", "L", "N", "N", 1.0, T, B)
    torch.cuda.synchronize()
tmp = os.path.join(tempfile.mkdtemp(), "t.json")
prof.export_chrome_trace(tmp)
ev = [e for e in json.load(open(tmp))["traceEvents"] if e.get("cat") == "kernel"]
ev.sort(key=lambda e: e["ts"])
span = ev[-1]["ts"] + ev[-1]["dur"] - ev[0]["ts"]
agg = collections.defaultdict(lambda: [0, 0.0])
for e in ev:
    k = e["name"].split("(")[0][-40:]
    agg[k][0] += 1; agg[k][1] += e["dur"]
print(json.dumps({"n": n, "kernels": len(ev), "span_us": round(span, 1),
                  "busy_us": round(sum(e["dur"] for e in ev), 1),
                  "by_kernel": {k: [c, round(t, 1)] for k, (c, t) in agg.items()}}, indent=1))
for e in ev[:12] + ev[-6:]:
    print(round(e["ts"] - ev[0]["ts"], 1), round(e["dur"], 1), e["args"].get("grid"), e["name"][:60])
