"""One STRSM call (after a warm-up) for ncu / trace captures: python tools/strsm_once.py [n]."""
import sys, torch
sys.path.insert(0, ".")
import paper_conf_ipps_cuiwxyf11_b200 as b3
n = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
T = b3.colmajor(n, n); T.uniform_(-1, 1); T.mul_(1.0 / n); T.diagonal().fill_(1.0)
B = b3.colmajor(n, n); B.uniform_(-1, 1)
X = b3.colmajor(n, n)
for _ in range(2):
    X.copy_(B); b3.strsm("L", "L", "N", "N", 1.0, T, X)
torch.cuda.synchronize()
