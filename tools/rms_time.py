"""Isolated RMSNorm fwd / fwd+bwd timing at the cfg1 shape (T = 8192 tokens, d = 4096) through menos_test_rmsnorm.
Each call ends in a device sync, so the per-call time includes one launch + sync gap (same for every variant).
Prints one JSON line: us per fwd, us per bwd (fwd+bwd minus fwd), and GB/s against DESIGN's algorithmic bytes
(fwd 6d+4 B/token, bwd 16d+4 B/token with the bf16 copy)."""
import json
import os
import sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_hul24_b200.menos import lib, check

T, d = (int(a) for a in sys.argv[1:3]) if len(sys.argv) > 2 else (8192, 4096)
dev = "cuda"
x = torch.randn(T, d, device=dev)
g = torch.randn(d, device=dev)
y = torch.empty(T, d, device=dev, dtype=torch.bfloat16)
rstd = torch.empty(T, device=dev)
dy = torch.randn(T, d, device=dev).bfloat16()
res = torch.randn(T, d, device=dev)
dx = torch.empty(T, d, device=dev)
dxb = torch.empty(T, d, device=dev, dtype=torch.bfloat16)
L = lib()


def run(bwd):
    check(L.menos_test_rmsnorm(T, d, x.data_ptr(), g.data_ptr(), 1e-5, y.data_ptr(), rstd.data_ptr(),
                               dy.data_ptr() if bwd else None, res.data_ptr(), dx.data_ptr(), dxb.data_ptr()))


def timeit(bwd, n=50):
    for _ in range(5):
        run(bwd)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    a.record()
    for _ in range(n):
        run(bwd)
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) * 1e3 / n


f = timeit(False)
fb = timeit(True)
bw = fb - f
print(json.dumps({"T": T, "d": d, "fwd_us": round(f, 2), "bwd_us": round(bw, 2),
                  "fwd_gbs": round(T * (6 * d + 4) / f / 1e3, 1), "bwd_gbs": round(T * (16 * d + 4) / bw / 1e3, 1)}))
