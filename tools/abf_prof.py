"""Per-phase cycle breakdown of the one-pass attention backward (tuning aid; needs a -DMENOS_ABF_PROF build:
MENOS_NVCC_DEFS=-DMENOS_ABF_PROF python -c 'from paper_conf_middleware_hul24_b200 import build as b; b.build(force=True)').

  python tools/abf_prof.py [lens=512x16] [H=32] [Hkv=32]

Runs menos_test_attention (forward + backward) at the given shape and prints the role threads' cycle totals per
phase (summed over CTAs) as fractions of the MMA thread's total."""
import ctypes as C
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_hul24_b200 import menos as M  # noqa: E402

NAMES = ["mma: wait Q/dO stage", "mma: wait sd_free", "mma: wait K/V", "mma: wait ew_done", "mma: wait acc_free",
         "mma: wait dq_free", "mma: issue/other", "ew: wait stage+S", "ew: compute+store", "ew: wait pd_free",
         "ew: epi wait acc", "ew: epilogue", "drain: wait dq_full", "drain: non-last", "drain: last", "-"]


def main():
    spec = sys.argv[1] if len(sys.argv) > 1 else "512x16"
    H = int(sys.argv[2]) if len(sys.argv) > 2 else 32
    Hkv = int(sys.argv[3]) if len(sys.argv) > 3 else 32
    L, n = (int(v) for v in spec.split("x"))
    lens = [L] * n
    hd = 128
    T, N = sum(lens), (H + 2 * Hkv) * hd
    lib = M.lib()
    M.check(lib.menos_test_set_attn_tc(46), testing=True)
    g = torch.Generator(device="cuda").manual_seed(0)
    qkv = torch.randn(T, N, device="cuda", generator=g).to(torch.bfloat16)
    dO = torch.randn(T, H * hd, device="cuda", generator=g).to(torch.bfloat16)
    O = torch.empty(T, H * hd, dtype=torch.bfloat16, device="cuda")
    lse = torch.empty(H, T, dtype=torch.float32, device="cuda")
    dqkv = torch.empty(T, N, dtype=torch.bfloat16, device="cuda")
    arr = (C.c_int32 * len(lens))(*lens)
    out = (C.c_ulonglong * 16)()
    import time
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for it in range(3):
        lib.menos_test_abf_prof(out)   # clear
        ev0.record()
        M.check(lib.menos_test_attention(len(lens), arr, H, Hkv, hd, qkv.data_ptr(), O.data_ptr(), lse.data_ptr(),
                                         dO.data_ptr(), dqkv.data_ptr(), 1e4), testing=True)
        ev1.record()
        torch.cuda.synchronize()
        ms = ev0.elapsed_time(ev1)
        lib.menos_test_abf_prof(out)
    v = [int(x) for x in out]
    tot = max(sum(v[0:7]), 1)
    print(json.dumps({"shape": {"lens": spec, "H": H, "Hkv": Hkv}, "fwd_bwd_call_ms": round(ms, 3),
                      "dbg": os.environ.get("MENOS_ABF_DBG", "0"),
                      "phases_frac_of_mma_total": {NAMES[k]: round(v[k] / tot, 4) for k in range(15)},
                      "mma_total_cycles": tot}, indent=1))


if __name__ == "__main__":
    main()
