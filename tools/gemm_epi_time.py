"""Time the dX GEMM shapes of a Llama-2-7B layer at cfg1's T through menos_test_gemm_time (CUDA events, back to
back launches) with the plain store epilogue and with the fused epilogue the server uses, so the epilogue's cost
is isolated.  Tuning aid; prints one JSON line.  python tools/gemm_epi_time.py [tag]"""
import ctypes as C
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_hul24_b200 import menos  # noqa: E402

lib = menos.lib()
T, d, f = 8192, 4096, 11008
res = {"tag": sys.argv[1] if len(sys.argv) > 1 else ""}
g = torch.Generator(device="cuda").manual_seed(0)


def rnd(*shape):
    return (torch.randn(*shape, device="cuda", generator=g) * 0.5).to(torch.bfloat16)


def t(name, M, N, K, b_mn, epi, aux=None, out_cols=None):
    A = rnd(M, K)
    B = rnd(K, N) if b_mn else rnd(N, K)
    out = torch.empty(M, out_cols or N, dtype=torch.bfloat16, device="cuda")
    ms = C.c_float()
    rc = lib.menos_test_gemm_time(M, N, K, b_mn, C.c_void_p(A.data_ptr()), C.c_void_p(B.data_ptr()),
                                  C.c_void_p(out.data_ptr()), epi, C.c_void_p(aux.data_ptr() if aux is not None else 0),
                                  20, C.byref(ms))
    assert rc == 0, rc
    res[name] = {"ms": round(ms.value, 4), "tflops": round(2.0 * M * N * K / ms.value / 1e9, 1)}


gu = rnd(T, 2 * f)
t("down_dx_store", T, f, d, 1, 0)
t("down_dx_swiglu_bwd", T, f, d, 1, 4, aux=gu, out_cols=2 * f)
t("gateup_dx_store", T, d, 2 * f, 1, 0)
t("qkv_dx_store", T, d, 3 * d, 1, 0)
t("gateup_fwd_store", T, 2 * f, d, 0, 0)
t("gateup_fwd_swiglu", T, 2 * f, d, 0, 3, out_cols=2 * f)
print(json.dumps(res))
