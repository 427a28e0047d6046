"""Fused-attention forward + backward at one shape through menos_test_attention (timing / ncu capture aid).

  python tools/attn_time.py <mode> <lens=512x16> <H> <Hkv> [iters=5] [hd=128]

mode = menos_test_set_attn_tc mode (14 = default two-kernel backward, 46 = one-pass fused backward).
Prints the mean fwd+bwd call time over the iterations after one warm-up call."""
import ctypes as C
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_hul24_b200 import menos as M  # noqa: E402


def main():
    mode, spec, H, Hkv = int(sys.argv[1]), sys.argv[2], int(sys.argv[3]), int(sys.argv[4])
    iters = int(sys.argv[5]) if len(sys.argv) > 5 else 5
    hd = int(sys.argv[6]) if len(sys.argv) > 6 else 128
    L, n = (int(v) for v in spec.split("x"))
    lens = [L] * n
    T, N = sum(lens), (H + 2 * Hkv) * hd
    lib = M.lib()
    M.check(lib.menos_test_set_attn_tc(mode), testing=True)
    g = torch.Generator(device="cuda").manual_seed(0)
    qkv = torch.randn(T, N, device="cuda", generator=g).to(torch.bfloat16)
    dO = torch.randn(T, H * hd, device="cuda", generator=g).to(torch.bfloat16)
    O = torch.empty(T, H * hd, dtype=torch.bfloat16, device="cuda")
    lse = torch.empty(H, T, dtype=torch.float32, device="cuda")
    dqkv = torch.empty(T, N, dtype=torch.bfloat16, device="cuda")
    arr = (C.c_int32 * len(lens))(*lens)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    call = lambda: M.check(lib.menos_test_attention(len(lens), arr, H, Hkv, hd, qkv.data_ptr(), O.data_ptr(),  # noqa
                                                    lse.data_ptr(), dO.data_ptr(), dqkv.data_ptr(), 1e4), testing=True)
    call()
    torch.cuda.synchronize()
    ev0.record()
    for _ in range(iters):
        call()
    ev1.record()
    torch.cuda.synchronize()
    print(f"mode {mode} {spec} H{H}/{Hkv} hd{hd}: {ev0.elapsed_time(ev1) / iters:.3f} ms per fwd+bwd call "
          f"(includes the harness's allocations)")


if __name__ == "__main__":
    main()
