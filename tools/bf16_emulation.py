"""How close can ANY bf16 implementation get to the oracle?  Evaluates the oracle with every GEMM / attention operand
rounded to bf16 (the kernels' operand precision, fp32 accumulation) and reports the worst gradient cosines against the
plain fp32 oracle.  Used to choose input recipes whose bars (BASELINE north_star: cos >= 0.999) an exact-bf16 kernel
can meet (R26).  CPU only.

  python tools/bf16_emulation.py"""
import dataclasses
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from oracle import menos_oracle as O  # noqa: E402
from tests.parity_util import compare_step, make_inputs, run_oracle_step  # noqa: E402
from workloads import ClientCfg, MODELS, ModelCfg, Workload, bf16_round  # noqa: E402

OPT_T = ("q", "k", "v", "o", "up", "down")


def _r(a):
    return bf16_round(np.asarray(a, np.float32))


def emulated(w, inputs):
    pf, pb, af, ab = O.proj_fwd, O.proj_bwd, O.attention_fwd, O.attention_bwd
    O.proj_fwd = lambda x, W, lora, s: pf(_r(x), W, lora, s)
    O.proj_bwd = lambda dy, x, W, lora, s, U: pb(_r(dy), _r(x), W, lora, s, None if U is None else _r(U))
    O.attention_fwd = lambda q, k, v: af(_r(q), _r(k), _r(v))
    O.attention_bwd = lambda dO, q, k, v: ab(_r(dO), _r(q), _r(k), _r(v))
    try:
        return run_oracle_step(w, inputs=inputs)
    finally:
        O.proj_fwd, O.proj_bwd, O.attention_fwd, O.attention_bwd = pf, pb, af, ab


def main():
    cases = [("opt_small", ModelCfg("opt-small", 256, 4, 4, 1024, 2, model_layers=3, arch="opt"),
              [ClientCfg(4, 8.0, ("q", "v"), [16, 16]), ClientCfg(8, 16.0, OPT_T, [33, 1, 70]),
               ClientCfg(16, 32.0, ("v", "up", "down"), [129])]),
             ("llama_tiny_mix", dataclasses.replace(MODELS["tiny"], n_kv_heads=2),
              [ClientCfg(4, 8.0, ("q", "k", "v", "o", "gate", "up", "down"), [1, 17, 3]),
               ClientCfg(16, 32.0, ("q", "v"), [129]), ClientCfg(8, 16.0, ("k", "o", "gate", "up", "down"), [64, 40])])]
    for name, m, cl in cases:
        w = Workload(name, m, cl)
        inputs = make_inputs(w, seed=21)
        rep = compare_step(emulated(w, inputs), run_oracle_step(w, inputs=inputs))
        worst = sorted((round(v["metric"], 6), k) for k, v in rep.items() if v["kind"] == "cos")[:4]
        print(name, "worst cosines of an exact-bf16 evaluation:", worst)


if __name__ == "__main__":
    main()
