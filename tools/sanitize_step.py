"""One forward + backward + AdamW step of small batches through libmenos.so, for compute-sanitizer
(memcheck / racecheck / synccheck) runs over every kernel family the server path launches:

  compute-sanitizer --tool memcheck   python tools/sanitize_step.py
  compute-sanitizer --tool racecheck  python tools/sanitize_step.py
  compute-sanitizer --tool synccheck  python tools/sanitize_step.py

Batches: BASELINE configs[0] (tiny, mma.sync attention), the tiny mix (GQA, all 7 targets, ragged), a head_dim-128
model (tcgen05 GEMM + persistent attention forward / one-pass and two-kernel backward), prefix-tuning clients, OPT.
Prints one line per batch; exit code 0 when every call returned OK."""
import dataclasses
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from tests.parity_util import make_inputs, new_server, register, run_gpu_step  # noqa: E402
from workloads import ClientCfg, MODELS, ModelCfg, PREFIX, TARGETS, Workload, workload  # noqa: E402


def batches():
    tiny_gqa = dataclasses.replace(MODELS["tiny"], n_kv_heads=2)
    hd128 = ModelCfg("hd128", 512, 4, 2, 1024, 2, model_layers=3)
    mix = [ClientCfg(4, 8.0, TARGETS, [1, 17, 3]), ClientCfg(16, 32.0, ("q", "v"), [129]),
           ClientCfg(8, 16.0, ("k", "o", "gate", "up", "down"), [64, 40])]
    yield workload("cfg0_tiny")
    yield Workload("tiny_mix", tiny_gqa, mix)
    yield Workload("hd128_mix", hd128, mix)
    yield Workload("prefix_mix", hd128, [ClientCfg(4, 8.0, ("q", "v"), [16, 16]), ClientCfg(4, 1.0, (PREFIX,), [9, 20])])
    yield Workload("opt_mix", MODELS["opt_tiny"], [ClientCfg(4, 8.0, ("q", "v"), [16, 16]),
                                                   ClientCfg(8, 16.0, ("q", "k", "v", "o", "up", "down"), [33, 1])])


def main():
    from paper_conf_middleware_hul24_b200 import menos as M
    modes = [int(m) for m in os.environ.get("MENOS_SANITIZE_MODES", "46,14").split(",")]
    for mode in modes:
        M.check(M.lib().menos_test_set_attn_tc(mode), testing=True)
        for w in batches():
            inputs = make_inputs(w, seed=1)
            srv = new_server(w, inputs[0])
            ids = register(srv, w, inputs[1])
            run_gpu_step(w, inputs=inputs, srv=srv, ids=ids)
            srv.adapter_step(ids)
            srv.sync()
            srv.close()
            print(f"attention mode {mode}: {w.name} OK", flush=True)


if __name__ == "__main__":
    main()
