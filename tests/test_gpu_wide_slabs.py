"""The fused LoRA dU + dB backward (`lora_dub_tc_kernel`) takes 256-column slabs for targets with
N_t >= 8192 and 128-column slabs otherwise (ranks <= 16; larger ranks take the mma.sync kernel,
`test_gpu_parity.py::test_tiny_ranks_above_16`).  The tiny recipe never reaches the
wide case (N_t <= 344), so these tests widen the MLP of the tiny model to d_ff = 8200 (gate / up: N_t = 8200 =
32 slabs of 256 + an 8-column tail; PAPER.md:294's LoRA on the projections, Alg. 1 L10-12 for the gradients) and
check (a) parity with the oracle and (b) that a client's results do not depend on who shares its batch."""
import dataclasses

import numpy as np
import pytest

from tests.parity_util import compare_step, make_inputs, run_gpu_step, run_oracle_step
from workloads import ClientCfg, MODELS, TARGETS, Workload

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _w():
    m = dataclasses.replace(MODELS["tiny"], d_ff=8200, n_layers=2, model_layers=3)
    cl = [ClientCfg(4, 8.0, ("gate", "up"), [37, 90]), ClientCfg(16, 32.0, TARGETS, [130]),
          ClientCfg(6, 12.0, ("up", "down"), [65]), ClientCfg(8, 16.0, ("q", "gate"), [3, 128])]
    return Workload("wide_mlp", m, cl)


def test_wide_slabs_parity_vs_oracle():
    w = _w()
    rep = compare_step(run_gpu_step(w, seed=21), run_oracle_step(w, seed=21))
    bad = {k: v for k, v in rep.items() if not v["ok"]}
    assert not bad, bad


def test_wide_slabs_batched_equals_alone_bitwise():
    w = _w()
    inputs = make_inputs(w, seed=22)
    full = run_gpu_step(w, inputs=inputs)
    for i, c in enumerate(w.clients):
        one = run_gpu_step(Workload("one", w.model, [c]), inputs=(inputs[0], [inputs[1][i]], [inputs[2][i]]))
        assert np.array_equal(full["x_s"][i], one["x_s"][0]), i
        assert np.array_equal(full["g_s"][i], one["g_s"][0]), i
        for l, d in enumerate(one["grads"][0]):
            for t, (dA, dB) in d.items():
                assert np.array_equal(full["grads"][i][l][t][0], dA), (i, l, t)
                assert np.array_equal(full["grads"][i][l][t][1], dB), (i, l, t)
