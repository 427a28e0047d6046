"""OPT server segment on the GPU (NEXT-4): pre-LayerNorm, biased projections, ReLU MLP, no RoPE,
through the same C-ABI (menos_model_cfg.arch = MENOS_ARCH_OPT) against the OPT oracle (tests/test_oracle_opt.py
pins it).  Bars as for Llama (BASELINE.json north_star); invariants (b) zero-B == base and (c) batched == alone
bitwise."""
import dataclasses

import numpy as np
import pytest

from tests.parity_util import compare_step, make_inputs, run_gpu_step, run_oracle_step, act_err
from workloads import ClientCfg, MODELS, Workload
from workloads.synth import ModelCfg

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")

OPT_T = ("q", "k", "v", "o", "up", "down")


def assert_ok(rep):
    bad = {k: v for k, v in rep.items() if not v["ok"]}
    assert not bad, bad


def test_opt_tiny_parity_mixed():
    w = Workload("opt_mix", MODELS["opt_tiny"],
                 [ClientCfg(4, 8.0, ("q", "v"), [16, 16]), ClientCfg(8, 16.0, OPT_T, [33, 1, 70]),
                  ClientCfg(16, 32.0, ("v", "up", "down"), [129])])
    assert_ok(compare_step(run_gpu_step(w, seed=21), run_oracle_step(w, seed=21)))


def test_opt_1p3b_width_two_layers():
    """OPT-1.3B widths (d 2048, 32 heads of 64, ffn 8192), 2 server layers, 2 clients (paper's q,v r=8 and all
    targets), ragged sequences spanning several 128-row tiles."""
    m = dataclasses.replace(MODELS["opt1.3b"], n_layers=2)
    w = Workload("opt13_2l", m, [ClientCfg(8, 16.0, ("q", "v"), [100, 100, 57]),
                                 ClientCfg(16, 32.0, OPT_T, [200, 33])])
    assert_ok(compare_step(run_gpu_step(w, seed=22), run_oracle_step(w, seed=22)))


@pytest.mark.parametrize("d,heads,ffn", [(4096, 32, 16384), (1024, 16, 4096)])
def test_opt_layernorm_widths_one_layer(d, heads, ffn):
    """LayerNorm launch shapes other than 1.3B's: d = 4096 (OPT-6.7B widths, head_dim 128 -> tcgen05 attention;
    four warps per row) and d = 1024 (one warp per row); 1 server layer, ragged sequences."""
    m = ModelCfg(f"opt-d{d}", d, heads, heads, ffn, 1, model_layers=2, arch="opt")
    w = Workload(f"opt_d{d}", m, [ClientCfg(8, 16.0, ("q", "v"), [130, 5]), ClientCfg(16, 32.0, OPT_T, [77])])
    assert_ok(compare_step(run_gpu_step(w, seed=23), run_oracle_step(w, seed=23)))


def test_opt_invariants_zero_b_and_batched_alone():
    m = MODELS["opt_tiny"]
    cl = [ClientCfg(4, 8.0, ("q", "v"), [20, 12]), ClientCfg(8, 16.0, OPT_T, [20, 12])]
    w = Workload("zb", m, cl)
    weights, adapters, io = make_inputs(w, seed=23, zero_b=True)
    io[1] = io[0]
    out = run_gpu_step(w, inputs=(weights, adapters, io), grads=False)
    assert np.array_equal(out["x_s"][0], out["x_s"][1])
    inputs = make_inputs(w, seed=24)
    full = run_gpu_step(w, inputs=inputs)
    for i, c in enumerate(w.clients):
        one = run_gpu_step(Workload("one", m, [c]), inputs=(inputs[0], [inputs[1][i]], [inputs[2][i]]))
        assert np.array_equal(full["x_s"][i], one["x_s"][0])
        assert np.array_equal(full["g_s"][i], one["g_s"][0])


def test_opt_nograd_reforward_bitwise():
    w = Workload("ng", MODELS["opt_tiny"], [ClientCfg(8, 16.0, OPT_T, [40, 9])])
    inputs = make_inputs(w, seed=25)
    a = run_gpu_step(w, inputs=inputs, flags=0)
    b = run_gpu_step(w, inputs=inputs, flags=1)
    assert np.array_equal(a["x_s"][0], b["x_s"][0]) and np.array_equal(a["g_s"][0], b["g_s"][0])


def test_opt_rejects_gate_target():
    from paper_conf_middleware_hul24_b200.menos import MenosError
    from tests.parity_util import new_server
    w = Workload("g", MODELS["opt_tiny"], [ClientCfg(4, 8.0, ("q",), [8])])
    weights, _, _ = make_inputs(w, seed=26)
    srv = new_server(w, weights)
    with pytest.raises(MenosError):
        srv.register_client(4, 8.0, ("gate",))
    srv.close()
