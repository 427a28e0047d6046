"""GPU parity at BASELINE.json full sizes (Llama-2-7B width), through the C-ABI, against the CPU oracle.

* 2-layer depth-truncated segment at 7B width with several clients (every output compared).
* The bench launch configuration (cfg1: 31 layers, 4 clients x 4 x 512 tokens, one batched pass): client 0 is
  recomputed by the oracle in full (x_s, g_s, every dA/dB); the other clients' rows are checked for
  finiteness and scale (the oracle computes one client at a time; a batched call is defined as the
  concatenation of per-client calls, and batch invariance is tested bitwise elsewhere).
Bars: activations max|d|/max|ref| <= 2e-2, every gradient tensor cosine >= 0.999 (BASELINE north_star).
"""
import numpy as np
import pytest

from tests.parity_util import compare_step, make_inputs, run_gpu_step, run_oracle_step
from workloads import ClientCfg, MODELS, TARGETS, Workload, workload

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def assert_report(rep):
    bad = {k: v for k, v in rep.items() if not v["ok"]}
    assert not bad, bad


def test_7b_width_two_layers_mixed_clients():
    m = MODELS["7b"].with_layers(2)
    cl = [ClientCfg(8, 16.0, ("q", "v"), [512, 300]), ClientCfg(16, 32.0, ("q", "k", "v", "o"), [129, 1]),
          ClientCfg(4, 8.0, ("gate", "up", "down"), [640])]
    w = Workload("7b_l2_mix", m, cl)
    inputs = make_inputs(w, seed=21)
    rep = compare_step(run_gpu_step(w, inputs=inputs), run_oracle_step(w, inputs=inputs))
    assert_report(rep)


@pytest.mark.parametrize("outlier", [False, True])
def test_7b_width_two_layers_plain_recipe(outlier):
    """SURVEY.md §8(d)'s recipe as written: every base projection N(0, 0.02^2) (no depth-scaled o / down, reading
    R27 off), and its massive-activation variant (two channels of x_c x100)."""
    m = MODELS["7b"].with_layers(2)
    cl = [ClientCfg(8, 16.0, ("q", "v"), [512, 77]), ClientCfg(16, 32.0, ("q", "k", "v", "o", "down"), [256])]
    w = Workload("7b_l2_plain", m, cl)
    inputs = make_inputs(w, seed=31, recipe="plain", outlier=outlier)
    rep = compare_step(run_gpu_step(w, inputs=inputs), run_oracle_step(w, inputs=inputs))
    assert_report(rep)


def test_13b_width_two_layers_cfg3_shapes():
    """BASELINE configs[3] shapes (Llama-2-13B: d 5120, 40 heads, f 13824; r = 16 on all 7 projections, one 2048-token
    sequence) at depth 2, plus a second client with a ragged pair of sequences."""
    m = MODELS["13b"].with_layers(2)
    cl = [ClientCfg(16, 32.0, TARGETS, [2048]), ClientCfg(16, 32.0, TARGETS, [700, 37])]
    w = Workload("13b_l2", m, cl)
    inputs = make_inputs(w, seed=33)
    rep = compare_step(run_gpu_step(w, inputs=inputs), run_oracle_step(w, inputs=inputs))
    assert_report(rep)


def test_bench_configuration_cfg1_full_depth():
    """The launch configuration bench.py times (31 layers, 4 clients x 4 x 512, one batched pass): clients 0 and 3 are
    recomputed by the oracle in full (x_s, g_s, every dA/dB; the oracle runs one client at a time); clients 1 and 2
    get finiteness / scale checks and are covered by the bitwise batched == alone invariant elsewhere."""
    w = workload("cfg1_7b_x4")
    inputs = make_inputs(w, seed=0)
    gpu = run_gpu_step(w, inputs=inputs)
    ora = run_oracle_step(w, inputs=inputs, clients=[0, 3])
    rep = compare_step(gpu, ora, clients=[0, 3])
    print({k: round(v["metric"], 5) for k, v in rep.items() if ".L" not in k or k.endswith("q.dA")})
    assert_report(rep)
    ref_scale = float(np.max(np.abs(ora["x_s"][0])))
    for i in (1, 2):
        assert np.all(np.isfinite(gpu["x_s"][i])) and np.all(np.isfinite(gpu["g_s"][i]))
        assert 0.5 * ref_scale < float(np.max(np.abs(gpu["x_s"][i]))) < 2.0 * ref_scale
