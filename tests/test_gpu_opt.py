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


OPT_SMALL = ModelCfg("opt-small", 256, 4, 4, 1024, 2, model_layers=3, arch="opt")   # head_dim 64: the tcgen05 kernels


def test_opt_tiny_parity_mixed():
    """A small OPT (d 256, 4 heads of 64 -- OPT-1.3B's head_dim, so the tcgen05 attention kernels -- f 1024) with
    mixed ranks / targets and ragged sequences.  (The d = 64 opt_tiny sits at cos 0.9984-0.9990 on its deepest LoRA
    grads with O(1) branches, R26: too few reduction terms to average the bf16 operand rounding; it still covers the
    bitwise invariants below.)"""
    w = Workload("opt_mix", OPT_SMALL,
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


def test_relu_mask_valid():
    """The ReLU mask is a decision several answers satisfy near z = 0 (where bf16 rounding of the GEMM operands can
    flip the sign).  Check the kernel's OWN decision (the saved a = relu(fc1) of a SAVE batch, a > 0) against the exact
    fp64 sign of the oracle's pre-activation z = fc1(LN2(h)) + LoRA: they must agree wherever |z| exceeds the a-priori
    bf16 bound tau = 2^-8 * sum_k |hn_k| |W_k| (+ the LoRA term), with a x4 margin from layer 1 on for the propagated
    input differences; and the band |z| <= tau must be a small fraction of the entries."""
    from tests.test_gpu_whitebox import gpu_layer_values
    from oracle import menos_oracle as O
    w = Workload("opt_relu", MODELS["opt_tiny"], [ClientCfg(8, 16.0, OPT_T, [33, 1, 70]),
                                                  ClientCfg(16, 32.0, ("v", "up", "down"), [129])])
    inputs = make_inputs(w, seed=27)
    weights, adapters, io = inputs
    gpu = gpu_layer_values(w, inputs)
    m = w.model
    F = np.float64
    zs, taus = [[] for _ in range(m.n_layers)], [[] for _ in range(m.n_layers)]
    for i, c in enumerate(w.clients):
        off = 0
        s = c.alpha / c.rank
        for S in c.seq_lens:
            x = np.asarray(io[i][0][off:off + S], F)
            off += S
            for l in range(m.n_layers):
                W = {k: np.asarray(v, F) for k, v in weights[l].items()}
                y, cache = O.opt_layer_fwd(x, W, {t: (np.asarray(a, F), np.asarray(b, F))
                                                  for t, (a, b) in adapters[i][l].items()}, s, m, F)
                hn = cache["hn"]
                z = hn @ W["wup"].T + W["bup"]
                tau = 2.0 ** -8 * (np.abs(hn) @ np.abs(W["wup"]).T)
                if "up" in adapters[i][l]:
                    A, B = (np.asarray(v, F) for v in adapters[i][l]["up"])
                    U = hn @ A.T
                    z = z + s * U @ B.T
                    tau = tau + 2.0 ** -8 * s * ((np.abs(hn) @ np.abs(A).T) + np.abs(U)) @ np.abs(B).T
                zs[l].append(z)
                taus[l].append(tau)
                x = y
    band_total = 0
    for l in range(m.n_layers):
        z, tau = np.concatenate(zs[l]), np.concatenate(taus[l]) * (1.0 if l == 0 else 4.0)
        gm = gpu[l]["a"][:, :m.d_ff] > 0
        clear = np.abs(z) > tau
        assert np.array_equal(gm[clear], (z > 0)[clear]), (l, int(np.sum(gm[clear] != (z > 0)[clear])))
        band_total += int(np.sum(~clear))
        if l == 0:   # exact inputs at layer 0: the a-priori band is tight; deeper layers carry the x4 margin
            assert np.mean(~clear) < 0.05, (l, float(np.mean(~clear)))
    print("entries inside the rounding band:", band_total)
