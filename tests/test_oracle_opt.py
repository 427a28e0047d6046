"""Pins of the OPT oracle (NEXT-4; oracle/menos_oracle.py opt_layer_*, layernorm_*) to things other than itself:
transformers' OPTDecoderLayer in fp64 with LoRA as a parametrisation W0 + s B A and torch.autograd; torch's
layer_norm; closed forms; finite differences in fp64 over a 2-layer segment."""
import numpy as np
import pytest
import torch

from oracle import menos_oracle as O
from workloads import ClientCfg, MODELS, ModelCfg, base_layer_weights, client_adapters, client_inputs

F64 = np.float64


def rel(a, b):
    return np.max(np.abs(a - b)) / max(np.max(np.abs(b)), 1e-300)


def opt_cfg(layers=1, d=64, H=4, f=256):
    return ModelCfg("opt-t", d, H, H, f, layers, model_layers=layers + 1, arch="opt")


def test_layernorm_closed_form_and_torch():
    r = np.random.default_rng(1)
    g, b = r.standard_normal(32), r.standard_normal(32)
    # a constant row has zero centred part: y = b exactly, and dx = 0 for any dy (the row has no direction left)
    x = np.full((3, 32), 2.5)
    y, rstd = O.layernorm_fwd(x, g, b, 1e-5)
    np.testing.assert_array_equal(y, np.broadcast_to(b, y.shape))
    x = r.standard_normal((5, 32)) * 3 + 1
    dy = r.standard_normal((5, 32))
    y, rstd = O.layernorm_fwd(x, g, b, 1e-5)
    xt = torch.from_numpy(x).requires_grad_(True)
    yt = torch.nn.functional.layer_norm(xt, (32,), torch.from_numpy(g), torch.from_numpy(b), 1e-5)
    (yt * torch.from_numpy(dy)).sum().backward()
    assert rel(y, yt.detach().numpy()) < 1e-12
    assert rel(O.layernorm_bwd(dy, x, g, rstd), xt.grad.numpy()) < 1e-12


def hf_opt_run(cfg, W, lora, s, x, g):
    from transformers import OPTConfig
    from transformers.models.opt.modeling_opt import OPTDecoderLayer
    c = OPTConfig(hidden_size=cfg.d_model, ffn_dim=cfg.d_ff, num_attention_heads=cfg.n_heads,
                  do_layer_norm_before=True, activation_function="relu", enable_bias=True,
                  layer_norm_elementwise_affine=True, dropout=0.0, attention_dropout=0.0)
    c._attn_implementation = "eager"
    L = OPTDecoderLayer(c, 0).double().eval()
    mods = {"q": L.self_attn.q_proj, "k": L.self_attn.k_proj, "v": L.self_attn.v_proj, "o": L.self_attn.out_proj,
            "up": L.fc1, "down": L.fc2}
    bias = {"q": "bq", "k": "bk", "v": "bv", "o": "bo", "up": "bup", "down": "bdown"}
    with torch.no_grad():
        for t, m in mods.items():
            m.weight.copy_(torch.from_numpy(W["w" + t].astype(F64)))
            m.bias.copy_(torch.from_numpy(W[bias[t]].astype(F64)))
        L.self_attn_layer_norm.weight.copy_(torch.from_numpy(W["g1"].astype(F64)))
        L.self_attn_layer_norm.bias.copy_(torch.from_numpy(W["b1"].astype(F64)))
        L.final_layer_norm.weight.copy_(torch.from_numpy(W["g2"].astype(F64)))
        L.final_layer_norm.bias.copy_(torch.from_numpy(W["b2"].astype(F64)))
    for p in L.parameters():
        p.requires_grad_(False)
    leaves = {}
    for t, (A, B) in lora.items():
        At = torch.from_numpy(A.astype(F64)).requires_grad_(True)
        Bt = torch.from_numpy(B.astype(F64)).requires_grad_(True)
        leaves[t] = (At, Bt)
        m = mods[t]
        W0, b0 = m.weight.detach().clone(), m.bias.detach().clone()
        m.forward = (lambda xx, W0=W0, b0=b0, At=At, Bt=Bt: xx @ (W0 + s * Bt @ At).T + b0)
    S = x.shape[0]
    xt = torch.from_numpy(x.astype(F64))[None].requires_grad_(True)
    mask = torch.full((S, S), float("-inf"), dtype=torch.float64).triu(1)[None, None]
    y = L(xt, attention_mask=mask)
    if isinstance(y, tuple):
        y = y[0]
    (y * torch.from_numpy(g.astype(F64))[None]).sum().backward()
    return y.detach().numpy()[0], xt.grad.numpy()[0], {t: (A.grad.numpy(), B.grad.numpy()) for t, (A, B) in leaves.items()}


@pytest.mark.parametrize("targets", [("q", "v"), ("q", "k", "v", "o", "up", "down")])
def test_opt_layer_vs_hf_fp64(targets):
    cfg = opt_cfg()
    W = base_layer_weights(cfg, 0, seed=31)
    c = ClientCfg(4, 8.0, targets, [19])
    lora = client_adapters(cfg, c, seed=32)[0]
    x, g = client_inputs(cfg, c, seed=33)
    s = c.alpha / c.rank
    y_hf, dx_hf, gr_hf = hf_opt_run(cfg, W, lora, s, x, g)
    y, cache = O.opt_layer_fwd(x.astype(F64), W, lora, s, cfg, F64)
    dx, gr = O.opt_layer_bwd(g.astype(F64), cache, W, lora, s, cfg, F64)
    # fp64 both sides; HF's eager attention runs its softmax in fp32 (~1e-7); a dropped term or sign shows up at >1e-3
    assert rel(y, y_hf) < 1e-6
    assert rel(dx, dx_hf) < 1e-6
    assert set(gr) == set(targets)
    for t in targets:
        assert rel(gr[t][0], gr_hf[t][0]) < 1e-6, t
        assert rel(gr[t][1], gr_hf[t][1]) < 1e-6, t


def test_opt_finite_differences_segment_fp64():
    cfg = opt_cfg(layers=2)
    Ws = [base_layer_weights(cfg, l, seed=41) for l in range(2)]
    c = ClientCfg(4, 8.0, ("q", "v", "up", "down"), [9])
    lora = client_adapters(cfg, c, seed=42)
    x, g = client_inputs(cfg, c, seed=43)
    x, g = x.astype(F64), g.astype(F64)
    s = 2.0
    xs, gs, gr = O.segment_fwd_bwd(x, g, Ws, lora, s, cfg, F64)

    def loss(xx, ll):
        return float(np.sum(O.segment_fwd(xx, Ws, ll, s, cfg, F64) * g))

    r = np.random.default_rng(44)
    eps = 1e-6
    dirx = r.standard_normal(x.shape)
    fd = (loss(x + eps * dirx, lora) - loss(x - eps * dirx, lora)) / (2 * eps)
    assert abs(fd - np.sum(gs * dirx)) < 1e-6 * max(1.0, abs(fd))
    for ell in range(2):
        for t in ("q", "up", "down"):
            for which in (0, 1):
                base = lora[ell][t][which]
                dirp = r.standard_normal(base.shape)

                def with_p(p):
                    ll = [dict(d) for d in lora]
                    A, B = ll[ell][t]
                    ll[ell][t] = (p, B) if which == 0 else (A, p)
                    return ll
                fd = (loss(x, with_p(base + eps * dirp)) - loss(x, with_p(base - eps * dirp))) / (2 * eps)
                an = np.sum(gr[ell][t][which] * dirp)
                assert abs(fd - an) < 1e-6 * max(1.0, abs(fd)), (ell, t, which, fd, an)


def test_opt_zero_b_is_base_and_models_registered():
    cfg = opt_cfg()
    W = base_layer_weights(cfg, 0, seed=51)
    assert "wgate" not in W and {"bq", "bk", "bv", "bo", "bup", "bdown", "b1", "b2"} <= set(W)
    c = ClientCfg(4, 8.0, ("q", "v"), [11])
    x, _ = client_inputs(cfg, c, seed=52)
    y0, _ = O.opt_layer_fwd(x, W, {}, 2.0, cfg)
    y1, _ = O.opt_layer_fwd(x, W, client_adapters(cfg, c, seed=53, zero_b=True)[0], 2.0, cfg)
    np.testing.assert_array_equal(y0, y1)
    m = MODELS["opt1.3b"]
    assert (m.d_model, m.n_heads, m.d_ff, m.total_layers, m.head_dim) == (2048, 32, 8192, 24, 64)


def test_relu_decision_in_kernel_precision_differs_only_where_ambiguous():
    """Reading R25: with relu_mask_bf16 the oracle decides the ReLU mask on bf16 operands (the kernel's precision).
    Pin: the decision agrees with the exact fp64 sign wherever the exact pre-activation is farther from 0 than the
    a-priori bound of the bf16 operand rounding, |z - z_bf16| <= 2^-8 (sum_k |hn_k W_k| + LoRA terms), and flips are
    rare; elsewhere both signs are correct results."""
    cfg = opt_cfg()
    W = base_layer_weights(cfg, 0, seed=61)
    c = ClientCfg(8, 16.0, ("up",), [200])
    lora = client_adapters(cfg, c, seed=62)[0]
    x, _ = client_inputs(cfg, c, seed=63)
    s = c.alpha / c.rank
    _, cache = O.opt_layer_fwd(x.astype(F64), W, lora, s, cfg, F64)
    hn = cache["hn"]
    A, B = (a.astype(F64) for a in lora["up"])
    z = hn @ W["wup"].astype(F64).T + s * (hn @ A.T) @ B.T + W["bup"].astype(F64)
    mask = O.relu_decision(hn, W["wup"], W["bup"], lora["up"], s)
    bound = 2.0 ** -8 * (np.abs(hn) @ np.abs(W["wup"].astype(F64)).T
                         + s * (np.abs(hn) @ np.abs(A).T) @ np.abs(B).T * 2.0) + 1e-6 * np.abs(z)
    flips = mask != (z > 0)
    assert np.all(np.abs(z[flips]) <= bound[flips])
    assert np.all(mask[np.abs(z) > bound] == (z[np.abs(z) > bound] > 0))
    assert flips.mean() < 5e-3


def test_opt_prefix_finite_differences_fp64():
    """Prefix tuning on the OPT layer (R28, no RoPE): finite differences of the prefix grads over 2 layers."""
    import dataclasses
    from workloads import PREFIX
    cfg = dataclasses.replace(MODELS["opt_tiny"], n_layers=2, d_model=32, n_heads=4, n_kv_heads=4, d_ff=48)
    Ws = [base_layer_weights(cfg, l, seed=71) for l in range(2)]
    c = ClientCfg(2, 1.0, (PREFIX,), [5, 3])
    ad = client_adapters(cfg, c, seed=72)
    x, g = client_inputs(cfg, c, seed=73)
    x, g = x.astype(np.float64), g.astype(np.float64)
    _, _, gr = O.client_step(x, g, c.seq_lens, Ws, ad, 1.0, cfg, np.float64)

    def loss(ll):
        return float(np.sum(O.client_step(x, np.zeros_like(g), c.seq_lens, Ws, ll, 1.0, cfg, np.float64)[0] * g))

    r = np.random.default_rng(74)
    for ell in range(2):
        for which in (0, 1):
            base = ad[ell][PREFIX][which]
            dirp = r.standard_normal(base.shape)

            def with_p(pp):
                ll = [dict(d) for d in ad]
                Pk, Pv = ll[ell][PREFIX]
                ll[ell][PREFIX] = (pp, Pv) if which == 0 else (Pk, pp)
                return ll
            fd = (loss(with_p(base + 1e-6 * dirp)) - loss(with_p(base - 1e-6 * dirp))) / 2e-6
            an = np.sum(gr[ell][PREFIX][which] * dirp)
            assert abs(fd - an) < 1e-6 * max(1.0, abs(fd)), (ell, which, fd, an)
