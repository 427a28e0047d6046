"""Pins of the CPU oracle to things other than itself (no GPU needed).

Each pin is external to oracle/: a library (transformers' LlamaDecoderLayer,
torch.autograd, torch SDPA, torch.optim.AdamW), a closed form, an invariant the
paper states, finite differences in float64, or a number the paper prints
(tests/golden/).  A plausible oracle bug (dropped term, wrong sign or index,
transposed operand) fails at least one of them.
"""
import json
import os

import numpy as np
import pytest
import torch

from oracle import menos_oracle as O
from workloads import (ClientCfg, MODELS, ModelCfg, TARGETS, base_layer_weights, bf16_round,
                       client_adapters, client_inputs, target_dims)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
F64 = np.float64


# ------------------------------------------------------------------ helpers
def hf_layer(cfg: ModelCfg, W, lora, s):
    """transformers' LlamaDecoderLayer in fp64 with LoRA merged: W' = W + s B A (textbook identity)."""
    from transformers import LlamaConfig
    from transformers.models.llama.modeling_llama import LlamaDecoderLayer
    c = LlamaConfig(hidden_size=cfg.d_model, intermediate_size=cfg.d_ff, num_attention_heads=cfg.n_heads,
                    num_key_value_heads=cfg.n_kv_heads, rms_norm_eps=cfg.rms_eps, rope_theta=cfg.rope_theta,
                    max_position_embeddings=4096)
    c._attn_implementation = "eager"
    L = LlamaDecoderLayer(c, 0).double()
    mods = {"q": L.self_attn.q_proj, "k": L.self_attn.k_proj, "v": L.self_attn.v_proj,
            "o": L.self_attn.o_proj, "gate": L.mlp.gate_proj, "up": L.mlp.up_proj, "down": L.mlp.down_proj}
    with torch.no_grad():
        for t, m in mods.items():
            m.weight.copy_(torch.from_numpy(W["w" + t].astype(F64)))
        L.input_layernorm.weight.copy_(torch.from_numpy(W["g1"].astype(F64)))
        L.post_attention_layernorm.weight.copy_(torch.from_numpy(W["g2"].astype(F64)))
    for p in L.parameters():
        p.requires_grad_(False)
    # LoRA as a parametrisation W0 + s B A with A, B leaves, so autograd yields dA, dB
    leaves = {}
    for t, (A, B) in lora.items():
        At = torch.from_numpy(A.astype(F64)).requires_grad_(True)
        Bt = torch.from_numpy(B.astype(F64)).requires_grad_(True)
        leaves[t] = (At, Bt)
        m = mods[t]
        W0 = m.weight.detach().clone()
        m.forward = (lambda x, W0=W0, At=At, Bt=Bt: x @ (W0 + s * Bt @ At).T)
    return c, L, leaves


def hf_run(cfg, W, lora, s, x, g):
    from transformers.models.llama.modeling_llama import LlamaRotaryEmbedding
    c, L, leaves = hf_layer(cfg, W, lora, s)
    S = x.shape[0]
    xt = torch.from_numpy(x.astype(F64))[None].requires_grad_(True)
    pos = torch.arange(S)[None]
    cos, sin = LlamaRotaryEmbedding(c)(xt, pos)
    mask = torch.full((S, S), float("-inf"), dtype=torch.float64).triu(1)[None, None]
    y = L(xt, attention_mask=mask, position_ids=pos, position_embeddings=(cos, sin))
    (y * torch.from_numpy(g.astype(F64))[None]).sum().backward()
    grads = {t: (A.grad.numpy(), B.grad.numpy()) for t, (A, B) in leaves.items()}
    return y.detach().numpy()[0], xt.grad.numpy()[0], grads


def small_cfg(H=4, Hkv=4, d=64, f=172, layers=1):
    return ModelCfg("t", d, H, Hkv, f, layers)


def rel(a, b):
    return np.max(np.abs(a - b)) / max(np.max(np.abs(b)), 1e-300)


# ------------------------------------------------------------------ RMSNorm
def test_rmsnorm_closed_form():
    d, c, eps = 64, 0.37, 1e-5
    g = np.linspace(0.5, 1.5, d)
    y, rstd = O.rmsnorm_fwd(np.full((3, d), c), g, eps)
    np.testing.assert_allclose(y, np.broadcast_to(g * c / np.sqrt(c * c + eps), (3, d)), rtol=1e-13)


def test_rmsnorm_vs_hf_autograd():
    from transformers.models.llama.modeling_llama import LlamaRMSNorm
    r = np.random.default_rng(0)
    x = r.standard_normal((5, 48))
    g = 1 + 0.1 * r.standard_normal(48)
    dy = r.standard_normal((5, 48))
    m = LlamaRMSNorm(48, eps=1e-5).double()
    with torch.no_grad():
        m.weight.copy_(torch.from_numpy(g))
    xt = torch.from_numpy(x).requires_grad_(True)
    yt = m(xt)
    (yt * torch.from_numpy(dy)).sum().backward()
    y, rstd = O.rmsnorm_fwd(x, g, 1e-5)
    # HF casts to fp32 inside LlamaRMSNorm even for fp64 modules: tolerance = fp32 rounding
    np.testing.assert_allclose(y, yt.detach().numpy(), rtol=2e-6, atol=1e-7)
    np.testing.assert_allclose(O.rmsnorm_bwd(dy, x, g, rstd), xt.grad.numpy(), rtol=1e-5, atol=1e-6)


# ------------------------------------------------------------------ RoPE
def test_rope_properties():
    S, hd = 40, 16
    cos, sin = O.rope_cos_sin(S, hd, 1e4, F64)
    r = np.random.default_rng(1)
    q = r.standard_normal((S, 2, hd))
    k = r.standard_normal((S, 2, hd))
    qr = O.rope_fwd(q, cos, sin)
    np.testing.assert_allclose(qr[0], q[0], rtol=0, atol=0)                   # position 0 = identity
    np.testing.assert_allclose(np.linalg.norm(qr, axis=-1), np.linalg.norm(q, axis=-1), rtol=1e-6)
    # <R_m q, R_n k> depends only on m - n: same q/k vectors placed at (m, n) and (m+7, n+7)
    qq = np.broadcast_to(q[3], q.shape).copy()
    kk = np.broadcast_to(k[5], k.shape).copy()
    qrr, krr = O.rope_fwd(qq, cos, sin), O.rope_fwd(kk, cos, sin)
    d1 = np.sum(qrr[10] * krr[4], axis=-1)
    d2 = np.sum(qrr[17] * krr[11], axis=-1)
    np.testing.assert_allclose(d1, d2, rtol=1e-5)
    # backward = adjoint (check <R x, y> = <x, R^T y>) and inverse (rotation by -angle)
    y = r.standard_normal(q.shape)
    np.testing.assert_allclose(np.sum(O.rope_fwd(q, cos, sin) * y), np.sum(q * O.rope_bwd(y, cos, sin)), rtol=1e-12)
    np.testing.assert_allclose(O.rope_bwd(O.rope_fwd(q, cos, sin), cos, sin), q, rtol=1e-6, atol=1e-6)


def test_rope_vs_hf():
    from transformers import LlamaConfig
    from transformers.models.llama.modeling_llama import LlamaRotaryEmbedding, apply_rotary_pos_emb
    S, hd = 33, 16
    c = LlamaConfig(hidden_size=64, num_attention_heads=4, rope_theta=1e4, max_position_embeddings=64)
    r = np.random.default_rng(2)
    q = r.standard_normal((S, 4, hd))
    qt = torch.from_numpy(q).transpose(0, 1)[None]  # [1, H, S, hd]
    cos, sin = LlamaRotaryEmbedding(c)(qt, torch.arange(S)[None])
    qe, _ = apply_rotary_pos_emb(qt, qt, cos, sin)
    mc, ms = O.rope_cos_sin(S, hd, 1e4, F64)
    np.testing.assert_allclose(O.rope_fwd(q, mc, ms), qe[0].transpose(0, 1).numpy(), rtol=1e-6, atol=1e-6)


# ------------------------------------------------------------------ attention
@pytest.mark.parametrize("H,Hkv", [(4, 4), (4, 2), (8, 1)])
def test_attention_vs_sdpa(H, Hkv):
    S, hd = 19, 16
    r = np.random.default_rng(3)
    q, k, v = r.standard_normal((S, H, hd)), r.standard_normal((S, Hkv, hd)), r.standard_normal((S, Hkv, hd))
    dO = r.standard_normal((S, H, hd))
    qt, kt, vt = (torch.from_numpy(a).transpose(0, 1)[None].requires_grad_(True) for a in (q, k, v))
    rep = H // Hkv
    ot = torch.nn.functional.scaled_dot_product_attention(
        qt, kt.repeat_interleave(rep, 1), vt.repeat_interleave(rep, 1), is_causal=True)
    (ot * torch.from_numpy(dO).transpose(0, 1)[None]).sum().backward()
    Ob, lse = O.attention_fwd(q, k, v)
    np.testing.assert_allclose(Ob, ot.detach()[0].transpose(0, 1).numpy(), rtol=1e-10, atol=1e-12)
    dq, dk, dv = O.attention_bwd(dO, q, k, v)
    for mine, ref in ((dq, qt), (dk, kt), (dv, vt)):
        np.testing.assert_allclose(mine, ref.grad[0].transpose(0, 1).numpy(), rtol=1e-9, atol=1e-11)
    # lse closed form on row 0: only key 0 visible -> lse = q0.k0/sqrt(hd)
    np.testing.assert_allclose(lse[:, 0], np.sum(q[0] * k[0, np.arange(H) // rep], -1) / 4.0, rtol=1e-12)


def test_attention_special_cases():
    r = np.random.default_rng(4)
    q, k, v = r.standard_normal((1, 2, 8)), r.standard_normal((1, 2, 8)), r.standard_normal((1, 2, 8))
    np.testing.assert_allclose(O.attention_fwd(q, k, v)[0], v, rtol=1e-14)     # S=1: O = v
    S = 9
    q = r.standard_normal((S, 1, 8))
    k = np.broadcast_to(r.standard_normal((1, 1, 8)), (S, 1, 8))                # identical keys
    v = r.standard_normal((S, 1, 8))
    Ob, _ = O.attention_fwd(q, k, v)
    running_mean = np.cumsum(v, axis=0) / np.arange(1, S + 1)[:, None, None]
    np.testing.assert_allclose(Ob, running_mean, rtol=1e-12)


# ------------------------------------------------------------------ SwiGLU
def test_swiglu_special_values_and_hf():
    from transformers import LlamaConfig
    from transformers.models.llama.modeling_llama import LlamaMLP
    assert O.silu(np.array(0.0)) == 0.0
    dgt, dup = O.swiglu_bwd(np.array(1.0), np.array(0.0), np.array(1.0))
    assert dgt == 0.5 and dup == 0.0                                            # silu'(0) = 1/2
    c = LlamaConfig(hidden_size=16, intermediate_size=24, num_attention_heads=2, num_key_value_heads=2)
    m = LlamaMLP(c).double()
    r = np.random.default_rng(5)
    x = r.standard_normal((3, 16))
    wg, wu, wd = (m.gate_proj.weight.detach().numpy(), m.up_proj.weight.detach().numpy(),
                  m.down_proj.weight.detach().numpy())
    ref = m(torch.from_numpy(x)).detach().numpy()
    np.testing.assert_allclose((O.silu(x @ wg.T) * (x @ wu.T)) @ wd.T, ref, rtol=1e-12, atol=1e-14)


# ------------------------------------------------------------------ full decoder layer vs HF
@pytest.mark.parametrize("H,Hkv,targets", [
    (4, 4, ("q", "v")),
    (4, 2, TARGETS),
    (4, 4, ("k", "o", "gate", "up", "down")),
])
def test_layer_vs_hf_fp64(H, Hkv, targets):
    cfg = small_cfg(H, Hkv)
    W = base_layer_weights(cfg, 0, seed=7)
    c = ClientCfg(4, 8.0, targets, [23])
    lora = client_adapters(cfg, c, seed=11)[0]
    x, g = client_inputs(cfg, c, seed=13)
    s = c.alpha / c.rank
    y_hf, dx_hf, gr_hf = hf_run(cfg, W, lora, s, x, g)
    y, cache = O.layer_fwd(x.astype(F64), W, lora, s, cfg, F64)
    dx, gr = O.layer_bwd(g.astype(F64), cache, W, lora, s, cfg, F64)
    # HF computes RMSNorm and cos/sin in fp32 even in an fp64 module -> ~1e-6 agreement
    assert rel(y, y_hf) < 1e-5
    assert rel(dx, dx_hf) < 1e-5
    assert set(gr) == set(targets)
    for t in targets:
        assert rel(gr[t][0], gr_hf[t][0]) < 1e-5, t
        assert rel(gr[t][1], gr_hf[t][1]) < 1e-5, t


# ------------------------------------------------------------------ finite differences (invariant a)
def test_finite_differences_segment_fp64():
    cfg = small_cfg(4, 2, layers=2)
    Ws = [base_layer_weights(cfg, l, seed=21) for l in range(2)]
    c = ClientCfg(4, 8.0, ("q", "v", "down"), [7])
    lora = client_adapters(cfg, c, seed=22)
    x, g = client_inputs(cfg, c, seed=23)
    x, g = x.astype(F64), g.astype(F64)
    s = 2.0
    xs, gs, gr = O.segment_fwd_bwd(x, g, Ws, lora, s, cfg, F64)

    def loss(xx, ll):
        return float(np.sum(O.segment_fwd(xx, Ws, ll, s, cfg, F64) * g))

    r = np.random.default_rng(24)
    eps = 1e-6
    dirx = r.standard_normal(x.shape)
    fd = (loss(x + eps * dirx, lora) - loss(x - eps * dirx, lora)) / (2 * eps)
    assert abs(fd - np.sum(gs * dirx)) < 1e-6 * max(1.0, abs(fd))
    for ell in range(2):
        for t in ("q", "v", "down"):
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


# ------------------------------------------------------------------ invariants (b), (c), (d)
def test_zero_b_gives_base_output_exactly():
    cfg = small_cfg(layers=2)
    Ws = [base_layer_weights(cfg, l, seed=31) for l in range(2)]
    c = ClientCfg(4, 8.0, TARGETS, [12])
    lz = client_adapters(cfg, c, seed=32, zero_b=True)
    x, _ = client_inputs(cfg, c, seed=33)
    with_lora = O.segment_fwd(x, Ws, lz, 2.0, cfg)
    base_only = O.segment_fwd(x, Ws, [{} for _ in range(2)], 2.0, cfg)
    np.testing.assert_array_equal(with_lora, base_only)


def test_batched_equals_alone_and_sequence_independence():
    cfg = small_cfg(layers=1)
    Ws = [base_layer_weights(cfg, 0, seed=41)]
    cs = [ClientCfg(4, 8.0, ("q", "v"), [5, 9]), ClientCfg(8, 16.0, ("q", "v"), [16])]
    ad = [client_adapters(cfg, c, seed=42 + i) for i, c in enumerate(cs)]
    io = [client_inputs(cfg, c, seed=50 + i) for i, c in enumerate(cs)]
    res = O.batched_step([a for a, _ in io], [b for _, b in io], cs, Ws, ad, cfg, F64)
    for i, c in enumerate(cs):
        alone = O.client_step(io[i][0], io[i][1], c.seq_lens, Ws, ad[i], c.alpha / c.rank, cfg, F64)
        np.testing.assert_array_equal(res[i][0], alone[0])
    # sequences are independent: the 2nd sequence of client 0 alone gives the same rows
    xs2, gs2, _ = O.segment_fwd_bwd(io[0][0][5:], io[0][1][5:], Ws, ad[0], 2.0, cfg, F64)
    np.testing.assert_allclose(res[0][0][5:], xs2, rtol=1e-12)
    np.testing.assert_allclose(res[0][1][5:], gs2, rtol=1e-12)


def test_no_base_gradient_and_base_unchanged():
    cfg = small_cfg(layers=1)
    W = base_layer_weights(cfg, 0, seed=61)
    snapshot = {k: v.copy() for k, v in W.items()}
    c = ClientCfg(4, 8.0, ("q", "v"), [6])
    lora = client_adapters(cfg, c, seed=62)[0]
    x, g = client_inputs(cfg, c, seed=63)
    y, cache = O.layer_fwd(x, W, lora, 2.0, cfg)
    dx, gr = O.layer_bwd(g, cache, W, lora, 2.0, cfg)
    assert set(gr) == {"q", "v"}                        # only adapter grads exist
    for t, (dA, dB) in gr.items():
        K, N = target_dims(cfg, t)
        assert dA.shape == (4, K) and dB.shape == (N, 4)
    for k in W:
        np.testing.assert_array_equal(W[k], snapshot[k])


# ------------------------------------------------------------------ AdamW
def test_adamw_vs_torch_and_closed_form():
    r = np.random.default_rng(71)
    p0 = r.standard_normal(50)
    gs = [r.standard_normal(50) for _ in range(4)]
    hp = dict(lr=1e-3, beta1=0.9, beta2=0.999, eps=1e-8, weight_decay=0.01)
    pt = torch.from_numpy(p0.copy()).requires_grad_(True)
    opt = torch.optim.AdamW([pt], lr=hp["lr"], betas=(hp["beta1"], hp["beta2"]), eps=hp["eps"],
                            weight_decay=hp["weight_decay"])
    p, m, v = p0.copy(), np.zeros(50), np.zeros(50)
    for t, g in enumerate(gs, start=1):
        pt.grad = torch.from_numpy(g.copy())
        opt.step()
        p, m, v = O.adamw_step(p, g, m, v, t, **hp)
        if t == 1:
            closed = p0 * (1 - hp["lr"] * hp["weight_decay"]) - hp["lr"] * g / (np.abs(g) + hp["eps"])
            np.testing.assert_allclose(p, closed, rtol=1e-12)
        np.testing.assert_allclose(p, pt.detach().numpy(), rtol=1e-12, atol=1e-15)


# ------------------------------------------------------------------ paper's printed numbers
def _two_point(vanilla_1, menos_n, N):
    """M and A+O from two printed persistent-memory figures: one client alone (vanilla = M + (A+O)) and Menos with N
    clients (M + N (A+O), Eq.3 without I)."""
    AO = (menos_n - vanilla_1) / (N - 1)
    return vanilla_1 - AO, AO


def test_persistent_reduction_pinned_to_printed_figures():
    """PAPER.md:352 (§5.2, Fig.5b): Llama-2-7B, 23.8 GB for the full model (one client), Menos 26.4 GB for 4 clients,
    "72.2% less than duplicating".  PAPER.md:350 (Fig.5a): OPT 4.7 GB -> 18.7 GB for 4 vanilla clients vs Menos 6.7 GB,
    "a 64.1% reduction".  M and A+O are solved from two printed figures; the third printed number (the reduction)
    must then come out of oracle.persistent_reduction, so a wrong formula (e.g. dividing by N*M, forgetting N on A+O)
    fails.  Tolerance: the GB figures are printed to 0.1 GB."""
    with open(os.path.join(GOLDEN, "paper_memory.json")) as fh:
        gold = json.load(fh)
    # Llama-2-7B: one-client figure printed directly
    M, AO = _two_point(23.8, 26.4, 4)
    assert abs(O.persistent_reduction(M, AO, 4) - 0.722) <= 0.001
    assert abs(O.memory_menos(M, AO, 0.0, 0.0, 4) - 26.4) < 1e-9                # Eq.3 with I = 0
    assert abs(O.memory_vanilla(M, AO, 0.0, 0.0, 4) - 4 * 23.8) < 1e-9           # Eq.2 with I = 0
    # OPT: the one-client figure is 18.7 / 4 (printed 4.7)
    Mo, AOo = _two_point(18.7 / 4, 6.7, 4)
    assert abs(18.7 / 4 - 4.7) <= 0.05
    assert abs(O.persistent_reduction(Mo, AOo, 4) - 0.641) <= 0.001
    for row in gold["reductions"]:
        v1 = row["vanilla_gb"] / 4
        m_, ao_ = _two_point(v1, row["menos_gb"], 4)
        assert abs(O.persistent_reduction(m_, ao_, 4) - row["paper_reduction"]) <= row["tol"], row
    # the formula is not symmetric in its arguments: swapping M and A+O must not reproduce the printed number
    assert abs(O.persistent_reduction(AO, M, 4) - 0.722) > 0.05
    # limits: one client saves nothing; N -> inf approaches 1 - (A+O)/(M+A+O)
    assert abs(O.persistent_reduction(M, AO, 1)) < 1e-12
    assert abs(O.persistent_reduction(M, AO, 10 ** 9) - (1 - AO / (M + AO))) < 1e-6


def test_memory_models_against_p105_breakdown():
    """PAPER.md:105 (§2.3): one Llama-2-7B client with batch 4 needs ~28.7 GB = 24 GB (M) + 246 MB (A+O) + 4 GB (I);
    Eq.2 at N = 1 must give that total (the paper leaves a ~0.45 GB residual, its CUDA context,
    cf. PAPER.md:354); Eq.3 keeps one I and one M for any N; base sharing keeps one M."""
    with open(os.path.join(GOLDEN, "paper_memory.json")) as fh:
        b = json.load(fh)["one_client_breakdown"]
    M, AO, I = b["M_gb"], b["AO_gb"], b["I_gb"]
    assert abs(O.memory_vanilla(M, AO, 0.0, I, 1) - b["total_gb"]) <= b["residual_tol_gb"]
    for N in (1, 2, 4, 8):
        # differences between consecutive N isolate the per-client term of each model
        dv = O.memory_vanilla(M, AO, 0.0, I, N + 1) - O.memory_vanilla(M, AO, 0.0, I, N)
        ds = O.memory_shared_base(M, AO, 0.0, I, N + 1) - O.memory_shared_base(M, AO, 0.0, I, N)
        dm = O.memory_menos(M, AO, 0.0, I, N + 1) - O.memory_menos(M, AO, 0.0, I, N)
        assert abs(dv - (M + AO + I)) < 1e-9 and abs(ds - (AO + I)) < 1e-9 and abs(dm - AO) < 1e-9
    assert O.memory_menos(M, AO, 0.0, I, 1) == O.memory_vanilla(M, AO, 0.0, I, 1)


# ------------------------------------------------------------------ client_step over several sequences
def test_finite_differences_client_with_several_sequences_fp64():
    """client_step sums each adapter's gradient over ALL of a client's sequences (reading R10) and returns g_s for
    every token: finite differences of L = sum(G * x_s) over the whole client (3 ragged sequences, positions
    restarting at 0 in each) against the analytic gradients.  Keeping only one sequence's gradient, or mixing
    sequences, fails."""
    import dataclasses
    cfg = dataclasses.replace(MODELS["tiny"], n_layers=2, n_kv_heads=2, d_model=32, n_heads=4, d_ff=48)
    Ws = [base_layer_weights(cfg, l, seed=81) for l in range(2)]
    c = ClientCfg(4, 8.0, ("q", "v", "o", "down"), [5, 1, 7])
    lora = client_adapters(cfg, c, seed=82)
    x, g = client_inputs(cfg, c, seed=83)
    x, g = x.astype(F64), g.astype(F64)
    s = c.alpha / c.rank
    xs, gs, gr = O.client_step(x, g, c.seq_lens, Ws, lora, s, cfg, F64)

    def loss(xx, ll):
        return float(np.sum(O.client_step(xx, np.zeros_like(g), c.seq_lens, Ws, ll, s, cfg, F64)[0] * g))

    r = np.random.default_rng(84)
    eps = 1e-6
    dirx = r.standard_normal(x.shape)
    fd = (loss(x + eps * dirx, lora) - loss(x - eps * dirx, lora)) / (2 * eps)
    assert abs(fd - np.sum(gs * dirx)) < 1e-6 * max(1.0, abs(fd))
    for ell in range(2):
        for t in c.targets:
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
    # and the sum really spans the sequences: each sequence alone gives a different, partial gradient
    off = 0
    parts = []
    for S in c.seq_lens:
        parts.append(O.segment_fwd_bwd(x[off:off + S], g[off:off + S], Ws, lora, s, cfg, F64)[2])
        off += S
    for ell in range(2):
        for t in c.targets:
            tot = sum(p[ell][t][0] for p in parts)
            np.testing.assert_allclose(gr[ell][t][0], tot, rtol=1e-10, atol=1e-14)
            assert np.linalg.norm(parts[-1][ell][t][0] - gr[ell][t][0]) > 1e-3 * np.linalg.norm(gr[ell][t][0])


def test_segment_composes_at_a_cut():
    """NEXT-3: a client with cut k runs the oracle's segment [k, L).  Pin the meaning of x_c / g_s at
    a cut by composition: f_[0,L) = f_[k,L) o f_[0,k), and g_s of [0,L) equals g_s of [0,k) driven by the g_s that
    [k,L) returns (chain rule); the adapter grads of layers >= k are those of the shorter segment (fp64)."""
    import dataclasses
    m = dataclasses.replace(MODELS["tiny"], n_layers=3, n_kv_heads=2)
    c = ClientCfg(4, 8.0, ("q", "v", "down"), [9, 5])
    W = [base_layer_weights(m, l, seed=21) for l in range(3)]
    ad = client_adapters(m, c, seed=22)
    x, g = client_inputs(m, c, seed=23)
    s = c.alpha / c.rank
    xs, gs, gr = O.client_step(x, g, c.seq_lens, W, ad, s, m, F64)
    k = 1
    mid, gmid, grk = O.client_step(x, np.zeros_like(x), c.seq_lens, W[:k], ad[:k], s, m.with_layers(k), F64)
    xs2, gk, gr2 = O.client_step(mid, g, c.seq_lens, W[k:], ad[k:], s, m.with_layers(3 - k), F64)
    _, gs2, gr1 = O.client_step(x, gk, c.seq_lens, W[:k], ad[:k], s, m.with_layers(k), F64)
    np.testing.assert_allclose(xs2, xs, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(gs2, gs, rtol=1e-10, atol=1e-12)
    for l in range(3 - k):
        for t in c.targets:
            np.testing.assert_allclose(gr2[l][t][0], gr[k + l][t][0], rtol=1e-10, atol=1e-13)
            np.testing.assert_allclose(gr2[l][t][1], gr[k + l][t][1], rtol=1e-10, atol=1e-13)


# ------------------------------------------------------------------ prefix tuning (NEXT-3, reading R28)
def _sdpa_prefix(q, k, v, pk, pv):
    """torch SDPA (fp64) over [prefix | sequence] keys with an explicit mask: prefix always visible, causal inside the
    sequence; GQA by repeating kv heads (HF repeat_kv)."""
    S, H, hd = q.shape
    P, Hkv = pk.shape[0], k.shape[1]
    rep = H // Hkv
    qt = q.permute(1, 0, 2)[None]
    kk = torch.cat([pk, k]).repeat_interleave(rep, dim=1).permute(1, 0, 2)[None]
    vv = torch.cat([pv, v]).repeat_interleave(rep, dim=1).permute(1, 0, 2)[None]
    mask = torch.cat([torch.ones(S, P, dtype=torch.bool), torch.tril(torch.ones(S, S, dtype=torch.bool))], dim=1)
    return torch.nn.functional.scaled_dot_product_attention(qt, kk, vv, attn_mask=mask)[0].permute(1, 0, 2)


@pytest.mark.parametrize("H,Hkv,P", [(4, 4, 3), (4, 2, 5), (2, 1, 1)])
def test_prefix_attention_vs_sdpa_autograd_fp64(H, Hkv, P):
    r = np.random.default_rng(91)
    S, hd = 9, 16
    q, k, v = (r.standard_normal((S, n, hd)) for n in (H, Hkv, Hkv))
    pk, pv = r.standard_normal((P, Hkv, hd)), r.standard_normal((P, Hkv, hd))
    dO = r.standard_normal((S, H, hd))
    O_, lse = O.attention_prefix_fwd(q, k, v, pk, pv)
    ts = [torch.from_numpy(a).requires_grad_(True) for a in (q, k, v, pk, pv)]
    ref = _sdpa_prefix(*ts)
    np.testing.assert_allclose(O_, ref.detach().numpy(), rtol=1e-10, atol=1e-12)
    ref.backward(torch.from_numpy(dO))
    got = O.attention_prefix_bwd(dO, q, k, v, pk, pv)
    for g, t in zip(got, ts):
        np.testing.assert_allclose(g, t.grad.numpy(), rtol=1e-9, atol=1e-11)
    # lse closed form at row 0: log(sum_j<P exp(s_0j) + exp(s_00)) per head
    sc = 1.0 / np.sqrt(hd)
    for h in range(H):
        kv = h // (H // Hkv)
        s0 = np.concatenate([pk[:, kv] @ q[0, h], [k[0, kv] @ q[0, h]]]) * sc
        assert abs(lse[h, 0] - np.log(np.sum(np.exp(s0)))) < 1e-12


def test_prefix_attention_reduces_to_causal_without_prefix():
    r = np.random.default_rng(92)
    q, k, v = (r.standard_normal((7, n, 8)) for n in (4, 2, 2))
    empty = np.zeros((0, 2, 8))
    a, la = O.attention_prefix_fwd(q, k, v, empty, empty)
    b, lb = O.attention_fwd(q, k, v)
    np.testing.assert_allclose(a, b, rtol=1e-13)
    np.testing.assert_allclose(la, lb, rtol=1e-13)
    dO = r.standard_normal(q.shape)
    for x, y in zip(O.attention_prefix_bwd(dO, q, k, v, empty, empty)[:3], O.attention_bwd(dO, q, k, v)):
        np.testing.assert_allclose(x, y, rtol=1e-12, atol=1e-14)


def test_prefix_finite_differences_client_fp64():
    """dL/dPk, dL/dPv of a prefix-tuning client over 2 layers and 2 sequences (summed over the client's tokens) by
    central differences of L = sum(G * x_s)."""
    import dataclasses
    from workloads import PREFIX
    cfg = dataclasses.replace(MODELS["tiny"], n_layers=2, n_kv_heads=2, d_model=32, n_heads=4, d_ff=48)
    Ws = [base_layer_weights(cfg, l, seed=93) for l in range(2)]
    c = ClientCfg(3, 1.0, (PREFIX,), [6, 4])
    ad = client_adapters(cfg, c, seed=94)
    x, g = client_inputs(cfg, c, seed=95)
    x, g = x.astype(F64), g.astype(F64)
    xs, gs, gr = O.client_step(x, g, c.seq_lens, Ws, ad, 1.0, cfg, F64)

    def loss(ll):
        return float(np.sum(O.client_step(x, np.zeros_like(g), c.seq_lens, Ws, ll, 1.0, cfg, F64)[0] * g))

    r = np.random.default_rng(96)
    eps = 1e-6
    for ell in range(2):
        for which in (0, 1):
            base = ad[ell][PREFIX][which]
            dirp = r.standard_normal(base.shape)

            def with_p(pp):
                ll = [dict(d) for d in ad]
                Pk, Pv = ll[ell][PREFIX]
                ll[ell][PREFIX] = (pp, Pv) if which == 0 else (Pk, pp)
                return ll
            fd = (loss(with_p(base + eps * dirp)) - loss(with_p(base - eps * dirp))) / (2 * eps)
            an = np.sum(gr[ell][PREFIX][which] * dirp)
            assert abs(fd - an) < 1e-6 * max(1.0, abs(fd)), (ell, which, fd, an)
