"""Menos server-segment oracle: plain, slow, obviously-correct CPU reference.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this module.  The product path
(paper_conf_middleware_hul24_b200 + libmenos.so) never imports it and shares no
code with it: no kernels, helpers, tables or constants.

What it computes (DESIGN.md §"Readings" lists every reading):

* The server segment f_s of split fine-tuning: x_s = f_s(x_c; theta_s, phi_s) and
  g_s = dL/dx_c given g_c = dL/dx_s  (§2.2, Fig.1).
* theta_s (the base) is read-only; only the adapters phi_s receive gradients
  (§2.1 Eq.1; §3.1).  No base gradient is ever formed.
* phi_s is LoRA on chosen projections, y += (alpha/r) (x A^T) B^T
  (§2.1; §5.1: q,v, r=8, alpha=16, config from PEFT [19]).
* The server holds decoder layers 2..L of Llama 2; the decoder
  layer itself is Llama-2's (PAPER.md:292 cites [32]; conventions readings R1-R5).
* Alg.1 lines 10-12: forward with gradient preparation,
  backward from g_c to g_s, then optimize phi_s (AdamW, reading R7).
* A batched multi-client call is DEFINED as the concatenation of per-client,
  per-sequence calls: Menos "only distributes computation while maintaining the
  same logical flow".

Precision: every function takes a dtype (np.float32 default, np.float64 for the
finite-difference pins).  Inputs are the same bf16-representable values the GPU
receives.  Library primitives used as steps: matmul, exp, sqrt, cos/sin.
"""
from __future__ import annotations

import numpy as np

TARGETS = ("q", "k", "v", "o", "gate", "up", "down")


# ============================================================ RMSNorm (reading R1)
def rmsnorm_fwd(x, g, eps):
    """y = x * rstd * g, rstd = 1/sqrt(mean(x^2) + eps), mean over the last axis."""
    rstd = 1.0 / np.sqrt(np.mean(x * x, axis=-1, keepdims=True) + eps)
    return x * rstd * g, rstd


def rmsnorm_bwd(dy, x, g, rstd):
    """d/dx of y = x*rstd*g:  rstd*(gh - xh*mean(gh*xh)),  gh = dy*g, xh = x*rstd."""
    gh = dy * g
    xh = x * rstd
    return rstd * (gh - xh * np.mean(gh * xh, axis=-1, keepdims=True))


# ============================================================ RoPE (reading R2)
def rope_cos_sin(S, hd, theta, dtype):
    """cos/sin [S, hd] with HF's rotate_half convention: emb = cat(freqs, freqs),
    freqs[p, i] = p * theta^(-2i/hd), computed in fp32 as HF does (angle fp32)."""
    inv_freq = (1.0 / (np.float32(theta) ** (np.arange(0, hd, 2, dtype=np.float32) / np.float32(hd))))
    inv_freq = inv_freq.astype(np.float32)
    pos = np.arange(S, dtype=np.float32)
    freqs = (pos[:, None] * inv_freq[None, :]).astype(np.float32)
    emb = np.concatenate([freqs, freqs], axis=-1)
    return np.cos(emb.astype(np.float64)).astype(dtype), np.sin(emb.astype(np.float64)).astype(dtype)


def rotate_half(x):
    h = x.shape[-1] // 2
    return np.concatenate([-x[..., h:], x[..., :h]], axis=-1)


def rotate_half_T(x):
    """Transpose of rotate_half (it is orthogonal, so this is its inverse)."""
    h = x.shape[-1] // 2
    return np.concatenate([x[..., h:], -x[..., :h]], axis=-1)


def rope_fwd(x, cos, sin):
    """x [S, nh, hd] -> x*cos + rotate_half(x)*sin (positions = row index)."""
    return x * cos[:, None, :] + rotate_half(x) * sin[:, None, :]


def rope_bwd(dy, cos, sin):
    """Adjoint of rope_fwd: dx = dy*cos + rotate_half^T(dy*sin)."""
    return dy * cos[:, None, :] + rotate_half_T(dy * sin[:, None, :])


# ============================================================ causal attention (reading R3)
def attention_fwd(q, k, v):
    """q [S,H,hd], k/v [S,Hkv,hd].  O[i] = softmax_j<=i(q_i.k_j/sqrt(hd)) v_j per head;
    GQA: head h uses kv head h // (H/Hkv) (HF repeat_kv).  Returns O [S,H,hd], lse [H,S]."""
    S, H, hd = q.shape
    rep = H // k.shape[1]
    scale = 1.0 / np.sqrt(hd)
    O = np.zeros_like(q)
    lse = np.zeros((H, S), dtype=q.dtype)
    mask = np.triu(np.ones((S, S), dtype=bool), 1)
    for h in range(H):
        kh, vh = k[:, h // rep, :], v[:, h // rep, :]
        s = (q[:, h, :] @ kh.T) * scale
        s = np.where(mask, -np.inf, s)
        m = np.max(s, axis=-1, keepdims=True)
        e = np.exp(s - m)
        z = np.sum(e, axis=-1, keepdims=True)
        O[:, h, :] = (e / z) @ vh
        lse[h] = (m + np.log(z))[:, 0]
    return O, lse


def attention_bwd(dO, q, k, v):
    """Textbook softmax-attention backward (P recomputed):
    dV = P^T dO; dP = dO V^T; dS = P*(dP - rowsum(P*dP)); dq = dS k/sqrt(hd); dk = dS^T q/sqrt(hd).
    GQA: kv-head gradients sum over the heads of their group."""
    S, H, hd = q.shape
    rep = H // k.shape[1]
    scale = 1.0 / np.sqrt(hd)
    dq = np.zeros_like(q)
    dk = np.zeros_like(k)
    dv = np.zeros_like(v)
    mask = np.triu(np.ones((S, S), dtype=bool), 1)
    for h in range(H):
        kh, vh = k[:, h // rep, :], v[:, h // rep, :]
        s = (q[:, h, :] @ kh.T) * scale
        s = np.where(mask, -np.inf, s)
        e = np.exp(s - np.max(s, axis=-1, keepdims=True))
        P = e / np.sum(e, axis=-1, keepdims=True)
        dv[:, h // rep, :] += P.T @ dO[:, h, :]
        dP = dO[:, h, :] @ vh.T
        dS = P * (dP - np.sum(P * dP, axis=-1, keepdims=True))
        dq[:, h, :] = (dS @ kh) * scale
        dk[:, h // rep, :] += (dS.T @ q[:, h, :]) * scale
    return dq, dk, dv


# ============================================================ prefix-tuning attention (NEXT-3; reading R28)
def attention_prefix_fwd(q, k, v, pk, pv):
    """Prefix tuning (§2.1, Li & Liang [16]; a client may pick it instead of LoRA): the layer
    holds P learned key/value vectors per KV head, pk/pv [P, Hkv, hd], which every query of the sequence attends to
    in addition to its causal keys -- one softmax over [prefix | causal keys], scale hd^-1/2 (reading R28: prefix
    keys are used as given, no RoPE; the sequence keeps positions 0..S-1).  Returns O [S,H,hd], lse [H,S]."""
    S, H, hd = q.shape
    P = pk.shape[0]
    rep = H // k.shape[1]
    scale = 1.0 / np.sqrt(hd)
    O = np.zeros_like(q)
    lse = np.zeros((H, S), dtype=q.dtype)
    mask = np.concatenate([np.zeros((S, P), dtype=bool), np.triu(np.ones((S, S), dtype=bool), 1)], axis=1)
    for h in range(H):
        kh = np.concatenate([pk[:, h // rep, :], k[:, h // rep, :]])
        vh = np.concatenate([pv[:, h // rep, :], v[:, h // rep, :]])
        s = (q[:, h, :] @ kh.T) * scale
        s = np.where(mask, -np.inf, s)
        m = np.max(s, axis=-1, keepdims=True)
        e = np.exp(s - m)
        z = np.sum(e, axis=-1, keepdims=True)
        O[:, h, :] = (e / z) @ vh
        lse[h] = (m + np.log(z))[:, 0]
    return O, lse


def attention_prefix_bwd(dO, q, k, v, pk, pv):
    """Backward of attention_prefix_fwd (same textbook softmax backward over the concatenated keys):
    returns dq, dk, dv, dpk, dpv (GQA: kv-head and prefix gradients sum over the heads of their group)."""
    S, H, hd = q.shape
    P = pk.shape[0]
    rep = H // k.shape[1]
    scale = 1.0 / np.sqrt(hd)
    dq, dk, dv = np.zeros_like(q), np.zeros_like(k), np.zeros_like(v)
    dpk, dpv = np.zeros_like(pk), np.zeros_like(pv)
    mask = np.concatenate([np.zeros((S, P), dtype=bool), np.triu(np.ones((S, S), dtype=bool), 1)], axis=1)
    for h in range(H):
        kv = h // rep
        kh = np.concatenate([pk[:, kv, :], k[:, kv, :]])
        vh = np.concatenate([pv[:, kv, :], v[:, kv, :]])
        s = (q[:, h, :] @ kh.T) * scale
        s = np.where(mask, -np.inf, s)
        e = np.exp(s - np.max(s, axis=-1, keepdims=True))
        Pm = e / np.sum(e, axis=-1, keepdims=True)
        dvh = Pm.T @ dO[:, h, :]
        dP = dO[:, h, :] @ vh.T
        dS = Pm * (dP - np.sum(Pm * dP, axis=-1, keepdims=True))
        dq[:, h, :] = (dS @ kh) * scale
        dkh = (dS.T @ q[:, h, :]) * scale
        dpk[:, kv, :] += dkh[:P]
        dk[:, kv, :] += dkh[P:]
        dpv[:, kv, :] += dvh[:P]
        dv[:, kv, :] += dvh[P:]
    return dq, dk, dv, dpk, dpv


# ============================================================ SwiGLU (reading R4)
def sigmoid(x):
    return 1.0 / (1.0 + np.exp(-x))


def silu(x):
    return x * sigmoid(x)


def swiglu_bwd(da, gt, up):
    """a = silu(gt)*up  ->  (dgt, dup)."""
    sg = sigmoid(gt)
    dgt = da * up * sg * (1.0 + gt * (1.0 - sg))
    dup = da * gt * sg
    return dgt, dup


# ============================================================ LoRA projection
def proj_fwd(x, W, lora, s):
    """y = x W^T (+ s (x A^T) B^T).  Returns y and U = x A^T (None without LoRA)."""
    y = x @ W.T
    if lora is None:
        return y, None
    A, B = lora
    U = x @ A.T
    return y + s * (U @ B.T), U


def proj_bwd(dy, x, W, lora, s, U):
    """Given dy = dL/dy: dx = dy W (+ s (dy B) A); dA = s (dy B)^T x; dB = s dy^T U.
    No gradient w.r.t. W is formed (base read-only)."""
    dx = dy @ W
    if lora is None:
        return dx, None
    A, B = lora
    dU = s * (dy @ B)
    dx = dx + dU @ A
    dA = dU.T @ x
    dB = s * (dy.T @ U)
    return dx, (dA, dB)


# ============================================================ one decoder layer
def _cast(a, dtype):
    return np.asarray(a, dtype=dtype)


def layer_fwd(x, W, lora, s, cfg, dtype=np.float32):
    """One Llama-2 decoder layer on ONE sequence x [S, d] (positions 0..S-1), steps
    in SURVEY.md §8(c) order:  xn = rms(x) g1;  q,k,v (+LoRA);  RoPE(q,k);
    O = causal attn;  h = x + O Wo^T (+LoRA);  hn = rms(h) g2;
    a = silu(gate) * up;  y = h + a Wd^T (+LoRA)."""
    S, d = x.shape
    H, Hkv, hd = cfg.n_heads, cfg.n_kv_heads, cfg.head_dim
    Wd = {k: _cast(v, dtype) for k, v in W.items()}
    L = {t: (_cast(a, dtype), _cast(b, dtype)) for t, (a, b) in lora.items()}
    c = {"x": x}
    xn, c["rstd1"] = rmsnorm_fwd(x, Wd["g1"], dtype(cfg.rms_eps))
    c["xn"] = xn
    U = {}
    qp, U["q"] = proj_fwd(xn, Wd["wq"], L.get("q"), s)
    kp, U["k"] = proj_fwd(xn, Wd["wk"], L.get("k"), s)
    vp, U["v"] = proj_fwd(xn, Wd["wv"], L.get("v"), s)
    cos, sin = rope_cos_sin(S, hd, cfg.rope_theta, dtype)
    c["cos"], c["sin"] = cos, sin
    q = rope_fwd(qp.reshape(S, H, hd), cos, sin)
    k = rope_fwd(kp.reshape(S, Hkv, hd), cos, sin)
    v = vp.reshape(S, Hkv, hd)
    if "prefix" in L:   # prefix-tuning client (NEXT-3): the layer's learned prefix keys / values join the attention
        pk, pv = (a.reshape(-1, Hkv, hd) for a in L["prefix"])
        O, c["lse"] = attention_prefix_fwd(q, k, v, pk, pv)
    else:
        O, c["lse"] = attention_fwd(q, k, v)
    c["q"], c["k"], c["v"] = q, k, v
    Of = O.reshape(S, H * hd)
    c["O"] = Of
    ao, U["o"] = proj_fwd(Of, Wd["wo"], L.get("o"), s)
    h = x + ao
    c["h"] = h
    hn, c["rstd2"] = rmsnorm_fwd(h, Wd["g2"], dtype(cfg.rms_eps))
    c["hn"] = hn
    gt, U["gate"] = proj_fwd(hn, Wd["wgate"], L.get("gate"), s)
    up, U["up"] = proj_fwd(hn, Wd["wup"], L.get("up"), s)
    c["gt"], c["up"] = gt, up
    a = silu(gt) * up
    c["a"] = a
    md, U["down"] = proj_fwd(a, Wd["wdown"], L.get("down"), s)
    y = h + md
    c["U"] = U
    return y, c


def layer_bwd(dy, c, W, lora, s, cfg, dtype=np.float32):
    """Backward of layer_fwd, in exact reverse order.
    Returns dx and {target: (dA, dB)}; never a base-weight gradient."""
    S = dy.shape[0]
    H, Hkv, hd = cfg.n_heads, cfg.n_kv_heads, cfg.head_dim
    Wd = {k: _cast(v, dtype) for k, v in W.items()}
    L = {t: (_cast(a, dtype), _cast(b, dtype)) for t, (a, b) in lora.items()}
    U = c["U"]
    grads = {}
    # A8: y = h + a Wd^T  (residual: dh = dy)
    da, gd = proj_bwd(dy, c["a"], Wd["wdown"], L.get("down"), s, U["down"])
    if gd is not None:
        grads["down"] = gd
    dgt, dup = swiglu_bwd(da, c["gt"], c["up"])
    # A9: gate/up projections of hn, then RMSNorm2 backward + residual
    dhn_g, gg = proj_bwd(dgt, c["hn"], Wd["wgate"], L.get("gate"), s, U["gate"])
    dhn_u, gu = proj_bwd(dup, c["hn"], Wd["wup"], L.get("up"), s, U["up"])
    if gg is not None:
        grads["gate"] = gg
    if gu is not None:
        grads["up"] = gu
    dh = dy + rmsnorm_bwd(dhn_g + dhn_u, c["h"], Wd["g2"], c["rstd2"])
    # A10: h = x + O Wo^T
    dO, go = proj_bwd(dh, c["O"], Wd["wo"], L.get("o"), s, U["o"])
    if go is not None:
        grads["o"] = go
    # A11: attention backward, then RoPE backward
    if "prefix" in L:
        pk, pv = (a.reshape(-1, Hkv, hd) for a in L["prefix"])
        dq, dk, dv, dpk, dpv = attention_prefix_bwd(dO.reshape(S, H, hd), c["q"], c["k"], c["v"], pk, pv)
        grads["prefix"] = (dpk.reshape(pk.shape[0], -1), dpv.reshape(pv.shape[0], -1))
    else:
        dq, dk, dv = attention_bwd(dO.reshape(S, H, hd), c["q"], c["k"], c["v"])
    dqp = rope_bwd(dq, c["cos"], c["sin"]).reshape(S, H * hd)
    dkp = rope_bwd(dk, c["cos"], c["sin"]).reshape(S, Hkv * hd)
    dvp = dv.reshape(S, Hkv * hd)
    # A12: q,k,v projections of xn, then RMSNorm1 backward + residual
    dxn = np.zeros_like(c["xn"])
    for t, dt in (("q", dqp), ("k", dkp), ("v", dvp)):
        dxt, gt_ = proj_bwd(dt, c["xn"], Wd["w" + t], L.get(t), s, U[t])
        dxn = dxn + dxt
        if gt_ is not None:
            grads[t] = gt_
    dx = dh + rmsnorm_bwd(dxn, c["x"], Wd["g1"], c["rstd1"])
    return dx, grads


# ============================================================ OPT decoder layer (NEXT-4)
# OPT-1.3B and up: pre-LayerNorm (do_layer_norm_before), biases on every projection, ReLU MLP, learned positions
# added by the client's embedding layer (so no positional term in the server segment).  Reading R23.
def layernorm_fwd(x, g, b, eps):
    """y = (x - mu) rstd g + b, mu = mean(x), rstd = 1/sqrt(var(x) + eps) (biased variance), last axis."""
    mu = np.mean(x, axis=-1, keepdims=True)
    xc = x - mu
    rstd = 1.0 / np.sqrt(np.mean(xc * xc, axis=-1, keepdims=True) + eps)
    return xc * rstd * g + b, rstd


def layernorm_bwd(dy, x, g, rstd):
    """dx of layernorm_fwd (g, b frozen): xh = (x - mu) rstd, gh = dy g,
    dx = rstd (gh - mean(gh) - xh mean(gh xh))."""
    xh = (x - np.mean(x, axis=-1, keepdims=True)) * rstd
    gh = dy * g
    return rstd * (gh - np.mean(gh, axis=-1, keepdims=True) - xh * np.mean(gh * xh, axis=-1, keepdims=True))


def _bf16(a):
    """Round to the nearest bf16 (ties to even), returned as float32: the kernel's GEMM-operand precision."""
    u = np.ascontiguousarray(a, dtype=np.float32).view(np.uint32)
    u = (u + (np.uint32(0x7FFF) + ((u >> 16) & np.uint32(1)))) & np.uint32(0xFFFF0000)
    return u.view(np.float32)


def relu_decision(hn, Wup, bup, lora, s):
    """Reading R25: the ReLU mask is a decision taken by floating point, so the oracle takes it in the
    kernel's precision for that op -- bf16 GEMM operands (hn, and the LoRA shrink output U), fp32 accumulation, fp32
    bias -- instead of on its own fp32 pre-activation (which differs by bf16 rounding and would flip the sign of
    near-zero entries).  Returns the boolean mask [S, f]."""
    hb = _bf16(hn)
    z = hb @ np.asarray(Wup, np.float32).T
    if lora is not None:
        A, B = lora
        z = z + _bf16(np.float32(s) * (hb @ np.asarray(A, np.float32).T)) @ np.asarray(B, np.float32).T
    return (z + np.asarray(bup, np.float32)) > 0


def opt_layer_fwd(x, W, lora, s, cfg, dtype=np.float32, relu_mask_bf16=False):
    """One OPT decoder layer on ONE sequence x [S, d]:  xn = LN1(x);  q,k,v = xn W^T + b (+LoRA);
    O = causal attn (scale hd^-1/2);  h = x + O Wo^T + bo (+LoRA);  hn = LN2(h);
    a = relu(hn W1^T + b1 (+LoRA up));  y = h + a W2^T + b2 (+LoRA down)."""
    S, d = x.shape
    H, hd = cfg.n_heads, cfg.head_dim
    Wd = {k: _cast(v, dtype) for k, v in W.items()}
    L = {t: (_cast(a, dtype), _cast(b, dtype)) for t, (a, b) in lora.items()}
    c = {"x": x}
    eps = dtype(cfg.rms_eps)
    xn, c["rstd1"] = layernorm_fwd(x, Wd["g1"], Wd["b1"], eps)
    c["xn"] = xn
    U = {}
    qp, U["q"] = proj_fwd(xn, Wd["wq"], L.get("q"), s)
    kp, U["k"] = proj_fwd(xn, Wd["wk"], L.get("k"), s)
    vp, U["v"] = proj_fwd(xn, Wd["wv"], L.get("v"), s)
    q = (qp + Wd["bq"]).reshape(S, H, hd)
    k = (kp + Wd["bk"]).reshape(S, H, hd)
    v = (vp + Wd["bv"]).reshape(S, H, hd)
    if "prefix" in L:   # prefix tuning (NEXT-3, R28): no RoPE in OPT, so exactly as for Llama minus the rotation
        pk, pv = (a.reshape(-1, H, hd) for a in L["prefix"])
        O, c["lse"] = attention_prefix_fwd(q, k, v, pk, pv)
    else:
        O, c["lse"] = attention_fwd(q, k, v)
    c["q"], c["k"], c["v"] = q, k, v
    Of = O.reshape(S, H * hd)
    c["O"] = Of
    ao, U["o"] = proj_fwd(Of, Wd["wo"], L.get("o"), s)
    h = x + ao + Wd["bo"]
    c["h"] = h
    hn, c["rstd2"] = layernorm_fwd(h, Wd["g2"], Wd["b2"], eps)
    c["hn"] = hn
    z, U["up"] = proj_fwd(hn, Wd["wup"], L.get("up"), s)
    if relu_mask_bf16:
        c["mask"] = relu_decision(hn, W["wup"], W["bup"], lora.get("up"), s)
        a = (z + Wd["bup"]) * c["mask"]
    else:
        a = np.maximum(z + Wd["bup"], 0)
        c["mask"] = a > 0
    c["a"] = a
    md, U["down"] = proj_fwd(a, Wd["wdown"], L.get("down"), s)
    y = h + md + Wd["bdown"]
    c["U"] = U
    return y, c


def opt_layer_bwd(dy, c, W, lora, s, cfg, dtype=np.float32):
    """Backward of opt_layer_fwd in exact reverse order; dx and {target: (dA, dB)}, no base or bias gradient."""
    S = dy.shape[0]
    H, hd = cfg.n_heads, cfg.head_dim
    Wd = {k: _cast(v, dtype) for k, v in W.items()}
    L = {t: (_cast(a, dtype), _cast(b, dtype)) for t, (a, b) in lora.items()}
    U = c["U"]
    grads = {}
    da, gd = proj_bwd(dy, c["a"], Wd["wdown"], L.get("down"), s, U["down"])
    if gd is not None:
        grads["down"] = gd
    dz = da * c["mask"]
    dhn, gu = proj_bwd(dz, c["hn"], Wd["wup"], L.get("up"), s, U["up"])
    if gu is not None:
        grads["up"] = gu
    dh = dy + layernorm_bwd(dhn, c["h"], Wd["g2"], c["rstd2"])
    dO, go = proj_bwd(dh, c["O"], Wd["wo"], L.get("o"), s, U["o"])
    if go is not None:
        grads["o"] = go
    if "prefix" in L:
        pk, pv = (a.reshape(-1, H, hd) for a in L["prefix"])
        dq, dk, dv, dpk, dpv = attention_prefix_bwd(dO.reshape(S, H, hd), c["q"], c["k"], c["v"], pk, pv)
        grads["prefix"] = (dpk.reshape(pk.shape[0], -1), dpv.reshape(pv.shape[0], -1))
    else:
        dq, dk, dv = attention_bwd(dO.reshape(S, H, hd), c["q"], c["k"], c["v"])
    dxn = np.zeros_like(c["xn"])
    for t, dt in (("q", dq), ("k", dk), ("v", dv)):
        dxt, gt_ = proj_bwd(dt.reshape(S, H * hd), c["xn"], Wd["w" + t], L.get(t), s, U[t])
        dxn = dxn + dxt
        if gt_ is not None:
            grads[t] = gt_
    dx = dh + layernorm_bwd(dxn, c["x"], Wd["g1"], c["rstd1"])
    return dx, grads


def _layer_fns(cfg, relu_mask_bf16=False):
    if getattr(cfg, "arch", "llama") == "opt":
        return (lambda *a, **k: opt_layer_fwd(*a, **k, relu_mask_bf16=relu_mask_bf16)), opt_layer_bwd
    return layer_fwd, layer_bwd


# ============================================================ server segment
def segment_fwd_bwd(x_c, g_c, weights, adapters, s, cfg, dtype=np.float32, relu_mask_bf16=False):
    """One client's ONE sequence through all server layers: forward from x_c, then
    backward from g_c (Alg.1 L10-11).
    weights: list over layers of base dicts; adapters: list over layers of {t: (A,B)}.
    Returns x_s, g_s, grads (list over layers of {t: (dA, dB)})."""
    fwd, bwd = _layer_fns(cfg, relu_mask_bf16)
    x = np.asarray(x_c, dtype=dtype)
    caches = []
    for ell in range(cfg.n_layers):
        x, cache = fwd(x, weights[ell], adapters[ell], dtype(s), cfg, dtype)
        caches.append(cache)
    x_s = x
    dy = np.asarray(g_c, dtype=dtype)
    grads = [None] * cfg.n_layers
    for ell in reversed(range(cfg.n_layers)):
        dy, grads[ell] = bwd(dy, caches[ell], weights[ell], adapters[ell], dtype(s), cfg, dtype)
    return x_s, dy, grads


def segment_fwd(x_c, weights, adapters, s, cfg, dtype=np.float32):
    fwd, _ = _layer_fns(cfg)
    x = np.asarray(x_c, dtype=dtype)
    for ell in range(cfg.n_layers):
        x, _ = fwd(x, weights[ell], adapters[ell], dtype(s), cfg, dtype)
    return x


def client_step(x_c, g_c, seq_lens, weights, adapters, s, cfg, dtype=np.float32, relu_mask_bf16=False):
    """One client: its sequences run independently (positions restart at 0, reading R5);
    LoRA grads are summed over all of the client's tokens (backward overwrites, reading R10).
    x_c, g_c: [T_c, d] client-major packed.  Returns x_s, g_s [T_c, d], grads."""
    outs, gins, total = [], [], None
    off = 0
    for S in seq_lens:
        xs, gs, gr = segment_fwd_bwd(x_c[off:off + S], g_c[off:off + S], weights, adapters, s, cfg, dtype,
                                     relu_mask_bf16)
        outs.append(xs)
        gins.append(gs)
        if total is None:
            total = gr
        else:
            total = [{t: (total[l][t][0] + gr[l][t][0], total[l][t][1] + gr[l][t][1]) for t in gr[l]}
                     for l in range(len(gr))]
        off += S
    return np.concatenate(outs), np.concatenate(gins), total


def batched_step(xs, gs, clients, weights, adapters_per_client, cfg, dtype=np.float32):
    """A batched multi-client call is DEFINED as the concatenation of per-client calls
    (PAPER.md:428).  xs/gs: per-client [T_c, d] arrays.  clients: ClientCfg-like objects
    with seq_lens, rank, alpha."""
    res = []
    for i, c in enumerate(clients):
        s = c.alpha / c.rank
        res.append(client_step(xs[i], gs[i], c.seq_lens, weights, adapters_per_client[i], s, cfg, dtype))
    return res


# ============================================================ AdamW (reading R7)
def adamw_step(p, g, m, v, t, lr, beta1, beta2, eps, weight_decay):
    """torch.optim.AdamW semantics (decoupled decay, bias correction), step number t>=1:
    p <- p(1 - lr*wd); m <- b1 m + (1-b1) g; v <- b2 v + (1-b2) g^2;
    p <- p - lr/(1-b1^t) * m / (sqrt(v)/sqrt(1-b2^t) + eps).  Returns new (p, m, v)."""
    p = p * (1.0 - lr * weight_decay)
    m = beta1 * m + (1.0 - beta1) * g
    v = beta2 * v + (1.0 - beta2) * g * g
    bc1 = 1.0 - beta1 ** t
    bc2 = 1.0 - beta2 ** t
    denom = np.sqrt(v) / np.sqrt(bc2) + eps
    p = p - (lr / bc1) * m / denom
    return p, m, v


# ============================================================ memory model (Eq.2 / Eq.3)
def memory_vanilla(M, A, O, I, N):
    """Eq.2: (M + A + O + I) * N."""
    return (M + A + O + I) * N


def memory_shared_base(M, A, O, I, N):
    """Base-model sharing: M + (A + O + I) * N."""
    return M + (A + O + I) * N


def memory_menos(M, A, O, I, N):
    """Eq.3: M + (A + O) * N + I."""
    return M + (A + O) * N + I


def persistent_reduction(M, AO, N):
    """Persistent-memory reduction the paper's way (Fig.5):
    1 - (M + N*(A+O)) / (N*(M + A+O))."""
    return 1.0 - (M + N * AO) / (N * (M + AO))
