"""Tensor-parallel decomposition (include/menos.h menos_tp_cfg), CPU, gloo,
world_size 2.

Each rank holds the shards `paper_conf_middleware_hul24_b200.tp` assigns (column-parallel q,k,v,gate,up;
row-parallel o,down; LoRA A replicated / B sharded for column targets, A sharded / B replicated for row targets)
and runs the SEQUENCE-PARALLEL exchange plan libmenos.so implements: the residual streams and the norms live on the
rank's token rows [r*Tl, (r+1)*Tl) (Tl = ceil(T / world), the last rank padded); per layer the norm outputs and the
incoming gradients dy, dh are all-gathered, the o / down partial sums (forward) and gate|up-dX / qkv-dX partial sums
(backward) are reduce-scattered, and once per backward the replicated adapters' gradient partial sums are
all-reduced; x_s and g_s are all-gathered at the end.  The shard arithmetic is composed from oracle primitives; the
result must equal the UNSHARDED oracle (fp64, up to re-association).  This pins the host-side shard layout, the row
split and the placement of every collective that the GPU path's tensor-parallel mode relies on.
"""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import menos_oracle as O
from paper_conf_middleware_hul24_b200 import tp as TP
from workloads import ClientCfg, ModelCfg, TARGETS, base_layer_weights, client_adapters, client_inputs

CFG = ModelCfg("tiny-gqa-tp", 64, 4, 2, 172, 2, model_layers=3)   # H=4, H_kv=2 (GQA), f=172 -> 2 ranks
CLIENT = ClientCfg(4, 8.0, TARGETS, [16, 9])                       # all 7 targets, ragged sequences: T = 25 (odd)
F64 = np.float64


def _allreduce(x):
    t = torch.from_numpy(np.ascontiguousarray(x))
    dist.all_reduce(t)
    return t.numpy()


def _rows(T):
    world, rank = dist.get_world_size(), dist.get_rank()
    loc = -(-T // world)
    return loc, loc * world, loc * rank


def _gather(x_loc, T):
    """all-gather of the ranks' [Tl, d] rows -> [T, d] (padding rows dropped)."""
    parts = [torch.empty_like(torch.from_numpy(x_loc)) for _ in range(dist.get_world_size())]
    dist.all_gather(parts, torch.from_numpy(np.ascontiguousarray(x_loc)))
    return torch.cat(parts).numpy()[:T]


def _scatter(part, T):
    """reduce-scatter of a [T, d] partial sum (padded to world * Tl rows) -> this rank's [Tl, d] rows."""
    loc, pad, r0 = _rows(T)
    full = np.zeros((pad, part.shape[1]), part.dtype)
    full[:T] = part
    return _allreduce(full)[r0:r0 + loc]


def _attn_fwd(q, k, v, lens):
    outs, off = [], 0
    for S in lens:
        o, _ = O.attention_fwd(q[off:off + S], k[off:off + S], v[off:off + S])
        outs.append(o)
        off += S
    return np.concatenate(outs)


def _attn_bwd(dO, q, k, v, lens):
    res, off = [], 0
    for S in lens:
        res.append(O.attention_bwd(dO[off:off + S], q[off:off + S], k[off:off + S], v[off:off + S]))
        off += S
    return [np.concatenate([r[i] for r in res]) for i in range(3)]


def _rope(lens, hd):
    cs, ss = zip(*[O.rope_cos_sin(S, hd, CFG.rope_theta, F64) for S in lens])
    return np.concatenate(cs), np.concatenate(ss)


def _shard_layer(rank, world, W, lora):
    hd = CFG.head_dim
    Ws = TP.shard_layer_weights(W, rank, world, CFG.n_heads, CFG.n_kv_heads, hd, CFG.d_ff)
    Ls = {t: TP.shard_adapter(t, A, B, rank, world, CFG.n_heads, CFG.n_kv_heads, hd, CFG.d_ff)
          for t, (A, B) in lora.items()}
    return ({k: np.asarray(v, F64) for k, v in Ws.items()},
            {t: (np.asarray(a, F64), np.asarray(b, F64)) for t, (a, b) in Ls.items()})


def _tp_layer_fwd(x_loc, T, lens, W, L, s, H, Hkv):
    hd = CFG.head_dim
    c = {"x": x_loc}
    xn_loc, c["rstd1"] = O.rmsnorm_fwd(x_loc, W["g1"], CFG.rms_eps)
    xn = _gather(xn_loc, T)                                           # exchange: all-gather xn
    c["xn"] = xn
    U = {}
    qp, U["q"] = O.proj_fwd(xn, W["wq"], L.get("q"), s)
    kp, U["k"] = O.proj_fwd(xn, W["wk"], L.get("k"), s)
    vp, U["v"] = O.proj_fwd(xn, W["wv"], L.get("v"), s)
    cos, sin = _rope(lens, hd)
    c["cos"], c["sin"] = cos, sin
    q = O.rope_fwd(qp.reshape(T, H, hd), cos, sin)
    k = O.rope_fwd(kp.reshape(T, Hkv, hd), cos, sin)
    v = vp.reshape(T, Hkv, hd)
    c["q"], c["k"], c["v"] = q, k, v
    c["O"] = _attn_fwd(q, k, v, lens).reshape(T, H * hd)
    ao, U["o"] = O.proj_fwd(c["O"], W["wo"], L.get("o"), s)          # row-parallel partial (+ s U_r B^T)
    h_loc = x_loc + _scatter(ao, T)                                   # exchange: reduce-scatter, residual add
    c["h"] = h_loc
    hn_loc, c["rstd2"] = O.rmsnorm_fwd(h_loc, W["g2"], CFG.rms_eps)
    hn = _gather(hn_loc, T)                                           # exchange: all-gather hn
    c["hn"] = hn
    gt, U["gate"] = O.proj_fwd(hn, W["wgate"], L.get("gate"), s)
    up, U["up"] = O.proj_fwd(hn, W["wup"], L.get("up"), s)
    c["gt"], c["up"] = gt, up
    a = O.silu(gt) * up
    c["a"] = a
    md, U["down"] = O.proj_fwd(a, W["wdown"], L.get("down"), s)
    y_loc = h_loc + _scatter(md, T)                                   # exchange: reduce-scatter, residual add
    c["U"] = U
    return y_loc, c


def _tp_layer_bwd(dy_loc, T, lens, c, W, L, s, H, Hkv):
    hd = CFG.head_dim
    U = c["U"]
    g = {}
    dy = _gather(dy_loc, T)                                           # exchange: all-gather dy
    da, g["down"] = O.proj_bwd(dy, c["a"], W["wdown"], L.get("down"), s, U["down"])
    dgt, dup = O.swiglu_bwd(da, c["gt"], c["up"])
    dg, g["gate"] = O.proj_bwd(dgt, c["hn"], W["wgate"], L.get("gate"), s, U["gate"])
    du, g["up"] = O.proj_bwd(dup, c["hn"], W["wup"], L.get("up"), s, U["up"])
    dhn_loc = _scatter(dg + du, T)                                    # exchange: reduce-scatter
    dh_loc = dy_loc + O.rmsnorm_bwd(dhn_loc, c["h"], W["g2"], c["rstd2"])
    dh = _gather(dh_loc, T)                                           # exchange: all-gather dh
    dO, g["o"] = O.proj_bwd(dh, c["O"], W["wo"], L.get("o"), s, U["o"])
    dq, dk, dv = _attn_bwd(dO.reshape(T, H, hd), c["q"], c["k"], c["v"], lens)
    dqp = O.rope_bwd(dq, c["cos"], c["sin"]).reshape(T, H * hd)
    dkp = O.rope_bwd(dk, c["cos"], c["sin"]).reshape(T, Hkv * hd)
    dxn = 0.0
    for t, d_t in (("q", dqp), ("k", dkp), ("v", dv.reshape(T, Hkv * hd))):
        dxt, g[t] = O.proj_bwd(d_t, c["xn"], W["w" + t], L.get(t), s, U[t])
        dxn = dxn + dxt
    dxn_loc = _scatter(dxn, T)                                        # exchange: reduce-scatter
    dx_loc = dh_loc + O.rmsnorm_bwd(dxn_loc, c["x"], W["g1"], c["rstd1"])
    return dx_loc, g


def _local(x, T):
    loc, pad, r0 = _rows(T)
    full = np.zeros((pad, x.shape[1]), x.dtype)
    full[:T] = x
    return full[r0:r0 + loc]


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        H, Hkv = CFG.n_heads // world, CFG.n_kv_heads // world
        Wf = [base_layer_weights(CFG, l, seed=0) for l in range(CFG.n_layers)]
        ad = client_adapters(CFG, CLIENT, seed=5)
        x_c, g_c = client_inputs(CFG, CLIENT, seed=6)
        s = CLIENT.alpha / CLIENT.rank
        T, lens = CLIENT.n_tokens, CLIENT.seq_lens
        shards = [_shard_layer(rank, world, Wf[l], ad[l]) for l in range(CFG.n_layers)]
        x = _local(x_c.astype(F64), T)
        caches = []
        for l in range(CFG.n_layers):
            x, c = _tp_layer_fwd(x, T, lens, *shards[l], s, H, Hkv)
            caches.append(c)
        xs = _gather(x, T)                                            # x_s on every rank
        dy = _local(g_c.astype(F64), T)
        grads = [None] * CFG.n_layers
        for l in reversed(range(CFG.n_layers)):
            dy, grads[l] = _tp_layer_bwd(dy, T, lens, caches[l], *shards[l], s, H, Hkv)
        gs = _gather(dy, T)
        # once per backward: the replicated adapters' gradient partial sums
        for l in range(CFG.n_layers):
            for t, (dA, dB) in grads[l].items():
                grads[l][t] = (_allreduce(dA), dB) if t in TP.COLUMN_PARALLEL else (dA, _allreduce(dB))
        q.put((rank, xs, gs, grads))
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_shard_slices_cover_and_reassemble():
    rng = np.random.default_rng(0)
    hd = CFG.head_dim
    for world in (1, 2):
        W = base_layer_weights(CFG, 0, seed=1)
        parts = [TP.shard_layer_weights(W, r, world, CFG.n_heads, CFG.n_kv_heads, hd, CFG.d_ff) for r in range(world)]
        for t in ("q", "k", "v", "gate", "up"):
            np.testing.assert_array_equal(np.concatenate([p["w" + t] for p in parts], 0), W["w" + t])
        for t in ("o", "down"):
            np.testing.assert_array_equal(np.concatenate([p["w" + t] for p in parts], 1), W["w" + t])
        for t in TARGETS:
            K, N = {"q": (64, 64), "k": (64, 32), "v": (64, 32), "o": (64, 64), "gate": (64, 172),
                    "up": (64, 172), "down": (172, 64)}[t]
            A, B = rng.standard_normal((4, K)), rng.standard_normal((N, 4))
            sh = [TP.shard_adapter(t, A, B, r, world, CFG.n_heads, CFG.n_kv_heads, hd, CFG.d_ff) for r in range(world)]
            A2, B2 = TP.gather_adapter(t, sh)
            np.testing.assert_array_equal(A2, A)
            np.testing.assert_array_equal(B2, B)


def test_gloo_tp2_equals_unsharded_oracle():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=300) for _ in procs], key=lambda r: r[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    Wf = [base_layer_weights(CFG, l, seed=0) for l in range(CFG.n_layers)]
    ad = client_adapters(CFG, CLIENT, seed=5)
    x_c, g_c = client_inputs(CFG, CLIENT, seed=6)
    xs, gs, gr = O.client_step(x_c, g_c, CLIENT.seq_lens, Wf, ad, CLIENT.alpha / CLIENT.rank, CFG, F64)

    def close(a, b):
        np.testing.assert_allclose(a, b, rtol=1e-9, atol=1e-11 * max(1.0, np.abs(b).max()))

    for r in range(world):                               # every rank ends with the same replicated outputs
        close(res[r][1], xs)
        close(res[r][2], gs)
    for l in range(CFG.n_layers):
        for t in TARGETS:
            dA, dB = TP.gather_adapter(t, [res[r][3][l][t] for r in range(world)])
            close(dA, gr[l][t][0])
            close(dB, gr[l][t][1])
            if t in TP.COLUMN_PARALLEL:                 # replicated gradients agree across ranks
                close(res[1][3][l][t][0], res[0][3][l][t][0])
            else:
                close(res[1][3][l][t][1], res[0][3][l][t][1])
