"""Tensor-parallel decomposition (include/menos.h menos_tp_cfg), CPU, gloo,
world_size 2.

Each rank holds the shards `paper_conf_middleware_hul24_b200.tp` assigns (column-parallel q,k,v,gate,up;
row-parallel o,down; LoRA A replicated / B sharded for column targets, A sharded / B replicated for row targets)
and runs the exchange plan libmenos.so implements: all-reduce of the o-proj and down-proj partial sums (rank 0's
partial carries the residual), of the gate|up-dX and qkv-dX partial sums, and once per backward of the
replicated adapters' gradient partial sums.  The shard arithmetic is composed from oracle primitives; the result
must equal the UNSHARDED oracle (fp64, up to re-association).  This pins the host-side shard layout and the
placement of every collective that the GPU path's TP mode relies on.
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
CLIENT = ClientCfg(4, 8.0, TARGETS, [16, 9])                       # all 7 targets, ragged sequences
F64 = np.float64


def _allreduce(x):
    t = torch.from_numpy(np.ascontiguousarray(x))
    dist.all_reduce(t)
    return t.numpy()


def _shard_layer(rank, world, W, lora):
    hd = CFG.head_dim
    Ws = TP.shard_layer_weights(W, rank, world, CFG.n_heads, CFG.n_kv_heads, hd, CFG.d_ff)
    Ls = {t: TP.shard_adapter(t, A, B, rank, world, CFG.n_heads, CFG.n_kv_heads, hd, CFG.d_ff)
          for t, (A, B) in lora.items()}
    return ({k: np.asarray(v, F64) for k, v in Ws.items()},
            {t: (np.asarray(a, F64), np.asarray(b, F64)) for t, (a, b) in Ls.items()})


def _tp_layer_fwd(rank, x, W, L, s, H, Hkv):
    S = x.shape[0]
    hd = CFG.head_dim
    c = {"x": x}
    xn, c["rstd1"] = O.rmsnorm_fwd(x, W["g1"], CFG.rms_eps)
    c["xn"] = xn
    U = {}
    qp, U["q"] = O.proj_fwd(xn, W["wq"], L.get("q"), s)
    kp, U["k"] = O.proj_fwd(xn, W["wk"], L.get("k"), s)
    vp, U["v"] = O.proj_fwd(xn, W["wv"], L.get("v"), s)
    cos, sin = O.rope_cos_sin(S, hd, CFG.rope_theta, F64)
    c["cos"], c["sin"] = cos, sin
    q = O.rope_fwd(qp.reshape(S, H, hd), cos, sin)
    k = O.rope_fwd(kp.reshape(S, Hkv, hd), cos, sin)
    v = vp.reshape(S, Hkv, hd)
    Oa, _ = O.attention_fwd(q, k, v)
    c["q"], c["k"], c["v"] = q, k, v
    c["O"] = Oa.reshape(S, H * hd)
    ao, U["o"] = O.proj_fwd(c["O"], W["wo"], L.get("o"), s)          # row-parallel partial (+ s U_r B^T)
    h = _allreduce((x if rank == 0 else 0.0) + ao)                    # exchange 1
    c["h"] = h
    hn, c["rstd2"] = O.rmsnorm_fwd(h, W["g2"], CFG.rms_eps)
    c["hn"] = hn
    gt, U["gate"] = O.proj_fwd(hn, W["wgate"], L.get("gate"), s)
    up, U["up"] = O.proj_fwd(hn, W["wup"], L.get("up"), s)
    c["gt"], c["up"] = gt, up
    a = O.silu(gt) * up
    c["a"] = a
    md, U["down"] = O.proj_fwd(a, W["wdown"], L.get("down"), s)
    y = _allreduce((h if rank == 0 else 0.0) + md)                    # exchange 2
    c["U"] = U
    return y, c


def _tp_layer_bwd(dy, c, W, L, s, H, Hkv):
    S = dy.shape[0]
    hd = CFG.head_dim
    U = c["U"]
    g = {}
    da, g["down"] = O.proj_bwd(dy, c["a"], W["wdown"], L.get("down"), s, U["down"])
    dgt, dup = O.swiglu_bwd(da, c["gt"], c["up"])
    dg, g["gate"] = O.proj_bwd(dgt, c["hn"], W["wgate"], L.get("gate"), s, U["gate"])
    du, g["up"] = O.proj_bwd(dup, c["hn"], W["wup"], L.get("up"), s, U["up"])
    dhn = _allreduce(dg + du)                                         # exchange 3
    dh = dy + O.rmsnorm_bwd(dhn, c["h"], W["g2"], c["rstd2"])
    dO, g["o"] = O.proj_bwd(dh, c["O"], W["wo"], L.get("o"), s, U["o"])
    dq, dk, dv = O.attention_bwd(dO.reshape(S, H, hd), c["q"], c["k"], c["v"])
    dqp = O.rope_bwd(dq, c["cos"], c["sin"]).reshape(S, H * hd)
    dkp = O.rope_bwd(dk, c["cos"], c["sin"]).reshape(S, Hkv * hd)
    dxn = 0.0
    for t, d_t in (("q", dqp), ("k", dkp), ("v", dv.reshape(S, Hkv * hd))):
        dxt, g[t] = O.proj_bwd(d_t, c["xn"], W["w" + t], L.get(t), s, U[t])
        dxn = dxn + dxt
    dxn = _allreduce(dxn)                                             # exchange 4
    dx = dh + O.rmsnorm_bwd(dxn, c["x"], W["g1"], c["rstd1"])
    return dx, g


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        H, Hkv = CFG.n_heads // world, CFG.n_kv_heads // world
        Wf = [base_layer_weights(CFG, l, seed=0) for l in range(CFG.n_layers)]
        ad = client_adapters(CFG, CLIENT, seed=5)
        x_c, g_c = client_inputs(CFG, CLIENT, seed=6)
        s = CLIENT.alpha / CLIENT.rank
        shards = [_shard_layer(rank, world, Wf[l], ad[l]) for l in range(CFG.n_layers)]
        xs_all, gs_all, grads = [], [], [{} for _ in range(CFG.n_layers)]
        off = 0
        for S in CLIENT.seq_lens:
            x = x_c[off:off + S].astype(F64)
            caches = []
            for l in range(CFG.n_layers):
                x, c = _tp_layer_fwd(rank, x, *shards[l], s, H, Hkv)
                caches.append(c)
            xs_all.append(x)
            dy = g_c[off:off + S].astype(F64)
            for l in reversed(range(CFG.n_layers)):
                dy, gl = _tp_layer_bwd(dy, caches[l], *shards[l], s, H, Hkv)
                for t, (dA, dB) in gl.items():
                    pa, pb = grads[l].get(t, (0.0, 0.0))
                    grads[l][t] = (pa + dA, pb + dB)
            gs_all.append(dy)
            off += S
        # once per backward: the replicated adapters' gradient partial sums
        for l in range(CFG.n_layers):
            for t, (dA, dB) in grads[l].items():
                grads[l][t] = (_allreduce(dA), dB) if t in TP.COLUMN_PARALLEL else (dA, _allreduce(dB))
        q.put((rank, np.concatenate(xs_all), np.concatenate(gs_all), grads))
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
