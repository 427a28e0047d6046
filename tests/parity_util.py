"""Helpers shared by the GPU parity tests, smoke() and bench.py's parity spot check.

run_gpu_step  : drives libmenos.so through its C-ABI (paper_conf_middleware_hul24_b200.Server).
run_oracle_step: the CPU oracle (oracle/menos_oracle.py) on the same seeded inputs.
compare_step  : BASELINE.json north_star bars -- activations max|d|/max|ref| <= 2e-2, every gradient tensor
                cosine >= 0.999 (DESIGN.md §"Tolerances") -- applied to x_s and g_s AND to the segment's branch
                deltas x_s - x_c and g_s - g_c (so an identity map, a dropped branch or a dropped adapter cannot hide
                behind the residual stream; tests/test_mutants.py proves each such mutant fails).
"""
from __future__ import annotations

import numpy as np

from workloads import TARGETS, Workload, base_layer_weights, client_adapters, client_inputs

ACT_TOL = 2e-2
COS_TOL = 0.999


def _bf16(a, device="cpu"):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(torch.bfloat16).to(device).contiguous()


def make_inputs(w: Workload, seed: int = 0, zero_b: bool = False, outlier: bool = False, recipe: str = "default"):
    m = w.model
    weights = [base_layer_weights(m, l, seed=seed, recipe=recipe) for l in range(m.n_layers)]
    adapters = [client_adapters(m, c, seed=1000 + 17 * seed + i, zero_b=zero_b) for i, c in enumerate(w.clients)]
    io = [client_inputs(m, c, seed=2000 + 17 * seed + i, outlier=outlier) for i, c in enumerate(w.clients)]
    return weights, adapters, io


def new_server(w: Workload, weights, arena_bytes=0, max_rank=16, device="cuda:0"):
    import torch
    from paper_conf_middleware_hul24_b200 import Server
    m = w.model
    wl = []
    for W in weights:
        wl.append({k: _bf16(v) for k, v in W.items()})
    names = {"wq": "wq", "wk": "wk", "wv": "wv", "wo": "wo", "wgate": "wgate", "wup": "wup", "wdown": "wdown"}
    del names
    # prefix-tuning clients (rank = P) attend over P + S rows: the library bounds that by max_seq_len too
    max_seq = max(max(c.seq_lens) + (c.rank if "prefix" in c.targets else 0) for c in w.clients)
    srv = Server(m.d_model, m.n_heads, m.n_kv_heads, m.d_ff, m.n_layers, first_layer=m.first_layer,
                 rms_eps=m.rms_eps, rope_theta=m.rope_theta, weights=wl, max_rank=max_rank,
                 max_seq_len=max(max_seq, 64), arena_bytes=arena_bytes, arch=m.arch)
    return srv


def register(srv, w: Workload, adapters, seed=0):
    ids = []
    for i, c in enumerate(w.clients):
        cid = srv.register_client(c.rank, c.alpha, c.targets, seed=seed + i,
                                  cut_layer=(w.model.first_layer + c.cut) if c.cut else None)
        for l, d in enumerate(adapters[i]):
            if l < c.cut:
                continue   # no adapters below the client's cut
            for t, (A, B) in d.items():
                srv.set_adapter(cid, l, t, "A", A)
                srv.set_adapter(cid, l, t, "B", B)
        ids.append(cid)
    return ids


def run_gpu_step(w: Workload, seed: int = 0, zero_b: bool = False, flags: int = 0, inputs=None, srv=None,
                 ids=None, keep=False, grads=True):
    """One forward + backward of the whole batch on cuda:0.  Returns per-client x_s, g_s and adapter grads."""
    import torch
    m = w.model
    weights, adapters, io = inputs if inputs is not None else make_inputs(w, seed, zero_b)
    own = srv is None
    if own:
        srv = new_server(w, weights)
        ids = register(srv, w, adapters)
    seq_client, seq_len = [], []
    for i, c in enumerate(w.clients):
        seq_client += [ids[i]] * len(c.seq_lens)
        seq_len += list(c.seq_lens)
    x = _bf16(np.concatenate([a for a, _ in io]), "cuda")
    g = _bf16(np.concatenate([b for _, b in io]), "cuda")
    xs = torch.empty_like(x)
    gs = torch.empty_like(x)
    b = srv.forward(seq_client, seq_len, x, xs, flags=flags)
    srv.backward(b, g, gs)
    torch.cuda.synchronize()
    out = {"x_s": [], "g_s": [], "grads": [], "x_c": [a for a, _ in io], "g_c": [b for _, b in io]}
    off = 0
    xs_h, gs_h = xs.float().cpu().numpy(), gs.float().cpu().numpy()
    for i, c in enumerate(w.clients):
        T = c.n_tokens
        out["x_s"].append(xs_h[off:off + T])
        out["g_s"].append(gs_h[off:off + T])
        off += T
        gr = []
        if grads:
            for l in range(c.cut, m.n_layers):   # the client's layers (grads index 0 = its cut layer)
                gr.append({t: (srv.get_adapter(ids[i], l, t, "dA"), srv.get_adapter(ids[i], l, t, "dB"))
                           for t in c.targets})
        out["grads"].append(gr)
    if keep:
        out["server"], out["ids"] = srv, ids
    elif own:
        srv.close()
    return out


def run_oracle_step(w: Workload, seed: int = 0, zero_b: bool = False, inputs=None, clients=None):
    from oracle import menos_oracle as O
    m = w.model
    weights, adapters, io = inputs if inputs is not None else make_inputs(w, seed, zero_b)
    out = {"x_s": [], "g_s": [], "grads": [], "x_c": [a for a, _ in io], "g_c": [b for _, b in io]}
    for i, c in enumerate(w.clients):
        if clients is not None and i not in clients:
            out["x_s"].append(None); out["g_s"].append(None); out["grads"].append(None)
            continue
        # a client with cut k runs the segment [k, L): the same oracle on the layers it sends its tokens through
        mc = m.with_layers(m.n_layers - c.cut) if c.cut else m
        # OPT: the ReLU mask is a floating-point decision; the oracle takes it in the kernel's precision (bf16 GEMM
        # operands, fp32 accumulation: reading R25).  r2a measured the plain fp32 decision on the GPU suite: fc1 dA/dB
        # cosines 0.9986-0.9990 on the tiny OPT mix, all from near-zero pre-activations (tests/test_gpu_opt.py
        # test_relu_mask_valid checks the kernel's own decision against the exact sign outside the rounding band).
        xs, gs, gr = O.client_step(io[i][0], io[i][1], c.seq_lens, weights[c.cut:], adapters[i][c.cut:],
                                   c.alpha / c.rank, mc, relu_mask_bf16=(m.arch == "opt"))
        out["x_s"].append(xs)
        out["g_s"].append(gs)
        out["grads"].append(gr)
    return out


def act_err(a, ref):
    return float(np.max(np.abs(a - ref)) / max(np.max(np.abs(ref)), 1e-30))


def bf16_ulp(x):
    """Spacing of bf16 numbers at |x| (8 significant bits): 2^(floor(log2|x|) - 7)."""
    ax = np.maximum(np.abs(np.asarray(x, np.float64)), 2.0 ** -126)
    return np.exp2(np.floor(np.log2(ax)) - 7)


def delta_err(xs_gpu, xs_ref, xc):
    """max|(x_s - x_c)_gpu - (x_s - x_c)_ref| / max|(x_s - x_c)_ref|, each element first discounted by one bf16 ulp of
    |x_s|: the kernels return x_s rounded to bf16 (RNE) after the residual add, so an element may sit one output ulp
    from the fp32 reference through rounding alone.  That ulp is what x_c's massive-activation channels (x100) make
    larger than the branch delta; a dropped or wrong branch is O(1) of the delta and still fails."""
    g = np.asarray(xs_gpu, np.float64) - xc
    r = np.asarray(xs_ref, np.float64) - xc
    err = np.maximum(np.abs(g - r) - bf16_ulp(xs_ref), 0.0)
    return float(np.max(err) / max(np.max(np.abs(r)), 1e-30))


def cosine(a, ref):
    a = np.asarray(a, np.float64).ravel()
    b = np.asarray(ref, np.float64).ravel()
    na, nb = np.linalg.norm(a), np.linalg.norm(b)
    if na < 1e-30 and nb < 1e-30:
        return 1.0
    return float(a @ b / max(na * nb, 1e-300))


def compare_step(gpu, ora, clients=None):
    rep = {}
    n = len(gpu["x_s"])
    for i in range(n):
        if clients is not None and i not in clients:
            continue
        e = act_err(gpu["x_s"][i], ora["x_s"][i])
        rep[f"c{i}.x_s"] = {"metric": e, "ok": e <= ACT_TOL, "kind": "maxrel"}
        cg = cosine(gpu["g_s"][i], ora["g_s"][i])
        rep[f"c{i}.g_s"] = {"metric": cg, "ok": cg >= COS_TOL, "kind": "cos"}
        # branch deltas: what the segment adds to its input / to the incoming gradient
        xc, gc = np.asarray(ora["x_c"][i], np.float64), np.asarray(ora["g_c"][i], np.float64)
        e = delta_err(gpu["x_s"][i], ora["x_s"][i], xc)
        rep[f"c{i}.x_s-x_c"] = {"metric": e, "ok": e <= ACT_TOL, "kind": "maxrel"}
        cg = cosine(gpu["g_s"][i] - gc, ora["g_s"][i] - gc)
        rep[f"c{i}.g_s-g_c"] = {"metric": cg, "ok": cg >= COS_TOL, "kind": "cos"}
        for l, d in enumerate(gpu["grads"][i]):
            for t, (dA, dB) in d.items():
                oA, oB = ora["grads"][i][l][t]
                ca, cb = cosine(dA, oA), cosine(dB, oB)
                rep[f"c{i}.L{l}.{t}.dA"] = {"metric": ca, "ok": ca >= COS_TOL, "kind": "cos"}
                rep[f"c{i}.L{l}.{t}.dB"] = {"metric": cb, "ok": cb >= COS_TOL, "kind": "cos"}
    return rep
