"""White-box GPU parity: every saved intermediate of every layer of a SAVE batch against the oracle's own
per-layer values (VERDICT r1 "next" #1).

x_s / g_s comparisons see a layer only through the residual stream; here each step of §8(a) is checked where it
lands: x (A1 input), xn (A1), q|k|v post-RoPE (A2), O (A3), lse (A3), h (A4), hn (A5), a = silu(gate)*up (A6, kept
when a client targets down) -- per layer, per client, through include/menos_testing.h menos_test_batch_tensor.
Bar: the activation bar of BASELINE.json north_star (max|d|/max|ref| <= 2e-2) on every tensor.
"""
import dataclasses

import numpy as np
import pytest

from tests.parity_util import ACT_TOL, _bf16, act_err, make_inputs, new_server, register
from workloads import ClientCfg, MODELS, TARGETS, Workload, bits_to_f32, workload

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def oracle_layer_values(w, inputs):
    """Per layer: token-major oracle intermediates of the whole batch (client-major, sequence-major)."""
    from oracle import menos_oracle as O
    m = w.model
    weights, adapters, io = inputs
    fwd = O.opt_layer_fwd if m.arch == "opt" else O.layer_fwd
    per_layer = [dict() for _ in range(m.n_layers)]
    for i, c in enumerate(w.clients):
        off = 0
        s = np.float32(c.alpha / c.rank)
        for S in c.seq_lens:
            x = np.asarray(io[i][0][off:off + S], np.float32)
            off += S
            for l in range(m.n_layers):
                y, cache = fwd(x, weights[l], adapters[i][l], s, m)
                vals = {"x": cache["x"], "xn": cache["xn"],
                        "qkv": np.concatenate([cache["q"].reshape(S, -1), cache["k"].reshape(S, -1),
                                               cache["v"].reshape(S, -1)], axis=1),
                        "O": cache["O"], "h": cache["h"], "hn": cache["hn"], "a": cache["a"], "lse": cache["lse"].T}
                for k, v in vals.items():
                    per_layer[l].setdefault(k, []).append(np.asarray(v, np.float32))
                x = y
    return [{k: np.concatenate(v, axis=0) for k, v in d.items()} for d in per_layer]


WHICH = {"x": (0, "f32"), "xn": (1, "bf16"), "qkv": (2, "bf16"), "O": (3, "bf16"), "h": (4, "f32"),
         "hn": (5, "bf16"), "a": (7, "bf16"), "lse": (12, "f32")}


def gpu_layer_values(w, inputs):
    m = w.model
    weights, adapters, io = inputs
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    seq_client, seq_len = [], []
    for i, c in enumerate(w.clients):
        seq_client += [ids[i]] * len(c.seq_lens)
        seq_len += list(c.seq_lens)
    x = _bf16(np.concatenate([a for a, _ in io]), "cuda")
    xs = torch.empty_like(x)
    b = srv.forward(seq_client, seq_len, x, xs)
    torch.cuda.synchronize()
    T = x.shape[0]
    save_a = m.arch == "opt" or any("down" in c.targets for c in w.clients)
    out = []
    for l in range(m.n_layers):
        d = {}
        for k, (wh, dt) in WHICH.items():
            if k == "a" and not save_a:
                continue
            raw = srv.batch_tensor(b, l, wh)
            v = raw.view(np.float32) if dt == "f32" else bits_to_f32(raw.view(np.uint16))
            if k == "lse":
                v = v.reshape(m.n_heads, T).T
            else:
                v = v.reshape(T, -1)
            if k == "a":
                v = v[:, :m.d_ff]
            d[k] = v
        out.append(d)
    srv.batch_free(b)
    srv.close()
    return out


def tiny_mix():
    m = dataclasses.replace(MODELS["tiny"], n_heads=4, n_kv_heads=2)
    cl = [ClientCfg(4, 8.0, TARGETS, [1, 17, 3]), ClientCfg(16, 32.0, ("q", "v"), [129]),
          ClientCfg(8, 16.0, ("k", "o", "gate", "up", "down"), [64, 40]), ClientCfg(5, 10.0, ("v", "down"), [200])]
    return Workload("tiny_mix", m, cl)


def opt_mix():
    return Workload("opt_mix", MODELS["opt_tiny"],
                    [ClientCfg(4, 8.0, ("q", "v"), [16, 16]),
                     ClientCfg(8, 16.0, ("q", "k", "v", "o", "up", "down"), [33, 1, 70])])


def seven_b_two_layers():
    m = MODELS["7b"].with_layers(2)
    return Workload("7b_l2", m, [ClientCfg(8, 16.0, ("q", "v"), [300, 5]),
                                 ClientCfg(16, 32.0, ("q", "v", "o", "down"), [200])])


@pytest.mark.parametrize("mk,seed", [(lambda: workload("cfg0_tiny"), 0), (tiny_mix, 3), (opt_mix, 5),
                                     (seven_b_two_layers, 7)])
def test_every_saved_intermediate_matches_oracle(mk, seed):
    w = mk()
    inputs = make_inputs(w, seed=seed)
    ora = oracle_layer_values(w, inputs)
    gpu = gpu_layer_values(w, inputs)
    bad, rep = {}, {}
    for l in range(w.model.n_layers):
        for k, v in gpu[l].items():
            e = act_err(v, ora[l][k])
            rep[f"L{l}.{k}"] = round(e, 5)
            if not e <= ACT_TOL:
                bad[f"L{l}.{k}"] = e
    print(w.name, rep)
    assert not bad, bad
