"""The parity harness must be able to FAIL.

Each mutant below is the oracle with one plausible kernel bug planted (a dropped branch, a missing RoPE, a client's
adapter ignored, the sequence mask leaking, the wrong GQA map, only one sequence's gradients kept, an identity map).
Its outputs go through exactly the comparison the GPU parity tests and smoke() use (tests/parity_util.compare_step)
against the true oracle, on the configs smoke() and the tiny GPU tests run (cfg0, tiny_mix).  A mutant that passes
every check would mean a GPU kernel with that bug would pass too, so each one must fail at least one check.
"""
import contextlib
import copy
import dataclasses

import numpy as np
import pytest

from oracle import menos_oracle as O
from tests.parity_util import compare_step, make_inputs, run_oracle_step
from workloads import ClientCfg, MODELS, TARGETS, Workload, workload


def tiny_mix():
    m = dataclasses.replace(MODELS["tiny"], n_heads=4, n_kv_heads=2)
    cl = [ClientCfg(4, 8.0, TARGETS, [1, 17, 3]), ClientCfg(16, 32.0, ("q", "v"), [129]),
          ClientCfg(8, 16.0, ("k", "o", "gate", "up", "down"), [64, 40]), ClientCfg(5, 10.0, ("v", "down"), [200])]
    return Workload("tiny_mix", m, cl)


def prefix_mix():
    from workloads import PREFIX
    return Workload("prefix_mix", MODELS["tiny"], [ClientCfg(4, 8.0, ("q", "v"), [16, 16]),
                                                   ClientCfg(4, 1.0, (PREFIX,), [9, 20]),
                                                   ClientCfg(2, 1.0, (PREFIX,), [1, 30, 5])])


CONFIGS = {"cfg0": (lambda: workload("cfg0_tiny"), 0), "tiny_mix": (tiny_mix, 3), "prefix_mix": (prefix_mix, 5)}


@contextlib.contextmanager
def patched(**fns):
    old = {k: getattr(O, k) for k in fns}
    for k, f in fns.items():
        setattr(O, k, f)
    try:
        yield
    finally:
        for k, f in old.items():
            setattr(O, k, f)


def _attn_zero_fwd(q, k, v):
    return np.zeros_like(q), np.zeros((q.shape[1], q.shape[0]), q.dtype)


def _attn_zero_bwd(dO, q, k, v):
    return np.zeros_like(q), np.zeros_like(k), np.zeros_like(v)


_true_attn_fwd, _true_attn_bwd = O.attention_fwd, O.attention_bwd


def _gqa_modulo(fn):
    """Head h reads kv head h % Hkv instead of h // (H/Hkv): permute q's heads so the true kernel sees that map."""
    def perm(H, Hkv):
        rep = H // Hkv
        # the true map gives position p kv head p // rep; place there an original head h with h % Hkv == p // rep
        return np.array([p // rep + Hkv * (p % rep) for p in range(H)])

    def fwd(q, k, v):
        P = perm(q.shape[1], k.shape[1])
        o, lse = _true_attn_fwd(q[:, P], k, v)
        out, l2 = np.empty_like(o), np.empty_like(lse)
        out[:, P], l2[P] = o, lse
        return out, l2

    def bwd(dO, q, k, v):
        P = perm(q.shape[1], k.shape[1])
        dq, dk, dv = _true_attn_bwd(dO[:, P], q[:, P], k, v)
        o = np.empty_like(dq)
        o[:, P] = dq
        return o, dk, dv
    return fwd if fn == "fwd" else bwd


def mutant(name, w, inputs):
    """Outputs of the oracle with bug `name` planted."""
    weights, adapters, io = inputs
    if name == "mlp_dropped":
        wz = [dict(W, wdown=np.zeros_like(W["wdown"])) for W in weights]
        return run_oracle_step(w, inputs=(wz, adapters, io))
    if name == "attention_skipped":
        with patched(attention_fwd=_attn_zero_fwd, attention_bwd=_attn_zero_bwd):
            return run_oracle_step(w, inputs=inputs)
    if name == "prefix_ignored":     # the attention of prefix clients runs without their prefix (grads left correct)
        if not any("prefix" in c.targets for c in w.clients):
            return None
        good = run_oracle_step(w, inputs=inputs)
        ad = [[{t: v for t, v in d.items() if t != "prefix"} for d in a] for a in adapters]
        bad = run_oracle_step(w, inputs=(weights, ad, io))
        bad["grads"] = good["grads"]
        return bad
    if name == "rope_off":
        with patched(rope_fwd=lambda x, c, s: x, rope_bwd=lambda dy, c, s: dy):
            return run_oracle_step(w, inputs=inputs)
    if name == "gqa_modulo":
        if w.model.n_kv_heads == w.model.n_heads:
            return None
        with patched(attention_fwd=_gqa_modulo("fwd"), attention_bwd=_gqa_modulo("bwd")):
            return run_oracle_step(w, inputs=inputs)
    if name == "client_lora_dropped":   # the forward ignores client 1's adapter; its gradients are left correct
        good = run_oracle_step(w, inputs=inputs)
        ad = list(adapters)
        ad[1] = [{} for _ in ad[1]]
        bad = run_oracle_step(w, inputs=(weights, ad, io))
        bad["grads"][1] = good["grads"][1]
        return bad
    if name == "lora_scale_one":      # alpha/r taken as 1
        w2 = copy.deepcopy(w)
        for c in w2.clients:
            c.alpha = float(c.rank)
        return run_oracle_step(w2, inputs=inputs)
    if name == "sequences_not_separated":   # varlen mask leaks: a client's sequences attend across each other
        if all(len(c.seq_lens) == 1 for c in w.clients):
            return None
        w2 = copy.deepcopy(w)
        for c in w2.clients:
            c.seq_lens = [sum(c.seq_lens)]
        return run_oracle_step(w2, inputs=inputs)
    if name == "last_sequence_grads_only":
        good = run_oracle_step(w, inputs=inputs)
        for i, c in enumerate(w.clients):
            if len(c.seq_lens) < 2:
                continue
            off = sum(c.seq_lens[:-1])
            wl = copy.deepcopy(w)
            wl.clients = [dataclasses.replace(c, seq_lens=[c.seq_lens[-1]])]
            io_i = (io[i][0][off:], io[i][1][off:])
            last = run_oracle_step(wl, inputs=(weights, [adapters[i]], [io_i]))
            good["grads"][i] = last["grads"][0]
        return good
    if name == "identity":
        good = run_oracle_step(w, inputs=inputs)
        good["x_s"] = [a.copy() for a in good["x_c"]]
        good["g_s"] = [b.copy() for b in good["g_c"]]
        return good
    raise KeyError(name)


MUTANTS = ["mlp_dropped", "attention_skipped", "prefix_ignored", "rope_off", "gqa_modulo", "client_lora_dropped", "lora_scale_one",
           "sequences_not_separated", "last_sequence_grads_only", "identity"]


@pytest.fixture(scope="module")
def truth():
    out = {}
    for cname, (mk, seed) in CONFIGS.items():
        w = mk()
        inputs = make_inputs(w, seed=seed)
        out[cname] = (w, inputs, run_oracle_step(w, inputs=inputs))
    return out


@pytest.mark.parametrize("cname", list(CONFIGS))
def test_oracle_passes_its_own_bars(truth, cname):
    w, inputs, ora = truth[cname]
    rep = compare_step(ora, ora)
    assert all(v["ok"] for v in rep.values())


@pytest.mark.parametrize("name", MUTANTS)
@pytest.mark.parametrize("cname", list(CONFIGS))
def test_mutant_fails_parity(truth, cname, name):
    w, inputs, ora = truth[cname]
    mut = mutant(name, w, inputs)
    if mut is None:
        pytest.skip(f"{name} does not apply to {cname}")
    rep = compare_step(mut, ora)
    failed = {k: round(v["metric"], 5) for k, v in rep.items() if not v["ok"]}
    assert failed, f"mutant {name} passes every parity check on {cname}"


def test_bf16_rounding_alone_passes(truth):
    """The bars are not so tight that the GPU's own precision fails them: the oracle run on bf16-rounded
    intermediates of the segment's output (x_s, g_s rounded to bf16, as the kernels return them) still passes."""
    from workloads import bf16_round
    for cname in CONFIGS:
        w, inputs, ora = truth[cname]
        r = {"x_s": [bf16_round(a) for a in ora["x_s"]], "g_s": [bf16_round(a) for a in ora["g_s"]],
             "grads": ora["grads"], "x_c": ora["x_c"], "g_c": ora["g_c"]}
        rep = compare_step(r, ora)
        assert all(v["ok"] for v in rep.values()), {k: v for k, v in rep.items() if not v["ok"]}
