"""Prefix-tuning clients on the GPU (SURVEY.md §8(f) NEXT-3; PAPER.md:59 §2.1, :121 §3.1; Li & Liang [16]; DESIGN.md
R28), mixed with LoRA clients in ONE batch over the shared base, against the oracle (attention_prefix_fwd / _bwd,
pinned in tests/test_oracle_pins.py).  The library runs the attention kernels on an extended batch whose prefix
clients' sequences are preceded by their prefix rows; these tests check x_s, g_s, the LoRA grads and the prefix
grads (dPk, dPv summed over the client's tokens) within the BASELINE.json bars, and the bitwise invariants."""
import dataclasses

import numpy as np
import pytest

from tests.parity_util import compare_step, make_inputs, new_server, register, run_gpu_step, run_oracle_step
from workloads import ClientCfg, MODELS, ModelCfg, PREFIX, TARGETS, Workload

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def assert_ok(rep):
    bad = {k: v for k, v in rep.items() if not v["ok"]}
    assert not bad, bad


def prefix_mix(m):
    return Workload("prefix_mix", m, [ClientCfg(4, 8.0, ("q", "v"), [16, 16]), ClientCfg(4, 1.0, (PREFIX,), [9, 20]),
                                      ClientCfg(8, 16.0, TARGETS, [33]), ClientCfg(2, 1.0, (PREFIX,), [1, 70, 5])])


@pytest.mark.parametrize("m", [MODELS["tiny"], dataclasses.replace(MODELS["tiny"], n_kv_heads=2),
                               ModelCfg("hd128", 512, 4, 2, 1024, 2, model_layers=3),   # tcgen05 attention kernels
                               ModelCfg("opt-small", 256, 4, 4, 1024, 2, model_layers=3, arch="opt")],
                         ids=["tiny", "tiny_gqa", "hd128_gqa", "opt_small_hd64"])
def test_prefix_clients_mixed_with_lora(m):
    w = prefix_mix(m)
    if m.arch == "opt":   # OPT has no gate projection
        w.clients[2] = ClientCfg(8, 16.0, ("q", "k", "v", "o", "up", "down"), [33])
    inputs = make_inputs(w, seed=61)
    assert_ok(compare_step(run_gpu_step(w, inputs=inputs), run_oracle_step(w, inputs=inputs)))


def test_prefix_batched_equals_alone_and_nograd_bitwise():
    m = MODELS["tiny"]
    w = prefix_mix(m)
    inputs = make_inputs(w, seed=62)
    weights, adapters, io = inputs
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    full = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids)
    ng = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids, flags=1)
    for i, c in enumerate(w.clients):
        assert np.array_equal(full["x_s"][i], ng["x_s"][i]) and np.array_equal(full["g_s"][i], ng["g_s"][i])
        alone = run_gpu_step(Workload("one", m, [c]), inputs=(weights, [adapters[i]], [io[i]]), srv=srv, ids=[ids[i]])
        assert np.array_equal(alone["x_s"][0], full["x_s"][i]), i
        assert np.array_equal(alone["g_s"][0], full["g_s"][i]), i
        for l in range(m.n_layers):
            for t in c.targets:
                for k in (0, 1):
                    assert np.array_equal(alone["grads"][0][l][t][k], full["grads"][i][l][t][k]), (i, l, t, k)
    srv.close()


def test_prefix_adamw_step_matches_oracle():
    """AdamW (A13) updates the prefix keys / values like any adapter tensor (torch.optim.AdamW semantics)."""
    from oracle import menos_oracle as O
    m = MODELS["tiny"]
    w = Workload("pa", m, [ClientCfg(3, 1.0, (PREFIX,), [12, 7])])
    inputs = make_inputs(w, seed=63)
    weights, adapters, io = inputs
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    out = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids)
    srv.adapter_step(ids)
    torch.cuda.synchronize()
    for l in range(m.n_layers):
        for k, which in ((0, "A"), (1, "B")):
            p0 = adapters[0][l][PREFIX][k].astype(np.float64)
            g = out["grads"][0][l][PREFIX][k].astype(np.float64)
            ref, _, _ = O.adamw_step(p0, g, np.zeros_like(p0), np.zeros_like(p0), 1, 1e-4, 0.9, 0.999, 1e-8, 0.01)
            got = srv.get_adapter(ids[0], l, PREFIX, which)
            np.testing.assert_allclose(got, ref, rtol=1e-5, atol=1e-6)
    srv.close()


def test_prefix_api_errors():
    from paper_conf_middleware_hul24_b200.menos import MenosError
    m = MODELS["tiny"]
    w = Workload("pe", m, [ClientCfg(3, 1.0, (PREFIX,), [4])])
    weights, _, _ = make_inputs(w, seed=64)
    srv = new_server(w, weights)
    with pytest.raises(MenosError):
        srv.register_client(4, 8.0, ("q", PREFIX))          # prefix is the client's only adapter
    cid = srv.register_client(4, 1.0, (PREFIX,))
    (ra, ca), (rb, cb) = srv.adapter_shape(cid, PREFIX)
    assert (ra, ca, rb, cb) == (4, m.n_kv_heads * m.head_dim, 4, m.n_kv_heads * m.head_dim)
    with pytest.raises(MenosError):
        srv.get_adapter(cid, 0, "q", "A")                    # not in its mask
    srv.close()
