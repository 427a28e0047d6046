"""Per-client cut points: clients whose tokens enter the server segment at
different layers share one batched pass.  Layer l runs on the prefix of clients with cut <= l; a client with cut k
is the oracle's segment [k, L) (tests/test_oracle_pins.py pins the composition at a cut)."""
import dataclasses

import numpy as np
import pytest

from tests.parity_util import (compare_step, make_inputs, new_server, register, run_gpu_step, run_oracle_step)
from workloads import ClientCfg, MODELS, TARGETS, Workload

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _w():
    m = dataclasses.replace(MODELS["tiny"], n_layers=4, n_kv_heads=2, model_layers=5)
    cl = [ClientCfg(4, 8.0, ("q", "v"), [17, 40], cut=0), ClientCfg(8, 16.0, TARGETS, [96], cut=0),
          ClientCfg(16, 32.0, ("q", "v", "o"), [130, 5], cut=1), ClientCfg(4, 8.0, ("v", "down"), [64], cut=3),
          ClientCfg(8, 16.0, ("q", "k", "gate", "up"), [33, 1, 70], cut=3)]
    return Workload("cuts_mix", m, cl)


def assert_ok(rep):
    bad = {k: v for k, v in rep.items() if not v["ok"]}
    assert not bad, bad


def test_mixed_cuts_parity_vs_oracle():
    w = _w()
    assert_ok(compare_step(run_gpu_step(w, seed=11), run_oracle_step(w, seed=11)))


@pytest.mark.parametrize("flags", [0, 1])
def test_mixed_cuts_batched_equals_alone_bitwise(flags):
    """Invariant (c) with cuts, in SAVE and NOGRAD (re-forward) mode."""
    w = _w()
    inputs = make_inputs(w, seed=12)
    full = run_gpu_step(w, inputs=inputs, flags=flags)
    for i, c in enumerate(w.clients):
        wi = Workload("one", w.model, [c])
        one = run_gpu_step(wi, inputs=(inputs[0], [inputs[1][i]], [inputs[2][i]]), flags=flags)
        assert np.array_equal(full["x_s"][i], one["x_s"][0]), i
        assert np.array_equal(full["g_s"][i], one["g_s"][0]), i
        for l, d in enumerate(one["grads"][0]):
            for t, (dA, dB) in d.items():
                assert np.array_equal(full["grads"][i][l][t][0], dA) and np.array_equal(full["grads"][i][l][t][1], dB)


def test_cut_api_errors():
    from paper_conf_middleware_hul24_b200.menos import MenosError
    w = _w()
    weights, adapters, io = make_inputs(w, seed=13)
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    with pytest.raises(MenosError):
        srv.get_adapter(ids[3], 1, "v", "A")                    # below client 3's cut (layer 3)
    with pytest.raises(MenosError):
        srv.register_client(4, 8.0, ("q",), cut_layer=w.model.first_layer + w.model.n_layers)   # past the segment
    x = torch.zeros(64 + 17, w.model.d_model, dtype=torch.bfloat16, device="cuda")
    xs = torch.empty_like(x)
    with pytest.raises(MenosError):                             # cut 3 before cut 0: not in cut order
        srv.forward([ids[3], ids[0]], [64, 17], x, xs)
    srv.close()


def test_all_clients_at_last_layer():
    m = dataclasses.replace(MODELS["tiny"], n_layers=3, model_layers=4)
    w = Workload("late", m, [ClientCfg(4, 8.0, ("q", "v"), [20, 9], cut=2), ClientCfg(8, 16.0, ("o",), [31], cut=2)])
    assert_ok(compare_step(run_gpu_step(w, seed=14), run_oracle_step(w, seed=14)))
