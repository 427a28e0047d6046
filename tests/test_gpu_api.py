"""C-ABI state rules (include/menos.h "Stream rule" / "Live batches") and the binding's argument checks.

* A registration that would grow the LoRA slot tables while a SAVE batch is alive is refused (MENOS_ESTATE): the
  batch's LoRA problem lists point into the tables.  One that fits in the existing tables is allowed, and the live
  batch's backward still matches a fresh run bitwise.
* A client inside a live batch cannot be unregistered (so its id cannot be reused under the batch).
* All of a server's work stays on one stream (MENOS_EINVAL otherwise).
* x_c / x_s / g_c / g_s of the wrong dtype, shape or layout are rejected by the binding before any device access.
"""
import numpy as np
import pytest

from tests.parity_util import _bf16, make_inputs, new_server, register
from workloads import ClientCfg, MODELS, Workload

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _setup(n_clients=2, rank=4):
    m = MODELS["tiny"]
    w = Workload("api", m, [ClientCfg(rank, 2.0 * rank, ("q", "v"), [24, 8]) for _ in range(n_clients)])
    weights, adapters, io = make_inputs(w, seed=51)
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    x = _bf16(np.concatenate([a for a, _ in io]), "cuda")
    g = _bf16(np.concatenate([b for _, b in io]), "cuda")
    sc = sum([[ids[i]] * 2 for i in range(n_clients)], [])
    sl = [24, 8] * n_clients
    return srv, ids, x, g, sc, sl


def test_live_save_batch_blocks_table_growth_and_unregister():
    from paper_conf_middleware_hul24_b200.menos import MenosError
    srv, ids, x, g, sc, sl = _setup()
    xs, gs = torch.empty_like(x), torch.empty_like(x)
    b = srv.forward(sc, sl, x, xs)
    # growth needed: the q/k/v slot table holds 64 columns, filled by 2 clients x 2 targets x 16; a client with
    # 3 targets x 16 columns cannot fit
    with pytest.raises(MenosError) as e:
        srv.register_client(16, 32.0, ("q", "k", "v"))
    assert e.value.code == -4
    with pytest.raises(MenosError) as e:
        srv.unregister_client(ids[0])
    assert e.value.code == -4
    srv.backward(b, g, gs)
    torch.cuda.synchronize()
    # after the backward both are allowed
    cid = srv.register_client(16, 32.0, ("q", "k", "v"))
    srv.unregister_client(cid)
    srv.close()


def test_registration_that_fits_under_live_batch_keeps_results():
    srv, ids, x, g, sc, sl = _setup()
    xs0, gs0 = torch.empty_like(x), torch.empty_like(x)
    b = srv.forward(sc, sl, x, xs0)
    srv.backward(b, g, gs0)
    dA0 = srv.get_adapter(ids[0], 0, "q", "dA")
    srv.unregister_client(srv.register_client(4, 8.0, ("q",)))   # leave a free slot of 16 columns
    xs1, gs1 = torch.empty_like(x), torch.empty_like(x)
    b = srv.forward(sc, sl, x, xs1)
    cid = srv.register_client(4, 8.0, ("v",))                     # fits in the freed 16 columns
    srv.backward(b, g, gs1)
    torch.cuda.synchronize()
    assert torch.equal(xs0, xs1) and torch.equal(gs0, gs1)
    assert np.array_equal(dA0, srv.get_adapter(ids[0], 0, "q", "dA"))
    srv.unregister_client(cid)
    srv.close()


def test_one_stream_per_server():
    from paper_conf_middleware_hul24_b200.menos import MenosError
    srv, ids, x, g, sc, sl = _setup()
    xs, gs = torch.empty_like(x), torch.empty_like(x)
    s1 = torch.cuda.Stream()
    b = srv.forward(sc, sl, x, xs, stream=s1)
    with pytest.raises(MenosError) as e:
        srv.backward(b, g, gs, stream=torch.cuda.Stream())
    assert e.value.code == -1
    srv.backward(b, g, gs, stream=s1)
    with pytest.raises(MenosError):
        srv.adapter_step(ids)                      # the legacy default stream is another stream
    srv.adapter_step(ids, stream=s1)
    s1.synchronize()
    srv.close()


def test_binding_rejects_bad_activation_buffers():
    from paper_conf_middleware_hul24_b200.menos import MenosError
    srv, ids, x, g, sc, sl = _setup()
    xs = torch.empty_like(x)
    for bad in (x.float(), x[:-1], x.t().contiguous().t(), torch.empty(x.shape[0], x.shape[1] + 1,
                                                                        dtype=torch.bfloat16, device="cuda")):
        with pytest.raises(MenosError):
            srv.forward(sc, sl, bad, xs)
    with pytest.raises(MenosError):
        srv.forward(sc, sl, x, xs[:, :-1])
    b = srv.forward(sc, sl, x, xs)
    with pytest.raises(MenosError):
        srv.backward(b, g.float(), torch.empty_like(x))
    srv.batch_free(b)
    srv.close()
