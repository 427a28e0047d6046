"""The Alg.2-driven serving loop on the GPU (paper_conf_middleware_hul24_b200/serve.py):
mixed forward / backward waves formed by the native scheduler under memory pressure.

* every wave's exact arena demand fits in what its grants reserved (MENOS_MEM_BOUND additivity) and no call
  returns ENOMEM;
* scheduling changes nothing a client sees: each client's x_s and g_s of every iteration and its
  adapters after the last AdamW step are BITWISE those of the client run alone, iteration by iteration;
* iteration 0 matches the CPU oracle within the north_star bars.
"""
import numpy as np
import pytest

from tests.parity_util import _bf16, act_err, cosine, make_inputs, new_server, register, run_oracle_step
from workloads import ClientCfg, MODELS, Workload, client_inputs

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _workload():
    m = MODELS["tiny"]
    cl = [ClientCfg(4, 8.0, ("q", "v"), [48, 16]), ClientCfg(16, 32.0, ("q", "v", "o"), [96]),
          ClientCfg(8, 16.0, ("q", "v", "down"), [7, 70]), ClientCfg(4, 8.0, ("q", "k", "v", "gate", "up"), [33]),
          ClientCfg(8, 16.0, ("q", "v"), [128, 64])]
    return Workload("serve_mix", m, cl)


def _iter_inputs(w, n_iters):
    """(seq_lens, x_c, g_c) per client and iteration; iteration 0 is the parity workload's."""
    weights, adapters, io = make_inputs(w, seed=4)
    out = {}
    for i, c in enumerate(w.clients):
        out[i] = []
        for k in range(n_iters):
            x, g = io[i] if k == 0 else client_inputs(w.model, c, seed=5000 + 97 * i + k)
            out[i].append((list(c.seq_lens), _bf16(x, "cuda"), _bf16(g, "cuda")))
    return (weights, adapters, io), out


def _adapters(srv, w, ids):
    return {(i, l, t, wh): srv.get_adapter(ids[i], l, t, wh)
            for i, c in enumerate(w.clients) for l in range(w.model.n_layers) for t in c.targets for wh in ("A", "B")}


def test_scheduled_serving_equals_alone_and_oracle():
    from paper_conf_middleware_hul24_b200 import menos as M
    from paper_conf_middleware_hul24_b200.serve import ClientTiming, MenosExecutor, ServeLoop, client_demands
    w = _workload()
    n_iters = 3
    inputs, per_iter = _iter_inputs(w, n_iters)
    weights, adapters, io = inputs

    # ---- scheduled run: memory for about two backwards at a time
    srv = new_server(w, weights, arena_bytes=64 << 20)
    ids = register(srv, w, adapters)
    dem = {i: client_demands(srv, ids[i], w.clients[i].n_tokens) for i in range(len(w.clients))}
    total = int(2.2 * max(mb for _, mb in dem.values()))
    assert total <= srv.stats()["arena_bytes"]
    sched = M.Scheduler(total, 16)
    for i, (mf, mb) in dem.items():
        sched.set_demand(i, mf, mb)
    timings = {i: ClientTiming(1e-3 * (1 + i % 3), 2e-3 * (1 + (i * 7) % 4)) for i in range(len(w.clients))}
    ex = MenosExecutor(srv, {i: ids[i] for i in range(len(w.clients))}, per_iter,
                       cost=lambda kind, toks: (2e-5 if kind == M.REQ_FWD else 6e-5) * toks + 1e-3)
    loop = ServeLoop(sched, ex, timings, n_iters).run()
    torch.cuda.synchronize()
    assert set(loop.finish) == set(range(len(w.clients)))
    assert any(len(x.clients) > 1 for x in loop.waves), "no batched wave formed"
    assert {x.kind for x in loop.waves} == {M.REQ_FWD, M.REQ_BWD}
    # the additive per-client bounds cover every wave's exact demand
    for (kind, cl, exact), wave in zip(ex.exact, loop.waves):
        assert wave.clients == cl and exact <= wave.reserved, (kind, cl, exact, wave.reserved)
    assert srv.stats()["arena_peak"] <= total   # the scheduler's accounting held on the real arena
    sched_ad = _adapters(srv, w, ids)
    srv.close()

    # ---- each client alone, iteration by iteration (SAVE forward + backward + step)
    srv = new_server(w, weights, arena_bytes=64 << 20)
    ids = register(srv, w, adapters)
    for i, c in enumerate(w.clients):
        for k in range(n_iters):
            lens, x, g = per_iter[i][k]
            xs, gs = torch.empty_like(x), torch.empty_like(g)
            b = srv.forward([ids[i]] * len(lens), lens, x, xs)
            srv.backward(b, g, gs)
            srv.adapter_step([ids[i]])
            torch.cuda.synchronize()
            assert torch.equal(xs, ex.x_s[(i, k)]), (i, k)
            assert torch.equal(gs, ex.g_s[(i, k)]), (i, k)
    alone_ad = _adapters(srv, w, ids)
    srv.close()
    for key in sched_ad:
        assert np.array_equal(sched_ad[key], alone_ad[key]), key

    # ---- iteration 0 against the oracle
    ora = run_oracle_step(w, inputs=inputs)
    for i in range(len(w.clients)):
        assert act_err(ex.x_s[(i, 0)].float().cpu().numpy(), ora["x_s"][i]) <= 2e-2
        assert cosine(ex.g_s[(i, 0)].float().cpu().numpy(), ora["g_s"][i]) >= 0.999


def test_mem_bound_is_additive_over_random_partitions():
    """menos_batch_memory(MENOS_MEM_BOUND) per client sums to at least the exact demand of any batch."""
    import random
    from paper_conf_middleware_hul24_b200 import menos as M
    w = _workload()
    weights, adapters, _ = make_inputs(w, seed=4)
    srv = new_server(w, weights, arena_bytes=64 << 20)
    ids = register(srv, w, adapters)
    rng = random.Random(1)
    for _ in range(200):
        k = rng.randint(1, len(ids))
        sub = rng.sample(range(len(ids)), k)
        toks = [rng.randint(1, 4096) for _ in sub]
        for flags in (M.FWD_SAVE, M.FWD_NOGRAD):
            ef, eb = srv.batch_memory([ids[i] for i in sub], toks, flags)
            bf = sum(srv.batch_memory([ids[i]], [t], flags | M.MEM_BOUND)[0] for i, t in zip(sub, toks))
            bb = sum(srv.batch_memory([ids[i]], [t], flags | M.MEM_BOUND)[1] for i, t in zip(sub, toks))
            assert ef <= bf and eb <= bb
    srv.close()
