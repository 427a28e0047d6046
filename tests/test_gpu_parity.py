"""End-to-end GPU parity through the C-ABI (libmenos.so) against the CPU oracle, plus the invariants the
BASELINE.json north_star names: (b) zero-B == base, (c) batched == alone, (d) the base is never modified.

Bars (BASELINE.json north_star; DESIGN.md §"Tolerances"): activations max|d|/max|ref| <= 2e-2, cosine >= 0.999
on every gradient tensor (g_s, every dA, dB).  Invariants (b), (c), re-forward (NEXT-1) are BITWISE on the GPU.
"""
import dataclasses

import numpy as np
import pytest

from tests.parity_util import (compare_step, make_inputs, new_server, register, run_gpu_step, run_oracle_step)
from workloads import ClientCfg, MODELS, TARGETS, Workload, workload

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def assert_report(rep):
    bad = {k: v for k, v in rep.items() if not v["ok"]}
    assert not bad, bad


def test_cfg0_tiny_parity():
    w = workload("cfg0_tiny")
    rep = compare_step(run_gpu_step(w, seed=0), run_oracle_step(w, seed=0))
    assert_report(rep)


def test_tiny_all_targets_gqa_ragged_mixed_ranks():
    m = dataclasses.replace(MODELS["tiny"], n_heads=4, n_kv_heads=2)
    cl = [ClientCfg(4, 8.0, TARGETS, [1, 17, 3]), ClientCfg(16, 32.0, ("q", "v"), [129]),
          ClientCfg(8, 16.0, ("k", "o", "gate", "up", "down"), [64, 40]), ClientCfg(5, 10.0, ("v", "down"), [200])]
    w = Workload("tiny_mix", m, cl)
    rep = compare_step(run_gpu_step(w, seed=3), run_oracle_step(w, seed=3))
    assert_report(rep)


def test_tiny_ranks_above_16():
    """Ranks 24 and 32: the fused dU + dB kernel runs two 16-wide rank tiles per slab, and a q|k|v slot of 96
    columns takes the one-pass dA over two 64-row tiles (three output segments)."""
    m = dataclasses.replace(MODELS["tiny"], n_heads=4, n_kv_heads=2)
    cl = [ClientCfg(32, 64.0, ("q", "v", "gate", "up"), [33, 90]), ClientCfg(24, 48.0, TARGETS, [57]),
          ClientCfg(4, 8.0, ("v",), [16])]
    w = Workload("tiny_big_rank", m, cl)
    inputs = make_inputs(w, seed=11)
    srv = new_server(w, inputs[0], max_rank=64)
    ids = register(srv, w, inputs[1])
    rep = compare_step(run_gpu_step(w, inputs=inputs, srv=srv, ids=ids), run_oracle_step(w, inputs=inputs))
    srv.close()
    assert_report(rep)


def test_zero_b_equals_base_bitwise():
    """Invariant (b): with B = 0 the LoRA contribution is exactly zero, whatever the targets."""
    m = MODELS["tiny"]
    cl = [ClientCfg(4, 8.0, ("q", "v"), [20, 12]), ClientCfg(8, 16.0, TARGETS, [20, 12])]
    w = Workload("zb", m, cl)
    weights, adapters, io = make_inputs(w, seed=5, zero_b=True)
    io[1] = io[0]  # same inputs for both clients
    out = run_gpu_step(w, inputs=(weights, adapters, io), grads=False)
    assert np.array_equal(out["x_s"][0], out["x_s"][1])
    ora = run_oracle_step(w, inputs=(weights, [[{} for _ in range(m.n_layers)]] * 2, io))
    from tests.parity_util import act_err
    assert act_err(out["x_s"][0], ora["x_s"][0]) < 2e-2


def test_batched_equals_alone_bitwise():
    """Invariant (c): a client's outputs and grads do not depend on who shares the batch."""
    m = MODELS["tiny"]
    # slot widths differ per group (the tcgen05 shrink's MMA N follows the widest client of the batch) and one rank
    # is above 16 (its dU + dB problems take the mma.sync kernel, the others the tcgen05 one)
    cl = [ClientCfg(4, 8.0, ("q", "v"), [50, 30]), ClientCfg(16, 32.0, ("q", "v", "o"), [100]),
          ClientCfg(8, 16.0, ("q", "v", "down"), [7, 70]), ClientCfg(16, 32.0, TARGETS, [45]),
          ClientCfg(24, 48.0, ("q", "k", "v", "gate"), [33])]
    w = Workload("bva", m, cl)
    inputs = make_inputs(w, seed=7)
    weights, adapters, io = inputs
    srv = new_server(w, weights, max_rank=32)
    ids = register(srv, w, adapters)
    full = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids)
    for i in range(len(cl)):
        wi = Workload("alone", m, [cl[i]])
        alone = run_gpu_step(wi, inputs=(weights, [adapters[i]], [io[i]]), srv=srv, ids=[ids[i]])
        assert np.array_equal(alone["x_s"][0], full["x_s"][i]), i
        assert np.array_equal(alone["g_s"][0], full["g_s"][i]), i
        for l in range(m.n_layers):
            for t in cl[i].targets:
                assert np.array_equal(alone["grads"][0][l][t][0], full["grads"][i][l][t][0]), (i, l, t)
                assert np.array_equal(alone["grads"][0][l][t][1], full["grads"][i][l][t][1]), (i, l, t)
    srv.close()


def test_base_unchanged_and_repeatable():
    """Invariant (d): no base gradient exists; after fwd+bwd+step the same call reproduces bit-identical
    outputs for unchanged adapters (the shared base is read-only)."""
    w = workload("cfg0_tiny")
    inputs = make_inputs(w, seed=9)
    weights, adapters, io = inputs
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    a = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids, grads=False)
    srv.adapter_step(ids)
    register_again = [srv.set_adapter(ids[i], l, t, wh, adapters[i][l][t][0 if wh == "A" else 1])
                      for i in range(len(ids)) for l in range(w.model.n_layers) for t in w.clients[i].targets
                      for wh in ("A", "B")]
    del register_again
    b = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids, grads=False)
    for i in range(len(ids)):
        assert np.array_equal(a["x_s"][i], b["x_s"][i])
        assert np.array_equal(a["g_s"][i], b["g_s"][i])
    st = srv.stats()
    assert st["base_bytes"] > 0
    srv.close()


def test_nograd_reforward_bitwise_equals_save():
    """NEXT-1 (Alg.1 L6/L10): NOGRAD forward + re-forward backward == SAVE mode, bitwise."""
    m = MODELS["tiny"]
    cl = [ClientCfg(4, 8.0, ("q", "v"), [33, 31]), ClientCfg(8, 16.0, TARGETS, [64])]
    w = Workload("ng", m, cl)
    inputs = make_inputs(w, seed=11)
    weights, adapters, io = inputs
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    a = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids, flags=0)
    b = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids, flags=1)
    for i in range(len(cl)):
        assert np.array_equal(a["x_s"][i], b["x_s"][i])
        assert np.array_equal(a["g_s"][i], b["g_s"][i])
        for l in range(m.n_layers):
            for t in cl[i].targets:
                assert np.array_equal(a["grads"][i][l][t][0], b["grads"][i][l][t][0])
                assert np.array_equal(a["grads"][i][l][t][1], b["grads"][i][l][t][1])
    srv.close()


def test_adamw_step_matches_oracle():
    from oracle import menos_oracle as O
    w = workload("cfg0_tiny")
    inputs = make_inputs(w, seed=13)
    weights, adapters, io = inputs
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    for step in range(1, 3):
        got = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids)
        before = {(i, l, t, wh): srv.get_adapter(ids[i], l, t, wh)
                  for i in range(len(ids)) for l in range(w.model.n_layers) for t in w.clients[i].targets
                  for wh in ("A", "B", "mA", "mB", "vA", "vB")}
        srv.adapter_step(ids)
        torch.cuda.synchronize()
        for i in range(len(ids)):
            for l in range(w.model.n_layers):
                for t in w.clients[i].targets:
                    for wh, gi in (("A", 0), ("B", 1)):
                        g = got["grads"][i][l][t][gi]
                        p, m_, v_ = O.adamw_step(before[(i, l, t, wh)], g, before[(i, l, t, "m" + wh)],
                                                 before[(i, l, t, "v" + wh)], step, 1e-4, 0.9, 0.999, 1e-8, 0.01)
                        np.testing.assert_allclose(srv.get_adapter(ids[i], l, t, wh), p, rtol=1e-5, atol=1e-7)
                        np.testing.assert_allclose(srv.get_adapter(ids[i], l, t, "m" + wh), m_, rtol=1e-5,
                                                   atol=1e-9)
                        np.testing.assert_allclose(srv.get_adapter(ids[i], l, t, "v" + wh), v_, rtol=1e-5,
                                                   atol=1e-12)
                        assert not np.any(srv.get_adapter(ids[i], l, t, "d" + wh))  # consumed and zeroed
    srv.close()


def test_enomem_returned_not_crash():
    from paper_conf_middleware_hul24_b200 import MenosError
    w = workload("cfg0_tiny")
    weights, adapters, io = make_inputs(w, seed=15)
    srv = new_server(w, weights, arena_bytes=64 * 1024)
    ids = register(srv, w, adapters)
    x = torch.zeros(64, 64, dtype=torch.bfloat16, device="cuda")
    with pytest.raises(MenosError) as e:
        srv.forward([ids[0]] * 2 + [ids[1]] * 2, [16] * 4, x, torch.empty_like(x))
    assert e.value.code == -2
    srv.close()


@pytest.mark.parametrize("flags", [0, 1])
def test_batch_memory_is_exact_bound(flags):
    """menos_batch_memory (the admission query, Alg.2 L2 PAPER.md:238): an arena of max(fwd, bwd) bytes runs the
    batch (SAVE, or NOGRAD + re-forward) and the observed arena peak P stays below it, with at most the metadata
    bound (<= 4 MB here) of slack; an arena just below P is refused with ENOMEM (never a crash)."""
    from paper_conf_middleware_hul24_b200 import MenosError
    m = MODELS["tiny"]
    cl = [ClientCfg(4, 8.0, ("q", "v"), [33, 60]), ClientCfg(16, 32.0, TARGETS, [100]), ClientCfg(8, 16.0, ("o", "down"), [7])]
    w = Workload("bm", m, cl)
    inputs = make_inputs(w, seed=21)
    weights, adapters, io = inputs
    x = torch.from_numpy(np.concatenate([a for a, _ in io])).to(torch.bfloat16).cuda()

    def run(cap):
        srv = new_server(w, weights, arena_bytes=cap)
        ids = register(srv, w, adapters)
        sc, sl = [], []
        for i, c in enumerate(cl):
            sc += [ids[i]] * len(c.seq_lens)
            sl += list(c.seq_lens)
        need = max(srv.batch_memory(ids, [c.n_tokens for c in cl], flags))
        try:
            b = srv.forward(sc, sl, x, torch.empty_like(x), flags=flags)
            srv.backward(b, x, torch.empty_like(x))
            torch.cuda.synchronize()
            return need, srv.stats()["arena_peak"], None
        except MenosError as e:
            return need, None, e
        finally:
            srv.close()

    need, _, _ = run(1 << 30)
    need2, peak, err = run(need)
    assert err is None and need2 == need
    assert peak <= need <= peak + (4 << 20)
    _, _, err = run(peak - 4096)
    assert err is not None and err.code == -2


def test_batch_memory_bounds_the_ds_stored_backward():
    """head_dim 128: the demand menos_batch_memory reports includes the dS^T chunk buffer's bound (the sequence
    lengths are not part of the query): an arena of exactly that many bytes runs the SAVE and the NOGRAD step, and the
    observed peak stays below it."""
    from workloads.synth import ModelCfg
    m = ModelCfg("hd128", 512, 4, 2, 1024, 2, model_layers=3)
    cl = [ClientCfg(8, 16.0, ("q", "v"), [300, 1, 129]), ClientCfg(16, 32.0, TARGETS, [700])]
    w = Workload("bm128", m, cl)
    inputs = make_inputs(w, seed=23)
    weights, adapters, io = inputs
    x = torch.from_numpy(np.concatenate([a for a, _ in io])).to(torch.bfloat16).cuda()
    for flags in (0, 1):
        srv = new_server(w, weights, arena_bytes=1 << 30)
        ids = register(srv, w, adapters)
        need = max(srv.batch_memory(ids, [c.n_tokens for c in cl], flags))
        srv.close()
        srv = new_server(w, weights, arena_bytes=need)
        ids = register(srv, w, adapters)
        sc, sl = [], []
        for i, c in enumerate(cl):
            sc += [ids[i]] * len(c.seq_lens)
            sl += list(c.seq_lens)
        b = srv.forward(sc, sl, x, torch.empty_like(x), flags=flags)
        srv.backward(b, x, torch.empty_like(x))
        torch.cuda.synchronize()
        assert srv.stats()["arena_peak"] <= need
        srv.close()


def test_host_buffers_e2e_path():
    """x_c / g_c given as (pinned) host buffers: same results as device buffers."""
    w = workload("cfg0_tiny")
    inputs = make_inputs(w, seed=17)
    weights, adapters, io = inputs
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    dev_out = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids, grads=False)
    x = torch.from_numpy(np.concatenate([a for a, _ in io])).to(torch.bfloat16).pin_memory()
    g = torch.from_numpy(np.concatenate([b for _, b in io])).to(torch.bfloat16).pin_memory()
    xs, gs = torch.empty_like(x).pin_memory(), torch.empty_like(g).pin_memory()
    b = srv.forward([ids[0]] * 2 + [ids[1]] * 2, [16] * 4, x, xs)
    srv.backward(b, g, gs)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(xs.float().numpy(), np.concatenate(dev_out["x_s"]))
    np.testing.assert_array_equal(gs.float().numpy(), np.concatenate(dev_out["g_s"]))
    srv.close()


def test_interleaved_save_batches_bitwise():
    """Two SAVE batches of different sizes outstanding at once (forward A, forward B, backward A, backward B):
    the per-call scratch block moves in between, and A's backward must still equal A run alone (bitwise)."""
    m = MODELS["tiny"]
    wa = Workload("a", m, [ClientCfg(4, 8.0, ("q", "v", "down"), [30, 9])])
    wb = Workload("b", m, [ClientCfg(8, 16.0, TARGETS, [200, 77])])
    ia, ib = make_inputs(wa, seed=31), make_inputs(wb, seed=32)
    ib = (ia[0], ib[1], ib[2])   # one shared base
    ref_a, ref_b = run_gpu_step(wa, inputs=ia), run_gpu_step(wb, inputs=ib)
    w = Workload("ab", m, wa.clients + wb.clients)
    srv = new_server(w, ia[0])
    ids = register(srv, w, ia[1] + ib[1])
    from tests.parity_util import _bf16
    xa, ga = (_bf16(np.concatenate([a for a, _ in ia[2]]), "cuda"), _bf16(np.concatenate([g for _, g in ia[2]]), "cuda"))
    xb, gb = (_bf16(np.concatenate([a for a, _ in ib[2]]), "cuda"), _bf16(np.concatenate([g for _, g in ib[2]]), "cuda"))
    xsa, gsa, xsb, gsb = (torch.empty_like(t) for t in (xa, ga, xb, gb))
    ba = srv.forward([ids[0]] * 2, [30, 9], xa, xsa)
    bb = srv.forward([ids[1]] * 2, [200, 77], xb, xsb)
    srv.backward(ba, ga, gsa)
    srv.backward(bb, gb, gsb)
    torch.cuda.synchronize()
    assert np.array_equal(xsa.float().cpu().numpy(), ref_a["x_s"][0])
    assert np.array_equal(gsa.float().cpu().numpy(), ref_a["g_s"][0])
    assert np.array_equal(xsb.float().cpu().numpy(), ref_b["x_s"][0])
    assert np.array_equal(gsb.float().cpu().numpy(), ref_b["g_s"][0])
    for l in range(m.n_layers):
        for t in ("q", "v", "down"):
            assert np.array_equal(srv.get_adapter(ids[0], l, t, "dA"), ref_a["grads"][0][l][t][0])
    srv.close()


def test_attention_ds_chunking_end_to_end():
    """The dS-stored attention backward through the server: parity vs the oracle on a head_dim-128 GQA model with
    ragged sequences; a chunk budget far below the batch's dS^T tiles (several (sequence, kv head) chunks, one
    buffer) gives bitwise the same step; the recompute path (mode 14) also meets the bars."""
    from paper_conf_middleware_hul24_b200.menos import check, lib
    from workloads.synth import ModelCfg
    m = ModelCfg("hd128", 512, 4, 2, 1024, 2, model_layers=3)
    cl = [ClientCfg(8, 16.0, ("q", "v"), [300, 129]), ClientCfg(16, 32.0, TARGETS, [700, 17, 1]),
          ClientCfg(4, 8.0, ("k", "o", "down"), [64])]
    w = Workload("hd128_ds", m, cl)
    inputs = make_inputs(w, seed=41)
    ora = run_oracle_step(w, inputs=inputs)
    try:
        full = run_gpu_step(w, inputs=inputs)
        assert_report(compare_step(full, ora))
        check(lib().menos_test_set_ds_cap(80), testing=True)    # 700-token unit = 2 x 36 tiles; several chunks
        chunked = run_gpu_step(w, inputs=inputs)
        for i in range(len(cl)):
            assert np.array_equal(full["x_s"][i], chunked["x_s"][i]) and np.array_equal(full["g_s"][i], chunked["g_s"][i])
            for l, d in enumerate(full["grads"][i]):
                for t, (dA, dB) in d.items():
                    assert np.array_equal(chunked["grads"][i][l][t][0], dA) and np.array_equal(chunked["grads"][i][l][t][1], dB)
        check(lib().menos_test_set_attn_tc(14), testing=True)   # recompute path
        assert_report(compare_step(run_gpu_step(w, inputs=inputs), ora))
    finally:
        check(lib().menos_test_set_ds_cap(32768), testing=True)
        check(lib().menos_test_set_attn_tc(78), testing=True)
