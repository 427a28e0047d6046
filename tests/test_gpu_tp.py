"""Tensor-parallel server segment on the GPU (include/menos.h menos_tp_cfg), checked
against the UNSHARDED CPU oracle.

Several ranks share cuda:0 (the only GPU a test box has; NCCL refuses two ranks on one GPU): each process creates its
own libmenos server shard with tp = (rank, world, torch.distributed collective over gloo), loads its weight / adapter
shards (paper_conf_middleware_hul24_b200.tp), and runs forward(SAVE or NOGRAD) + backward + adapter_step.  The
library runs the sequence-parallel schedule: bf16 all-gathers of the norm outputs / incoming gradients and bf16
reduce-scatters of the row-parallel partial sums (8 per layer), plus one fp32 all-reduce of the replicated adapters'
gradients per client per backward; everything else runs in its kernels.  The NCCL transport (the library drives
NCCL itself from a broadcast unique id) is exercised at world 1 on one GPU.  Bars as in test_gpu_parity.py:
activations max|d|/max|ref| <= 2e-2, cosine >= 0.999 on every gradient tensor (gathered over the shards).
"""
import os
import socket

import numpy as np
import pytest

from tests.parity_util import ACT_TOL, COS_TOL, act_err, cosine, make_inputs
from workloads import ClientCfg, ModelCfg, TARGETS, Workload

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, wl, flags, q, transport="gloo"):
    import torch.distributed as dist
    from paper_conf_middleware_hul24_b200 import Server
    from paper_conf_middleware_hul24_b200 import tp as TP
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        m = wl.model
        hd = m.head_dim
        weights, adapters, io = make_inputs(wl, seed=11)
        shards = []
        for W in weights:
            Ws = TP.shard_layer_weights(W, rank, world, m.n_heads, m.n_kv_heads, hd, m.d_ff)
            shards.append({k: torch.from_numpy(np.ascontiguousarray(v)).to(torch.bfloat16).cuda() for k, v in Ws.items()})
        del weights
        if transport == "nccl":   # the library drives NCCL itself from rank 0's unique id (broadcast here)
            uid = [TP.nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(uid, src=0)
            tpc = (rank, world, uid[0])
        else:
            tpc = (rank, world, TP.make_torch_collective())
        srv = Server(m.d_model, m.n_heads, m.n_kv_heads, m.d_ff, m.n_layers, first_layer=m.first_layer,
                     weights=shards, max_rank=16, max_seq_len=1024, arena_bytes=1 << 30, tp=tpc)
        ids = []
        for i, c in enumerate(wl.clients):
            cid = srv.register_client(c.rank, c.alpha, c.targets, seed=i)
            for l, d in enumerate(adapters[i]):
                for t, (A, B) in d.items():
                    A_l, B_l = TP.shard_adapter(t, A, B, rank, world, m.n_heads, m.n_kv_heads, hd, m.d_ff)
                    srv.set_adapter(cid, l, t, "A", A_l)
                    srv.set_adapter(cid, l, t, "B", B_l)
            ids.append(cid)
        seq_client, seq_len = [], []
        for i, c in enumerate(wl.clients):
            seq_client += [ids[i]] * len(c.seq_lens)
            seq_len += list(c.seq_lens)
        x = torch.from_numpy(np.concatenate([a for a, _ in io])).to(torch.bfloat16).cuda()
        g = torch.from_numpy(np.concatenate([b for _, b in io])).to(torch.bfloat16).cuda()
        xs, gs = torch.empty_like(x), torch.empty_like(x)
        b = srv.forward(seq_client, seq_len, x, xs, flags=flags)
        srv.backward(b, g, gs)
        torch.cuda.synchronize()
        grads = [[{t: (srv.get_adapter(ids[i], l, t, "dA"), srv.get_adapter(ids[i], l, t, "dB")) for t in c.targets}
                  for l in range(m.n_layers)] for i, c in enumerate(wl.clients)]
        srv.adapter_step(ids)
        torch.cuda.synchronize()
        params = [[{t: (srv.get_adapter(ids[i], l, t, "A"), srv.get_adapter(ids[i], l, t, "B")) for t in c.targets}
                   for l in range(m.n_layers)] for i, c in enumerate(wl.clients)]
        q.put((rank, xs.float().cpu().numpy(), gs.float().cpu().numpy(), grads, params, srv.tp_stats()))
        srv.close()
    except Exception as e:  # surface the failure to the parent instead of hanging it
        import traceback
        q.put((rank, "error", traceback.format_exc(), repr(e), None))
    finally:
        dist.destroy_process_group()


def _run(wl, flags=0, world=2, transport="gloo"):
    import gc
    import torch.multiprocessing as mp
    gc.collect()                 # the workers share this GPU: release what earlier tests left in this process
    torch.cuda.empty_cache()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, wl, flags, q, transport)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=1200) for _ in procs], key=lambda r: r[0])
    for p in procs:
        p.join(timeout=120)
    for r in res:
        assert not (isinstance(r[1], str) and r[1] == "error"), r[2]
    return res


def _check(wl, res, world=2, flags=0):
    from oracle import menos_oracle as O
    from paper_conf_middleware_hul24_b200 import tp as TP
    m = wl.model
    weights, adapters, io = make_inputs(wl, seed=11)
    # sequence-parallel exchanges: per layer 4 all-gathers + 4 reduce-scatters of bf16 [T, d] (fwd + bwd), 2 more
    # all-gathers for x_s / g_s, one fp32 all-reduce per client of the replicated adapter gradients
    if world > 1:
        st = res[0][5]
        per_layer = 8 if flags == 0 else 12   # NOGRAD: the forward's exchanges again in the backward's re-forward
        assert st["calls"] == per_layer * m.n_layers + 2 + len(wl.clients), st
    for r in range(1, world):          # replicated outputs are bitwise identical on every rank
        assert np.array_equal(res[r][1], res[0][1])
        assert np.array_equal(res[r][2], res[0][2])
    off = 0
    bad = {}
    for i, c in enumerate(wl.clients):
        xs, gs, gr = O.client_step(io[i][0], io[i][1], c.seq_lens, weights, adapters[i], c.alpha / c.rank, m)
        T = c.n_tokens
        e = act_err(res[0][1][off:off + T], xs)
        if e > ACT_TOL:
            bad[f"c{i}.x_s"] = e
        cg = cosine(res[0][2][off:off + T], gs)
        if cg < COS_TOL:
            bad[f"c{i}.g_s"] = cg
        off += T
        for l in range(m.n_layers):
            for t in c.targets:
                dA, dB = TP.gather_adapter(t, [res[r][3][i][l][t] for r in range(world)])
                for nm, a, ref in (("dA", dA, gr[l][t][0]), ("dB", dB, gr[l][t][1])):
                    cs = cosine(a, ref)
                    if cs < COS_TOL:
                        bad[f"c{i}.L{l}.{t}.{nm}"] = cs
                # replicated parameters stay identical across ranks after AdamW
                k = 0 if t in TP.COLUMN_PARALLEL else 1
                for r in range(1, world):
                    assert np.array_equal(res[r][4][i][l][t][k], res[0][4][i][l][t][k]), (i, l, t)
    assert not bad, bad


MODEL_HD64 = ModelCfg("tp-gqa-hd64", 256, 4, 2, 344, 2, model_layers=3)
MODEL_70B_LIKE = ModelCfg("tp-70b-like", 1024, 8, 2, 2816, 2, model_layers=80)   # hd 128, GQA 4:1 like 70B


def test_tp2_all_targets_gqa_hd64():
    wl = Workload("tp_hd64", MODEL_HD64, [ClientCfg(4, 8.0, TARGETS, [33, 7]), ClientCfg(8, 16.0, ("q", "v"), [64])])
    _check(wl, _run(wl))


def test_tp2_70b_like_hd128_qv_and_nograd():
    wl = Workload("tp_hd128", MODEL_70B_LIKE,
                  [ClientCfg(8, 16.0, ("q", "v"), [300, 129]), ClientCfg(16, 32.0, ("q", "v", "o", "down"), [256])])
    _check(wl, _run(wl))
    _check(wl, _run(wl, flags=1), flags=1)   # MENOS_FWD_NOGRAD: the re-forward inside backward exchanges the same way


def test_tp8_at_llama2_70b_width():
    """BASELINE configs[4] shard shapes: Llama-2-70B widths (d 8192, 64 heads of 128, 8 KV heads, f 28672) split 8
    ways, so every rank holds 8 query heads, 1 KV head and f/8 = 3584 (the cfg4 per-GPU shapes); 2 layers, two clients
    (q,v r=8 and q,v,o,down r=16), T = 407 tokens (not a multiple of 8: the last rank's padding rows are exercised)."""
    m = ModelCfg("llama2-70b-2l", 8192, 64, 8, 28672, 2, model_layers=80)
    wl = Workload("tp8_70b", m, [ClientCfg(8, 16.0, ("q", "v"), [200, 57]),
                                 ClientCfg(16, 32.0, ("q", "v", "o", "down"), [150])])
    _check(wl, _run(wl, world=8), world=8)


def test_nccl_transport_world1():
    """The library-driven NCCL path (menos_tp_unique_id -> menos_tp_cfg.nccl_id -> ncclCommInitRank) running the
    sequence-parallel schedule at world 1 on the one GPU: results match the oracle like every other configuration."""
    wl = Workload("tp_nccl1", MODEL_70B_LIKE,
                  [ClientCfg(8, 16.0, ("q", "v"), [100, 29]), ClientCfg(16, 32.0, ("q", "v", "o", "down"), [64])])
    _check(wl, _run(wl, world=1, transport="nccl"), world=1)
