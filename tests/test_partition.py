"""Host logic of the multi-GPU replica path: LPT client partitioning (deterministic on every rank, each client
exactly once) and the max-over-ranks timing reduction, exercised with torch.distributed gloo, world_size 2."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_middleware_hul24_b200.partition import lpt_partition, workload_partition
from workloads import workload


def test_lpt_properties():
    costs = [5, 3, 3, 2, 2, 2, 1]
    bins = lpt_partition(costs, 3)
    assert sorted(i for b in bins for i in b) == list(range(len(costs)))
    loads = [sum(costs[i] for i in b) for b in bins]
    assert max(loads) - min(loads) <= max(costs)
    assert lpt_partition(costs, 1) == [list(range(len(costs)))]
    assert lpt_partition([1, 1], 2) == [[0], [1]]            # ties -> lower GPU index first


def test_cfg2_partition_balanced():
    w = workload("cfg2_7b_x32_ragged")
    for n in (1, 2, 4, 8):
        bins = workload_partition(w, n)
        assert sorted(i for b in bins for i in b) == list(range(32))
        toks = [sum(w.clients[i].n_tokens for i in b) for b in bins]
        assert max(toks) <= 1.15 * (sum(toks) / n) + 4096


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    w = workload("cfg2_7b_x32_ragged")
    mine = workload_partition(w, world)[rank]
    gathered = [None] * world
    dist.all_gather_object(gathered, mine)
    t = torch.tensor([10.0 + rank])                      # per-rank device time -> max over ranks
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    q.put((rank, gathered, float(t.item())))
    dist.destroy_process_group()


def test_gloo_two_ranks_agree_and_cover_all_clients():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    g0, g1 = res[0][1], res[1][1]
    assert g0 == g1
    assert sorted(i for b in g0 for i in b) == list(range(32))
    assert all(r[2] == 11.0 for r in res)


def test_plan_waves():
    from paper_conf_middleware_hul24_b200.partition import plan_waves
    assert plan_waves([10, 10, 10], [1, 1, 1], 100) == [[0, 1, 2]]
    assert plan_waves([40, 40, 40], [5, 5, 5], 100) == [[0, 1], [2]]
    assert plan_waves([90, 5], [5, 1], 96) == [[0], [1]]
    with pytest.raises(MemoryError):
        plan_waves([200], [1], 100)


def test_plan_waves_exact_uses_joint_demand():
    from paper_conf_middleware_hul24_b200.partition import plan_waves_exact
    # joint demand grows faster than the sum (block-diagonal slot columns span the wave)
    sizes = [10, 10, 10, 10]
    demand = lambda idx: sum(sizes[i] for i in idx) + 5 * len(idx) ** 2
    waves = plan_waves_exact(4, demand, 60)
    assert waves == [[0, 1], [2, 3]]
    assert all(demand(w) <= 60 for w in waves)
    assert sorted(i for w in waves for i in w) == [0, 1, 2, 3]
    with pytest.raises(MemoryError):
        plan_waves_exact(1, lambda idx: 100, 60)
