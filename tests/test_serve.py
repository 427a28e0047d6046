"""Host logic of the serving loop (Alg.1 driven by Alg.2; paper_conf_middleware_hul24_b200/serve.py) with a fake
executor on a fake clock: no GPU.  The loop with the native scheduler makes exactly the waves the loop makes with
the oracle scheduler (oracle/menos_sched.py), every client runs its iterations in Alg.1 order, the GPU timeline
never overlaps, and the memory reserved by running tasks never exceeds M_avail."""
import random

from oracle.menos_sched import OracleScheduler
from paper_conf_middleware_hul24_b200 import menos as M
from paper_conf_middleware_hul24_b200.serve import ClientTiming, ServeLoop


class FakeExecutor:
    def __init__(self, toks):
        self.toks, self.log = toks, []

    def forward_wave(self, clients, its):
        self.log.append(("F", tuple(clients), tuple(its[c] for c in clients)))
        return 1e-4 * sum(self.toks[c] for c in clients) + 2e-3

    def backward_wave(self, clients, its):
        self.log.append(("B", tuple(clients), tuple(its[c] for c in clients)))
        return 3.5e-4 * sum(self.toks[c] for c in clients) + 5e-3


class OracleAdapter:
    """The oracle scheduler behind the native binding's interface."""

    def __init__(self, total):
        self.o = OracleScheduler(total)

    def set_demand(self, c, mf, mb):
        self.o.set_demand(c, mf, mb)

    def arrive(self, c, k):
        return self.o.arrive(c, k)

    def complete(self, c):
        return self.o.complete(c)


def _setup(seed):
    rng = random.Random(seed)
    n = rng.randint(2, 12)
    toks = {c: rng.randint(128, 1024) * 4 for c in range(n)}
    per_tok_f, per_tok_b = 50, 1000
    demands = {c: (per_tok_f * t + 4096, per_tok_b * t + 65536) for c, t in toks.items()}
    total = max(mb for _, mb in demands.values()) * rng.choice([1, 2, 3]) + rng.randint(0, 10 ** 6)
    timings = {c: ClientTiming(rng.uniform(0.01, 0.5), rng.uniform(0.05, 1.0)) for c in toks}
    return toks, demands, total, timings


def _loop(sched, toks, demands, timings, n_iters):
    for c, (mf, mb) in demands.items():
        sched.set_demand(c, mf, mb)
    ex = FakeExecutor(toks)
    return ServeLoop(sched, ex, timings, n_iters).run(), ex


def test_native_loop_equals_oracle_loop():
    for seed in range(40):
        toks, demands, total, timings = _setup(seed)
        a, exa = _loop(M.Scheduler(total, 16), toks, demands, timings, 3)
        b, exb = _loop(OracleAdapter(total), toks, demands, timings, 3)
        assert exa.log == exb.log, seed
        assert [(w.kind, w.clients, w.start, w.end) for w in a.waves] == \
               [(w.kind, w.clients, w.start, w.end) for w in b.waves]


def test_loop_alg1_order_memory_and_timeline():
    for seed in range(40):
        toks, demands, total, timings = _setup(100 + seed)
        loop, ex = _loop(M.Scheduler(total, 16), toks, demands, timings, 3)
        # every client completes every iteration: F(k) then B(k), k = 0..n-1
        seen = {c: [] for c in toks}
        for kind, cl, its in ex.log:
            for c, k in zip(cl, its):
                seen[c].append((kind, k))
        for c in toks:
            assert seen[c] == [(x, k) for k in range(3) for x in ("F", "B")], (seed, c)
        assert set(loop.finish) == set(toks)
        # the GPU runs one wave at a time
        for w0, w1 in zip(loop.waves, loop.waves[1:]):
            assert w1.start >= w0.end - 1e-12
        # memory reserved by the tasks holding it (granted .. completed) at any grant <= M_avail (Alg.2 L18-20)
        tasks = [(tg, x.end, b) for x in loop.waves for _, tg, b in x.tasks]
        for t0, _, _ in tasks:
            assert sum(b for tg, te, b in tasks if tg <= t0 < te) <= total


def test_memory_pressure_serialises_backwards_and_backfills_forwards():
    """Room for one backward at a time: no two BWD waves overlap, and forwards of other
    clients are granted while a backward runs."""
    toks = {c: 512 for c in range(4)}
    demands = {c: (10, 100) for c in toks}
    timings = {c: ClientTiming(0.001 * (c + 1), 0.001) for c in toks}
    loop, ex = _loop(M.Scheduler(115, 8), toks, demands, timings, 2)
    bw = [w for w in loop.waves if w.kind == M.REQ_BWD]
    assert len(bw) == 8 and all(len(w.clients) == 1 for w in bw)
    for a, b in zip(bw, bw[1:]):
        assert b.granted >= a.end - 1e-12           # the next backward is granted only when the last completes
    # forwards granted while a backward holds its memory (backfilling / FCFS head fits in the 15 B left)
    fw_during = [w for w in loop.waves if w.kind == M.REQ_FWD and any(b.granted <= w.granted < b.end for b in bw)]
    assert any(len(w.clients) > 1 for w in loop.waves)
    assert fw_during
    assert set(loop.finish) == set(toks)
