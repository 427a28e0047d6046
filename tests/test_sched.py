"""Algorithm 2 scheduler (§4.2): the oracle pinned to hand-worked
traces of the paper's prose and to invariants checked by brute force; the native scheduler (libmenos.so,
csrc/sched.cpp; host-only, no GPU needed) bit-exact against the oracle on random traces; decision latency."""
import json
import os
import random

import pytest

from oracle.menos_sched import BWD, FWD, OracleScheduler

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "sched_traces.json")


def _native():
    from paper_conf_middleware_hul24_b200 import menos as M
    return M


def _traces():
    return json.load(open(GOLDEN))["traces"]


def _run_golden(make, tr):
    s = make(tr["total"])
    for c, (mf, mb) in tr["demands"].items():
        s.set_demand(int(c), mf, mb)
    for k, e in enumerate(tr["events"]):
        g = s.arrive(e["client"], e["kind"]) if e["ev"] == "arrive" else s.complete(e["client"])
        assert [list(x) for x in g] == e["grants"], (tr["name"], k)
        avail, waiting = _state(s)
        assert avail == e["avail"], (tr["name"], k)
        assert waiting == e["waiting"], (tr["name"], k)


def _state(s):
    if isinstance(s, OracleScheduler):
        return s.M_avail, [c for c, _ in s.W]
    st = s.state()
    return st["m_avail"], st["waiting"]


@pytest.mark.parametrize("tr", _traces(), ids=lambda t: t["name"])
def test_oracle_golden_traces(tr):
    _run_golden(OracleScheduler, tr)


@pytest.mark.parametrize("tr", _traces(), ids=lambda t: t["name"])
def test_native_golden_traces(tr):
    M = _native()
    _run_golden(lambda total: M.Scheduler(total, 8), tr)


def _random_trace(rng, n_clients, total, n_events):
    """Demands and an event sequence that is legal for a serving process per client (R17): idle clients
    arrive with a forward or a backward request; running clients complete."""
    demands = {i: (rng.randint(0, total // 2), rng.randint(1, total)) for i in range(n_clients)}
    return demands, n_events


def _drive(sched_a, sched_b, rng, demands, n_events, check):
    idle = set(demands)
    running = set()
    waiting = set()
    for i, (mf, mb) in demands.items():
        sched_a.set_demand(i, mf, mb)
        if sched_b is not None:
            sched_b.set_demand(i, mf, mb)
    for _ in range(n_events):
        if idle and (not running or rng.random() < 0.55):
            i = rng.choice(sorted(idle))
            kind = rng.choice((FWD, BWD))
            ga = sched_a.arrive(i, kind)
            gb = sched_b.arrive(i, kind) if sched_b is not None else None
            idle.discard(i)
            waiting.add(i)
        elif running:
            i = rng.choice(sorted(running))
            ga = sched_a.complete(i)
            gb = sched_b.complete(i) if sched_b is not None else None
            running.discard(i)
            idle.add(i)
        else:
            break
        for c, _, _ in ga:
            waiting.discard(c)
            running.add(c)
        check(sched_a, ga, gb)


def test_oracle_invariants_brute_force():
    """After every event: memory is conserved (M_avail + sum A = total), never negative; the FCFS head never
    fits once SCHEDULE returns (otherwise it or a backfill would have been granted); grants follow W order."""
    rng = random.Random(7)
    for trial in range(300):
        total = rng.randint(1, 40)
        demands, n_ev = _random_trace(rng, rng.randint(1, 9), total, 60)
        demands = {i: (mf, min(mb, total)) for i, (mf, mb) in demands.items()}
        state = {"W_before": []}

        def check(s, g, _):
            assert s.M_avail >= 0
            assert s.M_avail + sum(s.A[i] for i in s.running) == s.total
            if s.W:
                i, k = s.W[0]
                assert (s.M_f[i] if k == FWD else s.M_b[i]) > s.M_avail
            # grant order = waiting-list order (the head first, then backfills in position order)
            order = [c for c in state["W_before"] if c in {x for x, _, _ in g}]
            new = [x for x, _, _ in g if x not in state["W_before"]]
            assert [x for x, _, _ in g] == order + new
            state["W_before"] = [c for c, _ in s.W]

        s = OracleScheduler(total)
        orig_arrive = s.arrive

        def arrive(i, kind):
            state["W_before"] = state["W_before"] + [i]
            return orig_arrive(i, kind)
        s.arrive = arrive
        _drive(s, None, rng, demands, n_ev, check)


def test_oracle_no_starvation_of_fcfs_head():
    """a long-waiting backward is not bypassed by a stream of smaller forwards.  While the head
    waits, no later request is granted unless the head itself was granted in the same SCHEDULE call."""
    s = OracleScheduler(10)
    for i in range(6):
        s.set_demand(i, 1, 8)
    assert s.arrive(0, BWD) == [(0, BWD, 8)]
    assert s.arrive(1, BWD) == []            # head: needs 8, 2 left
    for i in range(2, 6):
        assert s.arrive(i, FWD) == []        # 1 B each would fit, but the head blocks (FCFS)
    g = s.complete(0)
    assert g[0] == (1, BWD, 8) and [x for x, _, _ in g[1:]] == [2, 3]


def test_native_matches_oracle_random_traces():
    M = _native()
    rng = random.Random(11)
    for trial in range(200):
        total = rng.randint(1, 1 << 40)
        n = rng.randint(1, 24)
        demands = {i: (rng.randint(0, total // 3), rng.randint(1, total)) for i in range(n)}
        o = OracleScheduler(total)
        nat = M.Scheduler(total, 32)

        def check(so, ga, gb):
            assert [tuple(x) for x in ga] == [tuple(x) for x in gb]
            st = nat.state()
            assert st["m_avail"] == so.M_avail
            assert st["waiting"] == [c for c, _ in so.W]
            assert st["n_running"] == len(so.running)
        _drive(o, nat, rng, demands, 80, check)


def test_native_errors():
    M = _native()
    s = M.Scheduler(100, 4)
    with pytest.raises(M.MenosError) as e:
        s.arrive(0, M.REQ_FWD)                 # no demands yet
    assert e.value.code == -3
    s.set_demand(0, 10, 101)
    with pytest.raises(M.MenosError) as e:
        s.arrive(0, M.REQ_BWD)                 # can never fit (R19)
    assert e.value.code == -2
    assert s.arrive(0, M.REQ_FWD) == [(0, M.REQ_FWD, 10)]
    with pytest.raises(M.MenosError) as e:
        s.arrive(0, M.REQ_BWD)                 # already running (R17)
    assert e.value.code == -4
    with pytest.raises(M.MenosError) as e:
        s.complete(1)
    assert e.value.code == -4
    with pytest.raises(M.MenosError) as e:
        s.set_demand(9, 1, 1)
    assert e.value.code == -3
    assert s.complete(0) == [] and s.state()["m_avail"] == 100


def test_native_short_out_buffer_changes_nothing():
    """a grant buffer smaller than max_clients is rejected BEFORE any state change (no client is left
    marked running with its memory deducted and no grant reported)."""
    import ctypes as C
    M = _native()
    s = M.Scheduler(100, 4)
    for i in range(4):
        s.set_demand(i, 10, 10)
    out = (M.SchedGrant * 2)()
    n = C.c_int()
    rc = M.lib().menos_sched_arrive(s.h, 0, M.REQ_FWD, out, 2, C.byref(n))
    assert rc == -1 and n.value == 0
    assert s.state() == {"m_avail": 100, "waiting": [], "n_running": 0}
    assert s.arrive(0, M.REQ_FWD) == [(0, M.REQ_FWD, 10)]
    rc = M.lib().menos_sched_complete(s.h, 0, out, 3, C.byref(n))
    assert rc == -1 and s.state() == {"m_avail": 90, "waiting": [], "n_running": 1}
    assert s.complete(0) == [] and s.state()["m_avail"] == 100


def test_native_decision_latency():
    """the scheduler takes less than 0.1 ms per decision (the paper's Python one).  64 clients,
    a full waiting list; mean and max of the native SCHEDULE call."""
    M = _native()
    s = M.Scheduler(1 << 34, 64)
    for i in range(64):
        s.set_demand(i, 1 << 28, 1 << 31)
    rng = random.Random(3)
    running = []
    for rnd in range(50):
        for i in range(64):
            if i not in running and i not in s.state()["waiting"]:
                running += [c for c, _, _ in s.arrive(i, rng.choice((0, 1)))]
        while running:
            c = running.pop(0)
            running += [x for x, _, _ in s.complete(c)]
    t = s.timing()
    assert t["decisions"] > 1000
    assert t["mean_ns"] < 1e5, t
