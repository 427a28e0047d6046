"""Menos serving loop: Algorithm 1 driven by the Algorithm 2 scheduler,
with every SCHEDULE call's grants run as batched waves on the shared base.

Host logic only (argument marshalling + an event queue); the decisions are the native scheduler's (menos_sched_*,
csrc/sched.cpp) and every step of the compute is libmenos.so's.  Time is a caller-supplied clock model, so a run
is deterministic and testable without a GPU (tests/test_serve.py) and the same loop drives the real server
(MenosExecutor; tests/test_gpu_serve.py).

Per client i (one "serving process" S_i), iteration k:
  x_c arrives (client forward + uplink)          -> sched.arrive(i, FWD)       Alg.2 L7-9
  FWD task: x_s = f_s(x_c) without caching        -> NOGRAD forward, retains nothing   Alg.1 L6-7
  x_s returned; g_c arrives after the client's loss/backward + uplink -> sched.arrive(i, BWD)
  BWD task: re-forward with grad, backward, AdamW -> SAVE forward + backward + adapter step  Alg.1 L10-13
  g_s returned; the next x_c follows.
The GPU runs one batched wave at a time.  Requests granted while it is busy accumulate; when it frees up, all of
them start as at most two waves, back to back: one batched FWD wave, then one batched BWD wave.  A task completes
(Alg.2 L10-13) when its wave ends on the GPU timeline; it holds its reserved memory from its grant until then.
"""
from __future__ import annotations

import dataclasses
import heapq

from .menos import MEM_BOUND, FWD_NOGRAD, FWD_SAVE, REQ_BWD, REQ_FWD, Scheduler


@dataclasses.dataclass
class ClientTiming:
    """Client-side delays (seconds on the loop's clock): t_fwd = client forward + uplink of x_c (Fig.1 steps 1),
    t_bwd = downlink of x_s + client loss/backward + uplink of g_c (step 3)."""
    t_fwd: float
    t_bwd: float


@dataclasses.dataclass
class Wave:
    kind: int
    clients: list
    granted: float   # time of the SCHEDULE call that granted it
    start: float     # start on the GPU timeline (after the waves before it)
    end: float
    reserved: int
    tasks: list      # (client, grant time, reserved bytes) per task


class ServeLoop:
    """Discrete-event loop.  executor.forward_wave(clients, it) / executor.backward_wave(clients, it) run one
    batched wave (it[c] = client c's iteration) and return its duration on the loop clock."""

    def __init__(self, sched: Scheduler, executor, timings: dict, n_iters: int):
        self.sched, self.ex, self.timings, self.n_iters = sched, executor, timings, n_iters
        self.waves: list[Wave] = []
        self.it = {c: 0 for c in timings}
        self._q = []
        self._seq = 0
        self.busy_until = 0.0
        self.pending = []   # (grant time, grant) not yet on the GPU
        self.finish = {}

    def _push(self, t, kind, c):
        heapq.heappush(self._q, (t, self._seq, kind, c))
        self._seq += 1

    def _on_grants(self, t, grants):
        for g in grants:
            self.pending.append((t, g))
        self._launch(t)

    def _launch(self, t):
        """Run everything granted so far as the next waves if the GPU is free; otherwise they join the waves that
        start when it frees up (one batched wave per kind: the B200 runs one wave at a time)."""
        if not self.pending or t < self.busy_until:
            return
        start = t
        for kind in (REQ_FWD, REQ_BWD):
            sel = [(tg, g) for tg, g in self.pending if g[1] == kind]
            if not sel:
                continue
            cl = [g[0] for _, g in sel]
            its = {c: self.it[c] for c in cl}
            dur = (self.ex.forward_wave if kind == REQ_FWD else self.ex.backward_wave)(cl, its)
            end = start + dur
            self.waves.append(Wave(kind, cl, min(tg for tg, _ in sel), start, end, sum(g[2] for _, g in sel),
                                   [(g[0], tg, g[2]) for tg, g in sel]))
            for c in cl:
                self._push(end, "done_fwd" if kind == REQ_FWD else "done_bwd", c)
            start = end
        self.pending = []
        self.busy_until = start
        self._push(start, "gpu_free", -1)

    def run(self):
        for c in sorted(self.timings):
            self._push(self.timings[c].t_fwd, "xc", c)
        while self._q:
            t, _, kind, c = heapq.heappop(self._q)
            if kind == "gpu_free":
                self._launch(t)
                continue
            if kind == "xc":
                grants = self.sched.arrive(c, REQ_FWD)
            elif kind == "gc":
                grants = self.sched.arrive(c, REQ_BWD)
            else:
                grants = self.sched.complete(c)
                if kind == "done_fwd":
                    self._push(t + self.timings[c].t_bwd, "gc", c)
                else:
                    self.it[c] += 1
                    if self.it[c] < self.n_iters:
                        self._push(t + self.timings[c].t_fwd, "xc", c)
                    else:
                        self.finish[c] = t
            self._on_grants(t, grants)
        return self


def client_demands(server, cid: int, n_tokens: int) -> tuple[int, int]:
    """Alg.2 L2: (M_f, M_b) of client cid alone, as additive bounds (MENOS_MEM_BOUND) so that any
    set of granted requests fits in the bytes they reserved when run as one batched wave."""
    m_f = server.batch_memory([cid], [n_tokens], FWD_NOGRAD | MEM_BOUND)[0]
    m_b = server.batch_memory([cid], [n_tokens], FWD_SAVE | MEM_BOUND)[1]
    return m_f, m_b


class MenosExecutor:
    """Runs waves on a menos Server.  inputs[c][k] = (seq_lens, x_c, g_c) of client c's iteration k (bf16 device
    tensors [T_c, d]).  Records x_s / g_s per (client, iteration), and each wave's exact demand
    (menos_batch_memory) next to what its grants reserved.  Durations come from `cost(kind, n_tokens)` (the loop
    clock) so that a run's event order is deterministic; measured GPU times are recorded separately."""

    def __init__(self, server, ids: dict, inputs: dict, cost, stream=None):
        import torch
        self.torch = torch
        self.srv, self.ids, self.inputs, self.cost, self.stream = server, ids, inputs, cost, stream
        self.x_s, self.g_s = {}, {}
        self.exact = []   # (kind, clients, exact bytes)

    def _pack(self, clients, its, which):
        t = self.torch
        seq_client, seq_len, parts = [], [], []
        for c in clients:
            lens, x, g = self.inputs[c][its[c]]
            seq_client += [self.ids[c]] * len(lens)
            seq_len += list(lens)
            parts.append(x if which == 0 else g)
        return seq_client, seq_len, t.cat(parts).contiguous()

    def _split(self, clients, its, buf, store):
        off = 0
        for c in clients:
            T = int(sum(self.inputs[c][its[c]][0]))
            store[(c, its[c])] = buf[off:off + T].clone()
            off += T

    def forward_wave(self, clients, its):
        sc, sl, x = self._pack(clients, its, 0)
        toks = [int(sum(self.inputs[c][its[c]][0])) for c in clients]
        self.exact.append((REQ_FWD, list(clients),
                           self.srv.batch_memory([self.ids[c] for c in clients], toks, FWD_NOGRAD)[0]))
        xs = self.torch.empty_like(x)
        self.srv.forward(sc, sl, x, xs, flags=FWD_NOGRAD, stream=self.stream, retain=False)
        self._split(clients, its, xs, self.x_s)
        return self.cost(REQ_FWD, sum(toks))

    def backward_wave(self, clients, its):
        sc, sl, x = self._pack(clients, its, 0)
        _, _, g = self._pack(clients, its, 1)
        toks = [int(sum(self.inputs[c][its[c]][0])) for c in clients]
        self.exact.append((REQ_BWD, list(clients),
                           self.srv.batch_memory([self.ids[c] for c in clients], toks, FWD_SAVE)[1]))
        xs = self.torch.empty_like(x)
        gs = self.torch.empty_like(g)
        b = self.srv.forward(sc, sl, x, xs, flags=FWD_SAVE, stream=self.stream)   # Alg.1 L10
        self.srv.backward(b, g, gs, stream=self.stream)                           # Alg.1 L11
        self.srv.adapter_step([self.ids[c] for c in clients], stream=self.stream)  # Alg.1 L12
        self._split(clients, its, gs, self.g_s)
        return self.cost(REQ_BWD, sum(toks))
