// Menos task scheduler (§4.2, Algorithm 2): FCFS with backfilling over GPU memory.
// SURVEY.md §8(f) NEXT-2.  Host-side, native; no CUDA.  It decides WHICH waiting requests enter the batched
// menos_forward / menos_backward calls of the hot path; the caller turns the grants of one SCHEDULE call into
// one batched call per request kind.
//
// State (Alg.2 L1-4): M_avail, per-client demands M_f[i], M_b[i], the waiting list W (arrival order) and the
// allocation dictionary A[i].  Events:
//   arrive(i, kind)  -- Alg.2 L7-9: append S_i to W, then SCHEDULE;
//   complete(i)      -- Alg.2 L10-13: M_avail += A[i]; A[i] = 0; then SCHEDULE.
// SCHEDULE (Alg.2 L14-24): if W is non-empty, take s = W[0] with m = M_f or M_b; if M_avail < m stop (FCFS: the
// head is never bypassed while it does not fit); else grant s (L19-22) and scan the rest of W
// in order, granting every request that still fits (backfilling, L23-24).
// Readings (DESIGN.md §3 R17-R19): a client has at most one request waiting or running (each serving process S_i
// alternates forward and backward, Alg.1); a request whose demand exceeds the total memory could never run and
// would block the FCFS head forever, so arrive() rejects it with MENOS_ENOMEM (principle 1).
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <deque>
#include <new>
#include <vector>

#include "menos.h"

namespace menos {
void set_last_error(const char* fmt, ...);
}

struct menos_sched {
  size_t total = 0, avail = 0;
  struct C {
    bool known = false;
    int state = 0;       // 0 idle, 1 waiting, 2 running
    int kind = 0;
    size_t mf = 0, mb = 0, alloc = 0;
  };
  std::vector<C> cl;
  std::deque<int32_t> W;   // waiting list, arrival order
  size_t n_running = 0;
  double decide_ns_total = 0, decide_ns_max = 0;
  long long decisions = 0;
};

#define SFAIL(code, ...) do { menos::set_last_error(__VA_ARGS__); return code; } while (0)

namespace {

// Alg.2 L14-24.  Appends grants to out (up to max_out; the count is returned in *n_out even if larger is
// impossible: the caller sizes out for every client).
int schedule(menos_sched* s, menos_sched_grant* out, int max_out, int* n_out) {
  const auto t0 = std::chrono::steady_clock::now();
  int n = 0;
  auto grant = [&](int32_t i, size_t m) {   // L19-22
    auto& c = s->cl[i];
    s->avail -= m;
    c.alloc = m;
    c.state = 2;
    ++s->n_running;
    if (n < max_out) { out[n].client = i; out[n].kind = c.kind; out[n].bytes = m; }
    ++n;
  };
  auto demand = [&](int32_t i) { const auto& c = s->cl[i]; return c.kind == MENOS_REQ_FWD ? c.mf : c.mb; };
  if (!s->W.empty()) {                                  // L15
    const int32_t h = s->W.front();                     // L16
    const size_t m = demand(h);                         // L17
    if (s->avail >= m) {                                // L18
      grant(h, m);
      s->W.pop_front();                                 // L22
      for (auto it = s->W.begin(); it != s->W.end();) { // L23-24: backfill, in waiting-list order
        const size_t mr = demand(*it);
        if (s->avail >= mr) { grant(*it, mr); it = s->W.erase(it); }
        else ++it;
      }
    }
  }
  if (n_out) *n_out = n;
  const double ns = std::chrono::duration<double, std::nano>(std::chrono::steady_clock::now() - t0).count();
  s->decide_ns_total += ns;
  if (ns > s->decide_ns_max) s->decide_ns_max = ns;
  ++s->decisions;
  return n <= max_out ? MENOS_OK : MENOS_EINVAL;
}

}  // namespace

extern "C" {

MENOS_API int menos_sched_create(size_t m_avail, int max_clients, menos_sched** out) {
  if (!out || max_clients <= 0) SFAIL(MENOS_EINVAL, "sched_create: bad arguments");
  auto* s = new (std::nothrow) menos_sched();
  if (!s) SFAIL(MENOS_ENOMEM, "sched_create: host allocation failed");
  s->total = s->avail = m_avail;                        // L1
  s->cl.resize(max_clients);                            // L4: A = {}
  *out = s;                                             // L3: W = []
  return MENOS_OK;
}

MENOS_API void menos_sched_destroy(menos_sched* s) { delete s; }

MENOS_API int menos_sched_set_demand(menos_sched* s, int32_t client, size_t m_f, size_t m_b) {   // L2
  if (!s) SFAIL(MENOS_EINVAL, "null scheduler");
  if (client < 0 || client >= (int32_t)s->cl.size()) SFAIL(MENOS_ENOCLIENT, "sched: client %d out of range", client);
  auto& c = s->cl[client];
  if (c.state != 0) SFAIL(MENOS_ESTATE, "sched: client %d has a request waiting or running", client);
  c.known = true; c.mf = m_f; c.mb = m_b;
  return MENOS_OK;
}

MENOS_API int menos_sched_arrive(menos_sched* s, int32_t client, int kind, menos_sched_grant* out, int max_out,
                                 int* n_out) {                                                  // L7-9
  if (n_out) *n_out = 0;
  if (!s || (max_out > 0 && !out)) SFAIL(MENOS_EINVAL, "sched_arrive: bad arguments");
  // one SCHEDULE can grant every waiting client: out must hold max_clients entries, checked BEFORE any state change
  if (max_out < (int)s->cl.size()) SFAIL(MENOS_EINVAL, "sched_arrive: out holds %d < max_clients %zu", max_out, s->cl.size());
  if (kind != MENOS_REQ_FWD && kind != MENOS_REQ_BWD) SFAIL(MENOS_EINVAL, "sched_arrive: bad kind %d", kind);
  if (client < 0 || client >= (int32_t)s->cl.size() || !s->cl[client].known)
    SFAIL(MENOS_ENOCLIENT, "sched_arrive: client %d has no demands (menos_sched_set_demand)", client);
  auto& c = s->cl[client];
  if (c.state != 0) SFAIL(MENOS_ESTATE, "sched_arrive: client %d already has a request waiting or running", client);
  const size_t m = kind == MENOS_REQ_FWD ? c.mf : c.mb;
  if (m > s->total) SFAIL(MENOS_ENOMEM, "sched_arrive: client %d needs %zu B > %zu B total", client, m, s->total);
  c.kind = kind;
  c.state = 1;
  s->W.push_back(client);                               // L8
  return schedule(s, out, max_out, n_out);              // L9
}

MENOS_API int menos_sched_complete(menos_sched* s, int32_t client, menos_sched_grant* out, int max_out,
                                   int* n_out) {                                                // L10-13
  if (n_out) *n_out = 0;
  if (!s || (max_out > 0 && !out)) SFAIL(MENOS_EINVAL, "sched_complete: bad arguments");
  if (max_out < (int)s->cl.size()) SFAIL(MENOS_EINVAL, "sched_complete: out holds %d < max_clients %zu", max_out, s->cl.size());
  if (client < 0 || client >= (int32_t)s->cl.size()) SFAIL(MENOS_ENOCLIENT, "sched: client %d out of range", client);
  auto& c = s->cl[client];
  if (c.state != 2) SFAIL(MENOS_ESTATE, "sched_complete: client %d has no running task", client);
  s->avail += c.alloc;                                  // L11
  c.alloc = 0;                                          // L12
  c.state = 0;
  --s->n_running;
  return schedule(s, out, max_out, n_out);              // L13
}

MENOS_API int menos_sched_state(menos_sched* s, size_t* m_avail, int* n_waiting, int* n_running,
                                int32_t* waiting, int max_waiting) {
  if (!s) SFAIL(MENOS_EINVAL, "null scheduler");
  if (m_avail) *m_avail = s->avail;
  if (n_waiting) *n_waiting = (int)s->W.size();
  if (n_running) *n_running = (int)s->n_running;
  if (waiting) {
    int k = 0;
    for (int32_t i : s->W) { if (k >= max_waiting) break; waiting[k++] = i; }
  }
  return MENOS_OK;
}

MENOS_API int menos_sched_timing(menos_sched* s, long long* decisions, double* mean_ns, double* max_ns) {
  if (!s) SFAIL(MENOS_EINVAL, "null scheduler");
  if (decisions) *decisions = s->decisions;
  if (mean_ns) *mean_ns = s->decisions ? s->decide_ns_total / s->decisions : 0.0;
  if (max_ns) *max_ns = s->decide_ns_max;
  return MENOS_OK;
}

}  // extern "C"
