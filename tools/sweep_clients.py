"""Supplementary sweep (labelled extra -- not a bench line): paper-shaped clients on ONE B200.

Llama-2-7B server segment (31 layers), each client batch 4 x S=100 (the paper's inferred workload), LoRA
r=8 on q,v, N in {1, 2, 4, 8, 16, 32} clients.  Per N, on one shared base copy:
  * save     : one batched SAVE forward + backward + AdamW over all N clients (the data-parallel hot path);
  * menos    : the paper's on-demand mode (Alg.1 L6-12, Fig.3(d)): NOGRAD forward (retains nothing), then re-forward
               with grad + backward + AdamW -- its overhead over `save` is the B200 counterpart of Tab.2
               (0.46 s -> 1.15 s on a V100 at one client);
  * serve    : the Alg.2 scheduler loop (serve.py) with the arena capped at room for ~4 clients' backwards; client
               delays 0 (saturated), so grants accumulate while the GPU is busy and run as batched waves;
  * memory   : base M once, per-client A+O, the batch's arena demand I (menos_batch_memory), and the paper's
               comparison: vanilla N x (M + A + O + I) (Eq.2) vs Menos M + N (A + O) + I_peak (Eq.3).
Times are CUDA events on the launching stream (device time), after warm-up.  Prints one JSON line per N.

Usage: python tools/sweep_clients.py [--ns 1,2,4,8,16,32] [--steps 3] [--layers 31]
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ns", default="1,2,4,8,16,32")
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--layers", type=int, default=None)
    ap.add_argument("--seq", type=int, default=100)
    args = ap.parse_args()
    import numpy as np
    import torch
    import bench
    from paper_conf_middleware_hul24_b200 import menos as M
    from paper_conf_middleware_hul24_b200.serve import ClientTiming, ServeLoop, client_demands
    from workloads import ClientCfg, MODELS, Workload, target_dims

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    ns = [int(x) for x in args.ns.split(",")]
    m = MODELS["7b"] if args.layers is None else MODELS["7b"].with_layers(args.layers)
    nmax = max(ns)
    w = Workload("paper_sweep", m, [ClientCfg(8, 16.0, ("q", "v"), [args.seq] * 4) for _ in range(nmax)])
    srv = bench.build_server(torch, w, dev, seed=0, arena_gb=0)
    ids = bench.register_clients(np, srv, w, seed=1)
    st = srv.stats()
    stream = torch.cuda.current_stream(dev)
    gen = torch.Generator(device=dev)
    gen.manual_seed(3)
    Tc = 4 * args.seq
    x_all = torch.randn(nmax * Tc, m.d_model, generator=gen, device=dev).to(torch.bfloat16)
    g_all = torch.randn(nmax * Tc, m.d_model, generator=gen, device=dev).to(torch.bfloat16)
    hd = m.head_dim
    P = m.n_layers * (m.d_model * (m.n_heads + 2 * m.n_kv_heads) * hd + m.d_model * m.n_heads * hd
                      + 3 * m.d_model * m.d_ff)
    lora_kn = [target_dims(m, t) for t in ("q", "v")]

    def flops(n):
        T = n * Tc
        pairs = n * 4 * args.seq * (args.seq + 1) / 2
        return 4.0 * P * T + 12.0 * hd * m.n_heads * pairs * m.n_layers + \
            sum(6 * 8 * (K + N) * T * m.n_layers for K, N in lora_kn)

    def timed(fn, k):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(k):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / k

    for n in ns:
        sel = ids[:n]
        T = n * Tc
        sc = [c for c in sel for _ in range(4)]
        sl = [args.seq] * (4 * n)
        x, g = x_all[:T], g_all[:T]
        xs, gs = torch.empty_like(x), torch.empty_like(x)

        def save_step():
            b = srv.forward(sc, sl, x, xs, stream=stream)
            srv.backward(b, g, gs, stream=stream)
            srv.adapter_step(sel, stream=stream)

        def menos_step():
            srv.forward(sc, sl, x, xs, flags=M.FWD_NOGRAD, stream=stream, retain=False)   # Alg.1 L6-7
            b = srv.forward(sc, sl, x, xs, stream=stream)                                  # L10
            srv.backward(b, g, gs, stream=stream)                                           # L11
            srv.adapter_step(sel, stream=stream)                                            # L12

        for _ in range(args.warmup):
            save_step()
            menos_step()
        t_save = timed(save_step, args.steps)
        t_menos = timed(menos_step, args.steps)
        fwd_b, bwd_b = srv.batch_memory(sel, [Tc] * n, M.FWD_SAVE)
        ng_f, _ = srv.batch_memory(sel, [Tc] * n, M.FWD_NOGRAD)
        persist = srv.client_memory(sel[0], Tc)[0]
        I1 = max(srv.batch_memory([sel[0]], [Tc], M.FWD_SAVE))   # one client's activations (vanilla keeps them)
        vanilla = n * (st["base_bytes"] + persist + I1)             # Eq.2: N x (M + A + O + I)
        menos = st["base_bytes"] + n * persist + max(fwd_b, bwd_b)  # Eq.3: M + N(A + O) + I

        # Alg.2-driven serving: saturated clients, arena share for ~4 backwards at a time
        dem = {i: client_demands(srv, sel[i], Tc) for i in range(n)}
        cap = int(4.2 * max(mb for _, mb in dem.values()))
        sched = M.Scheduler(cap, 64)
        for i, (mf, mb) in dem.items():
            sched.set_demand(i, mf, mb)

        class Ex:
            def __init__(self):
                self.ms = 0.0

            def _run(self, cl, fn):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                fn(cl)
                e1.record(stream)
                torch.cuda.synchronize()
                dt = e0.elapsed_time(e1)
                self.ms += dt
                return dt / 1e3

            def forward_wave(self, cl, its):
                def f(cl):
                    idx = torch.cat([torch.arange(i * Tc, (i + 1) * Tc, device=dev) for i in cl])
                    xx = x_all[idx]
                    srv.forward([sel[i] for i in cl for _ in range(4)], [args.seq] * (4 * len(cl)), xx,
                                torch.empty_like(xx), flags=M.FWD_NOGRAD, stream=stream, retain=False)
                return self._run(cl, f)

            def backward_wave(self, cl, its):
                def f(cl):
                    idx = torch.cat([torch.arange(i * Tc, (i + 1) * Tc, device=dev) for i in cl])
                    xx, gg = x_all[idx], g_all[idx]
                    b = srv.forward([sel[i] for i in cl for _ in range(4)], [args.seq] * (4 * len(cl)), xx,
                                    torch.empty_like(xx), stream=stream)
                    srv.backward(b, gg, torch.empty_like(gg), stream=stream)
                    srv.adapter_step([sel[i] for i in cl], stream=stream)
                return self._run(cl, f)

        ex = Ex()
        iters = 3
        loop = ServeLoop(sched, ex, {i: ClientTiming(0.0, 0.0) for i in range(n)}, iters).run()
        span = max(wv.end for wv in loop.waves)
        tim = sched.timing()
        print(json.dumps({
            "N": n, "tokens_per_client": Tc, "layers": m.n_layers,
            "save": {"ms_per_step": t_save, "tokens_per_s": T / (t_save / 1e3),
                     "tflops": flops(n) / (t_save / 1e3) / 1e12},
            "menos_on_demand": {"ms_per_step": t_menos, "tokens_per_s": T / (t_menos / 1e3),
                                "overhead_vs_save": t_menos / t_save,
                                "paper_tab2_ratio_v100": round(1.15 / 0.46, 3)},
            "serve_alg2": {"tokens_per_s": n * Tc * iters / span, "waves": len(loop.waves),
                           "mean_wave_clients": sum(len(x.clients) for x in loop.waves) / len(loop.waves),
                           "sched_mean_us": tim["mean_ns"] / 1e3, "arena_cap_bytes": cap},
            "memory": {"base_M": st["base_bytes"], "per_client_AO": persist, "batch_I_save": max(fwd_b, bwd_b),
                       "batch_I_nograd_fwd": ng_f, "vanilla_eq2": vanilla, "menos_eq3": menos,
                       "reduction": 1 - menos / vanilla,
                       "paper": "PAPER.md:350-352: -64.1% / -72.2% at 4 clients on a V100 (fp32; context)"},
        }), flush=True)


if __name__ == "__main__":
    main()
