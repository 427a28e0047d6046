#!/usr/bin/env python
"""Menos server-segment benchmark (BASELINE.json metric: server fwd+bwd tokens/s at N clients, Llama-2-7B LoRA;
HBM bytes/client).

One step = menos_forward(SAVE) over every client's tokens on this GPU -> menos_backward -> menos_adapter_step
(SURVEY.md §8(d) timing protocol; Alg.1 L10-12).  Default workload = BASELINE.json configs[1]
(Llama-2-7B layers 2..32, 4 clients r=8 on q,v, batch 4 x 512 = 8,192 tokens) on each GPU; with --gpus N
every rank runs its own replica with its own 4 clients (weak scaling, no collective on the path).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl menos|reference]

Inputs are synthetic and resident in HBM before the timed region (value); `e2e` repeats the measurement
through the same C-ABI with pinned HOST buffers (H2D of x_c and g_c, D2H of x_s and g_s inside the timed
region).  The reference arm (--impl reference) is the CPU oracle (oracle/), timed on a bounded sample.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "server fwd+bwd tokens/s at N clients (Llama-2-7B LoRA); HBM bytes/client"


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as fh:
            p = json.load(fh)
        return p, "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


# ------------------------------------------------------------------------------------------------ clocks
class ClockSampler:
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        try:
            out, _ = self.p.communicate(timeout=5)
        except Exception:
            self.p.kill()
            out = ""
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                smax = float(f[2])
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        load = [v for v in sm if smax and v > 0.5 * smax] or sm
        return {"sm_mhz": statistics.median(load) if load else None, "sm_max_mhz": smax,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------------------------------------ CPU oracle
_ORACLE_CACHE = {}


def _oracle_weights(n_layers: int):
    """Base weights of the first n_layers Llama-2-7B server layers (fp32, the parity recipe), generated once."""
    from workloads import MODELS, base_layer_weights
    key = n_layers
    if key not in _ORACLE_CACHE:
        _ORACLE_CACHE.clear()
        m = MODELS["7b"].with_layers(n_layers)
        _ORACLE_CACHE[key] = (m, [base_layer_weights(m, l, seed=0) for l in range(n_layers)])
    return _ORACLE_CACHE[key]


def oracle_layers_that_fit() -> int:
    """All 31 server layers (cfg1 full depth) when the host holds their fp32 weights (25 GB) plus working space;
    otherwise the most that fit, and the line says so."""
    full = 31
    try:
        import psutil
        avail = psutil.virtual_memory().available
    except Exception:
        return full
    per_layer = 202_383_360 * 4 * 1.2
    return max(1, min(full, int((avail - (12 << 30)) // per_layer)))


def oracle_sample(seq: int = 512, n_layers: int | None = None):
    """Time the CPU oracle (as it stands, never tuned) on a bounded sample of the cfg1 workload: ONE sequence of `seq`
    tokens of one cfg1 client (r = 8 on q, v) through the Llama-2-7B server segment, forward + backward.  Full depth
    (31 layers) unless the host cannot hold the fp32 weights; then the truncation is stated and scaled."""
    import numpy as np
    from oracle import menos_oracle as O
    from workloads import ClientCfg, client_adapters, client_inputs
    cores = len(os.sched_getaffinity(0))
    full = 31
    n_layers = n_layers or oracle_layers_that_fit()
    m, W = _oracle_weights(n_layers)
    c = ClientCfg(8, 16.0, ("q", "v"), [seq])
    ad = client_adapters(m, c, seed=1)
    x, g = client_inputs(m, c, seed=2)
    t0 = time.perf_counter()
    O.client_step(x, g, c.seq_lens, W, ad, c.alpha / c.rank, m)
    dt = time.perf_counter() - t0
    scale = full / n_layers
    tps = c.n_tokens / (dt * scale)
    depth = (f"all {full} Llama-2-7B server layers" if n_layers == full else
             f"{n_layers} of {full} Llama-2-7B server layers (host RAM bound), time scaled x{scale:.2f} to {full}")
    return {"value": tps, "unit": "tokens/s", "cores": cores, "kind": "oracle", "sample_s": dt,
            "sample_tokens": c.n_tokens, "sample_layers": n_layers,
            "sample": f"1 cfg1 sequence of {seq} tokens (r=8 q,v) through {depth}, fwd+bwd, fp32 numpy on {cores} "
                      f"host threads: {dt:.2f} s"}


def run_reference(args):
    """The reference arm for this tier = the CPU oracle as it stands, rank 0 only.  Each step is a
    bounded sample of our arm's workload: one 128-token sequence of a cfg1 client through the whole 31-layer segment
    (no depth extrapolation when the host holds the weights); value = tokens/s of that sample."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    seq = 128
    for _ in range(args.warmup):
        oracle_sample(seq)
    vals = [oracle_sample(seq) for _ in range(args.steps)]
    v = statistics.median([r["value"] for r in vals])
    s_med = statistics.median([r["sample_s"] for r in vals])
    cb = dict(vals[-1])
    cb["value"] = v
    w = args.workload or "cfg1_7b_x4"
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "tokens/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": s_med * 1000.0, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": w, "model": "llama2-7b", "measured_sample": cb["sample"],
                       "sample_tokens_per_step": cb["sample_tokens"], "sample_layers": cb["sample_layers"],
                       "note": "ms_per_step is the measured time of one sample step, not of the whole workload"},
            "cpu_baseline": cb, "e2e": {"value": v, "unit": "tokens/s", "h2d_bytes_per_step": 0,
                                        "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


# ------------------------------------------------------------------------------------------------ launcher
def _free_port() -> int:
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def spawn_ranks(args) -> int:
    """`python bench.py --gpus N` without a torchrun environment: re-exec this script under torchrun with N ranks
    (one process per GPU, 127.0.0.1 rendezvous), NCCL init logs on stderr; rank 0 prints the JSON line."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__), *sys.argv[1:]]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    env.setdefault("OMP_NUM_THREADS", "4")
    return subprocess.run(cmd, env=env).returncode


def rank_plan(w, world: int, rank: int, tp_mode: bool, strong: bool):
    """The clients this rank serves: all of them (weak scaling / tensor parallel) or its LPT share (strong)."""
    from paper_conf_middleware_hul24_b200.partition import workload_partition
    if strong and not tp_mode:
        return workload_partition(w, world)[rank]
    return list(range(len(w.clients)))


def run_dry(args):
    """Launcher check without the library or a GPU: every rank computes its client share; rank 0 prints the rank map
    as one JSON line (gloo all_gather when world > 1)."""
    import torch.distributed as dist
    from workloads import workload
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if world > 1:
        dist.init_process_group("gloo")
    w = workload(args.workload)
    tp_mode = args.workload.startswith("cfg4")
    strong = args.workload in ("cfg2_7b_x32_ragged", "cfg3_13b_x16") or tp_mode
    mine = rank_plan(w, world, rank, tp_mode, strong)
    info = {"rank": rank, "pid": os.getpid(), "clients": mine, "tokens": sum(w.clients[i].n_tokens for i in mine)}
    allinfo = [None] * world
    if world > 1:
        dist.all_gather_object(allinfo, info)
    else:
        allinfo = [info]
    if rank == 0:
        print(json.dumps({"dry_run": True, "metric": METRIC, "n_gpus": world, "ranks_seen": len(allinfo),
                          "config": {"workload": args.workload, "scaling": "strong" if strong else "weak",
                                     "per_rank": allinfo}}))
    if world > 1:
        dist.destroy_process_group()
    return 0


# ------------------------------------------------------------------------------------------------ GPU arm
def build_server(torch, w, device, seed, arena_gb, tp=None):
    """One server (replica, or tensor-parallel shard when tp = (rank, world, allreduce)).  Weights are drawn on
    the GPU directly in the shapes this server holds (a shard draws its own values: perf runs never compare
    bytes)."""
    from paper_conf_middleware_hul24_b200 import Server
    m = w.model
    if arena_gb is None or arena_gb <= 0:   # everything the base copy and the clients' adapters leave, minus headroom
        from workloads import target_dims
        free = torch.cuda.mem_get_info(device)[0]
        W = tp[1] if tp else 1
        P = m.n_layers * (2 * m.d_model * (m.n_heads + m.n_kv_heads) * m.head_dim + 3 * m.d_model * m.d_ff) // W
        # A + O per client: fp32 p, g, m, v (16 B/param) + bf16 slot tables (A and B, rank padded to 16, tables
        # grown by doubling: x2)
        ao = sum(m.n_layers * sum(target_dims(m, t)[0] + target_dims(m, t)[1] for t in c.targets)
                 * (16 * c.rank + 2 * 2 * (-(-c.rank // 16) * 16)) for c in w.clients) // W
        arena_gb = max(4.0, (free - 2 * P - ao - (6 << 30)) / (1 << 30))
    srv = Server(m.d_model, m.n_heads, m.n_kv_heads, m.d_ff, m.n_layers, first_layer=m.first_layer,
                 rms_eps=m.rms_eps, rope_theta=m.rope_theta, weights=None, device=device.index,
                 max_rank=16, max_seq_len=max(max(c.seq_lens) for c in w.clients),
                 arena_bytes=int(arena_gb * (1 << 30)), tp=tp, arch=m.arch)
    gen = torch.Generator(device=device)
    hd = m.head_dim
    W = tp[1] if tp else 1
    Hl, Hkvl, fl = m.n_heads // W, m.n_kv_heads // W, m.d_ff // W
    shapes = {"wq": (Hl * hd, m.d_model), "wk": (Hkvl * hd, m.d_model),
              "wv": (Hkvl * hd, m.d_model), "wo": (m.d_model, Hl * hd),
              "wgate": (fl, m.d_model), "wup": (fl, m.d_model), "wdown": (m.d_model, fl)}
    out_std = 0.02 / (2.0 * m.total_layers) ** 0.5   # same recipe as workloads.base_layer_weights (R17)
    for l in range(m.n_layers):
        gen.manual_seed(seed * 1000 + l)
        lw = {k: (torch.randn(s, generator=gen, device=device, dtype=torch.float32)
                  * (out_std if k in ("wo", "wdown") else 0.02)).to(torch.bfloat16)
              for k, s in shapes.items()}
        for gname in ("g1", "g2"):
            lw[gname] = (1 + 0.1 * torch.randn(m.d_model, generator=gen, device=device)).to(torch.bfloat16)
        if m.arch == "opt":   # OPT (NEXT-4): no gate; biases and LayerNorm biases (workloads.base_layer_weights recipe)
            del lw["wgate"]
            for bname, n in (("bq", Hl * hd), ("bk", Hkvl * hd), ("bv", Hkvl * hd), ("bo", m.d_model),
                             ("bup", fl), ("bdown", m.d_model), ("b1", m.d_model), ("b2", m.d_model)):
                sd = 0.1 if bname in ("b1", "b2") else 0.02
                lw[bname] = (sd * torch.randn(n, generator=gen, device=device)).to(torch.bfloat16)
        srv.load_layer(l, lw)
        del lw
    torch.cuda.synchronize(device)
    return srv


def register_clients(np, srv, w, seed):
    ids = []
    rng = np.random.default_rng(seed)
    for i, c in enumerate(w.clients):
        cid = srv.register_client(c.rank, c.alpha, c.targets, seed=seed * 100 + i)
        for l in range(w.model.n_layers):
            for t in c.targets:
                (_, _), (rb, cb) = srv.adapter_shape(cid, t)
                srv.set_adapter(cid, l, t, "B", (rng.standard_normal((rb, cb)) * 0.02).astype(np.float32))
        ids.append(cid)
    return ids


def run_gpu(args):
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_middleware_hul24_b200 import menos as M
    from workloads import workload

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world} (launch with torchrun or let bench.py "
                         f"spawn the ranks)")
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    device = torch.device("cuda", local)
    torch.cuda.set_device(device)
    from paper_conf_middleware_hul24_b200.partition import plan_waves_exact, workload_partition
    if os.environ.get("MENOS_ATTN_TC") is not None:   # kernel-variant switch for A/B measurements
        M.lib().menos_test_set_attn_tc(int(os.environ["MENOS_ATTN_TC"]))
    w = workload(args.workload, n_layers=args.layers)
    # cfg2 / cfg3 (32 ragged 7B clients / 16 13B clients): LPT partition over the replica ranks (strong scaling);
    # cfg4 (70B): tensor-parallel over the ranks, every rank sees all clients' tokens (strong scaling);
    # otherwise every rank serves the workload's own client set on its replica (weak scaling)
    tp_mode = args.workload.startswith("cfg4") or args.tp_shard_only > 1
    strong = args.workload in ("cfg2_7b_x32_ragged", "cfg3_13b_x16") or tp_mode
    tp = None
    if tp_mode:
        from paper_conf_middleware_hul24_b200 import tp as TPM
        if args.tp_shard_only > 1:
            # single-GPU compute-only timing of rank 0's shard of a W-way split: the all-reduce is a no-op, so
            # this is NOT a bench value (no communication); it measures the per-GPU kernels of the TP path
            if world != 1:
                raise SystemExit("--tp-shard-only runs on one GPU")
            tp = (0, args.tp_shard_only, lambda op, snd, rcv, n, dt, st: 0)
        else:
            # NCCL driven by the library (no Python on the per-layer path): rank 0's unique id, broadcast once
            ids_ = [TPM.nccl_unique_id() if rank == 0 else None]
            if world > 1:
                dist.broadcast_object_list(ids_, src=0)
            tp = (rank, world, ids_[0]) if world > 1 else None
    elif strong:
        w.clients = [w.clients[i] for i in rank_plan(w, world, rank, tp_mode, strong)]
    T = w.n_tokens
    d = w.model.d_model
    torch.cuda.synchronize(device)
    free0 = torch.cuda.mem_get_info(device)[0]
    srv = build_server(torch, w, device, seed=rank, arena_gb=args.arena_gb, tp=tp)
    torch.cuda.synchronize(device)
    free1 = torch.cuda.mem_get_info(device)[0]
    ids = register_clients(np, srv, w, seed=rank + 1)
    torch.cuda.synchronize(device)
    free2 = torch.cuda.mem_get_info(device)[0]
    # waves: temporal sharing of the arena when the clients' saved activations do not fit at once
    mem = [srv.client_memory(ids[i], c.n_tokens) for i, c in enumerate(w.clients)]
    cap = srv.stats()["arena_bytes"] - (64 << 20)

    def demand(idx):   # exact peak arena bytes of one batched call (menos_batch_memory)
        return max(srv.batch_memory([ids[i] for i in idx], [w.clients[i].n_tokens for i in idx]))
    waves = plan_waves_exact(len(w.clients), demand, cap)
    props = torch.cuda.get_device_properties(device)
    my_info = {"rank": rank, "device": str(getattr(props, "uuid", local)),
               "clients": len(w.clients), "tokens": T, "waves": len(waves)}
    per_rank = [my_info]
    if world > 1:
        per_rank = [None] * world
        dist.all_gather_object(per_rank, my_info)
    toff = [0]
    for c in w.clients:
        toff.append(toff[-1] + c.n_tokens)
    wave_args = []
    for wv in waves:
        sc_, sl_ = [], []
        for i in wv:
            sc_ += [ids[i]] * len(w.clients[i].seq_lens)
            sl_ += list(w.clients[i].seq_lens)
        wave_args.append((sc_, sl_, toff[wv[0]], toff[wv[-1] + 1]))
    gen = torch.Generator(device=device)
    gen.manual_seed(7 + rank)
    x_c = torch.randn(T, d, generator=gen, device=device).to(torch.bfloat16)
    g_c = torch.randn(T, d, generator=gen, device=device).to(torch.bfloat16)
    x_s, g_s = torch.empty_like(x_c), torch.empty_like(x_c)
    stream = torch.cuda.current_stream(device)
    T_all = T
    if world > 1 and not tp_mode:
        tt = torch.tensor([float(T)], device=device)
        dist.all_reduce(tt)
        T_all = int(tt.item())

    def step(xc, xs, gc, gs):
        for sc_, sl_, a, b_ in wave_args:
            b = srv.forward(sc_, sl_, xc[a:b_], xs[a:b_], stream=stream)
            srv.backward(b, gc[a:b_], gs[a:b_], stream=stream)
        srv.adapter_step(ids, stream=stream)

    def barrier():
        if world > 1:
            dist.barrier()

    host_ms = [0.0]

    def timed(fn, K):
        barrier()
        torch.cuda.synchronize(device)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        h0 = time.perf_counter()
        for _ in range(K):
            fn()
        e1.record(stream)
        host_ms[0] = (time.perf_counter() - h0) * 1e3   # host time to enqueue the K steps (diagnostic)
        torch.cuda.synchronize(device)
        barrier()
        ms = e0.elapsed_time(e1)
        if world > 1:
            t = torch.tensor([ms], device=device)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms

    for _ in range(args.warmup):
        step(x_c, x_s, g_c, g_s)
    torch.cuda.synchronize(device)

    clocks = ClockSampler(device.index)
    if os.environ.get("MENOS_BENCH_CLOCKS", "1") != "0":   # =0: diagnostic runs without the nvidia-smi sampler
        clocks.start()
        time.sleep(0.3)
    # one more untimed step after the sampler's start-up pause, so the timed region does not begin on an idle GPU
    # (its clocks ramp back under the power cap: r2cl read 43.6 k tokens/s here vs 44.1 k for the e2e region)
    step(x_c, x_s, g_c, g_s)
    torch.cuda.synchronize(device)
    l0 = M.launch_count()
    ms = timed(lambda: step(x_c, x_s, g_c, g_s), args.steps)
    host_enqueue_ms = host_ms[0] / args.steps
    launches = M.launch_count() - l0
    clk = clocks.stop()
    ms_per_step = ms / args.steps
    value = T_all * args.steps / (ms / 1000.0)

    # host work of one step with the GPU idle before every call (no ring-slot / event waits): what the library's
    # host side costs per step when it cannot hide behind the previous call's kernels
    host_calls = {"forward": 0.0, "backward": 0.0, "adapter_step": 0.0}
    torch.cuda.synchronize(device)
    for sc_, sl_, a, b_ in wave_args:
        h0 = time.perf_counter()
        b = srv.forward(sc_, sl_, x_c[a:b_], x_s[a:b_], stream=stream)
        host_calls["forward"] += time.perf_counter() - h0
        torch.cuda.synchronize(device)
        h0 = time.perf_counter()
        srv.backward(b, g_c[a:b_], g_s[a:b_], stream=stream)
        host_calls["backward"] += time.perf_counter() - h0
        torch.cuda.synchronize(device)
    h0 = time.perf_counter()
    srv.adapter_step(ids, stream=stream)
    host_calls["adapter_step"] += time.perf_counter() - h0
    torch.cuda.synchronize(device)
    host_calls = {k: v * 1e3 for k, v in host_calls.items()}

    # per-kernel CUDA events (recorded by the library on the launching stream around every launch) over a
    # second timed region of the same K steps; kept out of the headline region because an event pair around
    # every cluster launch adds inter-kernel gaps
    M.profile_enable(True)
    ms_prof = timed(lambda: step(x_c, x_s, g_c, g_s), args.steps)
    prof = M.profile_read()
    M.profile_enable(False)

    # e2e through the same C-ABI with pinned host buffers (copies inside the timed region)
    e2e = None
    if not args.no_e2e:
        hx = x_c.cpu().pin_memory()
        hg = g_c.cpu().pin_memory()
        hxs, hgs = torch.empty_like(hx).pin_memory(), torch.empty_like(hg).pin_memory()
        step(hx, hxs, hg, hgs)
        ms_e = timed(lambda: step(hx, hxs, hg, hgs), args.steps)
        e2e = {"value": T_all * args.steps / (ms_e / 1000.0), "unit": "tokens/s",
               "h2d_bytes_per_step": int(hx.numel() * 2 + hg.numel() * 2),
               "d2h_bytes_per_step": int(hxs.numel() * 2 + hgs.numel() * 2),
               "ms_per_step": ms_e / args.steps}

    # roofline of the dominant kernel (tcgen05 GEMM) from the live per-launch CUDA events
    peaks, src = load_peaks()
    g = prof.get("gemm_tcgen05", {})
    total_ms = sum(v["ms"] for v in prof.values()) or 1.0
    achieved = g["flops"] / (g["ms"] / 1000.0) / 1e12 if g.get("ms") else None
    peak = peaks.get("bf16_tflops_sustained", peaks.get("bf16_tflops"))
    traffic = None
    tp = os.path.join(ROOT, "profiles", "gemm_traffic.json")
    if os.path.exists(tp) and args.workload == "cfg1_7b_x4" and not args.layers:   # measured at cfg1's shapes only
        try:
            traffic = json.load(open(tp)).get("bytes_per_launch")
        except Exception:
            traffic = None
    roofline = {"bound": "tensor", "kernel": "gemm_tcgen05", "achieved": achieved, "peak": peak,
                "unit": "TFLOP/s", "frac": (achieved / peak) if achieved else None, "traffic": traffic,
                "peak_source": f"{src} bf16_tflops_sustained (kernel timed inside a long step)",
                "launches": g.get("launches"), "share_of_kernel_time": g.get("ms", 0) / total_ms,
                "region": f"per-launch CUDA events over a second timed region of the same {args.steps} steps "
                          f"({ms_prof / args.steps:.1f} ms/step with events vs {ms_per_step:.1f} without)",
                "avg_launch_ms": g["ms"] / g["launches"] if g.get("launches") else None}
    kernels = {}
    for k, v in prof.items():
        if not v["launches"]:
            continue
        e = {"launches": v["launches"], "ms_per_step": v["ms"] / args.steps, "share": v["ms"] / total_ms}
        if v["flops"]:
            e["tflops"] = v["flops"] / (v["ms"] / 1000.0) / 1e12
        if v["bytes"]:
            e["gbs"] = v["bytes"] / (v["ms"] / 1000.0) / 1e9
            e["frac_hbm"] = e["gbs"] / peaks.get("hbm_gbs", 6650.0)
        kernels[k] = e
    # algorithmic FLOPs of the whole step (no recompute credit, no base dW): 4 P + attention + LoRA
    m = w.model
    hd = m.head_dim
    mlp_mats = 2 if m.arch == "opt" else 3   # OPT: fc1, fc2; Llama: gate, up, down
    P = m.n_layers * (m.d_model * (m.n_heads + 2 * m.n_kv_heads) * hd + m.d_model * m.n_heads * hd
                      + mlp_mats * m.d_model * m.d_ff)
    pairs = sum(s * (s + 1) / 2 for c in w.clients for s in c.seq_lens)
    attn = 12 * hd * m.n_heads * pairs * m.n_layers
    lora = 0.0
    from workloads import target_dims
    for c in w.clients:
        for t in c.targets:
            K_, N_ = target_dims(m, t)
            lora += 6 * c.rank * (K_ + N_) * c.n_tokens * m.n_layers
    step_flops = 4 * P * T + attn + lora
    if tp_mode:   # every rank computes 1/W of the (replicated-token) step; the job does the whole step once
        job_flops = step_flops / (args.tp_shard_only if args.tp_shard_only > 1 else 1)
    else:
        job_flops = step_flops * (T_all / T)
    step_tflops = job_flops * args.steps / (ms / 1000.0) / 1e12
    n_dev = world

    # HBM bytes per client (persistent A+O and the SAVE-forward arena share), Eq.3 accounting
    st = srv.stats()
    per_client = []
    for i, c in enumerate(w.clients):
        pers, fwd, bwd = srv.client_memory(ids[i], c.n_tokens)
        per_client.append({"persistent_AO": pers, "arena_I": fwd})
    AO = statistics.mean(p["persistent_AO"] for p in per_client)
    Mb = st["base_bytes"]
    Nc = len(w.clients)
    hbm = {"base_M_bytes_once_per_gpu": Mb, "per_client_persistent_AO_bytes": AO,
           "per_client_arena_I_bytes": statistics.mean(p["arena_I"] for p in per_client),
           "measured": {
               "how": "cudaMemGetInfo deltas around menos_server_create (base + arena + tables) and around the "
                      "clients' registration (A+O: fp32 p, g, m, v + bf16 slot tables incl. their growth); arena "
                      "high-water mark of the step from the library's allocator",
               "server_create_bytes": free0 - free1, "arena_bytes": st["arena_bytes"],
               "base_and_tables_bytes": free0 - free1 - st["arena_bytes"],
               "per_client_persistent_AO_bytes": (free1 - free2) / max(1, Nc),
               "arena_peak_bytes_per_token": st["arena_peak"] / max(1, max(
                   sum(w.clients[i].n_tokens for i in wv) for wv in waves))},
           "persistent_reduction_vs_vanilla": 1.0 - (Mb + Nc * AO) / (Nc * (Mb + AO)),
           "paper_reference": "PAPER.md:352: -72.2% for 4 Llama-2-7B clients on a V100 (fp32; context only)"}

    line = {"metric": METRIC, "value": value, "unit": "tokens/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "strong" if strong else "weak",
            "vs_baseline": None, "dtype": "bf16", "data": "synthetic (seeded random weights/activations)",
            "config": {"workload": args.workload, "model": w.model.name, "clients_per_gpu": len(w.clients),
                       "tokens_per_gpu_step": T, "tokens_per_step_all_gpus": T_all,
                       "waves_per_step": len(waves), "server_layers": w.model.n_layers,
                       "per_rank": per_rank, "gpus_active": len({r["device"] for r in per_rank}),
                       "lora": sorted({f"r{c.rank} {'+'.join(c.targets)}" for c in w.clients}),
                       "seq_lens": sorted({s for c in w.clients for s in c.seq_lens}),
                       "parallelism": (f"tensor-parallel x{world} (NCCL all-reduce per attention/MLP block)"
                                       if tp_mode and args.tp_shard_only <= 1 else
                                       f"rank-0 shard of TP-{args.tp_shard_only}, all-reduce elided: compute "
                                       f"only, NOT a bench value" if tp_mode else
                                       f"replica x{world} (clients partitioned, no collective)"),
                       "l2": f"inputs larger than L2: {srv.stats()['base_bytes'] / 1e9:.2f} GB bf16 weights + "
                             f"{sum(m_[1] for m_ in mem) / 1e9:.1f} GB saved activations "
                             f"streamed per step vs 126 MB L2"},
            "roofline": roofline, "step_tflops": step_tflops,
            "step_frac_of_peak": step_tflops / (peak * n_dev) if peak else None,
            "kernels": kernels, "gpu_launches": launches, "clocks": clk, "e2e": e2e, "hbm_bytes_per_client": hbm,
            "host_enqueue_ms_per_step": host_enqueue_ms, "host_ms_per_call_gpu_idle": host_calls}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            line["cpu_baseline"] = oracle_sample(512)
        except Exception as ex:  # never let the baseline kill the bench line
            line["cpu_baseline"] = {"value": None, "error": repr(ex)}
    if rank == 0:
        print(json.dumps(line))
    srv.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="menos", choices=["menos", "reference"])
    ap.add_argument("--workload", default=None,
                    help="default: cfg1_7b_x4 at --gpus 1, cfg2_7b_x32_ragged (LPT over the ranks) at --gpus > 1")
    ap.add_argument("--layers", type=int, default=None, help="truncate depth (debug only; not a bench value)")
    ap.add_argument("--arena-gb", type=float, default=0.0, help="activation arena; 0 = all memory the base leaves")
    ap.add_argument("--tp-shard-only", type=int, default=0,
                    help="time rank 0's shard of a W-way tensor-parallel split on 1 GPU (no all-reduce; not a "
                         "bench value)")
    ap.add_argument("--dry-run", action="store_true", help="launcher check: no library, no GPU; print the rank map")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.workload is None:
        args.workload = "cfg1_7b_x4" if args.gpus == 1 else "cfg2_7b_x32_ragged"
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return spawn_ranks(args)
    if args.impl == "reference":
        return run_reference(args)
    if args.dry_run:
        return run_dry(args)
    return run_gpu(args)


if __name__ == "__main__":
    sys.exit(main())
