"""Diagnose the gap between the device-resident step and the host-buffer (e2e) step of bench.py.

Prints: pinned H2D/D2H bandwidth of one x_c-sized tensor, the device-resident step time, the host enqueue time of
one device-resident step (wall time of the python call while the GPU is busy), and the host-buffer step time.
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from workloads import workload  # noqa: E402


def main():
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    w = workload(os.environ.get("WL", "cfg1_7b_x4"))
    srv = bench.build_server(torch, w, dev, seed=0, arena_gb=80)
    ids = bench.register_clients(np, srv, w, seed=1)
    T, d = w.n_tokens, w.model.d_model
    sc, sl = [], []
    for i, c in enumerate(w.clients):
        sc += [ids[i]] * len(c.seq_lens)
        sl += list(c.seq_lens)
    x = torch.randn(T, d, device=dev).to(torch.bfloat16)
    g = torch.randn(T, d, device=dev).to(torch.bfloat16)
    xs, gs = torch.empty_like(x), torch.empty_like(x)
    st = torch.cuda.current_stream()

    def step(a, b, c, e):
        bt = srv.forward(sc, sl, a, b, stream=st)
        srv.backward(bt, c, e, stream=st)
        srv.adapter_step(ids, stream=st)

    def ev_time(fn, k=3):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(k):
            fn()
        e1.record(st)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / k

    for _ in range(3):
        step(x, xs, g, gs)
    hx = x.cpu().pin_memory()
    hxs = torch.empty_like(hx).pin_memory()
    print("pinned:", hx.is_pinned(), hxs.is_pinned())
    h2d = ev_time(lambda: x.copy_(hx, non_blocking=True))
    d2h = ev_time(lambda: hxs.copy_(x, non_blocking=True))
    nb = x.numel() * 2
    print(f"H2D {nb/1e6:.0f} MB: {h2d:.2f} ms = {nb/h2d/1e6:.1f} GB/s; D2H {d2h:.2f} ms = {nb/d2h/1e6:.1f} GB/s")
    dev_ms = ev_time(lambda: step(x, xs, g, gs))
    print(f"device-resident step {dev_ms:.1f} ms")
    # host enqueue time: keep the GPU busy with a long step first, then time the python call of another
    torch.cuda.synchronize()
    step(x, xs, g, gs)
    t0 = time.perf_counter()
    step(x, xs, g, gs)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"host enqueue of one step (GPU busy): {(t1-t0)*1e3:.1f} ms")
    t0 = time.perf_counter()
    bt = srv.forward(sc, sl, x, xs, stream=st)
    t1 = time.perf_counter()
    srv.backward(bt, g, gs, stream=st)
    t2 = time.perf_counter()
    srv.adapter_step(ids, stream=st)
    t3 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"enqueue: fwd {(t1-t0)*1e3:.1f} ms, bwd {(t2-t1)*1e3:.1f} ms, step {(t3-t2)*1e3:.1f} ms")
    hg = g.cpu().pin_memory()
    hgs = torch.empty_like(hg).pin_memory()
    step(hx, hxs, hg, hgs)
    host_ms = ev_time(lambda: step(hx, hxs, hg, hgs))
    print(f"host-buffer step {host_ms:.1f} ms")
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    bt = srv.forward(sc, sl, hx, hxs, stream=st)
    t1 = time.perf_counter()
    srv.backward(bt, hg, hgs, stream=st)
    t2 = time.perf_counter()
    srv.adapter_step(ids, stream=st)
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    print(f"host-buffer wall: fwd {(t1-t0)*1e3:.1f} ms, bwd {(t2-t1)*1e3:.1f} ms, step+sync {(t3-t2)*1e3:.1f} ms")
    # per-call device segments over 4 host-buffer steps
    for it in range(int(os.environ.get('NSTEPS', '4'))):
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        w0 = time.perf_counter()
        ev[0].record(st)
        bt = srv.forward(sc, sl, hx, hxs, stream=st)
        ev[1].record(st)
        w1 = time.perf_counter()
        srv.backward(bt, hg, hgs, stream=st)
        ev[2].record(st)
        w2 = time.perf_counter()
        srv.adapter_step(ids, stream=st)
        ev[3].record(st)
        torch.cuda.synchronize()
        w3 = time.perf_counter()
        print(f"step {it}: device fwd {ev[0].elapsed_time(ev[1]):.1f} gap+bwd {ev[1].elapsed_time(ev[2]):.1f} "
              f"adam {ev[2].elapsed_time(ev[3]):.1f} ms | wall fwd {(w1-w0)*1e3:.1f} bwd {(w2-w1)*1e3:.1f} "
              f"rest {(w3-w2)*1e3:.1f}")
    srv.close()


if __name__ == "__main__":
    main()
