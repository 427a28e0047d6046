"""Debug: client 0 (LoRA) alone vs in a batch with prefix clients: first saved intermediate that differs."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from tests.parity_util import _bf16, make_inputs, new_server, register
from workloads import ClientCfg, MODELS, PREFIX, Workload

m = MODELS["tiny"]
w = Workload("mix", m, [ClientCfg(4, 8.0, ("q", "v"), [16, 16]), ClientCfg(4, 1.0, (PREFIX,), [9, 20]),
                        ClientCfg(2, 1.0, (PREFIX,), [1, 70, 5])])
inputs = make_inputs(w, seed=62)
weights, adapters, io = inputs
srv = new_server(w, weights)
ids = register(srv, w, adapters)

def fwd(clients):
    sc, sl, xs_ = [], [], []
    for i in clients:
        c = w.clients[i]
        sc += [ids[i]] * len(c.seq_lens); sl += list(c.seq_lens); xs_.append(io[i][0])
    x = _bf16(np.concatenate(xs_), "cuda")
    xs = torch.empty_like(x)
    b = srv.forward(sc, sl, x, xs)
    torch.cuda.synchronize()
    vals = {}
    for l in range(m.n_layers):
        for k, wh in (("x", 0), ("xn", 1), ("qkv", 2), ("O", 3), ("h", 4), ("hn", 5), ("lse", 12)):
            raw = srv.batch_tensor(b, l, wh)
            vals[(l, k)] = raw
    srv.batch_free(b)
    return xs.float().cpu().numpy(), vals

xa, va = fwd([0])
xb, vb = fwd([0, 1, 2])
T0 = 32
print("x_s equal:", np.array_equal(xa, xb[:T0]), float(np.max(np.abs(xa - xb[:T0]))))
Tb = sum(w.clients[i].n_tokens for i in range(3))
for key in va:
    a, b = va[key], vb[key]
    k = key[1]
    if k == "lse":
        A = a.view(np.float32).reshape(m.n_heads, -1)[:, :T0]
        B = b.view(np.float32).reshape(m.n_heads, -1)[:, :T0]
    else:
        A = a.reshape(T0, -1)
        B = b.reshape(Tb, -1)[:T0]
    print(key, "equal" if np.array_equal(A, B) else "DIFF", flush=True)
srv.close()
