"""Debug: SAVE vs NOGRAD forward x_s for batches with / without prefix clients (bitwise expected)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from tests.parity_util import _bf16, make_inputs, new_server, register
from workloads import ClientCfg, MODELS, PREFIX, Workload

def run(w, seed=62):
    inputs = make_inputs(w, seed=seed)
    weights, adapters, io = inputs
    srv = new_server(w, weights)
    ids = register(srv, w, adapters)
    sc, sl = [], []
    for i, c in enumerate(w.clients):
        sc += [ids[i]] * len(c.seq_lens); sl += list(c.seq_lens)
    x = _bf16(np.concatenate([a for a, _ in io]), "cuda")
    outs = []
    for flags in (0, 1, 0, 1):
        xs = torch.empty_like(x)
        b = srv.forward(sc, sl, x, xs, flags=flags)
        srv.batch_free(b)
        torch.cuda.synchronize()
        outs.append(xs.float().cpu().numpy())
    srv.close()
    return [float(np.max(np.abs(outs[k] - outs[0]))) for k in range(4)]

m = MODELS["tiny"]
for name, cl in [("lora", [ClientCfg(4, 8.0, ("q", "v"), [16, 16])]),
                 ("prefix_only", [ClientCfg(4, 1.0, (PREFIX,), [9, 20])]),
                 ("mix", [ClientCfg(4, 8.0, ("q", "v"), [16, 16]), ClientCfg(4, 1.0, (PREFIX,), [9, 20])]),
                 ("mix_plain_first", [ClientCfg(4, 1.0, (PREFIX,), [9, 20]), ClientCfg(4, 8.0, ("q", "v"), [16, 16])])]:
    print(name, run(Workload(name, m, cl)), flush=True)
