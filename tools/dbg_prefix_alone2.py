import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from tests.parity_util import make_inputs, new_server, register, run_gpu_step
from workloads import ClientCfg, MODELS, PREFIX, Workload
m = MODELS["tiny"]
w = Workload("mix", m, [ClientCfg(4, 8.0, ("q", "v"), [16, 16]), ClientCfg(4, 1.0, (PREFIX,), [9, 20]),
                        ClientCfg(8, 16.0, ("q","k","v","o","gate","up","down"), [33]), ClientCfg(2, 1.0, (PREFIX,), [1, 70, 5])])
inputs = make_inputs(w, seed=62)
weights, adapters, io = inputs
srv = new_server(w, weights)
ids = register(srv, w, adapters)
seq = os.environ.get("SEQ", "full,ng,alone")
res = {}
for step in seq.split(","):
    if step == "full": res["full"] = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids)
    if step == "full2": res["full2"] = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids)
    if step == "ng": res["ng"] = run_gpu_step(w, inputs=inputs, srv=srv, ids=ids, flags=1)
    if step == "alone":
        for i, c in enumerate(w.clients):
            res[f"alone{i}"] = run_gpu_step(Workload("one", m, [c]), inputs=(weights, [adapters[i]], [io[i]]), srv=srv, ids=[ids[i]])
f = res["full"]
for k, v in res.items():
    if k == "full": continue
    for i in range(len(w.clients)):
        j = 0 if k.startswith("alone") else i
        if k.startswith("alone") and k != f"alone{i}": continue
        print(k, i, "x_s", float(np.max(np.abs(v["x_s"][j] - f["x_s"][i]))), "g_s", float(np.max(np.abs(v["g_s"][j] - f["g_s"][i]))))
srv.close()
