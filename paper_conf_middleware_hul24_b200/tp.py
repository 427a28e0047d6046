"""Tensor parallelism for the largest model (Llama-2-70B, BASELINE.json configs[4]).

Host-side logic only (argument marshalling): which slice of every base weight and LoRA adapter a rank holds, how the
shards reassemble, and the all-reduce callback `menos_tp_cfg.allreduce` (include/menos.h) implemented with
torch.distributed (NCCL over NVLink on a multi-GPU box; gloo for the single-GPU / CPU tests).  Every step of the
path still runs in libmenos.so; the library calls the callback at the four per-layer exchange points.

Split (Megatron, the paper's P:133 "more GPUs" reading for a model that does not fit one GPU's share):
  column-parallel q, k, v (heads), gate, up (rows of f): LoRA A [r, d] replicated, B [N/W, r] sharded;
  row-parallel o (columns of the heads), down (columns of f): LoRA A [r, K/W] sharded, B [d, r] replicated.
"""
from __future__ import annotations

import ctypes as C

COLUMN_PARALLEL = ("q", "k", "v", "gate", "up")
ROW_PARALLEL = ("o", "down")


def _heads_slice(rank: int, world: int, n: int, hd: int) -> slice:
    per = n // world
    return slice(rank * per * hd, (rank + 1) * per * hd)


def shard_slices(rank: int, world: int, n_heads: int, n_kv_heads: int, head_dim: int, d_ff: int) -> dict:
    """Per projection: (axis, slice) of the natural [N, K] weight that rank `rank` holds."""
    for name, v in (("n_heads", n_heads), ("n_kv_heads", n_kv_heads), ("d_ff", d_ff)):
        if v % world:
            raise ValueError(f"{name}={v} not divisible by tensor-parallel world {world}")
    q = _heads_slice(rank, world, n_heads, head_dim)
    kv = _heads_slice(rank, world, n_kv_heads, head_dim)
    fp = d_ff // world
    f = slice(rank * fp, (rank + 1) * fp)
    return {"q": (0, q), "k": (0, kv), "v": (0, kv), "o": (1, q), "gate": (0, f), "up": (0, f), "down": (1, f)}


def _take(x, axis: int, sl: slice):
    return x[sl] if axis == 0 else x[:, sl]


def shard_layer_weights(w: dict, rank: int, world: int, n_heads: int, n_kv_heads: int, head_dim: int,
                        d_ff: int) -> dict:
    """The rank's shard of one layer's base weights (dict with wq..wdown, g1, g2; numpy or torch, natural
    layouts).  Returns contiguous arrays in the layouts include/menos.h documents for tensor parallelism."""
    sl = shard_slices(rank, world, n_heads, n_kv_heads, head_dim, d_ff)
    out = {}
    for t, (axis, s) in sl.items():
        v = _take(w["w" + t], axis, s)
        out["w" + t] = v.contiguous() if hasattr(v, "contiguous") else v.copy()
    out["g1"], out["g2"] = w["g1"], w["g2"]
    return out


def shard_adapter(t: str, A, B, rank: int, world: int, n_heads: int, n_kv_heads: int, head_dim: int, d_ff: int):
    """(A_local, B_local) of target t: column-parallel -> (A, B rows of the shard); row-parallel ->
    (A columns of the shard, B)."""
    axis, s = shard_slices(rank, world, n_heads, n_kv_heads, head_dim, d_ff)[t]
    if t in COLUMN_PARALLEL:
        return A, B[s]
    return A[:, s], B


def gather_adapter(t: str, shards: list, which: str = "grad"):
    """Reassemble a full (A, B) (or (dA, dB)) from the per-rank local tensors [(A_r, B_r), ...] (rank order).
    Replicated tensors must be identical on every rank; the first one is returned."""
    import numpy as np
    As, Bs = [a for a, _ in shards], [b for _, b in shards]
    if t in COLUMN_PARALLEL:
        return As[0], np.concatenate(Bs, axis=0)
    return np.concatenate(As, axis=1), Bs[0]


# ------------------------------------------------------------------------------------------- all-reduce callback
ALLREDUCE_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_size_t, C.c_int, C.c_void_p, C.c_void_p)


class _CudaArray:
    """Minimal __cuda_array_interface__ holder so torch can view a raw device pointer without a copy."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3,
                                         "strides": None}


def make_torch_allreduce(group=None, device=None):
    """A Python callable (buf, count, dtype, stream) -> int for menos_tp_cfg.allreduce: an in-place SUM
    all-reduce of the device buffer with torch.distributed on `group`, ordered on the library's stream
    (the collective waits for the work queued on `stream`; later work on `stream` waits for the collective)."""
    import torch
    import torch.distributed as dist
    dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
    views: dict = {}

    def fn(buf: int, count: int, dtype: int, stream: int) -> int:
        key = (buf, count, dtype)
        t = views.get(key)
        if t is None:
            if len(views) > 256:
                views.clear()
            if dtype == 0:
                t = torch.as_tensor(_CudaArray(buf, count, "<f4"), device=dev)
            else:
                t = torch.as_tensor(_CudaArray(buf, count, "<i2"), device=dev).view(torch.bfloat16)
            views[key] = t
        s = torch.cuda.ExternalStream(stream, device=dev) if stream else torch.cuda.default_stream(dev)
        with torch.cuda.stream(s):
            dist.all_reduce(t, group=group)
        return 0

    return fn


def wrap_allreduce(fn):
    """ctypes callback around a Python all-reduce callable; exceptions become a nonzero status (MENOS_ENCCL)."""
    import traceback

    def cb(buf, count, dtype, stream, user):
        try:
            return int(fn(buf or 0, int(count), int(dtype), stream or 0) or 0)
        except Exception:
            traceback.print_exc()
            return 1

    return ALLREDUCE_FN(cb)
