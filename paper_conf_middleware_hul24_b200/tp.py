"""Tensor parallelism for the largest model (Llama-2-70B, BASELINE.json configs[4]).

Host-side logic only (argument marshalling): which slice of every base weight and LoRA adapter a rank holds, how the
shards reassemble, the NCCL unique id handshake (the library then drives NCCL itself), and a torch.distributed
collective callback (`menos_tp_cfg.collective`, include/menos.h) for the single-GPU gloo tests.  Every step of the
path runs in libmenos.so.

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


# ------------------------------------------------------------------------------------------- collectives
# include/menos.h menos_collective_fn: (op, send, recv, count, dtype, stream, user) -> int
COLLECTIVE_FN = C.CFUNCTYPE(C.c_int, C.c_int, C.c_void_p, C.c_void_p, C.c_size_t, C.c_int, C.c_void_p, C.c_void_p)
OP_ALLREDUCE, OP_ALLGATHER, OP_REDUCE_SCATTER = 0, 1, 2


class _CudaArray:
    """Minimal __cuda_array_interface__ holder so torch can view a raw device pointer without a copy."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3,
                                         "strides": None}


def make_torch_collective(group=None, device=None):
    """A Python callable (op, send, recv, count, dtype, stream) -> int for menos_tp_cfg.collective, implemented with
    torch.distributed on `group` and ordered on the library's stream.  Used for the single-GPU tests (gloo: ranks share
    one GPU, which NCCL does not allow); multi-GPU runs give the library an NCCL id instead (menos_tp_unique_id) so no
    Python runs on the per-layer path.  gloo has no reduce-scatter: it is an all-reduce of the full buffer followed by
    a copy of this rank's chunk (same sum, more bytes)."""
    import torch
    import torch.distributed as dist
    dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
    gloo = dist.get_backend(group) == "gloo"

    def view(ptr: int, n: int, dtype: int):
        if dtype == 0:
            return torch.as_tensor(_CudaArray(ptr, n, "<f4"), device=dev)
        return torch.as_tensor(_CudaArray(ptr, n, "<i2"), device=dev).view(torch.bfloat16)

    def fn(op: int, send: int, recv: int, count: int, dtype: int, stream: int) -> int:
        world = dist.get_world_size(group)
        rank = dist.get_rank(group)
        s = torch.cuda.ExternalStream(stream, device=dev) if stream else torch.cuda.default_stream(dev)
        with torch.cuda.stream(s):
            if op == OP_ALLREDUCE:
                t = view(recv, count, dtype)
                if gloo and dtype == 1:   # sum in fp32, one rounding to bf16 at the end (as NCCL's bf16 kernels do)
                    f = t.float()
                    dist.all_reduce(f, group=group)
                    t.copy_(f)
                else:
                    dist.all_reduce(t, group=group)
            elif op == OP_ALLGATHER:
                out = view(recv, count * world, dtype)
                src = view(send, count, dtype)
                if gloo:
                    parts = [torch.empty_like(src) for _ in range(world)]
                    dist.all_gather(parts, src.clone(), group=group)
                    out.copy_(torch.cat(parts))
                else:
                    dist.all_gather_into_tensor(out, src, group=group)
            elif op == OP_REDUCE_SCATTER:
                src = view(send, count * world, dtype)
                out = view(recv, count, dtype)
                if gloo:
                    f = src.float()
                    dist.all_reduce(f, group=group)
                    out.copy_(f[rank * count:(rank + 1) * count])
                else:
                    dist.reduce_scatter_tensor(out, src, group=group)
            else:
                return 1
        return 0

    return fn


def nccl_unique_id(lib=None) -> bytes:
    """128-byte NCCL unique id from libmenos (menos_tp_unique_id); rank 0 makes it, the caller broadcasts it."""
    from .menos import check, lib as _lib
    buf = C.create_string_buffer(128)
    check((lib or _lib()).menos_tp_unique_id(buf))
    return buf.raw


def wrap_collective(fn):
    """ctypes callback around a Python collective; exceptions become a nonzero status (MENOS_ENCCL)."""
    import traceback

    def cb(op, send, recv, count, dtype, stream, user):
        try:
            return int(fn(int(op), send or 0, recv or 0, int(count), int(dtype), stream or 0) or 0)
        except Exception:
            traceback.print_exc()
            return 1

    return COLLECTIVE_FN(cb)
