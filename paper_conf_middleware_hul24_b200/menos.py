"""Thin ctypes binding of libmenos.so (include/menos.h) -- argument marshalling only.

Every step of the Menos server path runs in the library's sm_100a kernels.  There is no Python or CPU
fallback: if the shared library is missing or no sm_100 GPU is present, the calls raise.
Buffers may be torch tensors (device or pinned host), numpy arrays (host) or raw integer addresses.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "_lib", "libmenos.so")

TARGET_BITS = {"q": 1, "k": 2, "v": 4, "o": 8, "gate": 16, "up": 32, "down": 64, "prefix": 128}
TARGET_INDEX = {"q": 0, "k": 1, "v": 2, "o": 3, "gate": 4, "up": 5, "down": 6, "prefix": 7}
FWD_SAVE, FWD_NOGRAD = 0, 1
ARCH = {"llama": 0, "opt": 1}
MEM_BOUND = 2
REQ_FWD, REQ_BWD = 0, 1
WHICH = {"A": 0, "B": 1, "dA": 2, "dB": 3, "mA": 4, "mB": 5, "vA": 6, "vB": 7}
STATUS = {0: "OK", -1: "EINVAL", -2: "ENOMEM", -3: "ENOCLIENT", -4: "ESTATE", -5: "ECUDA", -6: "ENCCL"}


class MenosError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"menos {STATUS.get(code, code)}: {msg}")
        self.code = code


class ModelCfg(C.Structure):
    _fields_ = [("d_model", C.c_int), ("n_heads", C.c_int), ("n_kv_heads", C.c_int), ("d_ff", C.c_int),
                ("rms_eps", C.c_float), ("rope_theta", C.c_float), ("arch", C.c_int)]


class LayerWeights(C.Structure):
    _fields_ = [(n, C.c_void_p) for n in ("wq", "wk", "wv", "wo", "wgate", "wup", "wdown", "g1", "g2",
                                          "bq", "bk", "bv", "bo", "bup", "bdown", "b1", "b2")]


class AdamWCfg(C.Structure):
    _fields_ = [("lr", C.c_double), ("beta1", C.c_double), ("beta2", C.c_double), ("eps", C.c_double),
                ("weight_decay", C.c_double)]


from .tp import COLLECTIVE_FN, wrap_collective  # noqa: E402


class TPCfg(C.Structure):
    _fields_ = [("rank", C.c_int), ("world", C.c_int), ("collective", COLLECTIVE_FN), ("user", C.c_void_p),
                ("nccl_id", C.c_void_p)]


class ServerOpts(C.Structure):
    _fields_ = [("max_clients", C.c_int), ("max_rank", C.c_int), ("max_seq_len", C.c_int),
                ("arena_bytes", C.c_size_t), ("num_sms", C.c_int), ("tp", TPCfg)]


class Stats(C.Structure):
    _fields_ = [("base_bytes", C.c_size_t), ("adapters_bytes", C.c_size_t), ("arena_bytes", C.c_size_t),
                ("arena_used", C.c_size_t), ("arena_peak", C.c_size_t), ("n_clients", C.c_int),
                ("num_sms", C.c_int)]


class SchedGrant(C.Structure):
    _fields_ = [("client", C.c_int32), ("kind", C.c_int32), ("bytes", C.c_size_t)]


class KernelStat(C.Structure):
    _fields_ = [("name", C.c_char * 32), ("launches", C.c_int), ("ms", C.c_double), ("flops", C.c_double),
                ("bytes", C.c_double)]


_lib = None

# (name, restype, argtypes) for every symbol include/menos.h and include/menos_testing.h declare
_P, _I, _F, _S = C.c_void_p, C.c_int, C.c_float, C.c_size_t
_PI32 = C.POINTER(C.c_int32)
SIGNATURES = {
    "menos_server_create": (_I, [C.POINTER(ModelCfg), _I, _I, C.POINTER(LayerWeights), _I, C.POINTER(ServerOpts),
                                 C.POINTER(_P)]),
    "menos_server_load_layer": (_I, [_P, _I, C.POINTER(LayerWeights)]),
    "menos_server_destroy": (None, [_P]),
    "menos_register_client": (_I, [_P, _I, _F, C.c_uint32, C.POINTER(AdamWCfg), C.c_uint64, _PI32]),
    "menos_register_client_at": (_I, [_P, _I, _I, _F, C.c_uint32, C.POINTER(AdamWCfg), C.c_uint64, _PI32]),
    "menos_unregister_client": (_I, [_P, C.c_int32]),
    "menos_client_memory": (_I, [_P, C.c_int32, _I, C.POINTER(_S), C.POINTER(_S), C.POINTER(_S)]),
    "menos_batch_memory": (_I, [_P, _I, _PI32, _PI32, _I, C.POINTER(_S), C.POINTER(_S)]),
    "menos_forward": (_I, [_P, _I, _PI32, _PI32, _P, _P, _I, _P, C.POINTER(_P)]),
    "menos_backward": (_I, [_P, _P, _P, _P, _P]),
    "menos_batch_free": (_I, [_P, _P]),
    "menos_adapter_step": (_I, [_P, _I, _PI32, _P]),
    "menos_adapter_shape": (_I, [_P, C.c_int32, _I, C.POINTER(_I), C.POINTER(_I)]),
    "menos_get_adapter": (_I, [_P, C.c_int32, _I, _I, _I, C.POINTER(C.c_float)]),
    "menos_set_adapter": (_I, [_P, C.c_int32, _I, _I, _I, C.POINTER(C.c_float)]),
    "menos_get_stats": (_I, [_P, C.POINTER(Stats)]),
    "menos_launch_count": (C.c_ulonglong, []),
    "menos_profile_enable": (_I, [_I]),
    "menos_profile_read": (_I, [C.POINTER(KernelStat), _I, C.POINTER(_I)]),
    "menos_sync": (_I, [_P]),
    "menos_tp_unique_id": (_I, [_P]),
    "menos_tp_stats": (_I, [_P, C.POINTER(C.c_longlong), C.POINTER(C.c_double)]),
    "menos_last_error": (C.c_char_p, []),
    "menos_test_gemm": (_I, [_I, _I, _I, _I, _P, _I, _P, _I, _P, _I, _P, _I, _I, _PI32, _I, _P, _I, _P, _I, _P, _I,
                             _P, _I, _I, _I, _PI32, _F, _I]),
    "menos_test_attention": (_I, [_I, _PI32, _I, _I, _I, _P, _P, _P, _P, _P, _F]),
    "menos_test_rmsnorm": (_I, [_I, _I, _P, _P, _F, _P, _P, _P, _P, _P, _P]),
    "menos_test_batch_tensor": (_I, [_P, _P, _I, _I, _P, C.POINTER(_S)]),
    "menos_test_lora_rows": (_I, [_P, _P, _P, _I, _I, _I, _I, _I, _I, _I, _F]),
    "menos_test_lora_tokred": (_I, [_P, _P, _P, _I, _I, _I, _I, _I, _I, _I, _I, _F, _I]),
    "menos_test_set_gemm_cta_group": (_I, [_I]),
    "menos_test_gemm_time": (_I, [_I, _I, _I, _I, _P, _P, _P, _I, _P, _I, C.POINTER(C.c_float)]),
    "menos_test_set_attn_tc": (_I, [_I]),
    "menos_test_set_ds_cap": (_I, [C.c_longlong]),
    "menos_test_ds_plan": (_I, [_I, _PI32, _I, _I, C.c_longlong, _PI32, _PI32, _PI32, _I, _PI32, _PI32, _PI32]),
    "menos_test_ds_plan_q": (_I, [_I, _PI32, _I, _I, C.c_longlong, _I, _PI32, _I, _PI32, _PI32, _I, _PI32]),
    "menos_test_abf_prof": (_I, [C.POINTER(C.c_ulonglong)]),
    "menos_testing_last_error": (C.c_char_p, []),
    "menos_sched_create": (_I, [_S, _I, C.POINTER(_P)]),
    "menos_sched_destroy": (None, [_P]),
    "menos_sched_set_demand": (_I, [_P, C.c_int32, _S, _S]),
    "menos_sched_arrive": (_I, [_P, C.c_int32, _I, C.POINTER(SchedGrant), _I, C.POINTER(_I)]),
    "menos_sched_complete": (_I, [_P, C.c_int32, C.POINTER(SchedGrant), _I, C.POINTER(_I)]),
    "menos_sched_state": (_I, [_P, C.POINTER(_S), C.POINTER(_I), C.POINTER(_I), _PI32, _I]),
    "menos_sched_timing": (_I, [_P, C.POINTER(C.c_longlong), C.POINTER(C.c_double), C.POINTER(C.c_double)]),
}


def lib():
    """Load libmenos.so (built in-tree by build.py / __graft_entry__.build()).  Raises if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise FileNotFoundError(f"{LIB_PATH} not built: run __graft_entry__.build() (no CPU fallback exists)")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def ptr(x) -> int | None:
    """Address of a torch tensor / numpy array / int (None for None)."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    raise TypeError(type(x))


def check(rc: int, testing: bool = False):
    if rc != 0:
        msg = (lib().menos_testing_last_error() if testing else lib().menos_last_error()) or b""
        raise MenosError(rc, msg.decode(errors="replace"))


def _stream(stream) -> int | None:
    if stream is None:
        return None
    if hasattr(stream, "cuda_stream"):
        return stream.cuda_stream
    return int(stream)


def _i32(seq):
    arr = (C.c_int32 * len(seq))(*[int(v) for v in seq])
    return arr


def _check_act(name: str, x, n_tokens: int, d_model: int, device: int | None):
    """x_c / x_s / g_c / g_s must be bf16, contiguous, [sum(seq_len), d_model], on the server's GPU or in host memory:
    the library trusts T from seq_len, so a short, strided or fp32 buffer would be read / written out of bounds."""
    if isinstance(x, int):
        return   # raw address: the caller vouches for it (include/menos.h)
    want = n_tokens * d_model
    if hasattr(x, "data_ptr"):
        import torch
        if x.dtype != torch.bfloat16:
            raise MenosError(-1, f"{name}: dtype {x.dtype}, expected torch.bfloat16")
        if not x.is_contiguous():
            raise MenosError(-1, f"{name}: not contiguous")
        if x.numel() != want:
            raise MenosError(-1, f"{name}: {tuple(x.shape)} has {x.numel()} elements, expected [{n_tokens}, {d_model}]")
        if x.is_cuda and device is not None and x.device.index != device:
            raise MenosError(-1, f"{name}: on cuda:{x.device.index}, the server is on cuda:{device}")
        return
    if hasattr(x, "ctypes"):   # numpy: raw bf16 bits
        if x.dtype.itemsize != 2 or not x.flags["C_CONTIGUOUS"] or x.size != want:
            raise MenosError(-1, f"{name}: numpy buffer must be contiguous 2-byte bf16 bits of [{n_tokens}, {d_model}]")
        return
    raise TypeError(f"{name}: unsupported buffer type {type(x)}")


class Batch:
    def __init__(self, server: "Server", handle: int, n_tokens: int):
        self.server, self.handle, self.n_tokens = server, handle, n_tokens


class Server:
    """One Menos server segment on one GPU: menos_server_create ... menos_server_destroy."""

    def __init__(self, d_model, n_heads, n_kv_heads, d_ff, n_layers, first_layer=1, rms_eps=1e-5,
                 rope_theta=1e4, weights=None, device=0, max_clients=64, max_rank=64, max_seq_len=4096,
                 arena_bytes=0, num_sms=0, tp=None, arch="llama"):
        """tp = (rank, world, transport) for tensor parallelism (include/menos.h menos_tp_cfg): `weights` are then the
        rank's shards (tp.shard_layer_weights); transport is either the 128-byte NCCL unique id (bytes, from
        tp.nccl_unique_id on rank 0, broadcast by the caller: the library drives NCCL itself) or a Python collective
        (op, send, recv, count, dtype, stream) -> int (tp.make_torch_collective)."""
        self.cfg = ModelCfg(d_model, n_heads, n_kv_heads, d_ff, rms_eps, rope_theta, ARCH[arch])
        self.n_layers = n_layers
        self.device = device
        tpc = TPCfg(0, 1, COLLECTIVE_FN(), None, None)
        self._tp_cb = self._tp_id = None
        if tp is not None and (tp[1] > 1 or isinstance(tp[2], (bytes, bytearray))):
            if isinstance(tp[2], (bytes, bytearray)):
                self._tp_id = C.create_string_buffer(bytes(tp[2]), 128)
                tpc = TPCfg(tp[0], tp[1], COLLECTIVE_FN(), None, C.cast(self._tp_id, C.c_void_p))
            else:
                self._tp_cb = wrap_collective(tp[2])   # kept alive as long as the server
                tpc = TPCfg(tp[0], tp[1], self._tp_cb, None, None)
        self.tp_rank, self.tp_world = (tp[0], tp[1]) if tp is not None else (0, 1)
        opts = ServerOpts(max_clients, max_rank, max_seq_len, arena_bytes, num_sms, tpc)
        h = C.c_void_p()
        warr = None
        if weights is not None:
            warr = (LayerWeights * n_layers)(*[self._lw(w) for w in weights])
        check(lib().menos_server_create(C.byref(self.cfg), first_layer, n_layers, warr, device, C.byref(opts),
                                        C.byref(h)))
        self.h = h.value

    @staticmethod
    def _lw(w: dict) -> LayerWeights:
        return LayerWeights(*[ptr(w.get(k)) for k, _ in LayerWeights._fields_])

    def load_layer(self, layer: int, w: dict):
        lw = self._lw(w)
        check(lib().menos_server_load_layer(self.h, layer, C.byref(lw)))

    def close(self):
        if getattr(self, "h", None):
            lib().menos_server_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ---------------------------------------------------------------- clients
    def register_client(self, rank, alpha, targets=("q", "v"), lr=1e-4, betas=(0.9, 0.999), eps=1e-8,
                        weight_decay=0.01, seed=0, cut_layer=None) -> int:
        """cut_layer (absolute layer index, NEXT-3): where the client's tokens enter; None = the segment's first."""
        mask = 0
        for t in targets:
            mask |= TARGET_BITS[t]
        opt = AdamWCfg(lr, betas[0], betas[1], eps, weight_decay)
        cid = C.c_int32()
        if cut_layer is None:
            check(lib().menos_register_client(self.h, rank, alpha, mask, C.byref(opt), seed, C.byref(cid)))
        else:
            check(lib().menos_register_client_at(self.h, cut_layer, rank, alpha, mask, C.byref(opt), seed,
                                                 C.byref(cid)))
        return cid.value

    def unregister_client(self, cid: int):
        check(lib().menos_unregister_client(self.h, cid))

    def client_memory(self, cid: int, n_tokens: int):
        a, b, c = C.c_size_t(), C.c_size_t(), C.c_size_t()
        check(lib().menos_client_memory(self.h, cid, n_tokens, C.byref(a), C.byref(b), C.byref(c)))
        return a.value, b.value, c.value

    def batch_memory(self, client_ids, n_tokens, flags=FWD_SAVE):
        """(fwd_bytes, bwd_bytes): exact peak arena demand of one batched forward / backward over these clients."""
        a, b = C.c_size_t(), C.c_size_t()
        check(lib().menos_batch_memory(self.h, len(client_ids), _i32(client_ids), _i32(n_tokens), flags, C.byref(a),
                                       C.byref(b)))
        return a.value, b.value

    def adapter_shape(self, cid: int, target: str):
        r = (C.c_int * 2)()
        c = (C.c_int * 2)()
        check(lib().menos_adapter_shape(self.h, cid, TARGET_INDEX[target], r, c))
        return (r[0], c[0]), (r[1], c[1])

    def get_adapter(self, cid: int, layer: int, target: str, which: str):
        import numpy as np
        (ra, ca), (rb, cb) = self.adapter_shape(cid, target)
        shape = (ra, ca) if WHICH[which] % 2 == 0 else (rb, cb)
        out = np.empty(shape, np.float32)
        check(lib().menos_get_adapter(self.h, cid, layer, TARGET_INDEX[target], WHICH[which],
                                      out.ctypes.data_as(C.POINTER(C.c_float))))
        return out

    def set_adapter(self, cid: int, layer: int, target: str, which: str, value):
        import numpy as np
        v = np.ascontiguousarray(value, dtype=np.float32)
        check(lib().menos_set_adapter(self.h, cid, layer, TARGET_INDEX[target], WHICH[which],
                                      v.ctypes.data_as(C.POINTER(C.c_float))))

    # ---------------------------------------------------------------- the hot path
    def forward(self, seq_client, seq_len, x_c, x_s, flags=FWD_SAVE, stream=None, retain=True) -> Batch | None:
        """retain=False (NOGRAD only): nothing is kept after the call (Alg.1 L6-7); returns None."""
        T = int(sum(seq_len))
        _check_act("x_c", x_c, T, self.cfg.d_model, self.device)
        _check_act("x_s", x_s, T, self.cfg.d_model, self.device)
        b = C.c_void_p()
        check(lib().menos_forward(self.h, len(seq_client), _i32(seq_client), _i32(seq_len), ptr(x_c), ptr(x_s),
                                  flags, _stream(stream), C.byref(b) if retain else None))
        return Batch(self, b.value, int(sum(seq_len))) if retain else None

    def backward(self, batch: Batch, g_c, g_s, stream=None):
        _check_act("g_c", g_c, batch.n_tokens, self.cfg.d_model, self.device)
        _check_act("g_s", g_s, batch.n_tokens, self.cfg.d_model, self.device)
        check(lib().menos_backward(self.h, batch.handle, ptr(g_c), ptr(g_s), _stream(stream)))
        batch.handle = None

    def batch_free(self, batch: Batch):
        if batch.handle:
            check(lib().menos_batch_free(self.h, batch.handle))
            batch.handle = None

    def batch_tensor(self, batch: Batch, layer: int, which: int):
        """White-box test hook (include/menos_testing.h menos_test_batch_tensor): one saved intermediate of a live
        SAVE batch as raw bytes (numpy uint8); the caller interprets dtype / shape."""
        import numpy as np
        n = C.c_size_t()
        check(lib().menos_test_batch_tensor(self.h, batch.handle, layer, which, None, C.byref(n)), testing=False)
        out = np.empty(n.value, np.uint8)
        if n.value:
            check(lib().menos_test_batch_tensor(self.h, batch.handle, layer, which, out.ctypes.data, C.byref(n)))
        return out

    def adapter_step(self, client_ids, stream=None):
        check(lib().menos_adapter_step(self.h, len(client_ids), _i32(client_ids), _stream(stream)))

    def stats(self) -> dict:
        s = Stats()
        check(lib().menos_get_stats(self.h, C.byref(s)))
        return {k: getattr(s, k) for k, _ in Stats._fields_}

    def sync(self):
        check(lib().menos_sync(self.h))

    def tp_stats(self) -> dict:
        """Collectives the tensor-parallel path issued and their payload bytes (menos_tp_stats)."""
        n, b = C.c_longlong(), C.c_double()
        check(lib().menos_tp_stats(self.h, C.byref(n), C.byref(b)))
        return {"calls": n.value, "bytes": b.value}


def launch_count() -> int:
    return int(lib().menos_launch_count())


def profile_enable(on: bool = True):
    check(lib().menos_profile_enable(1 if on else 0))


def profile_read() -> dict:
    arr = (KernelStat * 16)()
    n = C.c_int()
    check(lib().menos_profile_read(arr, 16, C.byref(n)))
    return {arr[i].name.decode(): {"launches": arr[i].launches, "ms": arr[i].ms, "flops": arr[i].flops,
                                   "bytes": arr[i].bytes} for i in range(n.value)}


class Scheduler:
    """Algorithm 2: FCFS + backfilling over GPU memory; native (menos_sched_*)."""

    def __init__(self, m_avail: int, max_clients: int = 64):
        h = C.c_void_p()
        check(lib().menos_sched_create(m_avail, max_clients, C.byref(h)))
        self.h, self.max_clients = h.value, max_clients
        self._out = (SchedGrant * max_clients)()

    def close(self):
        if getattr(self, "h", None):
            lib().menos_sched_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_demand(self, client: int, m_f: int, m_b: int):
        check(lib().menos_sched_set_demand(self.h, client, m_f, m_b))

    def _grants(self, n):
        return [(self._out[i].client, self._out[i].kind, self._out[i].bytes) for i in range(n.value)]

    def arrive(self, client: int, kind: int) -> list[tuple[int, int, int]]:
        """Alg.2 L7-9; returns the grants [(client, kind, bytes)] of the SCHEDULE call, in grant order."""
        n = C.c_int()
        check(lib().menos_sched_arrive(self.h, client, kind, self._out, self.max_clients, C.byref(n)))
        return self._grants(n)

    def complete(self, client: int) -> list[tuple[int, int, int]]:
        """Alg.2 L10-13."""
        n = C.c_int()
        check(lib().menos_sched_complete(self.h, client, self._out, self.max_clients, C.byref(n)))
        return self._grants(n)

    def state(self) -> dict:
        a, w, r = C.c_size_t(), C.c_int(), C.c_int()
        buf = (C.c_int32 * self.max_clients)()
        check(lib().menos_sched_state(self.h, C.byref(a), C.byref(w), C.byref(r), buf, self.max_clients))
        return {"m_avail": a.value, "waiting": list(buf[:w.value]), "n_running": r.value}

    def timing(self) -> dict:
        n, mean, mx = C.c_longlong(), C.c_double(), C.c_double()
        check(lib().menos_sched_timing(self.h, C.byref(n), C.byref(mean), C.byref(mx)))
        return {"decisions": n.value, "mean_ns": mean.value, "max_ns": mx.value}
