"""Workload descriptions and seeded generators (no method arithmetic here).

Model dims are Llama-2's [ext] (SURVEY.md §8 "Model dims"); the paper names the
model at PAPER.md:292 (§5.1) but prints no dims.  Client mixes follow
BASELINE.json `configs` with the readings listed in DESIGN.md §"Readings".
"""
from __future__ import annotations

import dataclasses
from dataclasses import dataclass, field

import numpy as np

__all__ = [
    "ModelCfg", "ClientCfg", "Workload", "TARGETS", "MODELS", "target_dims",
    "bf16_round", "bf16_bits", "bits_to_f32", "base_layer_weights", "client_adapters", "PREFIX",
    "client_inputs", "workload", "WORKLOAD_NAMES",
]

# LoRA target projections, in the bit order of include/menos.h (MENOS_T_*).
TARGETS = ("q", "k", "v", "o", "gate", "up", "down")
# Prefix tuning (NEXT-3): a client with targets == (PREFIX,) holds, per server layer, P = `rank`
# learned key and value vectors per KV head ("A" = prefix keys, "B" = prefix values, both [P, H_kv * hd]).
PREFIX = "prefix"


@dataclass(frozen=True)
class ModelCfg:
    name: str
    d_model: int
    n_heads: int
    n_kv_heads: int
    d_ff: int
    n_layers: int            # server layers (the segment [cut, L))
    first_layer: int = 1     # 0-indexed first server layer (layer 1 stays on the client)
    rms_eps: float = 1e-5
    rope_theta: float = 10000.0
    model_layers: int = 0    # decoder layers of the full model (0: first_layer + n_layers)
    arch: str = "llama"      # "llama" (RMSNorm, RoPE, SwiGLU) or "opt" (LayerNorm+bias, biases, ReLU; NEXT-4)

    @property
    def head_dim(self) -> int:
        return self.d_model // self.n_heads

    @property
    def total_layers(self) -> int:
        """Decoder layers of the whole model (unchanged by depth truncation)."""
        return self.model_layers if self.model_layers > 0 else self.first_layer + self.n_layers

    def with_layers(self, n: int) -> "ModelCfg":
        return dataclasses.replace(self, n_layers=n)


MODELS = {
    # tiny: BASELINE.json configs[0]
    "tiny": ModelCfg("tiny", 64, 4, 4, 172, 2, model_layers=3),
    # OPT (NEXT-4): tiny, and OPT-1.3B (d 2048, 32 heads, ffn 8192, 24 layers) [ext, HF config]
    "opt_tiny": ModelCfg("opt-tiny", 64, 4, 4, 256, 2, model_layers=3, arch="opt"),
    "opt1.3b": ModelCfg("opt-1.3b", 2048, 32, 32, 8192, 23, model_layers=24, arch="opt"),
    # Llama-2-7B / 13B / 70B server segments (layers 2..L, 1-indexed) [ext]
    "7b": ModelCfg("llama2-7b", 4096, 32, 32, 11008, 31, model_layers=32),
    "13b": ModelCfg("llama2-13b", 5120, 40, 40, 13824, 39, model_layers=40),
    "70b": ModelCfg("llama2-70b", 8192, 64, 8, 28672, 79, model_layers=80),
}


def target_dims(cfg: ModelCfg, t: str) -> tuple[int, int]:
    """(K_in, N_out) of projection t: y[.., N] = x[.., K] W[N, K]^T.  For PREFIX: (0, H_kv * hd), the width of one
    prefix key / value row."""
    d, hd = cfg.d_model, cfg.head_dim
    if t == PREFIX:
        return 0, cfg.n_kv_heads * hd
    return {
        "q": (d, cfg.n_heads * hd),
        "k": (d, cfg.n_kv_heads * hd),
        "v": (d, cfg.n_kv_heads * hd),
        "o": (cfg.n_heads * hd, d),
        "gate": (d, cfg.d_ff),
        "up": (d, cfg.d_ff),
        "down": (cfg.d_ff, d),
    }[t]


@dataclass
class ClientCfg:
    rank: int
    alpha: float
    targets: tuple[str, ...]
    seq_lens: list[int] = field(default_factory=list)
    cut: int = 0   # local index of the first server layer this client's tokens enter (NEXT-3; 0 = segment start)

    @property
    def n_tokens(self) -> int:
        return int(sum(self.seq_lens))


@dataclass
class Workload:
    name: str
    model: ModelCfg
    clients: list[ClientCfg]
    n_gpus: int = 1
    note: str = ""

    @property
    def n_tokens(self) -> int:
        return sum(c.n_tokens for c in self.clients)


# ---------------------------------------------------------------- bf16 encoding
def bf16_bits(x: np.ndarray) -> np.ndarray:
    """Round fp32 -> bf16 (round-to-nearest-even) and return the raw uint16 bits."""
    u = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32)
    lsb = (u >> 16) & 1
    r = (u + 0x7FFF + lsb) >> 16
    nan = np.isnan(np.asarray(x, dtype=np.float32))
    r = np.where(nan, 0x7FC0, r)
    return r.astype(np.uint16)


def bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (np.asarray(b, dtype=np.uint16).astype(np.uint32) << 16).view(np.float32)


def bf16_round(x: np.ndarray) -> np.ndarray:
    """fp32 array whose values are exactly bf16-representable (RNE)."""
    return bits_to_f32(bf16_bits(x))


# ---------------------------------------------------------------- generators
def _rng(*key: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(list(key)))


RECIPES = ("default", "plain")


def is_small(cfg: ModelCfg) -> bool:
    """The tiny Llama parity configs (d < 1024): weights are width-scaled (reading R26).  OPT keeps the
    Llama-width recipe at every size: with O(1) branches its ReLU MLP's fc1 LoRA grads are ill-conditioned in bf16 --
    an exact-bf16 evaluation of the oracle itself reaches only cos 0.9985-0.9991 (tools/bf16_emulation.py) -- so no
    bf16 kernel could meet the bar there; the OPT white-box test checks every intermediate instead."""
    return cfg.d_model < 1024 and cfg.arch != "opt"


def weight_std(cfg: ModelCfg, t: str, recipe: str = "default") -> float:
    """Init std of base projection t:
    * tiny configs (R26): 1/sqrt(K) for every projection, so each attention / MLP branch is O(1) against the
      residual stream as it is at Llama-2 width (0.02 = 1.28/sqrt(4096)); with 0.02 at d = 64 the branches are ~1%
      of the residual and a kernel that dropped one would still pass the activation bar;
    * Llama-2 widths, recipe "plain": N(0, 0.02^2) everywhere (Llama init std);
    * Llama-2 widths, recipe "default" (R27): q, k, v, gate, up 0.02; the residual-branch outputs o and down use the
      GPT-2 / Megatron depth-scaled std 0.02 / sqrt(2 L) (L = decoder layers of the whole model), so a 31-79 layer
      random residual stream grows like a trained pre-norm network's instead of doubling every few layers."""
    K, _ = target_dims(cfg, t)
    if is_small(cfg):
        return 1.0 / np.sqrt(K)
    if recipe == "plain" or t not in ("o", "down"):
        return 0.02
    return 0.02 / np.sqrt(2.0 * cfg.total_layers)


def base_layer_weights(cfg: ModelCfg, layer: int, seed: int = 0, recipe: str = "default") -> dict[str, np.ndarray]:
    """Frozen base weights of one decoder layer, natural (HF) layouts, fp32 bf16-representable.

    W ~ N(0, weight_std(cfg, t, recipe)^2) (readings R26 / R27); gains g = 1 + 0.1 N(0,1).
    """
    if recipe not in RECIPES:
        raise KeyError(recipe)
    out = {}
    names = ["q", "k", "v", "o", "gate", "up", "down"]
    for i, t in enumerate(names):
        K, N = target_dims(cfg, t)
        r = _rng(seed, layer, i)
        std = weight_std(cfg, t, recipe)
        out["w" + t] = bf16_round(r.standard_normal((N, K), dtype=np.float32) * np.float32(std))
    for j, g in enumerate(["g1", "g2"]):
        r = _rng(seed, layer, 100 + j)
        out[g] = bf16_round(1.0 + 0.1 * r.standard_normal(cfg.d_model, dtype=np.float32))
    if cfg.arch == "opt":
        # OPT: no gate; biases of q, k, v, o, fc1 (up), fc2 (down) and the LayerNorm biases ~ 0.02 N(0,1), nonzero
        # so that every bias path is exercised (trained OPT biases are nonzero)
        del out["wgate"]
        for j, t in enumerate(["q", "k", "v", "o", "up", "down"]):
            r = _rng(seed, layer, 200 + j)
            out["b" + t] = bf16_round(0.02 * r.standard_normal(target_dims(cfg, t)[1], dtype=np.float32))
        for j, bname in enumerate(["b1", "b2"]):
            r = _rng(seed, layer, 300 + j)
            out[bname] = bf16_round(0.1 * r.standard_normal(cfg.d_model, dtype=np.float32))
    return out


def client_adapters(cfg: ModelCfg, c: ClientCfg, seed: int, zero_b: bool = False
                    ) -> list[dict[str, tuple[np.ndarray, np.ndarray]]]:
    """Per server layer: {target: (A [r, K], B [N, r])}, fp32 bf16-representable.

    A ~ U(-1/sqrt(K), 1/sqrt(K)) (PEFT kaiming-uniform a=sqrt(5) bound);
    B ~ N(0, 0.02^2), nonzero so that dA != 0 (zero for invariant (b)).  Tiny configs (R26): B ~ N(0, 0.25/r), so
    the LoRA delta s (x A^T) B^T is a sizeable fraction of its projection (as for a trained adapter) and a kernel
    that dropped one client's adapter fails the activation bar.
    """
    layers = []
    b_std = np.sqrt(0.25 / c.rank) if is_small(cfg) else 0.02
    for ell in range(cfg.n_layers):
        d = {}
        if PREFIX in c.targets:   # prefix keys / values ~ N(0, 1) (PEFT's nn.Embedding init; O(1) like the layer's k, v)
            r = _rng(seed, ell, 50)
            N = target_dims(cfg, PREFIX)[1]
            d[PREFIX] = (bf16_round(r.standard_normal((c.rank, N), dtype=np.float32)),
                         bf16_round(r.standard_normal((c.rank, N), dtype=np.float32)))
            layers.append(d)
            continue
        for ti, t in enumerate(TARGETS):
            if t not in c.targets:
                continue
            K, N = target_dims(cfg, t)
            r = _rng(seed, ell, ti)
            bound = 1.0 / np.sqrt(K)
            A = bf16_round(r.uniform(-bound, bound, (c.rank, K)).astype(np.float32))
            if zero_b:
                B = np.zeros((N, c.rank), np.float32)
            else:
                B = bf16_round(r.standard_normal((N, c.rank), dtype=np.float32) * np.float32(b_std))
            d[t] = (A, B)
        layers.append(d)
    return layers


def client_inputs(cfg: ModelCfg, c: ClientCfg, seed: int, outlier: bool = False
                  ) -> tuple[np.ndarray, np.ndarray]:
    """x_c ~ N(0,1) and g_c ~ N(0,1), [T_c, d] fp32 bf16-representable.

    `outlier` multiplies two channels of x_c by 100 (massive-activation variant).
    """
    T = c.n_tokens
    x = _rng(seed, 0).standard_normal((T, cfg.d_model), dtype=np.float32)
    if outlier:
        x[:, 3] *= 100.0
        x[:, cfg.d_model // 2 + 1] *= 100.0
    g = _rng(seed, 1).standard_normal((T, cfg.d_model), dtype=np.float32)
    return bf16_round(x), bf16_round(g)


# ---------------------------------------------------------------- BASELINE.json configs
WORKLOAD_NAMES = ("cfg0_tiny", "cfg1_7b_x4", "cfg2_7b_x32_ragged", "cfg3_13b_x16", "cfg4_70b_tp8_x16")


def workload(name: str, n_layers: int | None = None) -> Workload:
    """BASELINE.json configs[k] (k = index in WORKLOAD_NAMES); `n_layers` truncates depth."""
    if name == "cfg0_tiny":
        m = MODELS["tiny"]
        cl = [ClientCfg(4, 8.0, ("q", "v"), [16, 16]) for _ in range(2)]
        w = Workload(name, m, cl, 1, "tiny 2-layer segment, 2 clients r=4 (alpha=2r), batch 2 x 16")
    elif name == "cfg1_7b_x4":
        m = MODELS["7b"]
        cl = [ClientCfg(8, 16.0, ("q", "v"), [512] * 4) for _ in range(4)]
        w = Workload(name, m, cl, 1, "Llama-2-7B layers 2..32, 4 clients r=8 q,v, batch 4 x 512")
    elif name == "cfg2_7b_x32_ragged":
        m = MODELS["7b"]
        r = _rng(42)
        cl = []
        for i in range(32):
            rank = [4, 8, 16][i % 3]
            lens = [int(s) for s in r.integers(128, 1025, size=4)]
            cl.append(ClientCfg(rank, 2.0 * rank, ("q", "v"), lens))
        w = Workload(name, m, cl, 8, "Llama-2-7B, 32 clients r in {4,8,16}, batch 4 x U{128..1024}")
    elif name == "cfg3_13b_x16":
        m = MODELS["13b"]
        cl = [ClientCfg(16, 32.0, TARGETS, [2048]) for _ in range(16)]
        w = Workload(name, m, cl, 8, "Llama-2-13B, 16 clients r=16 all projections, 1 x 2048")
    elif name == "opt13_x16_paper":
        # NEXT-4 extra (not a BASELINE config): the paper's OPT setting -- OPT-1.3B server layers
        # 2..24, LoRA r=8 alpha=16 on q,v, batch 16 x S~100 per client (S15) -- with 16 clients on one GPU
        m = MODELS["opt1.3b"]
        cl = [ClientCfg(8, 16.0, ("q", "v"), [100] * 16) for _ in range(16)]
        w = Workload(name, m, cl, 1, "OPT-1.3B, 16 clients r=8 q,v, batch 16 x 100 (paper's OPT setting)")
    elif name == "cfg4_70b_tp8_x16":
        m = MODELS["70b"]
        cl = [ClientCfg(8, 16.0, ("q", "v"), [1024, 1024]) for _ in range(16)]
        w = Workload(name, m, cl, 8, "Llama-2-70B TP-8, 16 clients r=8 q,v, 2 x 1024")
    else:
        raise KeyError(name)
    if n_layers is not None:
        w.model = w.model.with_layers(n_layers)
    return w
