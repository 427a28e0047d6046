"""Client -> GPU partitioning for replica mode (reading S19).

Clients are independent units (adapters per client, frozen shared base, no cross-client reduction:
PAPER.md:69, :119, :428), so the path shards by client with no collective: each GPU holds one base replica and
serves the clients assigned to it.  Assignment = LPT (longest processing time first) on per-client algorithmic
FLOPs (not tokens: attention adds an S^2 term); ties go to the lower GPU index, so every rank computes the same
deterministic assignment without communicating.
"""
from __future__ import annotations


def client_flops(d_model: int, n_heads: int, n_kv_heads: int, d_ff: int, n_layers: int, seq_lens, rank: int,
                 targets_dims) -> float:
    """Algorithmic fwd+bwd FLOPs of one client's tokens through the server segment (no recompute, no dW):
    4 P T + 12 hd H pairs L + sum_t 6 r (K+N) T L."""
    hd = d_model // n_heads
    P = n_layers * (d_model * (n_heads + 2 * n_kv_heads) * hd + d_model * n_heads * hd + 3 * d_model * d_ff)
    T = sum(seq_lens)
    pairs = sum(s * (s + 1) / 2 for s in seq_lens)
    lora = sum(6 * rank * (K + N) * T * n_layers for K, N in targets_dims)
    return 4.0 * P * T + 12.0 * hd * n_heads * pairs * n_layers + lora


def lpt_partition(costs, n_gpus: int) -> list[list[int]]:
    """Assign items (by index) to n_gpus bins: largest cost first onto the least-loaded bin (lowest index on
    ties).  Returns per-GPU lists of item indices, each in ascending index order (client-major packing)."""
    if n_gpus < 1:
        raise ValueError("n_gpus >= 1")
    order = sorted(range(len(costs)), key=lambda i: (-costs[i], i))
    load = [0.0] * n_gpus
    bins: list[list[int]] = [[] for _ in range(n_gpus)]
    for i in order:
        g = min(range(n_gpus), key=lambda k: (load[k], k))
        bins[g].append(i)
        load[g] += costs[i]
    return [sorted(b) for b in bins]


def workload_partition(w, n_gpus: int) -> list[list[int]]:
    """LPT partition of a workloads.Workload's clients over n_gpus replicas."""
    from workloads import target_dims  # input description only (no method arithmetic)
    m = w.model
    costs = [client_flops(m.d_model, m.n_heads, m.n_kv_heads, m.d_ff, m.n_layers, c.seq_lens, c.rank,
                          [target_dims(m, t) for t in c.targets]) for c in w.clients]
    return lpt_partition(costs, n_gpus)


def plan_waves(fwd_bytes, scratch_bytes, capacity: int) -> list[list[int]]:
    """Temporal sharing of the activation arena: split clients (in batch order) into
    consecutive waves whose SAVE activations plus the wave's scratch fit `capacity` bytes; each wave runs
    forward then backward before the next starts.  A client that cannot fit alone raises MemoryError (the
    caller would otherwise see MENOS_ENOMEM)."""
    waves: list[list[int]] = []
    cur: list[int] = []
    fb = sb = 0
    for i, (f, s) in enumerate(zip(fwd_bytes, scratch_bytes)):
        if f + s > capacity:
            raise MemoryError(f"client {i} needs {f + s} B > arena {capacity} B")
        if cur and fb + f + sb + s > capacity:
            waves.append(cur)
            cur, fb, sb = [], 0, 0
        cur.append(i)
        fb += f
        sb += s
    if cur:
        waves.append(cur)
    return waves


def plan_waves_exact(n_clients: int, demand, capacity: int) -> list[list[int]]:
    """Same greedy wave formation as plan_waves, with the EXACT peak arena demand of a candidate wave:
    demand(list_of_client_indices) -> bytes (the library's menos_batch_memory, which accounts for the block-diagonal
    LoRA slot columns a wave spans and the per-call scratch).  Clients keep batch order (client-major packing)."""
    waves: list[list[int]] = []
    cur: list[int] = []
    for i in range(n_clients):
        if demand([i]) > capacity:
            raise MemoryError(f"client {i} needs {demand([i])} B > arena {capacity} B")
        if cur and demand(cur + [i]) > capacity:
            waves.append(cur)
            cur = []
        cur.append(i)
    if cur:
        waves.append(cur)
    return waves
