"""Host logic of the dS-stored attention backward (no GPU): the dS^T tile count per sequence, the bound
menos_batch_memory charges for it, and the chunk plan (attn_ds_plan through menos_test_ds_plan).

The tile layout: per (sequence, head), key block kb (128 keys) pairs with the 64-query blocks
qb = 2 kb .. ceil(L/64) - 1 (the causal ones: a query block before the key block sees none of its keys)."""
import ctypes as C
import math

import numpy as np
import pytest


@pytest.fixture(scope="module")
def lib():
    from paper_conf_middleware_hul24_b200 import build
    build.build()
    from paper_conf_middleware_hul24_b200 import menos as M
    return M.lib()


def brute_tiles(L):
    """(key block, 64-query block) pairs with at least one causal (query >= key) position: kb*128 <= qb*64 + 63."""
    n = 0
    for kb in range(math.ceil(L / 128)):
        for qb in range(math.ceil(L / 64)):
            if qb * 64 + 63 >= kb * 128:
                n += 1
    return n


def plan(lib, lens, H, Hkv, cap, max_chunks=4096):
    n = len(lens)
    arr = (C.c_int32 * n)(*lens)
    tiles = (C.c_int32 * n)()
    base = (C.c_int32 * (n * Hkv))()
    chunks = (C.c_int32 * (4 * max_chunks))()
    nc, nkv, nq = C.c_int32(), C.c_int32(), C.c_int32()
    rc = lib.menos_test_ds_plan(n, arr, H, Hkv, cap, tiles, base, chunks, max_chunks, C.byref(nc), C.byref(nkv),
                                C.byref(nq))
    assert rc == 0
    return (list(tiles), list(base), [tuple(chunks[4 * c:4 * c + 4]) for c in range(max(nc.value, 0))], nc.value,
            nkv.value, nq.value)


def test_tile_count_matches_brute_force(lib):
    lens = list(range(1, 300)) + [511, 512, 513, 700, 1024, 2047, 2048, 4096]
    got, *_ = plan(lib, lens, 1, 1, 1 << 40)
    assert got == [brute_tiles(L) for L in lens]


def test_memory_bound_covers_every_split():
    """menos_batch_memory charges H * T * (1 + max_seq_len / 16384) tiles: tiles(L) <= L + L^2 / 16384 for every L,
    so any split of T tokens into sequences of at most max_seq_len is covered."""
    for L in list(range(1, 2000)) + [4095, 4096, 8191, 8192, 16384]:
        assert brute_tiles(L) <= L + L * L / 16384.0, L


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_plan_invariants(lib, seed):
    rng = np.random.default_rng(seed)
    H, Hkv = [(8, 2), (4, 4), (6, 1)][seed]
    rep = H // Hkv
    lens = [int(x) for x in rng.integers(1, 900, size=int(rng.integers(1, 12)))]
    unit = [rep * brute_tiles(L) for L in lens for _ in range(Hkv)]
    for cap in (max(unit), max(unit) + 7, sum(unit), 10 ** 9):
        tiles, base, chunks, nc, nkv, nq = plan(lib, lens, H, Hkv, cap)
        assert nc >= 1
        # units in (sequence, kv head) order; a chunk starts where the base resets to 0
        starts = [i for i, b in enumerate(base) if b == 0]
        assert starts[0] == 0 and len(starts) == nc
        bounds = starts + [len(base)]
        for c in range(nc):
            off = 0
            for u in range(bounds[c], bounds[c + 1]):
                assert base[u] == off          # contiguous, disjoint tile ranges inside the chunk
                off += unit[u]
            assert off <= cap                  # the chunk fits the buffer
        # the chunks' work lists cover every item exactly once, in order
        assert nkv == sum(Hkv * math.ceil(L / 128) for L in lens)
        assert nq == sum(H * math.ceil(L / 128) for L in lens)
        assert sum(c[1] for c in chunks) == nkv and sum(c[3] for c in chunks) == nq
        assert all(chunks[c][0] == sum(x[1] for x in chunks[:c]) for c in range(nc))
        assert all(chunks[c][2] == sum(x[3] for x in chunks[:c]) for c in range(nc))
        if cap >= sum(unit):
            assert nc == 1
    # a unit larger than the budget: no plan (the recompute path)
    assert plan(lib, lens, H, Hkv, max(unit) - 1)[3] == -1


def plan_q(lib, lens, H, Hkv, cap, grid):
    n = len(lens)
    arr = (C.c_int32 * n)(*lens)
    n_items, nc = C.c_int32(), C.c_int32()
    assert lib.menos_test_ds_plan_q(n, arr, H, Hkv, cap, grid, None, 0, C.byref(n_items), None, 0, C.byref(nc)) == 0
    items = (C.c_int32 * (4 * max(1, n_items.value)))()
    chunks = (C.c_int32 * (4 * max(1, nc.value)))()
    assert lib.menos_test_ds_plan_q(n, arr, H, Hkv, cap, grid, items, n_items.value, C.byref(n_items), chunks,
                                    nc.value, C.byref(nc)) == 0
    it = np.array(items[:4 * n_items.value], dtype=np.int64).reshape(-1, 4)
    return it, [tuple(chunks[4 * c:4 * c + 4]) for c in range(nc.value)]


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_dq_runs_plan(lib, seed):
    """The dQ list for a persistent grid (r2ck): per chunk, every (sequence, query block, head) exactly once; CTA c
    (entries c, c + grid, ...) holds its real items before its padding; the items of a CTA come in runs of one
    (sequence, query block); the CTAs' costs (kv blocks per item = query block + 1) differ by at most one item's."""
    rng = np.random.default_rng(seed)
    H, Hkv = [(32, 32), (8, 2), (6, 1)][seed]
    rep = H // Hkv
    lens = [int(x) for x in rng.integers(1, 1100, size=int(rng.integers(1, 20)))]
    grid = [148, 7, 64][seed]
    unit = [rep * brute_tiles(L) for L in lens for _ in range(Hkv)]
    for cap in (max(unit) + 3, 10 ** 9):
        items, chunks = plan_q(lib, lens, H, Hkv, cap, grid)
        seen = set()
        for (_, _, q_off, q_n) in chunks:
            assert q_n % grid == 0
            ch = items[q_off:q_off + q_n]
            real = [tuple(x[:3]) for x in ch if x[0] >= 0]
            assert len(real) == len(set(real))
            seen |= set(real)
            costs = []
            for c in range(grid):
                col = ch[c::grid]
                flags = col[:, 0] >= 0
                k = int(flags.sum())
                assert flags[:k].all() and not flags[k:].any()      # padding only at the tail
                col = col[:k]
                runs = 1 + int(np.sum((col[1:, 0] != col[:-1, 0]) | (col[1:, 1] != col[:-1, 1]))) if k else 0
                fams = len({(int(a), int(b)) for a, b in col[:, :2]})
                assert runs == fams                                  # one run per (sequence, query block)
                costs.append(int(np.sum(col[:, 1] // 128 + 1)) if k else 0)
            mx = max(int(x[1]) // 128 + 1 for x in ch if x[0] >= 0)
            assert max(costs) - min(costs) <= 2 * mx
        want = {(s, q, h) for s, L in enumerate(lens) for q in range(0, L, 128) for h in range(H)}
        assert seen == want
