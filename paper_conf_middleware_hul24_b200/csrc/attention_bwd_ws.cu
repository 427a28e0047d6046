// Varlen causal flash-attention BACKWARD, persistent warp-specialized tcgen05 kernels, head_dim 128 or 64 (OPT-1.3B,
// NEXT-4: one 128-byte swizzle atom per head row; the RoPE pairs are (j, j + hd/2)).
// SURVEY.md §8(a) A11.  Same contract and math as attention_bwd_tc.cu (deterministic: no atomics; blocks never
// cross a sequence, so never a client; GQA; RoPE backward applied to dq / dk before the store),
// restructured so that the per-block fill / drain of the non-persistent kernels overlaps with useful work:
//   * one CTA per SM loops over work items (dK/dV: (sequence, kv head, 128-key block); dQ: (sequence, head,
//     128-query block)); the TMA producer loads the next item's resident operand (K|V, resp. Q|dO) as soon as the
//     current item's last S / dP MMA has consumed it, and the streamed operand ring runs across item boundaries;
//   * the MMA warp starts the next item's S / dP MMAs while the elementwise warps run the previous epilogue; only
//     the first accumulation into dK|dV (resp. dQ) waits for the epilogue to have read the TMEM accumulators;
//   * epilogue: each thread reads the accumulator columns j and j+64 of its row, applies the RoPE backward in
//     registers, stages bf16 rows (swizzled) in the freed P/dS buffers and the warps write them row-contiguously.
// Elementwise work: P = exp2(S c - lse) (a quarter on the FMA pipe), dS = P (dP - D) scale, bf16 packed into
// 128B-swizzled K-major tiles for the accumulation MMAs.
#include <algorithm>
#include "common.cuh"
#include "kernels.h"

namespace menos {

bool tma_map_2d(CUtensorMap* out, const void* ptr, uint64_t rows, uint64_t cols, uint64_t ld, uint32_t bc,
                uint32_t br);

namespace {

#ifndef MENOS_BWS_EW
#define MENOS_BWS_EW 8
#endif
// EW_WARPS elementwise warps: EW_WARPS / 4 per TMEM lane quadrant, each thread owning CPT of a block's 64 columns
constexpr int STAGES = 3, EW_WARPS = MENOS_BWS_EW, NTHREADS = 64 + 32 * EW_WARPS;
constexpr int NGRP = EW_WARPS / 4, CPT = 64 / NGRP;   // column groups per lane quadrant, columns per thread
static_assert(CPT == 16 || CPT == 32, "EW_WARPS must be 8 or 16");
constexpr float LOG2E_W = 1.4426950408889634f;
// MENOS_BWS_TMEM_P (default 1): the elementwise warps write P^T / dS^T (dK/dV kernel) and dS (dQ kernel) as packed
// bf16 into the TMEM columns of the S / dP tile they have just read, and the accumulation MMAs take them as the A
// operand from TMEM ("ts" form): no shared-memory round trip (16-32 KB of stores and MMA operand reads per block),
// no proxy fence, no buffer-free barrier.  0: the shared-memory path (tuning A/B only).
#ifndef MENOS_BWS_TMEM_P
#define MENOS_BWS_TMEM_P 1
#endif
// MENOS_BWS_ALT (default 1, needs MENOS_BWS_TMEM_P and 8 elementwise warps): the elementwise warps form two groups of
// four (one warp per TMEM lane quadrant) that take ALTERNATE blocks -- group = block parity = its S / dP buffer -- and a
// thread owns all 64 columns of its row in its group's blocks (two halves of 32).  The SM's TMEM read port moves
// 64 B / cycle, so a block's S + dP (64 KB) takes ~1000 cycles to read: with both groups on the same block every warp
// waits for the port, then every warp computes; alternating, one group's loads overlap the other group's arithmetic.
// The dK / dV epilogue stages dK, then dV, through one 32 KB buffer (frees 32 KB of shared memory for the lse / D ring).
#ifndef MENOS_BWS_ALT
#define MENOS_BWS_ALT MENOS_BWS_TMEM_P
#endif
#if MENOS_BWS_ALT
static_assert(MENOS_BWS_TMEM_P && EW_WARPS == 8, "MENOS_BWS_ALT needs the TMEM operand path and 8 elementwise warps");
#endif
// MENOS_BWS_DV_DIRECT (tuning variant, default 0; ALT path): the dK/dV epilogue sends dK out by TMA store and writes
// dV straight from registers instead of staging it after the dK store's read -- measured slower (cfg1 214 -> 230 us,
// cfg3 2.34 -> 2.46 ms per layer, r2bs): 16-byte stores of 32 rows per warp instruction cost more than the wait
#ifndef MENOS_BWS_DV_DIRECT
#define MENOS_BWS_DV_DIRECT 0
#endif
// TMEM column (relative to the tile) of K-chunk kk (16 queries / keys) of a packed operand: thread group g wrote its
// CPT columns' values into the first CPT / 2 of the CPT columns it had read (columns [CPT g, CPT g + CPT / 2))
__device__ __forceinline__ uint32_t packed_col(int kk) {
  return (uint32_t)((kk * 16 / CPT) * CPT + (kk * 16 % CPT) / 2);
}
template <int N>
__device__ __forceinline__ void tmem_st_half(uint32_t taddr, const uint32_t (&u)[N]) {
  if constexpr (N == 16) tmem_st16_nw(taddr, u); else tmem_st8_nw(taddr, u);
}
// pack CPT fp32 values into CPT / 2 bf16x2 words (even column in the low half)
__device__ __forceinline__ void pack_row(const float (&v)[CPT], uint32_t (&u)[CPT / 2]) {
#pragma unroll
  for (int i = 0; i < CPT / 2; ++i) u[i] = pack_bf16x2(v[2 * i], v[2 * i + 1]);
}

struct BwParams {
  const int* cu_seqlens;
  const int4* items;       // (seq, block start, head (dQ) / kv head (dK/dV), -)
  int n_items;
  const float* lse;        // [H, T] natural log
  const float* D;          // [H, T]
  bf16* dqkv; int ld_dqkv;
  const float2* rope_cs;   // [max_pos][hd/2] (cos, sin)
  const int* pos_shift;    // [n_seqs] prefix rows before each sequence (extended batch) or nullptr
  int T, H, Hkv;
  float scale;
  // dS^T tiles for the dQ pass (attn_bwd_dq_ds_kernel) or nullptr: the dK/dV kernel stores every block's bf16
  // dS^T [128 keys][64 queries] at tile ds_tile(...) of `ds`; ds_base[seq * Hkv + kv head] = first tile of the unit
  bf16* ds;
  const int* ds_base;
};

// dS^T tiles of one sequence of length L and one head: key block kb (128 keys) pairs with the 64-query blocks
// qb = 2 kb .. nqb - 1 (causal); tiles are numbered key block by key block
__host__ __device__ __forceinline__ int ds_tiles_of(int L) {
  const int nqb = (L + 63) / 64, nkb = (L + 127) / 128;
  return nkb * nqb - nkb * (nkb - 1);
}
__device__ __forceinline__ int ds_tile_in_head(int L, int kb, int qb) {
  const int nqb = (L + 63) / 64;
  return kb * nqb - kb * (kb - 1) + (qb - 2 * kb);
}

__device__ __forceinline__ void wait_bar(uint64_t* bar, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile("{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  }
}
// 1-D bulk copy global -> shared (16-byte aligned source and destination, size % 16 == 0), completion on `bar`
__device__ __forceinline__ void bulk_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void ew_sync() { asm volatile("bar.sync 1, %0;" ::"n"(32 * EW_WARPS) : "memory"); }

// CPT consecutive TMEM columns (32x32b.x16 / .x32), no wait
template <int N>
__device__ __forceinline__ void tmem_ldc_nw(uint32_t taddr, uint32_t (&r)[N]) {
  if constexpr (N == 32) {
    tmem_ld32_nw(taddr, r);
  } else if constexpr (N == 8) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                 : "r"(taddr));
  } else {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
  }
}

// columns [CPT g, CPT g + CPT) (bf16) of one row of a [rows][64] SWIZZLE_128B K-major tile
__device__ __forceinline__ void st_half_row(uint8_t* tile, int row, int g, const float (&v)[CPT]) {
  uint8_t* prow = tile + row * 128;
#pragma unroll
  for (int c = 0; c < CPT / 8; ++c) {
    const int c8 = (CPT / 8) * g + c;
    uint4 u = make_uint4(pack_bf16x2(v[8 * c + 0], v[8 * c + 1]), pack_bf16x2(v[8 * c + 2], v[8 * c + 3]),
                         pack_bf16x2(v[8 * c + 4], v[8 * c + 5]), pack_bf16x2(v[8 * c + 6], v[8 * c + 7]));
    *reinterpret_cast<uint4*>(prow + ((c8 ^ (row & 7)) << 4)) = u;
  }
}

// Single-round epilogue: every elementwise thread converts its TMEM row (columns [32g, 32g+32) and [64+32g, ..),
// i.e. the RoPE pairs (j, j+64)) to bf16 in registers -- RoPE backward applied there, with the (cos, sin) pairs
// loaded BEFORE the wait for the accumulator (rope_cs_load) so the table's L2 latency hides behind it -- and writes it
// into a bf16 staging matrix in the TMA SWIZZLE_128B layout: HD / 64 atoms of [128 rows][128 B], 16-byte chunk k
// of row rr at atom (k / 8), rr * 128 + (((k % 8) ^ (rr & 7)) << 4).  The x half (columns < HD/2) lands in the first
// half of the atoms, the y half in the second.  A full 128-row block leaves by TMA store (one thread, async: the
// warps go on with the next item); a sequence's ragged last block by row-masked 16-byte stores (stage16_store).
// Same fp32 ops in the same order as before: the bf16 result is bitwise identical.
template <int HD>
struct RopeCS { float4 v[HD / (4 * NGRP)]; };   // (c_2i, s_2i, c_2i+1, s_2i+1) for the thread's HD / (2 NGRP) pairs
template <int HD>
__device__ __forceinline__ void rope_cs_load(RopeCS<HD>& c, const float2* cs, int pos, int g, bool rope) {
  if (!rope) return;
  const float4* c4 = reinterpret_cast<const float4*>(cs + (size_t)pos * (HD / 2) + (HD / (2 * NGRP)) * g);
#pragma unroll
  for (int i = 0; i < HD / (4 * NGRP); ++i) c.v[i] = __ldg(c4 + i);
}
// the thread's accumulator row chunk -> bf16 (RoPE backward applied when rope): x half (columns < HD/2) in ux, y in uy
template <int HD>
struct RowPack { uint4 x[HD / (16 * NGRP)], y[HD / (16 * NGRP)]; };
template <int HD>
__device__ __forceinline__ void acc_row_pack(uint32_t tacc, int g, const RopeCS<HD>& cs, bool rope, RowPack<HD>& o) {
  constexpr int EC = HD / (2 * NGRP);   // columns per group per half
  uint32_t a[EC], b[EC];
  tmem_ldc_nw(tacc + EC * g, a);
  tmem_ldc_nw(tacc + HD / 2 + EC * g, b);
  tmem_wait_ld();
  float x[EC], y[EC];
#pragma unroll
  for (int i = 0; i < EC; ++i) { x[i] = __uint_as_float(a[i]); y[i] = __uint_as_float(b[i]); }
  if (rope) {   // dx_j = dy_j c + dy_{j+hd/2} s,  dx_{j+hd/2} = dy_{j+hd/2} c - dy_j s
#pragma unroll
    for (int i = 0; i < EC / 2; ++i) {
      const float4 e = cs.v[i];
      const float x0 = x[2 * i] * e.x + y[2 * i] * e.y, y0 = y[2 * i] * e.x - x[2 * i] * e.y;
      const float x1 = x[2 * i + 1] * e.z + y[2 * i + 1] * e.w, y1 = y[2 * i + 1] * e.z - x[2 * i + 1] * e.w;
      x[2 * i] = x0; y[2 * i] = y0; x[2 * i + 1] = x1; y[2 * i + 1] = y1;
    }
  }
#pragma unroll
  for (int c = 0; c < EC / 8; ++c) {
    o.x[c] = make_uint4(pack_bf16x2(x[8 * c], x[8 * c + 1]), pack_bf16x2(x[8 * c + 2], x[8 * c + 3]),
                        pack_bf16x2(x[8 * c + 4], x[8 * c + 5]), pack_bf16x2(x[8 * c + 6], x[8 * c + 7]));
    o.y[c] = make_uint4(pack_bf16x2(y[8 * c], y[8 * c + 1]), pack_bf16x2(y[8 * c + 2], y[8 * c + 3]),
                        pack_bf16x2(y[8 * c + 4], y[8 * c + 5]), pack_bf16x2(y[8 * c + 6], y[8 * c + 7]));
  }
}
template <int HD>
__device__ __forceinline__ void stage_row(uint8_t* stg, int rr, int g, const RowPack<HD>& o) {
  constexpr int EC = HD / (2 * NGRP);
  uint8_t* row = stg + rr * 128;
#pragma unroll
  for (int c = 0; c < EC / 8; ++c) {
    const int kx = (EC / 8) * g + c, ky = HD / 16 + kx;   // 16-byte chunk indices of the row
    *reinterpret_cast<uint4*>(row + (kx >> 3) * 16384 + (((kx & 7) ^ (rr & 7)) << 4)) = o.x[c];
    *reinterpret_cast<uint4*>(row + (ky >> 3) * 16384 + (((ky & 7) ^ (rr & 7)) << 4)) = o.y[c];
  }
}
template <int HD>
__device__ __forceinline__ void acc_row_to_bf16(uint32_t tacc, uint8_t* stg, int rr, int g, const RopeCS<HD>& cs,
                                                bool rope) {
  RowPack<HD> o;
  acc_row_pack<HD>(tacc, g, cs, rope, o);
  stage_row<HD>(stg, rr, g, o);
}
// n_tiles staged bf16 matrices (128 rows each, 128 * 2 HD bytes apart, atom layout above) -> rows [0, n_valid) of
// dst[t] (row stride ld): HD / 8 lanes per row, 256 / HD rows per store instruction
template <int HD>
__device__ __forceinline__ void stage16_store(const uint8_t* stg, int n_tiles, int w8, int lane, int n_valid,
                                              bf16* dst0, bf16* dst1, int ld) {
  constexpr int NCH = HD / 8, RPI = 32 / NCH, MATB = 128 * HD * 2;
  const int k = lane % NCH;
#pragma unroll 4
  for (int i = 0; i < 128 * n_tiles / (RPI * EW_WARPS); ++i) {
    const int R = i * (RPI * EW_WARPS) + w8 * RPI + lane / NCH, t = R >> 7, rr = R & 127;
    if (rr >= n_valid) continue;
    const uint4 v = *reinterpret_cast<const uint4*>(stg + t * MATB + (k >> 3) * 16384 + rr * 128 +
                                                    (((k & 7) ^ (rr & 7)) << 4));
    *reinterpret_cast<uint4*>((t ? dst1 : dst0) + (size_t)rr * ld + k * 8) = v;
  }
}
// one staged matrix (HD / 64 atoms) -> 128 rows of dqkv from (row, col) by TMA store; called by one thread after the
// staging writes, fence.proxy.async and a barrier
template <int HD>
__device__ __forceinline__ void stage_tma_store(const CUtensorMap* m, const uint8_t* stg, int row, int col) {
#pragma unroll
  for (int a = 0; a < HD / 64; ++a) tma_store_2d(m, stg + a * 16384, col + 64 * a, row);
}

// Work-item geometry, pipelined so that no role stalls on global loads at an item boundary: the items entry of
// item + 2G is loaded at the top of item, the sequence's cu_seqlens / pos_shift entries of item + G (whose items entry
// arrived one item earlier) too, and both are consumed one item later.
struct ItemPipe {
  int4 raw;         // items[i + 2G] (x = -1: past the end)
  int4 cur;         // items[i + G]
  int c0, c1, sh;   // cu_seqlens[cur.x], cu_seqlens[cur.x + 1], pos_shift[cur.x]
};
__device__ __forceinline__ int4 item_at(const int4* items, int n, int i) {
  return i < n ? items[i] : make_int4(-1, 0, 0, 0);
}
__device__ __forceinline__ void ip_fetch(ItemPipe& q, const int* cu, const int* ps) {
  q.c0 = 0; q.c1 = 0; q.sh = 0;
  if (q.cur.x >= 0) { q.c0 = cu[q.cur.x]; q.c1 = cu[q.cur.x + 1]; q.sh = ps ? ps[q.cur.x] : 0; }
}
struct Geo { int base, L, blk0, head, n, sh, seq; };   // sh: RoPE position shift of the sequence (prefix rows)

// -DMENOS_BWS_PROF: per-phase clock64 accounting (dK/dV kernel: one elementwise thread and the MMA lane)
#ifdef MENOS_BWS_PROF
__device__ unsigned long long g_bws_prof[16];
#define BP_DECL long long bp_t = clock64(); unsigned long long bpr_[16] = {0};
#define BP(k) do { const long long t_ = clock64(); bpr_[k] += t_ - bp_t; bp_t = t_; } while (0)
#define BP_FLUSH(cond) do { if (cond) for (int k_ = 0; k_ < 16; ++k_) if (bpr_[k_]) atomicAdd(&g_bws_prof[k_], bpr_[k_]); } while (0)
#else
#define BP_DECL
#define BP(k) do {} while (0)
#define BP_FLUSH(cond) do {} while (0)
#endif

// P = exp2(S c - lse) (every fourth on the FMA pipe), dS = P (dP - D) scale for the thread's CPT columns; MASK: the
// causal / sequence-end mask (columns outside [cmin, cmax) are 0) -- interior blocks take the unmasked instance
template <bool MASK>
__device__ __forceinline__ void pds_math(const uint32_t (&su)[CPT], const uint32_t (&du)[CPT], const float* lse_s,
                                         const float* d_s, float sl2, float scale, int cmin, int cmax,
                                         float (&pv)[CPT], float (&dsv)[CPT]) {
#pragma unroll
  for (int c4 = 0; c4 < CPT; c4 += 4) {
    const float4 lz = *reinterpret_cast<const float4*>(lse_s + c4);
    const float4 dz = *reinterpret_cast<const float4*>(d_s + c4);
    const float lzv[4] = {lz.x, lz.y, lz.z, lz.w}, dzv[4] = {dz.x, dz.y, dz.z, dz.w};
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int c = c4 + u;
      const float x = fmaf(__uint_as_float(su[c]), sl2, -lzv[u]);
      const float e = u == 3 ? poly_exp2(x) : fast_exp2(x);
      const float ds = e * fmaf(__uint_as_float(du[c]), scale, -dzv[u]);
      if (MASK) {
        const bool ok = c >= cmin && c < cmax;
        pv[c] = ok ? e : 0.f;
        dsv[c] = ok ? ds : 0.f;
      } else {
        pv[c] = e;
        dsv[c] = ds;
      }
    }
  }
}

// ======================================================================================= dK / dV
constexpr int KV_ROWS = 128, QB = 64;
constexpr uint32_t LD_BYTES = (QB + 4) * 4;    // a block's lse (or D) row from the aligned start: 272 B
constexpr int PT_TILE = KV_ROWS * QB * 2;      // 16 KB (1 atom [128][64])
constexpr int KVA = KV_ROWS * 128, QBA = QB * 128;   // one SW128 atom (64 columns) of a K / V tile, of a Q / dO tile
template <int HD> struct DkdvGeo {
  static constexpr int KV_TILE = KV_ROWS * HD * 2;   // HD 128: 32 KB (2 atoms [128][64]); 64: 16 KB
  static constexpr int QB_TILE = QB * HD * 2;        // 16 KB (2 atoms [64][64]); 8 KB
  static constexpr int SMEM = 2 * KV_TILE + 2 * STAGES * QB_TILE + (MENOS_BWS_ALT ? 2 : 4) * PT_TILE + 1024;
};

template <int HD>
__global__ void __launch_bounds__(NTHREADS, 1)
attn_bwd_dkdv_ws_kernel(const __grid_constant__ CUtensorMap tmQKV128, const __grid_constant__ CUtensorMap tmQKV64,
                        const __grid_constant__ CUtensorMap tmDO64, const __grid_constant__ CUtensorMap tmOut,
                        const __grid_constant__ CUtensorMap tmDS, const BwParams p) {
  constexpr int KV_TILE = DkdvGeo<HD>::KV_TILE, QB_TILE = DkdvGeo<HD>::QB_TILE;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* const sK = smem;
  uint8_t* const sV = sK + KV_TILE;
  uint8_t* const sQ0 = sV + KV_TILE;                  // Q stages
  uint8_t* const sO0 = sQ0 + STAGES * QB_TILE;        // dO stages
  uint8_t* const sP0 = sO0 + STAGES * QB_TILE;        // P^T  (2 buffers) -- dK staging in the epilogue
  uint8_t* const sS0 = sP0 + 2 * PT_TILE;             // dS^T (2 buffers) -- dV staging in the epilogue
  __shared__ __align__(8) uint64_t kv_full, kv_empty, full[STAGES], empty[STAGES], s_full[2], ew_done[2], pd_free[2];
  __shared__ __align__(8) uint64_t acc_full, acc_free;
  __shared__ uint32_t tmem_sh;
#if MENOS_BWS_ALT
  // raw lse | D of each Q / dO stage's 64 queries, brought by the TMA warp with the stage (two 272-byte bulk copies
  // from the 16-byte-aligned start at or below the first query; `off` = the first query's index inside), and the
  // group's scaled copy (lse in the log2 domain, D pre-scaled), a ring of 2 blocks
  __shared__ __align__(16) float s_ldr[STAGES][2][QB + 4];
  __shared__ __align__(16) float s_ld[2][2][2 * QB];
#else
  // lse (log2 domain) | D (pre-scaled) of a block's 64 queries, ring of 3 blocks filled by cp.async two blocks ahead
  __shared__ __align__(16) float s_ld[3][2 * QB];
#endif

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int rep = p.H / p.Hkv;
  if (threadIdx.x == 0) {
    tma_prefetch(&tmQKV128); tma_prefetch(&tmQKV64); tma_prefetch(&tmDO64);
    mbar_init(&kv_full, 1); mbar_init(&kv_empty, 1);
    for (int i = 0; i < STAGES; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&s_full[i], 1); mbar_init(&ew_done[i], MENOS_BWS_ALT ? EW_WARPS / 2 : EW_WARPS); mbar_init(&pd_free[i], 1);
    }
    mbar_init(&acc_full, 1); mbar_init(&acc_free, EW_WARPS);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  const uint32_t tdV = tmem + 256, tdK = tmem + 384;   // S^T buffers at 0/64, dP^T at 128/192

  auto ip_init = [&](ItemPipe& q) {
    q.cur = item_at(p.items, p.n_items, blockIdx.x);
    ip_fetch(q, p.cu_seqlens, p.pos_shift);
    q.raw = item_at(p.items, p.n_items, blockIdx.x + gridDim.x);
  };
  auto ip_advance = [&](ItemPipe& q, int item) {   // at the top of `item`: q moves on to item + G
    q.cur = q.raw;
    ip_fetch(q, p.cu_seqlens, p.pos_shift);
    q.raw = item_at(p.items, p.n_items, item + 2 * gridDim.x);
  };
  auto decode = [&](const ItemPipe& q) {
    Geo g{q.c0, q.c1 - q.c0, q.cur.y, q.cur.z, 0, q.sh, q.cur.x};
    g.n = rep * ((g.L - g.blk0 + QB - 1) / QB);      // (head of the group, 64-query block) pairs; 0 past the end
    return g;
  };

  if (warp == 0) {
    // ------------------------------------------------ TMA producer
    if (elect_one()) {
      ItemPipe ip;
      ip_init(ip);
      int it = 0, gb = 0;
      for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
        const Geo G = decode(ip);
        ip_advance(ip, item);
        const int k0 = G.blk0, hk = G.head, nqb = (G.L - k0 + QB - 1) / QB;
        const int kcol = (p.H + hk) * HD, vcol = (p.H + p.Hkv + hk) * HD;
        wait_bar(&kv_empty, (it & 1) ^ 1);
        mbar_expect_tx(&kv_full, 2 * KV_TILE);
#pragma unroll
        for (int a = 0; a < HD / 64; ++a) {
          tma_load_2d(sK + a * KVA, &tmQKV128, &kv_full, kcol + 64 * a, G.base + k0);
          tma_load_2d(sV + a * KVA, &tmQKV128, &kv_full, vcol + 64 * a, G.base + k0);
        }
        for (int j = 0; j < G.n; ++j, ++gb) {
          const int st = gb % STAGES;
          const int h = hk * rep + j / nqb, q0 = k0 + (j % nqb) * QB;
          wait_bar(&empty[st], ((gb / STAGES) & 1) ^ 1);
#if MENOS_BWS_ALT
          mbar_expect_tx(&full[st], 2 * QB_TILE + 2 * LD_BYTES);
          {
            const size_t i0 = ((size_t)h * p.T + G.base + q0) & ~(size_t)3;   // 16-byte aligned start
            bulk_load_1d(&s_ldr[st][0][0], p.lse + i0, LD_BYTES, &full[st]);
            bulk_load_1d(&s_ldr[st][1][0], p.D + i0, LD_BYTES, &full[st]);
          }
#else
          mbar_expect_tx(&full[st], 2 * QB_TILE);
#endif
          uint8_t* q = sQ0 + st * QB_TILE;
          uint8_t* o = sO0 + st * QB_TILE;
#pragma unroll
          for (int a = 0; a < HD / 64; ++a) {
            tma_load_2d(q + a * QBA, &tmQKV64, &full[st], h * HD + 64 * a, G.base + q0);
            tma_load_2d(o + a * QBA, &tmDO64, &full[st], h * HD + 64 * a, G.base + q0);
          }
        }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer
    constexpr uint32_t ID_S = umma_idesc_bf16(128, QB, 0);     // [128 kv] x [64 q], K = hd
    constexpr uint32_t ID_ACC = umma_idesc_bf16(128, HD, 1);   // [128 kv] x [hd], K = 64 q, B MN-major
    ItemPipe ip;
    ip_init(ip);
    BP_DECL
    int it = 0, gb = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
      const Geo G = decode(ip);
      ip_advance(ip, item);
      auto issue_acc = [&](int gp, int jp) {  // dV += P^T dO ; dK += dS^T Q   for global block gp (item block jp)
        const int bp = gp & 1, sp = gp % STAGES;
        BP(10);
        wait_bar(&ew_done[bp], (gp >> 1) & 1);
        BP(11);
        if (jp == 0) wait_bar(&acc_free, (it & 1) ^ 1);   // previous item's epilogue has read dV / dK
        BP(12);
        tc_fence_after();
        __syncwarp();
        if (elect_one()) {
          const uint32_t ob = smem_u32(sO0 + sp * QB_TILE), qb = smem_u32(sQ0 + sp * QB_TILE);
#if MENOS_BWS_TMEM_P
          const uint64_t od0 = umma_desc_sw128(ob, 8192, 1024), qd0 = umma_desc_sw128(qb, 8192, 1024);
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {   // A = P^T / dS^T packed in the S^T / dP^T tiles of buffer bp
            const uint32_t acc = (jp > 0 || kk > 0) ? 1u : 0u;   // B: base descriptor + constant K-step offset
            tc_mma_bf16_ts(tdV, tmem + 64 * bp + packed_col(kk), od0 + (uint64_t)((kk * 2048) >> 4), ID_ACC, acc);
            tc_mma_bf16_ts(tdK, tmem + 128 + 64 * bp + packed_col(kk), qd0 + (uint64_t)((kk * 2048) >> 4), ID_ACC, acc);
          }
          tc_commit(&empty[sp]);     // Q/dO stage free
#else
          const uint32_t pa = smem_u32(sP0 + bp * PT_TILE), sa = smem_u32(sS0 + bp * PT_TILE);
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {
            const uint32_t acc = (jp > 0 || kk > 0) ? 1u : 0u;
            tc_mma_bf16(tdV, umma_desc_sw128(pa + kk * 32, 16, 1024), umma_desc_sw128(ob + kk * 2048, 8192, 1024), ID_ACC, acc);
            tc_mma_bf16(tdK, umma_desc_sw128(sa + kk * 32, 16, 1024), umma_desc_sw128(qb + kk * 2048, 8192, 1024), ID_ACC, acc);
          }
          tc_commit(&empty[sp]);     // Q/dO stage free
          tc_commit(&pd_free[bp]);   // P^T/dS^T buffer free
#endif
        }
        __syncwarp();
        BP(13);
      };
      BP(10);
      wait_bar(&kv_full, it & 1);
      BP(15);
      tc_fence_after();
      for (int j = 0; j < G.n; ++j, ++gb) {
        const int b = gb & 1, st = gb % STAGES;
        BP(10);
        wait_bar(&full[st], (gb / STAGES) & 1);
        BP(14);
        tc_fence_after();
        __syncwarp();
        if (elect_one()) {
          // one base descriptor per operand, K steps as constant 16-byte-unit offsets (no carry: smem < 256 KB)
          const uint64_t kd0 = umma_desc_sw128(smem_u32(sK), 16, 1024), vd0 = umma_desc_sw128(smem_u32(sV), 16, 1024);
          const uint64_t qd0 = umma_desc_sw128(smem_u32(sQ0 + st * QB_TILE), 16, 1024);
          const uint64_t od0 = umma_desc_sw128(smem_u32(sO0 + st * QB_TILE), 16, 1024);
#pragma unroll
          for (int kk = 0; kk < HD / 16; ++kk) {
            const uint64_t offa = (uint64_t)(((kk >> 2) * KVA + (kk & 3) * 32) >> 4);
            const uint64_t offb = (uint64_t)(((kk >> 2) * QBA + (kk & 3) * 32) >> 4);
            tc_mma_bf16(tmem + 64 * b, kd0 + offa, qd0 + offb, ID_S, kk > 0);
            tc_mma_bf16(tmem + 128 + 64 * b, vd0 + offa, od0 + offb, ID_S, kk > 0);
          }
          tc_commit(&s_full[b]);
          if (j == G.n - 1) tc_commit(&kv_empty);   // K / V free once the item's last S^T / dP^T completes
        }
        __syncwarp();
        if (j > 0) issue_acc(gb - 1, j - 1);
      }
      if (G.n > 0) issue_acc(gb - 1, G.n - 1);
      __syncwarp();
      if (elect_one()) tc_commit(&acc_full);
      __syncwarp();
    }
    BP(10);
    BP_FLUSH(blockIdx.x < 8 && lane == 0);
  } else {
#if MENOS_BWS_ALT
    // ------------------------------------------------ elementwise warps: group gr = w8 / 4 takes the blocks of parity
    //                                                  gr; thread = key row = TMEM lane, all 64 query columns
    const int w4 = warp & 3, w8 = warp - 2, gr = w8 >> 2, t = threadIdx.x - 64, tt = t & 127;
    const int r = w4 * 32 + lane;           // key row within the block
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_W;
    ItemPipe ip;
    ip_init(ip);
    BP_DECL
    auto gsync = [&]() {   // the group's four warps
      if (gr == 0) asm volatile("bar.sync 2, 128;" ::: "memory"); else asm volatile("bar.sync 3, 128;" ::: "memory");
    };
    bool tma_pending = false;   // this thread (t == 0) has TMA stores reading the staging buffer
    int it = 0, gb = 0, kb = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
      const Geo G = decode(ip);
      ip_advance(ip, item);
      const int k0 = G.blk0, L = G.L, base = G.base, nqb = (L - k0 + QB - 1) / QB;
      const int kpos = k0 + r;
      // dS^T tiles of this unit (sequence, kv head) for the dQ pass
      const int ds_unit = (p.ds && G.n > 0) ? __ldg(p.ds_base + G.seq * p.Hkv + G.head) : 0;
      for (int j = 0; j < G.n; ++j, ++gb) {
        if ((gb & 1) != gr) continue;
        const int q0 = k0 + (j % nqb) * QB, sl = kb & 1;
        // dS^T of this block -> the group's staging tile (128-byte swizzled rows) -> one TMA store (dS-stored variant)
        // (sP0: idle between item epilogues; group gr stages in its half)
        uint8_t* const ds_stg = sP0 + gr * PT_TILE + r * 128;
        const bool ds_lead = p.ds != nullptr && w4 == 0 && lane == 0;
        {   // this block's lse / D arrived with its Q / dO stage (the MMA warp already waited for it): scale one each
          const int st = gb % STAGES, h = G.head * rep + j / nqb;
          wait_bar(&full[st], (gb / STAGES) & 1);
          const int off = (int)(((size_t)h * p.T + base + q0) & 3);
          const float v = s_ldr[st][tt >= QB][off + (tt & (QB - 1))];
          s_ld[gr][sl][tt] = v * (tt < QB ? LOG2E_W : p.scale);   // lse to the log2 domain, D pre-scaled
        }
        if (p.ds && w4 == 0 && lane == 0) bulk_wait_read0();   // the group's staging tile is free again
        BP(9);
        gsync();
        BP(1);
        BP(0);
        wait_bar(&s_full[gr], (gb >> 1) & 1);
        BP(2);
        tc_fence_after();
        __syncwarp();
#pragma unroll 1
        for (int hf = 0; hf < 2; ++hf) {   // query columns [32 hf, 32 hf + 32)
          uint32_t su[CPT], du[CPT];
          tmem_ldc_nw(tmem + 64 * gr + 32 * hf + lane_off, su);
          tmem_ldc_nw(tmem + 128 + 64 * gr + 32 * hf + lane_off, du);
          tmem_wait_ld();
          const int cmin = kpos - q0 - 32 * hf;   // P = 0 for queries before the key (causal) ...
          const int cmax = L - q0 - 32 * hf;      // ... and past the end of the sequence
          float pv[CPT], dsv[CPT];
          if (cmin <= 0 && cmax >= CPT)
            pds_math<false>(su, du, &s_ld[gr][sl][32 * hf], &s_ld[gr][sl][QB + 32 * hf], sl2, p.scale, cmin, cmax, pv,
                            dsv);
          else
            pds_math<true>(su, du, &s_ld[gr][sl][32 * hf], &s_ld[gr][sl][QB + 32 * hf], sl2, p.scale, cmin, cmax, pv,
                           dsv);
          uint32_t up[CPT / 2], ud[CPT / 2];
          pack_row(pv, up);
          pack_row(dsv, ud);
          tmem_st_half(tmem + 64 * gr + 32 * hf + lane_off, up);
          tmem_st_half(tmem + 128 + 64 * gr + 32 * hf + lane_off, ud);
          if (p.ds) {   // the same bf16 dS^T row (queries 32 hf .. 32 hf + 31): four 16-byte chunks of the staged row
#pragma unroll
            for (int c = 0; c < CPT / 8; ++c) {
              const int c8 = (CPT / 8) * hf + c;
              *reinterpret_cast<uint4*>(ds_stg + ((c8 ^ (r & 7)) << 4)) =
                  make_uint4(ud[4 * c], ud[4 * c + 1], ud[4 * c + 2], ud[4 * c + 3]);
            }
          }
        }
        BP(3);
        tmem_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&ew_done[gr]);
        if (p.ds) {   // the staged dS^T tile leaves by TMA (async; the leader waits for its read before the next fill)
          fence_proxy_async();
          gsync();
          if (ds_lead) {
            const int tile = ds_unit + (j / nqb) * ds_tiles_of(L) + ds_tile_in_head(L, k0 / KV_ROWS, q0 / QB);
            tma_store_2d(&tmDS, sP0 + gr * PT_TILE, 0, tile * KV_ROWS);
            bulk_commit();
          }
        }
        ++kb;
        BP(5);
      }
      // ------------------------------------------------ epilogue: dK (RoPE bwd), then dV, through one 32 KB staging
      const int nv = min(KV_ROWS, L - k0);
      const bool rope = p.rope_cs != nullptr && r < nv, full = nv == KV_ROWS;
      RopeCS<HD> csk;
      rope_cs_load<HD>(csk, p.rope_cs, max(0, k0 + r - G.sh), gr, rope);   // in flight during the wait below
      BP(0);
      wait_bar(&acc_full, it & 1);
      BP(6);
      tc_fence_after();
      if (t == 0 && tma_pending) bulk_wait_read0();   // the previous item's dV store has read the staging
      if (p.ds && w4 == 0 && lane == 0) bulk_wait_read0();   // ... and the groups' dS^T stores (same buffer)
      tma_pending = false;
      ew_sync();
      bf16* dst = p.dqkv + (size_t)(base + k0) * p.ld_dqkv;
      acc_row_to_bf16<HD>(tdK + lane_off, sP0, r, gr, csk, rope);
      RowPack<HD> vpk;
      acc_row_pack<HD>(tdV + lane_off, gr, csk, false, vpk);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&acc_free);   // the next item's dK / dV accumulation may start
      BP(7);
      if (full) fence_proxy_async();
      ew_sync();
#if MENOS_BWS_DV_DIRECT
      if (full) {   // dK leaves by TMA store; dV straight from registers (no second staging round, no wait between)
        if (t == 0) {
          stage_tma_store<HD>(&tmOut, sP0, base + k0, (p.H + G.head) * HD);
          bulk_commit();
        }
        tma_pending = true;
        constexpr int EC = HD / (2 * NGRP);
        bf16* vrow = dst + (size_t)r * p.ld_dqkv + (p.H + p.Hkv + G.head) * HD + EC * gr;
#pragma unroll
        for (int c = 0; c < EC / 8; ++c) {
          *reinterpret_cast<uint4*>(vrow + 8 * c) = vpk.x[c];
          *reinterpret_cast<uint4*>(vrow + HD / 2 + 8 * c) = vpk.y[c];
        }
      } else
#endif
      {
      if (full) {
        if (t == 0) {
          stage_tma_store<HD>(&tmOut, sP0, base + k0, (p.H + G.head) * HD);
          bulk_commit();
          bulk_wait_read0();
        }
      } else {
        stage16_store<HD>(sP0, 1, w8, lane, nv, dst + (p.H + G.head) * HD, dst, p.ld_dqkv);
      }
      ew_sync();
      stage_row<HD>(sP0, r, gr, vpk);
      if (full) {
        fence_proxy_async();
        ew_sync();
        if (t == 0) {
          stage_tma_store<HD>(&tmOut, sP0, base + k0, (p.H + p.Hkv + G.head) * HD);
          bulk_commit();
        }
        tma_pending = true;
      } else {
        ew_sync();
        stage16_store<HD>(sP0, 1, w8, lane, nv, dst + (p.H + p.Hkv + G.head) * HD, dst, p.ld_dqkv);
        ew_sync();
      }
      }
      if (p.ds) {   // the next item's dS^T staging reuses sP0: the dK / dV store must have read it
        if (t == 0 && tma_pending) { bulk_wait_read0(); tma_pending = false; }
        ew_sync();
      }
      BP(8);
    }
#else
    // ------------------------------------------------ elementwise warps (thread = key row = TMEM lane;
    //                                                  warp group g owns query columns [CPT g, CPT g + CPT))
    const int w4 = warp & 3, w8 = warp - 2, g = w8 >> 2, t = threadIdx.x - 64;
    const int r = w4 * 32 + lane;           // key row within the block
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_W;
    ItemPipe ip;
    ip_init(ip);
    BP_DECL
    // the stager threads' (t < 128) lse / D values arrive by 4-byte cp.async two blocks ahead of their use (ring
    // s_ld[gb % 3]; issued after block gb's barrier, when every thread is done with block gb - 1's slot), so their
    // latency (L2 or HBM) hides behind two blocks of work without a register dependency; a value whose block lies
    // beyond the next item (items of one block) is issued one block ahead instead
    auto issue = [&](int slot, const Geo& G, int jj) {
      const float* src = p.lse;
      int sz = 0;
      if (jj < G.n) {
        const int nqb = (G.L - G.blk0 + QB - 1) / QB;
        const int h = G.head * rep + jj / nqb, qpos = G.blk0 + (jj % nqb) * QB + (t & (QB - 1));
        if (qpos < G.L) { src = (t < QB ? p.lse : p.D) + (size_t)h * p.T + G.base + qpos; sz = 4; }
      }
      cp_async4(smem_u32(&s_ld[slot][t]), src, sz);
    };
    bool nxt_issued = false, cur_wait0 = true;
    bool tma_pending = false;   // this thread (t == 0) has TMA stores reading the staging buffers
    int it = 0, gb = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
      const Geo G = decode(ip);
      ip_advance(ip, item);
      const int k0 = G.blk0, L = G.L, base = G.base, nqb = (L - k0 + QB - 1) / QB;
      const int kpos = k0 + r;
      for (int j = 0; j < G.n; ++j, ++gb) {
        const int b = gb & 1, sl = gb % 3;
        const int q0 = k0 + (j % nqb) * QB;
        if (t < 2 * QB) {   // this block's value: wait for its copy, scale in place
          if (gb == 0) { issue(0, G, 0); cp_async_commit(); }
          if (cur_wait0) cp_async_wait<0>(); else cp_async_wait<1>();
          s_ld[sl][t] *= t < QB ? LOG2E_W : p.scale;   // lse to the log2 domain, D pre-scaled
          BP(9);
        }
        BP(0);
        ew_sync();
        BP(1);
        if (t < 2 * QB) {   // copies of block gb + 1 (if not issued a block ago) and gb + 2 (if its item is known)
          const Geo N = j + 2 >= G.n ? decode(ip) : G;
          const bool late = !nxt_issued;
          if (late) {
            if (j + 1 < G.n) issue((gb + 1) % 3, G, j + 1); else issue((gb + 1) % 3, N, j + 1 - G.n);
          }
          nxt_issued = true;
          if (j + 2 < G.n) issue((gb + 2) % 3, G, j + 2);
          else if (j + 2 - G.n < N.n) issue((gb + 2) % 3, N, j + 2 - G.n);
          else nxt_issued = false;
          cp_async_commit();
          cur_wait0 = late;
        }
        wait_bar(&s_full[b], (gb >> 1) & 1);
        BP(2);
        tc_fence_after();
        __syncwarp();
        uint32_t su[CPT], du[CPT];
        tmem_ldc_nw(tmem + 64 * b + CPT * g + lane_off, su);
        tmem_ldc_nw(tmem + 128 + 64 * b + CPT * g + lane_off, du);
        tmem_wait_ld();
        const int cmin = kpos - q0 - CPT * g;   // P = 0 for queries before the key (causal) ...
        const int cmax = L - q0 - CPT * g;      // ... and past the end of the sequence
        float pv[CPT], dsv[CPT];
        if (cmin <= 0 && cmax >= CPT)   // interior: no mask in this row's columns
          pds_math<false>(su, du, &s_ld[sl][CPT * g], &s_ld[sl][QB + CPT * g], sl2, p.scale, cmin, cmax, pv, dsv);
        else
          pds_math<true>(su, du, &s_ld[sl][CPT * g], &s_ld[sl][QB + CPT * g], sl2, p.scale, cmin, cmax, pv, dsv);
        BP(3);
#if MENOS_BWS_TMEM_P
        {   // P^T, dS^T -> the first 16 of the 32 S^T / dP^T columns this thread group read
          uint32_t up[CPT / 2], ud[CPT / 2];
          pack_row(pv, up);
          pack_row(dsv, ud);
          tmem_st_half(tmem + 64 * b + CPT * g + lane_off, up);
          tmem_st_half(tmem + 128 + 64 * b + CPT * g + lane_off, ud);
          tmem_wait_st();
        }
        BP(4);
#else
        if (gb >= 2) wait_bar(&pd_free[b], ((gb - 2) >> 1) & 1);
        if (j == 0 && tma_pending) {   // the previous item's dK / dV TMA stores have read the staging buffers
          if (t == 0) bulk_wait_read0();
          ew_sync();
          tma_pending = false;
        }
        BP(4);
        st_half_row(sP0 + b * PT_TILE, r, g, pv);
        st_half_row(sS0 + b * PT_TILE, r, g, dsv);
        fence_proxy_async();
#endif
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&ew_done[b]);
        BP(5);
      }
      // ------------------------------------------------ epilogue: dK (RoPE bwd), dV rows -> dqkv
      const int nv = min(KV_ROWS, L - k0);
      const bool rope = p.rope_cs != nullptr && r < nv;
      RopeCS<HD> csk;
      rope_cs_load<HD>(csk, p.rope_cs, max(0, k0 + r - G.sh), g, rope);   // in flight during the wait below
      BP(0);
      wait_bar(&acc_full, it & 1);
      BP(6);
      tc_fence_after();
#if MENOS_BWS_TMEM_P
      if (t == 0 && tma_pending) bulk_wait_read0();   // the previous item's TMA stores have read the staging
      tma_pending = false;
#endif
      ew_sync();   // order every warp's last P^T / dS^T stores before the staging writes (the mbarrier chain through
                   // the MMAs already does; the named barrier makes it visible to compute-sanitizer racecheck)
      // all MMAs of this item completed: P^T / dS^T buffers (64 KB, contiguous) = bf16 staging of dK | dV
      acc_row_to_bf16<HD>(tdK + lane_off, sP0, r, g, csk, rope);
      acc_row_to_bf16<HD>(tdV + lane_off, sP0 + 128 * HD * 2, r, g, csk, false);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&acc_free);   // the next item's dK / dV accumulation may start
      BP(7);
      if (nv == KV_ROWS) {   // full block: TMA stores, the warps go on with the next item
        fence_proxy_async();
        ew_sync();
        if (t == 0) {
          stage_tma_store<HD>(&tmOut, sP0, base + k0, (p.H + G.head) * HD);
          stage_tma_store<HD>(&tmOut, sP0 + 128 * HD * 2, base + k0, (p.H + p.Hkv + G.head) * HD);
          bulk_commit();
        }
        tma_pending = true;
      } else {               // the sequence's ragged last block: row-masked stores
        bf16* dst = p.dqkv + (size_t)(base + k0) * p.ld_dqkv;
        ew_sync();
        stage16_store<HD>(sP0, 2, w8, lane, nv, dst + (p.H + G.head) * HD, dst + (p.H + p.Hkv + G.head) * HD,
                          p.ld_dqkv);
        ew_sync();
      }
      BP(8);
    }
#endif
    if (t == 0 || (p.ds && (warp & 3) == 0 && lane == 0)) bulk_wait0();   // epilogue / dS^T stores complete
    BP_FLUSH(blockIdx.x < 8 && t == 0);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

// ======================================================================================= dQ
constexpr int Q_ROWS = 128, KB = 64;
constexpr int DS_TILE = Q_ROWS * KB * 2;      // 16 KB
constexpr int QA = Q_ROWS * 128, KBA = KB * 128;   // one SW128 atom of a Q / dO tile, of a K / V stage
template <int HD> struct DqGeo {
  static constexpr int Q_TILE = Q_ROWS * HD * 2;   // HD 128: 32 KB; 64: 16 KB
  static constexpr int KB_TILE = KB * HD * 2;      // 16 KB; 8 KB
  static constexpr int SMEM = 2 * Q_TILE + 2 * STAGES * KB_TILE + 2 * DS_TILE + 1024;
};

template <int HD>
__global__ void __launch_bounds__(NTHREADS, 1)
attn_bwd_dq_ws_kernel(const __grid_constant__ CUtensorMap tmQKV128, const __grid_constant__ CUtensorMap tmQKV64,
                      const __grid_constant__ CUtensorMap tmDO128, const __grid_constant__ CUtensorMap tmOut,
                      const BwParams p) {
  constexpr int Q_TILE = DqGeo<HD>::Q_TILE, KB_TILE = DqGeo<HD>::KB_TILE;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* const sQ = smem;
  uint8_t* const sO = sQ + Q_TILE;
  uint8_t* const sK0 = sO + Q_TILE;                  // K stages
  uint8_t* const sV0 = sK0 + STAGES * KB_TILE;       // V stages
  uint8_t* const sS0 = sV0 + STAGES * KB_TILE;       // dS (2 buffers) -- dQ staging in the epilogue
  __shared__ __align__(8) uint64_t q_full, q_empty, full[STAGES], empty[STAGES], s_full[2], ew_done[2], pd_free[2];
  __shared__ __align__(8) uint64_t acc_full, acc_free;
  __shared__ uint32_t tmem_sh;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    tma_prefetch(&tmQKV128); tma_prefetch(&tmQKV64); tma_prefetch(&tmDO128);
    mbar_init(&q_full, 1); mbar_init(&q_empty, 1);
    for (int i = 0; i < STAGES; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&s_full[i], 1); mbar_init(&ew_done[i], MENOS_BWS_ALT ? EW_WARPS / 2 : EW_WARPS); mbar_init(&pd_free[i], 1);
    }
    mbar_init(&acc_full, 1); mbar_init(&acc_free, EW_WARPS);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  const uint32_t tdQ = tmem + 256;   // S buffers at 0/64, dP at 128/192

  auto ip_init = [&](ItemPipe& q) {
    q.cur = item_at(p.items, p.n_items, blockIdx.x);
    ip_fetch(q, p.cu_seqlens, p.pos_shift);
    q.raw = item_at(p.items, p.n_items, blockIdx.x + gridDim.x);
  };
  auto ip_advance = [&](ItemPipe& q, int item) {
    q.cur = q.raw;
    ip_fetch(q, p.cu_seqlens, p.pos_shift);
    q.raw = item_at(p.items, p.n_items, item + 2 * gridDim.x);
  };
  auto decode = [&](const ItemPipe& q) {
    Geo g{q.c0, q.c1 - q.c0, q.cur.y, q.cur.z, 0, q.sh, q.cur.x};
    g.n = (min(g.L, g.blk0 + Q_ROWS) + KB - 1) / KB;   // 0 past the end
    return g;
  };

  if (warp == 0) {
    if (elect_one()) {
      ItemPipe ip;
      ip_init(ip);
      int it = 0, gb = 0;
      for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
        const Geo G = decode(ip);
        ip_advance(ip, item);
        const int h = G.head, hk = h / (p.H / p.Hkv), q0 = G.blk0;
        const int kcol = (p.H + hk) * HD, vcol = (p.H + p.Hkv + hk) * HD;
        wait_bar(&q_empty, (it & 1) ^ 1);
        mbar_expect_tx(&q_full, 2 * Q_TILE);
#pragma unroll
        for (int a = 0; a < HD / 64; ++a) {
          tma_load_2d(sQ + a * QA, &tmQKV128, &q_full, h * HD + 64 * a, G.base + q0);
          tma_load_2d(sO + a * QA, &tmDO128, &q_full, h * HD + 64 * a, G.base + q0);
        }
        for (int j = 0; j < G.n; ++j, ++gb) {
          const int st = gb % STAGES;
          wait_bar(&empty[st], ((gb / STAGES) & 1) ^ 1);
          mbar_expect_tx(&full[st], 2 * KB_TILE);
          uint8_t* k = sK0 + st * KB_TILE;
          uint8_t* v = sV0 + st * KB_TILE;
#pragma unroll
          for (int a = 0; a < HD / 64; ++a) {
            tma_load_2d(k + a * KBA, &tmQKV64, &full[st], kcol + 64 * a, G.base + j * KB);
            tma_load_2d(v + a * KBA, &tmQKV64, &full[st], vcol + 64 * a, G.base + j * KB);
          }
        }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    constexpr uint32_t ID_S = umma_idesc_bf16(128, KB, 0);     // [128 q] x [64 keys], K = hd
    constexpr uint32_t ID_ACC = umma_idesc_bf16(128, HD, 1);   // [128 q] x [hd], K = 64 keys, B MN-major
    ItemPipe ip;
    ip_init(ip);
    int it = 0, gb = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
      const Geo G = decode(ip);
      ip_advance(ip, item);
      auto issue_acc = [&](int gp, int jp) {  // dQ += dS K
        const int bp = gp & 1, sp = gp % STAGES;
        wait_bar(&ew_done[bp], (gp >> 1) & 1);
        if (jp == 0) wait_bar(&acc_free, (it & 1) ^ 1);
        tc_fence_after();
        __syncwarp();
        if (elect_one()) {
          const uint32_t kb_ = smem_u32(sK0 + sp * KB_TILE);
#if MENOS_BWS_TMEM_P
#pragma unroll
          for (int kk = 0; kk < 4; ++kk)   // A = dS packed in the S tile of buffer bp
            tc_mma_bf16_ts(tdQ, tmem + 64 * bp + packed_col(kk), umma_desc_sw128(kb_ + kk * 2048, 8192, 1024), ID_ACC,
                           (jp > 0 || kk > 0) ? 1u : 0u);
          tc_commit(&empty[sp]);
#else
          const uint32_t sa = smem_u32(sS0 + bp * DS_TILE);
#pragma unroll
          for (int kk = 0; kk < 4; ++kk)
            tc_mma_bf16(tdQ, umma_desc_sw128(sa + kk * 32, 16, 1024), umma_desc_sw128(kb_ + kk * 2048, 8192, 1024), ID_ACC,
                        (jp > 0 || kk > 0) ? 1u : 0u);
          tc_commit(&empty[sp]);
          tc_commit(&pd_free[bp]);
#endif
        }
        __syncwarp();
      };
      wait_bar(&q_full, it & 1);
      tc_fence_after();
      for (int j = 0; j < G.n; ++j, ++gb) {
        const int b = gb & 1, st = gb % STAGES;
        wait_bar(&full[st], (gb / STAGES) & 1);
        tc_fence_after();
        __syncwarp();
        if (elect_one()) {
          const uint32_t q = smem_u32(sQ), o = smem_u32(sO);
          const uint32_t k = smem_u32(sK0 + st * KB_TILE), v = smem_u32(sV0 + st * KB_TILE);
#pragma unroll
          for (int kk = 0; kk < HD / 16; ++kk) {
            const uint32_t offa = (kk >> 2) * QA + (kk & 3) * 32, offb = (kk >> 2) * KBA + (kk & 3) * 32;
            tc_mma_bf16(tmem + 64 * b, umma_desc_sw128(q + offa, 16, 1024), umma_desc_sw128(k + offb, 16, 1024), ID_S, kk > 0);
            tc_mma_bf16(tmem + 128 + 64 * b, umma_desc_sw128(o + offa, 16, 1024), umma_desc_sw128(v + offb, 16, 1024), ID_S, kk > 0);
          }
          tc_commit(&s_full[b]);
          if (j == G.n - 1) tc_commit(&q_empty);   // Q / dO free once the item's last S / dP completes
        }
        __syncwarp();
        if (j > 0) issue_acc(gb - 1, j - 1);
      }
      if (G.n > 0) issue_acc(gb - 1, G.n - 1);
      __syncwarp();
      if (elect_one()) tc_commit(&acc_full);
      __syncwarp();
    }
  } else {
#if MENOS_BWS_ALT
    // group gr = w8 / 4 takes the key blocks of parity gr (its S / dP buffer); thread = query row, all 64 key columns
    const int w4 = warp & 3, w8 = warp - 2, gr = w8 >> 2, t = threadIdx.x - 64;
    const int r = w4 * 32 + lane;           // query row
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_W;
    ItemPipe ip;
    ip_init(ip);
    // lse (log2 domain) and pre-scaled D of this thread's query row in item G; loaded one item ahead
    auto row_stats = [&](const Geo& G, float& l2, float& dq) {
      const int qpos = G.blk0 + r;
      const bool ok = G.n > 0 && qpos < G.L;
      l2 = ok ? __ldg(p.lse + (size_t)G.head * p.T + G.base + qpos) : 0.f;
      dq = ok ? __ldg(p.D + (size_t)G.head * p.T + G.base + qpos) : 0.f;
    };
    float lse_n = 0.f, D_n = 0.f;
    bool tma_pending = false;
    int it = 0, gb = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
      const Geo G = decode(ip);
      ip_advance(ip, item);
      const int h = G.head, q0 = G.blk0, L = G.L, base = G.base;
      const int qpos = q0 + r;
      const bool qok = qpos < L;
      if (it == 0) row_stats(G, lse_n, D_n);
      const float lse2 = lse_n * LOG2E_W, Dq = D_n * p.scale;   // Dq pre-scaled
      bool stats_next = false;
      for (int j = 0; j < G.n; ++j, ++gb) {
        if ((gb & 1) != gr) continue;
        wait_bar(&s_full[gr], (gb >> 1) & 1);
        tc_fence_after();
        __syncwarp();
#pragma unroll 1
        for (int hf = 0; hf < 2; ++hf) {   // key columns [32 hf, 32 hf + 32)
          uint32_t su[CPT], du[CPT];
          tmem_ldc_nw(tmem + 64 * gr + 32 * hf + lane_off, su);
          tmem_ldc_nw(tmem + 128 + 64 * gr + 32 * hf + lane_off, du);
          tmem_wait_ld();
          const int cmax = qok ? qpos - j * KB - 32 * hf : -1;   // keys <= query
          float dsv[CPT];
          if (cmax >= CPT - 1) {   // no masked column
#pragma unroll
            for (int c = 0; c < CPT; ++c) {
              const float x = fmaf(__uint_as_float(su[c]), sl2, -lse2);
              const float e = (c & 3) == 3 ? poly_exp2(x) : fast_exp2(x);
              dsv[c] = e * fmaf(__uint_as_float(du[c]), p.scale, -Dq);
            }
          } else {
#pragma unroll
            for (int c = 0; c < CPT; ++c) {
              const float x = fmaf(__uint_as_float(su[c]), sl2, -lse2);
              const float e = (c & 3) == 3 ? poly_exp2(x) : fast_exp2(x);
              const float v = e * fmaf(__uint_as_float(du[c]), p.scale, -Dq);
              dsv[c] = c <= cmax ? v : 0.f;
            }
          }
          uint32_t ud[CPT / 2];
          pack_row(dsv, ud);
          tmem_st_half(tmem + 64 * gr + 32 * hf + lane_off, ud);
        }
        if (!stats_next) { row_stats(decode(ip), lse_n, D_n); stats_next = true; }   // next item's (geometry arrived)
        tmem_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&ew_done[gr]);
      }
      if (!stats_next) row_stats(decode(ip), lse_n, D_n);   // this group had no block in the item
      const int nv = min(Q_ROWS, L - q0);
      const bool rope = p.rope_cs != nullptr && r < nv;
      RopeCS<HD> csq;
      rope_cs_load<HD>(csq, p.rope_cs, max(0, q0 + r - G.sh), gr, rope);   // in flight during the wait below
      wait_bar(&acc_full, it & 1);
      tc_fence_after();
      if (t == 0 && tma_pending) bulk_wait_read0();   // the previous item's TMA store has read the staging
      tma_pending = false;
      ew_sync();
      // dS buffers (32 KB) = bf16 staging of dQ
      acc_row_to_bf16<HD>(tdQ + lane_off, sS0, r, gr, csq, rope);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&acc_free);
      if (nv == Q_ROWS) {
        fence_proxy_async();
        ew_sync();
        if (t == 0) {
          stage_tma_store<HD>(&tmOut, sS0, base + q0, h * HD);
          bulk_commit();
        }
        tma_pending = true;
      } else {
        ew_sync();
        bf16* dq = p.dqkv + (size_t)(base + q0) * p.ld_dqkv + h * HD;
        stage16_store<HD>(sS0, 1, w8, lane, nv, dq, dq, p.ld_dqkv);
        ew_sync();
      }
    }
#else
    const int w4 = warp & 3, w8 = warp - 2, g = w8 >> 2, t = threadIdx.x - 64;   // warp group g owns key columns [CPT g, CPT g + CPT)
    const int r = w4 * 32 + lane;           // query row
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_W;
    ItemPipe ip;
    ip_init(ip);
    // lse (log2 domain) and pre-scaled D of this thread's query row in item G; loaded one item ahead
    auto row_stats = [&](const Geo& G, float& l2, float& dq) {
      const int qpos = G.blk0 + r;
      const bool ok = G.n > 0 && qpos < G.L;
      l2 = ok ? __ldg(p.lse + (size_t)G.head * p.T + G.base + qpos) : 0.f;
      dq = ok ? __ldg(p.D + (size_t)G.head * p.T + G.base + qpos) : 0.f;
    };
    float lse_n = 0.f, D_n = 0.f;
    bool tma_pending = false;
    int it = 0, gb = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
      const Geo G = decode(ip);
      ip_advance(ip, item);
      const int h = G.head, q0 = G.blk0, L = G.L, base = G.base;
      const int qpos = q0 + r;
      const bool qok = qpos < L;
      if (it == 0) row_stats(G, lse_n, D_n);
      const float lse2 = lse_n * LOG2E_W, Dq = D_n * p.scale;   // Dq pre-scaled
      for (int j = 0; j < G.n; ++j, ++gb) {
        const int b = gb & 1;
        wait_bar(&s_full[b], (gb >> 1) & 1);
        tc_fence_after();
        __syncwarp();
        uint32_t su[CPT], du[CPT];
        tmem_ldc_nw(tmem + 64 * b + CPT * g + lane_off, su);
        tmem_ldc_nw(tmem + 128 + 64 * b + CPT * g + lane_off, du);
        tmem_wait_ld();
        const int cmax = qok ? qpos - j * KB - CPT * g : -1;   // keys <= query
        float dsv[CPT];
        if (cmax >= CPT - 1) {   // no masked column in this row
#pragma unroll
          for (int c = 0; c < CPT; ++c) {
            const float x = fmaf(__uint_as_float(su[c]), sl2, -lse2);
            const float e = (c & 3) == 3 ? poly_exp2(x) : fast_exp2(x);
            dsv[c] = e * fmaf(__uint_as_float(du[c]), p.scale, -Dq);
          }
        } else {
#pragma unroll
          for (int c = 0; c < CPT; ++c) {
            const float x = fmaf(__uint_as_float(su[c]), sl2, -lse2);
            const float e = (c & 3) == 3 ? poly_exp2(x) : fast_exp2(x);
            const float v = e * fmaf(__uint_as_float(du[c]), p.scale, -Dq);
            dsv[c] = c <= cmax ? v : 0.f;
          }
        }
        if (j == 0) row_stats(decode(ip), lse_n, D_n);   // next item's row statistics (its geometry has arrived)
#if MENOS_BWS_TMEM_P
        {   // dS -> the first 16 of the 32 S columns this thread group read
          uint32_t ud[CPT / 2];
          pack_row(dsv, ud);
          tmem_st_half(tmem + 64 * b + CPT * g + lane_off, ud);
          tmem_wait_st();
        }
#else
        if (gb >= 2) wait_bar(&pd_free[b], ((gb - 2) >> 1) & 1);
        if (j == 0 && tma_pending) {   // the previous item's dQ TMA store has read the staging buffers
          if (t == 0) bulk_wait_read0();
          ew_sync();
          tma_pending = false;
        }
        st_half_row(sS0 + b * DS_TILE, r, g, dsv);
        fence_proxy_async();
#endif
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&ew_done[b]);
      }
      const int nv = min(Q_ROWS, L - q0);
      const bool rope = p.rope_cs != nullptr && r < nv;
      RopeCS<HD> csq;
      rope_cs_load<HD>(csq, p.rope_cs, max(0, q0 + r - G.sh), g, rope);   // in flight during the wait below
      wait_bar(&acc_full, it & 1);
      tc_fence_after();
#if MENOS_BWS_TMEM_P
      if (t == 0 && tma_pending) bulk_wait_read0();   // the previous item's TMA store has read the staging
      tma_pending = false;
#endif
      ew_sync();   // as in the dK / dV epilogue: the dS^T stores of every warp precede the staging writes
      // dS buffers (32 KB) = bf16 staging of dQ
      acc_row_to_bf16<HD>(tdQ + lane_off, sS0, r, g, csq, rope);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&acc_free);
      if (nv == Q_ROWS) {
        fence_proxy_async();
        ew_sync();
        if (t == 0) {
          stage_tma_store<HD>(&tmOut, sS0, base + q0, h * HD);
          bulk_commit();
        }
        tma_pending = true;
      } else {
        ew_sync();
        bf16* dq = p.dqkv + (size_t)(base + q0) * p.ld_dqkv + h * HD;
        stage16_store<HD>(sS0, 1, w8, lane, nv, dq, dq, p.ld_dqkv);
        ew_sync();
      }
    }
#endif
    if (t == 0) bulk_wait0();
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

// ======================================================================================= dQ from stored dS^T
// dQ[q, :] = sum over key blocks kb <= q-block of dS[q, keys of kb] K[keys of kb, :], with dS^T read back from the
// tiles the dK/dV kernel stored (bf16 [128 keys][64 queries], linear; TMA applies the 128-byte swizzle), so S, P and
// dP are computed ONCE per (key, query) pair: this pass is a memory-bound varlen GEMM (M = 128 queries = two
// 64-query tiles read as one MN-major A operand one M-atom apart, N = head_dim, K = 128 keys per block).
// Roles: warp 0 TMA (dS^T pair + K block per stage, 3-stage ring across items), warp 1 MMA (dQ in one of two TMEM
// accumulators, so an item's epilogue overlaps the next item's MMAs), warps 2-9 the epilogue (RoPE backward, bf16,
// TMA store) exactly as in attn_bwd_dq_ws_kernel.
constexpr int DSQ_STAGES = 3;
template <int HD> struct DqDsGeo {
  static constexpr int DS2 = 2 * KV_ROWS * QB * 2;   // two dS^T tiles: 32 KB
  static constexpr int KT = KV_ROWS * HD * 2;        // K block: 32 KB (HD 128) / 16 KB
  static constexpr int STAGE = DS2 + KT;
  static constexpr int STG = Q_ROWS * HD * 2;        // bf16 staging of one dQ block
  static constexpr int SMEM = DSQ_STAGES * STAGE + STG + 1024;
};
static_assert(DqDsGeo<128>::SMEM <= 232448, "dQ-from-dS shared memory");

template <int HD>
__global__ void __launch_bounds__(NTHREADS, 1)
attn_bwd_dq_ds_kernel(const __grid_constant__ CUtensorMap tmDS, const __grid_constant__ CUtensorMap tmQKV128,
                      const __grid_constant__ CUtensorMap tmOut, const BwParams p) {
  using Gm = DqDsGeo<HD>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* const sStage = smem;                              // [stage][dS^T pair | K block]
  uint8_t* const sStg = smem + DSQ_STAGES * Gm::STAGE;       // dQ staging
  __shared__ __align__(8) uint64_t full[DSQ_STAGES], empty[DSQ_STAGES], acc_full[2], acc_free[2];
  __shared__ uint32_t tmem_sh;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int rep = p.H / p.Hkv;
  if (threadIdx.x == 0) {
    tma_prefetch(&tmDS); tma_prefetch(&tmQKV128);
    for (int i = 0; i < DSQ_STAGES; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&acc_full[i], 1); mbar_init(&acc_free[i], EW_WARPS); }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<2 * HD>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  // item -> (sequence geometry, q0, head); items are read directly (the producer runs ahead of everyone else)
  auto geo = [&](int item, int& base, int& L, int& q0, int& h, int& seq) {
    const int4 it = p.items[item];
    seq = it.x; q0 = it.y; h = it.z;
    base = p.cu_seqlens[seq]; L = p.cu_seqlens[seq + 1] - base;
  };

  if (warp == 0) {
    if (elect_one()) {
      int gb = 0;
      for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
        if (p.items[item].x < 0) continue;   // padding (attn_ds_plan): a CTA's tail
        int base, L, q0, h, seq;
        geo(item, base, L, q0, h, seq);
        const int hk = h / rep;
        const int t_head = __ldg(p.ds_base + seq * p.Hkv + hk) + (h - hk * rep) * ds_tiles_of(L);
        const int kcol = (p.H + hk) * HD;
        for (int kb = 0; kb <= q0 / KV_ROWS; ++kb, ++gb) {
          const int st = gb % DSQ_STAGES;
          wait_bar(&empty[st], ((gb / DSQ_STAGES) & 1) ^ 1);
          mbar_expect_tx(&full[st], Gm::STAGE);
          uint8_t* sd = sStage + st * Gm::STAGE;
          const int tile = t_head + ds_tile_in_head(L, kb, q0 / QB);   // (kb, 2 qb128) and the next tile
          tma_load_2d(sd, &tmDS, &full[st], 0, tile * KV_ROWS);
#pragma unroll
          for (int a = 0; a < HD / 64; ++a)
            tma_load_2d(sd + Gm::DS2 + a * KVA, &tmQKV128, &full[st], kcol + 64 * a, base + kb * KV_ROWS);
        }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    constexpr uint32_t ID_DQ = umma_idesc_bf16(128, HD, 1) | (1u << 15);   // A (dS) and B (K) MN-major
    int gb = 0, it = 0;   // it counts real items only (accumulator buffer and phase)
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
      if (p.items[item].x < 0) continue;
      const int q0 = p.items[item].y;
      const int buf = it & 1;
      wait_bar(&acc_free[buf], ((it >> 1) & 1) ^ 1);
      tc_fence_after();
      for (int kb = 0; kb <= q0 / KV_ROWS; ++kb, ++gb) {
        const int st = gb % DSQ_STAGES;
        wait_bar(&full[st], (gb / DSQ_STAGES) & 1);
        tc_fence_after();
        __syncwarp();
        if (elect_one()) {
          const uint32_t sd = smem_u32(sStage + st * Gm::STAGE), sk = sd + Gm::DS2;
          const uint64_t dd0 = umma_desc_sw128(sd, 16384, 1024), kd0 = umma_desc_sw128(sk, 16384, 1024);
#pragma unroll
          for (int kk = 0; kk < KV_ROWS / 16; ++kk)   // 16 keys = 2048 B of both the dS^T pair and the K block
            tc_mma_bf16(tmem + buf * HD, dd0 + (uint64_t)((kk * 2048) >> 4), kd0 + (uint64_t)((kk * 2048) >> 4), ID_DQ,
                        (kb > 0 || kk > 0) ? 1u : 0u);
          tc_commit(&empty[st]);
        }
        __syncwarp();
      }
      if (elect_one()) tc_commit(&acc_full[buf]);
      __syncwarp();
      ++it;
    }
  } else {
    const int w4 = warp & 3, w8 = warp - 2, g = w8 >> 2, t = threadIdx.x - 64;
    const int r = w4 * 32 + lane;   // query row = TMEM lane
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    bool tma_pending = false;
    int it = 0, prev_seq = -1, prev_q0 = -1;
    RopeCS<HD> csq;   // kept across a run of items at the same (sequence, query block): loaded once per run
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
      if (p.items[item].x < 0) continue;
      int base, L, q0, h, seq;
      geo(item, base, L, q0, h, seq);
      const int sh = p.pos_shift ? p.pos_shift[seq] : 0;
      const int buf = it & 1;
      const int nv = min(Q_ROWS, L - q0);
      const bool rope = p.rope_cs != nullptr && r < nv;
      if (seq != prev_seq || q0 != prev_q0)
        rope_cs_load<HD>(csq, p.rope_cs, max(0, q0 + r - sh), g, rope);   // in flight during the wait below
      prev_seq = seq; prev_q0 = q0;
      wait_bar(&acc_full[buf], (it >> 1) & 1);
      tc_fence_after();
      if (t == 0 && tma_pending) bulk_wait_read0();   // the previous item's TMA store has read the staging
      tma_pending = false;
      ew_sync();
      acc_row_to_bf16<HD>(tmem + buf * HD + lane_off, sStg, r, g, csq, rope);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&acc_free[buf]);
      if (nv == Q_ROWS) {
        fence_proxy_async();
        ew_sync();
        if (t == 0) {
          stage_tma_store<HD>(&tmOut, sStg, base + q0, h * HD);
          bulk_commit();
        }
        tma_pending = true;
      } else {
        ew_sync();
        bf16* dq = p.dqkv + (size_t)(base + q0) * p.ld_dqkv + h * HD;
        stage16_store<HD>(sStg, 1, w8, lane, nv, dq, dq, p.ld_dqkv);
        ew_sync();
      }
      ++it;
    }
    if (t == 0) bulk_wait0();
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<2 * HD>(tmem);
  }
}

}  // namespace

#ifdef MENOS_BWS_PROF
int attn_bws_prof_read(unsigned long long* out) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out, g_bws_prof, sizeof(unsigned long long) * 16);
  unsigned long long z[16] = {0};
  cudaMemcpyToSymbol(g_bws_prof, z, sizeof z);
  return 0;
}
#endif

// items_kv: (seq, k0, kv head) per 128-key block for dK/dV; items_q: (seq, q0, head) per 128-query block for dQ
template <int HD>
static int launch_bwd_ws(const AttnArgs& a, const int4* items_kv, int n_items_kv, const int4* items_q, int n_items_q,
                         int num_sms, cudaStream_t st) {
  CUtensorMap mQKV128, mQKV64, mDO64, mDO128, mOut;
  if (!tma_map_2d(&mQKV128, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, 128)) return -2;
  if (!tma_map_2d(&mOut, a.dqkv, a.T, (a.H + 2 * a.Hkv) * HD, a.ld_dqkv, 64, 128)) return -2;   // dK / dV / dQ stores
  if (!tma_map_2d(&mQKV64, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, 64)) return -2;
  if (!tma_map_2d(&mDO64, a.dO, a.T, a.H * HD, a.ld_do, 64, 64)) return -2;
  if (!tma_map_2d(&mDO128, a.dO, a.T, a.H * HD, a.ld_do, 64, 128)) return -2;
  BwParams p;
  memset(&p, 0, sizeof p);
  p.cu_seqlens = a.cu_seqlens; p.lse = a.lse; p.D = a.D; p.dqkv = a.dqkv;
  p.ld_dqkv = a.ld_dqkv; p.rope_cs = a.rope_cs; p.pos_shift = a.pos_shift; p.T = a.T; p.H = a.H; p.Hkv = a.Hkv;
  p.scale = a.scale;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_bwd_dkdv_ws_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, DkdvGeo<HD>::SMEM);
    cudaFuncSetAttribute(attn_bwd_dq_ws_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, DqGeo<HD>::SMEM);
    attr = true;
  }
  p.items = items_kv; p.n_items = n_items_kv;
  if (n_items_kv > 0)
    attn_bwd_dkdv_ws_kernel<HD><<<min(n_items_kv, num_sms), NTHREADS, DkdvGeo<HD>::SMEM, st>>>(mQKV128, mQKV64, mDO64,
                                                                                                mOut, mQKV128, p);
  ++g_launch_count;
  p.items = items_q; p.n_items = n_items_q;
  if (n_items_q > 0)
    attn_bwd_dq_ws_kernel<HD><<<min(n_items_q, num_sms), NTHREADS, DqGeo<HD>::SMEM, st>>>(mQKV128, mQKV64, mDO128,
                                                                                            mOut, p);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

// dS-stored variant: dK/dV (storing dS^T tiles) then dQ from the tiles
template <int HD>
static int launch_bwd_ws_ds(const AttnArgs& a, const int4* items_kv, int n_items_kv, const int4* items_q, int n_items_q,
                            bf16* ds, long long ds_tiles, const int* ds_base, int num_sms, cudaStream_t st) {
  CUtensorMap mQKV128, mQKV64, mDO64, mOut, mDS;
  if (!tma_map_2d(&mQKV128, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, 128)) return -2;
  if (!tma_map_2d(&mOut, a.dqkv, a.T, (a.H + 2 * a.Hkv) * HD, a.ld_dqkv, 64, 128)) return -2;
  if (!tma_map_2d(&mQKV64, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, 64)) return -2;
  if (!tma_map_2d(&mDO64, a.dO, a.T, a.H * HD, a.ld_do, 64, 64)) return -2;
  if (!tma_map_2d(&mDS, ds, (uint64_t)ds_tiles * KV_ROWS, QB, QB, 64, KV_ROWS)) return -2;      // dK/dV: store
  CUtensorMap mDS2;
  if (!tma_map_2d(&mDS2, ds, (uint64_t)ds_tiles * KV_ROWS, QB, QB, 64, 2 * KV_ROWS)) return -2;  // dQ: tile pairs
  BwParams p;
  memset(&p, 0, sizeof p);
  p.cu_seqlens = a.cu_seqlens; p.lse = a.lse; p.D = a.D; p.dqkv = a.dqkv;
  p.ld_dqkv = a.ld_dqkv; p.rope_cs = a.rope_cs; p.pos_shift = a.pos_shift; p.T = a.T; p.H = a.H; p.Hkv = a.Hkv;
  p.scale = a.scale; p.ds = ds; p.ds_base = ds_base;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_bwd_dkdv_ws_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, DkdvGeo<HD>::SMEM);
    cudaFuncSetAttribute(attn_bwd_dq_ds_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, DqDsGeo<HD>::SMEM);
    attr = true;
  }
  p.items = items_kv; p.n_items = n_items_kv;
  if (n_items_kv > 0) {
    attn_bwd_dkdv_ws_kernel<HD><<<min(n_items_kv, num_sms), NTHREADS, DkdvGeo<HD>::SMEM, st>>>(mQKV128, mQKV64, mDO64,
                                                                                                mOut, mDS, p);
    ++g_launch_count;
  }
  p.items = items_q; p.n_items = n_items_q;
  if (n_items_q > 0) {
    attn_bwd_dq_ds_kernel<HD><<<min(n_items_q, num_sms), NTHREADS, DqDsGeo<HD>::SMEM, st>>>(mDS2, mQKV128, mOut, p);
    ++g_launch_count;
  }
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

int attn_bwd_ws_ds(const AttnArgs& a, const int4* items_kv, int n_items_kv, const int4* items_q, int n_items_q,
                   bf16* ds, long long ds_tiles, const int* ds_base, int num_sms, cudaStream_t st) {
  if (!MENOS_BWS_ALT) return -1;   // the dS^T stores live in the alternating-group elementwise path
  if (n_items_kv <= 0 && n_items_q <= 0) return 0;
  if (a.hd == 128) return launch_bwd_ws_ds<128>(a, items_kv, n_items_kv, items_q, n_items_q, ds, ds_tiles, ds_base, num_sms, st);
  if (a.hd == 64) return launch_bwd_ws_ds<64>(a, items_kv, n_items_kv, items_q, n_items_q, ds, ds_tiles, ds_base, num_sms, st);
  return -1;
}
int attn_ds_tiles(int L) { return ds_tiles_of(L); }

long long attn_ds_total_tiles(const int* seq_len, int n_seqs, int H) {
  long long t = 0;
  for (int i = 0; i < n_seqs; ++i) t += (long long)H * ds_tiles_of(seq_len[i]);
  return t;
}

bool attn_ds_plan(const int* seq_len, int n_seqs, int H, int Hkv, long long cap_tiles, AttnDsPlan& out, int grid) {
  const int rep = H / Hkv;
  out.base.assign((size_t)n_seqs * Hkv, 0);
  out.items_kv.clear(); out.items_q.clear(); out.chunks.clear();
  std::vector<int2> units;   // (seq, kv head) of the open chunk
  long long cur = 0;
  int grp = 0;               // (sequence, head) groups of dQ items so far (rotation of their query-block order)
  auto flush = [&]() {
    if (units.empty()) return;
    const int kv0 = (int)out.items_kv.size(), q0 = (int)out.items_q.size();
    for (const int2& u : units) {
      const int L = seq_len[u.x];
      for (int k = 0; k < L; k += 128) out.items_kv.push_back(make_int4(u.x, k, u.y, 0));
      const int nq = (L + 127) / 128;
      if (grid <= 0)
        for (int h = u.y * rep; h < (u.y + 1) * rep; ++h, ++grp)
          for (int j = 0; j < nq; ++j) out.items_q.push_back(make_int4(u.x, (nq - 1 - (j + grp) % nq) * 128, h, 0));
    }
    if (grid > 0) {
      // dQ items for a persistent grid of `grid` CTAs (CTA c takes list entries c, c + grid, ...): each CTA gets a
      // RUN of items with the same (sequence, query block) over consecutive heads, so its epilogue loads the RoPE
      // rows once per run instead of once per item (r2cj: the RoPE-table loads bound the dQ pass).  Natural order
      // (sequence, query block, head) split into `grid` contiguous ranges of equal cost (kv blocks per item), then
      // interleaved; CTAs with shorter ranges are padded with (-1, ...) entries at their tail (the kernel stops there).
      std::vector<int4> nat;
      std::vector<int> cost;
      for (size_t i = 0; i < units.size(); ++i) {
        const int sq = units[i].x;
        if (i > 0 && units[i - 1].x == sq) continue;   // units of one sequence are adjacent
        const int nq = (seq_len[sq] + 127) / 128;
        for (int j = nq - 1; j >= 0; --j)
          for (size_t k = i; k < units.size() && units[k].x == sq; ++k)
            for (int h = units[k].y * rep; h < (units[k].y + 1) * rep; ++h) {
              nat.push_back(make_int4(sq, j * 128, h, 0));
              cost.push_back(j + 1);
            }
      }
      long long total = 0;
      for (int c : cost) total += c;
      std::vector<int> lo(grid + 1, (int)nat.size());
      lo[0] = 0;
      long long acc = 0;
      int c = 1;
      for (size_t i = 0; i < nat.size() && c < grid; ++i) {
        while (c < grid && acc >= total * c / grid) lo[c++] = (int)i;
        acc += cost[i];
      }
      int mx = 0;
      for (int k = 0; k < grid; ++k) mx = std::max(mx, lo[k + 1] - lo[k]);
      const size_t at = out.items_q.size();
      out.items_q.resize(at + (size_t)mx * grid, make_int4(-1, 0, 0, 0));
      for (int k = 0; k < grid; ++k)
        for (int t = 0; t < lo[k + 1] - lo[k]; ++t) out.items_q[at + (size_t)t * grid + k] = nat[lo[k] + t];
    }
    // dK/dV: LPT for the persistent grid's static round-robin (largest = most query blocks after the key block)
    std::stable_sort(out.items_kv.begin() + kv0, out.items_kv.end(), [&](const int4& a, const int4& b) {
      return seq_len[a.x] - a.y > seq_len[b.x] - b.y;
    });
    attn_snake_waves(out.items_kv, kv0, grid);
    // dQ items stay grouped by (sequence, head) so neighbouring CTAs read the same K blocks at the same time (one
    // L2 fill instead of one per query block); inside a group the query blocks are ROTATED by the group's index, so
    // the static round-robin (stride = grid, a multiple of 4 when the grid is 148) does not hand one CTA the same
    // query-block position -- the same cost -- in every group (r2bn: 1.6x load imbalance at cfg1)
    out.chunks.push_back(make_int4(kv0, (int)out.items_kv.size() - kv0, q0, (int)out.items_q.size() - q0));
    units.clear();
    cur = 0;
  };
  for (int i = 0; i < n_seqs; ++i)
    for (int hk = 0; hk < Hkv; ++hk) {
      const long long ut = (long long)rep * ds_tiles_of(seq_len[i]);
      if (ut > cap_tiles) return false;
      if (cur + ut > cap_tiles) flush();
      out.base[(size_t)i * Hkv + hk] = (int)cur;
      cur += ut;
      units.push_back(make_int2(i, hk));
    }
  flush();
  return true;
}

int attn_bwd_ws(const AttnArgs& a, const int4* items_kv, int n_items_kv, const int4* items_q, int n_items_q,
                int num_sms, cudaStream_t st) {
  if (n_items_kv <= 0 && n_items_q <= 0) return 0;
  if (a.hd == 128) return launch_bwd_ws<128>(a, items_kv, n_items_kv, items_q, n_items_q, num_sms, st);
  if (a.hd == 64) return launch_bwd_ws<64>(a, items_kv, n_items_kv, items_q, n_items_q, num_sms, st);
  return -1;
}

}  // namespace menos
