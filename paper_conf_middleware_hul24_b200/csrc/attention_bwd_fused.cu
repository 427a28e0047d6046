// Varlen causal flash-attention BACKWARD in ONE pass, persistent warp-specialized tcgen05, head_dim 128.
// SURVEY.md §8(a) A11; VERDICT r1 "next" #3.
//
// Work item = (sequence, kv head): the CTA walks the item's 128-key blocks j = 0, 1, ... and, for each, every (query
// head of the GQA group, 64-query block at or after the key block).  S^T = K Q^T, dP^T = V dO^T and
// P^T = exp2(S^T c - lse), dS^T = P^T (dP^T - D) scale are computed ONCE per (key block, query block) and feed all
// three gradient products:
//     dV_j += P^T dO        dK_j += dS^T Q        dQ_i = dS K_j (two 64-query blocks per MMA, M = 128)
// (10 hd MMA FLOP per causal pair, against 14 hd and twice the exponentials for the separate dK/dV and dQ kernels).
//
// dV_j, dK_j accumulate in TMEM over the key block's query blocks and are written once per key block.  dQ_i collects
// one contribution per key block j <= i; since one CTA owns all key blocks of the (sequence, kv head), every dQ element
// is accumulated by ONE thread in program order through an fp32 buffer (L2-resident): j = 0 stores, later blocks
// red.add (fire-and-forget), the last contributor (j = q0 / 128) loads the sum, adds its own, applies the RoPE
// backward and writes the bf16 dq -- deterministic (batched == alone, SAVE == re-forward, bitwise)
// without atomics ordering, semaphores or a separate reduction pass.  Items are in LPT order (longest sequence first).
//
// Warp roles (448 threads, one CTA per SM):
//   warp 0       TMA producer: K and V of the key block (two 32 KB buffers that swap roles every key block, so the next
//                block's K is loaded as soon as the last dP^T MMA has read V), Q / dO 64-row stages (ring of 3) with
//                the block's lse and D staged beside them by the warp's lanes
//   warp 1       MMA issuer (tcgen05.mma, one elected lane)
//   warps 2-9    softmax-gradient warps: one TMEM lane (= key row) per thread, 32 query columns each
//   warps 2-9    (also, once per key block, the dK (RoPE backward) / dV epilogue, straight from TMEM to global)
//   warps 10-13  dQ drain: one TMEM lane (= query row of a block pair) per thread, all 128 head dims (the RoPE pairs
//                are in-thread): TMEM -> program-ordered fp32 accumulate -> RoPE backward -> bf16
// TMEM (512 columns): S^T 0..63 | dP^T 64..127 | dQ (a block pair: 128 query rows x 128 hd) 128..255 | dV 256..383 |
// dK 384..511.
#include "common.cuh"
#include "kernels.h"

#include <cstdlib>

namespace menos {

bool tma_map_2d(CUtensorMap* out, const void* ptr, uint64_t rows, uint64_t cols, uint64_t ld, uint32_t bc,
                uint32_t br);

namespace {

constexpr int HD = 128, STAGES = 3, EW_WARPS = 8, DR_WARPS = 4;
constexpr int NTHREADS = 64 + 32 * EW_WARPS + 32 * DR_WARPS;   // 448
constexpr int CPT = 32;                                        // query columns per softmax-gradient thread
constexpr float LOG2E_F = 1.4426950408889634f;
constexpr int KV_ROWS = 128, QB = 64;
constexpr int KV_TILE = KV_ROWS * HD * 2;      // 32 KB (2 SW128 atoms [128][64])
constexpr int QB_TILE = QB * HD * 2;           // 16 KB (2 atoms [64][64])
constexpr int PT_TILE = KV_ROWS * QB * 2;      // 16 KB (1 atom [128][64])
constexpr int SMEM_FUSED = 2 * KV_TILE + 2 * STAGES * QB_TILE + 4 * PT_TILE + 1024;
constexpr uint32_t T_S = 0, T_DP = 64, T_DQ = 128, T_DV = 256, T_DK = 384;   // TMEM columns

struct FParams {
  const int* cu_seqlens;
  const int4* items;       // (seq, -, kv head, -), LPT order (longest sequence first)
  int n_items;
  const float* lse;        // [H, T] natural log
  const float* D;          // [H, T]
  bf16* dqkv; int ld_dqkv;
  const float2* rope_cs;   // [max_pos][HD/2] (cos, sin) or nullptr (no RoPE: OPT)
  float* dq_acc;           // [T, H*HD] fp32 partial sums of dQ
  const int* pos_shift;    // [n_seqs] prefix rows before each sequence (extended batch) or nullptr
  int T, H, Hkv;
  float scale;
  int dbg;                 // tuning only (MENOS_ABF_DBG): 1 drain skips the global accumulation, 3 no RoPE
                           // exchange (results wrong for 1, 3)
};

__device__ __forceinline__ void ew_sync() { asm volatile("bar.sync 1, %0;" ::"n"(32 * EW_WARPS) : "memory"); }
__device__ __forceinline__ void wait_bar(uint64_t* bar, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile("{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  }
}


// bf16x2 pack with round-to-nearest-even on the integer pipe (finite inputs): offloads the conversion unit
__device__ __forceinline__ uint32_t pack_bf16x2_alu(float lo, float hi) {
  const uint32_t a = __float_as_uint(lo), b = __float_as_uint(hi);
  const uint32_t ra = a + 0x7FFFu + ((a >> 16) & 1u), rb = b + 0x7FFFu + ((b >> 16) & 1u);
  return __byte_perm(ra, rb, 0x7632);
}

// Instruction descriptor kind::f16 with both operand majors selectable (bit 15: A MN-major, bit 16: B MN-major).
__host__ __device__ constexpr uint32_t idesc_ab(int M, int N, int a_mn, int b_mn) {
  return umma_idesc_bf16(M, N, b_mn) | ((uint32_t)a_mn << 15);
}

// columns [CPT g, CPT g + CPT) of one row of a [rows][64] SWIZZLE_128B bf16 tile, from packed bf16x2 pairs
__device__ __forceinline__ void st_half_row_packed(uint8_t* tile, int row, int g, const uint32_t (&u)[CPT / 2]) {
  uint8_t* prow = tile + row * 128;
#pragma unroll
  for (int c = 0; c < CPT / 8; ++c) {
    const int c8 = (CPT / 8) * g + c;
    *reinterpret_cast<uint4*>(prow + ((c8 ^ (row & 7)) << 4)) =
        make_uint4(u[4 * c], u[4 * c + 1], u[4 * c + 2], u[4 * c + 3]);
  }
}

struct Geo { int seq, base, L, hk, nkv; };

// -DMENOS_ABF_PROF: per-phase clock64 accounting of one thread per role (read with menos_test_abf_prof)
#ifdef MENOS_ABF_PROF
__device__ unsigned long long g_abf_prof[16];
#define PF_DECL long long pf_t = clock64(); unsigned long long pfr_[16] = {0};
#define PF(k) do { const long long t_ = clock64(); pfr_[k] += t_ - pf_t; pf_t = t_; } while (0)
#define PF_FLUSH(cond) do { if (cond) for (int k_ = 0; k_ < 16; ++k_) if (pfr_[k_]) atomicAdd(&g_abf_prof[k_], pfr_[k_]); } while (0)
#else
#define PF_DECL
#define PF(k) do {} while (0)
#define PF_FLUSH(cond) do {} while (0)
#endif

__global__ void __launch_bounds__(NTHREADS, 1)
attn_bwd_fused_kernel(const __grid_constant__ CUtensorMap tmQKV128, const __grid_constant__ CUtensorMap tmQKV64,
                      const __grid_constant__ CUtensorMap tmDO64, const FParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* const sX0 = smem;                          // K / V buffers (roles swap every key block)
  uint8_t* const sQ0 = sX0 + 2 * KV_TILE;             // Q stages
  uint8_t* const sO0 = sQ0 + STAGES * QB_TILE;        // dO stages
  uint8_t* const sP0 = sO0 + STAGES * QB_TILE;        // P^T  (2 buffers) -- dK staging in the epilogue
  uint8_t* const sS0 = sP0 + 2 * PT_TILE;             // dS^T (2 buffers) -- dV staging in the epilogue
  __shared__ __align__(8) uint64_t x_full[2], x_empty[2], full[STAGES], empty[STAGES];
  __shared__ __align__(8) uint64_t s_full, sd_free, ew_done[2], pd_free[2], dq_full[2], dq_free[2];
  __shared__ __align__(8) uint64_t acc_full, acc_free;
  __shared__ uint32_t tmem_sh;
  __shared__ __align__(16) float s_lse[STAGES][QB], s_D[STAGES][QB];   // per stage: lse (log2 domain), D (scaled)

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int rep = p.H / p.Hkv;
  if (threadIdx.x == 0) {
    tma_prefetch(&tmQKV128); tma_prefetch(&tmQKV64); tma_prefetch(&tmDO64);
    for (int i = 0; i < 2; ++i) {   // dq_full / dq_free: only [0] is used (one dQ accumulator)
      mbar_init(&x_full[i], 1); mbar_init(&x_empty[i], 1);
      mbar_init(&ew_done[i], EW_WARPS); mbar_init(&pd_free[i], 1);
      mbar_init(&dq_full[i], 1); mbar_init(&dq_free[i], DR_WARPS);
    }
    for (int i = 0; i < STAGES; ++i) { mbar_init(&full[i], 2); mbar_init(&empty[i], 1); }   // TMA tx + lse/D stores
    mbar_init(&s_full, 1); mbar_init(&sd_free, EW_WARPS);
    mbar_init(&acc_full, 1); mbar_init(&acc_free, EW_WARPS);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;

  auto load_geo = [&](int item) {
    Geo g{0, 0, 0, 0, 0};
    if (item < p.n_items) {
      const int4 it = p.items[item];
      g.seq = it.x; g.base = p.cu_seqlens[it.x]; g.L = p.cu_seqlens[it.x + 1] - g.base; g.hk = it.z;
      g.nkv = (g.L + KV_ROWS - 1) / KV_ROWS;
    }
    return g;
  };
  // key block j of an item: query blocks [k0, L) in 64-row blocks, DESCENDING, heads of the GQA group inner
  auto nqb_of = [&](const Geo& G, int j) { return (G.L - j * KV_ROWS + QB - 1) / QB; };
  auto blk = [&](const Geo& G, int j, int nqb, int jj, int& h, int& q0) {
    h = G.hk * rep + jj % rep;
    q0 = j * KV_ROWS + (nqb - 1 - jj / rep) * QB;
  };

  if (warp == 0) {
    // ------------------------------------------------ TMA producer (lane 0 issues TMA; the warp stages lse / D)
    const bool leader = elect_one();
    const float sl2 = LOG2E_F;
    int kvit = 0, gb = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
      const Geo G = load_geo(item);
      const int kcol = (p.H + G.hk) * HD, vcol = (p.H + p.Hkv + G.hk) * HD;
      for (int j = 0; j < G.nkv; ++j, ++kvit) {
        const int kb = kvit & 1, vb = kb ^ 1, k0 = j * KV_ROWS, nqb = nqb_of(G, j), n = rep * nqb;
        uint8_t* sK = sX0 + kb * KV_TILE;
        uint8_t* sV = sX0 + vb * KV_TILE;
        if (leader) {
          wait_bar(&x_empty[kb], (kvit & 1) ^ 1);
          mbar_expect_tx(&x_full[kb], KV_TILE);
          tma_load_2d(sK, &tmQKV128, &x_full[kb], kcol, G.base + k0);
          tma_load_2d(sK + 16384, &tmQKV128, &x_full[kb], kcol + 64, G.base + k0);
        }
        for (int jj = 0; jj < n; ++jj, ++gb) {
          const int st = gb % STAGES;
          int h, q0;
          blk(G, j, nqb, jj, h, q0);
          if (jj == 1 && leader) {   // V of this key block: its buffer held the previous block's K until now
            wait_bar(&x_empty[vb], (kvit & 1) ^ 1);
            mbar_expect_tx(&x_full[vb], KV_TILE);
            tma_load_2d(sV, &tmQKV128, &x_full[vb], vcol, G.base + k0);
            tma_load_2d(sV + 16384, &tmQKV128, &x_full[vb], vcol + 64, G.base + k0);
          }
          wait_bar(&empty[st], ((gb / STAGES) & 1) ^ 1);
          if (leader) {
            mbar_expect_tx(&full[st], 2 * QB_TILE);
            uint8_t* q = sQ0 + st * QB_TILE;
            uint8_t* o = sO0 + st * QB_TILE;
            tma_load_2d(q, &tmQKV64, &full[st], h * HD, G.base + q0);
            tma_load_2d(q + 8192, &tmQKV64, &full[st], h * HD + 64, G.base + q0);
            tma_load_2d(o, &tmDO64, &full[st], h * HD, G.base + q0);
            tma_load_2d(o + 8192, &tmDO64, &full[st], h * HD + 64, G.base + q0);
          }
          // lse (log2 domain) and D (pre-scaled) of the block's 64 queries: 2 per lane; 0 past the sequence end
#pragma unroll
          for (int u = 0; u < 2; ++u) {
            const int c = lane + 32 * u, qpos = q0 + c;
            const size_t o = (size_t)h * p.T + G.base + qpos;
            s_lse[st][c] = qpos < G.L ? __ldg(p.lse + o) * sl2 : 0.f;
            s_D[st][c] = qpos < G.L ? __ldg(p.D + o) * p.scale : 0.f;
          }
          __syncwarp();
          if (lane == 0) mbar_arrive(&full[st]);
          if (n == 1 && leader) {    // a one-block key block: V was not issued inside the loop
            wait_bar(&x_empty[vb], (kvit & 1) ^ 1);
            mbar_expect_tx(&x_full[vb], KV_TILE);
            tma_load_2d(sV, &tmQKV128, &x_full[vb], vcol, G.base + k0);
            tma_load_2d(sV + 16384, &tmQKV128, &x_full[vb], vcol + 64, G.base + k0);
          }
        }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer
    constexpr uint32_t ID_S = idesc_ab(128, QB, 0, 0);    // S^T, dP^T: [128 kv] x [64 q], K = hd
    constexpr uint32_t ID_ACC = idesc_ab(128, HD, 0, 1);  // dV, dK: [128 kv] x [128 hd], K = 64 q, B MN-major
    constexpr uint32_t ID_DQ = idesc_ab(128, HD, 1, 1);   // dQ: [128 q (two blocks)] x [128 hd], K = 128 kv
    PF_DECL
    int kvit = 0, gb = 0, npair = 0, use[2] = {0, 0};
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
      const Geo G = load_geo(item);
      for (int j = 0; j < G.nkv; ++j, ++kvit) {
        const int kb = kvit & 1, vb = kb ^ 1, n = rep * nqb_of(G, j);
        const uint32_t k_s = smem_u32(sX0 + kb * KV_TILE), v_s = smem_u32(sX0 + vb * KV_TILE);
        // dV += P^T dO ; dK += dS^T Q for block jp (P/dS buffer jp & 1); after the second block of a pair (or a
        // unit's unpaired last block) dQ[2 x 64 q][hd] = dS (both dS^T buffers read MN-major as one M = 128 operand:
        // they sit 16 KB apart = one M-atom stride) . K_j
        auto issue_acc = [&](int gp, int jp) {
          const int bp = jp & 1, sp = gp % STAGES;
          const bool dq_now = (jp & 1) || jp == n - 1;
          PF(6);
          wait_bar(&ew_done[bp], use[bp] & 1);
          PF(3);
          if (jp == 0) wait_bar(&acc_free, (kvit & 1) ^ 1);   // previous key block's epilogue has read dV / dK
          PF(4);
          if (dq_now) wait_bar(&dq_free[0], (npair & 1) ^ 1);   // the drain has read the previous pair's dQ
          PF(5);
          tc_fence_after();
          __syncwarp();
          if (elect_one()) {
            const uint32_t pa = smem_u32(sP0 + bp * PT_TILE), sa = smem_u32(sS0 + bp * PT_TILE);
            const uint32_t ob = smem_u32(sO0 + sp * QB_TILE), qb = smem_u32(sQ0 + sp * QB_TILE);
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) {
              const uint32_t acc = (jp > 0 || kk > 0) ? 1u : 0u;
              tc_mma_bf16(tmem + T_DV, umma_desc_sw128(pa + kk * 32, 16, 1024), umma_desc_sw128(ob + kk * 2048, 8192, 1024), ID_ACC, acc);
              tc_mma_bf16(tmem + T_DK, umma_desc_sw128(sa + kk * 32, 16, 1024), umma_desc_sw128(qb + kk * 2048, 8192, 1024), ID_ACC, acc);
            }
            tc_commit(&empty[sp]);     // Q/dO stage free
            if (dq_now) {
              const uint32_t s0 = smem_u32(sS0);
#pragma unroll
              for (int kk = 0; kk < 8; ++kk)   // K-steps of 16 key rows = 2048 B in both the dS^T tiles and K
                tc_mma_bf16(tmem + T_DQ, umma_desc_sw128(s0 + kk * 2048, 16384, 1024),
                            umma_desc_sw128(k_s + kk * 2048, 16384, 1024), ID_DQ, kk > 0 ? 1u : 0u);
              tc_commit(&dq_full[0]);
              tc_commit(&pd_free[0]);                  // both P^T/dS^T buffers read for the last time
              if (jp & 1) tc_commit(&pd_free[1]);
            }
            if (jp == n - 1) { tc_commit(&x_empty[kb]); tc_commit(&acc_full); }   // K read for the last time
          }
          __syncwarp();
          ++use[bp];
          if (dq_now) ++npair;
        };
        PF(6);
        wait_bar(&x_full[kb], kvit & 1);
        PF(2);
        for (int jj = 0; jj < n; ++jj, ++gb) {
          const int st = gb % STAGES;
          PF(6);
          wait_bar(&full[st], (gb / STAGES) & 1);
          PF(0);
          wait_bar(&sd_free, (gb & 1) ^ 1);           // softmax warps have read S^T / dP^T of block gb - 1
          PF(1);
          tc_fence_after();
          __syncwarp();
          const uint32_t q = smem_u32(sQ0 + st * QB_TILE), o = smem_u32(sO0 + st * QB_TILE);
          if (elect_one()) {
#pragma unroll
            for (int kk = 0; kk < 8; ++kk) {
              const uint32_t offa = (kk >> 2) * 16384 + (kk & 3) * 32, offb = (kk >> 2) * 8192 + (kk & 3) * 32;
              tc_mma_bf16(tmem + T_S, umma_desc_sw128(k_s + offa, 16, 1024), umma_desc_sw128(q + offb, 16, 1024), ID_S, kk > 0);
            }
          }
          __syncwarp();
          PF(6);
          if (jj == 0) { wait_bar(&x_full[vb], kvit & 1); tc_fence_after(); }   // V lands after the first S^T
          PF(2);
          __syncwarp();
          if (elect_one()) {
#pragma unroll
            for (int kk = 0; kk < 8; ++kk) {
              const uint32_t offa = (kk >> 2) * 16384 + (kk & 3) * 32, offb = (kk >> 2) * 8192 + (kk & 3) * 32;
              tc_mma_bf16(tmem + T_DP, umma_desc_sw128(v_s + offa, 16, 1024), umma_desc_sw128(o + offb, 16, 1024), ID_S, kk > 0);
            }
            tc_commit(&s_full);
            if (jj == n - 1) tc_commit(&x_empty[vb]);   // V read for the last time: the next block's K goes here
          }
          __syncwarp();
          if (jj > 0) issue_acc(gb - 1, jj - 1);
        }
        if (n > 0) issue_acc(gb - 1, n - 1);
        __syncwarp();
      }
    }
    PF(6);
    PF_FLUSH(lane == 0);
  } else if (warp < 2 + EW_WARPS) {
    // ------------------------------------------------ softmax-gradient warps (thread = key row = TMEM lane;
    //                                                  warp group g owns query columns [CPT g, CPT g + CPT))
    const int w4 = warp & 3, w8 = warp - 2, g = w8 >> 2;
    const int r = w4 * 32 + lane;
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_F;
    PF_DECL
    int kvit = 0, gb = 0, use[2] = {0, 0};
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
      const Geo G = load_geo(item);
      for (int j = 0; j < G.nkv; ++j, ++kvit) {
        const int k0 = j * KV_ROWS, nqb = nqb_of(G, j), n = rep * nqb;
        const int kpos = k0 + r;
        PF(8);
        for (int jj = 0; jj < n; ++jj, ++gb) {
          const int b = jj & 1, st = gb % STAGES;
          int h, q0;
          blk(G, j, nqb, jj, h, q0);
          PF(8);
          wait_bar(&full[st], (gb / STAGES) & 1);     // the stage's lse / D (stored by the producer lanes)
          wait_bar(&s_full, gb & 1);
          PF(7);
          tc_fence_after();
          __syncwarp();
          uint32_t su[CPT], du[CPT];
          tmem_ld32_nw(tmem + T_S + CPT * g + lane_off, su);
          tmem_ld32_nw(tmem + T_DP + CPT * g + lane_off, du);
          tmem_wait_ld();
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&sd_free);    // the next S^T / dP^T may overwrite TMEM
          const int cmin = kpos - q0 - CPT * g;   // P = 0 for queries before the key (causal) ...
          const int cmax = G.L - q0 - CPT * g;    // ... and past the end of the sequence
          const bool fullb = cmin <= 0 && cmax >= CPT;
          uint32_t pk[CPT / 2], dk[CPT / 2];       // bf16x2-packed P^T and dS^T (packed as produced)
#pragma unroll
          for (int c4 = 0; c4 < CPT; c4 += 4) {
            const float4 lz = *reinterpret_cast<const float4*>(&s_lse[st][CPT * g + c4]);   // stage st is live:
            const float4 dz = *reinterpret_cast<const float4*>(&s_D[st][CPT * g + c4]);     // freed after acc(gb)
            const float lzv[4] = {lz.x, lz.y, lz.z, lz.w}, dzv[4] = {dz.x, dz.y, dz.z, dz.w};
            float pv[4], dsv[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              const int c = c4 + u;
              const bool ok = fullb || (c >= cmin && c < cmax);
              const float x = fmaf(__uint_as_float(su[c]), sl2, -lzv[u]);
              const float e = (u == 3 || ((p.dbg == 4 || p.dbg == 6) && u == 1)) ? poly_exp2(x) : fast_exp2(x);
              pv[u] = ok ? e : 0.f;
              dsv[u] = ok ? e * fmaf(__uint_as_float(du[c]), p.scale, -dzv[u]) : 0.f;
            }
            if (p.dbg == 5 || p.dbg == 6) {
              pk[c4 / 2] = pack_bf16x2_alu(pv[0], pv[1]); pk[c4 / 2 + 1] = pack_bf16x2_alu(pv[2], pv[3]);
            } else {
              pk[c4 / 2] = pack_bf16x2(pv[0], pv[1]); pk[c4 / 2 + 1] = pack_bf16x2(pv[2], pv[3]);
            }
            dk[c4 / 2] = pack_bf16x2(dsv[0], dsv[1]); dk[c4 / 2 + 1] = pack_bf16x2(dsv[2], dsv[3]);
          }
          PF(8);
          wait_bar(&pd_free[b], (use[b] & 1) ^ 1);   // the buffer's previous block has been read by its MMAs
          PF(9);
          st_half_row_packed(sP0 + b * PT_TILE, r, g, pk);
          st_half_row_packed(sS0 + b * PT_TILE, r, g, dk);
          fence_proxy_async();
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&ew_done[b]);
          ++use[b];
        }
        // ---------------------------------------------- epilogue of key block j: key row r, columns [32g, 32g+32) of
        // dK (and their RoPE partners 64 + ..., in-thread) and of dV -> bf16 rows staged (swizzled) in the P^T / dS^T
        // buffers (all of the key block's MMAs are done), then written by whole rows; the first half of the thread's
        // RoPE table row is fetched before the wait for the key block's last MMA
        const int nv = min(KV_ROWS, G.L - k0), kr = k0 + r;
        const int sh = p.pos_shift ? p.pos_shift[G.seq] : 0;   // prefix rows: position < 0 -> identity (R28)
        const bool rope = p.rope_cs != nullptr && r < nv;
        const float4* c4 = reinterpret_cast<const float4*>(p.rope_cs + (size_t)(r < nv ? max(0, kr - sh) : 0) * (HD / 2) +
                                                           CPT * g);
        float4 cs8[8];
        if (rope) {
#pragma unroll
          for (int k = 0; k < 8; ++k) cs8[k] = __ldg(c4 + k);
        }
        PF(8);
        wait_bar(&acc_full, kvit & 1);
        PF(10);
        tc_fence_after();
        ew_sync();   // every warp's last P^T / dS^T stores precede the staging writes (visible to racecheck)
        uint8_t* row_k = sP0 + r * 256;            // dK staging tile [128 rows][256 B]
        uint8_t* row_v = sP0 + 32768 + r * 256;    // dV staging tile
#pragma unroll
        for (int hh = 0; hh < 2; ++hh) {           // 16 dims of the thread's 32 at a time (and their partners)
          uint32_t ka[16], kb2[16];
          asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                       : "=r"(ka[0]), "=r"(ka[1]), "=r"(ka[2]), "=r"(ka[3]), "=r"(ka[4]), "=r"(ka[5]), "=r"(ka[6]), "=r"(ka[7]),
                         "=r"(ka[8]), "=r"(ka[9]), "=r"(ka[10]), "=r"(ka[11]), "=r"(ka[12]), "=r"(ka[13]), "=r"(ka[14]), "=r"(ka[15])
                       : "r"(tmem + T_DK + CPT * g + 16 * hh + lane_off));
          asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                       : "=r"(kb2[0]), "=r"(kb2[1]), "=r"(kb2[2]), "=r"(kb2[3]), "=r"(kb2[4]), "=r"(kb2[5]), "=r"(kb2[6]), "=r"(kb2[7]),
                         "=r"(kb2[8]), "=r"(kb2[9]), "=r"(kb2[10]), "=r"(kb2[11]), "=r"(kb2[12]), "=r"(kb2[13]), "=r"(kb2[14]), "=r"(kb2[15])
                       : "r"(tmem + T_DK + 64 + CPT * g + 16 * hh + lane_off));
          tmem_wait_ld();
          float x[16], y[16];
#pragma unroll
          for (int k = 0; k < 16; ++k) { x[k] = __uint_as_float(ka[k]); y[k] = __uint_as_float(kb2[k]); }
          if (rope) {   // dx_i = dy_i c + dy_{i+64} s ; dx_{i+64} = dy_{i+64} c - dy_i s
            if (hh == 1) {
#pragma unroll
              for (int k = 0; k < 8; ++k) cs8[k] = __ldg(c4 + 8 + k);
            }
#pragma unroll
            for (int k = 0; k < 8; ++k) {
              const float4 e = cs8[k];
              const float x0 = x[2 * k] * e.x + y[2 * k] * e.y, y0 = y[2 * k] * e.x - x[2 * k] * e.y;
              const float x1 = x[2 * k + 1] * e.z + y[2 * k + 1] * e.w, y1 = y[2 * k + 1] * e.z - x[2 * k + 1] * e.w;
              x[2 * k] = x0; y[2 * k] = y0; x[2 * k + 1] = x1; y[2 * k + 1] = y1;
            }
          }
#pragma unroll
          for (int k = 0; k < 2; ++k) {   // 16-byte chunk c of the row at ((c ^ (r & 15)) << 4)
            const int ck = (CPT / 8) * g + 2 * hh + k;
            *reinterpret_cast<uint4*>(row_k + ((ck ^ (r & 15)) << 4)) =
                make_uint4(pack_bf16x2(x[8 * k], x[8 * k + 1]), pack_bf16x2(x[8 * k + 2], x[8 * k + 3]),
                           pack_bf16x2(x[8 * k + 4], x[8 * k + 5]), pack_bf16x2(x[8 * k + 6], x[8 * k + 7]));
            *reinterpret_cast<uint4*>(row_k + (((8 + ck) ^ (r & 15)) << 4)) =
                make_uint4(pack_bf16x2(y[8 * k], y[8 * k + 1]), pack_bf16x2(y[8 * k + 2], y[8 * k + 3]),
                           pack_bf16x2(y[8 * k + 4], y[8 * k + 5]), pack_bf16x2(y[8 * k + 6], y[8 * k + 7]));
          }
        }
#pragma unroll
        for (int hh = 0; hh < 2; ++hh) {   // dV columns [32g, 32g+32) and [64+32g, ..)
          uint32_t va[32];
          tmem_ld32_nw(tmem + T_DV + 64 * hh + CPT * g + lane_off, va);
          tmem_wait_ld();
          if (hh == 1) {
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&acc_free);   // dK / dV read: the next key block may accumulate
          }
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const int ck = 8 * hh + (CPT / 8) * g + k;
            *reinterpret_cast<uint4*>(row_v + ((ck ^ (r & 15)) << 4)) =
                make_uint4(pack_bf16x2(__uint_as_float(va[8 * k]), __uint_as_float(va[8 * k + 1])),
                           pack_bf16x2(__uint_as_float(va[8 * k + 2]), __uint_as_float(va[8 * k + 3])),
                           pack_bf16x2(__uint_as_float(va[8 * k + 4]), __uint_as_float(va[8 * k + 5])),
                           pack_bf16x2(__uint_as_float(va[8 * k + 6]), __uint_as_float(va[8 * k + 7])));
          }
        }
        ew_sync();
        {   // whole rows: 16 lanes x 16 B per 256-byte row, 2 rows per instruction
          bf16* dst0 = p.dqkv + (size_t)(G.base + k0) * p.ld_dqkv + (p.H + G.hk) * HD;
          bf16* dst1 = dst0 + p.Hkv * HD;
          const int kq = lane & 15;
#pragma unroll 4
          for (int i = 0; i < 128 * 2 / (2 * EW_WARPS); ++i) {
            const int R = i * (2 * EW_WARPS) + w8 * 2 + (lane >> 4), t = R >> 7, rr = R & 127;
            if (rr >= nv) continue;
            const uint4 v = *reinterpret_cast<const uint4*>(sP0 + t * 32768 + rr * 256 + ((kq ^ (rr & 15)) << 4));
            *reinterpret_cast<uint4*>((t ? dst1 : dst0) + (size_t)rr * p.ld_dqkv + kq * 8) = v;
          }
        }
        ew_sync();
        PF(11);
      }
    }
    PF_FLUSH(threadIdx.x == 64);
  } else {
    // ------------------------------------------------ dQ drain: thread = one query row of a block pair (TMEM lane:
    // rows 0-63 the pair's first block, 64-127 its second), all 128 head dims -- the RoPE pairs (d, d + 64) are in the
    // same thread.  The CTA owns every key block of its (sequence, kv head), so each dQ element is touched only by the
    // thread that owns its row: the contributions of key blocks j = 0, 1, ... are ordered by program order alone
    // (j = 0 stores, later blocks red.add, the last one loads the sum) -- deterministic without cross-CTA sync.
    const int w4 = warp & 3;
    const int r = w4 * 32 + lane, mem = r >> 6, qr = r & 63;
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    const int ldq = p.H * HD;
    const bool rope = p.rope_cs != nullptr && p.dbg != 3;
    PF_DECL
    int npair = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
      const Geo G = load_geo(item);
      for (int j = 0; j < G.nkv; ++j) {
        const int nqb = nqb_of(G, j), n = rep * nqb;
        for (int jp = 0; jp < n; jp += 2, ++npair) {
          const int jj = jp + mem;
          int h = 0, q0 = 0;
          if (jj < n) blk(G, j, nqb, jj, h, q0);
          const int q = q0 + qr;
          const bool active = jj < n && q < G.L && p.dbg != 1;
          const bool last = j == q0 / KV_ROWS;        // contributors to query q: key blocks 0..last
          float* acc = p.dq_acc + (size_t)(G.base + q) * ldq + h * HD;
          PF(14);
          wait_bar(&dq_full[0], npair & 1);
          PF(12);
          tc_fence_after();
          __syncwarp();
#pragma unroll
          for (int c = 0; c < 2; ++c) {   // columns [32c, 32c+32) and their RoPE partners [64+32c, ..)
            uint32_t ua[32], ub[32];
            tmem_ld32_nw(tmem + T_DQ + 32 * c + lane_off, ua);
            tmem_ld32_nw(tmem + T_DQ + 64 + 32 * c + lane_off, ub);
            tmem_wait_ld();
            if (c == 1) {
              tc_fence_before();
              __syncwarp();
              if (lane == 0) mbar_arrive(&dq_free[0]);
            }
            if (!active) continue;
            float4* a0 = reinterpret_cast<float4*>(acc + 32 * c);
            float4* a1 = reinterpret_cast<float4*>(acc + 64 + 32 * c);
            if (!last) {
              if (j == 0) {
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                  __stcg(a0 + k, make_float4(__uint_as_float(ua[4 * k]), __uint_as_float(ua[4 * k + 1]),
                                             __uint_as_float(ua[4 * k + 2]), __uint_as_float(ua[4 * k + 3])));
                  __stcg(a1 + k, make_float4(__uint_as_float(ub[4 * k]), __uint_as_float(ub[4 * k + 1]),
                                             __uint_as_float(ub[4 * k + 2]), __uint_as_float(ub[4 * k + 3])));
                }
              } else {
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                  asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(a0 + k),
                               "r"(ua[4 * k]), "r"(ua[4 * k + 1]), "r"(ua[4 * k + 2]), "r"(ua[4 * k + 3]) : "memory");
                  asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(a1 + k),
                               "r"(ub[4 * k]), "r"(ub[4 * k + 1]), "r"(ub[4 * k + 2]), "r"(ub[4 * k + 3]) : "memory");
                }
              }
              continue;
            }
            float x[32], y[32];
#pragma unroll
            for (int k = 0; k < 32; ++k) { x[k] = __uint_as_float(ua[k]); y[k] = __uint_as_float(ub[k]); }
            if (j > 0) {
#pragma unroll
              for (int k = 0; k < 8; ++k) {
                const float4 e = __ldcg(a0 + k), f = __ldcg(a1 + k);
                x[4 * k] += e.x; x[4 * k + 1] += e.y; x[4 * k + 2] += e.z; x[4 * k + 3] += e.w;
                y[4 * k] += f.x; y[4 * k + 1] += f.y; y[4 * k + 2] += f.z; y[4 * k + 3] += f.w;
              }
            }
            if (rope) {   // dx_d = dy_d c + dy_{d+64} s ; dx_{d+64} = dy_{d+64} c - dy_d s   (d = 32c + k)
              const int sh = p.pos_shift ? p.pos_shift[G.seq] : 0;
              const float4* c4 = reinterpret_cast<const float4*>(p.rope_cs + (size_t)max(0, q - sh) * (HD / 2) + 32 * c);
#pragma unroll
              for (int k = 0; k < 16; ++k) {
                const float4 e = __ldg(c4 + k);   // (cos, sin) of dims 2k, 2k + 1
                const float x0 = x[2 * k] * e.x + y[2 * k] * e.y, y0 = y[2 * k] * e.x - x[2 * k] * e.y;
                const float x1 = x[2 * k + 1] * e.z + y[2 * k + 1] * e.w, y1 = y[2 * k + 1] * e.z - x[2 * k + 1] * e.w;
                x[2 * k] = x0; y[2 * k] = y0; x[2 * k + 1] = x1; y[2 * k + 1] = y1;
              }
            }
            uint4* o0 = reinterpret_cast<uint4*>(p.dqkv + (size_t)(G.base + q) * p.ld_dqkv + h * HD + 32 * c);
            uint4* o1 = reinterpret_cast<uint4*>(p.dqkv + (size_t)(G.base + q) * p.ld_dqkv + h * HD + 64 + 32 * c);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              o0[k] = make_uint4(pack_bf16x2(x[8 * k], x[8 * k + 1]), pack_bf16x2(x[8 * k + 2], x[8 * k + 3]),
                                 pack_bf16x2(x[8 * k + 4], x[8 * k + 5]), pack_bf16x2(x[8 * k + 6], x[8 * k + 7]));
              o1[k] = make_uint4(pack_bf16x2(y[8 * k], y[8 * k + 1]), pack_bf16x2(y[8 * k + 2], y[8 * k + 3]),
                                 pack_bf16x2(y[8 * k + 4], y[8 * k + 5]), pack_bf16x2(y[8 * k + 6], y[8 * k + 7]));
            }
          }
          PF(13);
        }
      }
    }
    PF_FLUSH(threadIdx.x == 64 + 32 * EW_WARPS);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

}  // namespace

// per-phase cycle counters of the last MENOS_ABF_PROF build (zeros otherwise); reading clears them
int attn_bwd_fused_prof(unsigned long long* out16) {
#ifdef MENOS_ABF_PROF
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out16, g_abf_prof, sizeof(unsigned long long) * 16);
  unsigned long long z[16] = {0};
  cudaMemcpyToSymbol(g_abf_prof, z, sizeof z);
#else
  for (int k = 0; k < 16; ++k) out16[k] = 0;
#endif
  return 0;
}

int attn_bwd_fused(const AttnArgs& a, const int4* items_seq, int n_items, int num_sms, cudaStream_t st) {
  if (a.hd != HD) return -1;
  if (n_items <= 0) return 0;
  if (!a.dq_acc) return -1;
  CUtensorMap mQKV128, mQKV64, mDO64;
  if (!tma_map_2d(&mQKV128, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, 128)) return -2;
  if (!tma_map_2d(&mQKV64, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, 64)) return -2;
  if (!tma_map_2d(&mDO64, a.dO, a.T, a.H * HD, a.ld_do, 64, 64)) return -2;
  FParams p;
  p.cu_seqlens = a.cu_seqlens; p.items = items_seq; p.n_items = n_items; p.lse = a.lse; p.D = a.D;
  p.dqkv = a.dqkv; p.ld_dqkv = a.ld_dqkv; p.rope_cs = a.rope_cs; p.dq_acc = a.dq_acc; p.pos_shift = a.pos_shift;
  p.T = a.T; p.H = a.H; p.Hkv = a.Hkv; p.scale = a.scale;
  static const int dbg = getenv("MENOS_ABF_DBG") ? atoi(getenv("MENOS_ABF_DBG")) : 0;
  p.dbg = dbg;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_bwd_fused_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_FUSED);
    attr = true;
  }
  attn_bwd_fused_kernel<<<min(n_items, num_sms), NTHREADS, SMEM_FUSED, st>>>(mQKV128, mQKV64, mDO64, p);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

}  // namespace menos
