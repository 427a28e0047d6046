// Varlen causal flash-attention BACKWARD on the 5th-gen tensor cores (tcgen05 / TMEM / TMA), head_dim 128.
// SURVEY.md §8(a) A11.  Same contract as attn_bwd (attention.cu): deterministic (no atomics), blocks never cross a
// sequence, GQA, RoPE backward applied to dq / dk before the store.
//
// Two warp-specialized kernels, each a small "GEMM -> elementwise -> GEMM" pipeline:
//   dK/dV  (one CTA per 128-key block x kv head; loop over the group's heads x 64-query blocks):
//       S^T = K Q^T, dP^T = V dO^T          (tcgen05 -> TMEM, double-buffered)
//       P^T = exp(S^T c - lse), dS^T = P^T (dP^T - D) scale          (4 elementwise warps, thread = key row)
//       dV += P^T dO, dK += dS^T Q          (tcgen05, P^T / dS^T from swizzled smem, accumulators in TMEM)
//   dQ     (one CTA per 128-query block x head; loop over 64-key blocks):
//       S = Q K^T, dP = dO V^T -> dS = P (dP - D) scale -> dQ += dS K
// Warp roles: warp 0 TMA producer, warp 1 MMA issuer (elected lane), warps 2-5 elementwise + epilogue.
#include <cstdio>
#include "common.cuh"
#include "kernels.h"

namespace menos {

bool tma_map_2d(CUtensorMap* out, const void* ptr, uint64_t rows, uint64_t cols, uint64_t ld, uint32_t bc,
                uint32_t br);

namespace {

constexpr int HD = 128;
constexpr float LOG2E_B = 1.4426950408889634f;

struct TcBwdParams {
  const int* cu_seqlens;
  const int2* blocks;      // dkdv: (seq, k0) per 128-key block; dq: (seq, q0) per 128-query block
  const float* lse;        // [H, T] natural log
  const float* D;          // [H, T]
  bf16* dqkv; int ld_dqkv;
  const float2* rope_cs;
  int T, H, Hkv;
  float scale;
};

// mbarrier wait with a 2 s watchdog: a pipeline bug traps (launch error) instead of hanging the device
__device__ __forceinline__ void bw_wait(uint64_t* bar, uint32_t parity) {
  uint64_t t0 = 0;
  for (uint32_t n = 0;; ++n) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    if (ok) return;
    if ((n & 255) == 255) {
      uint64_t t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      if (t0 == 0) t0 = t;
      else if (t - t0 > 2000000000ull) __trap();
    }
  }
}

// write 64 bf16 of one row into a [rows][64] SWIZZLE_128B K-major tile
__device__ __forceinline__ void st_row64_sw128(uint8_t* tile, int row, const float (&v)[64]) {
  uint8_t* prow = tile + row * 128;
#pragma unroll
  for (int c8 = 0; c8 < 8; ++c8) {
    uint4 u = make_uint4(pack_bf16x2(v[8 * c8 + 0], v[8 * c8 + 1]), pack_bf16x2(v[8 * c8 + 2], v[8 * c8 + 3]),
                         pack_bf16x2(v[8 * c8 + 4], v[8 * c8 + 5]), pack_bf16x2(v[8 * c8 + 6], v[8 * c8 + 7]));
    *reinterpret_cast<uint4*>(prow + ((c8 ^ (row & 7)) << 4)) = u;
  }
}

__device__ __forceinline__ void tmem_ld64(uint32_t taddr, float (&v)[64]) {
  float a[32], b[32];
  tmem_ld32(taddr, a);
  tmem_ld32(taddr + 32, b);
#pragma unroll
  for (int c = 0; c < 32; ++c) { v[c] = a[c]; v[32 + c] = b[c]; }
}

// RoPE backward on a full 128-wide row held as 4 chunks of 32 (pairs j, j+64): dx_j = dy_j c + dy_{j+64} s,
// dx_{j+64} = dy_{j+64} c - dy_j s
__device__ __forceinline__ void rope_bwd_row(float (&r0)[32], float (&r1)[32], float (&r2)[32], float (&r3)[32],
                                             const float2* cs) {
#pragma unroll
  for (int j = 0; j < 32; ++j) {
    float2 e = cs[j];
    float y1 = r0[j], y2 = r2[j];
    r0[j] = y1 * e.x + y2 * e.y;
    r2[j] = y2 * e.x - y1 * e.y;
    e = cs[32 + j];
    y1 = r1[j]; y2 = r3[j];
    r1[j] = y1 * e.x + y2 * e.y;
    r3[j] = y2 * e.x - y1 * e.y;
  }
}

__device__ __forceinline__ void st_row32_bf16(bf16* dst, const float (&v)[32]) {
  uint4* d = reinterpret_cast<uint4*>(dst);
#pragma unroll
  for (int q = 0; q < 4; ++q)
    d[q] = make_uint4(pack_bf16x2(v[8 * q], v[8 * q + 1]), pack_bf16x2(v[8 * q + 2], v[8 * q + 3]),
                      pack_bf16x2(v[8 * q + 4], v[8 * q + 5]), pack_bf16x2(v[8 * q + 6], v[8 * q + 7]));
}

// ======================================================================================= dK / dV kernel
constexpr int KV_ROWS = 128, QB = 64;
constexpr int KV_TILE = KV_ROWS * HD * 2;      // 32 KB (2 atoms [128][64])
constexpr int QB_TILE = QB * HD * 2;           // 16 KB (2 atoms [64][64])
constexpr int PT_TILE = KV_ROWS * QB * 2;      // 16 KB (1 atom [128][64])
constexpr int SMEM_DKDV = 2 * KV_TILE + 4 * QB_TILE + 4 * PT_TILE + 1024;   // 193 KB

__global__ void __launch_bounds__(192, 1)
attn_bwd_dkdv_tc_kernel(const __grid_constant__ CUtensorMap tmQKV128, const __grid_constant__ CUtensorMap tmQKV64,
                        const __grid_constant__ CUtensorMap tmDO64, const TcBwdParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sK = smem;
  uint8_t* sV = sK + KV_TILE;
  // stage b of each double buffer at base + b * tile
  uint8_t* const sQ0 = sV + KV_TILE;              // Q stages
  uint8_t* const sO0 = sQ0 + 2 * QB_TILE;         // dO stages
  uint8_t* const sP0 = sO0 + 2 * QB_TILE;         // P^T
  uint8_t* const sS0 = sP0 + 2 * PT_TILE;         // dS^T
#define sQ(b) (sQ0 + (b) * QB_TILE)
#define sO(b) (sO0 + (b) * QB_TILE)
#define sP(b) (sP0 + (b) * PT_TILE)
#define sS(b) (sS0 + (b) * PT_TILE)
  __shared__ __align__(8) uint64_t bar_kv, full[2], empty[2], s_full[2], ew_done[2], acc_done;
  __shared__ uint32_t tmem_sh;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int2 kb = p.blocks[blockIdx.x];
  const int hk = blockIdx.y, rep = p.H / p.Hkv;
  const int base = p.cu_seqlens[kb.x], L = p.cu_seqlens[kb.x + 1] - base, k0 = kb.y;
  const int kcol = (p.H + hk) * HD, vcol = (p.H + p.Hkv + hk) * HD;
  const int nqb = (L - k0 + QB - 1) / QB;      // q blocks [k0, L)
  const int nblk = rep * nqb;

  if (threadIdx.x == 0) {
    tma_prefetch(&tmQKV128); tma_prefetch(&tmQKV64); tma_prefetch(&tmDO64);
    mbar_init(&bar_kv, 1);
    for (int i = 0; i < 2; ++i) {
      mbar_init(&full[i], 1); mbar_init(&empty[i], 1); mbar_init(&s_full[i], 1); mbar_init(&ew_done[i], 4);
    }
    mbar_init(&acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
#define tS(b) (tmem + 64 * (b))
#define tP(b) (tmem + 128 + 64 * (b))
  const uint32_t tdV = tmem + 256, tdK = tmem + 384;

  if (warp == 0) {
    // ------------------------------------------------ TMA producer
    if (elect_one()) {
      mbar_expect_tx(&bar_kv, 2 * KV_TILE);
      tma_load_2d(sK, &tmQKV128, &bar_kv, kcol, base + k0);
      tma_load_2d(sK + 16384, &tmQKV128, &bar_kv, kcol + 64, base + k0);
      tma_load_2d(sV, &tmQKV128, &bar_kv, vcol, base + k0);
      tma_load_2d(sV + 16384, &tmQKV128, &bar_kv, vcol + 64, base + k0);
      for (int it = 0; it < nblk; ++it) {
        const int b = it & 1;
        const int h = hk * rep + it / nqb, q0 = k0 + (it % nqb) * QB;
        bw_wait(&empty[b], ((it >> 1) & 1) ^ 1);
        mbar_expect_tx(&full[b], 2 * QB_TILE);
        tma_load_2d(sQ(b), &tmQKV64, &full[b], h * HD, base + q0);
        tma_load_2d(sQ(b) + 8192, &tmQKV64, &full[b], h * HD + 64, base + q0);
        tma_load_2d(sO(b), &tmDO64, &full[b], h * HD, base + q0);
        tma_load_2d(sO(b) + 8192, &tmDO64, &full[b], h * HD + 64, base + q0);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer
    constexpr uint32_t ID_S = umma_idesc_bf16(128, QB, 0);     // [128 kv] x [64 q], K = hd
    constexpr uint32_t ID_ACC = umma_idesc_bf16(128, HD, 1);   // [128 kv] x [128 hd], K = 64 q, B MN-major
    bw_wait(&bar_kv, 0);
    tc_fence_after();
    auto issue_acc = [&](int itp) {  // dV += P^T dO ; dK += dS^T Q   for block itp
      const int bp = itp & 1;
      bw_wait(&ew_done[bp], (itp >> 1) & 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t pa = smem_u32(sP(bp)), sa = smem_u32(sS(bp));
        const uint32_t ob = smem_u32(sO(bp)), qb = smem_u32(sQ(bp));
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
          const uint32_t acc = (itp > 0 || kk > 0) ? 1u : 0u;
          tc_mma_bf16(tdV, umma_desc_sw128(pa + kk * 32, 16, 1024), umma_desc_sw128(ob + kk * 2048, 8192, 1024), ID_ACC, acc);
          tc_mma_bf16(tdK, umma_desc_sw128(sa + kk * 32, 16, 1024), umma_desc_sw128(qb + kk * 2048, 8192, 1024), ID_ACC, acc);
        }
        tc_commit(&empty[bp]);   // frees the Q/dO stage and the P/dS buffer of block itp
      }
      __syncwarp();
    };
    for (int it = 0; it < nblk; ++it) {
      const int b = it & 1;
      bw_wait(&full[b], (it >> 1) & 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t k = smem_u32(sK), v = smem_u32(sV), q = smem_u32(sQ(b)), o = smem_u32(sO(b));
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
          const uint32_t offa = (kk >> 2) * 16384 + (kk & 3) * 32, offb = (kk >> 2) * 8192 + (kk & 3) * 32;
          tc_mma_bf16(tS(b), umma_desc_sw128(k + offa, 16, 1024), umma_desc_sw128(q + offb, 16, 1024), ID_S, kk > 0);
          tc_mma_bf16(tP(b), umma_desc_sw128(v + offa, 16, 1024), umma_desc_sw128(o + offb, 16, 1024), ID_S, kk > 0);
        }
        tc_commit(&s_full[b]);
      }
      __syncwarp();
      if (it > 0) issue_acc(it - 1);
    }
    if (nblk > 0) issue_acc(nblk - 1);
    __syncwarp();
    if (elect_one()) tc_commit(&acc_done);
    __syncwarp();
  } else {
    // ------------------------------------------------ elementwise warps (thread = key row = TMEM lane)
    const int q4 = warp & 3;
    const int r = q4 * 32 + lane;           // key row within the block
    const int kpos = k0 + r;
    const uint32_t lane_off = (uint32_t)(q4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_B;
    for (int it = 0; it < nblk; ++it) {
      const int b = it & 1;
      const int h = hk * rep + it / nqb, q0 = k0 + (it % nqb) * QB;
      bw_wait(&s_full[b], (it >> 1) & 1);
      tc_fence_after();
      __syncwarp();
      float s[64], dp[64];
      tmem_ld64(tS(b) + lane_off, s);
      tmem_ld64(tP(b) + lane_off, dp);
      const float* lse_h = p.lse + (size_t)h * p.T + base;
      const float* D_h = p.D + (size_t)h * p.T + base;
#pragma unroll
      for (int c = 0; c < 64; ++c) {
        const int qpos = q0 + c;
        float pv = 0.f, dsv = 0.f;
        if (qpos < L && kpos <= qpos) {
          pv = exp2f(s[c] * sl2 - __ldg(lse_h + qpos) * LOG2E_B);
          dsv = pv * (dp[c] - __ldg(D_h + qpos)) * p.scale;
        }
        s[c] = pv;
        dp[c] = dsv;
      }
      // the P^T / dS^T buffer b was last read by the dV/dK MMAs of block it-2
      if (it >= 2) bw_wait(&empty[b], ((it - 2) >> 1) & 1);
      st_row64_sw128(sP(b), r, s);
      st_row64_sw128(sS(b), r, dp);
      fence_proxy_async();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&ew_done[b]);
    }
    // ------------------------------------------------ epilogue: dK (RoPE bwd), dV rows -> dqkv
    bw_wait(&acc_done, 0);
    tc_fence_after();
    __syncwarp();
    const bool rok = kpos < L;
    float a0[32], a1[32], a2[32], a3[32];
    tmem_ld32(tdK + lane_off, a0);
    tmem_ld32(tdK + lane_off + 32, a1);
    tmem_ld32(tdK + lane_off + 64, a2);
    tmem_ld32(tdK + lane_off + 96, a3);
    const int ps = rok ? kpos : 0;
    rope_bwd_row(a0, a1, a2, a3, p.rope_cs + (size_t)ps * (HD / 2));
    bf16* krow = p.dqkv + (size_t)(base + ps) * p.ld_dqkv + kcol;
    if (rok) { st_row32_bf16(krow, a0); st_row32_bf16(krow + 32, a1); st_row32_bf16(krow + 64, a2); st_row32_bf16(krow + 96, a3); }
    tmem_ld32(tdV + lane_off, a0);
    tmem_ld32(tdV + lane_off + 32, a1);
    tmem_ld32(tdV + lane_off + 64, a2);
    tmem_ld32(tdV + lane_off + 96, a3);
    bf16* vrow = p.dqkv + (size_t)(base + ps) * p.ld_dqkv + vcol;
    if (rok) { st_row32_bf16(vrow, a0); st_row32_bf16(vrow + 32, a1); st_row32_bf16(vrow + 64, a2); st_row32_bf16(vrow + 96, a3); }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

// ======================================================================================= dQ kernel
constexpr int Q_ROWS = 128, KB = 64;
constexpr int Q_TILE = Q_ROWS * HD * 2;       // 32 KB
constexpr int KB_TILE = KB * HD * 2;          // 16 KB
constexpr int DS_TILE = Q_ROWS * KB * 2;      // 16 KB
constexpr int SMEM_DQ = 2 * Q_TILE + 4 * KB_TILE + 2 * DS_TILE + 1024;   // 161 KB

__global__ void __launch_bounds__(192, 1)
attn_bwd_dq_tc_kernel(const __grid_constant__ CUtensorMap tmQKV128, const __grid_constant__ CUtensorMap tmQKV64,
                      const __grid_constant__ CUtensorMap tmDO128, const TcBwdParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* const sQ1 = smem;
  uint8_t* const sO1 = sQ1 + Q_TILE;
  uint8_t* const sK0 = sO1 + Q_TILE;
  uint8_t* const sV0 = sK0 + 2 * KB_TILE;
  uint8_t* const sS0 = sV0 + 2 * KB_TILE;
#define sK(b) (sK0 + (b) * KB_TILE)
#define sV(b) (sV0 + (b) * KB_TILE)
  __shared__ __align__(8) uint64_t bar_q, full[2], empty[2], s_full[2], ew_done[2], acc_done;
  __shared__ uint32_t tmem_sh;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int2 qb = p.blocks[blockIdx.x];
  const int h = blockIdx.y, hk = h / (p.H / p.Hkv);
  const int base = p.cu_seqlens[qb.x], L = p.cu_seqlens[qb.x + 1] - base, q0 = qb.y;
  const int kcol = (p.H + hk) * HD, vcol = (p.H + p.Hkv + hk) * HD;
  const int nkb = (min(L, q0 + Q_ROWS) + KB - 1) / KB;

  if (threadIdx.x == 0) {
    tma_prefetch(&tmQKV128); tma_prefetch(&tmQKV64); tma_prefetch(&tmDO128);
    mbar_init(&bar_q, 1);
    for (int i = 0; i < 2; ++i) {
      mbar_init(&full[i], 1); mbar_init(&empty[i], 1); mbar_init(&s_full[i], 1); mbar_init(&ew_done[i], 4);
    }
    mbar_init(&acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  const uint32_t tdQ = tmem + 256;

  if (warp == 0) {
    if (elect_one()) {
      mbar_expect_tx(&bar_q, 2 * Q_TILE);
      tma_load_2d(sQ1, &tmQKV128, &bar_q, h * HD, base + q0);
      tma_load_2d(sQ1 + 16384, &tmQKV128, &bar_q, h * HD + 64, base + q0);
      tma_load_2d(sO1, &tmDO128, &bar_q, h * HD, base + q0);
      tma_load_2d(sO1 + 16384, &tmDO128, &bar_q, h * HD + 64, base + q0);
      for (int it = 0; it < nkb; ++it) {
        const int b = it & 1;
        bw_wait(&empty[b], ((it >> 1) & 1) ^ 1);
        mbar_expect_tx(&full[b], 2 * KB_TILE);
        tma_load_2d(sK(b), &tmQKV64, &full[b], kcol, base + it * KB);
        tma_load_2d(sK(b) + 8192, &tmQKV64, &full[b], kcol + 64, base + it * KB);
        tma_load_2d(sV(b), &tmQKV64, &full[b], vcol, base + it * KB);
        tma_load_2d(sV(b) + 8192, &tmQKV64, &full[b], vcol + 64, base + it * KB);
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t ID_S = umma_idesc_bf16(128, KB, 0);     // [128 q] x [64 keys], K = hd
    constexpr uint32_t ID_ACC = umma_idesc_bf16(128, HD, 1);   // [128 q] x [128 hd], K = 64 keys, B MN-major
    bw_wait(&bar_q, 0);
    tc_fence_after();
    auto issue_acc = [&](int itp) {  // dQ += dS K  for key block itp
      const int bp = itp & 1;
      bw_wait(&ew_done[bp], (itp >> 1) & 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t sa = smem_u32(sS(bp)), kb_ = smem_u32(sK(bp));
#pragma unroll
        for (int kk = 0; kk < 4; ++kk)
          tc_mma_bf16(tdQ, umma_desc_sw128(sa + kk * 32, 16, 1024), umma_desc_sw128(kb_ + kk * 2048, 8192, 1024), ID_ACC,
                      (itp > 0 || kk > 0) ? 1u : 0u);
        tc_commit(&empty[bp]);
      }
      __syncwarp();
    };
    for (int it = 0; it < nkb; ++it) {
      const int b = it & 1;
      bw_wait(&full[b], (it >> 1) & 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t q = smem_u32(sQ1), o = smem_u32(sO1), k = smem_u32(sK(b)), v = smem_u32(sV(b));
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
          const uint32_t offa = (kk >> 2) * 16384 + (kk & 3) * 32, offb = (kk >> 2) * 8192 + (kk & 3) * 32;
          tc_mma_bf16(tS(b), umma_desc_sw128(q + offa, 16, 1024), umma_desc_sw128(k + offb, 16, 1024), ID_S, kk > 0);
          tc_mma_bf16(tP(b), umma_desc_sw128(o + offa, 16, 1024), umma_desc_sw128(v + offb, 16, 1024), ID_S, kk > 0);
        }
        tc_commit(&s_full[b]);
      }
      __syncwarp();
      if (it > 0) issue_acc(it - 1);
    }
    if (nkb > 0) issue_acc(nkb - 1);
    __syncwarp();
    if (elect_one()) tc_commit(&acc_done);
    __syncwarp();
  } else {
    const int q4 = warp & 3;
    const int r = q4 * 32 + lane;           // query row
    const int qpos = q0 + r;
    const uint32_t lane_off = (uint32_t)(q4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_B;
    const bool qok = qpos < L;
    const float lse2 = qok ? p.lse[(size_t)h * p.T + base + qpos] * LOG2E_B : 0.f;
    const float Dq = qok ? p.D[(size_t)h * p.T + base + qpos] : 0.f;
    for (int it = 0; it < nkb; ++it) {
      const int b = it & 1;
      bw_wait(&s_full[b], (it >> 1) & 1);
      tc_fence_after();
      __syncwarp();
      float s[64], dp[64];
      tmem_ld64(tS(b) + lane_off, s);
      tmem_ld64(tP(b) + lane_off, dp);
#pragma unroll
      for (int c = 0; c < 64; ++c) {
        const int key = it * KB + c;
        float dsv = 0.f;
        if (qok && key <= qpos) dsv = exp2f(s[c] * sl2 - lse2) * (dp[c] - Dq) * p.scale;
        dp[c] = dsv;
      }
      if (it >= 2) bw_wait(&empty[b], ((it - 2) >> 1) & 1);
      st_row64_sw128(sS(b), r, dp);
      fence_proxy_async();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&ew_done[b]);
    }
    bw_wait(&acc_done, 0);
    tc_fence_after();
    __syncwarp();
    float a0[32], a1[32], a2[32], a3[32];
    tmem_ld32(tdQ + lane_off, a0);
    tmem_ld32(tdQ + lane_off + 32, a1);
    tmem_ld32(tdQ + lane_off + 64, a2);
    tmem_ld32(tdQ + lane_off + 96, a3);
    const int ps = qok ? qpos : 0;
    rope_bwd_row(a0, a1, a2, a3, p.rope_cs + (size_t)ps * (HD / 2));
    bf16* qrow = p.dqkv + (size_t)(base + ps) * p.ld_dqkv + h * HD;
    if (qok) { st_row32_bf16(qrow, a0); st_row32_bf16(qrow + 32, a1); st_row32_bf16(qrow + 64, a2); st_row32_bf16(qrow + 96, a3); }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

}  // namespace

// blocks128: (seq, local start) per 128-row block (key blocks for dK/dV, query blocks for dQ)
int attn_bwd_tc(const AttnArgs& a, const int2* blocks128, int n_blocks128, cudaStream_t st) {
  if (a.hd != HD) return -1;
  if (n_blocks128 <= 0) return 0;
  CUtensorMap mQKV128, mQKV64, mDO64, mDO128;
  if (!tma_map_2d(&mQKV128, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, 128)) return -2;
  if (!tma_map_2d(&mQKV64, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, 64)) return -2;
  if (!tma_map_2d(&mDO64, a.dO, a.T, a.H * HD, a.ld_do, 64, 64)) return -2;
  if (!tma_map_2d(&mDO128, a.dO, a.T, a.H * HD, a.ld_do, 64, 128)) return -2;
  TcBwdParams p;
  p.cu_seqlens = a.cu_seqlens; p.blocks = blocks128; p.lse = a.lse; p.D = a.D; p.dqkv = a.dqkv;
  p.ld_dqkv = a.ld_dqkv; p.rope_cs = a.rope_cs; p.T = a.T; p.H = a.H; p.Hkv = a.Hkv; p.scale = a.scale;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_bwd_dkdv_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_DKDV);
    cudaFuncSetAttribute(attn_bwd_dq_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_DQ);
    attr = true;
  }
  attn_bwd_dkdv_tc_kernel<<<dim3(n_blocks128, a.Hkv), 192, SMEM_DKDV, st>>>(mQKV128, mQKV64, mDO64, p);
  ++g_launch_count;
  attn_bwd_dq_tc_kernel<<<dim3(n_blocks128, a.H), 192, SMEM_DQ, st>>>(mQKV128, mQKV64, mDO128, p);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

}  // namespace menos
