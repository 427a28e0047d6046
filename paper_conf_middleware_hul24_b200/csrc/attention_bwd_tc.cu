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
// Warp roles: warp 0 TMA producer (3-stage ring of the streamed operand), warp 1 MMA issuer (elected lane),
// warps 2-9 elementwise (thread = TMEM lane = row; warpgroup g of them owns half the columns) + epilogue.  The epilogue stages the fp32 accumulator rows in
// shared memory and re-reads them warp-per-row so the RoPE table reads and the bf16 row stores are coalesced.
#include <cstdio>
#include "common.cuh"
#include "kernels.h"

namespace menos {

bool tma_map_2d(CUtensorMap* out, const void* ptr, uint64_t rows, uint64_t cols, uint64_t ld, uint32_t bc,
                uint32_t br);

namespace {

constexpr int HD = 128;
constexpr int STAGES = 3;
constexpr int STG_LD = HD + 1;   // fp32 staging row stride (bank-conflict-free column writes)
constexpr float LOG2E_B = 1.4426950408889634f;

struct TcBwdParams {
  const int* cu_seqlens;
  const int2* blocks;      // dkdv: (seq, k0) per 128-key block; dq: (seq, q0) per 128-query block
  const float* lse;        // [H, T] natural log
  const float* D;          // [H, T]
  bf16* dqkv; int ld_dqkv;
  const float2* rope_cs;   // [max_pos][HD/2] (cos, sin)
  const int* pos_shift;    // [n_seqs] prefix rows before each sequence (extended batch) or nullptr
  int T, H, Hkv;
  float scale;
};

// mbarrier wait with a 2 s watchdog: a pipeline bug traps (launch error) instead of hanging the device
__device__ __forceinline__ void bw_wait(uint64_t* bar, uint32_t parity) {
  uint64_t t0 = 0;
  for (uint32_t n = 0;; ++n) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred P;\n\tmbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}"
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

#ifdef MENOS_BWD_TRACE
__device__ __forceinline__ unsigned long long gtime() { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
#define TRACED() ((blockIdx.x == 0 || blockIdx.x == 36) && (blockIdx.y == 0 || blockIdx.y == 20))
#define TR_DECL const unsigned long long T0 = gtime(); unsigned long long tr_a[8] = {0}, tr_b[8] = {0}, tr_c[4] = {0};
#define TR_A(i) if ((i) < 8) tr_a[i] = gtime() - T0;
#define TR_B(i) if ((i) < 8) tr_b[i] = gtime() - T0;
#define TR_C(i) tr_c[i] = gtime() - T0;
#define TR_PRINT(tag) if (TRACED()) printf("%s %d,%d n %d: a %llu %llu %llu %llu %llu %llu %llu %llu | b %llu %llu %llu %llu %llu %llu %llu %llu | c %llu %llu %llu %llu\n", tag, blockIdx.x, blockIdx.y, nblk, \
  tr_a[0], tr_a[1], tr_a[2], tr_a[3], tr_a[4], tr_a[5], tr_a[6], tr_a[7], tr_b[0], tr_b[1], tr_b[2], tr_b[3], tr_b[4], tr_b[5], tr_b[6], tr_b[7], tr_c[0], tr_c[1], tr_c[2], tr_c[3]);
#else
#define TR_DECL
#define TR_A(i)
#define TR_B(i)
#define TR_C(i)
#define TR_PRINT(tag)
#endif

constexpr int EW_WARPS = 8;                 // two warpgroups: each owns half of the S / dP columns
constexpr int NTHREADS = 64 + 32 * EW_WARPS;

// named barrier over the elementwise warps
__device__ __forceinline__ void ew_sync() { asm volatile("bar.sync 1, %0;" ::"n"(32 * EW_WARPS) : "memory"); }

// long waits of the producer / MMA warps: suspend-capable try_wait so they do not steal issue slots from the
// elementwise warps that share their schedulers
__device__ __forceinline__ void bw_wait_idle(uint64_t* bar, uint32_t parity) {
  uint64_t t0 = 0;
  for (uint32_t n = 0;; ++n) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    if (ok) return;
    if ((n & 15) == 15) {
      uint64_t t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      if (t0 == 0) t0 = t;
      else if (t - t0 > 2000000000ull) __trap();
    }
  }
}

// write columns [32 g, 32 g + 32) (bf16) of one row of a [rows][64] SWIZZLE_128B K-major tile
__device__ __forceinline__ void st_half_row_sw128(uint8_t* tile, int row, int g, const float (&v)[32]) {
  uint8_t* prow = tile + row * 128;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const int c8 = 4 * g + c;
    uint4 u = make_uint4(pack_bf16x2(v[8 * c + 0], v[8 * c + 1]), pack_bf16x2(v[8 * c + 2], v[8 * c + 3]),
                         pack_bf16x2(v[8 * c + 4], v[8 * c + 5]), pack_bf16x2(v[8 * c + 6], v[8 * c + 7]));
    *reinterpret_cast<uint4*>(prow + ((c8 ^ (row & 7)) << 4)) = u;
  }
}

// Epilogue phase A: thread (row r, column half g) moves accumulator columns [64 g, 64 g + 64) to staging row r.
__device__ __forceinline__ void stage_acc(uint32_t tacc, float* stg, int r, int g) {
  float* row = stg + r * STG_LD + 64 * g;
  uint32_t a[32], b[32];
  tmem_ld32_nw(tacc + 64 * g, a);
  tmem_ld32_nw(tacc + 64 * g + 32, b);
  tmem_wait_ld();
#pragma unroll
  for (int i = 0; i < 32; ++i) { row[i] = __uint_as_float(a[i]); row[32 + i] = __uint_as_float(b[i]); }
}

// Epilogue phase B: elementwise warp w8 (0..7) writes staged rows [16 w8, 16 w8 + 16) to dst (bf16), lanes across
// columns (coalesced), 8 rows in flight; with rope, applies the RoPE backward (pairs j, j+64):
// dx_j = dy_j c + dy_{j+64} s, dx_{j+64} = dy_{j+64} c - dy_j s.
__device__ __forceinline__ void store_rows(const float* stg, int w8, int lane, int row0, int n_valid,
                                           bf16* dst, int ld, const float2* cs, bool rope) {
  const int j = 2 * lane;   // this lane: columns j, j+1 and j+64, j+65
#pragma unroll
  for (int half = 0; half < 2; ++half) {
    float4 e[8];
    float a0[8], a1[8], b0[8], b1[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int rr = w8 * 16 + half * 8 + u;
      const float* s = stg + rr * STG_LD;
      a0[u] = s[j]; a1[u] = s[j + 1]; b0[u] = s[64 + j]; b1[u] = s[65 + j];
      if (rope && rr < n_valid) e[u] = *reinterpret_cast<const float4*>(cs + (size_t)max(0, row0 + rr) * (HD / 2) + j);
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int rr = w8 * 16 + half * 8 + u;
      if (rr >= n_valid) continue;
      float x0 = a0[u], x1 = a1[u], y0 = b0[u], y1 = b1[u];
      if (rope) {   // e = (c_j, s_j, c_j+1, s_j+1)
        x0 = a0[u] * e[u].x + b0[u] * e[u].y; y0 = b0[u] * e[u].x - a0[u] * e[u].y;
        x1 = a1[u] * e[u].z + b1[u] * e[u].w; y1 = b1[u] * e[u].z - a1[u] * e[u].w;
      }
      bf16* d = dst + (size_t)rr * ld;
      *reinterpret_cast<uint32_t*>(d + j) = pack_bf16x2(x0, x1);
      *reinterpret_cast<uint32_t*>(d + 64 + j) = pack_bf16x2(y0, y1);
    }
  }
}

// ======================================================================================= dK / dV kernel
constexpr int KV_ROWS = 128, QB = 64;
constexpr int KV_TILE = KV_ROWS * HD * 2;      // 32 KB (2 atoms [128][64])
constexpr int QB_TILE = QB * HD * 2;           // 16 KB (2 atoms [64][64])
constexpr int PT_TILE = KV_ROWS * QB * 2;      // 16 KB (1 atom [128][64])
constexpr int SMEM_DKDV = 2 * KV_TILE + 2 * STAGES * QB_TILE + 4 * PT_TILE + 1024;   // 225 KB
static_assert(2 * KV_ROWS * STG_LD * 4 <= SMEM_DKDV - 1024, "dK/dV staging must fit in the freed buffers");

__global__ void __launch_bounds__(NTHREADS, 1)
attn_bwd_dkdv_tc_kernel(const __grid_constant__ CUtensorMap tmQKV128, const __grid_constant__ CUtensorMap tmQKV64,
                        const __grid_constant__ CUtensorMap tmDO64, const TcBwdParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* const sK = smem;
  uint8_t* const sV = sK + KV_TILE;
  uint8_t* const sQ0 = sV + KV_TILE;                  // Q stages
  uint8_t* const sO0 = sQ0 + STAGES * QB_TILE;        // dO stages
  uint8_t* const sP0 = sO0 + STAGES * QB_TILE;        // P^T  (2 buffers)
  uint8_t* const sS0 = sP0 + 2 * PT_TILE;             // dS^T (2 buffers)
  __shared__ __align__(8) uint64_t bar_kv, full[STAGES], empty[STAGES], s_full[2], ew_done[2], pd_free[2], acc_done;
  __shared__ uint32_t tmem_sh;
  __shared__ __align__(16) float s_lse[2][QB], s_D[2][QB];

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int2 kb = p.blocks[blockIdx.x];
  const int hk = blockIdx.y, rep = p.H / p.Hkv;
  const int base = p.cu_seqlens[kb.x], L = p.cu_seqlens[kb.x + 1] - base, k0 = kb.y;
  const int kcol = (p.H + hk) * HD, vcol = (p.H + p.Hkv + hk) * HD;
  const int nqb = (L - k0 + QB - 1) / QB;      // q blocks [k0, L)
  const int nblk = rep * nqb;

  TR_DECL
  if (threadIdx.x == 0) {
    tma_prefetch(&tmQKV128); tma_prefetch(&tmQKV64); tma_prefetch(&tmDO64);
    mbar_init(&bar_kv, 1);
    for (int i = 0; i < STAGES; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&s_full[i], 1); mbar_init(&ew_done[i], EW_WARPS); mbar_init(&pd_free[i], 1); }
    mbar_init(&acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  const uint32_t tdV = tmem + 256, tdK = tmem + 384;   // S^T buffers at 0/64, dP^T at 128/192

  if (warp == 0) {
    // ------------------------------------------------ TMA producer
    if (elect_one()) {
      mbar_expect_tx(&bar_kv, 2 * KV_TILE);
      tma_load_2d(sK, &tmQKV128, &bar_kv, kcol, base + k0);
      tma_load_2d(sK + 16384, &tmQKV128, &bar_kv, kcol + 64, base + k0);
      tma_load_2d(sV, &tmQKV128, &bar_kv, vcol, base + k0);
      tma_load_2d(sV + 16384, &tmQKV128, &bar_kv, vcol + 64, base + k0);
      for (int it = 0; it < nblk; ++it) {
        const int st = it % STAGES;
        const int h = hk * rep + it / nqb, q0 = k0 + (it % nqb) * QB;
        bw_wait_idle(&empty[st], ((it / STAGES) & 1) ^ 1);
        mbar_expect_tx(&full[st], 2 * QB_TILE);
        uint8_t* q = sQ0 + st * QB_TILE;
        uint8_t* o = sO0 + st * QB_TILE;
        tma_load_2d(q, &tmQKV64, &full[st], h * HD, base + q0);
        tma_load_2d(q + 8192, &tmQKV64, &full[st], h * HD + 64, base + q0);
        tma_load_2d(o, &tmDO64, &full[st], h * HD, base + q0);
        tma_load_2d(o + 8192, &tmDO64, &full[st], h * HD + 64, base + q0);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------ MMA issuer
    constexpr uint32_t ID_S = umma_idesc_bf16(128, QB, 0);     // [128 kv] x [64 q], K = hd
    constexpr uint32_t ID_ACC = umma_idesc_bf16(128, HD, 1);   // [128 kv] x [128 hd], K = 64 q, B MN-major
    bw_wait_idle(&bar_kv, 0);
    TR_C(0)
    tc_fence_after();
    auto issue_acc = [&](int itp) {  // dV += P^T dO ; dK += dS^T Q   for block itp
      const int bp = itp & 1, sp = itp % STAGES;
      bw_wait_idle(&ew_done[bp], (itp >> 1) & 1);
      TR_B(itp)
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t pa = smem_u32(sP0 + bp * PT_TILE), sa = smem_u32(sS0 + bp * PT_TILE);
        const uint32_t ob = smem_u32(sO0 + sp * QB_TILE), qb = smem_u32(sQ0 + sp * QB_TILE);
#pragma unroll
        for (int kk = 0; kk < 4; ++kk) {
          const uint32_t acc = (itp > 0 || kk > 0) ? 1u : 0u;
          tc_mma_bf16(tdV, umma_desc_sw128(pa + kk * 32, 16, 1024), umma_desc_sw128(ob + kk * 2048, 8192, 1024), ID_ACC, acc);
          tc_mma_bf16(tdK, umma_desc_sw128(sa + kk * 32, 16, 1024), umma_desc_sw128(qb + kk * 2048, 8192, 1024), ID_ACC, acc);
        }
        tc_commit(&empty[sp]);     // Q/dO stage free
        tc_commit(&pd_free[bp]);   // P^T/dS^T buffer free
      }
      __syncwarp();
    };
    for (int it = 0; it < nblk; ++it) {
      const int b = it & 1, st = it % STAGES;
      bw_wait_idle(&full[st], (it / STAGES) & 1);
      TR_A(it)
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t k = smem_u32(sK), v = smem_u32(sV);
        const uint32_t q = smem_u32(sQ0 + st * QB_TILE), o = smem_u32(sO0 + st * QB_TILE);
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
          const uint32_t offa = (kk >> 2) * 16384 + (kk & 3) * 32, offb = (kk >> 2) * 8192 + (kk & 3) * 32;
          tc_mma_bf16(tmem + 64 * b, umma_desc_sw128(k + offa, 16, 1024), umma_desc_sw128(q + offb, 16, 1024), ID_S, kk > 0);
          tc_mma_bf16(tmem + 128 + 64 * b, umma_desc_sw128(v + offa, 16, 1024), umma_desc_sw128(o + offb, 16, 1024), ID_S, kk > 0);
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
    TR_C(1)
    if (lane == 0) { TR_PRINT("MMA") }
  } else {
    // ------------------------------------------------ elementwise warps (thread = key row = TMEM lane;
    //                                                  warpgroup g owns query columns [32 g, 32 g + 32))
    const int w4 = warp & 3, w8 = warp - 2, g = w8 >> 2, t = threadIdx.x - 64;
    const int r = w4 * 32 + lane;           // key row within the block
    const int kpos = k0 + r;
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_B;
    for (int it = 0; it < nblk; ++it) {
      const int b = it & 1;
      const int h = hk * rep + it / nqb, q0 = k0 + (it % nqb) * QB;
      if (t < 2 * QB) {  // stage lse (log2 domain) and D of the block's 64 queries
        const int c = t & (QB - 1), qpos = q0 + c;
        const float* src = (t < QB ? p.lse : p.D) + (size_t)h * p.T + base + qpos;
        const float v = qpos < L ? __ldg(src) : 0.f;
        if (t < QB) s_lse[b][c] = v * LOG2E_B; else s_D[b][c] = v;
      }
      ew_sync();
      bw_wait(&s_full[b], (it >> 1) & 1);
      TR_A(it)
      tc_fence_after();
      __syncwarp();
      uint32_t su[32], du[32];
      tmem_ld32_nw(tmem + 64 * b + 32 * g + lane_off, su);
      tmem_ld32_nw(tmem + 128 + 64 * b + 32 * g + lane_off, du);
      tmem_wait_ld();
      const int cmin = kpos - q0 - 32 * g;   // P = 0 for queries before the key (causal) ...
      const int cmax = L - q0 - 32 * g;      // ... and past the end of the sequence
      float pv[32], dsv[32];
#pragma unroll
      for (int c4 = 0; c4 < 32; c4 += 4) {
        const float4 lz = *reinterpret_cast<const float4*>(&s_lse[b][32 * g + c4]);
        const float4 dz = *reinterpret_cast<const float4*>(&s_D[b][32 * g + c4]);
        const float lzv[4] = {lz.x, lz.y, lz.z, lz.w}, dzv[4] = {dz.x, dz.y, dz.z, dz.w};
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int c = c4 + u;
          const bool ok = c >= cmin && c < cmax;
          const float x = fmaf(__uint_as_float(su[c]), sl2, -lzv[u]);
          const float e = u == 3 ? poly_exp2(x) : fast_exp2(x);   // a quarter on the FMA pipe (SFU-bound loop)
          pv[c] = ok ? e : 0.f;
          dsv[c] = ok ? e * (__uint_as_float(du[c]) - dzv[u]) * p.scale : 0.f;
        }
      }
      if (it >= 2) bw_wait(&pd_free[b], ((it - 2) >> 1) & 1);
      st_half_row_sw128(sP0 + b * PT_TILE, r, g, pv);
      st_half_row_sw128(sS0 + b * PT_TILE, r, g, dsv);
      fence_proxy_async();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&ew_done[b]);
      TR_B(it)
    }
    TR_C(0)
    // ------------------------------------------------ epilogue: dK (RoPE bwd), dV rows -> dqkv
    bw_wait(&acc_done, 0);
    TR_C(1)
    tc_fence_after();
    __syncwarp();
    float* stgK = reinterpret_cast<float*>(smem);            // every MMA has completed: all buffers are free
    float* stgV = stgK + KV_ROWS * STG_LD;
    stage_acc(tdK + lane_off, stgK, r, g);
    stage_acc(tdV + lane_off, stgV, r, g);
    ew_sync();
    TR_C(2)
    const int nv = min(KV_ROWS, L - k0);
    store_rows(stgK, w8, lane, k0 - (p.pos_shift ? p.pos_shift[kb.x] : 0), nv,
               p.dqkv + (size_t)(base + k0) * p.ld_dqkv + kcol, p.ld_dqkv, p.rope_cs, p.rope_cs != nullptr);
    store_rows(stgV, w8, lane, k0, nv, p.dqkv + (size_t)(base + k0) * p.ld_dqkv + vcol, p.ld_dqkv, p.rope_cs, false);
    TR_C(3)
    if (threadIdx.x == 64) { TR_PRINT("EW") }
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
constexpr int SMEM_DQ = 2 * Q_TILE + 2 * STAGES * KB_TILE + 2 * DS_TILE + 1024;   // 193 KB
static_assert(Q_ROWS * STG_LD * 4 <= SMEM_DQ - 1024, "dQ staging must fit in the freed buffers");

__global__ void __launch_bounds__(NTHREADS, 1)
attn_bwd_dq_tc_kernel(const __grid_constant__ CUtensorMap tmQKV128, const __grid_constant__ CUtensorMap tmQKV64,
                      const __grid_constant__ CUtensorMap tmDO128, const TcBwdParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* const sQ = smem;
  uint8_t* const sO = sQ + Q_TILE;
  uint8_t* const sK0 = sO + Q_TILE;                  // K stages
  uint8_t* const sV0 = sK0 + STAGES * KB_TILE;       // V stages
  uint8_t* const sS0 = sV0 + STAGES * KB_TILE;       // dS (2 buffers)
  __shared__ __align__(8) uint64_t bar_q, full[STAGES], empty[STAGES], s_full[2], ew_done[2], pd_free[2], acc_done;
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
    for (int i = 0; i < STAGES; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&s_full[i], 1); mbar_init(&ew_done[i], EW_WARPS); mbar_init(&pd_free[i], 1); }
    mbar_init(&acc_done, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  const uint32_t tdQ = tmem + 256;   // S buffers at 0/64, dP at 128/192

  if (warp == 0) {
    if (elect_one()) {
      mbar_expect_tx(&bar_q, 2 * Q_TILE);
      tma_load_2d(sQ, &tmQKV128, &bar_q, h * HD, base + q0);
      tma_load_2d(sQ + 16384, &tmQKV128, &bar_q, h * HD + 64, base + q0);
      tma_load_2d(sO, &tmDO128, &bar_q, h * HD, base + q0);
      tma_load_2d(sO + 16384, &tmDO128, &bar_q, h * HD + 64, base + q0);
      for (int it = 0; it < nkb; ++it) {
        const int st = it % STAGES;
        bw_wait_idle(&empty[st], ((it / STAGES) & 1) ^ 1);
        mbar_expect_tx(&full[st], 2 * KB_TILE);
        uint8_t* k = sK0 + st * KB_TILE;
        uint8_t* v = sV0 + st * KB_TILE;
        tma_load_2d(k, &tmQKV64, &full[st], kcol, base + it * KB);
        tma_load_2d(k + 8192, &tmQKV64, &full[st], kcol + 64, base + it * KB);
        tma_load_2d(v, &tmQKV64, &full[st], vcol, base + it * KB);
        tma_load_2d(v + 8192, &tmQKV64, &full[st], vcol + 64, base + it * KB);
      }
    }
  } else if (warp == 1) {
    constexpr uint32_t ID_S = umma_idesc_bf16(128, KB, 0);     // [128 q] x [64 keys], K = hd
    constexpr uint32_t ID_ACC = umma_idesc_bf16(128, HD, 1);   // [128 q] x [128 hd], K = 64 keys, B MN-major
    bw_wait_idle(&bar_q, 0);
    tc_fence_after();
    auto issue_acc = [&](int itp) {  // dQ += dS K  for key block itp
      const int bp = itp & 1, sp = itp % STAGES;
      bw_wait_idle(&ew_done[bp], (itp >> 1) & 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t sa = smem_u32(sS0 + bp * DS_TILE), kb_ = smem_u32(sK0 + sp * KB_TILE);
#pragma unroll
        for (int kk = 0; kk < 4; ++kk)
          tc_mma_bf16(tdQ, umma_desc_sw128(sa + kk * 32, 16, 1024), umma_desc_sw128(kb_ + kk * 2048, 8192, 1024), ID_ACC,
                      (itp > 0 || kk > 0) ? 1u : 0u);
        tc_commit(&empty[sp]);
        tc_commit(&pd_free[bp]);
      }
      __syncwarp();
    };
    for (int it = 0; it < nkb; ++it) {
      const int b = it & 1, st = it % STAGES;
      bw_wait_idle(&full[st], (it / STAGES) & 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t q = smem_u32(sQ), o = smem_u32(sO);
        const uint32_t k = smem_u32(sK0 + st * KB_TILE), v = smem_u32(sV0 + st * KB_TILE);
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) {
          const uint32_t offa = (kk >> 2) * 16384 + (kk & 3) * 32, offb = (kk >> 2) * 8192 + (kk & 3) * 32;
          tc_mma_bf16(tmem + 64 * b, umma_desc_sw128(q + offa, 16, 1024), umma_desc_sw128(k + offb, 16, 1024), ID_S, kk > 0);
          tc_mma_bf16(tmem + 128 + 64 * b, umma_desc_sw128(o + offa, 16, 1024), umma_desc_sw128(v + offb, 16, 1024), ID_S, kk > 0);
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
    const int w4 = warp & 3, w8 = warp - 2, g = w8 >> 2;   // warpgroup g owns key columns [32 g, 32 g + 32)
    const int r = w4 * 32 + lane;           // query row
    const int qpos = q0 + r;
    const uint32_t lane_off = (uint32_t)(w4 * 32) << 16;
    const float sl2 = p.scale * LOG2E_B;
    const bool qok = qpos < L;
    const float lse2 = qok ? p.lse[(size_t)h * p.T + base + qpos] * LOG2E_B : 0.f;
    const float Dq = qok ? p.D[(size_t)h * p.T + base + qpos] : 0.f;
    for (int it = 0; it < nkb; ++it) {
      const int b = it & 1;
      bw_wait(&s_full[b], (it >> 1) & 1);
      tc_fence_after();
      __syncwarp();
      uint32_t su[32], du[32];
      tmem_ld32_nw(tmem + 64 * b + 32 * g + lane_off, su);
      tmem_ld32_nw(tmem + 128 + 64 * b + 32 * g + lane_off, du);
      tmem_wait_ld();
      const int cmax = qok ? qpos - it * KB - 32 * g : -1;   // keys <= query
      float dsv[32];
#pragma unroll
      for (int c = 0; c < 32; ++c) {
        const float x = fmaf(__uint_as_float(su[c]), sl2, -lse2);
        const float e = (c & 3) == 3 ? poly_exp2(x) : fast_exp2(x);   // a quarter on the FMA pipe
        const float v = e * (__uint_as_float(du[c]) - Dq) * p.scale;
        dsv[c] = c <= cmax ? v : 0.f;
      }
      if (it >= 2) bw_wait(&pd_free[b], ((it - 2) >> 1) & 1);
      st_half_row_sw128(sS0 + b * DS_TILE, r, g, dsv);
      fence_proxy_async();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&ew_done[b]);
    }
    bw_wait(&acc_done, 0);
    tc_fence_after();
    __syncwarp();
    float* stg = reinterpret_cast<float*>(smem);
    stage_acc(tdQ + lane_off, stg, r, g);
    ew_sync();
    const int nv = min(Q_ROWS, L - q0);
    store_rows(stg, w8, lane, q0 - (p.pos_shift ? p.pos_shift[qb.x] : 0), nv,
               p.dqkv + (size_t)(base + q0) * p.ld_dqkv + h * HD, p.ld_dqkv, p.rope_cs, p.rope_cs != nullptr);
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
  p.ld_dqkv = a.ld_dqkv; p.rope_cs = a.rope_cs; p.pos_shift = a.pos_shift; p.T = a.T; p.H = a.H; p.Hkv = a.Hkv;
  p.scale = a.scale;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_bwd_dkdv_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_DKDV);
    cudaFuncSetAttribute(attn_bwd_dq_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_DQ);
    attr = true;
  }
  attn_bwd_dkdv_tc_kernel<<<dim3(n_blocks128, a.Hkv), NTHREADS, SMEM_DKDV, st>>>(mQKV128, mQKV64, mDO64, p);
  ++g_launch_count;
  attn_bwd_dq_tc_kernel<<<dim3(n_blocks128, a.H), NTHREADS, SMEM_DQ, st>>>(mQKV128, mQKV64, mDO128, p);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

}  // namespace menos
