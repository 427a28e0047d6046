// Varlen causal flash-attention FORWARD on the 5th-gen tensor cores (tcgen05 / TMEM / TMA), head_dim 128.
// SURVEY.md §8(a) A3.  Same contract as attn_fwd_kernel (attention.cu): blocks never cross a sequence (so never
// a client), GQA head h -> kv head h / (H/Hkv), LSE saved for the backward.
//
// Design (B200-native): one CTA = 128 query rows of one (sequence, head); thread r of the 4 warps owns query
// row r = TMEM lane r.  Two passes over the causal key blocks (64 keys each):
//   pass 1  S = Q K^T (tcgen05, fp32 in TMEM) -> per-row running max / sum  -> LSE
//   pass 2  S again -> P = exp(S - LSE) (already normalised) -> bf16 in swizzled smem -> O += P V (tcgen05, TMEM)
// so O never needs rescaling (no TMEM read-modify-write); the extra Q K^T costs 1/2 of the forward FLOPs but
// keeps the softmax warps' work per block minimal.  S is double-buffered in TMEM so the next block's Q K^T runs
// while the current block's softmax executes; 112 KB smem and 256 TMEM columns per CTA -> 2 CTAs per SM.
#include <cstdio>
#include "common.cuh"
#include "kernels.h"

namespace menos {
namespace {

constexpr int HD = 128, BQ = 128, BKV = 64;
constexpr int Q_BYTES = BQ * HD * 2;        // 32 KB: 2 swizzle atoms [128][64]
constexpr int K_BYTES = BKV * HD * 2;       // 16 KB: 2 atoms [64][64]
constexpr int V_BYTES = BKV * HD * 2;       // 16 KB: MN-major [2 hd blocks][64 keys][64]
constexpr int P_BYTES = BQ * BKV * 2;       // 16 KB: 1 atom [128][64]
// P_j is written into the K_j stage buffer (free once S_j completed): 97 KB -> 2 CTAs per SM
constexpr int SMEM_FWD = Q_BYTES + 2 * (K_BYTES + V_BYTES) + 1024;
static_assert(P_BYTES == K_BYTES, "P reuses the K stage buffer");
constexpr float LOG2E = 1.4426950408889634f;

struct TcFwdParams {
  const int* cu_seqlens;
  const int2* qblocks;   // (seq, local q start) per 128-row block
  bf16* O; int ld_o;
  float* lse;
  int T, H, Hkv;
  float scale;
};

#ifdef MENOS_ATTN_DEBUG
// watchdog wait: report which barrier never completed instead of hanging
__device__ __forceinline__ void mbar_wait_dbg(uint64_t* bar, uint32_t parity, int id) {
  uint64_t t0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  for (long long it = 0;; ++it) {
    uint32_t ok;
    asm volatile("{\n\t.reg .pred P;\n\tmbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    if (ok) return;
    uint64_t t1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    if (t1 - t0 > 2000000000ull) {
      printf("attn_fwd_tc hang: block (%d,%d) tid %d barrier %d parity %u\n", blockIdx.x, blockIdx.y, threadIdx.x, id,
             parity);
      __trap();
    }
  }
}
#define MBAR_WAIT(b, p) mbar_wait_dbg(b, p, __LINE__)
#else
// spin on test_wait (no suspend hint): these waits are short and on the critical path of every key block
__device__ __forceinline__ void mbar_wait_spin(uint64_t* bar, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile("{\n\t.reg .pred P;\n\tmbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  }
}
#define MBAR_WAIT(b, p) mbar_wait_spin(b, p)
#endif

__global__ void __launch_bounds__(128, 2)
attn_fwd_tc_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmKV,
                   const TcFwdParams p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK[2] = {sQ + Q_BYTES, sQ + Q_BYTES + K_BYTES + V_BYTES};
  uint8_t* sV[2] = {sK[0] + K_BYTES, sK[1] + K_BYTES};
  __shared__ __align__(8) uint64_t bar_q, bar_kv[2], bar_s[2], bar_pv;
  __shared__ uint32_t tmem_sh;

  const int tid = threadIdx.x, warp = tid >> 5;
  const int2 qb = p.qblocks[blockIdx.x];
  const int h = blockIdx.y, hk = h / (p.H / p.Hkv);
  const int base = p.cu_seqlens[qb.x], L = p.cu_seqlens[qb.x + 1] - base, q0 = qb.y;
  const int qcol = h * HD, kcol = (p.H + hk) * HD, vcol = (p.H + p.Hkv + hk) * HD;
  const int nkv = (min(L, q0 + BQ) + BKV - 1) / BKV;

#ifdef MENOS_ATTN_DEBUG
  if (tid == 0 && blockIdx.x == 0 && blockIdx.y == 0) printf("attn_fwd_tc start nkv=%d L=%d\n", nkv, L);
#endif
  if (tid == 0) {
    tma_prefetch(&tmQ); tma_prefetch(&tmKV);
    mbar_init(&bar_q, 1);
    for (int i = 0; i < 2; ++i) { mbar_init(&bar_kv[i], 1); mbar_init(&bar_s[i], 1); }
    mbar_init(&bar_pv, 1);
    fence_barrier_init();
  }
  if (warp == 0) tmem_alloc<256>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
#ifdef MENOS_ATTN_DEBUG
#define DBG(msg) do { if (blockIdx.x == 0 && blockIdx.y == 0 && (threadIdx.x == 0 || threadIdx.x == 33)) printf("tid %d: %s\n", threadIdx.x, msg); } while (0)
#else
#define DBG(msg) do {} while (0)
#endif
  DBG("alloc done");
  const uint32_t tS[2] = {tmem, tmem + 64};
  const uint32_t tO = tmem + 128;
  const uint32_t lane_off = (uint32_t)(warp * 32) << 16;

  constexpr uint32_t IDESC_S = umma_idesc_bf16(128, BKV, 0);
  constexpr uint32_t IDESC_PV = umma_idesc_bf16(128, HD, 1);
  uint32_t ph_kv[2] = {0, 0}, ph_s[2] = {0, 0}, ph_pv = 0;

  // control-thread helpers
  auto load_k = [&](int j, int s) {
    mbar_expect_tx(&bar_kv[s], K_BYTES);
    tma_load_2d(sK[s], &tmKV, &bar_kv[s], kcol, base + j * BKV);
    tma_load_2d(sK[s] + 8192, &tmKV, &bar_kv[s], kcol + 64, base + j * BKV);
  };
  auto load_kv = [&](int j, int s) {
    mbar_expect_tx(&bar_kv[s], K_BYTES + V_BYTES);
    tma_load_2d(sK[s], &tmKV, &bar_kv[s], kcol, base + j * BKV);
    tma_load_2d(sK[s] + 8192, &tmKV, &bar_kv[s], kcol + 64, base + j * BKV);
    tma_load_2d(sV[s], &tmKV, &bar_kv[s], vcol, base + j * BKV);
    tma_load_2d(sV[s] + 8192, &tmKV, &bar_kv[s], vcol + 64, base + j * BKV);
  };
  auto issue_s = [&](int s) {  // S[s] = Q K[s]^T  (M=128, N=64, K=128: 8 x K16)
    const uint32_t q = smem_u32(sQ), k = smem_u32(sK[s]);
#pragma unroll
    for (int kk = 0; kk < 8; ++kk) {
      const uint64_t ad = umma_desc_sw128(q + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024);
      const uint64_t bd = umma_desc_sw128(k + (kk >> 2) * 8192 + (kk & 3) * 32, 16, 1024);
      tc_mma_bf16(tS[s], ad, bd, IDESC_S, kk > 0 ? 1u : 0u);
    }
    tc_commit(&bar_s[s]);
  };

  const int row = tid;                   // query row inside the block (TMEM lane)
  const int qpos = q0 + row;             // position in the sequence
  const float sl2 = p.scale * LOG2E;

  // ---------------- pass 1: row max / sum -> LSE
  if (tid == 0) {
    mbar_expect_tx(&bar_q, Q_BYTES);
    tma_load_2d(sQ, &tmQ, &bar_q, qcol, base + q0);
    tma_load_2d(sQ + 16384, &tmQ, &bar_q, qcol + 64, base + q0);
    load_k(0, 0);
    if (nkv > 1) load_k(1, 1);
    MBAR_WAIT(&bar_q, 0);
    MBAR_WAIT(&bar_kv[0], ph_kv[0]);
    tc_fence_after();
    issue_s(0);
  }
  DBG("pass1 setup done");
  float m = -INFINITY, l = 0.f;
  for (int j = 0; j < nkv; ++j) {
    const int s = j & 1;
    if (tid == 0 && j + 1 < nkv) {     // next block's Q K^T runs during this block's softmax
      MBAR_WAIT(&bar_kv[s ^ 1], ph_kv[s ^ 1]);
      tc_fence_after();
      issue_s(s ^ 1);
    }
    __syncwarp();                      // warp 0 reconverges before the .sync.aligned TMEM loads
    MBAR_WAIT(&bar_s[s], ph_s[s]);
    tc_fence_after();
    float v[64];
    {
      float a[32], b[32];
      tmem_ld32(tS[s] + lane_off, a);
      tmem_ld32(tS[s] + lane_off + 32, b);
#pragma unroll
      for (int c = 0; c < 32; ++c) { v[c] = a[c]; v[32 + c] = b[c]; }
    }
    float mx = -INFINITY;
#pragma unroll
    for (int c = 0; c < 64; ++c) {
      const int kpos = j * BKV + c;
      v[c] = (kpos <= qpos && kpos < L) ? v[c] * sl2 : -INFINITY;
      mx = fmaxf(mx, v[c]);
    }
    const float mn = fmaxf(m, mx);
    float sum = 0.f;
#pragma unroll
    for (int c = 0; c < 64; ++c) sum += exp2f(v[c] - mn);
    l = (m == -INFINITY ? 0.f : l * exp2f(m - mn)) + sum;
    m = mn;
    ph_s[s] ^= 1;
    tc_fence_before();
    __syncthreads();                   // S[s] fully read before it is overwritten by block j+2
    if (tid == 0) {
      ph_kv[s] ^= 1;                   // stage s consumed by S_j (waited above via bar_s)
      if (j + 2 < nkv) load_k(j + 2, s);
    }
  }
  const float lse2 = m + log2f(l);     // log2-domain LSE of this row
  DBG("pass1 done");

  // ---------------- pass 2: P = exp(S - LSE) -> smem -> O += P V
  if (tid == 0) {
    // all pass-1 TMA completions have been waited; reload K and V for block 0 (and 1)
    load_kv(0, 0);
    if (nkv > 1) load_kv(1, 1);
    MBAR_WAIT(&bar_kv[0], ph_kv[0]);
    tc_fence_after();
    issue_s(0);
  }
  for (int j = 0; j < nkv; ++j) {
    const int s = j & 1;
    if (tid == 0 && j + 1 < nkv) {
      MBAR_WAIT(&bar_kv[s ^ 1], ph_kv[s ^ 1]);
      tc_fence_after();
      issue_s(s ^ 1);
    }
    __syncwarp();
    MBAR_WAIT(&bar_s[s], ph_s[s]);
    tc_fence_after();
    float v[64];
    {
      float a[32], b[32];
      tmem_ld32(tS[s] + lane_off, a);
      tmem_ld32(tS[s] + lane_off + 32, b);
#pragma unroll
      for (int c = 0; c < 32; ++c) { v[c] = a[c]; v[32 + c] = b[c]; }
    }
    // previous P V must have consumed sP before it is overwritten
    if (j > 0) { MBAR_WAIT(&bar_pv, ph_pv); ph_pv ^= 1; }
    uint8_t* prow = sK[s] + row * 128;   // P_j overwrites K_j (S_j has completed)
#pragma unroll
    for (int c8 = 0; c8 < 8; ++c8) {
      float e[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int c = c8 * 8 + i;
        const int kpos = j * BKV + c;
        e[i] = (kpos <= qpos && kpos < L) ? exp2f(v[c] * sl2 - lse2) : 0.f;
      }
      uint4 u = make_uint4(pack_bf16x2(e[0], e[1]), pack_bf16x2(e[2], e[3]), pack_bf16x2(e[4], e[5]),
                           pack_bf16x2(e[6], e[7]));
      *reinterpret_cast<uint4*>(prow + ((c8 ^ (row & 7)) << 4)) = u;
    }
    fence_proxy_async();               // generic-proxy smem writes -> visible to the tensor core
    ph_s[s] ^= 1;
    tc_fence_before();
    __syncthreads();
    if (tid == 0) {
      tc_fence_after();
      const uint32_t pa = smem_u32(sK[s]), vb = smem_u32(sV[s]);
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const uint64_t ad = umma_desc_sw128(pa + kk * 32, 16, 1024);
        const uint64_t bd = umma_desc_sw128(vb + kk * 2048, 8192, 1024);
        tc_mma_bf16(tO, ad, bd, IDESC_PV, (j > 0 || kk > 0) ? 1u : 0u);
      }
      tc_commit(&bar_pv);
      ph_kv[s] ^= 1;
      if (j + 2 < nkv) {
        // stage s is free once P V_j (and S_j) completed
        MBAR_WAIT(&bar_pv, ph_pv);
        load_kv(j + 2, s);
      }
    }
    // keep every thread's view of the bar_pv phase in step with the control thread's extra wait above
    if (j + 2 < nkv) { MBAR_WAIT(&bar_pv, ph_pv); }
  }
  DBG("pass2 loop done");
  // the last P V commit
  __syncwarp();
  MBAR_WAIT(&bar_pv, ph_pv);
  tc_fence_after();
  // ---------------- epilogue: O row (normalised already) -> bf16, LSE
  // TMEM loads are warp-collective (.sync.aligned): every lane loads, only rows inside the sequence store
  const bool rok = qpos < L;
  bf16* orow = p.O + (size_t)(base + (rok ? qpos : 0)) * p.ld_o + h * HD;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    float o[32];
    tmem_ld32(tO + lane_off + c * 32, o);
    if (rok) {
      uint4* dst = reinterpret_cast<uint4*>(orow + c * 32);
#pragma unroll
      for (int q = 0; q < 4; ++q)
        dst[q] = make_uint4(pack_bf16x2(o[8 * q], o[8 * q + 1]), pack_bf16x2(o[8 * q + 2], o[8 * q + 3]),
                            pack_bf16x2(o[8 * q + 4], o[8 * q + 5]), pack_bf16x2(o[8 * q + 6], o[8 * q + 7]));
    }
  }
  if (rok) p.lse[(size_t)h * p.T + base + qpos] = lse2 / LOG2E;
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_dealloc<256>(tmem);
  }
}

}  // namespace

bool tma_map_2d(CUtensorMap* out, const void* ptr, uint64_t rows, uint64_t cols, uint64_t ld, uint32_t bc,
                uint32_t br);

// qblocks128: (seq, local q start) per 128-row block
int attn_fwd_tc(const AttnArgs& a, const int2* qblocks128, int n_qblocks128, cudaStream_t st) {
  if (a.hd != HD) return -1;
  if (n_qblocks128 <= 0) return 0;
  CUtensorMap mQ, mKV;
  const int Nqkv = a.ld_qkv;
  if (!tma_map_2d(&mQ, a.qkv, a.T, Nqkv, a.ld_qkv, 64, BQ)) return -2;
  if (!tma_map_2d(&mKV, a.qkv, a.T, Nqkv, a.ld_qkv, 64, BKV)) return -2;
  TcFwdParams p;
  p.cu_seqlens = a.cu_seqlens; p.qblocks = qblocks128; p.O = a.O; p.ld_o = a.ld_o; p.lse = a.lse;
  p.T = a.T; p.H = a.H; p.Hkv = a.Hkv; p.scale = a.scale;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_fwd_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_FWD);
    attr = true;
  }
#ifdef MENOS_ATTN_DEBUG
  fprintf(stderr, "attn_fwd_tc launch grid %d x %d smem %d\n", n_qblocks128, a.H, SMEM_FWD);
#endif
  attn_fwd_tc_kernel<<<dim3(n_qblocks128, a.H), 128, SMEM_FWD, st>>>(mQ, mKV, p);
#ifdef MENOS_ATTN_DEBUG
  fprintf(stderr, "attn_fwd_tc launched: %s\n", cudaGetErrorString(cudaPeekAtLastError()));
#endif
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

}  // namespace menos
