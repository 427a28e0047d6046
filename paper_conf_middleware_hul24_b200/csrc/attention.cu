// Varlen causal flash attention, forward and backward.
//
// Sequences are packed token-major; cu_seqlens bounds every q/kv block to ONE sequence of ONE client, so
// attention never mixes clients' (or sequences') tokens -- the batched pass equals each client alone
// (PAPER.md:428).  Causal, GQA (head h -> kv head h / (H/Hkv)), online softmax in fp32, LSE saved.
// Backward is deterministic: one kernel owns dK/dV per kv block (loop over q), another owns dQ per q block
// (loop over kv); both recompute P from the saved LSE.  RoPE backward is applied to dq/dk in registers
// before the store, so dqkv holds gradients w.r.t. the pre-RoPE projections.
// Tensor-core path: mma.sync m16n8k16 (bf16 -> fp32) with ldmatrix from XOR-swizzled smem.
#include "common.cuh"
#include "kernels.h"

namespace menos {
namespace {

constexpr float LOG2E = 1.4426950408889634f;

template <int HD>
__device__ __forceinline__ int swz(int row, int chunk) {
  constexpr int NCH = HD / 8;
  constexpr int MSK = NCH - 1 < 7 ? NCH - 1 : 7;
  return row * HD + ((chunk ^ (row & MSK)) << 3);
}

// cp.async a [ROWS x HD] tile: rows [r0, r0+ROWS) of a sequence starting at token `base` with length L,
// columns [col0, col0+HD) of a row-major matrix with leading dim ld.  Rows outside the sequence are zeroed.
template <int HD, int ROWS, int NT>
__device__ __forceinline__ void load_tile(bf16* s, const bf16* g, int ld, int base, int r0, int L, int col0) {
  constexpr int NCH = HD / 8;
  for (int i = threadIdx.x; i < ROWS * NCH; i += NT) {
    const int r = i / NCH, c = i % NCH;
    const int lr = r0 + r;
    const bool ok = lr < L;
    const bf16* src = g + (size_t)(ok ? base + lr : base) * ld + col0 + c * 8;
    cp_async16(smem_u32(s + swz<HD>(r, c)), src, ok ? 16 : 0);
  }
}

// A fragment (16 x 16) from row-major smem tile rows [r0, r0+16), cols [k0, k0+16)
template <int HD>
__device__ __forceinline__ void ld_a(const bf16* s, int r0, int k0, uint32_t (&a)[4]) {
  const int l = threadIdx.x & 31, mat = l >> 3, r = l & 7;
  const int row = r0 + (mat & 1) * 8 + r, col = k0 + (mat >> 1) * 8;
  ldsm_x4(smem_u32(s + swz<HD>(row, col >> 3)), a[0], a[1], a[2], a[3]);
}
// B fragments for n-tiles (n0, n0+8) x k16 at k0, from smem stored [n][k] (k contiguous): non-trans
template <int HD>
__device__ __forceinline__ void ld_b_nk(const bf16* s, int n0, int k0, uint32_t& b0, uint32_t& b1, uint32_t& b2,
                                        uint32_t& b3) {
  const int l = threadIdx.x & 31, mat = l >> 3, r = l & 7;
  const int row = n0 + (mat >> 1) * 8 + r, col = k0 + (mat & 1) * 8;
  ldsm_x4(smem_u32(s + swz<HD>(row, col >> 3)), b0, b1, b2, b3);
}
// B fragments for n-tiles (n0, n0+8) x k16 at k0, from smem stored [k][n] (n contiguous): trans
template <int HD>
__device__ __forceinline__ void ld_b_kn(const bf16* s, int k0, int n0, uint32_t& b0, uint32_t& b1, uint32_t& b2,
                                        uint32_t& b3) {
  const int l = threadIdx.x & 31, mat = l >> 3, r = l & 7;
  const int row = k0 + (mat & 1) * 8 + r, col = n0 + (mat >> 1) * 8;
  ldsm_x4_t(smem_u32(s + swz<HD>(row, col >> 3)), b0, b1, b2, b3);
}

// ======================================================================== forward
template <int HD>
__global__ void __launch_bounds__(128) attn_fwd_kernel(const AttnArgs a) {
  constexpr int BQ = 64, BKV = 64, NKS = HD / 16, NON = HD / 8;
  extern __shared__ __align__(128) uint8_t sm[];
  bf16* Qs = reinterpret_cast<bf16*>(sm);
  bf16* Ks = Qs + BQ * HD;             // [2][BKV*HD]
  bf16* Vs = Ks + 2 * BKV * HD;        // [2][BKV*HD]

  const int2 qb = a.qblocks[blockIdx.x];
  const int h = blockIdx.y, hk = h / (a.H / a.Hkv);
  const int base = a.cu_seqlens[qb.x], L = a.cu_seqlens[qb.x + 1] - base, q0 = qb.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int kcol = (a.H + hk) * HD, vcol = (a.H + a.Hkv + hk) * HD;

  load_tile<HD, BQ, 128>(Qs, a.qkv, a.ld_qkv, base, q0, L, h * HD);
  cp_async_commit();
  const int kv_end = min(L, q0 + BQ);
  const int nkv = (kv_end + BKV - 1) / BKV;
  load_tile<HD, BKV, 128>(Ks, a.qkv, a.ld_qkv, base, 0, L, kcol);
  load_tile<HD, BKV, 128>(Vs, a.qkv, a.ld_qkv, base, 0, L, vcol);
  cp_async_commit();
  cp_async_wait<1>();
  __syncthreads();
  uint32_t qf[NKS][4];
#pragma unroll
  for (int ks = 0; ks < NKS; ++ks) ld_a<HD>(Qs, warp * 16, ks * 16, qf[ks]);

  float o[NON][4];
#pragma unroll
  for (int i = 0; i < NON; ++i) o[i][0] = o[i][1] = o[i][2] = o[i][3] = 0.f;
  float mrow[2] = {-INFINITY, -INFINITY}, lrow[2] = {0.f, 0.f};
  const float sl2 = a.scale * LOG2E;
  const int qr0 = q0 + warp * 16 + g;  // local row of c[0], c[1]; +8 for c[2], c[3]

  for (int j = 0; j < nkv; ++j) {
    if (j + 1 < nkv) {
      load_tile<HD, BKV, 128>(Ks + ((j + 1) & 1) * BKV * HD, a.qkv, a.ld_qkv, base, (j + 1) * BKV, L, kcol);
      load_tile<HD, BKV, 128>(Vs + ((j + 1) & 1) * BKV * HD, a.qkv, a.ld_qkv, base, (j + 1) * BKV, L, vcol);
      cp_async_commit();
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    const bf16* Kb = Ks + (j & 1) * BKV * HD;
    const bf16* Vb = Vs + (j & 1) * BKV * HD;
    float s[8][4];
#pragma unroll
    for (int i = 0; i < 8; ++i) s[i][0] = s[i][1] = s[i][2] = s[i][3] = 0.f;
#pragma unroll
    for (int ks = 0; ks < NKS; ++ks)
#pragma unroll
      for (int nt = 0; nt < 8; nt += 2) {
        uint32_t b0, b1, b2, b3;
        ld_b_nk<HD>(Kb, nt * 8, ks * 16, b0, b1, b2, b3);
        mma_bf16_16816(s[nt], qf[ks], b0, b1);
        mma_bf16_16816(s[nt + 1], qf[ks], b2, b3);
      }
    // scale, causal + sequence-end mask, online softmax (log2 domain)
    float mx[2] = {-INFINITY, -INFINITY};
#pragma unroll
    for (int nt = 0; nt < 8; ++nt)
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int key = j * BKV + nt * 8 + 2 * t + (e & 1);
        const int qr = qr0 + (e >> 1) * 8;
        float v = s[nt][e] * sl2;
        if (key > qr || key >= L) v = -INFINITY;
        s[nt][e] = v;
        mx[e >> 1] = fmaxf(mx[e >> 1], v);
      }
    float alpha[2];
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], 1));
      mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], 2));
      const float mn = fmaxf(mrow[r], mx[r]);
      alpha[r] = (mrow[r] == -INFINITY) ? 0.f : exp2f(mrow[r] - mn);
      mrow[r] = mn;
      lrow[r] *= alpha[r];
    }
#pragma unroll
    for (int nt = 0; nt < 8; ++nt)
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float m = mrow[e >> 1];
        const float p = (s[nt][e] == -INFINITY) ? 0.f : exp2f(s[nt][e] - m);
        s[nt][e] = p;
        lrow[e >> 1] += p;
      }
#pragma unroll
    for (int i = 0; i < NON; ++i) {
      o[i][0] *= alpha[0]; o[i][1] *= alpha[0]; o[i][2] *= alpha[1]; o[i][3] *= alpha[1];
    }
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      uint32_t pa[4];
      pa[0] = pack_bf16x2(s[2 * kk][0], s[2 * kk][1]);
      pa[1] = pack_bf16x2(s[2 * kk][2], s[2 * kk][3]);
      pa[2] = pack_bf16x2(s[2 * kk + 1][0], s[2 * kk + 1][1]);
      pa[3] = pack_bf16x2(s[2 * kk + 1][2], s[2 * kk + 1][3]);
#pragma unroll
      for (int nt = 0; nt < NON; nt += 2) {
        uint32_t b0, b1, b2, b3;
        ld_b_kn<HD>(Vb, kk * 16, nt * 8, b0, b1, b2, b3);
        mma_bf16_16816(o[nt], pa, b0, b1);
        mma_bf16_16816(o[nt + 1], pa, b2, b3);
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    lrow[r] += __shfl_xor_sync(0xffffffffu, lrow[r], 1);
    lrow[r] += __shfl_xor_sync(0xffffffffu, lrow[r], 2);
  }
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int qr = qr0 + r * 8;
    if (qr >= L) continue;
    const float inv = 1.f / lrow[r];
    bf16* orow = a.O + (size_t)(base + qr) * a.ld_o + h * HD;
#pragma unroll
    for (int nt = 0; nt < NON; ++nt)
      *reinterpret_cast<uint32_t*>(orow + nt * 8 + 2 * t) = pack_bf16x2(o[nt][2 * r] * inv, o[nt][2 * r + 1] * inv);
    if (t == 0) a.lse[(size_t)h * a.T + base + qr] = (mrow[r] + log2f(lrow[r])) / LOG2E;
  }
}

// RoPE backward on a per-thread accumulator fragment set (cols nt*8 + 2t + e); partner n-tile = nt + HD/16
template <int HD>
__device__ __forceinline__ void rope_bwd_frag(float (&acc)[HD / 8][4], const float2* cs, int pos0, int pos1) {
  constexpr int HALF = HD / 2, PN = HD / 16;
  const int t = (threadIdx.x & 31) & 3;
#pragma unroll
  for (int nt = 0; nt < PN; ++nt)
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int j = nt * 8 + 2 * t + (e & 1);   // < HALF
      const int p = (e >> 1) ? pos1 : pos0;
      const float2 c = cs[(size_t)p * HALF + j];
      const float y1 = acc[nt][e], y2 = acc[nt + PN][e];
      acc[nt][e] = y1 * c.x + y2 * c.y;          // dx_j      = dy_j c + dy_{j+h} s
      acc[nt + PN][e] = y2 * c.x - y1 * c.y;     // dx_{j+h}  = dy_{j+h} c - dy_j s
    }
}

// ======================================================================== backward: dK, dV per kv block
template <int HD>
__global__ void __launch_bounds__(128) attn_bwd_dkdv_kernel(const AttnArgs a) {
  constexpr int BKV = 64, BQ = 32, NKS = HD / 16, NON = HD / 8;
  extern __shared__ __align__(128) uint8_t sm[];
  bf16* Ks = reinterpret_cast<bf16*>(sm);
  bf16* Vs = Ks + BKV * HD;
  bf16* Qs = Vs + BKV * HD;           // [2][BQ*HD]
  bf16* dOs = Qs + 2 * BQ * HD;       // [2][BQ*HD]
  float* lses = reinterpret_cast<float*>(dOs + 2 * BQ * HD);  // [2][BQ]
  float* Ds = lses + 2 * BQ;                                   // [2][BQ]

  const int2 kb = a.kvblocks[blockIdx.x];
  const int hk = blockIdx.y, rep = a.H / a.Hkv;
  const int base = a.cu_seqlens[kb.x], L = a.cu_seqlens[kb.x + 1] - base, k0 = kb.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int kcol = (a.H + hk) * HD, vcol = (a.H + a.Hkv + hk) * HD;
  const float sl2 = a.scale * LOG2E;

  load_tile<HD, BKV, 128>(Ks, a.qkv, a.ld_qkv, base, k0, L, kcol);
  load_tile<HD, BKV, 128>(Vs, a.qkv, a.ld_qkv, base, k0, L, vcol);
  cp_async_commit();

  float dk[NON][4], dv[NON][4];
#pragma unroll
  for (int i = 0; i < NON; ++i)
#pragma unroll
    for (int e = 0; e < 4; ++e) dk[i][e] = dv[i][e] = 0.f;

  const int nqb = (L - k0 + BQ - 1) / BQ;      // q blocks [k0, L)
  const int total = rep * nqb;
  auto issue = [&](int it, int buf) {
    const int hh = hk * rep + it / nqb, qs = k0 + (it % nqb) * BQ;
    load_tile<HD, BQ, 128>(Qs + buf * BQ * HD, a.qkv, a.ld_qkv, base, qs, L, hh * HD);
    load_tile<HD, BQ, 128>(dOs + buf * BQ * HD, a.dO, a.ld_do, base, qs, L, hh * HD);
    if (threadIdx.x < BQ) {
      const int r = qs + threadIdx.x;
      const bool ok = r < L;
      lses[buf * BQ + threadIdx.x] = ok ? a.lse[(size_t)hh * a.T + base + r] * LOG2E : 0.f;
      Ds[buf * BQ + threadIdx.x] = ok ? a.D[(size_t)hh * a.T + base + r] : 0.f;
    }
  };
  if (total > 0) issue(0, 0);
  cp_async_commit();
  const int kr0 = k0 + warp * 16 + g;   // local kv row of c[0], c[1]; +8 for c[2], c[3]

  for (int it = 0; it < total; ++it) {
    const int buf = it & 1;
    if (it + 1 < total) {
      issue(it + 1, buf ^ 1);
      cp_async_commit();
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    const int qs = k0 + (it % nqb) * BQ;
    const bf16* Qb = Qs + buf * BQ * HD;
    const bf16* dOb = dOs + buf * BQ * HD;
    // S^T = K Q^T  (rows: kv, cols: q)
    float s[4][4], dp[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int e = 0; e < 4; ++e) s[i][e] = dp[i][e] = 0.f;
#pragma unroll
    for (int ks = 0; ks < NKS; ++ks) {
      uint32_t kf[4], vf[4];
      ld_a<HD>(Ks, warp * 16, ks * 16, kf);
      ld_a<HD>(Vs, warp * 16, ks * 16, vf);
#pragma unroll
      for (int nt = 0; nt < 4; nt += 2) {
        uint32_t b0, b1, b2, b3;
        ld_b_nk<HD>(Qb, nt * 8, ks * 16, b0, b1, b2, b3);
        mma_bf16_16816(s[nt], kf, b0, b1);
        mma_bf16_16816(s[nt + 1], kf, b2, b3);
        ld_b_nk<HD>(dOb, nt * 8, ks * 16, b0, b1, b2, b3);
        mma_bf16_16816(dp[nt], vf, b0, b1);
        mma_bf16_16816(dp[nt + 1], vf, b2, b3);
      }
    }
    // P^T and dS^T
#pragma unroll
    for (int nt = 0; nt < 4; ++nt)
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int qc = nt * 8 + 2 * t + (e & 1);     // col within q block
        const int qr = qs + qc;
        const int kr = kr0 + (e >> 1) * 8;
        float p = 0.f;
        if (qr < L && kr <= qr && kr < L) p = exp2f(s[nt][e] * sl2 - lses[buf * BQ + qc]);
        s[nt][e] = p;
        dp[nt][e] = p * (dp[nt][e] - Ds[buf * BQ + qc]);
      }
    // dV += P^T dO ; dK += dS^T Q   (k dimension = q rows of the block: 2 steps of 16)
#pragma unroll
    for (int kk = 0; kk < 2; ++kk) {
      uint32_t pa[4], da[4];
      pa[0] = pack_bf16x2(s[2 * kk][0], s[2 * kk][1]);
      pa[1] = pack_bf16x2(s[2 * kk][2], s[2 * kk][3]);
      pa[2] = pack_bf16x2(s[2 * kk + 1][0], s[2 * kk + 1][1]);
      pa[3] = pack_bf16x2(s[2 * kk + 1][2], s[2 * kk + 1][3]);
      da[0] = pack_bf16x2(dp[2 * kk][0], dp[2 * kk][1]);
      da[1] = pack_bf16x2(dp[2 * kk][2], dp[2 * kk][3]);
      da[2] = pack_bf16x2(dp[2 * kk + 1][0], dp[2 * kk + 1][1]);
      da[3] = pack_bf16x2(dp[2 * kk + 1][2], dp[2 * kk + 1][3]);
#pragma unroll
      for (int nt = 0; nt < NON; nt += 2) {
        uint32_t b0, b1, b2, b3;
        ld_b_kn<HD>(dOb, kk * 16, nt * 8, b0, b1, b2, b3);
        mma_bf16_16816(dv[nt], pa, b0, b1);
        mma_bf16_16816(dv[nt + 1], pa, b2, b3);
        ld_b_kn<HD>(Qb, kk * 16, nt * 8, b0, b1, b2, b3);
        mma_bf16_16816(dk[nt], da, b0, b1);
        mma_bf16_16816(dk[nt + 1], da, b2, b3);
      }
    }
    __syncthreads();
  }
  if (total == 0) { cp_async_wait<0>(); }
#pragma unroll
  for (int i = 0; i < NON; ++i)
#pragma unroll
    for (int e = 0; e < 4; ++e) dk[i][e] *= a.scale;
  const int sh = a.pos_shift ? a.pos_shift[kb.x] : 0;   // prefix rows of an extended batch: position < 0 -> identity
  const int p0 = min(kr0, L - 1) - sh, p1 = min(kr0 + 8, L - 1) - sh;
  if (a.rope_cs) rope_bwd_frag<HD>(dk, a.rope_cs, p0 < 0 ? 0 : p0, p1 < 0 ? 0 : p1);   // none for OPT
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int kr = kr0 + r * 8;
    if (kr >= L) continue;
    bf16* krow = a.dqkv + (size_t)(base + kr) * a.ld_dqkv + kcol;
    bf16* vrow = a.dqkv + (size_t)(base + kr) * a.ld_dqkv + vcol;
#pragma unroll
    for (int nt = 0; nt < NON; ++nt) {
      *reinterpret_cast<uint32_t*>(krow + nt * 8 + 2 * t) = pack_bf16x2(dk[nt][2 * r], dk[nt][2 * r + 1]);
      *reinterpret_cast<uint32_t*>(vrow + nt * 8 + 2 * t) = pack_bf16x2(dv[nt][2 * r], dv[nt][2 * r + 1]);
    }
  }
}

// ======================================================================== backward: dQ per q block
template <int HD>
__global__ void __launch_bounds__(128) attn_bwd_dq_kernel(const AttnArgs a) {
  constexpr int BQ = 64, BKV = 32, NKS = HD / 16, NON = HD / 8;
  extern __shared__ __align__(128) uint8_t sm[];
  bf16* Qs = reinterpret_cast<bf16*>(sm);
  bf16* dOs = Qs + BQ * HD;
  bf16* Ks = dOs + BQ * HD;            // [2][BKV*HD]
  bf16* Vs = Ks + 2 * BKV * HD;        // [2][BKV*HD]

  const int2 qb = a.qblocks[blockIdx.x];
  const int h = blockIdx.y, hk = h / (a.H / a.Hkv);
  const int base = a.cu_seqlens[qb.x], L = a.cu_seqlens[qb.x + 1] - base, q0 = qb.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int kcol = (a.H + hk) * HD, vcol = (a.H + a.Hkv + hk) * HD;
  const float sl2 = a.scale * LOG2E;

  load_tile<HD, BQ, 128>(Qs, a.qkv, a.ld_qkv, base, q0, L, h * HD);
  load_tile<HD, BQ, 128>(dOs, a.dO, a.ld_do, base, q0, L, h * HD);
  cp_async_commit();
  const int kv_end = min(L, q0 + BQ);
  const int nkv = (kv_end + BKV - 1) / BKV;
  load_tile<HD, BKV, 128>(Ks, a.qkv, a.ld_qkv, base, 0, L, kcol);
  load_tile<HD, BKV, 128>(Vs, a.qkv, a.ld_qkv, base, 0, L, vcol);
  cp_async_commit();
  cp_async_wait<1>();
  __syncthreads();
  uint32_t qf[NKS][4], df[NKS][4];
#pragma unroll
  for (int ks = 0; ks < NKS; ++ks) {
    ld_a<HD>(Qs, warp * 16, ks * 16, qf[ks]);
    ld_a<HD>(dOs, warp * 16, ks * 16, df[ks]);
  }
  const int qr0 = q0 + warp * 16 + g;
  float lse2[2], Dr[2];
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int qr = qr0 + r * 8;
    const bool ok = qr < L;
    lse2[r] = ok ? a.lse[(size_t)h * a.T + base + qr] * LOG2E : 0.f;
    Dr[r] = ok ? a.D[(size_t)h * a.T + base + qr] : 0.f;
  }
  float dq[NON][4];
#pragma unroll
  for (int i = 0; i < NON; ++i) dq[i][0] = dq[i][1] = dq[i][2] = dq[i][3] = 0.f;

  for (int j = 0; j < nkv; ++j) {
    if (j + 1 < nkv) {
      load_tile<HD, BKV, 128>(Ks + ((j + 1) & 1) * BKV * HD, a.qkv, a.ld_qkv, base, (j + 1) * BKV, L, kcol);
      load_tile<HD, BKV, 128>(Vs + ((j + 1) & 1) * BKV * HD, a.qkv, a.ld_qkv, base, (j + 1) * BKV, L, vcol);
      cp_async_commit();
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    const bf16* Kb = Ks + (j & 1) * BKV * HD;
    const bf16* Vb = Vs + (j & 1) * BKV * HD;
    float s[4][4], dp[4][4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int e = 0; e < 4; ++e) s[i][e] = dp[i][e] = 0.f;
#pragma unroll
    for (int ks = 0; ks < NKS; ++ks)
#pragma unroll
      for (int nt = 0; nt < 4; nt += 2) {
        uint32_t b0, b1, b2, b3;
        ld_b_nk<HD>(Kb, nt * 8, ks * 16, b0, b1, b2, b3);
        mma_bf16_16816(s[nt], qf[ks], b0, b1);
        mma_bf16_16816(s[nt + 1], qf[ks], b2, b3);
        ld_b_nk<HD>(Vb, nt * 8, ks * 16, b0, b1, b2, b3);
        mma_bf16_16816(dp[nt], df[ks], b0, b1);
        mma_bf16_16816(dp[nt + 1], df[ks], b2, b3);
      }
#pragma unroll
    for (int nt = 0; nt < 4; ++nt)
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int key = j * BKV + nt * 8 + 2 * t + (e & 1);
        const int qr = qr0 + (e >> 1) * 8;
        float p = 0.f;
        if (qr < L && key <= qr) p = exp2f(s[nt][e] * sl2 - lse2[e >> 1]);
        dp[nt][e] = p * (dp[nt][e] - Dr[e >> 1]);
      }
#pragma unroll
    for (int kk = 0; kk < 2; ++kk) {
      uint32_t da[4];
      da[0] = pack_bf16x2(dp[2 * kk][0], dp[2 * kk][1]);
      da[1] = pack_bf16x2(dp[2 * kk][2], dp[2 * kk][3]);
      da[2] = pack_bf16x2(dp[2 * kk + 1][0], dp[2 * kk + 1][1]);
      da[3] = pack_bf16x2(dp[2 * kk + 1][2], dp[2 * kk + 1][3]);
#pragma unroll
      for (int nt = 0; nt < NON; nt += 2) {
        uint32_t b0, b1, b2, b3;
        ld_b_kn<HD>(Kb, kk * 16, nt * 8, b0, b1, b2, b3);
        mma_bf16_16816(dq[nt], da, b0, b1);
        mma_bf16_16816(dq[nt + 1], da, b2, b3);
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < NON; ++i)
#pragma unroll
    for (int e = 0; e < 4; ++e) dq[i][e] *= a.scale;
  const int sh = a.pos_shift ? a.pos_shift[qb.x] : 0;
  const int p0 = min(qr0, L - 1) - sh, p1 = min(qr0 + 8, L - 1) - sh;
  if (a.rope_cs) rope_bwd_frag<HD>(dq, a.rope_cs, p0 < 0 ? 0 : p0, p1 < 0 ? 0 : p1);
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int qr = qr0 + r * 8;
    if (qr >= L) continue;
    bf16* qrow = a.dqkv + (size_t)(base + qr) * a.ld_dqkv + h * HD;
#pragma unroll
    for (int nt = 0; nt < NON; ++nt)
      *reinterpret_cast<uint32_t*>(qrow + nt * 8 + 2 * t) = pack_bf16x2(dq[nt][2 * r], dq[nt][2 * r + 1]);
  }
}

template <int HD>
int launch_fwd(const AttnArgs& a, cudaStream_t st) {
  const int smem = (64 * HD + 4 * 64 * HD) * 2;
  static bool set = false;
  if (!set) { cudaFuncSetAttribute(attn_fwd_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); set = true; }
  attn_fwd_kernel<HD><<<dim3(a.n_qblocks, a.H), 128, smem, st>>>(a);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}
template <int HD>
int launch_bwd(const AttnArgs& a, cudaStream_t st) {
  const int smem1 = (2 * 64 * HD + 4 * 32 * HD) * 2 + 4 * 32 * 4;
  const int smem2 = (2 * 64 * HD + 4 * 32 * HD) * 2;
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(attn_bwd_dkdv_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem1);
    cudaFuncSetAttribute(attn_bwd_dq_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2);
    set = true;
  }
  attn_bwd_dkdv_kernel<HD><<<dim3(a.n_kvblocks, a.Hkv), 128, smem1, st>>>(a);
  ++g_launch_count;
  attn_bwd_dq_kernel<HD><<<dim3(a.n_qblocks, a.H), 128, smem2, st>>>(a);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

}  // namespace

int attn_fwd(const AttnArgs& a, cudaStream_t st) {
  if (a.n_qblocks <= 0) return 0;
  switch (a.hd) {
    case 16: return launch_fwd<16>(a, st);
    case 32: return launch_fwd<32>(a, st);
    case 64: return launch_fwd<64>(a, st);
    case 128: return launch_fwd<128>(a, st);
    default: return -1;
  }
}
int attn_bwd(const AttnArgs& a, cudaStream_t st) {
  if (a.n_qblocks <= 0) return 0;
  switch (a.hd) {
    case 16: return launch_bwd<16>(a, st);
    case 32: return launch_bwd<32>(a, st);
    case 64: return launch_bwd<64>(a, st);
    case 128: return launch_bwd<128>(a, st);
    default: return -1;
  }
}

}  // namespace menos
