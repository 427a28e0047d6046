// Segmented multi-client LoRA side contractions (SURVEY.md §8(a) A2/A4/A6/A7 shrink, A8-A12 LoRA backward).
//
//   rows kernel (one client's ROWS_BM-token block, full reduction):
//     shrink   U_c  = s_c * X_c A_c^T      (B operand = A_cat rows   [W, K], "nk")
//     dU       dU_c = s_c * dY_c B_c       (B operand = B_cat        [K, W], "kn")
//   token-reduction kernel (reduce over ONE client's tokens, fixed order -> deterministic, no atomics):
//     dB_t     = dY_t^T (s U_t)            (fp32 [N_t, r])
//     dA_t     = dU_t^T X                  (fp32 [r, K_t])
//
// Paper: LoRA y += (alpha/r)(x A^T) B^T on the targeted projections (§2.1, §5.1);
// only phi = {A, B} receives gradients (Eq.1).  These are skinny contractions (r <= 16 per
// target): they are bound by streaming X / dY from HBM once, so the kernels stage 16-byte cp.async tiles
// (double-buffered) and use mma.sync m16n8k16 for the little arithmetic there is.
#include "common.cuh"
#include "kernels.h"

namespace menos {
namespace {

// swizzled element offset inside a [rows][COLS] bf16 tile (16-byte chunk XOR row)
template <int COLS>
__device__ __forceinline__ int tsw(int row, int chunk) {
  constexpr int NCH = COLS / 8;
  constexpr int MSK = NCH - 1 < 7 ? NCH - 1 : 7;
  return row * COLS + ((chunk ^ (row & MSK)) << 3);
}

// ============================================================================ rows kernel
// C[t, j] = scale * sum_k A[t, k] * Bop(j, k) for t in [m0, m0+64), j in [0, NT)
// 4-stage cp.async ring of 128-wide K tiles: ~96-192 KB of X / dY in flight per SM, enough to stream the
// activations at HBM rate with one CTA per 64-token block.
#ifndef MENOS_LORA_ROWS_BM
#define MENOS_LORA_ROWS_BM 64
#endif
// ROWS_BM tokens per CTA, one warp per 16 of them.  64 (default) vs 32 measured at cfg1 shapes
// (profiles/r1n_lora_rows_bm.txt): 32-token blocks double the CTAs but each CTA still re-stages the whole
// [N, K] adapter operand from L2, so the shrink is no faster and the per-target dU is 38% slower.
// 4 stages: 8 (one CTA per SM) measured no faster at cfg1 (35 us per layer either way: the 128 CTAs are bound by
// their per-warp issue chain, not by bytes in flight) and 1.5x slower at cfg3 (r2bc, profiles/r2bc_lora.txt)
constexpr int ROWS_BM = MENOS_LORA_ROWS_BM, ROWS_BK = 128, ROWS_NTH = ROWS_BM / 16 * 32;
template <int NT>
__host__ __device__ constexpr int rows_stages() { return 4; }
template <int NT>
constexpr int rows_smem_bytes() { return rows_stages<NT>() * (ROWS_BM + NT) * ROWS_BK * 2; }

template <int NT>
__global__ void __launch_bounds__(ROWS_NTH) lora_rows_kernel(const LoraRowsProblem* __restrict__ probs,
                                                        const int2* __restrict__ tiles) {
  constexpr int BM = ROWS_BM, BK = ROWS_BK, NNT = NT / 8, NS = rows_stages<NT>();
  extern __shared__ __align__(128) uint8_t rows_smem[];
  bf16* As_base = reinterpret_cast<bf16*>(rows_smem);                 // [NS][BM * BK]
  bf16* Bs_base = As_base + NS * BM * BK;                             // [NS][NT * BK]  ("nk": [NT][BK]; "kn": [BK][NT])
  const int2 tl = tiles[blockIdx.x];
  const LoraRowsProblem P = probs[tl.x];
  const int m0 = tl.y;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, g = lane >> 2, t = lane & 3;

  auto load = [&](int buf, int k0) {
    bf16* As = As_base + buf * BM * BK;
    bf16* Bs = Bs_base + buf * NT * BK;
    for (int i = tid; i < BM * (BK / 8); i += ROWS_NTH) {
      const int r = i / (BK / 8), c = i % (BK / 8);
      const int gr = m0 + r, gk = k0 + c * 8;
      const bool ok = gr < P.M && gk < P.K;
      cp_async16(smem_u32(&As[tsw<BK>(r, c)]), P.A + (ok ? (size_t)gr * P.lda + gk : 0), ok ? 16 : 0);
    }
    if (!P.b_kn) {
      for (int i = tid; i < NT * (BK / 8); i += ROWS_NTH) {
        const int r = i / (BK / 8), c = i % (BK / 8);
        const int gk = k0 + c * 8;
        const bool ok = r < P.N && gk < P.K;
        cp_async16(smem_u32(&Bs[tsw<BK>(r, c)]), P.B + (ok ? (size_t)r * P.ldb + gk : 0), ok ? 16 : 0);
      }
    } else {
      for (int i = tid; i < BK * (NT / 8); i += ROWS_NTH) {
        const int r = i / (NT / 8), c = i % (NT / 8);
        const int gk = k0 + r;
        const bool ok = gk < P.K && c * 8 < P.N;
        cp_async16(smem_u32(&Bs[tsw<NT>(r, c)]), P.B + (ok ? (size_t)gk * P.ldb + c * 8 : 0), ok ? 16 : 0);
      }
    }
  };

  float acc[NNT][4];
#pragma unroll
  for (int j = 0; j < NNT; ++j) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
  const int nk = (P.K + BK - 1) / BK;
#pragma unroll
  for (int s = 0; s < NS - 1; ++s) {
    if (s < nk) load(s, s * BK);
    cp_async_commit();
  }
  for (int kb = 0; kb < nk; ++kb) {
    cp_async_wait<NS - 2>();
    __syncthreads();
    {  // refill the stage freed by iteration kb-1 (everyone passed the barrier above)
      const int nx = kb + NS - 1;
      if (nx < nk) load(nx % NS, nx * BK);
      cp_async_commit();
    }
    const bf16* a_s = As_base + (kb % NS) * BM * BK;
    const bf16* b_s = Bs_base + (kb % NS) * NT * BK;
#pragma unroll
    for (int kk = 0; kk < BK; kk += 16) {
      uint32_t a[4];
      {
        const int mat = lane >> 3, r = lane & 7;
        const int row = warp * 16 + (mat & 1) * 8 + r, col = kk + (mat >> 1) * 8;
        ldsm_x4(smem_u32(a_s + tsw<BK>(row, col >> 3)), a[0], a[1], a[2], a[3]);
      }
#pragma unroll
      for (int j = 0; j < NNT; j += 2) {
        uint32_t b0, b1, b2, b3;
        const int mat = lane >> 3, r = lane & 7;
        if (!P.b_kn) {
          const int row = j * 8 + (mat >> 1) * 8 + r, col = kk + (mat & 1) * 8;
          ldsm_x4(smem_u32(b_s + tsw<BK>(row, col >> 3)), b0, b1, b2, b3);
        } else {
          const int row = kk + (mat & 1) * 8 + r, col = j * 8 + (mat >> 1) * 8;
          ldsm_x4_t(smem_u32(b_s + tsw<NT>(row, col >> 3)), b0, b1, b2, b3);
        }
        mma_bf16_16816(acc[j], a, b0, b1);
        mma_bf16_16816(acc[j + 1], a, b2, b3);
      }
    }
  }
  cp_async_wait<0>();
#pragma unroll
  for (int j = 0; j < NNT; ++j)
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int r = m0 + warp * 16 + g + h * 8;
      const int c = j * 8 + 2 * t;
      if (r >= P.M || c >= P.N) continue;
      *reinterpret_cast<uint32_t*>(P.C + (size_t)r * P.ldc + c) =
          pack_bf16x2(acc[j][2 * h] * P.scale, acc[j][2 * h + 1] * P.scale);
    }
}

// ============================================================================ token-reduction kernel
// C[m, n] = scale * sum_t P[t, map(m)] * Q[t, n]  over t in [0, T); tile (MT x NT) at (m0, n0)
// 4-stage cp.async ring of 64-token stages (~54 KB of P / Q in flight per CTA): the reduction streams one client's
// activations once, so bytes in flight, not math, set its speed
constexpr int TR_BK = 64, TR_STAGES = 4;
template <int MT, int NT>
constexpr int tokred_smem_bytes() { return TR_STAGES * TR_BK * (MT + NT) * 2; }

template <int MT, int NT>
__global__ void __launch_bounds__(128) lora_tokred_kernel(const LoraTokRedProblem* __restrict__ probs,
                                                          const int4* __restrict__ tiles) {
  constexpr int BK = TR_BK, NS = TR_STAGES;    // tokens per stage, stages
  constexpr int WM = MT >= 64 ? MT / 4 : MT;   // rows per warp (4 warps split M when MT is large)
  constexpr int WN = MT >= 64 ? NT : NT / 4;   // cols per warp (else split N)
  constexpr int NMI = WM / 16, NNJ = WN / 8;
  extern __shared__ __align__(128) uint8_t tr_smem[];
  bf16* Ps_base = reinterpret_cast<bf16*>(tr_smem);   // [NS][BK * MT]  ([token][m])
  bf16* Qs_base = Ps_base + NS * BK * MT;             // [NS][BK * NT]  ([token][n])
  const int4 tl = tiles[blockIdx.x];
  const LoraTokRedProblem P = probs[tl.x];
  const int m0 = tl.y, n0 = tl.z;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, g = lane >> 2, t = lane & 3;
  const int wm0 = MT >= 64 ? warp * WM : 0, wn0 = MT >= 64 ? 0 : warp * WN;
  // P columns of this tile are contiguous: m0 is a multiple of MT and p_blk (128) is a multiple of MT
  const int pcol0 = (m0 / P.p_blk) * P.p_blk_stride + m0 % P.p_blk;

  auto load = [&](int buf, int t0) {
    bf16* Ps = Ps_base + buf * BK * MT;
    bf16* Qs = Qs_base + buf * BK * NT;
    for (int i = tid; i < BK * (MT / 8); i += 128) {
      const int r = i / (MT / 8), c = i % (MT / 8);
      const int tok = t0 + r;
      const bool ok = tok < P.T && m0 + c * 8 < P.M;
      cp_async16(smem_u32(&Ps[tsw<MT>(r, c)]), P.P + (ok ? (size_t)tok * P.ldp + pcol0 + c * 8 : 0), ok ? 16 : 0);
    }
    for (int i = tid; i < BK * (NT / 8); i += 128) {
      const int r = i / (NT / 8), c = i % (NT / 8);
      const int tok = t0 + r;
      const bool ok = tok < P.T && n0 + c * 8 < P.N;
      cp_async16(smem_u32(&Qs[tsw<NT>(r, c)]), P.Q + (ok ? (size_t)tok * P.ldq + n0 + c * 8 : 0), ok ? 16 : 0);
    }
  };

  float acc[NMI][NNJ][4];
#pragma unroll
  for (int i = 0; i < NMI; ++i)
#pragma unroll
    for (int j = 0; j < NNJ; ++j) acc[i][j][0] = acc[i][j][1] = acc[i][j][2] = acc[i][j][3] = 0.f;
  const int nk = (P.T + BK - 1) / BK;
#pragma unroll
  for (int s = 0; s < NS - 1; ++s) {
    if (s < nk) load(s, s * BK);
    cp_async_commit();
  }
  for (int kb = 0; kb < nk; ++kb) {
    cp_async_wait<NS - 2>();
    __syncthreads();
    {
      const int nx = kb + NS - 1;
      if (nx < nk) load(nx % NS, nx * BK);
      cp_async_commit();
    }
    const bf16* p_s = Ps_base + (kb % NS) * BK * MT;
    const bf16* q_s = Qs_base + (kb % NS) * BK * NT;
#pragma unroll
    for (int kk = 0; kk < BK; kk += 16) {
      const int mat = lane >> 3, r = lane & 7;
      uint32_t a[NMI][4];
#pragma unroll
      for (int i = 0; i < NMI; ++i) {
        // A(m, k) = P[k][m]: transposed ldmatrix of the [token][m] tile
        const int row = kk + (mat >> 1) * 8 + r, col = wm0 + i * 16 + (mat & 1) * 8;
        ldsm_x4_t(smem_u32(p_s + tsw<MT>(row, col >> 3)), a[i][0], a[i][1], a[i][2], a[i][3]);
      }
#pragma unroll
      for (int j = 0; j < NNJ; j += 2) {
        uint32_t b0, b1, b2, b3;
        const int row = kk + (mat & 1) * 8 + r, col = wn0 + j * 8 + (mat >> 1) * 8;
        ldsm_x4_t(smem_u32(q_s + tsw<NT>(row, col >> 3)), b0, b1, b2, b3);
#pragma unroll
        for (int i = 0; i < NMI; ++i) {
          mma_bf16_16816(acc[i][j], a[i], b0, b1);
          mma_bf16_16816(acc[i][j + 1], a[i], b2, b3);
        }
      }
    }
  }
  cp_async_wait<0>();
#pragma unroll
  for (int i = 0; i < NMI; ++i)
#pragma unroll
    for (int j = 0; j < NNJ; ++j)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int r = m0 + wm0 + i * 16 + g + h * 8;
        const int c = n0 + wn0 + j * 8 + 2 * t;
        if (r >= P.M) continue;
        const int seg = P.m_seg > 0 ? r / P.m_seg : 0, mr = P.m_seg > 0 ? r % P.m_seg : r;
        if (P.m_valid > 0 && mr >= P.m_valid) continue;
        float* C = seg == 0 ? P.C : seg == 1 ? P.C1 : P.C2;
        if (c < P.N) C[(size_t)mr * P.ldc + c] = acc[i][j][2 * h] * P.scale;
        if (c + 1 < P.N) C[(size_t)mr * P.ldc + c + 1] = acc[i][j][2 * h + 1] * P.scale;
      }
}

// ============================================================================ fused dU + dB kernel
// CTA = (problem, slab of MT dY columns, 16-wide rank tile); streams the client's T tokens once in 64-token stages
// (4-stage cp.async ring of the [64, MT] dY tile and the [64, 16] U tile).  Per stage:
//   dB[slab, n]  += dY_tile^T U_tile     (accumulated in registers over all tokens; one fixed order)
//   W[slab][t, n] = dY_tile B_slab       (this slab's share of dU for the stage's tokens, written once)
// Replaces the two passes (dU rows kernel + dB token reduction) that each read dY from HBM.
constexpr int DUB_BK = 64, DUB_STAGES = 4, DUB_NT = 16;
template <int MT>
constexpr int dub_smem_bytes() { return DUB_STAGES * DUB_BK * (MT + DUB_NT) * 2 + MT * DUB_NT * 2; }

// NJ: n8 tiles of the 16-wide rank tile that carry data (1 when rank <= 8: half the MMAs, which the kernel needs --
// at r = 8 it does 8 MACs per dY byte on mma.sync)
template <int MT, int NJ>
__global__ void __launch_bounds__(128) lora_dub_kernel(const LoraDUBProblem* __restrict__ probs, int n_rt) {
  constexpr int BK = DUB_BK, NS = DUB_STAGES, NT = DUB_NT;
  constexpr int WM = MT / 4, NMI = WM / 16;   // dB: each warp owns WM of the slab's columns
  constexpr int CPR = MT / 8;                 // 16-byte chunks per dY row of a stage
  static_assert(128 % CPR == 0, "one fixed chunk column per thread");
  extern __shared__ __align__(128) uint8_t dub_smem[];
  bf16* Ps_base = reinterpret_cast<bf16*>(dub_smem);   // [NS][BK * MT]  ([token][m])
  bf16* Us_base = Ps_base + NS * BK * MT;              // [NS][BK * NT]  ([token][n])
  bf16* Bs = Us_base + NS * BK * NT;                   // [MT * NT]      ([m][n])
  const LoraDUBProblem P = probs[blockIdx.y];
  const int slab = blockIdx.x / n_rt, n0 = (blockIdx.x % n_rt) * NT;
  if (slab >= P.n_slabs || n0 >= P.rank) return;
  const int m0 = slab * MT;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, g = lane >> 2, t = lane & 3;
  // the slab's dY columns are contiguous (p_blk is a multiple of MT, host-checked)
  const int pcol0 = (m0 / P.p_blk) * P.p_blk_stride + m0 % P.p_blk;

  // this slab's B rows (indexed like dY's columns), once
  for (int i = tid; i < MT * (NT / 8); i += 128) {
    const int r = i / (NT / 8), c = i % (NT / 8);
    const bool ok = m0 + r < P.Nt && n0 + c * 8 < P.rs;
    cp_async16(smem_u32(&Bs[tsw<NT>(r, c)]), P.B + (ok ? (size_t)(pcol0 + r) * P.ldb + n0 + c * 8 : 0), ok ? 16 : 0);
  }
  // per-thread fixed dY chunk column, rows r0 + (128 / CPR) k
  const int yc = tid % CPR, yr0 = tid / CPR;
  const bool ycol_ok = m0 + yc * 8 < P.Nt;
  const bf16* ysrc = P.dY + pcol0 + yc * 8;
  const int uc = tid & 1, ur0 = tid >> 1;   // U: 2 chunks per row (NT = 16)
  const bool ucol_ok = n0 + uc * 8 < P.rank;
  const bf16* usrc = P.U + n0 + uc * 8;
  auto load = [&](int buf, int t0) {
    bf16* Ps = Ps_base + buf * BK * MT;
    bf16* Us = Us_base + buf * BK * NT;
#pragma unroll
    for (int r = yr0; r < BK; r += 128 / CPR) {
      const int tok = t0 + r;
      const bool ok = ycol_ok && tok < P.T;
      cp_async16(smem_u32(&Ps[tsw<MT>(r, yc)]), ok ? ysrc + (size_t)tok * P.ldy : P.dY, ok ? 16 : 0);
    }
    if (ur0 < BK) {
      const int tok = t0 + ur0;
      const bool ok = ucol_ok && tok < P.T;
      cp_async16(smem_u32(&Us[tsw<NT>(ur0, uc)]), ok ? usrc + (size_t)tok * P.ldu : P.U, ok ? 16 : 0);
    }
  };

  float accb[NMI][NJ][4];
#pragma unroll
  for (int i = 0; i < NMI; ++i)
#pragma unroll
    for (int j = 0; j < NJ; ++j) accb[i][j][0] = accb[i][j][1] = accb[i][j][2] = accb[i][j][3] = 0.f;
  const int nk = (P.T + BK - 1) / BK;
#pragma unroll
  for (int s = 0; s < NS - 1; ++s) {
    if (s < nk) load(s, s * BK);
    cp_async_commit();   // the first group also carries the B slab
  }
  const int mat = lane >> 3, rr = lane & 7;
  float* const Wb = P.W + (size_t)slab * P.T * P.rank;
  for (int kb = 0; kb < nk; ++kb) {
    cp_async_wait<NS - 2>();
    __syncthreads();
    {
      const int nx = kb + NS - 1;
      if (nx < nk) load(nx % NS, nx * BK);
      cp_async_commit();
    }
    const bf16* p_s = Ps_base + (kb % NS) * BK * MT;
    const bf16* u_s = Us_base + (kb % NS) * BK * NT;
    // dB: A(m, k=token) = dY^T via transposed ldmatrix, B(k=token, n) = U
#pragma unroll
    for (int kk = 0; kk < BK; kk += 16) {
      uint32_t a[NMI][4];
#pragma unroll
      for (int i = 0; i < NMI; ++i) {
        const int row = kk + (mat >> 1) * 8 + rr, col = warp * WM + i * 16 + (mat & 1) * 8;
        ldsm_x4_t(smem_u32(p_s + tsw<MT>(row, col >> 3)), a[i][0], a[i][1], a[i][2], a[i][3]);
      }
      uint32_t b[4];
      {
        const int row = kk + (mat & 1) * 8 + rr, col = (mat >> 1) * 8;
        ldsm_x4_t(smem_u32(u_s + tsw<NT>(row, col >> 3)), b[0], b[1], b[2], b[3]);
      }
#pragma unroll
      for (int i = 0; i < NMI; ++i)
#pragma unroll
        for (int j = 0; j < NJ; ++j) mma_bf16_16816(accb[i][j], a[i], b[2 * j], b[2 * j + 1]);
    }
    // dU share: warp w takes the stage's tokens 16w..16w+15, reduction over the slab's MT columns in two independent
    // accumulator chains (even / odd 16-column steps) summed at the end -- the same order for every NJ, so a
    // client's dU does not depend on the ranks of the clients sharing its batch
    {
      float acc2[NJ][2][4];
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int c = 0; c < 2; ++c) acc2[j][c][0] = acc2[j][c][1] = acc2[j][c][2] = acc2[j][c][3] = 0.f;
#pragma unroll
      for (int kk = 0; kk < MT; kk += 16) {
        uint32_t a[4], b[4];
        {
          const int row = warp * 16 + (mat & 1) * 8 + rr, col = kk + (mat >> 1) * 8;
          ldsm_x4(smem_u32(p_s + tsw<MT>(row, col >> 3)), a[0], a[1], a[2], a[3]);
        }
        {
          const int row = kk + (mat & 1) * 8 + rr, col = (mat >> 1) * 8;
          ldsm_x4_t(smem_u32(Bs + tsw<NT>(row, col >> 3)), b[0], b[1], b[2], b[3]);
        }
#pragma unroll
        for (int j = 0; j < NJ; ++j) mma_bf16_16816(acc2[j][(kk >> 4) & 1], a, b[2 * j], b[2 * j + 1]);
      }
      float accu[NJ][4];
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int e = 0; e < 4; ++e) accu[j][e] = acc2[j][0][e] + acc2[j][1][e];
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int tok = kb * BK + warp * 16 + g + h * 8;
          const int n = n0 + j * 8 + 2 * t;
          if (tok >= P.T) continue;
          float* w = Wb + (size_t)tok * P.rank + n;
          if (n < P.rank) w[0] = accu[j][2 * h];
          if (n + 1 < P.rank) w[1] = accu[j][2 * h + 1];
        }
    }
  }
  cp_async_wait<0>();
#pragma unroll
  for (int i = 0; i < NMI; ++i)
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int m = m0 + warp * WM + i * 16 + g + h * 8;
        const int n = n0 + j * 8 + 2 * t;
        if (m >= P.Nt) continue;
        float* d = P.dB + (size_t)m * P.rank + n;
        if (n < P.rank) d[0] = accb[i][j][2 * h];
        if (n + 1 < P.rank) d[1] = accb[i][j][2 * h + 1];
      }
}

// dU[t, n] = bf16(scale * sum over slabs, in slab order, of W[s][t, n]); zero in the slot's padding columns
__global__ void __launch_bounds__(256) lora_du_reduce_kernel(const LoraDUBProblem* __restrict__ probs) {
  const LoraDUBProblem P = probs[blockIdx.y];
  if ((P.rank & 3) == 0 && (P.rs & 3) == 0 && (P.lddu & 3) == 0 && (reinterpret_cast<uintptr_t>(P.W) & 15) == 0) {
    const long long e4 = (long long)blockIdx.x * 256 + threadIdx.x;
    if (e4 * 4 >= (long long)P.T * P.rs) return;
    const int tok = (int)(e4 * 4 / P.rs), n = (int)(e4 * 4 % P.rs);
    float4 a = make_float4(0.f, 0.f, 0.f, 0.f);
    if (n < P.rank) {
      const float4* w = reinterpret_cast<const float4*>(P.W + (size_t)tok * P.rank + n);
      const size_t step = (size_t)P.T * P.rank / 4;
#pragma unroll 8
      for (int i = 0; i < P.n_slabs; ++i) {
        const float4 v = w[i * step];
        a.x += v.x; a.y += v.y; a.z += v.z; a.w += v.w;
      }
    }
    uint2 o = make_uint2(pack_bf16x2(a.x * P.scale, a.y * P.scale), pack_bf16x2(a.z * P.scale, a.w * P.scale));
    *reinterpret_cast<uint2*>(P.dU + (size_t)tok * P.lddu + n) = o;
    return;
  }
  const long long e = (long long)blockIdx.x * 256 + threadIdx.x;
  if (e >= (long long)P.T * P.rs) return;
  const int tok = (int)(e / P.rs), n = (int)(e % P.rs);
  float s = 0.f;
  if (n < P.rank) {
    const float* w = P.W + (size_t)tok * P.rank + n;
    const size_t step = (size_t)P.T * P.rank;
#pragma unroll 8
    for (int i = 0; i < P.n_slabs; ++i) s += w[i * step];
  }
  P.dU[(size_t)tok * P.lddu + n] = __float2bfloat16_rn(s * P.scale);
}

// ============================================================================ shrink on tcgen05
// U[t0 + m, col + n] = bf16(scale * sum_k X[t0 + m, k] Acat[col + n, k])  (m < T, n < w): a [128 x K] . [K x N]
// skinny GEMM per 128-token tile of one client.  TMA streams X and the client's Acat rows (both K-major, 128-byte
// swizzle) through a ring of ~200 KB, one elected thread issues tcgen05.mma into a [128 x N] TMEM accumulator, four
// warps scale, convert and store.  Pure streaming of X: on mma.sync the same contraction ran at ~2 TB/s (r2bc).
constexpr int SHK_BK = 64;
template <int N> struct ShkGeo {
  static constexpr int A_BYTES = 128 * SHK_BK * 2, B_BYTES = N * SHK_BK * 2, STAGE = A_BYTES + B_BYTES;
  static constexpr int STAGES = (200 * 1024) / STAGE;
  static constexpr int SMEM = STAGES * STAGE + 1024;
  static constexpr int TCOLS = N < 32 ? 32 : N;
};

template <int N>
__global__ void __launch_bounds__(192, 1)
lora_shrink_tc_kernel(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmA,
                      const LoraShrinkProblem* __restrict__ probs, const int2* __restrict__ tiles, int K, bf16* U,
                      int ldu) {
  using G = ShkGeo<N>;
  constexpr int S = G::STAGES;
  extern __shared__ uint8_t shk_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(shk_raw) + 1023) & ~uintptr_t(1023));
  __shared__ __align__(8) uint64_t full[S], empty[S], acc_full;
  __shared__ uint32_t tmem_sh;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int2 tl = tiles[blockIdx.x];
  const LoraShrinkProblem P = probs[tl.x];
  const int m0 = tl.y, nk = (K + SHK_BK - 1) / SHK_BK;
  if (threadIdx.x == 0) {
    tma_prefetch(&tmX); tma_prefetch(&tmA);
    for (int i = 0; i < S; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    mbar_init(&acc_full, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<G::TCOLS>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  if (warp == 0) {
    if (elect_one()) {
      for (int kb = 0; kb < nk; ++kb) {
        const int st = kb % S;
        mbar_wait(&empty[st], ((kb / S) & 1) ^ 1);
        mbar_expect_tx(&full[st], G::STAGE);
        uint8_t* sa = smem + st * G::STAGE;
        tma_load_2d(sa, &tmX, &full[st], kb * SHK_BK, P.t0 + m0);
        tma_load_2d(sa + G::A_BYTES, &tmA, &full[st], kb * SHK_BK, P.col);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    constexpr uint32_t ID = umma_idesc_bf16(128, N, 0);
    for (int kb = 0; kb < nk; ++kb) {
      const int st = kb % S;
      mbar_wait(&full[st], (kb / S) & 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t sa = smem_u32(smem + st * G::STAGE), sb = sa + G::A_BYTES;
#pragma unroll
        for (int kk = 0; kk < SHK_BK / 16; ++kk)
          tc_mma_bf16(tmem, umma_desc_sw128(sa + kk * 32, 16, 1024), umma_desc_sw128(sb + kk * 32, 16, 1024), ID,
                      (kb > 0 || kk > 0) ? 1u : 0u);
        tc_commit(&empty[st]);
        if (kb == nk - 1) tc_commit(&acc_full);
      }
      __syncwarp();
    }
  } else {
    const int q = warp & 3, row = q * 32 + lane;   // TMEM lane quadrant of this warp
    mbar_wait(&acc_full, 0);
    tc_fence_after();
    const bool ok = m0 + row < P.T;
    bf16* dst = U + (size_t)(P.t0 + m0 + row) * ldu + P.col;
#pragma unroll
    for (int c0 = 0; c0 < N; c0 += 32) {
      uint32_t r[32];
      tmem_ld32_nw(tmem + c0 + ((uint32_t)(q * 32) << 16), r);
      tmem_wait_ld();
      if (ok) {
#pragma unroll
        for (int j = 0; j < 32; j += 8)
          if (c0 + j < P.w) {
            uint4 v;
            v.x = pack_bf16x2(__uint_as_float(r[j]) * P.scale, __uint_as_float(r[j + 1]) * P.scale);
            v.y = pack_bf16x2(__uint_as_float(r[j + 2]) * P.scale, __uint_as_float(r[j + 3]) * P.scale);
            v.z = pack_bf16x2(__uint_as_float(r[j + 4]) * P.scale, __uint_as_float(r[j + 5]) * P.scale);
            v.w = pack_bf16x2(__uint_as_float(r[j + 6]) * P.scale, __uint_as_float(r[j + 7]) * P.scale);
            *reinterpret_cast<uint4*>(dst + c0 + j) = v;
          }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<G::TCOLS>(tmem);
  }
}

// ============================================================================ fused dU + dB on tcgen05
// Same contract as lora_dub_kernel for rank <= 16, with the contractions on the 5th-gen tensor cores: CTA = (problem,
// 128-column slab), 128-token stages.  One staged dY tile [128 tokens][128 columns] (two TMA boxes, 128-byte
// swizzle) is BOTH the MN-major A operand of dB[slab] += dY^T U (M = 128 columns, K = tokens) and the K-major A
// operand of this slab's dU share W = dY B_slab (M = 128 tokens, K = columns); the two small B operands (U^T of the
// stage, B_slab^T once) are transposed by the epilogue warps into K-major swizzled tiles.  dB accumulates in TMEM
// over all stages; each stage's dU share lands in one of two TMEM buffers and is written out as fp32 partial rows
// while the next stage runs.  Rows past the client's tokens and columns past the target's are zeroed in the
// transposed operands, so they contribute nothing.
// MTS = dY columns per CTA (slab): 128, or 256 for large grids (half the fp32 dU partials to write and sum; two
// M = 128 dB accumulators)
constexpr int DUBT_BK = 128, DUBT_ST = 2;
constexpr int DUBT_U = 128 * 16 * 2;             // U stage, linear [128][16]
constexpr int DUBT_UT = 16 * 128 * 2;            // U^T: [16][128 tokens] K-major (two [16][64] atoms)
template <int MTS> struct DubtGeo {
  static constexpr int Y = 128 * MTS * 2;        // dY stage: MTS / 64 atoms of [128 rows][64 cols]
  static constexpr int BT = 16 * MTS * 2;        // B_slab^T: [16][MTS] K-major (MTS / 64 atoms of [16][64])
  static constexpr int STAGE = Y + DUBT_U + DUBT_UT;
  static constexpr int SMEM = DUBT_ST * STAGE + BT + 1024;
};

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// the first `rank` (<= 16) of 16 fp32 values -> dst; 16-byte stores when rank % 4 == 0 and dst is aligned
__device__ __forceinline__ void store_row16(float* dst, const uint32_t (&r)[16], int rank) {
  if ((rank & 3) == 0 && (reinterpret_cast<uintptr_t>(dst) & 15) == 0) {
#pragma unroll
    for (int n = 0; n < 16; n += 4)
      if (n < rank) *reinterpret_cast<uint4*>(dst + n) = make_uint4(r[n], r[n + 1], r[n + 2], r[n + 3]);
  } else {
#pragma unroll
    for (int n = 0; n < 16; ++n)
      if (n < rank) dst[n] = __uint_as_float(r[n]);
  }
}
// element (row n < 16, k < 128) of a K-major [16][128] bf16 tile in two 128-byte-swizzled [16][64] atoms
__device__ __forceinline__ uint32_t kt_off(int n, int k) {
  return (uint32_t)((k >> 6) * 2048 + n * 128 + ((((k & 63) >> 3) ^ (n & 7)) << 4) + (k & 7) * 2);
}

template <int MTS>
__global__ void __launch_bounds__(192, MTS == 128 ? 2 : 1)
lora_dub_tc_kernel(const __grid_constant__ CUtensorMap tmY, const __grid_constant__ CUtensorMap tmU,
                   const LoraDUBProblem* __restrict__ probs) {
  using Gd = DubtGeo<MTS>;
  constexpr int NH = MTS / 128;                  // dB accumulators (M = 128 each)
  constexpr int DUBT_Y = Gd::Y, DUBT_STAGE = Gd::STAGE;
  extern __shared__ uint8_t dubt_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(dubt_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* const sBT = smem + DUBT_ST * DUBT_STAGE;
  __shared__ __align__(8) uint64_t full[DUBT_ST], empty[DUBT_ST], ut_full[DUBT_ST], bt_ready, du_full[2], du_free[2],
      db_full;
  __shared__ uint32_t tmem_sh;
  const LoraDUBProblem P = probs[blockIdx.y];
  const int slab = blockIdx.x;
  if (slab >= P.n_slabs) return;
  const int m0 = slab * MTS, nst = (P.T + DUBT_BK - 1) / DUBT_BK;
  auto pcol = [&](int m) { return (m / P.p_blk) * P.p_blk_stride + m % P.p_blk; };   // per 64-column atom
  const int pcol0 = pcol(m0);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    tma_prefetch(&tmY); tma_prefetch(&tmU);
    for (int i = 0; i < DUBT_ST; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); mbar_init(&ut_full[i], 4); }
    mbar_init(&bt_ready, 4);
    for (int i = 0; i < 2; ++i) { mbar_init(&du_full[i], 1); mbar_init(&du_free[i], 4); }
    mbar_init(&db_full, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<64>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;   // dB halves at columns 0 (/ 16), dU buffers after them
  if (warp == 0) {
    if (elect_one()) {
      for (int s = 0; s < nst; ++s) {
        const int st = s % DUBT_ST;
        mbar_wait(&empty[st], ((s / DUBT_ST) & 1) ^ 1);
        mbar_expect_tx(&full[st], DUBT_Y + DUBT_U);
        uint8_t* sy = smem + st * DUBT_STAGE;
        const int row = P.t0 + s * DUBT_BK;
#pragma unroll
        for (int a = 0; a < MTS / 64; ++a) tma_load_2d(sy + a * 16384, &tmY, &full[st], P.ycol0 + pcol(m0 + 64 * a), row);
        tma_load_2d(sy + DUBT_Y, &tmU, &full[st], P.ucol0, row);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    constexpr uint32_t ID_DB = umma_idesc_bf16(128, 16, 0) | (1u << 15);   // A (dY^T) MN-major, B (U^T) K-major
    constexpr uint32_t ID_DU = umma_idesc_bf16(128, 16, 0);                // A (dY) K-major, B (B_slab^T) K-major
    mbar_wait(&bt_ready, 0);
    for (int s = 0; s < nst; ++s) {
      const int st = s % DUBT_ST, b = s & 1;
      mbar_wait(&full[st], (s / DUBT_ST) & 1);
      mbar_wait(&ut_full[st], (s / DUBT_ST) & 1);
      mbar_wait(&du_free[b], ((s >> 1) & 1) ^ 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t sy = smem_u32(smem + st * DUBT_STAGE), sut = sy + DUBT_Y + DUBT_U, sbt = smem_u32(sBT);
#pragma unroll
        for (int h = 0; h < NH; ++h)                 // dB half h: slab columns 128 h .. 128 h + 127 (atoms 2h, 2h+1)
#pragma unroll
          for (int kk = 0; kk < DUBT_BK / 16; ++kk)   // K = 16 tokens = 16 rows of the dY atoms, of U^T
            tc_mma_bf16(tmem + 16 * h, umma_desc_sw128(sy + h * 32768 + kk * 2048, 16384, 1024),
                        umma_desc_sw128(sut + (kk >> 2) * 2048 + (kk & 3) * 32, 16, 1024), ID_DB,
                        (s > 0 || kk > 0) ? 1u : 0u);
#pragma unroll
        for (int kk = 0; kk < MTS / 16; ++kk)       // dU share: K = 16 slab columns
          tc_mma_bf16(tmem + 16 * NH + 16 * b, umma_desc_sw128(sy + (kk >> 2) * 16384 + (kk & 3) * 32, 16, 1024),
                      umma_desc_sw128(sbt + (kk >> 2) * 2048 + (kk & 3) * 32, 16, 1024), ID_DU, kk > 0 ? 1u : 0u);
        tc_commit(&empty[st]);
        tc_commit(&du_full[b]);
        if (s == nst - 1) tc_commit(&db_full);
      }
      __syncwarp();
    }
  } else {
    const int q = warp & 3, row = q * 32 + lane;   // TMEM lane quadrant; row = token (dU) / slab column (dB)
    const uint32_t loff = (uint32_t)(q * 32) << 16;
#pragma unroll
    for (int h = 0; h < NH; ++h) {   // B_slab^T [16][MTS]: row n = rank column n, k = slab column; zero past the
                                     // target's columns / the rank
      const int k = 128 * h + row;
      const bool ok = m0 + k < P.Nt;
      const uint4* src = reinterpret_cast<const uint4*>(P.B + (size_t)(ok ? pcol(m0 + k) : 0) * P.ldb);
      uint4 v0 = ok ? src[0] : make_uint4(0, 0, 0, 0), v1 = ok ? src[1] : make_uint4(0, 0, 0, 0);
      const bf16* e0 = reinterpret_cast<const bf16*>(&v0);
      const bf16* e1 = reinterpret_cast<const bf16*>(&v1);
      const bf16 z = __float2bfloat16_rn(0.f);
#pragma unroll
      for (int n = 0; n < 16; ++n)
        *reinterpret_cast<bf16*>(sBT + kt_off(n, k)) = n < P.rank ? (n < 8 ? e0[n] : e1[n - 8]) : z;
    }
    {
      fence_proxy_async();
      __syncwarp();
      if (lane == 0) mbar_arrive(&bt_ready);
    }
    float* const Wb = P.W + (size_t)slab * P.T * P.rank;
    auto du_out = [&](int s) {   // stage s's dU share -> fp32 partial rows
      const int b = s & 1;
      mbar_wait(&du_full[b], (s >> 1) & 1);
      tc_fence_after();
      uint32_t r[16];
      tmem_ld16(tmem + 16 * NH + 16 * b + loff, r);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&du_free[b]);
      const int tok = s * DUBT_BK + row;
      if (tok < P.T) store_row16(Wb + (size_t)tok * P.rank, r, P.rank);
    };
    for (int s = 0; s < nst; ++s) {
      const int st = s % DUBT_ST;
      mbar_wait(&full[st], (s / DUBT_ST) & 1);
      {   // U^T [16][128 tokens] of this stage, zero past the client's tokens and the rank
        const uint8_t* su = smem + st * DUBT_STAGE + DUBT_Y;
        uint8_t* sut = smem + st * DUBT_STAGE + DUBT_Y + DUBT_U;
        const bool ok = s * DUBT_BK + row < P.T;
        uint4 v0 = ok ? reinterpret_cast<const uint4*>(su + row * 32)[0] : make_uint4(0, 0, 0, 0);
        uint4 v1 = ok ? reinterpret_cast<const uint4*>(su + row * 32)[1] : make_uint4(0, 0, 0, 0);
        const bf16* e0 = reinterpret_cast<const bf16*>(&v0);
        const bf16* e1 = reinterpret_cast<const bf16*>(&v1);
        const bf16 z = __float2bfloat16_rn(0.f);
#pragma unroll
        for (int n = 0; n < 16; ++n)
          *reinterpret_cast<bf16*>(sut + kt_off(n, row)) = n < P.rank ? (n < 8 ? e0[n] : e1[n - 8]) : z;
        fence_proxy_async();
        __syncwarp();
        if (lane == 0) mbar_arrive(&ut_full[st]);
      }
      if (s > 0) du_out(s - 1);
    }
    if (nst > 0) du_out(nst - 1);
    mbar_wait(&db_full, 0);
    tc_fence_after();
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      uint32_t r[16];
      tmem_ld16(tmem + 16 * h + loff, r);
      const int m = m0 + 128 * h + row;
      if (m < P.Nt) store_row16(P.dB + (size_t)m * P.rank, r, P.rank);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<64>(tmem);
  }
}

// ============================================================================ dA on tcgen05
// dA^T[k, m] = sum_t X[t, k] dU[t, m] for one client's group: CTA = (problem, 128 columns of X), 128-token stages.
// The staged X tile [128 tokens][128 columns] (two TMA boxes, 128-byte swizzle) is the MN-major A operand (M = 128
// columns, K = tokens); the stage's dU columns [128 tokens][NW] are transposed by the epilogue warps into a K-major
// [NW][128] operand (rows past the client's tokens / slot width zeroed).  The [128 x NW] accumulator stays in TMEM
// over all stages; one thread per column k writes it to every target's dA rows.
constexpr int DAT_BK = 128;
// STG stages: 4 (one CTA per SM, ~200 KB in flight) when the grid is small (cfg1: 128 CTAs; 25.0 -> 19.7 us per
// layer), 2 (two CTAs per SM) when it is large (cfg3: 4 stages measured 217 -> 246 us), r2bh / r2bi
template <int NW, int STG> struct DatGeo {
  static constexpr int X = 128 * 128 * 2, U = 128 * NW * 2, UT = NW * 128 * 2, STAGE = X + U + UT;
  static constexpr int ST = STG;
  static constexpr int SMEM = ST * STAGE + 1024;
  static constexpr int TCOLS = NW < 32 ? 32 : NW;
};

template <int NW, int STG>
__global__ void __launch_bounds__(192, 1)
lora_da_tc_kernel(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmU,
                  const LoraTokRedProblem* __restrict__ probs) {
  using G = DatGeo<NW, STG>;
  constexpr int DAT_ST = G::ST;
  extern __shared__ uint8_t dat_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(dat_raw) + 1023) & ~uintptr_t(1023));
  __shared__ __align__(8) uint64_t full[DAT_ST], empty[DAT_ST], ut_full[DAT_ST], acc_full;
  __shared__ uint32_t tmem_sh;
  const LoraTokRedProblem P = probs[blockIdx.y];
  const int k0 = blockIdx.x * 128;
  if (k0 >= P.N) return;
  const int nst = (P.T + DAT_BK - 1) / DAT_BK;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    tma_prefetch(&tmX); tma_prefetch(&tmU);
    for (int i = 0; i < DAT_ST; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); mbar_init(&ut_full[i], 4); }
    mbar_init(&acc_full, 1);
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<G::TCOLS>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  if (warp == 0) {
    if (elect_one()) {
      for (int s = 0; s < nst; ++s) {
        const int st = s % DAT_ST;
        mbar_wait(&empty[st], ((s / DAT_ST) & 1) ^ 1);
        mbar_expect_tx(&full[st], G::X + G::U);
        uint8_t* sx = smem + st * G::STAGE;
        const int row = P.t0 + s * DAT_BK;
        tma_load_2d(sx, &tmX, &full[st], k0, row);
        tma_load_2d(sx + 16384, &tmX, &full[st], k0 + 64, row);
        tma_load_2d(sx + G::X, &tmU, &full[st], P.pcol0, row);
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    constexpr uint32_t ID = umma_idesc_bf16(128, NW, 0) | (1u << 15);   // A (X^T) MN-major, B (dU^T) K-major
    for (int s = 0; s < nst; ++s) {
      const int st = s % DAT_ST;
      mbar_wait(&full[st], (s / DAT_ST) & 1);
      mbar_wait(&ut_full[st], (s / DAT_ST) & 1);
      tc_fence_after();
      __syncwarp();
      if (elect_one()) {
        const uint32_t sx = smem_u32(smem + st * G::STAGE), sut = sx + G::X + G::U;
#pragma unroll
        for (int kk = 0; kk < DAT_BK / 16; ++kk)
          tc_mma_bf16(tmem, umma_desc_sw128(sx + kk * 2048, 16384, 1024),
                      umma_desc_sw128(sut + (kk >> 2) * (NW * 128) + (kk & 3) * 32, 16, 1024), ID,
                      (s > 0 || kk > 0) ? 1u : 0u);
        tc_commit(&empty[st]);
        if (s == nst - 1) tc_commit(&acc_full);
      }
      __syncwarp();
    }
  } else {
    const int q = warp & 3, row = q * 32 + lane;
    for (int s = 0; s < nst; ++s) {
      const int st = s % DAT_ST;
      mbar_wait(&full[st], (s / DAT_ST) & 1);
      const uint8_t* su = smem + st * G::STAGE + G::X;
      uint8_t* sut = smem + st * G::STAGE + G::X + G::U;
      const bool ok = s * DAT_BK + row < P.T;
      const bf16 z = __float2bfloat16_rn(0.f);
#pragma unroll
      for (int c = 0; c < NW / 8; ++c) {
        uint4 v = ok ? reinterpret_cast<const uint4*>(su + row * (NW * 2))[c] : make_uint4(0, 0, 0, 0);
        const bf16* e = reinterpret_cast<const bf16*>(&v);
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int n = c * 8 + i;   // dU^T row n, K = token `row`: atom (row >> 6) of [NW][64]
          *reinterpret_cast<bf16*>(sut + (row >> 6) * (NW * 128) + n * 128 + ((((row & 63) >> 3) ^ (n & 7)) << 4) +
                                   (row & 7) * 2) = n < P.M ? e[i] : z;
        }
      }
      fence_proxy_async();
      __syncwarp();
      if (lane == 0) mbar_arrive(&ut_full[st]);
    }
    mbar_wait(&acc_full, 0);
    tc_fence_after();
    const int k = k0 + row;
#pragma unroll
    for (int c0 = 0; c0 < NW; c0 += 16) {
      uint32_t r[16];
      tmem_ld16(tmem + c0 + ((uint32_t)(q * 32) << 16), r);
      if (k < P.N) {
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          const int m = c0 + i;
          if (m >= P.M) continue;
          const int seg = P.m_seg > 0 ? m / P.m_seg : 0, mr = P.m_seg > 0 ? m % P.m_seg : m;
          if (P.m_valid > 0 && mr >= P.m_valid) continue;
          float* C = seg == 0 ? P.C : seg == 1 ? P.C1 : P.C2;
          C[(size_t)mr * P.ldc + k] = __uint_as_float(r[i]) * P.scale;
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<G::TCOLS>(tmem);
  }
}

}  // namespace

void lora_rows_tiles(const LoraRowsProblem* probs, int n, std::vector<int2>& out) {
  for (int i = 0; i < n; ++i)
    for (int m = 0; m < probs[i].M; m += ROWS_BM) out.push_back(make_int2(i, m));
}
void lora_tokred_tiles(const LoraTokRedProblem* probs, int n, int mt, int nt, std::vector<int4>& out) {
  for (int i = 0; i < n; ++i)
    for (int m = 0; m < probs[i].M; m += mt)
      for (int c = 0; c < probs[i].N; c += nt) out.push_back(make_int4(i, m, c, 0));
}

int lora_rows_run(const LoraRowsProblem* d_probs, const int2* d_tiles, int n_tiles, int max_n, cudaStream_t st) {
  if (n_tiles <= 0) return 0;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(lora_rows_kernel<32>, cudaFuncAttributeMaxDynamicSharedMemorySize, rows_smem_bytes<32>());
    cudaFuncSetAttribute(lora_rows_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, rows_smem_bytes<64>());
    cudaFuncSetAttribute(lora_rows_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, rows_smem_bytes<128>());
    attr = true;
  }
  if (max_n <= 32) lora_rows_kernel<32><<<n_tiles, ROWS_NTH, rows_smem_bytes<32>(), st>>>(d_probs, d_tiles);
  else if (max_n <= 64) lora_rows_kernel<64><<<n_tiles, ROWS_NTH, rows_smem_bytes<64>(), st>>>(d_probs, d_tiles);
  else if (max_n <= 128) lora_rows_kernel<128><<<n_tiles, ROWS_NTH, rows_smem_bytes<128>(), st>>>(d_probs, d_tiles);
  else return -1;
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

int lora_tokred_run(const LoraTokRedProblem* d_probs, const int4* d_tiles, int n_tiles, int mt, int nt, cudaStream_t st) {
  if (n_tiles <= 0) return 0;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(lora_tokred_kernel<128, 16>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         tokred_smem_bytes<128, 16>());
    cudaFuncSetAttribute(lora_tokred_kernel<16, 128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         tokred_smem_bytes<16, 128>());
    cudaFuncSetAttribute(lora_tokred_kernel<32, 128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         tokred_smem_bytes<32, 128>());
    cudaFuncSetAttribute(lora_tokred_kernel<64, 128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         tokred_smem_bytes<64, 128>());

    attr = true;
  }
#define TOKRED_CASE(MT_, NT_) \
  else if (mt == MT_ && nt == NT_) lora_tokred_kernel<MT_, NT_><<<n_tiles, 128, tokred_smem_bytes<MT_, NT_>(), st>>>(d_probs, d_tiles);
  if (false) {}
  TOKRED_CASE(128, 16)
  TOKRED_CASE(16, 128)
  TOKRED_CASE(32, 128)
  TOKRED_CASE(64, 128)
#undef TOKRED_CASE
  else return -1;
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

int lora_dub_run(const LoraDUBProblem* d_probs, int n_probs, int max_slabs, int max_rank, cudaStream_t st) {
  if (n_probs <= 0 || max_slabs <= 0 || max_rank <= 0) return 0;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(lora_dub_kernel<LORA_DUB_MT, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         dub_smem_bytes<LORA_DUB_MT>());
    cudaFuncSetAttribute(lora_dub_kernel<LORA_DUB_MT, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         dub_smem_bytes<LORA_DUB_MT>());
    attr = true;
  }
  const int n_rt = (max_rank + DUB_NT - 1) / DUB_NT;
  const dim3 grid(max_slabs * n_rt, n_probs);
  if (max_rank <= 8) lora_dub_kernel<LORA_DUB_MT, 1><<<grid, 128, dub_smem_bytes<LORA_DUB_MT>(), st>>>(d_probs, n_rt);
  else lora_dub_kernel<LORA_DUB_MT, 2><<<grid, 128, dub_smem_bytes<LORA_DUB_MT>(), st>>>(d_probs, n_rt);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

int lora_du_reduce_run(const LoraDUBProblem* d_probs, int n_probs, long long max_elems, cudaStream_t st) {
  if (n_probs <= 0 || max_elems <= 0) return 0;
  lora_du_reduce_kernel<<<dim3((unsigned)((max_elems + 255) / 256), n_probs), 256, 0, st>>>(d_probs);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

}  // namespace menos

namespace menos {
bool tma_map_2d(CUtensorMap* out, const void* ptr, uint64_t rows, uint64_t cols, uint64_t ld, uint32_t bc,
                uint32_t br);
bool tma_map_2d_plain(CUtensorMap* out, const void* ptr, uint64_t rows, uint64_t cols, uint64_t ld, uint32_t bc,
                      uint32_t br);

template <int NW, int STG>
static int da_tc_launch(const CUtensorMap& mX, const CUtensorMap& mU, const LoraTokRedProblem* d_probs, int n_probs,
                        int max_n, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(lora_da_tc_kernel<NW, STG>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         DatGeo<NW, STG>::SMEM);
    attr = true;
  }
  lora_da_tc_kernel<NW, STG><<<dim3((max_n + 127) / 128, n_probs), 192, DatGeo<NW, STG>::SMEM, st>>>(mX, mU, d_probs);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

int lora_da_tc_run(const LoraTokRedProblem* d_probs, int n_probs, int max_n, int max_w, const bf16* X, int rows,
                   int ldx, const bf16* dU, int lddu, cudaStream_t st) {
  if (n_probs <= 0 || max_n <= 0) return 0;
  const int NW = max_w <= 16 ? 16 : max_w <= 32 ? 32 : max_w <= 64 ? 64 : -1;
  if (NW < 0 || ldx % 8 || lddu % 8) return -1;
  CUtensorMap mX, mU;
  if (!tma_map_2d(&mX, X, rows, max_n, ldx, 64, 128)) return -2;
  if (!tma_map_2d_plain(&mU, dU, rows, lddu, lddu, NW, 128)) return -2;
  int sms = 148, dev = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const bool deep = (long long)((max_n + 127) / 128) * n_probs < 2LL * sms;
  if (NW == 16) return deep ? da_tc_launch<16, 4>(mX, mU, d_probs, n_probs, max_n, st)
                            : da_tc_launch<16, 2>(mX, mU, d_probs, n_probs, max_n, st);
  if (NW == 32) return deep ? da_tc_launch<32, 4>(mX, mU, d_probs, n_probs, max_n, st)
                            : da_tc_launch<32, 2>(mX, mU, d_probs, n_probs, max_n, st);
  return deep ? da_tc_launch<64, 3>(mX, mU, d_probs, n_probs, max_n, st)
              : da_tc_launch<64, 2>(mX, mU, d_probs, n_probs, max_n, st);
}

int lora_dub_tc_run(const LoraDUBProblem* d_probs, int n_probs, int max_slabs, const bf16* dY, int y_rows, int ldy,
                    const bf16* U, int ldu, int mts, cudaStream_t st) {
  if (n_probs <= 0 || max_slabs <= 0) return 0;
  if (ldy % 8 || ldu % 8 || (mts != 128 && mts != 256)) return -1;
  CUtensorMap mY, mU;
  if (!tma_map_2d(&mY, dY, y_rows, ldy, ldy, 64, 128)) return -2;
  if (!tma_map_2d_plain(&mU, U, y_rows, ldu, ldu, 16, 128)) return -2;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(lora_dub_tc_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, DubtGeo<128>::SMEM);
    cudaFuncSetAttribute(lora_dub_tc_kernel<256>, cudaFuncAttributeMaxDynamicSharedMemorySize, DubtGeo<256>::SMEM);
    attr = true;
  }
  if (mts == 256) lora_dub_tc_kernel<256><<<dim3(max_slabs, n_probs), 192, DubtGeo<256>::SMEM, st>>>(mY, mU, d_probs);
  else lora_dub_tc_kernel<128><<<dim3(max_slabs, n_probs), 192, DubtGeo<128>::SMEM, st>>>(mY, mU, d_probs);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

void lora_shrink_tiles(const LoraShrinkProblem* probs, int n, std::vector<int2>& out) {
  for (int i = 0; i < n; ++i)
    for (int m = 0; m < probs[i].T; m += 128) out.push_back(make_int2(i, m));
}

template <int N>
static int shrink_launch(const CUtensorMap& mX, const CUtensorMap& mA, const LoraShrinkProblem* d_probs,
                         const int2* d_tiles, int n_tiles, int K, bf16* U, int ldu, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(lora_shrink_tc_kernel<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, ShkGeo<N>::SMEM);
    attr = true;
  }
  lora_shrink_tc_kernel<N><<<n_tiles, 192, ShkGeo<N>::SMEM, st>>>(mX, mA, d_probs, d_tiles, K, U, ldu);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

int lora_shrink_tc_run(const bf16* X, int x_rows, int ldx, const bf16* Acat, int a_rows, int lda, int K,
                       const LoraShrinkProblem* d_probs, const int2* d_tiles, int n_tiles, int max_w, bf16* U, int ldu,
                       cudaStream_t st) {
  if (n_tiles <= 0) return 0;
  const int N = max_w <= 16 ? 16 : max_w <= 32 ? 32 : max_w <= 64 ? 64 : max_w <= 128 ? 128 : -1;
  if (N < 0 || ldx % 8 || lda % 8 || ldu % 8) return -1;   // TMA: 16-byte row strides; any K (OOB columns read 0)
  CUtensorMap mX, mA;
  if (!tma_map_2d(&mX, X, x_rows, K, ldx, SHK_BK, 128)) return -2;
  if (!tma_map_2d(&mA, Acat, a_rows, K, lda, SHK_BK, N)) return -2;
  switch (N) {
    case 16: return shrink_launch<16>(mX, mA, d_probs, d_tiles, n_tiles, K, U, ldu, st);
    case 32: return shrink_launch<32>(mX, mA, d_probs, d_tiles, n_tiles, K, U, ldu, st);
    case 64: return shrink_launch<64>(mX, mA, d_probs, d_tiles, n_tiles, K, U, ldu, st);
    default: return shrink_launch<128>(mX, mA, d_probs, d_tiles, n_tiles, K, U, ldu, st);
  }
}
}  // namespace menos
