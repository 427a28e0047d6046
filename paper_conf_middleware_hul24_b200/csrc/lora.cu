// Segmented multi-client LoRA side GEMMs (SURVEY.md §8(a) A2/A4/A6/A7 shrink, A8-A12 LoRA backward):
//   shrink   U_c  = s_c * X_c A_c^T          (bf16 block-diagonal operand of the GEMM's extra-K segment)
//   dU       dU_c = s_c * dY_c B_c            (operand of the dX GEMM's extra-K segment, and of dA)
//   dB       dB_c = s_c * dY_c^T U_c          (fp32, reduced over the client's tokens only)
//   dA       dA_c = dU_c^T X_c                (fp32, reduced over the client's tokens only)
// Every problem is one client's token segment; every output tile is owned by one CTA that loops over the
// whole reduction in a fixed order, so results are deterministic and never mix clients.
// These are tiny contractions (rank r <= 16); they run on mma.sync tensor cores with smem staging.
#include "common.cuh"
#include "kernels.h"

namespace menos {
namespace {

constexpr int BM = 64, BN = 64, BKK = 32, PAD = 8;

__global__ void __launch_bounds__(128) small_gemm_kernel(const SmallGemmProblem* __restrict__ probs,
                                                         const int4* __restrict__ tiles) {
  __shared__ __align__(16) bf16 As[BM][BKK + PAD];
  __shared__ __align__(16) bf16 Bs[BN][BKK + PAD];
  const int4 tl = tiles[blockIdx.x];
  const SmallGemmProblem P = probs[tl.x];
  const int m0 = tl.y, n0 = tl.z;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int wm = (warp >> 1) * 32, wn = (warp & 1) * 32;
  const int g = lane >> 2, t = lane & 3;
  float acc[2][4][4];
#pragma unroll
  for (int i = 0; i < 2; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int k = 0; k < 4; ++k) acc[i][j][k] = 0.f;

  const bf16 zero = __float2bfloat16_rn(0.f);
  for (int k0 = 0; k0 < P.K; k0 += BKK) {
    // stage A tile [BM][BKK] and B tile [BN][BKK] (K contiguous in smem), coalesced along the source's fast dim
    for (int idx = tid; idx < BM * BKK; idx += 128) {
      int m, k;
      if (!P.a_t) { m = idx / BKK; k = idx % BKK; } else { k = idx / BM; m = idx % BM; }
      const int gm = m0 + m, gk = k0 + k;
      bf16 v = zero;
      if (gm < P.M && gk < P.K) {
        if (P.a_t) {
          const int mm = (gm / P.a_blk) * P.a_blk_stride + gm % P.a_blk;
          v = P.A[(size_t)gk * P.lda + mm];
        } else {
          v = P.A[(size_t)gm * P.lda + gk];
        }
      }
      As[m][k] = v;
    }
    for (int idx = tid; idx < BN * BKK; idx += 128) {
      int n, k;
      if (!P.b_t) { n = idx / BKK; k = idx % BKK; } else { k = idx / BN; n = idx % BN; }
      const int gn = n0 + n, gk = k0 + k;
      bf16 v = zero;
      if (gn < P.N && gk < P.K) v = P.b_t ? P.B[(size_t)gk * P.ldb + gn] : P.B[(size_t)gn * P.ldb + gk];
      Bs[n][k] = v;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < BKK; kk += 16) {
      uint32_t a[2][4];
#pragma unroll
      for (int i = 0; i < 2; ++i) {
        const int r = wm + i * 16 + g;
        a[i][0] = *reinterpret_cast<const uint32_t*>(&As[r][kk + 2 * t]);
        a[i][1] = *reinterpret_cast<const uint32_t*>(&As[r + 8][kk + 2 * t]);
        a[i][2] = *reinterpret_cast<const uint32_t*>(&As[r][kk + 2 * t + 8]);
        a[i][3] = *reinterpret_cast<const uint32_t*>(&As[r + 8][kk + 2 * t + 8]);
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int c = wn + j * 8 + g;
        const uint32_t b0 = *reinterpret_cast<const uint32_t*>(&Bs[c][kk + 2 * t]);
        const uint32_t b1 = *reinterpret_cast<const uint32_t*>(&Bs[c][kk + 2 * t + 8]);
#pragma unroll
        for (int i = 0; i < 2; ++i) mma_bf16_16816(acc[i][j], a[i], b0, b1);
      }
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 2; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int r = m0 + wm + i * 16 + g + h * 8;
        const int c = n0 + wn + j * 8 + 2 * t;
        if (r >= P.M) continue;
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          if (c + e >= P.N) continue;
          const float v = acc[i][j][2 * h + e] * P.scale;
          if (P.Cf) P.Cf[(size_t)r * P.ldc + c + e] = v;
          if (P.Cb) P.Cb[(size_t)r * P.ldc + c + e] = __float2bfloat16_rn(v);
        }
      }
}

}  // namespace

void small_gemm_tiles(const SmallGemmProblem* probs, int n, int4* out, int* n_out) {
  int k = 0;
  for (int i = 0; i < n; ++i)
    for (int m = 0; m < probs[i].M; m += BM)
      for (int c = 0; c < probs[i].N; c += BN) out[k++] = make_int4(i, m, c, 0);
  *n_out = k;
}

int small_gemm_run(const SmallGemmProblem* d_probs, const int4* d_tiles, int n_tiles, cudaStream_t st) {
  if (n_tiles <= 0) return 0;
  small_gemm_kernel<<<n_tiles, 128, 0, st>>>(d_probs, d_tiles);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

}  // namespace menos
