// Prefix-tuning adapters (§2.1 and :121 §3.1; Li & Liang [16]; R28).
//
// A prefix client's P learned key / value vectors per layer join every one of its sequences' attention.  The varlen
// causal attention kernels are reused unchanged on an EXTENDED batch: each such sequence is preceded by P rows whose
// k, v are the layer's prefix (q = 0), so "causal over [prefix | sequence]" is exactly "every query sees the whole
// prefix plus its causal keys"; the prefix rows' own outputs are dropped and their incoming gradient is zero, so
// they contribute nothing else.  The kernels below move rows between the batch and its extension:
//   prefix_gather    qkv -> qkv_ext (sequence rows copied, prefix rows from the client's bf16 prefix table)
//   rows_map         dst[r] = src[map[r]] or 0 (O_ext -> O, dO -> dO_ext; bf16 rows)
//   lse_map          D / lse per head [H, n] under the same row map (fp32)
//   dqkv_from_ext    dqkv rows <- dqkv_ext rows with the RoPE backward on q and k (the attention backward runs on the
//                    extension without RoPE: prefix keys are not rotated, R28)
//   prefix_grad      dPk, dPv of every (prefix client, layer): the client's sequences' prefix-row dk, dv summed in
//                    sequence order (fixed order: deterministic), fp32, overwriting the client's gradient buffer.
#include "common.cuh"
#include "kernels.h"

namespace menos {

namespace {

__global__ void prefix_gather_kernel(const bf16* __restrict__ qkv, int ld, const int2* __restrict__ src, int n_rows,
                                     const PrefixClient* __restrict__ pc, int layer, int Nq, int Nkv,
                                     bf16* __restrict__ out) {
  const int Nqkv = Nq + 2 * Nkv, v8 = Nqkv / 8;
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < (long long)n_rows * v8;
       e += (long long)gridDim.x * blockDim.x) {
    const int r = (int)(e / v8), c = (int)(e % v8) * 8;
    const int2 s = src[r];
    uint4 v = make_uint4(0, 0, 0, 0);
    if (s.x >= 0) {
      v = *reinterpret_cast<const uint4*>(qkv + (size_t)s.x * ld + c);
    } else if (c >= Nq) {   // prefix row p of batch client k: q = 0, k / v from the layer's table
      const PrefixClient P = pc[s.y >> 16];
      const int p = s.y & 0xFFFF;
      const bf16* tab = P.table + (size_t)(layer - P.first_layer) * 2 * P.n * Nkv;
      const int kv = c < Nq + Nkv ? 0 : 1, col = c - Nq - kv * Nkv;
      v = *reinterpret_cast<const uint4*>(tab + ((size_t)kv * P.n + p) * Nkv + col);
    }
    *reinterpret_cast<uint4*>(out + (size_t)r * Nqkv + c) = v;
  }
}

__global__ void rows_map_kernel(const bf16* __restrict__ src, int lds, const int* __restrict__ map, int n_rows,
                                int width, bf16* __restrict__ dst, int ldd) {
  const int v8 = width / 8;
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < (long long)n_rows * v8;
       e += (long long)gridDim.x * blockDim.x) {
    const int r = (int)(e / v8), c = (int)(e % v8) * 8;
    const int m = map[r];
    const uint4 v = m >= 0 ? *reinterpret_cast<const uint4*>(src + (size_t)m * lds + c) : make_uint4(0, 0, 0, 0);
    *reinterpret_cast<uint4*>(dst + (size_t)r * ldd + c) = v;
  }
}

__global__ void lse_map_kernel(const float* __restrict__ src, int n_src, const int* __restrict__ map, int n_rows, int H,
                               float* __restrict__ dst) {
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < (long long)n_rows * H;
       e += (long long)gridDim.x * blockDim.x) {
    const int h = (int)(e / n_rows), r = (int)(e % n_rows);
    const int m = map[r];
    dst[(size_t)h * n_rows + r] = m >= 0 ? src[(size_t)h * n_src + m] : 0.f;
  }
}

// one thread per (token, RoPE pair (i, i + hd/2) of one head of q or k) or per 8 v columns
__global__ void dqkv_from_ext_kernel(const bf16* __restrict__ ext, const int* __restrict__ ext_row, int T, int H,
                                     int Hkv, int hd, const float2* __restrict__ cs, const int* __restrict__ pos,
                                     bf16* __restrict__ dqkv) {
  const int Nq = H * hd, Nkv = Hkv * hd, Nqkv = Nq + 2 * Nkv, half = hd / 2;
  const int rot = (H + Hkv) * half;   // rotated pairs per row
  const int per_row = rot + Nkv / 8;
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < (long long)T * per_row;
       e += (long long)gridDim.x * blockDim.x) {
    const int t = (int)(e / per_row), k = (int)(e % per_row);
    const bf16* s = ext + (size_t)ext_row[t] * Nqkv;
    bf16* d = dqkv + (size_t)t * Nqkv;
    if (k < rot) {
      const int head = k / half, i = k % half, c0 = head * hd + i;   // q heads, then k heads (contiguous)
      const float x = bf2f(s[c0]), y = bf2f(s[c0 + half]);
      if (cs) {   // dx_i = dy_i c + dy_{i+half} s ; dx_{i+half} = dy_{i+half} c - dy_i s
        const float2 e2 = cs[(size_t)pos[t] * half + i];
        d[c0] = f2bf(x * e2.x + y * e2.y);
        d[c0 + half] = f2bf(y * e2.x - x * e2.y);
      } else {
        d[c0] = s[c0];
        d[c0 + half] = s[c0 + half];
      }
    } else {
      const int c = Nq + Nkv + (k - rot) * 8;
      *reinterpret_cast<uint4*>(d + c) = *reinterpret_cast<const uint4*>(s + c);
    }
  }
}

// grid: x over (client slot, p, column chunk of 256); dPk / dPv [P, Nkv] of one layer = sum over the client's sequences
__global__ void prefix_grad_kernel(const bf16* __restrict__ dqkv_ext, int Nq, int Nkv, const PrefixClient* __restrict__ pc,
                                   int n_pc, const int* __restrict__ seq_ext0, int layer) {
  const int chunks = (Nkv + 255) / 256;
  int b = blockIdx.x;
  // locate (client slot k, prefix row p, column chunk)
  int k = 0;
  for (; k < n_pc; ++k) {
    const int nb = pc[k].n * chunks;
    if (b < nb) break;
    b -= nb;
  }
  if (k >= n_pc) return;
  const PrefixClient P = pc[k];
  if (layer < P.first_layer) return;
  const int p = b / chunks, col = (b % chunks) * 256 + threadIdx.x;
  if (col >= Nkv) return;
  const int Nqkv = Nq + 2 * Nkv;
  float sk = 0.f, sv = 0.f;
  for (int i = P.seq0; i < P.seq1; ++i) {   // the client's sequences, in batch order
    const bf16* row = dqkv_ext + (size_t)(seq_ext0[i] + p) * Nqkv;
    sk += bf2f(row[Nq + col]);
    sv += bf2f(row[Nq + Nkv + col]);
  }
  float* g = P.grad + (size_t)(layer - P.first_layer) * 2 * P.n * Nkv;
  g[(size_t)p * Nkv + col] = sk;
  g[((size_t)P.n + p) * Nkv + col] = sv;
}

inline int grid_for(long long n) { return (int)std::min<long long>(std::max<long long>((n + 255) / 256, 1), 4 * 148 * 8); }

}  // namespace

#define PFX_LAUNCH_CHECK() (++g_launch_count, cudaPeekAtLastError() == cudaSuccess ? 0 : -3)

int prefix_gather(const bf16* qkv, int ld, const int2* src, int n_rows, const PrefixClient* pc, int layer, int Nq,
                  int Nkv, bf16* out, cudaStream_t st) {
  if (n_rows <= 0) return 0;
  if ((Nq + 2 * Nkv) % 8 || ld % 8) return -1;
  prefix_gather_kernel<<<grid_for((long long)n_rows * (Nq + 2 * Nkv) / 8), 256, 0, st>>>(qkv, ld, src, n_rows, pc,
                                                                                         layer, Nq, Nkv, out);
  return PFX_LAUNCH_CHECK();
}
int rows_map(const bf16* src, int lds, const int* map, int n_rows, int width, bf16* dst, int ldd, cudaStream_t st) {
  if (n_rows <= 0) return 0;
  if (width % 8 || lds % 8 || ldd % 8) return -1;
  rows_map_kernel<<<grid_for((long long)n_rows * width / 8), 256, 0, st>>>(src, lds, map, n_rows, width, dst, ldd);
  return PFX_LAUNCH_CHECK();
}
int lse_map(const float* src, int n_src, const int* map, int n_rows, int H, float* dst, cudaStream_t st) {
  if (n_rows <= 0) return 0;
  lse_map_kernel<<<grid_for((long long)n_rows * H), 256, 0, st>>>(src, n_src, map, n_rows, H, dst);
  return PFX_LAUNCH_CHECK();
}
int dqkv_from_ext(const bf16* ext, const int* ext_row, int T, int H, int Hkv, int hd, const float2* cs, const int* pos,
                  bf16* dqkv, cudaStream_t st) {
  if (T <= 0) return 0;
  const long long n = (long long)T * ((H + Hkv) * (hd / 2) + Hkv * hd / 8);
  dqkv_from_ext_kernel<<<grid_for(n), 256, 0, st>>>(ext, ext_row, T, H, Hkv, hd, cs, pos, dqkv);
  return PFX_LAUNCH_CHECK();
}
int prefix_grad(const bf16* dqkv_ext, int Nq, int Nkv, const PrefixClient* pc, int n_pc, int total_rows,
                const int* seq_ext0, int layer, cudaStream_t st) {
  if (n_pc <= 0 || total_rows <= 0) return 0;
  const int chunks = (Nkv + 255) / 256;
  prefix_grad_kernel<<<total_rows * chunks, 256, 0, st>>>(dqkv_ext, Nq, Nkv, pc, n_pc, seq_ext0, layer);
  return PFX_LAUNCH_CHECK();
}

}  // namespace menos
