// HBM-bound row kernels: RMSNorm fwd/bwd, attention-backward row sums
// (A11 prologue), fused multi-tensor AdamW over all stepped clients' adapters (A13, Alg.1 L12),
// RoPE table.  One warp per row, 16-byte vector loads, warp-shuffle fp32 reductions.
#include <type_traits>
#include "common.cuh"
#include "kernels.h"

namespace menos {

unsigned long long g_launch_count = 0;

namespace {

// 8 consecutive fp32 values / bf16 values <-> registers
__device__ __forceinline__ void ld8f(const float* p, float (&v)[8]) {
  const float4 a = reinterpret_cast<const float4*>(p)[0], b = reinterpret_cast<const float4*>(p)[1];
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}
__device__ __forceinline__ void st8f(float* p, const float (&v)[8]) {
  reinterpret_cast<float4*>(p)[0] = make_float4(v[0], v[1], v[2], v[3]);
  reinterpret_cast<float4*>(p)[1] = make_float4(v[4], v[5], v[6], v[7]);
}
__device__ __forceinline__ void ld8b(const bf16* p, float (&v)[8]) {
  const uint4 u = *reinterpret_cast<const uint4*>(p);
  float2 a = unpack_bf16x2(u.x), b = unpack_bf16x2(u.y), c = unpack_bf16x2(u.z), e = unpack_bf16x2(u.w);
  v[0] = a.x; v[1] = a.y; v[2] = b.x; v[3] = b.y; v[4] = c.x; v[5] = c.y; v[6] = e.x; v[7] = e.y;
}
__device__ __forceinline__ void st8b(bf16* p, const float (&v)[8]) {
  *reinterpret_cast<uint4*>(p) = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]),
                                            pack_bf16x2(v[4], v[5]), pack_bf16x2(v[6], v[7]));
}
__device__ __forceinline__ void ld8(const bf16* p, float (&v)[8]) { ld8b(p, v); }
__device__ __forceinline__ void ld8(const float* p, float (&v)[8]) { ld8f(p, v); }

// ------------------------------------------------------------------ RMSNorm forward
// y = x * rstd * g, rstd = rsqrt(mean(x^2) + eps); x fp32 residual stream [T, d]; y bf16 (GEMM operand);
// g fp32 [d]; d % 8 == 0
__global__ void rmsnorm_fwd_kernel(const float* __restrict__ x, const float* __restrict__ g, bf16* __restrict__ y,
                                   float* __restrict__ rstd, int T, int d, float eps) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= T) return;
  const float* xr = x + (size_t)warp * d;
  float ss = 0.f;
  for (int i = lane * 8; i < d; i += 256) {
    float v[8];
    ld8f(xr + i, v);
#pragma unroll
    for (int k = 0; k < 8; ++k) ss += v[k] * v[k];
  }
  ss = warp_sum(ss);
  const float r = rsqrtf(ss / (float)d + eps);
  if (lane == 0) rstd[warp] = r;
  bf16* yr = y + (size_t)warp * d;
  for (int i = lane * 8; i < d; i += 256) {
    float v[8], gg[8];
    ld8f(xr + i, v);
    ld8f(g + i, gg);
#pragma unroll
    for (int k = 0; k < 8; ++k) v[k] = v[k] * r * gg[k];
    st8b(yr + i, v);
  }
}

// ------------------------------------------------------------------ RMSNorm backward (+ residual)
// dx = resid + rstd*(gh - xh*mean(gh*xh)),  gh = dy*g,  xh = x*rstd.   dy bf16 (GEMM output), x / resid / dx
// fp32 (residual streams); dxb = bf16 copy of dx for the next dX GEMM's A operand (optional).
template <typename TDY>
__global__ void rmsnorm_bwd_kernel(const TDY* __restrict__ dy, const float* __restrict__ x,
                                   const float* __restrict__ g, const float* __restrict__ rstd,
                                   const float* __restrict__ resid, float* __restrict__ dx, bf16* __restrict__ dxb,
                                   int T, int d) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= T) return;
  const size_t ro = (size_t)warp * d;
  const float r = rstd[warp];
  float dot = 0.f;
  for (int i = lane * 8; i < d; i += 256) {
    float a[8], b[8], gg[8];
    ld8(dy + ro + i, a);
    ld8f(x + ro + i, b);
    ld8f(g + i, gg);
#pragma unroll
    for (int k = 0; k < 8; ++k) dot += a[k] * gg[k] * b[k];
  }
  dot = warp_sum(dot);
  const float mean = dot * r / (float)d;  // mean(gh * xh) = r * mean(gh * x)
  for (int i = lane * 8; i < d; i += 256) {
    float a[8], b[8], c[8], gg[8], o[8];
    ld8(dy + ro + i, a);
    ld8f(x + ro + i, b);
    ld8f(resid + ro + i, c);
    ld8f(g + i, gg);
#pragma unroll
    for (int k = 0; k < 8; ++k) o[k] = c[k] + r * (a[k] * gg[k] - b[k] * r * mean);
    st8f(dx + ro + i, o);
    if (dxb) st8b(dxb + ro + i, o);
  }
}

// ------------------------------------------------------------------ single-pass RMSNorm (row cached in registers)
// TPR threads per row (128, or 256 for wide rows such as d = 8192), 8-element chunks, up to NC chunks per thread
// (d <= TPR * 8 * NC); block = 256 threads = 256 / TPR rows.
template <int TPR>
__device__ __forceinline__ float block_row_sum(float v, float* red, int wr) {
  // reduce over the TPR / 32 warps of this row's threads (fixed order)
  constexpr int W = TPR / 32;
  v = warp_sum(v);
  const int lane = threadIdx.x & 31, w = (threadIdx.x % TPR) >> 5;
  if (lane == 0) red[wr * W + w] = v;
  __syncthreads();
  float s = red[wr * W];
#pragma unroll
  for (int k = 1; k < W; ++k) s += red[wr * W + k];
  return s;
}

template <int NC, int TPR>
__global__ void __launch_bounds__(256) rmsnorm_fwd_reg_kernel(const float* __restrict__ x, const float* __restrict__ g,
                                                              bf16* __restrict__ y, float* __restrict__ rstd, int T,
                                                              int d, float eps) {
  __shared__ float red[8];
  const int wr = threadIdx.x / TPR, t = threadIdx.x % TPR;
  const int row = blockIdx.x * (256 / TPR) + wr;
  const bool ok = row < T;
  const float* xr = x + (size_t)(ok ? row : 0) * d;
  float v[NC][8];
  float ss = 0.f;
#pragma unroll
  for (int c = 0; c < NC; ++c) {
    const int i = (c * TPR + t) * 8;
    if (ok && i < d) {
      ld8f(xr + i, v[c]);
#pragma unroll
      for (int k = 0; k < 8; ++k) ss += v[c][k] * v[c][k];
    }
  }
  ss = block_row_sum<TPR>(ss, red, wr);
  const float r = rsqrtf(ss / (float)d + eps);
  if (!ok) return;
  if (t == 0) rstd[row] = r;
  bf16* yr = y + (size_t)row * d;
#pragma unroll
  for (int c = 0; c < NC; ++c) {
    const int i = (c * TPR + t) * 8;
    if (i < d) {
      float gg[8];
      ld8f(g + i, gg);
#pragma unroll
      for (int k = 0; k < 8; ++k) v[c][k] = v[c][k] * r * gg[k];
      st8b(yr + i, v[c]);
    }
  }
}

template <int NC, int TPR, typename TDY>
__global__ void __launch_bounds__(256) rmsnorm_bwd_reg_kernel(const TDY* __restrict__ dy, const float* __restrict__ x,
                                                              const float* __restrict__ g, const float* __restrict__ rstd,
                                                              const float* __restrict__ resid, float* __restrict__ dx,
                                                              bf16* __restrict__ dxb, int T, int d) {
  __shared__ float red[8];
  const int wr = threadIdx.x / TPR, t = threadIdx.x % TPR;
  const int row = blockIdx.x * (256 / TPR) + wr;
  const bool ok = row < T;
  const size_t ro = (size_t)(ok ? row : 0) * d;
  const float r = ok ? rstd[row] : 0.f;
  float a[NC][8], b[NC][8], res[NC][8];
  float dot = 0.f;
#pragma unroll
  for (int c = 0; c < NC; ++c) {
    const int i = (c * TPR + t) * 8;
    if (ok && i < d) {
      float gg[8];
      ld8(dy + ro + i, a[c]);
      ld8f(x + ro + i, b[c]);
      ld8f(resid + ro + i, res[c]);   // issued with the others: its latency overlaps the row reduction
      ld8f(g + i, gg);
#pragma unroll
      for (int k = 0; k < 8; ++k) { a[c][k] *= gg[k]; dot += a[c][k] * b[c][k]; }   // a = gh = dy * g
    }
  }
  dot = block_row_sum<TPR>(dot, red, wr);
  if (!ok) return;
  const float mean = dot * r / (float)d;
#pragma unroll
  for (int c = 0; c < NC; ++c) {
    const int i = (c * TPR + t) * 8;
    if (i < d) {
      float o[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) o[k] = res[c][k] + r * (a[c][k] - b[c][k] * r * mean);
      st8f(dx + ro + i, o);
      if (dxb) st8b(dxb + ro + i, o);
    }
  }
}

__global__ void f32_to_bf16_kernel(const float* __restrict__ s, bf16* __restrict__ d, long long n8) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n8; i += (long long)gridDim.x * blockDim.x) {
    float v[8];
    ld8f(s + 8 * i, v);
    st8b(d + 8 * i, v);
  }
}
__global__ void bf16_to_f32_vec_kernel(const bf16* __restrict__ s, float* __restrict__ d, long long n8) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n8; i += (long long)gridDim.x * blockDim.x) {
    float v[8];
    ld8b(s + 8 * i, v);
    st8f(d + 8 * i, v);
  }
}
// out = x + float(delta): the sequence-parallel residual add after a reduce-scatter (A16); x, out fp32, delta bf16
__global__ void add_bf16_f32_kernel(const float* x, const bf16* __restrict__ delta, float* out,
                                    long long n8) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n8; i += (long long)gridDim.x * blockDim.x) {
    float a[8], b[8];
    ld8f(x + 8 * i, a);
    ld8b(delta + 8 * i, b);
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] += b[k];
    st8f(out + 8 * i, a);
  }
}

// ------------------------------------------------------------------ D = rowsum(dO * O) per (token, head)
__global__ void attn_prep_kernel(const bf16* __restrict__ dO, const bf16* __restrict__ O, float* __restrict__ D,
                                 int T, int H, int hd) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= T * H) return;
  const int t = warp / H, h = warp % H;
  const bf16* a = dO + (size_t)t * H * hd + h * hd;
  const bf16* b = O + (size_t)t * H * hd + h * hd;
  float s = 0.f;
  for (int i = lane * 2; i < hd; i += 64) {
    float2 x = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(a + i));
    float2 y = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(b + i));
    s += x.x * y.x + x.y * y.y;
  }
  s = warp_sum(s);
  if (lane == 0) D[(size_t)h * T + t] = s;
}

// ------------------------------------------------------------------ AdamW (torch semantics) + bf16 refresh
// work item = (segment, start, len, 0); one CTA per work item.
__global__ void adamw_kernel(const AdamSeg* __restrict__ segs, const int4* __restrict__ work,
                             const AdamHyper* __restrict__ hyp) {
  const int4 w = work[blockIdx.x];
  const AdamSeg sg = segs[w.x];
  const AdamHyper hp = hyp[sg.client];
  // 4 elements per thread with 16-byte loads / stores when the block, its row length and the bf16 copy allow it
  // (the same fp32 operations per element as the scalar loop below: results are bitwise identical)
  const bool vec = (sg.p_off & 3) == 0 && (sg.cols & 3) == 0 && (w.y & 3) == 0 && (w.z & 3) == 0 &&
                   (sg.dst_ld & 3) == 0 && (reinterpret_cast<uintptr_t>(sg.dst) & 7) == 0;
  if (vec) {
    for (int e = w.y + 4 * threadIdx.x; e < w.y + w.z; e += 4 * blockDim.x) {
      const long long i = sg.p_off + e;
      float4 p = *reinterpret_cast<const float4*>(hp.p + i);
      if (hp.do_update) {
        const float4 g = *reinterpret_cast<const float4*>(hp.g + i);
        float4 m = *reinterpret_cast<const float4*>(hp.m + i), v = *reinterpret_cast<const float4*>(hp.v + i);
        float* pp = &p.x; const float* gg = &g.x; float* mm = &m.x; float* vv = &v.x;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          pp[k] = pp[k] * hp.decay;
          mm[k] = hp.beta1 * mm[k] + hp.omb1 * gg[k];
          vv[k] = hp.beta2 * vv[k] + hp.omb2 * (gg[k] * gg[k]);
          const float denom = sqrtf(vv[k]) / hp.bc2_sqrt + hp.eps;
          pp[k] = pp[k] - hp.step_size * (mm[k] / denom);
        }
        *reinterpret_cast<float4*>(hp.p + i) = p; *reinterpret_cast<float4*>(hp.m + i) = m;
        *reinterpret_cast<float4*>(hp.v + i) = v; *reinterpret_cast<float4*>(hp.g + i) = make_float4(0.f, 0.f, 0.f, 0.f);
      }
      const int rr = e / sg.cols, cc = e % sg.cols;   // the 4 elements share a row (cols % 4 == 0)
      const size_t drow = !sg.is_b ? (size_t)rr
                                   : (size_t)(sg.row_base + (rr / sg.row_blk) * sg.row_blk_stride + rr % sg.row_blk);
      *reinterpret_cast<uint2*>(sg.dst + drow * sg.dst_ld + cc) = make_uint2(pack_bf16x2(p.x, p.y), pack_bf16x2(p.z, p.w));
    }
    return;
  }
  for (int e = w.y + threadIdx.x; e < w.y + w.z; e += blockDim.x) {
    const long long i = sg.p_off + e;
    float p = hp.p[i];
    if (hp.do_update) {
      const float g = hp.g[i];
      float m = hp.m[i], v = hp.v[i];
      p = p * hp.decay;
      m = hp.beta1 * m + hp.omb1 * g;
      v = hp.beta2 * v + hp.omb2 * (g * g);
      const float denom = sqrtf(v) / hp.bc2_sqrt + hp.eps;
      p = p - hp.step_size * (m / denom);
      hp.p[i] = p; hp.m[i] = m; hp.v[i] = v; hp.g[i] = 0.f;
    }
    const int rr = e / sg.cols, cc = e % sg.cols;
    size_t dst;
    if (!sg.is_b) {
      dst = (size_t)rr * sg.dst_ld + cc;
    } else {
      const int drow = sg.row_base + (rr / sg.row_blk) * sg.row_blk_stride + rr % sg.row_blk;
      dst = (size_t)drow * sg.dst_ld + cc;
    }
    sg.dst[dst] = __float2bfloat16_rn(p);
  }
}

__global__ void rope_table_kernel(float2* cs, int max_pos, int hd, float theta) {
  const int half = hd / 2;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= max_pos * half) return;
  const int p = idx / half, i = idx % half;
  // inv_freq and angle in fp32 (HF convention), cos/sin evaluated accurately (fp64) then rounded
  const float ex = (float)(2 * i) / (float)hd;                 // arange(0, hd, 2) / hd in fp32
  const float pw = (float)pow((double)theta, (double)ex);        // theta ** ex, correctly rounded to fp32
  const float inv_freq = 1.0f / pw;
  const float ang = (float)p * inv_freq;
  cs[idx] = make_float2((float)cos((double)ang), (float)sin((double)ang));
}

__global__ void bf16_to_f32_kernel(const bf16* __restrict__ s, float* __restrict__ d, long long n) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    d[i] = __bfloat162float(s[i]);
}

// ------------------------------------------------------------------ LayerNorm (OPT, NEXT-4)
// WPR warps per row, the row cached in registers (NCH 8-element chunks per lane, d <= 256 * WPR * NCH), two-pass
// statistics in fp32.  fwd: y = (x - mu) * rstd * g + b.  bwd (+ residual; g, b frozen so no dg, db):
// dx = resid + rstd * (gh - mean(gh) - xh * mean(gh * xh)), gh = dy * g, xh = (x - mu) * rstd; mu and rstd are
// recomputed from x with the forward's own reduction order.
// WPR warps per row (1 for d <= 1024, 2 above: d = 2048 at one warp per row held 215 registers in the backward,
// one CTA per SM); the row sums go warp_sum -> shared slots of the row's warps (fixed order), the same helper in
// fwd and bwd so the backward's recomputed mu / rstd equal the forward's bit for bit.
// the row's WPR warps synchronise on their own named barrier (1 + the row's index in the CTA), not the whole CTA:
// the rows of a CTA do not wait for each other (same summation order as before: results unchanged)
template <int WPR>
__device__ __forceinline__ void ln_row_bar() {
  const int id = 1 + (int)(threadIdx.x >> 5) / WPR;
  asm volatile("bar.sync %0, %1;" ::"r"(id), "n"(32 * WPR) : "memory");
}
template <int WPR>
__device__ __forceinline__ float ln_row_sum(float v, float* red) {
  v = warp_sum(v);
  if constexpr (WPR == 1) {
    return v;
  } else {
    const int w = threadIdx.x >> 5, base = (w / WPR) * WPR;
    if ((threadIdx.x & 31) == 0) red[w] = v;
    ln_row_bar<WPR>();
    float s = red[base];
#pragma unroll
    for (int k = 1; k < WPR; ++k) s += red[base + k];
    ln_row_bar<WPR>();   // red is reused by the next reduction
    return s;
  }
}
// two row sums in one exchange (the backward's mean(gh) and mean(gh * xh)); each in the order ln_row_sum uses
template <int WPR>
__device__ __forceinline__ void ln_row_sum2(float& a, float& b, float2* red2) {
  a = warp_sum(a);
  b = warp_sum(b);
  if constexpr (WPR > 1) {
    const int w = threadIdx.x >> 5, base = (w / WPR) * WPR;
    if ((threadIdx.x & 31) == 0) red2[w] = make_float2(a, b);
    ln_row_bar<WPR>();
    float2 s = red2[base];
#pragma unroll
    for (int k = 1; k < WPR; ++k) { s.x += red2[base + k].x; s.y += red2[base + k].y; }
    ln_row_bar<WPR>();
    a = s.x; b = s.y;
  }
}

template <int NCH, int WPR>
__device__ __forceinline__ void ln_stats(const float (&v)[NCH][8], int tr, int d, float eps, float& mu, float& r,
                                         float* red) {
  float s = 0.f;
#pragma unroll
  for (int c = 0; c < NCH; ++c)
    if ((c * 32 * WPR + tr) * 8 < d)
#pragma unroll
      for (int k = 0; k < 8; ++k) s += v[c][k];
  mu = ln_row_sum<WPR>(s, red) / (float)d;
  float q = 0.f;
#pragma unroll
  for (int c = 0; c < NCH; ++c)
    if ((c * 32 * WPR + tr) * 8 < d)
#pragma unroll
      for (int k = 0; k < 8; ++k) { const float e = v[c][k] - mu; q += e * e; }
  r = rsqrtf(ln_row_sum<WPR>(q, red) / (float)d + eps);
}

template <int NCH, int WPR>
__global__ void __launch_bounds__(256) layernorm_fwd_kernel(const float* __restrict__ x, const float* __restrict__ g,
                                                            const float* __restrict__ b, bf16* __restrict__ y,
                                                            float* __restrict__ rstd, int T, int d, float eps) {
  __shared__ float red[8];
  const int row = blockIdx.x * (8 / WPR) + threadIdx.x / (32 * WPR), tr = threadIdx.x % (32 * WPR);
  const bool ok = row < T;   // no early return: the row sums may synchronise the CTA
  const float* xr = x + (size_t)(ok ? row : 0) * d;
  float v[NCH][8];
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    const int i = (c * 32 * WPR + tr) * 8;
    if (i < d) ld8f(xr + i, v[c]);
  }
  float mu, r;
  ln_stats<NCH, WPR>(v, tr, d, eps, mu, r, red);
  if (!ok) return;
  if (tr == 0) rstd[row] = r;
  bf16* yr = y + (size_t)row * d;
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    const int i = (c * 32 * WPR + tr) * 8;
    if (i >= d) continue;
    float gg[8], bb[8], o[8];
    ld8f(g + i, gg);
    ld8f(b + i, bb);
#pragma unroll
    for (int k = 0; k < 8; ++k) o[k] = (v[c][k] - mu) * r * gg[k] + bb[k];
    st8b(yr + i, o);
  }
}

template <int NCH, int WPR, typename TDY>
__global__ void __launch_bounds__(256) layernorm_bwd_kernel(const TDY* __restrict__ dy, const float* __restrict__ x,
                                                            const float* __restrict__ g,
                                                            const float* __restrict__ resid, float* __restrict__ dx,
                                                            bf16* __restrict__ dxb, int T, int d, float eps) {
  __shared__ float red[8];
  __shared__ float2 red2[8];
  const int row = blockIdx.x * (8 / WPR) + threadIdx.x / (32 * WPR), tr = threadIdx.x % (32 * WPR);
  const bool ok = row < T;
  const size_t ro = (size_t)(ok ? row : 0) * d;
  float v[NCH][8], gh[NCH][8];
  // residual loads first: in flight during the loads and reductions below instead of after them
  const float4* rr4 = reinterpret_cast<const float4*>(resid + ro);
  float4 rq[NCH][2];
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    const int i = (c * 32 * WPR + tr) * 8;
    if (i < d) { rq[c][0] = rr4[i / 4]; rq[c][1] = rr4[i / 4 + 1]; }
  }
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    const int i = (c * 32 * WPR + tr) * 8;
    if (i < d) {
      ld8f(x + ro + i, v[c]);
      float a[8], gg[8];
      ld8(dy + ro + i, a);
      ld8f(g + i, gg);
#pragma unroll
      for (int k = 0; k < 8; ++k) gh[c][k] = a[k] * gg[k];
    }
  }
  float mu, r;
  ln_stats<NCH, WPR>(v, tr, d, eps, mu, r, red);
  float sg = 0.f, sgx = 0.f;
#pragma unroll
  for (int c = 0; c < NCH; ++c)
    if ((c * 32 * WPR + tr) * 8 < d)
#pragma unroll
      for (int k = 0; k < 8; ++k) { sg += gh[c][k]; sgx += gh[c][k] * (v[c][k] - mu) * r; }
  ln_row_sum2<WPR>(sg, sgx, red2);
  const float mg = sg / (float)d, mgx = sgx / (float)d;
  if (!ok) return;
#pragma unroll
  for (int c = 0; c < NCH; ++c) {
    const int i = (c * 32 * WPR + tr) * 8;
    if (i >= d) continue;
    const float rr[8] = {rq[c][0].x, rq[c][0].y, rq[c][0].z, rq[c][0].w, rq[c][1].x, rq[c][1].y, rq[c][1].z, rq[c][1].w};
    float o[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) o[k] = rr[k] + r * (gh[c][k] - mg - (v[c][k] - mu) * r * mgx);
    st8f(dx + ro + i, o);
    if (dxb) st8b(dxb + ro + i, o);
  }
}

}  // namespace

#ifndef MENOS_RMS_WIDE4K
#define MENOS_RMS_WIDE4K 1
#endif
#define LAUNCH_CHECK() (++g_launch_count, cudaPeekAtLastError() == cudaSuccess ? 0 : -3)

int rmsnorm_fwd(const float* x, const float* g, bf16* y, float* rstd, int T, int d, float eps, cudaStream_t st) {
  if (T <= 0) return 0;
  if (d % 8) return -1;
  const int nc = (d + 1023) / 1024, g2 = (T + 1) / 2;
  switch (nc) {  // single pass: the row stays in registers between the reduction and the write
    case 1: rmsnorm_fwd_reg_kernel<1, 128><<<g2, 256, 0, st>>>(x, g, y, rstd, T, d, eps); break;
    case 2: rmsnorm_fwd_reg_kernel<2, 128><<<g2, 256, 0, st>>>(x, g, y, rstd, T, d, eps); break;
#if MENOS_RMS_WIDE4K   // one row per 256 threads, 2-3 chunks per thread (r1q: bwd 100 -> 80 us at 8192 x 4096)
    case 3: case 4: rmsnorm_fwd_reg_kernel<2, 256><<<T, 256, 0, st>>>(x, g, y, rstd, T, d, eps); break;
    case 5: rmsnorm_fwd_reg_kernel<3, 256><<<T, 256, 0, st>>>(x, g, y, rstd, T, d, eps); break;
#else
    case 3: case 4: rmsnorm_fwd_reg_kernel<4, 128><<<g2, 256, 0, st>>>(x, g, y, rstd, T, d, eps); break;
    case 5: rmsnorm_fwd_reg_kernel<5, 128><<<g2, 256, 0, st>>>(x, g, y, rstd, T, d, eps); break;
#endif
    case 6: case 7: case 8: rmsnorm_fwd_reg_kernel<4, 256><<<T, 256, 0, st>>>(x, g, y, rstd, T, d, eps); break;
    default: {
      const int warps = 8;
      rmsnorm_fwd_kernel<<<(T + warps - 1) / warps, warps * 32, 0, st>>>(x, g, y, rstd, T, d, eps);
    }
  }
  return LAUNCH_CHECK();
}
template <typename TDY>
static int rmsnorm_bwd_t(const TDY* dy, const float* x, const float* g, const float* rstd, const float* resid,
                         float* dx, bf16* dxb, int T, int d, cudaStream_t st) {
  if (T <= 0) return 0;
  if (d % 8) return -1;
  const int nc = (d + 1023) / 1024, g2 = (T + 1) / 2;
  switch (nc) {
    case 1: rmsnorm_bwd_reg_kernel<1, 128, TDY><<<g2, 256, 0, st>>>(dy, x, g, rstd, resid, dx, dxb, T, d); break;
    case 2: rmsnorm_bwd_reg_kernel<2, 128, TDY><<<g2, 256, 0, st>>>(dy, x, g, rstd, resid, dx, dxb, T, d); break;
#if MENOS_RMS_WIDE4K
    case 3: case 4: rmsnorm_bwd_reg_kernel<2, 256, TDY><<<T, 256, 0, st>>>(dy, x, g, rstd, resid, dx, dxb, T, d); break;
    case 5: rmsnorm_bwd_reg_kernel<3, 256, TDY><<<T, 256, 0, st>>>(dy, x, g, rstd, resid, dx, dxb, T, d); break;
#else
    case 3: case 4: rmsnorm_bwd_reg_kernel<4, 128, TDY><<<g2, 256, 0, st>>>(dy, x, g, rstd, resid, dx, dxb, T, d); break;
    case 5: rmsnorm_bwd_reg_kernel<5, 128, TDY><<<g2, 256, 0, st>>>(dy, x, g, rstd, resid, dx, dxb, T, d); break;
#endif
    case 6: case 7: case 8:   // wide rows (70B: d = 8192): one row per 256 threads keeps 4 chunks per thread
      rmsnorm_bwd_reg_kernel<4, 256, TDY><<<T, 256, 0, st>>>(dy, x, g, rstd, resid, dx, dxb, T, d); break;
    default: {
      const int warps = 8;
      rmsnorm_bwd_kernel<TDY><<<(T + warps - 1) / warps, warps * 32, 0, st>>>(dy, x, g, rstd, resid, dx, dxb, T, d);
    }
  }
  return LAUNCH_CHECK();
}
int rmsnorm_bwd(const bf16* dy, const float* x, const float* g, const float* rstd, const float* resid, float* dx,
                bf16* dxb, int T, int d, cudaStream_t st) {
  return rmsnorm_bwd_t(dy, x, g, rstd, resid, dx, dxb, T, d, st);
}
int rmsnorm_bwd_f32dy(const float* dy, const float* x, const float* g, const float* rstd, const float* resid,
                      float* dx, bf16* dxb, int T, int d, cudaStream_t st) {
  return rmsnorm_bwd_t(dy, x, g, rstd, resid, dx, dxb, T, d, st);
}
int convert_f32_to_bf16(const float* src, bf16* dst, long long n, cudaStream_t st) {
  if (n <= 0) return 0;
  if (n % 8) return -1;
  f32_to_bf16_kernel<<<1184, 256, 0, st>>>(src, dst, n / 8);
  return LAUNCH_CHECK();
}
int convert_bf16_to_f32_vec(const bf16* src, float* dst, long long n, cudaStream_t st) {
  if (n <= 0) return 0;
  if (n % 8) return -1;
  bf16_to_f32_vec_kernel<<<1184, 256, 0, st>>>(src, dst, n / 8);
  return LAUNCH_CHECK();
}
int add_bf16_to_f32(const float* x, const bf16* delta, float* out, long long n, cudaStream_t st) {
  if (n <= 0) return 0;
  if (n % 8) return -1;
  add_bf16_f32_kernel<<<1184, 256, 0, st>>>(x, delta, out, n / 8);
  return LAUNCH_CHECK();
}
int attn_bwd_prep(const bf16* dO, const bf16* O, float* D, int T, int H, int hd, cudaStream_t st) {
  if (T <= 0) return 0;
  const int warps = 8;
  const long long n = (long long)T * H;
  attn_prep_kernel<<<(unsigned)((n + warps - 1) / warps), warps * 32, 0, st>>>(dO, O, D, T, H, hd);
  return LAUNCH_CHECK();
}
int adamw_run(const AdamSeg* d_segs, const int4* d_work, int n_work, const AdamHyper* d_hyp, cudaStream_t st) {
  if (n_work <= 0) return 0;
  adamw_kernel<<<n_work, 256, 0, st>>>(d_segs, d_work, d_hyp);
  return LAUNCH_CHECK();
}
int fill_rope_table(float2* cs, int max_pos, int hd, float theta, cudaStream_t st) {
  const int n = max_pos * (hd / 2);
  rope_table_kernel<<<(n + 255) / 256, 256, 0, st>>>(cs, max_pos, hd, theta);
  return LAUNCH_CHECK();
}
int convert_bf16_to_f32(const bf16* src, float* dst, long long n, cudaStream_t st) {
  if (n <= 0) return 0;
  bf16_to_f32_kernel<<<1024, 256, 0, st>>>(src, dst, n);
  return LAUNCH_CHECK();
}


// ------------------------------------------------------------------ LayerNorm launchers (OPT)
template <typename F>
static int ln_dispatch(int d, F&& f) {   // (chunks per lane, warps per row); d <= 4096 as before
  using std::integral_constant;
  const int nch = (d + 255) / 256;
  if (nch <= 1) return f(integral_constant<int, 1>{}, integral_constant<int, 1>{});
  if (nch <= 2) return f(integral_constant<int, 2>{}, integral_constant<int, 1>{});
  if (nch <= 4) return f(integral_constant<int, 4>{}, integral_constant<int, 1>{});
  if (nch <= 8) return f(integral_constant<int, 4>{}, integral_constant<int, 2>{});
  if (nch <= 16) return f(integral_constant<int, 4>{}, integral_constant<int, 4>{});
  return -1;
}
int layernorm_fwd(const float* x, const float* g, const float* b, bf16* y, float* rstd, int T, int d, float eps,
                  cudaStream_t st) {
  if (T <= 0) return 0;
  if (d % 8) return -1;
  return ln_dispatch(d, [&](auto n, auto w) {
    constexpr int RPB = 8 / decltype(w)::value;   // rows per 256-thread CTA
    layernorm_fwd_kernel<decltype(n)::value, decltype(w)::value><<<(T + RPB - 1) / RPB, 256, 0, st>>>(
        x, g, b, y, rstd, T, d, eps);
    return LAUNCH_CHECK();
  });
}
template <typename TDY>
static int layernorm_bwd_t(const TDY* dy, const float* x, const float* g, const float* resid, float* dx, bf16* dxb,
                           int T, int d, float eps, cudaStream_t st) {
  if (T <= 0) return 0;
  if (d % 8) return -1;
  return ln_dispatch(d, [&](auto n, auto w) {
    constexpr int RPB = 8 / decltype(w)::value;
    layernorm_bwd_kernel<decltype(n)::value, decltype(w)::value, TDY><<<(T + RPB - 1) / RPB, 256, 0, st>>>(
        dy, x, g, resid, dx, dxb, T, d, eps);
    return LAUNCH_CHECK();
  });
}
int layernorm_bwd(const bf16* dy, const float* x, const float* g, const float* resid, float* dx, bf16* dxb, int T,
                  int d, float eps, cudaStream_t st) {
  return layernorm_bwd_t(dy, x, g, resid, dx, dxb, T, d, eps, st);
}

}  // namespace menos
