// HBM-bound row kernels: RMSNorm fwd/bwd, attention-backward row sums
// (A11 prologue), fused multi-tensor AdamW over all stepped clients' adapters (A13, Alg.1 L12),
// RoPE table.  One warp per row, 16-byte vector loads, warp-shuffle fp32 reductions.
#include "common.cuh"
#include "kernels.h"

namespace menos {

unsigned long long g_launch_count = 0;

namespace {

// ------------------------------------------------------------------ RMSNorm forward
// y = x * rstd * g, rstd = rsqrt(mean(x^2) + eps); x, y bf16 [T, d]; g fp32 [d]; d % 8 == 0
__global__ void rmsnorm_fwd_kernel(const bf16* __restrict__ x, const float* __restrict__ g, bf16* __restrict__ y,
                                   float* __restrict__ rstd, int T, int d, float eps) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= T) return;
  const uint4* xr = reinterpret_cast<const uint4*>(x + (size_t)warp * d);
  const int nv = d >> 3;
  float ss = 0.f;
  for (int i = lane; i < nv; i += 32) {
    uint4 u = xr[i];
    uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) { float2 f = unpack_bf16x2(w[k]); ss += f.x * f.x + f.y * f.y; }
  }
  ss = warp_sum(ss);
  const float r = rsqrtf(ss / (float)d + eps);
  if (lane == 0) rstd[warp] = r;
  uint4* yr = reinterpret_cast<uint4*>(y + (size_t)warp * d);
  const float4* g4 = reinterpret_cast<const float4*>(g);
  for (int i = lane; i < nv; i += 32) {
    uint4 u = xr[i];
    float4 ga = g4[2 * i], gb = g4[2 * i + 1];
    float2 f0 = unpack_bf16x2(u.x), f1 = unpack_bf16x2(u.y), f2 = unpack_bf16x2(u.z), f3 = unpack_bf16x2(u.w);
    uint4 o;
    o.x = pack_bf16x2(f0.x * r * ga.x, f0.y * r * ga.y);
    o.y = pack_bf16x2(f1.x * r * ga.z, f1.y * r * ga.w);
    o.z = pack_bf16x2(f2.x * r * gb.x, f2.y * r * gb.y);
    o.w = pack_bf16x2(f3.x * r * gb.z, f3.y * r * gb.w);
    yr[i] = o;
  }
}

// ------------------------------------------------------------------ RMSNorm backward (+ residual)
// dx = resid + rstd*(gh - xh*mean(gh*xh)),  gh = dy*g,  xh = x*rstd
__global__ void rmsnorm_bwd_kernel(const bf16* __restrict__ dy, const bf16* __restrict__ x,
                                   const float* __restrict__ g, const float* __restrict__ rstd,
                                   const bf16* __restrict__ resid, bf16* __restrict__ dx, int T, int d) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= T) return;
  const size_t ro = (size_t)warp * d;
  const uint4* dyr = reinterpret_cast<const uint4*>(dy + ro);
  const uint4* xr = reinterpret_cast<const uint4*>(x + ro);
  const float4* g4 = reinterpret_cast<const float4*>(g);
  const int nv = d >> 3;
  const float r = rstd[warp];
  float dot = 0.f;
  for (int i = lane; i < nv; i += 32) {
    uint4 a = dyr[i], b = xr[i];
    float4 ga = g4[2 * i], gb = g4[2 * i + 1];
    float gg[8] = {ga.x, ga.y, ga.z, ga.w, gb.x, gb.y, gb.z, gb.w};
    uint32_t wa[4] = {a.x, a.y, a.z, a.w}, wb[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      float2 fa = unpack_bf16x2(wa[k]), fb = unpack_bf16x2(wb[k]);
      dot += fa.x * gg[2 * k] * fb.x + fa.y * gg[2 * k + 1] * fb.y;
    }
  }
  dot = warp_sum(dot);
  const float mean = dot * r / (float)d;  // mean(gh * xh) = r * mean(gh * x)
  const uint4* rr = reinterpret_cast<const uint4*>(resid + ro);
  uint4* out = reinterpret_cast<uint4*>(dx + ro);
  for (int i = lane; i < nv; i += 32) {
    uint4 a = dyr[i], b = xr[i], c = rr[i];
    float4 ga = g4[2 * i], gb = g4[2 * i + 1];
    float gg[8] = {ga.x, ga.y, ga.z, ga.w, gb.x, gb.y, gb.z, gb.w};
    uint32_t wa[4] = {a.x, a.y, a.z, a.w}, wb[4] = {b.x, b.y, b.z, b.w}, wc[4] = {c.x, c.y, c.z, c.w};
    uint32_t wo[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      float2 fa = unpack_bf16x2(wa[k]), fb = unpack_bf16x2(wb[k]), fc = unpack_bf16x2(wc[k]);
      const float o0 = fc.x + r * (fa.x * gg[2 * k] - fb.x * r * mean);
      const float o1 = fc.y + r * (fa.y * gg[2 * k + 1] - fb.y * r * mean);
      wo[k] = pack_bf16x2(o0, o1);
    }
    out[i] = make_uint4(wo[0], wo[1], wo[2], wo[3]);
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

}  // namespace

#define LAUNCH_CHECK() (++g_launch_count, cudaPeekAtLastError() == cudaSuccess ? 0 : -3)

int rmsnorm_fwd(const bf16* x, const float* g, bf16* y, float* rstd, int T, int d, float eps, cudaStream_t st) {
  if (T <= 0) return 0;
  if (d % 8) return -1;
  const int warps = 8;
  rmsnorm_fwd_kernel<<<(T + warps - 1) / warps, warps * 32, 0, st>>>(x, g, y, rstd, T, d, eps);
  return LAUNCH_CHECK();
}
int rmsnorm_bwd(const bf16* dy, const bf16* x, const float* g, const float* rstd, const bf16* resid, bf16* dx, int T,
                int d, cudaStream_t st) {
  if (T <= 0) return 0;
  if (d % 8) return -1;
  const int warps = 8;
  rmsnorm_bwd_kernel<<<(T + warps - 1) / warps, warps * 32, 0, st>>>(dy, x, g, rstd, resid, dx, T, d);
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

}  // namespace menos
