// Kernel-level test entry points (include/menos_testing.h): same kernels as the server path.
#include <algorithm>
#include <cstdlib>
#include <cmath>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/menos.h"
#include "../../include/menos_testing.h"
#include "kernels.h"

using namespace menos;

namespace {
thread_local std::string t_err;
int fail(const char* m) { t_err = m; return MENOS_ECUDA; }
}  // namespace

extern "C" const char* menos_testing_last_error(void) { return t_err.c_str(); }

extern "C" int menos_test_gemm(int M, int N, int K, int b_mn, const void* A, int lda, const void* B, int ldb,
                               const void* A2, int lda2, const void* B2, int ldb2, int R, const int32_t* mtile_extra,
                               int epi, void* out, int ldo, const void* resid, int ldr, void* out2, int ldo2,
                               const void* aux, int ldaux, int head_dim, int rope_cols, const int32_t* pos,
                               float theta, int num_sms) {
  GemmArgs a;
  memset(&a, 0, sizeof a);
  a.M = M; a.N = N; a.K = K; a.b_mn_major = b_mn;
  a.A = (const bf16*)A; a.lda = lda; a.B = (const bf16*)B; a.ldb = ldb;
  a.A2 = (const bf16*)A2; a.lda2 = lda2; a.B2 = (const bf16*)B2; a.ldb2 = ldb2; a.R = R;
  a.epi = epi; a.out = (bf16*)out; a.ldo = ldo; a.resid = (const float*)resid; a.ldr = ldr;
  a.outf = (float*)out;  // EPI_RESID: fp32 residual in, fp32 out
  a.out2 = (bf16*)out2; a.ldo2 = ldo2; a.aux = (const bf16*)aux; a.ldaux = ldaux;
  a.head_dim = head_dim; a.rope_cols = rope_cols;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  a.num_sms = num_sms > 0 ? num_sms : sms;
  const int n_mt = (M + 127) / 128;
  int2* d_mt = nullptr; int* d_pos = nullptr; float2* d_cs = nullptr;
  if (R > 0) {
    if (cudaMalloc(&d_mt, n_mt * sizeof(int2)) != cudaSuccess) return fail("alloc");
    cudaMemcpy(d_mt, mtile_extra, n_mt * sizeof(int2), cudaMemcpyHostToDevice);
    a.mtile_extra = d_mt;
  }
  if (epi == EPI_ROPE) {
    int maxp = 1;
    for (int i = 0; i < M; ++i) maxp = std::max(maxp, pos[i] + 1);
    cudaMalloc(&d_pos, M * sizeof(int));
    cudaMemcpy(d_pos, pos, M * sizeof(int), cudaMemcpyHostToDevice);
    cudaMalloc(&d_cs, (size_t)maxp * (head_dim / 2) * sizeof(float2));
    fill_rope_table(d_cs, maxp, head_dim, theta, 0);
    a.pos = d_pos; a.rope_cs = d_cs;
  }
  int rc = gemm_run(a, 0);
  cudaError_t e = cudaDeviceSynchronize();
  if (d_mt) cudaFree(d_mt);
  if (d_pos) cudaFree(d_pos);
  if (d_cs) cudaFree(d_cs);
  if (rc != 0) return fail("gemm_run rejected the arguments");
  if (e != cudaSuccess) return fail(cudaGetErrorString(e));
  return MENOS_OK;
}

static int sms_of_device() {
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms;
}

extern "C" int menos_test_attention(int n_seqs, const int32_t* seq_len, int H, int Hkv, int hd, const void* qkv,
                                    void* O, float* lse, const void* dO, void* dqkv, float theta) {
  std::vector<int> cu(1, 0);
  std::vector<int2> blocks;
  int maxL = 1;
  for (int i = 0; i < n_seqs; ++i) {
    for (int q = 0; q < seq_len[i]; q += 64) blocks.push_back(make_int2(i, q));
    cu.push_back(cu.back() + seq_len[i]);
    maxL = std::max(maxL, seq_len[i]);
  }
  const int T = cu.back();
  int* d_cu; int2* d_blk; float2* d_cs; float* d_D;
  cudaMalloc(&d_cu, cu.size() * 4);
  cudaMalloc(&d_blk, std::max<size_t>(1, blocks.size()) * sizeof(int2));
  cudaMalloc(&d_cs, (size_t)maxL * (hd / 2) * sizeof(float2));
  cudaMalloc(&d_D, (size_t)H * T * 4);
  cudaMemcpy(d_cu, cu.data(), cu.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(d_blk, blocks.data(), blocks.size() * sizeof(int2), cudaMemcpyHostToDevice);
  fill_rope_table(d_cs, maxL, hd, theta, 0);
  AttnArgs a;
  memset(&a, 0, sizeof a);
  const int Nqkv = (H + 2 * Hkv) * hd;
  a.qkv = (const bf16*)qkv; a.ld_qkv = Nqkv; a.O = (bf16*)O; a.ld_o = H * hd; a.lse = lse;
  a.cu_seqlens = d_cu; a.qblocks = d_blk; a.n_qblocks = (int)blocks.size(); a.kvblocks = d_blk;
  a.n_kvblocks = (int)blocks.size(); a.T = T; a.H = H; a.Hkv = Hkv; a.hd = hd; a.scale = 1.f / std::sqrt((float)hd);
  int rc;
  std::vector<int2> b128;
  for (int i = 0; i < n_seqs; ++i)
    for (int q = 0; q < seq_len[i]; q += 128) b128.push_back(make_int2(i, q));
  int2* d_b128;
  cudaMalloc(&d_b128, std::max<size_t>(1, b128.size()) * sizeof(int2));
  cudaMemcpy(d_b128, b128.data(), b128.size() * sizeof(int2), cudaMemcpyHostToDevice);
  const bool ws_fwd = (hd == 128 || hd == 64) && (g_attn_tc & 4);
  std::vector<int4> items;
  attn_ws_items(seq_len, n_seqs, H, items, g_attn_order ? 1 : 0, sms_of_device());
  int4* d_items;
  cudaMalloc(&d_items, std::max<size_t>(1, items.size()) * sizeof(int4));
  cudaMemcpy(d_items, items.data(), items.size() * sizeof(int4), cudaMemcpyHostToDevice);
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  rc = ws_fwd ? attn_fwd_ws(a, d_items, (int)items.size(), sms, 0)
              : attn_fwd(a, 0);
  if (rc == 0 && dO) {
    attn_bwd_prep((const bf16*)dO, (const bf16*)O, d_D, T, H, hd, 0);
    a.dO = (const bf16*)dO; a.ld_do = H * hd; a.D = d_D; a.dqkv = (bf16*)dqkv; a.ld_dqkv = Nqkv;
    a.rope_cs = theta > 0.f ? d_cs : nullptr;   // theta <= 0: no RoPE backward (OPT)
    std::vector<int4> items_kv;
    attn_ws_items(seq_len, n_seqs, Hkv, items_kv, g_attn_order ? 2 : 0, sms_of_device());
    int4* d_items_kv;
    cudaMalloc(&d_items_kv, std::max<size_t>(1, items_kv.size()) * sizeof(int4));
    cudaMemcpy(d_items_kv, items_kv.data(), items_kv.size() * sizeof(int4), cudaMemcpyHostToDevice);
    const bool ws_bwd = (hd == 128 || hd == 64) && (g_attn_tc & 8);
    const bool fused_bwd = hd == 128 && (g_attn_tc & 32);
    float* d_acc = nullptr;
    std::vector<int4> items_seq;
    int4* d_items_seq = nullptr;
    if (fused_bwd) {
      attn_seq_items(seq_len, n_seqs, Hkv, items_seq);
      cudaMalloc(&d_items_seq, items_seq.size() * sizeof(int4));
      cudaMemcpy(d_items_seq, items_seq.data(), items_seq.size() * sizeof(int4), cudaMemcpyHostToDevice);
      cudaMalloc(&d_acc, (size_t)T * H * hd * sizeof(float));
      a.dq_acc = d_acc;
    }
    // bit 6: the dS-stored backward, chunked under g_attn_ds_cap_tiles exactly as the server runs it
    AttnDsPlan plan;
    const bool ds_bwd = ws_bwd && !fused_bwd && (g_attn_tc & 64) &&
                        attn_ds_plan(seq_len, n_seqs, H, Hkv, g_attn_ds_cap_tiles, plan, sms_of_device());
    if (ds_bwd) {
      const long long cap = std::min(g_attn_ds_cap_tiles, attn_ds_total_tiles(seq_len, n_seqs, H));
      bf16* d_ds; int* d_base; int4 *d_ikv, *d_iq;
      cudaMalloc(&d_ds, (size_t)std::max(1LL, cap) * 128 * 64 * 2);
      cudaMalloc(&d_base, std::max<size_t>(1, plan.base.size()) * 4);
      cudaMalloc(&d_ikv, std::max<size_t>(1, plan.items_kv.size()) * sizeof(int4));
      cudaMalloc(&d_iq, std::max<size_t>(1, plan.items_q.size()) * sizeof(int4));
      cudaMemcpy(d_base, plan.base.data(), plan.base.size() * 4, cudaMemcpyHostToDevice);
      cudaMemcpy(d_ikv, plan.items_kv.data(), plan.items_kv.size() * sizeof(int4), cudaMemcpyHostToDevice);
      cudaMemcpy(d_iq, plan.items_q.data(), plan.items_q.size() * sizeof(int4), cudaMemcpyHostToDevice);
      rc = 0;
      for (const int4& c : plan.chunks)
        if (!rc) rc = attn_bwd_ws_ds(a, d_ikv + c.x, c.y, d_iq + c.z, c.w, d_ds, cap, d_base, sms, 0);
      cudaDeviceSynchronize();
      cudaFree(d_ds); cudaFree(d_base); cudaFree(d_ikv); cudaFree(d_iq);
    } else {
      rc = fused_bwd ? attn_bwd_fused(a, d_items_seq, (int)items_seq.size(), sms, 0)
           : ws_bwd ? attn_bwd_ws(a, d_items_kv, (int)items_kv.size(), d_items, (int)items.size(), sms, 0)
                    : attn_bwd(a, 0);
    }
    cudaDeviceSynchronize();
    cudaFree(d_items_kv); cudaFree(d_acc); cudaFree(d_items_seq);
  }
  cudaError_t e = cudaDeviceSynchronize();
  cudaFree(d_cu); cudaFree(d_blk); cudaFree(d_cs); cudaFree(d_D); cudaFree(d_b128); cudaFree(d_items);
  if (rc != 0) return fail("attention launch rejected");
  if (e != cudaSuccess) return fail(cudaGetErrorString(e));
  return MENOS_OK;
}

extern "C" int menos_test_rmsnorm(int T, int d, const float* x, const float* g, float eps, void* y, float* rstd,
                                  const void* dy, const float* resid, float* dx, void* dxb) {
  int rc = rmsnorm_fwd(x, g, (bf16*)y, rstd, T, d, eps, 0);
  if (rc == 0 && dy) rc = rmsnorm_bwd((const bf16*)dy, x, g, rstd, resid, dx, (bf16*)dxb, T, d, 0);
  cudaError_t e = cudaDeviceSynchronize();
  if (rc != 0) return fail("rmsnorm launch rejected");
  if (e != cudaSuccess) return fail(cudaGetErrorString(e));
  return MENOS_OK;
}

extern "C" int menos_test_lora_rows(const void* A, const void* B, void* C, int M, int N, int K, int lda, int ldb,
                                    int ldc, int b_kn, float scale) {
  LoraRowsProblem p{};
  p.A = (const bf16*)A; p.B = (const bf16*)B; p.C = (bf16*)C;
  p.M = M; p.N = N; p.K = K; p.lda = lda; p.ldb = ldb; p.ldc = ldc; p.b_kn = b_kn; p.scale = scale;
  std::vector<int2> tiles;
  lora_rows_tiles(&p, 1, tiles);
  LoraRowsProblem* dp; int2* dt;
  cudaMalloc(&dp, sizeof p);
  cudaMalloc(&dt, tiles.size() * sizeof(int2) + 8);
  cudaMemcpy(dp, &p, sizeof p, cudaMemcpyHostToDevice);
  cudaMemcpy(dt, tiles.data(), tiles.size() * sizeof(int2), cudaMemcpyHostToDevice);
  int rc = lora_rows_run(dp, dt, (int)tiles.size(), N, 0);
  cudaError_t e = cudaDeviceSynchronize();
  cudaFree(dp); cudaFree(dt);
  if (rc) return fail("lora rows rejected");
  if (e != cudaSuccess) return fail(cudaGetErrorString(e));
  return MENOS_OK;
}

extern "C" int menos_test_lora_tokred(const void* P, const void* Q, float* C, int M, int N, int T, int ldp, int ldq,
                                      int ldc, int p_blk, int p_blk_stride, float scale, int mt) {
  LoraTokRedProblem p{};
  p.P = (const bf16*)P; p.Q = (const bf16*)Q; p.C = C;
  p.M = M; p.N = N; p.T = T; p.ldp = ldp; p.ldq = ldq; p.ldc = ldc;
  p.p_blk = p_blk > 0 ? p_blk : (1 << 30); p.p_blk_stride = p_blk_stride; p.scale = scale;
  std::vector<int4> tiles;
  lora_tokred_tiles(&p, 1, mt, mt == 128 ? 16 : 128, tiles);
  LoraTokRedProblem* dp; int4* dt;
  cudaMalloc(&dp, sizeof p);
  cudaMalloc(&dt, tiles.size() * sizeof(int4) + 16);
  cudaMemcpy(dp, &p, sizeof p, cudaMemcpyHostToDevice);
  cudaMemcpy(dt, tiles.data(), tiles.size() * sizeof(int4), cudaMemcpyHostToDevice);
  int rc = lora_tokred_run(dp, dt, (int)tiles.size(), mt, mt == 128 ? 16 : 128, 0);
  cudaError_t e = cudaDeviceSynchronize();
  cudaFree(dp); cudaFree(dt);
  if (rc) return fail("lora tokred rejected");
  if (e != cudaSuccess) return fail(cudaGetErrorString(e));
  return MENOS_OK;
}

namespace menos { extern int g_gemm_cta_group; }
extern "C" int menos_test_set_gemm_cta_group(int cg) {
  if (cg != 1 && cg != 2) return fail("cta_group must be 1 or 2");
  menos::g_gemm_cta_group = cg;
  return MENOS_OK;
}

// Time `iters` back-to-back launches of one plain GEMM (out = A B^T or A B) with CUDA events (tuning aid).
extern "C" int menos_test_gemm_time(int M, int N, int K, int b_mn, const void* A, const void* B, void* out, int epi,
                                    const void* aux, int iters, float* ms_out) {
  GemmArgs a;
  memset(&a, 0, sizeof a);
  a.M = M; a.N = N; a.K = K; a.b_mn_major = b_mn;
  a.A = (const bf16*)A; a.lda = K; a.B = (const bf16*)B; a.ldb = b_mn ? N : K;
  a.epi = epi; a.out = (bf16*)out; a.ldo = epi == EPI_SWIGLU_BWD ? 2 * N : N;
  a.out2 = (bf16*)out; a.ldo2 = N / 2; a.aux = (const bf16*)aux; a.ldaux = 2 * N;
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  a.num_sms = sms;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  int rc = gemm_run(a, 0);
  cudaEventRecord(e0, 0);
  for (int i = 0; i < iters && rc == 0; ++i) rc = gemm_run(a, 0);
  cudaEventRecord(e1, 0);
  cudaError_t e = cudaEventSynchronize(e1);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0); cudaEventDestroy(e1);
  if (rc) return fail("gemm rejected");
  if (e != cudaSuccess) return fail(cudaGetErrorString(e));
  *ms_out = ms / iters;
  return MENOS_OK;
}

// Attention variant for head_dim 128 / 64, bitmask (bits 0, 1: round-1 non-persistent tcgen05 kernels, removed in
// round 2; ignored): 4 = persistent warp-specialized tcgen05 forward (attention_fwd_ws.cu; else mma.sync),
// 8 = persistent warp-specialized tcgen05 backward (attention_bwd_ws.cu; else mma.sync).
// 64 = with 8: the dK/dV kernel stores dS^T and dQ is computed from it (S, P, dP once per pair; chunked under
// g_attn_ds_cap_tiles, 16 KB tiles).
// Default 78: the persistent tcgen05 forward and the dS-stored persistent backward (LPT work order, bit 4 selects
// (sequence, head) order).
namespace menos {
int g_attn_tc = 78; int g_attn_order = 1;
// MENOS_DS_CAP_TILES: tuning override of the dS-stored backward's chunk budget (16 KB tiles; default 32768 = 512 MB)
long long g_attn_ds_cap_tiles = [] { const char* e = getenv("MENOS_DS_CAP_TILES"); return e ? atoll(e) : 32768LL; }();
}
extern "C" int menos_test_abf_prof(unsigned long long* out16) {
  if (!out16) return fail("null output");
  return menos::attn_bwd_fused_prof(out16);
}

extern "C" int menos_test_set_attn_tc(int mode) {
  if (mode < 0 || mode > 127) { fail("attention mode must be in [0, 127]"); return MENOS_EINVAL; }
  menos::g_attn_order = (mode & 16) ? 0 : 1;   // bit 4: (sequence, head)-grouped work order instead of LPT
  mode &= 111;                                 // bit 5: one-pass fused backward; bit 6: dS-stored backward
  menos::g_attn_tc = mode;
  return MENOS_OK;
}

// dS-stored backward: tile budget of one chunk (16 KB tiles; default 32768 = 512 MB); small values force chunking
extern "C" int menos_test_set_ds_cap(long long tiles) {
  if (tiles < 1) { fail("ds cap must be >= 1 tile"); return MENOS_EINVAL; }
  menos::g_attn_ds_cap_tiles = tiles;
  return MENOS_OK;
}

// Host-only: the dS-stored backward's dQ item list for a persistent grid of `grid` CTAs (attn_ds_plan with grid > 0):
// items[4 i .. 4 i + 3] = (sequence, q0, head, 0), or sequence -1 for padding; chunks as menos_test_ds_plan.
extern "C" int menos_test_ds_plan_q(int n_seqs, const int32_t* seq_len, int H, int Hkv, long long cap, int grid,
                                    int32_t* items, int max_items, int32_t* n_items, int32_t* chunks, int max_chunks,
                                    int32_t* n_chunks) {
  if (n_seqs < 0 || !seq_len || H <= 0 || Hkv <= 0 || H % Hkv || grid <= 0 || !n_items || !n_chunks)
    return fail("bad arguments");
  menos::AttnDsPlan plan;
  std::vector<int> lens(seq_len, seq_len + n_seqs);
  if (!menos::attn_ds_plan(lens.data(), n_seqs, H, Hkv, cap, plan, grid)) { *n_chunks = -1; return MENOS_OK; }
  *n_items = (int)plan.items_q.size();
  *n_chunks = (int)plan.chunks.size();
  for (int i = 0; i < (int)plan.items_q.size() && i < max_items && items; ++i) {
    items[4 * i] = plan.items_q[i].x; items[4 * i + 1] = plan.items_q[i].y;
    items[4 * i + 2] = plan.items_q[i].z; items[4 * i + 3] = plan.items_q[i].w;
  }
  for (int c = 0; c < (int)plan.chunks.size() && c < max_chunks && chunks; ++c) {
    chunks[4 * c] = plan.chunks[c].x; chunks[4 * c + 1] = plan.chunks[c].y;
    chunks[4 * c + 2] = plan.chunks[c].z; chunks[4 * c + 3] = plan.chunks[c].w;
  }
  return MENOS_OK;
}

// Host plan of the dS-stored attention backward (no GPU needed): per-sequence tile counts, unit bases and chunks.
// tiles[i] = attn_ds_tiles(seq_len[i]); base[seq * Hkv + hk]; chunks[c] = (kv item offset, count, q offset, count).
extern "C" int menos_test_ds_plan(int n_seqs, const int32_t* seq_len, int H, int Hkv, long long cap, int32_t* tiles,
                                  int32_t* base, int32_t* chunks, int max_chunks, int32_t* n_chunks,
                                  int32_t* n_items_kv, int32_t* n_items_q) {
  if (n_seqs < 0 || !seq_len || H <= 0 || Hkv <= 0 || H % Hkv || !n_chunks) return fail("bad arguments");
  for (int i = 0; i < n_seqs; ++i) if (tiles) tiles[i] = menos::attn_ds_tiles(seq_len[i]);
  menos::AttnDsPlan plan;
  std::vector<int> lens(seq_len, seq_len + n_seqs);
  if (!menos::attn_ds_plan(lens.data(), n_seqs, H, Hkv, cap, plan)) { *n_chunks = -1; return MENOS_OK; }
  *n_chunks = (int)plan.chunks.size();
  if (n_items_kv) *n_items_kv = (int)plan.items_kv.size();
  if (n_items_q) *n_items_q = (int)plan.items_q.size();
  if (base) for (size_t i = 0; i < plan.base.size(); ++i) base[i] = plan.base[i];
  if (chunks)
    for (int c = 0; c < (int)plan.chunks.size() && c < max_chunks; ++c) {
      chunks[4 * c] = plan.chunks[c].x; chunks[4 * c + 1] = plan.chunks[c].y;
      chunks[4 * c + 2] = plan.chunks[c].z; chunks[4 * c + 3] = plan.chunks[c].w;
    }
  return MENOS_OK;
}
