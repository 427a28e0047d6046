/*
 * menos_testing.h -- kernel-level entry points of libmenos.so used ONLY by the GPU unit tests
 * (tests/test_gpu_kernels.py).  They run exactly the kernels the server path launches, on caller-owned
 * DEVICE buffers, and synchronise the device before returning.  Not part of the user-facing boundary
 * (include/menos.h); same error conventions (0 = OK, menos_last_error() for the message).
 */
#ifndef MENOS_TESTING_H_
#define MENOS_TESTING_H_
#include <stddef.h>
#include <stdint.h>
#include "menos.h"
#ifndef MENOS_API
#define MENOS_API __attribute__((visibility("default")))
#endif

#ifdef __cplusplus
extern "C" {
#endif

/* tcgen05 GEMM:
 *   out[M, N] = epi( A[M, K] . B^T  +  A2[M, window] . B2[window]^T )
 *   b_mn = 0: B is [N, K] row-major (ldb); b_mn = 1: B is [K, N] row-major (dX form).  B2 follows B's form
 *   with R columns / rows.  mtile_extra (host, 2 ints per 128-row tile: col_start, n16) selects each tile's
 *   extra-K window; R = 0 disables it.  epi: 0 store, 1 +resid (resid and out fp32: the residual stream),
 *   2 RoPE (head_dim, rope_cols, pos, theta), 3 SwiGLU fwd (out = gu, out2 = a), 4 SwiGLU bwd (aux = saved gu,
 *   out = dgu).  Operands bf16, device. */
MENOS_API int menos_test_gemm(int M, int N, int K, int b_mn, const void* A, int lda, const void* B, int ldb, const void* A2,
                    int lda2, const void* B2, int ldb2, int R, const int32_t* mtile_extra, int epi, void* out, int ldo,
                    const void* resid, int ldr, void* out2, int ldo2, const void* aux, int ldaux, int head_dim,
                    int rope_cols, const int32_t* pos, float theta, int num_sms);

/* Varlen causal flash attention forward + backward (A3, A11) on a packed qkv [T, (H+2Hkv)hd] (q,k post-RoPE):
 * O [T, H*hd], lse [H, T] fp32; if dO != NULL also dqkv [T, (H+2Hkv)hd] = gradients w.r.t. the PRE-RoPE
 * q, k and v (RoPE backward with theta applied; theta <= 0: no RoPE, as for OPT).  seq_len: host [n_seqs]. */
MENOS_API int menos_test_attention(int n_seqs, const int32_t* seq_len, int H, int Hkv, int hd, const void* qkv, void* O,
                         float* lse, const void* dO, void* dqkv, float theta);

/* RMSNorm forward (y bf16, rstd) of the fp32 residual stream x, and backward dx = resid + norm_bwd(dy) with
 * dy bf16, resid / dx fp32 and dxb = bf16(dx) (optional); g fp32 [d].  Device buffers. */
MENOS_API int menos_test_rmsnorm(int T, int d, const float* x, const float* g, float eps, void* y, float* rstd,
                                 const void* dy, const float* resid, float* dx, void* dxb);

/* Copy one saved intermediate of a live SAVE batch to host (debugging / white-box tests).
 * which: 0 x, 1 xn, 2 qkv, 3 O, 4 h, 5 hn, 6 gu (Llama: warp-tile order, see gu_tile_off in gemm_tcgen05.cu), 7 a, 8 U_qkv, 9 U_o, 10 U_gu, 11 U_down (bf16), 12 lse (fp32 [H,T]).
 * *bytes receives the size; host_out may be NULL to query it. */
MENOS_API int menos_test_batch_tensor(menos_server* s, menos_batch* b, int layer, int which, void* host_out,
                                      size_t* bytes);

/* LoRA side contractions (device buffers, one problem):
 *   rows:   C[t, j] = scale * sum_k A[t, k] * (b_kn ? B[k, j] : B[j, k])         (bf16 out; shrink / dU)
 *   tokred: C[m, n] = scale * sum_t P[t, map(m)] * Q[t, n]                       (fp32 out; dA / dB)
 *           map(m) = (m / p_blk) * p_blk_stride + m % p_blk (p_blk <= 0: identity); mt = 128 (dB) or 16 (dA). */
MENOS_API int menos_test_lora_rows(const void* A, const void* B, void* C, int M, int N, int K, int lda, int ldb,
                                   int ldc, int b_kn, float scale);
MENOS_API int menos_test_lora_tokred(const void* P, const void* Q, float* C, int M, int N, int T, int ldp, int ldq,
                                     int ldc, int p_blk, int p_blk_stride, float scale, int mt);

/* Select the tcgen05 GEMM variant for subsequent launches: 2 = CTA pair (cta_group::2, default), 1 = single CTA. */
MENOS_API int menos_test_set_gemm_cta_group(int cta_group);

/* Time `iters` back-to-back launches of one GEMM (ld = natural) with CUDA events; *ms_out = ms per launch. */
MENOS_API int menos_test_gemm_time(int M, int N, int K, int b_mn, const void* A, const void* B, void* out, int epi,
                                   const void* aux, int iters, float* ms_out);

/* Attention kernels for head_dim 128 / 64, bitmask: bits 0, 1 = ignored (round-1 non-persistent tcgen05 kernels,
   removed), bit 2 = persistent warp-specialized tcgen05 forward (else mma.sync), bit 3 = persistent
   warp-specialized tcgen05 backward (else mma.sync), bit 4 = (sequence, head)-grouped
   work order instead of LPT, bit 5 = one-pass fused tcgen05 backward (overrides bits 3 and 1), bit 6 (with bit 3)
   = dS-stored backward: the dK/dV kernel also stores bf16 dS^T tiles and dQ = dS K is computed from them, so S, P and
   dP are evaluated once per (key, query) pair.  Default mode 78 (persistent forward + dS-stored
   persistent backward).  Returns MENOS_EINVAL outside [0, 127]. */
MENOS_API int menos_test_set_attn_tc(int mode);

/* dS-stored backward: most 16 KB dS^T tiles one chunk may use (default 32768 = 512 MB; the server reserves
   min(this, what the batch needs) in its scratch and runs larger batches in chunks of (sequence, kv head) units).
   Small values force chunking (tests).  MENOS_EINVAL if tiles < 1. */
MENOS_API int menos_test_set_ds_cap(long long tiles);

/* Host-only (no GPU): the dS-stored backward's plan for n_seqs sequences -- tiles[i] = dS^T tiles of sequence i per
   head, base[seq * Hkv + kv head] = the unit's first tile in its chunk, chunks[4c..4c+3] = (kv item offset, count,
   q item offset, count) for c < min(*n_chunks, max_chunks); *n_chunks = -1 when a unit alone exceeds `cap` (the
   recompute path).  Any output pointer but n_chunks may be NULL. */
/* Host-only (no GPU): the dS-stored backward's dQ item list for a persistent grid of `grid` CTAs (CTA c takes entries
   c, c + grid, ...): items[4i..4i+3] = (sequence, first query row, head, 0), sequence -1 = padding at a CTA's tail;
   each CTA's items form runs of one (sequence, query block) over consecutive heads (the epilogue loads the RoPE rows
   once per run).  *n_items = list length (copied up to max_items), chunks as menos_test_ds_plan (*n_chunks = -1:
   no plan).  items / chunks may be NULL. */
MENOS_API int menos_test_ds_plan_q(int n_seqs, const int32_t* seq_len, int H, int Hkv, long long cap, int grid,
                                   int32_t* items, int max_items, int32_t* n_items, int32_t* chunks, int max_chunks,
                                   int32_t* n_chunks);

MENOS_API int menos_test_ds_plan(int n_seqs, const int32_t* seq_len, int H, int Hkv, long long cap, int32_t* tiles,
                                 int32_t* base, int32_t* chunks, int max_chunks, int32_t* n_chunks,
                                 int32_t* n_items_kv, int32_t* n_items_q);

/* Tuning aid: per-phase clock64 totals of the one-pass attention backward's role threads (16 counters, cleared by the
 * read) when libmenos.so was built with -DMENOS_ABF_PROF (MENOS_NVCC_DEFS); zeros otherwise. */
MENOS_API int menos_test_abf_prof(unsigned long long* out16);

MENOS_API const char* menos_testing_last_error(void);

#ifdef __cplusplus
}
#endif
#endif
