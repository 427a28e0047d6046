// Internal launcher interface between the Menos host runtime (server.cu) and the sm_100a kernels.
// Not part of the C-ABI; see include/menos.h for the public boundary.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <vector>

namespace menos {

typedef __nv_bfloat16 bf16;

// Counts every kernel this library launches (reported as gpu_launches by bench.py).
extern unsigned long long g_launch_count;

// ---------------------------------------------------------------- tcgen05 GEMM
enum EpiMode : int {
  EPI_STORE = 0,       // out = bf16(acc)
  EPI_RESID = 1,       // outf = acc + residf   (fp32 residual stream; resid == nullptr: outf = acc)
  EPI_ROPE = 2,        // columns < rope_cols rotated by RoPE at pos[row]; out = bf16
  EPI_SWIGLU_FWD = 3,  // tile = [128 gate | 128 up]: out = bf16(acc) (saved gu, warp-tile order, see gu_tile_off), out2 = bf16(silu(g) u)
  EPI_SWIGLU_BWD = 4,  // acc = da over f columns; aux = saved gu (warp-tile order); out = dgu (row-major, interleaved like gu)
  EPI_RELU_FWD = 5,    // OPT fc1: out = bf16(relu(acc + bias))
  EPI_RELU_BWD = 6,    // OPT fc2 dX: out = bf16(acc * (aux > 0)), aux = saved relu output
  EPI_STORE_DSUM = 7,  // o-proj dX: out = dO = bf16(acc), and per head h of width dsum_hd (% 32 == 0):
                       // dsum[h * dsum_ld + row] = sum_j bf16(dO)[row, j] * aux[row, j] (aux = saved O): the
                       // attention backward's D = rowsum(dO . O), fused so dO and O are not re-read
  // EPI_STORE and EPI_RESID add `bias[col]` (fp32) when bias != nullptr (OPT projections)
};

struct GemmArgs {
  int M, N, K;               // out[M, N] = A[M, K] . B^T  (B K-major [N, K] or MN-major [K, N])
  int b_mn_major;            // 0: B is [N, K] row-major (weights, fwd); 1: B is [K, N] row-major (dX)
  const bf16* A; int lda;
  const bf16* B; int ldb;
  // optional extra-K segment (segmented LoRA expand, block-diagonal U): A2 [M, R] K-major, B2 like B
  const bf16* A2; int lda2;
  const bf16* B2; int ldb2;
  int R;                      // columns of A2 / K-extent of B2 (0 = no extra segment)
  const int2* mtile_extra;    // device [ceil(M/128)]: (col_start, n16 = # of 16-wide K steps)
  const uint8_t* ntile_extra; // device [ceil(N/256)] or nullptr (= all tiles)
  // epilogue
  int epi;
  bf16* out; int ldo;
  const float* resid; int ldr;     // EPI_RESID: fp32 residual in, fp32 `outf` out (ld = ldo)
  float* outf;
  bf16* out2; int ldo2;            // EPI_SWIGLU_FWD: a
  const bf16* aux; int ldaux;      // EPI_SWIGLU_BWD: saved gu; EPI_RELU_BWD: saved relu output
  const float* bias;               // [N] fp32 or nullptr (EPI_STORE, EPI_RESID, EPI_RELU_FWD)
  float* dsum; int dsum_ld, dsum_hd;   // EPI_STORE_DSUM
  const float2* rope_cs;           // EPI_ROPE: [max_pos][hd/2] (cos, sin)
  const int* pos;                  // EPI_ROPE: per-row position
  int head_dim, rope_cols;
  int num_sms;
};

// Tensor maps are cached by (ptr, rows, cols, ld, box) on the host.
int gemm_run(const GemmArgs& a, cudaStream_t st);

// ---------------------------------------------------------------- segmented LoRA side contractions
// rows: C[t, j] = scale * sum_k A[t, k] * Bop(j, k);  Bop(j,k) = b_kn ? B[k*ldb + j] : B[j*ldb + k]  (bf16 out)
struct LoraRowsProblem {
  const bf16* A; const bf16* B; bf16* C;
  int M, N, K, lda, ldb, ldc, b_kn;
  float scale;
};
// token reduction: C[m, n] = scale * sum_t P[t, map(m)] * Q[t, n]   (fp32 out, overwrite)
//   map(m) = (m / p_blk) * p_blk_stride + m % p_blk   (gate/up interleaved 128-blocks)
//   output rows may be split in segments (one client's q|k|v or gate|up dA in one pass over X): row m goes to
//   segment m / m_seg (C, C1, C2) at row m % m_seg, and only rows with m % m_seg < m_valid are written
//   (m_seg <= 0: one segment; m_valid <= 0: every row)
struct LoraTokRedProblem {
  const bf16* P; const bf16* Q; float* C;
  int M, N, T, ldp, ldq, ldc, p_blk, p_blk_stride;
  float scale;
  float* C1; float* C2;
  int m_seg, m_valid;
  int t0, pcol0;   // tcgen05 dA: the client's first row and its dU slot column in the whole buffers
};
// dA on tcgen05 (lists of per-(client, group) problems with M = slot width <= 64): dA_seg[m % m_seg][k] =
// sum_t dU[t0 + t, pcol0 + m] X[t0 + t, k]; X [rows, ldx] and dU [rows, lddu] are whole buffers
int lora_da_tc_run(const LoraTokRedProblem* d_probs, int n_probs, int max_n, int max_w, const bf16* X, int rows,
                   int ldx, const bf16* dU, int lddu, cudaStream_t st);
// fused dU + dB of one (client, target) in ONE pass over its dY columns:
//   dB[m, n]  = sum_t dY[t, map(m)] U[t, n]                                  (fp32 [Nt, rank], overwrite)
//   W[s][t,n] = sum_{m in slab s} dY[t, map(m)] B[map(m), n]                 (fp32 partials, [n_slabs][T][rank])
//   dU[t, n]  = bf16(scale * sum_s W[s][t, n])  for n < rank, 0 for rank <= n < rs   (second, tiny kernel)
// U = the saved s * X A^T of the target, B = its Bcat rows (indexed like dY's columns), map as above.
struct LoraDUBProblem {
  const bf16* dY; const bf16* U; const bf16* B;
  float* dB; float* W; bf16* dU;
  int Nt, rank, rs, T, ldy, ldu, ldb, lddu, p_blk, p_blk_stride, n_slabs;
  float scale;
  int t0, ycol0, ucol0;   // tcgen05 variant: the problem's first row and its dY / U columns in the whole buffers
};
int lora_rows_run(const LoraRowsProblem* d_probs, const int2* d_tiles, int n_tiles, int max_n, cudaStream_t st);
int lora_tokred_run(const LoraTokRedProblem* d_probs, const int4* d_tiles, int n_tiles, int mt, int nt, cudaStream_t st);
void lora_rows_tiles(const LoraRowsProblem* probs, int n, std::vector<int2>& out);
void lora_tokred_tiles(const LoraTokRedProblem* probs, int n, int mt, int nt, std::vector<int4>& out);
// shrink on tcgen05: U[t0 + m, col + n] = bf16(scale * sum_k X[t0 + m, k] Acat[col + n, k]), m < T, n < w
// (w <= 128, w % 8 == 0 and col % 8 == 0); X [x_rows, K] (ld ldx) and Acat [a_rows, K] (ld lda) are whole buffers
// (one TMA map each), problems index into them; tiles = (problem, 128-token tile start) from lora_shrink_tiles
struct LoraShrinkProblem { int t0, T, col, w; float scale; };
void lora_shrink_tiles(const LoraShrinkProblem* probs, int n, std::vector<int2>& out);
int lora_shrink_tc_run(const bf16* X, int x_rows, int ldx, const bf16* Acat, int a_rows, int lda, int K,
                       const LoraShrinkProblem* d_probs, const int2* d_tiles, int n_tiles, int max_w, bf16* U, int ldu,
                       cudaStream_t st);
// dU/dB slab width (dY columns per CTA) used for n_slabs
constexpr int LORA_DUB_MT = 128;
// grid: (max n_slabs * ceil(max rank / 16), n_probs); CTAs past a problem's slabs exit
int lora_dub_run(const LoraDUBProblem* d_probs, int n_probs, int max_slabs, int max_rank, cudaStream_t st);
// tcgen05 variant (rank <= 16): the same contract; dY [y_rows, ldy] and U [y_rows, ldu] are the whole buffers the
// problems index with (t0, ycol0) / (t0, ucol0); 128-token stages by TMA, dB and the per-stage dU share on tcgen05
// mts: dY columns per CTA (128, or 256: half the partials; the problems' n_slabs must use the same width)
int lora_dub_tc_run(const LoraDUBProblem* d_probs, int n_probs, int max_slabs, const bf16* dY, int y_rows, int ldy,
                    const bf16* U, int ldu, int mts, cudaStream_t st);
// grid: (ceil(max T * rs / 256), n_probs)
int lora_du_reduce_run(const LoraDUBProblem* d_probs, int n_probs, long long max_elems, cudaStream_t st);

// ---------------------------------------------------------------- norms / elementwise
// residual streams (x, h forward; dy, dh backward) are fp32; GEMM operands (xn, hn, dxn ...) are bf16
int rmsnorm_fwd(const float* x, const float* g, bf16* y, float* rstd, int T, int d, float eps, cudaStream_t st);
// LayerNorm (OPT, NEXT-4): y = (x - mu) rstd g + b (bf16 out, rstd saved); bwd recomputes mu, rstd from x:
// dx = resid + rstd (gh - mean(gh) - xh mean(gh xh)), gh = dy g; dxb = optional bf16 copy
int layernorm_fwd(const float* x, const float* g, const float* b, bf16* y, float* rstd, int T, int d, float eps,
                  cudaStream_t st);
int layernorm_bwd(const bf16* dy, const float* x, const float* g, const float* resid, float* dx, bf16* dxb, int T,
                  int d, float eps, cudaStream_t st);
// dx = resid + rstd*(gh - xh*mean(gh*xh)), gh = dy*g, xh = x*rstd; dxb (optional) = bf16(dx)
int rmsnorm_bwd(const bf16* dy, const float* x, const float* g, const float* rstd, const float* resid, float* dx,
                bf16* dxb, int T, int d, cudaStream_t st);
// same with an fp32 incoming gradient (tensor-parallel path: dy is the fp32 all-reduced dX partial sum)
int rmsnorm_bwd_f32dy(const float* dy, const float* x, const float* g, const float* rstd, const float* resid,
                      float* dx, bf16* dxb, int T, int d, cudaStream_t st);
int convert_f32_to_bf16(const float* src, bf16* dst, long long n, cudaStream_t st);       // n % 8 == 0
int convert_bf16_to_f32_vec(const bf16* src, float* dst, long long n, cudaStream_t st);   // n % 8 == 0
int attn_bwd_prep(const bf16* dO, const bf16* O, float* D, int T, int H, int hd, cudaStream_t st);
// out = x + float(delta) (fp32 residual add of a bf16 reduce-scatter result; n % 8 == 0); out may alias x
int add_bf16_to_f32(const float* x, const bf16* delta, float* out, long long n, cudaStream_t st);

// ---------------------------------------------------------------- attention (varlen causal, GQA)
struct AttnArgs {
  const bf16* qkv; int ld_qkv;   // q at col 0, k at H*hd, v at (H+Hkv)*hd
  bf16* O; int ld_o;
  float* lse;                    // [H, T]
  const int* cu_seqlens;         // [n_seq+1]
  const int2* qblocks;           // (seq, local q start) per 64-row q block
  int n_qblocks;
  const int2* kvblocks;          // (seq, local kv start) per 64-row kv block
  int n_kvblocks;
  int T, H, Hkv, hd;
  float scale;
  // backward
  const bf16* dO; int ld_do;
  const float* D;                // [H, T]
  bf16* dqkv; int ld_dqkv;       // dq/dk/dv written pre-RoPE (RoPE backward applied)
  const float2* rope_cs;         // [max_pos][hd/2]
  // one-pass backward (attention_bwd_fused.cu): per-thread ordered fp32 dQ accumulation
  float* dq_acc;                 // [T, H*hd] fp32 scratch
  // prefix tuning (NEXT-3): per sequence, the number of prefix rows in front of it in this (extended) batch: the RoPE
  // backward uses position = row - shift (clamped at 0, the identity rotation: prefix rows are not rotated, R28)
  const int* pos_shift;          // [n_seqs] or nullptr
};
int attn_fwd(const AttnArgs& a, cudaStream_t st);
// persistent warp-specialized tcgen05 forward for head_dim 128 (attention_fwd_ws.cu); items = (seq, q0, head, -)
int attn_fwd_ws(const AttnArgs& a, const int4* items, int n_items, int num_sms, cudaStream_t st);
// order: 0 = (sequence, head) groups (L2 locality), 1 = largest forward / dQ work first, 2 = largest dK/dV first
// grid > 0 (with order 1 / 2): the LPT list is laid out in boustrophedon waves of `grid` items (every second wave
// reversed), so the persistent kernels' static round-robin (item i -> CTA i % grid) balances the per-CTA work
void attn_ws_items(const int* seq_len, int n_seqs, int H, std::vector<int4>& out, int order = 0, int grid = 0);
void attn_snake_waves(std::vector<int4>& v, size_t first, int grid);
// persistent warp-specialized tcgen05 backward for head_dim 128 (attention_bwd_ws.cu): items_kv = (seq, k0, kv
// head, -) per 128-key block, items_q = (seq, q0, head, -) per 128-query block
int attn_bwd_ws(const AttnArgs& a, const int4* items_kv, int n_items_kv, const int4* items_q, int n_items_q,
                int num_sms, cudaStream_t st);
// same, with S / P / dP computed once per (key, query) pair: the dK/dV kernel also stores bf16 dS^T tiles
// ([128 keys][64 queries], `ds`, ds_tiles of them) and a second kernel computes dQ = dS K from them.
// ds_base[seq * Hkv + kv head] = first tile of that (sequence, kv head) unit; a unit holds, per head of its group,
// attn_ds_tiles(L) tiles numbered key block by key block (64-query blocks 2 kb .. ceil(L/64) - 1 of key block kb).
// The items must cover exactly the units whose tiles fit in `ds` (the caller chunks larger batches).
int attn_bwd_ws_ds(const AttnArgs& a, const int4* items_kv, int n_items_kv, const int4* items_q, int n_items_q,
                   bf16* ds, long long ds_tiles, const int* ds_base, int num_sms, cudaStream_t st);
int attn_ds_tiles(int L);
long long attn_ds_total_tiles(const int* seq_len, int n_seqs, int H);
// Host plan of the dS-stored backward over sequences [0, n_seqs): units (sequence, kv head) packed in order into
// chunks of at most cap_tiles tiles; base[seq * Hkv + kv head] = the unit's first tile within its chunk; per chunk c
// the work lists items_kv[chunks[c].x, + .y) and items_q[chunks[c].z, + .w) (LPT-ordered).  false: a single unit
// is larger than cap_tiles (the caller takes the recompute path).
struct AttnDsPlan { std::vector<int> base; std::vector<int4> items_kv, items_q, chunks; };
bool attn_ds_plan(const int* seq_len, int n_seqs, int H, int Hkv, long long cap_tiles, AttnDsPlan& out,
                  int grid = 0);
// tiles the dS-stored backward may use at most (the buffer a chunk fills): 16 KB each
extern long long g_attn_ds_cap_tiles;
// one-pass persistent tcgen05 backward for head_dim 128 (attention_bwd_fused.cu): items = (seq, -, kv head, -), one
// per (sequence, kv head), longest sequence first (attn_seq_items)
int attn_bwd_fused(const AttnArgs& a, const int4* items_seq, int n_items, int num_sms, cudaStream_t st);
void attn_seq_items(const int* seq_len, int n_seqs, int Hkv, std::vector<int4>& out);
int attn_bwd_fused_prof(unsigned long long* out16);   // tuning: per-phase cycles (-DMENOS_ABF_PROF builds)
// head_dim 128 / 64 variant bitmask: 4 = persistent warp-specialized tcgen05 forward, 8 = persistent
// warp-specialized tcgen05 backward, 64 (with 8) = the dS-stored backward, 32 = one-pass fused tcgen05 backward
// (head_dim 128; takes precedence over 8); without 4 / 8 the mma.sync kernels (attention.cu)
extern int g_attn_tc;
extern int g_attn_order;   // persistent attention work order: 1 = LPT (default), 0 = (sequence, head) grouped
int attn_bwd(const AttnArgs& a, cudaStream_t st);


// ---------------------------------------------------------------- prefix tuning (prefix.cu; NEXT-3, R28)
struct PrefixClient {        // one prefix-tuning client of a batch
  const bf16* table;         // bf16 prefix [layers from first_layer][2 (k, v)][n][Nkv]
  float* grad;               // fp32 gradient, same layout
  int n;                     // prefix length P
  int first_layer;           // the client's cut (local layer index)
  int seq0, seq1;            // its sequences [seq0, seq1) in the batch
};
// ext row r: src[r].x >= 0 -> copy qkv row src[r].x; else prefix row (src[r].y & 0xFFFF) of batch client
// (src[r].y >> 16): q = 0, k / v from that client's table at `layer`
int prefix_gather(const bf16* qkv, int ld, const int2* src, int n_rows, const PrefixClient* pc, int layer, int Nq,
                  int Nkv, bf16* out, cudaStream_t st);
int rows_map(const bf16* src, int lds, const int* map, int n_rows, int width, bf16* dst, int ldd, cudaStream_t st);
int lse_map(const float* src, int n_src, const int* map, int n_rows, int H, float* dst, cudaStream_t st);
int dqkv_from_ext(const bf16* ext, const int* ext_row, int T, int H, int Hkv, int hd, const float2* cs, const int* pos,
                  bf16* dqkv, cudaStream_t st);
int prefix_grad(const bf16* dqkv_ext, int Nq, int Nkv, const PrefixClient* pc, int n_pc, int total_rows,
                const int* seq_ext0, int layer, cudaStream_t st);

// ---------------------------------------------------------------- AdamW + bf16 refresh
struct AdamSeg {              // one (client, layer, target, A|B) parameter block
  long long p_off;            // offset into the client's flat fp32 buffers
  int rows, cols;             // source [rows, cols] row-major
  int client;                 // index into AdamHyper array
  bf16* dst;                  // bf16 copy destination base
  int dst_ld;
  int is_b;                   // B [N, r]: row n -> dst row map; col i -> dst col i
  int row_blk, row_blk_stride, row_base;  // dst_row = row_base + (n / row_blk)*row_blk_stride + n % row_blk
};
struct AdamHyper {
  float* p; float* g; float* m; float* v;
  // torch.optim.AdamW scalar conventions: every scalar below is formed in double on the host, then rounded
  float beta1, beta2, omb1, omb2;   // beta, 1 - beta
  float decay;                       // 1 - lr * weight_decay
  float step_size;                   // lr / (1 - beta1^t)
  float bc2_sqrt;                    // sqrt(1 - beta2^t)
  float eps;
  int do_update;              // 0: only refresh the bf16 copy (set_adapter / register)
};
int adamw_run(const AdamSeg* d_segs, const int4* d_work, int n_work, const AdamHyper* d_hyp, cudaStream_t st);

int fill_rope_table(float2* cs, int max_pos, int hd, float theta, cudaStream_t st);
int convert_bf16_to_f32(const bf16* src, float* dst, long long n, cudaStream_t st);

}  // namespace menos
