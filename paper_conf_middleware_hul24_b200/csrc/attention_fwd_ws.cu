// Varlen causal flash-attention FORWARD, persistent and warp-specialized on the 5th-gen tensor cores
// (tcgen05 / TMEM / TMA), head_dim 128 (Llama-2, OPT-6.7B+) or 64 (OPT-1.3B: NEXT-4; one 128-byte swizzle atom per row).  SURVEY.md §8(a) A3.  Same contract as attn_fwd_kernel (attention.cu):
// a work item never crosses a sequence (so never a client: PAPER.md:428), GQA head h -> kv head h / (H/Hkv),
// LSE saved for the backward.
//
// At the paper's sequence lengths (S <= 2048, hd 128) attention is bound by streaming q, k, v and O through HBM
// and by the softmax, not by the MMAs, so the design is about keeping loads in flight and the exp units busy:
//   * persistent grid (one CTA per SM, 192 KB smem), static round-robin over work items = (sequence, head,
//     128-row q block); items of one (sequence, head) are adjacent so their K/V reads are shared through L2;
//   * warps 0 and 2 = TMA producers: Q (double-buffered across items) and K into a 4-stage ring of 64-key
//     blocks released as soon as S = Q K^T completes; V into its own 4-stage ring released after P V -- so K runs
//     further ahead than V and both run ahead across item boundaries;
//   * warp 1 = MMA issuer (one elected lane): S = Q K^T into a double-buffered TMEM tile, O += P V into a
//     double-buffered TMEM accumulator (the next item's O does not wait for this item's epilogue);
//   * warps 4-7 = softmax, one query row per thread (= TMEM lane): online softmax in the log2 domain with a
//     lazy max (O in TMEM is rescaled only when a row max grows by more than 2^8; P values stay <= 256),
//     P = exp2(S - m) in bf16 written into a 128B-swizzled smem tile that is the next PV MMA's A operand.
#include <algorithm>
#include "common.cuh"
#include "kernels.h"

namespace menos {
namespace {

constexpr int BQ = 128, BKV = 64, K_STAGES = 4, V_STAGES = 4;
constexpr int QA_BYTES = BQ * 64 * 2;                // one SW128 atom of Q: [128 rows][64 cols] = 16 KB
constexpr int KA_BYTES = BKV * 64 * 2;               // one atom of a K / V tile: [64][64] = 8 KB
constexpr int P_BYTES = BQ * BKV * 2;                // 16 KB: 1 atom [128][64]
template <int HD> struct FwdGeo {
  static constexpr int Q_BYTES = BQ * HD * 2;        // HD 128: 2 atoms; 64: 1
  static constexpr int K_BYTES = BKV * HD * 2;
  static constexpr int SMEM = 2 * Q_BYTES + (K_STAGES + V_STAGES) * K_BYTES + 2 * P_BYTES + 1024;
};
constexpr float LOG2E = 1.4426950408889634f;
constexpr float RESCALE_THRESHOLD = 8.0f;            // log2 units
constexpr int NTHREADS = 256;
// MENOS_FWS_TMEM_P (default 1): the softmax threads write P as packed bf16 into the TMEM columns of the S tile they
// have just read and the PV MMA takes it as the A operand from TMEM ("ts" tcgen05.mma), as in the backward: no
// shared-memory P tile, no proxy fence.  The S buffer is only reissued after the PV that reads its P (the MMA warp
// issues PV(j) before S(j + 2), and the tensor pipe runs a thread's MMAs in order).  0: P through shared memory.
#ifndef MENOS_FWS_TMEM_P
#define MENOS_FWS_TMEM_P 1
#endif

// -DMENOS_WS_PROF: per-phase clock64 accounting of one softmax thread and the MMA lane (tuning aid only)
#ifdef MENOS_WS_PROF
__device__ unsigned long long g_ws_prof[16];
#define WSP_DECL long long wsp_t = clock64(); unsigned long long wsp[16] = {0};
#define WSP(k) do { const long long t_ = clock64(); wsp[k] += t_ - wsp_t; wsp_t = t_; } while (0)
#define WSP_FLUSH(cond) do { if (cond) for (int k_ = 0; k_ < 16; ++k_) if (wsp[k_]) atomicAdd(&g_ws_prof[k_], wsp[k_]); } while (0)
#else
#define WSP_DECL
#define WSP(k) do {} while (0)
#define WSP_FLUSH(cond) do {} while (0)
#endif

struct WsParams {
  const int* cu_seqlens;
  const int4* items;      // (seq, q0, head, -)
  int n_items;
  bf16* O; int ld_o;
  float* lse;
  int T, H, Hkv;
  float scale;
};

// try_wait (not a test_wait spin): a waiting producer / MMA warp is suspended by the hardware instead of issuing
// a poll loop that would steal issue slots from the softmax warp sharing its SM sub-partition
__device__ __forceinline__ void wait_spin(uint64_t* bar, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok) {
    asm volatile("{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  }
}

template <int HD>
__global__ void __launch_bounds__(NTHREADS, 1)
attn_fwd_ws_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmKV,
                   const WsParams p) {
  constexpr int Q_BYTES = FwdGeo<HD>::Q_BYTES, K_BYTES = FwdGeo<HD>::K_BYTES;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;                                   // [2][Q_BYTES]
  uint8_t* sK = sQ + 2 * Q_BYTES;                       // [K_STAGES][K_BYTES]
  uint8_t* sV = sK + K_STAGES * K_BYTES;                // [V_STAGES][K_BYTES]
  uint8_t* sP = sV + V_STAGES * K_BYTES;                // [2][P_BYTES]
  __shared__ __align__(8) uint64_t q_full[2], q_empty[2], k_full[K_STAGES], k_empty[K_STAGES];
  __shared__ __align__(8) uint64_t v_full[V_STAGES], v_empty[V_STAGES];
  __shared__ __align__(8) uint64_t s_full[2], s_free[2], p_full[2], pv_done[2], o_free[2];
  __shared__ uint32_t tmem_sh;
  const int tid = threadIdx.x, warp = tid >> 5;

  if (tid == 0) {
    tma_prefetch(&tmQ); tma_prefetch(&tmKV);
    for (int i = 0; i < 2; ++i) {
      mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1);
      mbar_init(&s_full[i], 1); mbar_init(&s_free[i], 128);
      mbar_init(&p_full[i], 128); mbar_init(&pv_done[i], 1); mbar_init(&o_free[i], 128);
    }
    for (int i = 0; i < K_STAGES; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
    for (int i = 0; i < V_STAGES; ++i) { mbar_init(&v_full[i], 1); mbar_init(&v_empty[i], 1); }
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc<512>(&tmem_sh);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_sh;
  // TMEM columns: S[0] 0..63, S[1] 64..127, O[0] 128..128+HD, O[1] 256..256+HD
  const uint32_t tS0 = tmem, tO0 = tmem + 128;

  // work-item geometry, two items deep so that no role stalls on a dependent load at an item boundary: at the top
  // of item i the items entry of i + 2G is loaded and the cu_seqlens entries of i + G (whose items entry arrived an
  // item earlier) are fetched; i + G's values are consumed one item later
  struct GeoPipe { int4 far, nxt; int c0, c1; };
  auto fetch = [&](GeoPipe& g) {
    g.c0 = 0; g.c1 = 0;
    if (g.nxt.x >= 0) { g.c0 = p.cu_seqlens[g.nxt.x]; g.c1 = p.cu_seqlens[g.nxt.x + 1]; }
  };
  auto entry = [&](int item) { return item < p.n_items ? p.items[item] : make_int4(-1, 0, 0, 0); };
  auto pipe_init = [&]() {
    GeoPipe g;
    g.nxt = entry(blockIdx.x);
    fetch(g);
    g.far = entry(blockIdx.x + gridDim.x);
    return g;
  };
  auto item_geom = [&](GeoPipe& g, int item, int& base, int& L, int& q0, int& h, int& nkv) {
    base = g.c0; L = g.c1 - g.c0; q0 = g.nxt.y; h = g.nxt.z;
    nkv = g.nxt.x >= 0 ? (min(L, q0 + BQ) + BKV - 1) / BKV : 0;
    g.nxt = g.far;
    fetch(g);
    g.far = entry(item + 2 * gridDim.x);
  };

  if (warp == 0 || warp == 2) {
    // ============================================================ TMA producers (warp 0: Q, K; warp 2: V)
    if (elect_one()) {
      int it = 0, kc = 0;
      GeoPipe nxt = pipe_init();
      for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
        int base, L, q0, h, nkv;
        item_geom(nxt, item, base, L, q0, h, nkv);
        const int hk = h / (p.H / p.Hkv);
        if (warp == 0) {
          const int qcol = h * HD, kcol = (p.H + hk) * HD;
          const int qb = it & 1;
          wait_spin(&q_empty[qb], ((it >> 1) & 1) ^ 1);
          uint8_t* q = sQ + qb * Q_BYTES;
          mbar_expect_tx(&q_full[qb], Q_BYTES);
#pragma unroll
          for (int a = 0; a < HD / 64; ++a) tma_load_2d(q + a * QA_BYTES, &tmQ, &q_full[qb], qcol + 64 * a, base + q0);
          for (int j = 0; j < nkv; ++j, ++kc) {
            const int s = kc % K_STAGES;
            wait_spin(&k_empty[s], ((kc / K_STAGES) & 1) ^ 1);
            uint8_t* k = sK + s * K_BYTES;
            mbar_expect_tx(&k_full[s], K_BYTES);
#pragma unroll
            for (int a = 0; a < HD / 64; ++a) tma_load_2d(k + a * KA_BYTES, &tmKV, &k_full[s], kcol + 64 * a, base + j * BKV);
          }
        } else {
          const int vcol = (p.H + p.Hkv + hk) * HD;
          for (int j = 0; j < nkv; ++j, ++kc) {
            const int s = kc % V_STAGES;
            wait_spin(&v_empty[s], ((kc / V_STAGES) & 1) ^ 1);
            uint8_t* v = sV + s * K_BYTES;
            mbar_expect_tx(&v_full[s], K_BYTES);
#pragma unroll
            for (int a = 0; a < HD / 64; ++a) tma_load_2d(v + a * KA_BYTES, &tmKV, &v_full[s], vcol + 64 * a, base + j * BKV);
          }
        }
      }
    }
    __syncwarp();
  } else if (warp == 1) {
    // ============================================================ MMA issuer
    constexpr uint32_t IDESC_S = umma_idesc_bf16(BQ, BKV, 0);
    constexpr uint32_t IDESC_PV = umma_idesc_bf16(BQ, HD, 1);
    GeoPipe nxt = pipe_init();
    WSP_DECL
    int it = 0, kvc = 0, sc = 0;   // kvc: global 64-key block counter (K and V rings), sc: S / P buffer counter
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
      int base, L, q0, h, nkv;
      item_geom(nxt, item, base, L, q0, h, nkv);
      const int qb = it & 1, ob = it & 1;
      const uint32_t tO = tO0 + ob * 128;
      wait_spin(&q_full[qb], (it >> 1) & 1);   // (TMEM: O[ob] at 128 + 128 ob, HD columns)
      const uint32_t qa = smem_u32(sQ + qb * Q_BYTES);
      int prev_kv = 0, prev_b = 0, prev_sc = 0;
      auto issue_pv = [&](int j, int gkv, int b, int gsc) {
        const int s = gkv % V_STAGES;
        WSP(15);
        if (j == 0) wait_spin(&o_free[ob], ((it >> 1) & 1) ^ 1);   // previous user of O[ob] fully read
        WSP(14);
        wait_spin(&v_full[s], (gkv / V_STAGES) & 1);
        WSP(13);
        wait_spin(&p_full[b], (gsc >> 1) & 1);
        WSP(14);
        tc_fence_after();
        if (elect_one()) {
          const uint32_t pa = smem_u32(sP + b * P_BYTES), vb = smem_u32(sV + s * K_BYTES);
          const uint64_t vd0 = umma_desc_sw128(vb, KA_BYTES, 1024);
#pragma unroll
          for (int kk = 0; kk < BKV / 16; ++kk) {
            const uint64_t bd = vd0 + (uint64_t)((kk * 2048) >> 4);
#if MENOS_FWS_TMEM_P
            (void)pa;   // A = P packed in S[b]'s first 32 columns: 8 columns (16 keys) per K step
            tc_mma_bf16_ts(tO, tS0 + b * 64 + kk * 8, bd, IDESC_PV, (j > 0 || kk > 0) ? 1u : 0u);
#else
            const uint64_t ad = umma_desc_sw128(pa + kk * 32, 16, 1024);
            tc_mma_bf16(tO, ad, bd, IDESC_PV, (j > 0 || kk > 0) ? 1u : 0u);
#endif
          }
          tc_commit(&pv_done[b]);
          tc_commit(&v_empty[s]);
        }
        __syncwarp();
      };
      for (int j = 0; j < nkv; ++j, ++kvc, ++sc) {
        const int s = kvc % K_STAGES, b = sc & 1;
        WSP(12);
        wait_spin(&k_full[s], (kvc / K_STAGES) & 1);
        WSP(10);
        wait_spin(&s_free[b], ((sc >> 1) & 1) ^ 1);
        WSP(11);
        tc_fence_after();
        if (elect_one()) {
          // descriptors: one base per operand, the K steps as constant 16-byte-unit offsets (the start-address field
          // cannot carry: shared memory is < 256 KB)
          const uint64_t ad0 = umma_desc_sw128(qa, 16, 1024);
          const uint64_t bd0 = umma_desc_sw128(smem_u32(sK + s * K_BYTES), 16, 1024);
#pragma unroll
          for (int kk = 0; kk < HD / 16; ++kk) {
            const uint64_t ad = ad0 + (uint64_t)(((kk >> 2) * QA_BYTES + (kk & 3) * 32) >> 4);
            const uint64_t bd = bd0 + (uint64_t)(((kk >> 2) * KA_BYTES + (kk & 3) * 32) >> 4);
            tc_mma_bf16(tS0 + b * 64, ad, bd, IDESC_S, kk > 0 ? 1u : 0u);
          }
          tc_commit(&s_full[b]);
          tc_commit(&k_empty[s]);                      // K[s] free once S completes
          if (j == nkv - 1) tc_commit(&q_empty[qb]);   // Q free once this item's last S completes
        }
        __syncwarp();
        if (j > 0) issue_pv(j - 1, prev_kv, prev_b, prev_sc);
        prev_kv = kvc; prev_b = b; prev_sc = sc;
      }
      issue_pv(nkv - 1, prev_kv, prev_b, prev_sc);
    }
    WSP(15);
    WSP_FLUSH(blockIdx.x < 8 && (tid & 31) == 0);
  } else if (warp >= 4) {
    // ============================================================ softmax / epilogue (one row per thread)
    const int row = tid - 128;
    const int wq = warp & 3;                        // TMEM lane quadrant of this warp
    const uint32_t lane_off = (uint32_t)(wq * 32) << 16;
    const float sl2 = p.scale * LOG2E;
    int it = 0, sc = 0;
    GeoPipe nxt = pipe_init();
    WSP_DECL
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x, ++it) {
      int base, L, q0, h, nkv;
      item_geom(nxt, item, base, L, q0, h, nkv);
      const int ob = it & 1;
      const uint32_t tO = tO0 + ob * 128 + lane_off;
      const int qpos = q0 + row;
      float m_used = -INFINITY, l = 0.f;
      for (int j = 0; j < nkv; ++j, ++sc) {
        const int b = sc & 1;
        WSP(9);
        wait_spin(&s_full[b], (sc >> 1) & 1);
        WSP(0);
        tc_fence_after();
        float v[64];
        {
          uint32_t a[32], c[32];
          tmem_ld32_nw(tS0 + b * 64 + lane_off, a);
          tmem_ld32_nw(tS0 + b * 64 + 32 + lane_off, c);
          tmem_wait_ld();
#pragma unroll
          for (int i = 0; i < 32; ++i) { v[i] = __uint_as_float(a[i]); v[32 + i] = __uint_as_float(c[i]); }
        }
        tc_fence_before();
        mbar_arrive(&s_free[b]);                    // S[b] is in registers: the next-next S may overwrite it
        WSP(1);
        const int k0 = j * BKV;
        if (k0 + BKV - 1 > q0 || k0 + BKV > L) {    // diagonal / sequence-end block: keys k0+i valid iff i <= lim
          const int lim = min(qpos, L - 1) - k0;
#pragma unroll
          for (int i = 0; i < 64; ++i) v[i] = i <= lim ? v[i] : -INFINITY;
        }
        float mx4[4] = {v[0], v[1], v[2], v[3]};    // 4 independent chains (ILP for the one warp per SMSP)
#pragma unroll
        for (int i = 4; i < 64; ++i) mx4[i & 3] = fmaxf(mx4[i & 3], v[i]);
        float mx = fmaxf(fmaxf(mx4[0], mx4[1]), fmaxf(mx4[2], mx4[3]));
        mx *= sl2;                                  // log2-domain row max (sl2 > 0 commutes with max)
        if (j == 0) {
          m_used = mx;                              // key 0 <= qpos: always finite
        } else {
          const bool need = mx > m_used + RESCALE_THRESHOLD;
          if (__any_sync(0xffffffffu, need)) {
            // O[ob] holds the PV of blocks < j: wait for the last one, then rescale this warp's rows in TMEM
            const int last = sc - 1;
            wait_spin(&pv_done[last & 1], (last >> 1) & 1);
            tc_fence_after();
            const float f = need ? exp2f(m_used - mx) : 1.f;
#pragma unroll 1
            for (int c = 0; c < HD / 32; ++c) {
              float o[32];
              tmem_ld32(tO + c * 32, o);
#pragma unroll
              for (int i = 0; i < 32; ++i) o[i] *= f;
              tmem_st32(tO + c * 32, o);
            }
            if (need) { l *= f; m_used = mx; }
            WSP(3);
          }
        }
        WSP(2);
#if !MENOS_FWS_TMEM_P
        // P[b] was last read by the PV of block sc-2
        if (sc >= 2) wait_spin(&pv_done[b], ((sc - 2) >> 1) & 1);
#endif
        WSP(4);
        uint8_t* prow = sP + b * P_BYTES + row * 128;
        float sum = 0.f;
#if MENOS_FWS_TMEM_P
        uint32_t pw[32];
#endif
#pragma unroll
        for (int c8 = 0; c8 < 8; ++c8) {
          float e[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const float x = fmaf(v[c8 * 8 + i], sl2, -m_used);
            // a quarter of the exponentials on the FMA pipe: the SFU (ex2 + bf16 packing) is this loop's limit
            e[i] = (i & 3) == 3 ? poly_exp2(x) : fast_exp2(x);
            sum += e[i];
          }
          const uint4 u = make_uint4(pack_bf16x2(e[0], e[1]), pack_bf16x2(e[2], e[3]), pack_bf16x2(e[4], e[5]),
                                     pack_bf16x2(e[6], e[7]));
#if MENOS_FWS_TMEM_P
          pw[4 * c8] = u.x; pw[4 * c8 + 1] = u.y; pw[4 * c8 + 2] = u.z; pw[4 * c8 + 3] = u.w;
#else
          *reinterpret_cast<uint4*>(prow + ((c8 ^ (row & 7)) << 4)) = u;
#endif
        }
        l += sum;
        WSP(5);
#if MENOS_FWS_TMEM_P
        {
          uint32_t lo[16], hi[16];
#pragma unroll
          for (int i = 0; i < 16; ++i) { lo[i] = pw[i]; hi[i] = pw[16 + i]; }
          tmem_st16_nw(tS0 + b * 64 + lane_off, lo);
          tmem_st16_nw(tS0 + b * 64 + 16 + lane_off, hi);
          tmem_wait_st();
        }
        (void)prow;
#else
        fence_proxy_async();                        // generic smem writes -> async proxy (tensor core)
#endif
        tc_fence_before();
        mbar_arrive(&p_full[b]);
        WSP(6);
      }
      // epilogue: wait for the last PV, normalise, store O (bf16) and LSE
      const int last = sc - 1;
      wait_spin(&pv_done[last & 1], (last >> 1) & 1);
      WSP(7);
      tc_fence_after();
      const bool rok = qpos < L;
      const float inv = 1.f / l;
      uint32_t o[HD / 32][32];
#pragma unroll
      for (int c = 0; c < HD / 32; ++c) tmem_ld32_nw(tO + c * 32, o[c]);
      tmem_wait_ld();
      // stage this warp's 32 rows (256 B each) in its own P rows (free: every PV of this item has completed), then
      // write them out row-contiguously: one store instruction covers 2 full rows instead of 32 scattered ones
      {
        const int lane = row & 31;
        auto stage = [&](int r, int c) -> uint8_t* {   // 16-byte chunk c (0..15) of staged row r (0..31)
          return sP + (c >> 3) * P_BYTES + (wq * 32 + r) * 128 + (((c & 7) ^ (r & 7)) << 4);
        };
#pragma unroll
        for (int c = 0; c < HD / 32; ++c)
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const uint32_t* w = o[c] + 8 * q;
            *reinterpret_cast<uint4*>(stage(lane, c * 4 + q)) =
                make_uint4(pack_bf16x2(__uint_as_float(w[0]) * inv, __uint_as_float(w[1]) * inv),
                           pack_bf16x2(__uint_as_float(w[2]) * inv, __uint_as_float(w[3]) * inv),
                           pack_bf16x2(__uint_as_float(w[4]) * inv, __uint_as_float(w[5]) * inv),
                           pack_bf16x2(__uint_as_float(w[6]) * inv, __uint_as_float(w[7]) * inv));
          }
        __syncwarp();
        constexpr int LPR = HD / 8, RPI = 32 / LPR;   // lanes per staged row (16-byte chunks), rows per instruction
        const int half = lane / LPR, c = lane % LPR;
#pragma unroll 4
        for (int r2 = 0; r2 < 32; r2 += RPI) {
          const int r = r2 + half, qp = q0 + wq * 32 + r;
          const uint4 u = *reinterpret_cast<const uint4*>(stage(r, c));
          if (qp < L) *reinterpret_cast<uint4*>(p.O + (size_t)(base + qp) * p.ld_o + h * HD + c * 8) = u;
        }
        __syncwarp();
      }
      tc_fence_before();
      mbar_arrive(&o_free[ob]);
      if (rok) p.lse[(size_t)h * p.T + base + qpos] = (m_used + log2f(l)) / LOG2E;
      WSP(8);
    }
    WSP_FLUSH(blockIdx.x < 8 && tid == 128);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

}  // namespace

bool tma_map_2d(CUtensorMap* out, const void* ptr, uint64_t rows, uint64_t cols, uint64_t ld, uint32_t bc,
                uint32_t br);

void attn_snake_waves(std::vector<int4>& v, size_t first, int grid) {
  if (grid <= 1) return;
  const size_t n = v.size() - first, G = (size_t)grid;
  if (n <= G) return;   // one wave: the launch grid is n, nothing to balance
  for (size_t w = 1; w * G < n; w += 2) {
    const size_t a = first + w * G, b = first + std::min(n, (w + 1) * G);
    if (b - a == G) std::reverse(v.begin() + a, v.begin() + b);   // a partial last wave stays as it is (the kernels
                                                                   // take no placeholder items)
  }
}

void attn_ws_items(const int* seq_len, int n_seqs, int H, std::vector<int4>& out, int order, int grid) {
  // (sequence, head) groups, q blocks of a group adjacent and largest first: the group's K/V stays in L2
  const size_t first = out.size();
  for (int i = 0; i < n_seqs; ++i)
    for (int h = 0; h < H; ++h)
      for (int q = ((seq_len[i] - 1) / BQ) * BQ; q >= 0; q -= BQ) out.push_back(make_int4(i, q, h, 0));
  if (order == 0) return;
  // LPT for the static round-robin of the persistent grids: stable sort by work, largest first.  order 1:
  // work ~ causal kv blocks of a query block (forward, dQ); order 2: ~ query blocks after a key block (dK/dV)
  std::vector<int> len(seq_len, seq_len + n_seqs);
  auto cost = [&](const int4& it) {
    const int L = len[it.x];
    return order == 1 ? std::min(L, it.y + BQ) : L - it.y;
  };
  std::stable_sort(out.begin() + first, out.end(), [&](const int4& a, const int4& b) { return cost(a) > cost(b); });
  attn_snake_waves(out, first, grid);
}

// (sequence, kv head) items of the one-pass backward, LPT: longest sequence first (stable)
void attn_seq_items(const int* seq_len, int n_seqs, int Hkv, std::vector<int4>& out) {
  const size_t first = out.size();
  for (int i = 0; i < n_seqs; ++i)
    for (int h = 0; h < Hkv; ++h) out.push_back(make_int4(i, 0, h, 0));
  std::stable_sort(out.begin() + first, out.end(),
                   [&](const int4& a, const int4& b) { return seq_len[a.x] > seq_len[b.x]; });
}

#ifdef MENOS_WS_PROF
int attn_ws_prof_read(unsigned long long* out) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out, g_ws_prof, sizeof(unsigned long long) * 16);
  unsigned long long z[16] = {0};
  cudaMemcpyToSymbol(g_ws_prof, z, sizeof z);
  return 0;
}
#endif

template <int HD>
static int launch_fwd_ws(const AttnArgs& a, const int4* items, int n_items, int num_sms, cudaStream_t st) {
  CUtensorMap mQ, mKV;
  if (!tma_map_2d(&mQ, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, BQ)) return -2;
  if (!tma_map_2d(&mKV, a.qkv, a.T, a.ld_qkv, a.ld_qkv, 64, BKV)) return -2;
  WsParams p;
  p.cu_seqlens = a.cu_seqlens; p.items = items; p.n_items = n_items; p.O = a.O; p.ld_o = a.ld_o; p.lse = a.lse;
  p.T = a.T; p.H = a.H; p.Hkv = a.Hkv; p.scale = a.scale;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(attn_fwd_ws_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize, FwdGeo<HD>::SMEM);
    attr = true;
  }
  const int grid = n_items < num_sms ? n_items : num_sms;
  attn_fwd_ws_kernel<HD><<<grid, NTHREADS, FwdGeo<HD>::SMEM, st>>>(mQ, mKV, p);
  ++g_launch_count;
  return cudaPeekAtLastError() == cudaSuccess ? 0 : -3;
}

int attn_fwd_ws(const AttnArgs& a, const int4* items, int n_items, int num_sms, cudaStream_t st) {
  if (n_items <= 0) return 0;
  if (a.hd == 128) return launch_fwd_ws<128>(a, items, n_items, num_sms, st);
  if (a.hd == 64) return launch_fwd_ws<64>(a, items, n_items, num_sms, st);
  return -1;
}

}  // namespace menos
