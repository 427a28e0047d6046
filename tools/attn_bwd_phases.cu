// Per-phase clock accounting of the persistent dK/dV backward kernel at the cfg1 shape (tuning aid).
// Build (on the GPU box): MENOS_NVCC_DEFS=-DMENOS_BWS_PROF python -m paper_conf_middleware_hul24_b200.build -f, then
//   nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_bwd_phases.cu -I<pkg>/csrc <pkg>/_lib/*.o -lcuda -ldl
// Run: ./a.out [ds]   (ds: the dS-stored backward; else the recompute path)
#include <cstdio>
#include <vector>
#include <cmath>
#include <cstring>
#include "../paper_conf_middleware_hul24_b200/csrc/kernels.h"
namespace menos { int attn_bws_prof_read(unsigned long long* out); extern int g_attn_order; }
using namespace menos;
int main(int argc, char** argv) {
  const bool ds_path = argc > 1 && argv[1][0] == 'd';   // "ds": the dS-stored backward (default path since r2)
  const int nseq = 16, S = 512, H = 32, Hkv = 32, hd = 128, T = nseq * S, N = (H + 2 * Hkv) * hd;
  std::vector<int> cu(nseq + 1), lens(nseq, S);
  for (int i = 0; i <= nseq; ++i) cu[i] = i * S;
  std::vector<uint16_t> h(size_t(T) * N);
  unsigned x = 1;
  for (auto& v : h) { x = x * 1664525u + 1013904223u; float f = ((x >> 9) / 8388608.f - 0.5f) * 2.f; unsigned u; memcpy(&u, &f, 4); v = u >> 16; }
  bf16 *qkv, *dO, *dqkv; float *lse, *D; int* dcu; int4 *ikv, *iq; float2* cs;
  cudaMalloc(&qkv, h.size() * 2); cudaMemcpy(qkv, h.data(), h.size() * 2, cudaMemcpyHostToDevice);
  cudaMalloc(&dO, size_t(T) * H * hd * 2); cudaMemcpy(dO, h.data(), size_t(T) * H * hd * 2, cudaMemcpyHostToDevice);
  cudaMalloc(&dqkv, h.size() * 2); cudaMalloc(&lse, size_t(H) * T * 4); cudaMalloc(&D, size_t(H) * T * 4);
  cudaMemset(lse, 0, size_t(H) * T * 4); cudaMemset(D, 0, size_t(H) * T * 4);
  cudaMalloc(&cs, size_t(S) * 64 * 8); fill_rope_table(cs, S, hd, 1e4f, 0);
  cudaMalloc(&dcu, cu.size() * 4); cudaMemcpy(dcu, cu.data(), cu.size() * 4, cudaMemcpyHostToDevice);
  std::vector<int4> a1, a2; attn_ws_items(lens.data(), nseq, Hkv, a1, 2); attn_ws_items(lens.data(), nseq, H, a2, 1);
  cudaMalloc(&ikv, a1.size() * 16); cudaMemcpy(ikv, a1.data(), a1.size() * 16, cudaMemcpyHostToDevice);
  cudaMalloc(&iq, a2.size() * 16); cudaMemcpy(iq, a2.data(), a2.size() * 16, cudaMemcpyHostToDevice);
  AttnArgs a; memset(&a, 0, sizeof a);
  a.qkv = qkv; a.ld_qkv = N; a.cu_seqlens = dcu; a.T = T; a.H = H; a.Hkv = Hkv; a.hd = hd; a.scale = 1.f / sqrtf(hd);
  a.dO = dO; a.ld_do = H * hd; a.D = D; a.lse = lse; a.dqkv = dqkv; a.ld_dqkv = N; a.rope_cs = cs;
  unsigned long long pr[16];
  AttnDsPlan plan;
  attn_ds_plan(lens.data(), nseq, H, Hkv, 32768, plan);
  bf16* ds; int* dbase; int4 *pkv, *pq;
  const long long cap = attn_ds_total_tiles(lens.data(), nseq, H);
  cudaMalloc(&ds, (size_t)cap * 16384); cudaMalloc(&dbase, plan.base.size() * 4);
  cudaMalloc(&pkv, plan.items_kv.size() * 16); cudaMalloc(&pq, plan.items_q.size() * 16);
  cudaMemcpy(dbase, plan.base.data(), plan.base.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(pkv, plan.items_kv.data(), plan.items_kv.size() * 16, cudaMemcpyHostToDevice);
  cudaMemcpy(pq, plan.items_q.data(), plan.items_q.size() * 16, cudaMemcpyHostToDevice);
  auto run = [&]() {
    if (ds_path) attn_bwd_ws_ds(a, pkv, (int)plan.items_kv.size(), pq, (int)plan.items_q.size(), ds, cap, dbase, 148, 0);
    else attn_bwd_ws(a, ikv, (int)a1.size(), iq, (int)a2.size(), 148, 0);
  };
  for (int r = 0; r < 3; ++r) run();
  attn_bws_prof_read(pr);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int r = 0; r < 10; ++r) run();
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  attn_bws_prof_read(pr);
  printf("err %s  %.1f us per dkdv+dq launch pair\n", cudaGetErrorString(cudaGetLastError()), ms * 100.f);
  const char* nm[16] = {"ew lse stage/loop", "ew ew_sync", "ew wait S", "ew tmem+math", "ew pack+TMEM st (or pd_free wait)", "ew arrive (or smem P/dS store)", "ew epi wait acc", "ew epi tmem->stage", "ew epi copy-out", "ew lse: value wait+store", "mma loop", "mma wait ew_done", "mma wait acc_free", "mma issue acc", "mma wait Q/dO", "mma wait K/V (item start)"};
  unsigned long long te = 0, tm = 0;
  for (int k = 0; k < 10; ++k) te += pr[k];
  for (int k = 10; k < 16; ++k) tm += pr[k];
  for (int k = 0; k < 16; ++k) printf("%-22s %6.1f%%  %.0f cycles/CTA/launch\n", nm[k], 100.0 * pr[k] / (k < 10 ? te : tm), pr[k] / 80.0);
  return 0;
}
