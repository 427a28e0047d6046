// Per-phase clock accounting of the persistent attention FORWARD kernel at the cfg1 shape (tuning aid).
// Build (on the GPU box): MENOS_NVCC_DEFS=-DMENOS_WS_PROF python -m paper_conf_middleware_hul24_b200.build -f, then
//   nvcc -std=c++17 -gencode arch=compute_100a,code=sm_100a tools/attn_fwd_phases.cu -I<pkg>/csrc -Iinclude <pkg>/_lib/*.o -lcuda -ldl
#include <cstdio>
#include <cstring>
#include <cmath>
#include <vector>
#include "../paper_conf_middleware_hul24_b200/csrc/kernels.h"
namespace menos { int attn_ws_prof_read(unsigned long long* out); }
using namespace menos;
int main() {
  const int nseq = 16, S = 512, H = 32, Hkv = 32, hd = 128, T = nseq * S, N = (H + 2 * Hkv) * hd;
  std::vector<int> cu(nseq + 1), lens(nseq, S);
  for (int i = 0; i <= nseq; ++i) cu[i] = i * S;
  std::vector<uint16_t> h(size_t(T) * N);
  unsigned x = 1;
  for (auto& v : h) { x = x * 1664525u + 1013904223u; float f = ((x >> 9) / 8388608.f - 0.5f) * 2.f; unsigned u; memcpy(&u, &f, 4); v = u >> 16; }
  bf16 *qkv, *O; float* lse; int* dcu; int4* items;
  cudaMalloc(&qkv, h.size() * 2); cudaMemcpy(qkv, h.data(), h.size() * 2, cudaMemcpyHostToDevice);
  cudaMalloc(&O, size_t(T) * H * hd * 2); cudaMalloc(&lse, size_t(H) * T * 4);
  cudaMalloc(&dcu, cu.size() * 4); cudaMemcpy(dcu, cu.data(), cu.size() * 4, cudaMemcpyHostToDevice);
  std::vector<int4> it; attn_ws_items(lens.data(), nseq, H, it, 1, 148);
  cudaMalloc(&items, it.size() * 16); cudaMemcpy(items, it.data(), it.size() * 16, cudaMemcpyHostToDevice);
  AttnArgs a; memset(&a, 0, sizeof a);
  a.qkv = qkv; a.ld_qkv = N; a.O = O; a.ld_o = H * hd; a.lse = lse; a.cu_seqlens = dcu; a.T = T; a.H = H; a.Hkv = Hkv;
  a.hd = hd; a.scale = 1.f / sqrtf(hd);
  unsigned long long pr[16];
  for (int r = 0; r < 3; ++r) attn_fwd_ws(a, items, (int)it.size(), 148, 0);
  attn_ws_prof_read(pr);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  for (int r = 0; r < 10; ++r) attn_fwd_ws(a, items, (int)it.size(), 148, 0);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  attn_ws_prof_read(pr);
  printf("err %s  %.1f us per forward\n", cudaGetErrorString(cudaGetLastError()), ms * 100.f);
  const char* nm[16] = {"sm wait S", "sm S ld + release", "sm max/mask", "sm rescale O", "sm (P buffer wait)",
                        "sm exp + pack + P store", "sm arrive", "sm epi wait PV", "sm epilogue", "sm loop top",
                        "mma wait s_free", "mma issue S", "mma wait K", "mma wait V", "mma wait P / o_free", "mma other"};
  unsigned long long ts = 0, tm = 0;
  for (int k = 0; k < 10; ++k) ts += pr[k];
  for (int k = 10; k < 16; ++k) tm += pr[k];
  for (int k = 0; k < 16; ++k) printf("%-26s %6.1f%%  %.0f cycles/CTA/launch\n", nm[k], 100.0 * pr[k] / (k < 10 ? ts : tm), pr[k] / 80.0);
  return 0;
}
