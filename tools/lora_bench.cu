// Isolated timing of the segmented LoRA side kernels at BASELINE cfg1 shapes (tuning aid; not a bench value).
// 4 clients x 2048 tokens, q,v r=8 (slot width 16 per target).
#include <cstdio>
#include <vector>
#include "../paper_conf_middleware_hul24_b200/csrc/kernels.h"
using namespace menos;
template <class F> float timeit(F f) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) f();
  cudaEventRecord(a); for (int i = 0; i < 20; ++i) f(); cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); return ms * 1000.f / 20;
}
int main() {
  const int T = 8192, d = 4096, Nqkv = 12288, R = 128, nc = 4, Tc = 2048;
  bf16 *X, *dY, *A, *B, *U, *dU; float* G;
  cudaMalloc(&X, (size_t)T * d * 2); cudaMalloc(&dY, (size_t)T * Nqkv * 2);
  cudaMalloc(&A, (size_t)R * d * 2); cudaMalloc(&B, (size_t)Nqkv * R * 2);
  cudaMalloc(&U, (size_t)T * R * 2); cudaMalloc(&dU, (size_t)T * R * 2); cudaMalloc(&G, (size_t)64 << 20);
  cudaMemset(X, 0, (size_t)T * d * 2); cudaMemset(dY, 0, (size_t)T * Nqkv * 2);
  std::vector<LoraRowsProblem> f, du, du1; std::vector<LoraTokRedProblem> db, da;
  for (int c = 0; c < nc; ++c) {
    LoraRowsProblem p{}; p.A = X + (size_t)c * Tc * d; p.lda = d; p.B = A + (size_t)c * 32 * d; p.ldb = d; p.b_kn = 0;
    p.C = U + (size_t)c * Tc * R + c * 32; p.ldc = R; p.M = Tc; p.N = 32; p.K = d; p.scale = 2.f; f.push_back(p);
    LoraRowsProblem q{}; q.A = dY + (size_t)c * Tc * Nqkv; q.lda = Nqkv; q.B = B + c * 32; q.ldb = R; q.b_kn = 1;
    q.C = dU + (size_t)c * Tc * R + c * 32; q.ldc = R; q.M = Tc; q.N = 32; q.K = Nqkv; q.scale = 2.f; du1.push_back(q);
    for (int t = 0; t < 2; ++t) {
      const int base = t == 0 ? 0 : 8192;
      LoraRowsProblem r{}; r.A = dY + (size_t)c * Tc * Nqkv + base; r.lda = Nqkv; r.B = B + (size_t)base * R + c * 32 + 16 * t;
      r.ldb = R; r.b_kn = 1; r.C = dU + (size_t)c * Tc * R + c * 32 + 16 * t; r.ldc = R; r.M = Tc; r.N = 16; r.K = 4096;
      r.scale = 2.f; du.push_back(r);
      LoraTokRedProblem pb{}; pb.P = dY + (size_t)c * Tc * Nqkv + base; pb.ldp = Nqkv; pb.p_blk = 1 << 30; pb.p_blk_stride = 0;
      pb.Q = U + (size_t)c * Tc * R + c * 32 + 16 * t; pb.ldq = R; pb.C = G + (c * 2 + t) * 65536; pb.ldc = 8; pb.M = 4096; pb.N = 8;
      pb.T = Tc; pb.scale = 1.f; db.push_back(pb);
      LoraTokRedProblem pa{}; pa.P = dU + (size_t)c * Tc * R + c * 32 + 16 * t; pa.ldp = R; pa.p_blk = 1 << 30; pa.p_blk_stride = 0;
      pa.Q = X + (size_t)c * Tc * d; pa.ldq = d; pa.C = G + (8 + c * 2 + t) * 65536; pa.ldc = d; pa.M = 8; pa.N = d;
      pa.T = Tc; pa.scale = 1.f; da.push_back(pa);
    }
  }
  auto up = [](const void* h, size_t n) { void* d; cudaMalloc(&d, n); cudaMemcpy(d, h, n, cudaMemcpyHostToDevice); return d; };
  std::vector<int2> tf, tdu, tdu1; std::vector<int4> tdb, tda;
  lora_rows_tiles(f.data(), (int)f.size(), tf); lora_rows_tiles(du.data(), (int)du.size(), tdu);
  lora_rows_tiles(du1.data(), (int)du1.size(), tdu1);
  lora_tokred_tiles(db.data(), (int)db.size(), 128, 16, tdb); lora_tokred_tiles(da.data(), (int)da.size(), 16, 128, tda);
  auto *df = (LoraRowsProblem*)up(f.data(), f.size() * sizeof f[0]), *ddu = (LoraRowsProblem*)up(du.data(), du.size() * sizeof du[0]);
  auto *ddu1 = (LoraRowsProblem*)up(du1.data(), du1.size() * sizeof du1[0]);
  auto *ddb = (LoraTokRedProblem*)up(db.data(), db.size() * sizeof db[0]), *dda = (LoraTokRedProblem*)up(da.data(), da.size() * sizeof da[0]);
  auto *dtf = (int2*)up(tf.data(), tf.size() * 8), *dtdu = (int2*)up(tdu.data(), tdu.size() * 8), *dtdu1 = (int2*)up(tdu1.data(), tdu1.size() * 8);
  auto *dtdb = (int4*)up(tdb.data(), tdb.size() * 16), *dtda = (int4*)up(tda.data(), tda.size() * 16);
  float t1 = timeit([&] { lora_rows_run(df, dtf, (int)tf.size(), 32, 0); });
  float t2 = timeit([&] { lora_rows_run(ddu1, dtdu1, (int)tdu1.size(), 32, 0); });
  float t3 = timeit([&] { lora_rows_run(ddu, dtdu, (int)tdu.size(), 16, 0); });
  float t4 = timeit([&] { lora_tokred_run(ddb, dtdb, (int)tdb.size(), 128, 0); });
  float t5 = timeit([&] { lora_tokred_run(dda, dtda, (int)tda.size(), 16, 0); });
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
  printf("shrink fwd  %7.1f us  %5.0f GB/s (X %d MB)\n", t1, T * d * 2.0 / t1 / 1e3, T * d * 2 >> 20);
  printf("dU group    %7.1f us  %5.0f GB/s (dY %d MB)\n", t2, T * (double)Nqkv * 2 / t2 / 1e3, int(T * (double)Nqkv * 2 / 1048576));
  printf("dU per-tgt  %7.1f us  %5.0f GB/s (dY q,v %d MB)\n", t3, T * 8192.0 * 2 / t3 / 1e3, T * 8192 * 2 >> 20);
  printf("dB tokred   %7.1f us  %5.0f GB/s\n", t4, T * 8192.0 * 2 / t4 / 1e3);
  printf("dA tokred   %7.1f us  %5.0f GB/s\n", t5, T * (double)d * 2 / t5 / 1e3);
  return 0;
}
