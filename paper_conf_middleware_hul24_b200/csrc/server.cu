// Menos server runtime behind include/menos.h: WeightStore (one bf16 base copy), ClientRegistry (LoRA
// adapters + AdamW state in shared slot tables), BatchPacker (segment tables), ActivationArena (temporal
// sharing), and the per-layer forward / backward schedules over the sm_100a kernels.
//
// Paper anchors: spatial sharing of theta (§3.1), on-demand allocation of I and release
// after backward (§3.2, Eq.3), the serving process Alg.1, the 4-step
// cycle, client profiling of M_f / M_b (Alg.2 L2).
#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <memory>
#include <string>
#include <vector>

#include "../../include/menos.h"
#include "../../include/menos_testing.h"
#include <type_traits>
#include "kernels.h"
#include "comm.h"

using namespace menos;

// =====================================================================================================
// errors
// =====================================================================================================
static thread_local std::string tl_err;
static void set_err(const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  tl_err = buf;
}
#define FAIL(code, ...) do { set_err(__VA_ARGS__); return (code); } while (0)
namespace menos {
// shared with sched.cpp (the Alg.2 scheduler reports through the same thread-local message)
void set_last_error(const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  tl_err = buf;
}
}  // namespace menos
#define CUDA_TRY(x)                                                                         \
  do {                                                                                      \
    cudaError_t e_ = (x);                                                                   \
    if (e_ != cudaSuccess) FAIL(MENOS_ECUDA, "%s: %s (%s:%d)", #x, cudaGetErrorString(e_), __FILE__, __LINE__); \
  } while (0)
#define K_TRY(x)                                                                              \
  do {                                                                                        \
    int r_ = (x);                                                                             \
    if (r_ != 0) {                                                                            \
      cudaError_t e_ = cudaGetLastError();                                                    \
      FAIL(MENOS_ECUDA, "%s failed (%d): %s (%s:%d)", #x, r_, cudaGetErrorString(e_), __FILE__, __LINE__); \
    }                                                                                         \
  } while (0)

static inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }
constexpr size_t kDsTileBytes = 128 * 64 * 2;   // one bf16 dS^T tile [128 keys][64 queries]
// lse / D rows are read by 272-byte bulk copies from a 16-byte-aligned start (attention backward): 512 B of slack
constexpr size_t kLsePad = 512;

// =====================================================================================================
// per-kernel-class CUDA-event profiler (bench.py's live roofline; off by default)
// =====================================================================================================
enum ProfClass { PC_GEMM = 0, PC_ATTN_FWD, PC_ATTN_BWD, PC_LORA, PC_NORM, PC_ATTN_PREP, PC_ADAMW, PC_N };
static const char* kProfName[PC_N] = {"gemm_tcgen05", "attn_fwd", "attn_bwd", "lora_side", "rmsnorm",
                                      "attn_bwd_prep", "adamw"};
struct ProfRec { cudaEvent_t a, b; int cls; double flops, bytes; };
static bool g_prof_on = false;
static std::vector<ProfRec> g_prof;
static std::vector<cudaEvent_t> g_ev_pool;
static size_t g_ev_used = 0;
static cudaEvent_t prof_event() {
  if (g_ev_used == g_ev_pool.size()) {
    cudaEvent_t e;
    cudaEventCreate(&e);
    g_ev_pool.push_back(e);
  }
  return g_ev_pool[g_ev_used++];
}
struct ProfScope {
  bool on; ProfRec r; cudaStream_t st;
  ProfScope(int cls, double flops, double bytes, cudaStream_t s) : on(g_prof_on), st(s) {
    if (!on) return;
    r.cls = cls; r.flops = flops; r.bytes = bytes; r.a = prof_event(); r.b = prof_event();
    cudaEventRecord(r.a, st);
  }
  ~ProfScope() {
    if (!on) return;
    cudaEventRecord(r.b, st);
    g_prof.push_back(r);
  }
};
static inline int ceil_div(int a, int b) { return (a + b - 1) / b; }

// =====================================================================================================
// target / group geometry
// =====================================================================================================
enum { TQ = 0, TK, TV, TO, TG, TU, TD, NT };
constexpr int TPFX = 7;   // target index of the prefix-tuning adapter in get/set_adapter (MENOS_T_PREFIX, NEXT-3)
enum { GQKV = 0, GO, GGU, GD, NG };
static const int kTargetGroup[NT] = {GQKV, GQKV, GQKV, GO, GGU, GGU, GD};

struct Dims {
  // local (per tensor-parallel rank) extents: H, Hkv, f are the global ones / tp_world
  int d, H, Hkv, hd, f, fpad, Nq, Nkv, Nqkv;
  int arch;                        // MENOS_ARCH_LLAMA / MENOS_ARCH_OPT (NEXT-4)
  int gu_cols;                     // columns of the saved MLP activation: [gate|up] 2*fpad (Llama), relu(fc1) fpad (OPT)
  int tp_rank, tp_world;
  bool sp;                         // tensor parallel with sequence-parallel residual streams (include/menos.h)
  int K_glob[NT];                  // global input dim of each projection (LoRA A init bound, A slicing)
  bool a_rep[NT];                  // A replicated across ranks (column-parallel); else B replicated (row-parallel)
  float eps, theta;
  int K_t[NT], N_t[NT];            // projection input/output dims (natural)
  int K_g[NG], N_g[NG], ldK_g[NG]; // group GEMM input dim, output dim, Acat leading dim
  // Bcat row map per target: row = base + (n / blk) * stride + n % blk
  int rb_base[NT], rb_blk[NT], rb_stride[NT];
};

static Dims make_dims(const menos_model_cfg& c, int tp_rank = 0, int tp_world = 1, bool sp = false) {
  Dims D;
  D.tp_rank = tp_rank; D.tp_world = tp_world; D.sp = sp;
  D.d = c.d_model; D.H = c.n_heads / tp_world; D.Hkv = c.n_kv_heads / tp_world; D.hd = c.d_model / c.n_heads;
  D.f = c.d_ff / tp_world; D.fpad = (int)align_up(D.f, 128);
  D.Nq = D.H * D.hd; D.Nkv = D.Hkv * D.hd; D.Nqkv = D.Nq + 2 * D.Nkv;
  D.eps = c.rms_eps; D.theta = c.rope_theta;
  D.arch = c.arch;
  const bool opt = c.arch == MENOS_ARCH_OPT;
  D.gu_cols = opt ? D.fpad : 2 * D.fpad;
  const int K[NT] = {D.d, D.d, D.d, D.Nq, D.d, D.d, D.f};
  const int N[NT] = {D.Nq, D.Nkv, D.Nkv, D.d, D.f, D.f, D.d};
  for (int t = 0; t < NT; ++t) {
    D.K_t[t] = K[t]; D.N_t[t] = N[t];
    D.a_rep[t] = !(t == TO || t == TD);
    D.K_glob[t] = D.a_rep[t] ? K[t] : K[t] * tp_world;
  }
  D.K_g[GQKV] = D.d;  D.N_g[GQKV] = D.Nqkv;    D.ldK_g[GQKV] = D.d;
  D.K_g[GO] = D.Nq;   D.N_g[GO] = D.d;         D.ldK_g[GO] = D.Nq;
  D.K_g[GGU] = D.d;   D.N_g[GGU] = D.gu_cols;  D.ldK_g[GGU] = D.d;
  D.K_g[GD] = D.f;    D.N_g[GD] = D.d;         D.ldK_g[GD] = D.fpad;
  const int big = 1 << 30;
  int base[NT] = {0, D.Nq, D.Nq + D.Nkv, 0, 0, 128, 0};
  int blk[NT] = {big, big, big, big, 128, 128, big};
  int str[NT] = {0, 0, 0, 0, 256, 256, 0};
  if (opt) { base[TU] = 0; blk[TU] = big; str[TU] = 0; }   // fc1 rows, not interleaved (gate does not exist)
  for (int t = 0; t < NT; ++t) { D.rb_base[t] = base[t]; D.rb_blk[t] = blk[t]; D.rb_stride[t] = str[t]; }
  return D;
}

// token rows under sequence parallelism: rank r owns rows [r*Tloc, (r+1)*Tloc), Tpad = world*Tloc >= T (the last
// rank's rows past T are padding); without it Tloc = Tpad = T
struct Rows { int T, Tloc, Tpad, row0; };
static inline Rows rows_of(const Dims& D, int T) {
  if (!D.sp) return Rows{T, T, T, 0};
  const int loc = ceil_div(T, D.tp_world);
  return Rows{T, loc, loc * D.tp_world, loc * D.tp_rank};
}

// =====================================================================================================
// arena (first-fit, no cudaMalloc on the hot path)
// =====================================================================================================
struct Arena {
  uint8_t* base = nullptr;
  size_t cap = 0, used = 0, peak = 0;
  std::map<size_t, size_t> free_;  // offset -> size
  std::map<size_t, size_t> live_;
  void init(uint8_t* b, size_t c) { base = b; cap = c; free_.clear(); live_.clear(); free_[0] = c; used = peak = 0; }
  void* alloc(size_t n) {
    n = align_up(n ? n : 256, 256);
    for (auto it = free_.begin(); it != free_.end(); ++it) {
      if (it->second >= n) {
        size_t off = it->first, sz = it->second;
        free_.erase(it);
        if (sz > n) free_[off + n] = sz - n;
        live_[off] = n;
        used += n; peak = std::max(peak, used);
        return base + off;
      }
    }
    return nullptr;
  }
  void release(void* p) {
    if (!p) return;
    size_t off = (uint8_t*)p - base;
    auto it = live_.find(off);
    if (it == live_.end()) return;
    size_t n = it->second;
    live_.erase(it);
    used -= n;
    auto nx = free_.lower_bound(off);
    if (nx != free_.end() && off + n == nx->first) { n += nx->second; free_.erase(nx); }
    auto pv = free_.lower_bound(off);
    if (pv != free_.begin()) {
      --pv;
      if (pv->first + pv->second == off) { off = pv->first; n += pv->second; free_.erase(pv); }
    }
    free_[off] = n;
  }
};

// =====================================================================================================
// clients
// =====================================================================================================
struct Client {
  bool used = false;
  int rank = 0, rs = 0;
  float alpha = 0, s = 0;
  uint32_t mask = 0;
  menos_adamw_cfg opt{};
  int step = 0;
  int cut = 0;                      // first server layer (local index) the client's tokens enter (NEXT-3)
  int col_off[NG] = {0, 0, 0, 0}, width[NG] = {0, 0, 0, 0};
  int sub[NT];                      // slot sub-offset of target t inside the group slot (j * rs), -1 if absent
  float* buf = nullptr;             // P | G | M | V, each n_params fp32
  size_t n_params = 0;
  size_t n_rep = 0;                 // params [0, n_rep) are replicated across tensor-parallel ranks
  std::vector<long long> offA, offB;  // [layer * NT + t]
  int n_prefix = 0;                 // prefix tuning (NEXT-3, R28): P prefix rows per layer; params [layer >= cut][k|v][P][Nkv]
  bf16* pfx = nullptr;              // its bf16 copy, same layout (read by the attention's prefix gather)
  float *P() const { return buf; }
  float *G() const { return buf + n_params; }
  float *M() const { return buf + 2 * n_params; }
  float *V() const { return buf + 3 * n_params; }
};

// column allocator over the slot tables of one group (16-column units)
struct ColAlloc {
  std::map<int, int> free_;  // off -> width
  int cap = 0;
  int alloc(int w) {
    for (auto it = free_.begin(); it != free_.end(); ++it)
      if (it->second >= w) {
        int off = it->first, sz = it->second;
        free_.erase(it);
        if (sz > w) free_[off + w] = sz - w;
        return off;
      }
    return -1;
  }
  void release(int off, int w) {
    free_[off] = w;
    // coalesce
    auto it = free_.begin();
    while (it != free_.end()) {
      auto nx = std::next(it);
      if (nx != free_.end() && it->first + it->second == nx->first) { it->second += nx->second; free_.erase(nx); }
      else it = nx;
    }
  }
  void grow(int newcap) {
    if (newcap > cap) release(cap, newcap - cap);
    cap = newcap;
  }
  bool fits(int w) const {
    for (const auto& kv : free_) if (kv.second >= w) return true;
    return false;
  }
  int max_end() const {  // end of the highest allocated column
    int end = cap;
    auto it = free_.rbegin();
    if (it != free_.rend() && it->first + it->second == cap) end = it->first;
    return end;
  }
};

// =====================================================================================================
// batch
// =====================================================================================================
struct LayerSave {
  float *x, *h;                       // fp32 residual stream (layer input, post-attention residual)
  bf16 *xn, *qkv, *O, *hn, *gu, *a;   // bf16 GEMM operands / attention inputs
  float *rstd1, *rstd2, *lse;
  bf16* U[NG];
};
struct SGList {
  int probs_off = 0, n_probs = 0, tiles_off = 0, n_tiles = 0, max_n = 0; double flops = 0;
  int max_rank = 0; long long max_elems = 0;   // fused dU+dB lists: widest rank, largest T * rs
  int tile_n = 0;                              // token-reduction lists: tile width
  int n_small = 0;                             // fused dU+dB lists: problems [0, n_small) have rank <= 16 (tcgen05),
  int n_wide = 0;                              // of which [0, n_wide) use 256-column slabs
};

struct menos_batch {
  int T = 0, n_seqs = 0;
  bool nograd = false;
  std::vector<int> seq_client, seq_len, cu;
  std::vector<int> bclients, btok_off, btok_n;  // unique clients in batch order, their token ranges
  std::vector<int> pos;
  int R_used[NG] = {0, 0, 0, 0};
  bool g_active[NG] = {false, false, false, false};
  bool save_a = false;
  int n_mt = 0, n_blocks = 0, n_blocks128 = 0;
  int2* d_blocks128 = nullptr;
  double pairs = 0;   // causal (query, key) pairs summed over sequences
  // per-client cut points: the batch is ordered by non-decreasing cut, so
  // the clients active at layer l (cut <= l) are a prefix: tokens [0, Tl[l]), sequences [0, nseq_l[l])
  std::vector<int> Tl, nseq_l, view_of;
  struct AttnView {
    int n_seqs = 0, n_blocks = 0, n_blocks128 = 0, n_items = 0, n_items_kv = 0, n_items_seq = 0;
    double pairs = 0;
    size_t o_items = 0, o_items_kv = 0, o_items_q = 0, o_items_seq = 0;
    int4 *items = nullptr, *items_kv = nullptr, *items_q = nullptr, *items_seq = nullptr;
    // dS-stored backward plan over this view's sequences (attn_ds_plan): per chunk (kv off, n, q off, n)
    bool ds_ok = false;
    std::vector<int4> ds_chunks;
    size_t o_ds_kv = 0, o_ds_q = 0, o_ds_base = 0;
    int4 *ds_kv = nullptr, *ds_q = nullptr;
    int* ds_base = nullptr;
  };
  std::vector<AttnView> views;
  // device metadata
  uint8_t* meta = nullptr;  // arena
  int* d_cu = nullptr; int* d_pos = nullptr; int2* d_blocks = nullptr;
  int2* d_mtile[NG] = {nullptr, nullptr, nullptr, nullptr};
  uint8_t* d_ntile_qkv = nullptr;
  LoraRowsProblem* d_rprobs = nullptr; int2* d_rtiles = nullptr;
  LoraTokRedProblem* d_tprobs = nullptr; int4* d_ttiles = nullptr;
  LoraDUBProblem* d_dprobs = nullptr;
  // forward LoRA shrink on tcgen05, per layer and group: whole-buffer operands + (client, 128-column chunk) problems
  struct ShkList {
    const bf16* X = nullptr; int x_rows = 0, ldx = 0; const bf16* A = nullptr; int a_rows = 0, lda = 0, K = 0;
    bf16* U = nullptr; int ldu = 0;
    int probs_off = 0, tiles_off = 0, n_tiles = 0, max_w = 0; double flops = 0;
  };
  std::vector<ShkList> sg_shk;   // [layer * NG + g]
  // whole-buffer operands of the tcgen05 dU + dB kernel, per layer and group (dY lives in the per-call scratch)
  struct DubBufs { const bf16* Y = nullptr; int ldy = 0; const bf16* U = nullptr; int ldu = 0, rows = 0; };
  std::vector<DubBufs> dub_bufs;
  // dA on tcgen05 (clients whose group slot is <= 64 wide), per layer and group
  struct DaTc {
    int probs_off = 0, n = 0, max_w = 0, max_n = 0; double flops = 0;
    const bf16* X = nullptr; int rows = 0, ldx = 0; const bf16* dU = nullptr; int lddu = 0;
  };
  std::vector<DaTc> da_tc;
  LoraTokRedProblem* d_daprobs = nullptr;
  std::vector<LoraTokRedProblem> h_daprobs;
  LoraShrinkProblem* d_sprobs = nullptr; int2* d_stiles = nullptr;
  // dS-stored attention backward: chunk buffer tiles (0 = the recompute path for this batch)
  long long ds_tiles = 0;
  // per layer, per group: fwd shrink, bwd fused dU + dB (one pass over dY per target), bwd dA (one pass over X per
  // client and group)
  std::vector<SGList> sg_fwd, sg_dub, sg_da;  // [layer * NG + g]
  // saved activations (SAVE) or x_c copy (NOGRAD)
  uint8_t* slab = nullptr;
  std::vector<LayerSave> L;
  // LoRA side problem lists reference the per-call scratch block (dY, dU); the scratch may move between this
  // batch's forward and its backward (another call of a different size in between), so the host copies are kept
  // and relocated before the backward (relocate_scratch_refs)
  std::vector<LoraRowsProblem> h_rprobs;
  std::vector<LoraTokRedProblem> h_tprobs;
  std::vector<LoraDUBProblem> h_dprobs;
  uint8_t* scratch_base = nullptr; size_t scratch_span = 0;
  // live-batch accounting (menos_server::batch_refs / live_save): set when the handle is returned to the caller
  bool counted = false, counted_save = false;
  // prefix tuning (NEXT-3, R28): the attention runs on an EXTENDED batch in which every sequence of a prefix client
  // is preceded by the client's P prefix rows (q = 0, k / v = the layer's prefix); Text = its rows (T without)
  bool has_pfx = false;
  int Text = 0, n_pc = 0, pc_rows = 0;
  std::vector<int> ext_len;           // per sequence: P + L
  AttnView xview;                     // attention work lists over the extension (prefix batches have no mixed cuts)
  int* d_cu_ext = nullptr; int2* d_blocks_ext = nullptr; int2* d_blocks128_ext = nullptr;
  int2* d_ext_src = nullptr;          // per ext row: (token row, -) or (-1, client slot << 16 | prefix row)
  int* d_ext_tok = nullptr;           // per ext row: token row or -1
  int* d_tok_ext = nullptr;           // per token: its ext row
  int* d_seq_ext0 = nullptr;          // per sequence: its first ext row
  int* d_seq_shift = nullptr;         // per sequence: its client's prefix length (RoPE position shift in the kernels)
  PrefixClient* d_pc = nullptr;
  double pairs_ext = 0;
};

// =====================================================================================================
// server
// =====================================================================================================
struct menos_server {
  menos_model_cfg cfg{};
  Dims D{};
  int first_layer = 0, n_layers = 0, device = 0, num_sms = 148;
  menos_server_opts opts{};
  menos_tp_cfg tp{0, 1, nullptr, nullptr, nullptr};  // tensor parallelism (world 1 = replica)
  Comm comm;                                          // its transport (comm.cpp): NCCL or the caller's callback
  // WeightStore: one bf16 copy of every server layer, packed for the kernels
  uint8_t* wbuf = nullptr; size_t wbytes = 0;
  struct LW {
    bf16 *wqkv, *wo, *wgu, *wd;
    float *g1, *g2;
    float *be1, *be2, *bqkv, *bo, *bu, *bd;   // OPT: LayerNorm biases, projection biases (fp32; zero for Llama)
  };
  std::vector<LW> W;
  std::vector<bool> loaded;
  // LoRA slot tables per layer per group (bf16): Bcat [N_g, cap], Acat [cap, ldK_g]
  ColAlloc cols[NG];
  std::vector<bf16*> Bcat[NG], Acat[NG];
  // registry
  std::vector<Client> clients;
  // rope table
  float2* rope = nullptr;
  // arena + scratch
  Arena arena;
  uint8_t* arena_mem = nullptr;
  uint8_t* scratch = nullptr; size_t scratch_bytes = 0;
  // pinned host staging for metadata uploads
  static constexpr int kRing = 4;
  struct Slot { uint8_t* buf = nullptr; size_t bytes = 0; cudaEvent_t ev = nullptr; };
  Slot ring[kRing];
  int ring_next = 0;
  // device copies of the AdamW tables (hyper-params, segments, work list): a ring reused once the kernel that
  // last read an entry has completed (its event), so adapter_step never allocates on the hot path
  Slot dring[kRing];
  int dring_next = 0;
  // live batches: a SAVE batch's LoRA problem lists hold raw slot-table pointers, leading dimensions and each
  // client's gradient buffer, so while one is alive the slot tables may not move (registration that would grow them
  // returns MENOS_ESTATE) and none of its clients may be unregistered (MENOS_ESTATE)
  int live_save = 0;
  std::vector<int> batch_refs;   // per client id: live batches that contain it
  // the one stream this server's work is ordered on (arena slabs and the scratch block are reused in stream order):
  // bound by the first forward / backward / adapter_step, any other stream afterwards is MENOS_EINVAL
  bool stream_bound = false;
  cudaStream_t stream = nullptr;
};

static int bind_stream(menos_server* s, cudaStream_t st) {
  if (!s->stream_bound) { s->stream_bound = true; s->stream = st; return MENOS_OK; }
  if (s->stream != st)
    FAIL(MENOS_EINVAL, "server work must stay on one stream (bound to %p, got %p): arena memory is reused in "
         "stream order", (void*)s->stream, (void*)st);
  return MENOS_OK;
}

// =====================================================================================================
// helpers: weights
// =====================================================================================================
// OPT (NEXT-4): q|k|v, o as for Llama; fc1 -> wgu [fpad, d] (rows >= f zero), fc2 -> wd [d, fpad]; LayerNorm gains
// and biases and the projection biases -> fp32
static int upload_layer_opt(menos_server* s, int l, const menos_layer_weights* w) {
  const Dims& D = s->D;
  auto& L = s->W[l];
  const size_t b2 = 2;
  cudaStream_t st = 0;
  CUDA_TRY(cudaMemcpyAsync(L.wqkv, w->wq, (size_t)D.Nq * D.d * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpyAsync(L.wqkv + (size_t)D.Nq * D.d, w->wk, (size_t)D.Nkv * D.d * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpyAsync(L.wqkv + (size_t)(D.Nq + D.Nkv) * D.d, w->wv, (size_t)D.Nkv * D.d * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpyAsync(L.wo, w->wo, (size_t)D.d * D.Nq * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpyAsync(L.wgu, w->wup, (size_t)D.f * D.d * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpy2DAsync(L.wd, (size_t)D.fpad * b2, w->wdown, (size_t)D.f * b2, (size_t)D.f * b2, D.d,
                             cudaMemcpyDefault, st));
  struct V { const void* src; float* dst; int n; };
  const V vs[] = {{w->g1, L.g1, D.d}, {w->g2, L.g2, D.d}, {w->b1, L.be1, D.d}, {w->b2, L.be2, D.d},
                  {w->bo, L.bo, D.d}, {w->bdown, L.bd, D.d}, {w->bq, L.bqkv, D.Nq}, {w->bk, L.bqkv + D.Nq, D.Nkv},
                  {w->bv, L.bqkv + D.Nq + D.Nkv, D.Nkv}, {w->bup, L.bu, D.f}};
  bf16* tmp = nullptr;
  CUDA_TRY(cudaMalloc(&tmp, (size_t)std::max(D.Nqkv, D.fpad) * b2));
  for (const V& v : vs) {
    CUDA_TRY(cudaMemcpyAsync(tmp, v.src, (size_t)v.n * b2, cudaMemcpyDefault, st));
    K_TRY(convert_bf16_to_f32(tmp, v.dst, v.n, st));
    CUDA_TRY(cudaStreamSynchronize(st));
  }
  CUDA_TRY(cudaFree(tmp));
  s->loaded[l] = true;
  return MENOS_OK;
}

static int upload_layer(menos_server* s, int l, const menos_layer_weights* w) {
  const Dims& D = s->D;
  auto& L = s->W[l];
  const size_t b2 = 2;
  const bool opt = D.arch == MENOS_ARCH_OPT;
  if (!w || !w->wq || !w->wk || !w->wv || !w->wo || (!opt && !w->wgate) || !w->wup || !w->wdown || !w->g1 || !w->g2)
    FAIL(MENOS_EINVAL, "layer %d: null weight pointer", l);
  if (opt && (!w->bq || !w->bk || !w->bv || !w->bo || !w->bup || !w->bdown || !w->b1 || !w->b2))
    FAIL(MENOS_EINVAL, "layer %d: OPT needs every bias", l);
  cudaStream_t st = 0;
  if (opt) return upload_layer_opt(s, l, w);
  CUDA_TRY(cudaMemcpyAsync(L.wqkv, w->wq, (size_t)D.Nq * D.d * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpyAsync(L.wqkv + (size_t)D.Nq * D.d, w->wk, (size_t)D.Nkv * D.d * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpyAsync(L.wqkv + (size_t)(D.Nq + D.Nkv) * D.d, w->wv, (size_t)D.Nkv * D.d * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpyAsync(L.wo, w->wo, (size_t)D.d * D.Nq * b2, cudaMemcpyDefault, st));
  // gate/up interleaved in 128-row blocks: rows [fb*256, +128) gate, [fb*256+128, +128) up
  const int nfull = D.f / 128, tail = D.f % 128;
  const size_t rowb = (size_t)D.d * b2;
  if (nfull > 0) {
    CUDA_TRY(cudaMemcpy2DAsync(L.wgu, 256 * rowb, w->wgate, 128 * rowb, 128 * rowb, nfull, cudaMemcpyDefault, st));
    CUDA_TRY(cudaMemcpy2DAsync(L.wgu + (size_t)128 * D.d, 256 * rowb, w->wup, 128 * rowb, 128 * rowb, nfull,
                               cudaMemcpyDefault, st));
  }
  if (tail) {
    CUDA_TRY(cudaMemcpyAsync(L.wgu + (size_t)nfull * 256 * D.d, (const uint8_t*)w->wgate + (size_t)nfull * 128 * rowb,
                             tail * rowb, cudaMemcpyDefault, st));
    CUDA_TRY(cudaMemcpyAsync(L.wgu + ((size_t)nfull * 256 + 128) * D.d,
                             (const uint8_t*)w->wup + (size_t)nfull * 128 * rowb, tail * rowb, cudaMemcpyDefault, st));
  }
  CUDA_TRY(cudaMemcpy2DAsync(L.wd, (size_t)D.fpad * b2, w->wdown, (size_t)D.f * b2, (size_t)D.f * b2, D.d,
                             cudaMemcpyDefault, st));
  // gains -> fp32
  bf16* tmp = nullptr;
  CUDA_TRY(cudaMalloc(&tmp, (size_t)2 * D.d * b2));
  CUDA_TRY(cudaMemcpyAsync(tmp, w->g1, D.d * b2, cudaMemcpyDefault, st));
  CUDA_TRY(cudaMemcpyAsync(tmp + D.d, w->g2, D.d * b2, cudaMemcpyDefault, st));
  K_TRY(convert_bf16_to_f32(tmp, L.g1, D.d, st));
  K_TRY(convert_bf16_to_f32(tmp + D.d, L.g2, D.d, st));
  CUDA_TRY(cudaStreamSynchronize(st));
  CUDA_TRY(cudaFree(tmp));
  s->loaded[l] = true;
  return MENOS_OK;
}

// =====================================================================================================
// helpers: slot tables
// =====================================================================================================
static int grow_group(menos_server* s, int g, int need_end) {
  int cap = s->cols[g].cap;
  if (need_end <= cap) return MENOS_OK;
  int nc = std::max(64, cap);
  while (nc < need_end) nc *= 2;
  const Dims& D = s->D;
  for (int l = 0; l < s->n_layers; ++l) {
    bf16 *nb = nullptr, *na = nullptr;
    if (cudaMalloc(&nb, (size_t)D.N_g[g] * nc * 2) != cudaSuccess) FAIL(MENOS_ENOMEM, "slot table growth");
    if (cudaMalloc(&na, (size_t)nc * D.ldK_g[g] * 2) != cudaSuccess) FAIL(MENOS_ENOMEM, "slot table growth");
    CUDA_TRY(cudaMemset(nb, 0, (size_t)D.N_g[g] * nc * 2));
    CUDA_TRY(cudaMemset(na, 0, (size_t)nc * D.ldK_g[g] * 2));
    if (cap > 0) {
      CUDA_TRY(cudaMemcpy2D(nb, (size_t)nc * 2, s->Bcat[g][l], (size_t)cap * 2, (size_t)cap * 2, D.N_g[g],
                            cudaMemcpyDeviceToDevice));
      CUDA_TRY(cudaMemcpy(na, s->Acat[g][l], (size_t)cap * D.ldK_g[g] * 2, cudaMemcpyDeviceToDevice));
      CUDA_TRY(cudaFree(s->Bcat[g][l]));
      CUDA_TRY(cudaFree(s->Acat[g][l]));
    }
    s->Bcat[g][l] = nb;
    s->Acat[g][l] = na;
  }
  s->cols[g].grow(nc);
  return MENOS_OK;
}

// AdamW / refresh segments of one client (both A and B of every targeted (layer, target))
static void client_segments(menos_server* s, const Client& c, int hyp_idx, std::vector<AdamSeg>& segs) {
  const Dims& D = s->D;
  if (c.n_prefix) {   // prefix keys and values of every layer: rows P, cols Nkv, bf16 copy in the same layout
    for (int l = c.cut; l < s->n_layers; ++l)
      for (int kv = 0; kv < 2; ++kv) {
        AdamSeg a{};
        a.p_off = ((long long)(l - c.cut) * 2 + kv) * c.n_prefix * D.Nkv; a.rows = c.n_prefix; a.cols = D.Nkv;
        a.client = hyp_idx; a.dst = c.pfx + a.p_off; a.dst_ld = D.Nkv; a.is_b = 0;
        a.row_blk = 1 << 30; a.row_blk_stride = 0; a.row_base = 0;
        segs.push_back(a);
      }
    return;
  }
  for (int l = c.cut; l < s->n_layers; ++l)
    for (int t = 0; t < NT; ++t) {
      if (!(c.mask >> t & 1)) continue;
      const int g = kTargetGroup[t];
      AdamSeg a{};
      a.p_off = c.offA[l * NT + t]; a.rows = c.rank; a.cols = D.K_t[t]; a.client = hyp_idx;
      a.dst = s->Acat[g][l] + (size_t)(c.col_off[g] + c.sub[t]) * D.ldK_g[g];
      a.dst_ld = D.ldK_g[g]; a.is_b = 0; a.row_blk = 1 << 30; a.row_blk_stride = 0; a.row_base = 0;
      segs.push_back(a);
      AdamSeg b{};
      b.p_off = c.offB[l * NT + t]; b.rows = D.N_t[t]; b.cols = c.rank; b.client = hyp_idx;
      b.dst = s->Bcat[g][l] + c.col_off[g] + c.sub[t];
      b.dst_ld = s->cols[g].cap; b.is_b = 1;
      b.row_blk = D.rb_blk[t]; b.row_blk_stride = D.rb_stride[t]; b.row_base = D.rb_base[t];
      segs.push_back(b);
    }
}

// Host->device upload through a ring of pinned staging slots; a slot is reused only after the copy that last
// used it has completed (its event), so uploads never synchronise the stream with the host.
static int upload(menos_server* s, void* dst, const void* src, size_t n, cudaStream_t st) {
  auto& slot = s->ring[s->ring_next];
  s->ring_next = (s->ring_next + 1) % menos_server::kRing;
  if (slot.ev) CUDA_TRY(cudaEventSynchronize(slot.ev));
  else CUDA_TRY(cudaEventCreateWithFlags(&slot.ev, cudaEventDisableTiming));
  if (n > slot.bytes) {
    if (slot.buf) CUDA_TRY(cudaFreeHost(slot.buf));
    slot.buf = nullptr;
    const size_t nb = std::max(n, (size_t)1 << 20);
    CUDA_TRY(cudaMallocHost(&slot.buf, nb));
    slot.bytes = nb;
  }
  memcpy(slot.buf, src, n);
  CUDA_TRY(cudaMemcpyAsync(dst, slot.buf, n, cudaMemcpyHostToDevice, st));
  CUDA_TRY(cudaEventRecord(slot.ev, st));
  return MENOS_OK;
}

// run AdamW (do_update) or plain bf16 refresh over a set of clients; synchronous w.r.t. host staging
static int run_adam(menos_server* s, const std::vector<int>& ids, bool update, cudaStream_t st,
                    const std::vector<AdamSeg>* only = nullptr) {
  std::vector<AdamHyper> hyp;
  std::vector<AdamSeg> segs;
  for (size_t i = 0; i < ids.size(); ++i) {
    Client& c = s->clients[ids[i]];
    AdamHyper h{};
    h.p = c.P(); h.g = c.G(); h.m = c.M(); h.v = c.V();
    h.do_update = update ? 1 : 0;
    if (update) {
      c.step += 1;
      const double lr = c.opt.lr, b1 = c.opt.beta1, b2 = c.opt.beta2;
      h.beta1 = (float)b1; h.beta2 = (float)b2; h.omb1 = (float)(1.0 - b1); h.omb2 = (float)(1.0 - b2);
      h.decay = (float)(1.0 - lr * (double)c.opt.weight_decay);
      h.step_size = (float)(lr / (1.0 - std::pow(b1, (double)c.step)));
      h.bc2_sqrt = (float)std::sqrt(1.0 - std::pow(b2, (double)c.step));
      h.eps = (float)c.opt.eps;
    }
    hyp.push_back(h);
    if (!only) client_segments(s, c, (int)i, segs);
  }
  if (only) segs = *only;
  std::vector<int4> work;
  for (size_t k = 0; k < segs.size(); ++k) {
    const long long n = (long long)segs[k].rows * segs[k].cols;
    for (long long o = 0; o < n; o += 4096) work.push_back(make_int4((int)k, (int)o, (int)std::min<long long>(4096, n - o), 0));
  }
  if (work.empty()) return MENOS_OK;
  const size_t b1 = hyp.size() * sizeof(AdamHyper), b2 = segs.size() * sizeof(AdamSeg), b3 = work.size() * sizeof(int4);
  const size_t o2 = align_up(b1, 256), o3 = o2 + align_up(b2, 256), tot = o3 + b3;
  auto& ds = s->dring[s->dring_next];
  s->dring_next = (s->dring_next + 1) % menos_server::kRing;
  if (ds.ev) CUDA_TRY(cudaEventSynchronize(ds.ev));
  else CUDA_TRY(cudaEventCreateWithFlags(&ds.ev, cudaEventDisableTiming));
  if (tot > ds.bytes) {
    if (ds.buf) CUDA_TRY(cudaFree(ds.buf));
    ds.buf = nullptr;
    const size_t nb = std::max(align_up(tot * 5 / 4, 1 << 16), (size_t)1 << 20);
    if (cudaMalloc(&ds.buf, nb) != cudaSuccess) { cudaGetLastError(); ds.bytes = 0; FAIL(MENOS_ENOMEM, "adamw tables"); }
    ds.bytes = nb;
  }
  uint8_t* dbuf = ds.buf;
  std::vector<uint8_t> blob(tot);
  memcpy(blob.data(), hyp.data(), b1);
  memcpy(blob.data() + o2, segs.data(), b2);
  memcpy(blob.data() + o3, work.data(), b3);
  int rc = upload(s, dbuf, blob.data(), tot, st);
  if (rc) return rc;
  double nparam = 0;
  for (auto& sg : segs) nparam += (double)sg.rows * sg.cols;
  {
    ProfScope ps(PC_ADAMW, 0, nparam * (update ? 30.0 : 6.0), st);
    K_TRY(adamw_run((AdamSeg*)(dbuf + o2), (int4*)(dbuf + o3), (int)work.size(), (AdamHyper*)dbuf, st));
  }
  CUDA_TRY(cudaEventRecord(ds.ev, st));
  return MENOS_OK;
}

// =====================================================================================================
// C-ABI: server lifecycle
// =====================================================================================================
extern "C" int menos_server_create(const menos_model_cfg* cfg, int first_layer, int n_layers,
                                   const menos_layer_weights* w, int device, const menos_server_opts* opts,
                                   menos_server** out) {
  if (!cfg || !out || n_layers <= 0 || first_layer < 0) FAIL(MENOS_EINVAL, "null cfg/out or bad layer range");
  *out = nullptr;
  if (cfg->d_model <= 0 || cfg->n_heads <= 0 || cfg->n_kv_heads <= 0 || cfg->d_ff <= 0 ||
      cfg->d_model % cfg->n_heads || cfg->n_heads % cfg->n_kv_heads)
    FAIL(MENOS_EINVAL, "bad model dims");
  const int hd = cfg->d_model / cfg->n_heads;
  if (hd != 16 && hd != 32 && hd != 64 && hd != 128) FAIL(MENOS_EINVAL, "head_dim %d unsupported (16/32/64/128)", hd);
  if (cfg->d_model % 64) FAIL(MENOS_EINVAL, "d_model must be a multiple of 64");
  if (cfg->arch != MENOS_ARCH_LLAMA && cfg->arch != MENOS_ARCH_OPT) FAIL(MENOS_EINVAL, "unknown arch %d", cfg->arch);
  if (cfg->arch == MENOS_ARCH_OPT && cfg->n_kv_heads != cfg->n_heads) FAIL(MENOS_EINVAL, "OPT has no GQA");
  if (cfg->arch == MENOS_ARCH_OPT && opts && opts->tp.world > 1) FAIL(MENOS_EINVAL, "tensor parallelism is Llama-only");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) FAIL(MENOS_ECUDA, "no CUDA device %d", device);
  cudaDeviceProp prop;
  CUDA_TRY(cudaGetDeviceProperties(&prop, device));
  if (prop.major != 10) FAIL(MENOS_ECUDA, "device %d is sm_%d%d; this library is built for sm_100a", device, prop.major, prop.minor);
  CUDA_TRY(cudaSetDevice(device));

  menos_server_opts o{};
  if (opts) o = *opts;
  menos_tp_cfg tp = o.tp;
  if (tp.world <= 1 && !tp.nccl_id) tp = menos_tp_cfg{0, 1, nullptr, nullptr, nullptr};
  if (tp.world < 1) tp.world = 1;
  if (tp.world > 1 || tp.nccl_id) {
    if (tp.rank < 0 || tp.rank >= tp.world || (!tp.collective && !tp.nccl_id)) FAIL(MENOS_EINVAL, "bad tensor-parallel cfg");
    if (cfg->n_heads % tp.world || cfg->n_kv_heads % tp.world || cfg->d_ff % tp.world)
      FAIL(MENOS_EINVAL, "H=%d, H_kv=%d, f=%d not divisible by tp world %d", cfg->n_heads, cfg->n_kv_heads,
           cfg->d_ff, tp.world);
  }
  std::unique_ptr<menos_server> s(new menos_server());
  s->cfg = *cfg; s->D = make_dims(*cfg, tp.rank, tp.world, tp.world > 1 || tp.nccl_id != nullptr); s->tp = tp;
  if (int rc = s->comm.init(tp, device)) return rc;
  s->tp.nccl_id = nullptr;   // the caller's id buffer is not kept
  s->first_layer = first_layer; s->n_layers = n_layers; s->device = device;
  if (o.max_clients <= 0) o.max_clients = 64;
  if (o.max_rank <= 0) o.max_rank = 64;
  if (o.max_seq_len <= 0) o.max_seq_len = 4096;
  s->num_sms = o.num_sms > 0 ? o.num_sms : prop.multiProcessorCount;
  s->opts = o;
  const Dims& D = s->D;

  // WeightStore: one allocation for all layers (a single preloaded copy)
  const size_t per = align_up((size_t)D.Nqkv * D.d * 2, 256) + align_up((size_t)D.d * D.Nq * 2, 256) +
                     align_up((size_t)D.gu_cols * D.d * 2, 256) + align_up((size_t)D.d * D.fpad * 2, 256) +
                     6 * align_up((size_t)D.d * 4, 256) + align_up((size_t)D.Nqkv * 4, 256) +   // g1 g2 be1 be2 bo bd
                     align_up((size_t)D.fpad * 4, 256);
  s->wbytes = per * n_layers;
  if (cudaMalloc(&s->wbuf, s->wbytes) != cudaSuccess) { cudaGetLastError(); FAIL(MENOS_ENOMEM, "weight store (%zu B)", s->wbytes); }
  CUDA_TRY(cudaMemset(s->wbuf, 0, s->wbytes));
  s->W.resize(n_layers);
  s->loaded.assign(n_layers, false);
  for (int l = 0; l < n_layers; ++l) {
    uint8_t* p = s->wbuf + per * l;
    auto& L = s->W[l];
    L.wqkv = (bf16*)p; p += align_up((size_t)D.Nqkv * D.d * 2, 256);
    L.wo = (bf16*)p; p += align_up((size_t)D.d * D.Nq * 2, 256);
    L.wgu = (bf16*)p; p += align_up((size_t)D.gu_cols * D.d * 2, 256);
    L.wd = (bf16*)p; p += align_up((size_t)D.d * D.fpad * 2, 256);
    L.g1 = (float*)p; p += align_up((size_t)D.d * 4, 256);
    L.g2 = (float*)p; p += align_up((size_t)D.d * 4, 256);
    L.be1 = (float*)p; p += align_up((size_t)D.d * 4, 256);
    L.be2 = (float*)p; p += align_up((size_t)D.d * 4, 256);
    L.bo = (float*)p; p += align_up((size_t)D.d * 4, 256);
    L.bd = (float*)p; p += align_up((size_t)D.d * 4, 256);
    L.bqkv = (float*)p; p += align_up((size_t)D.Nqkv * 4, 256);
    L.bu = (float*)p;
  }
  for (int g = 0; g < NG; ++g) { s->Bcat[g].assign(n_layers, nullptr); s->Acat[g].assign(n_layers, nullptr); }
  CUDA_TRY(cudaMalloc(&s->rope, (size_t)o.max_seq_len * (D.hd / 2) * sizeof(float2)));
  K_TRY(fill_rope_table(s->rope, o.max_seq_len, D.hd, D.theta, 0));
  s->clients.resize(o.max_clients);
  s->batch_refs.assign(o.max_clients, 0);
  if (w) {
    for (int l = 0; l < n_layers; ++l) {
      int rc = upload_layer(s.get(), l, &w[l]);
      if (rc) { menos_server_destroy(s.release()); return rc; }
    }
  }
  // activation arena I (Eq.3)
  size_t fb = 0, tb = 0;
  CUDA_TRY(cudaMemGetInfo(&fb, &tb));
  size_t ab = o.arena_bytes;
  if (ab == 0) ab = fb > ((size_t)8 << 30) ? fb - ((size_t)8 << 30) : fb / 2;
  if (cudaMalloc(&s->arena_mem, ab) != cudaSuccess) { cudaGetLastError(); menos_server_destroy(s.release()); FAIL(MENOS_ENOMEM, "arena (%zu B)", ab); }
  s->arena.init(s->arena_mem, ab);
  CUDA_TRY(cudaDeviceSynchronize());
  *out = s.release();
  return MENOS_OK;
}

extern "C" int menos_server_load_layer(menos_server* s, int layer, const menos_layer_weights* w) {
  if (!s || layer < 0 || layer >= s->n_layers) FAIL(MENOS_EINVAL, "bad server/layer");
  CUDA_TRY(cudaSetDevice(s->device));
  return upload_layer(s, layer, w);
}

extern "C" void menos_server_destroy(menos_server* s) {
  if (!s) return;
  cudaSetDevice(s->device);
  cudaDeviceSynchronize();
  for (auto& c : s->clients) { if (c.buf) cudaFree(c.buf); if (c.pfx) cudaFree(c.pfx); }
  for (int g = 0; g < NG; ++g)
    for (int l = 0; l < s->n_layers; ++l) { if (s->Bcat[g][l]) cudaFree(s->Bcat[g][l]); if (s->Acat[g][l]) cudaFree(s->Acat[g][l]); }
  if (s->wbuf) cudaFree(s->wbuf);
  if (s->rope) cudaFree(s->rope);
  if (s->arena_mem) cudaFree(s->arena_mem);
  s->comm.destroy();
  for (auto& sl : s->ring) {
    if (sl.buf) cudaFreeHost(sl.buf);
    if (sl.ev) cudaEventDestroy(sl.ev);
  }
  for (auto& sl : s->dring) {
    if (sl.buf) cudaFree(sl.buf);
    if (sl.ev) cudaEventDestroy(sl.ev);
  }
  delete s;
}

// =====================================================================================================
// C-ABI: clients
// =====================================================================================================
static uint64_t splitmix(uint64_t& x) {
  uint64_t z = (x += 0x9e3779b97f4a7c15ull);
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebull;
  return z ^ (z >> 31);
}

extern "C" int menos_register_client(menos_server* s, int rank, float alpha, uint32_t target_mask,
                                     const menos_adamw_cfg* opt, uint64_t init_seed, int32_t* client_id) {
  if (!s) FAIL(MENOS_EINVAL, "null server");
  return menos_register_client_at(s, s->first_layer, rank, alpha, target_mask, opt, init_seed, client_id);
}

extern "C" int menos_register_client_at(menos_server* s, int cut_layer, int rank, float alpha, uint32_t target_mask,
                                        const menos_adamw_cfg* opt, uint64_t init_seed, int32_t* client_id) {
  if (!s || !client_id) FAIL(MENOS_EINVAL, "null server/id");
  if (cut_layer < s->first_layer || cut_layer >= s->first_layer + s->n_layers)
    FAIL(MENOS_EINVAL, "cut layer %d outside the server segment [%d, %d)", cut_layer, s->first_layer,
         s->first_layer + s->n_layers);
  if (rank < 1 || rank > s->opts.max_rank) FAIL(MENOS_EINVAL, "rank %d outside [1, %d]", rank, s->opts.max_rank);
  const bool prefix = (target_mask >> TPFX) & 1;
  if (!(alpha > 0.f) || target_mask == 0 || (target_mask >> (TPFX + 1))) FAIL(MENOS_EINVAL, "bad alpha/target mask");
  if (prefix && target_mask != (1u << TPFX)) FAIL(MENOS_EINVAL, "a prefix-tuning client has no LoRA targets");
  if (prefix && s->D.sp) FAIL(MENOS_EINVAL, "prefix tuning is not supported with tensor parallelism");
  if (s->D.arch == MENOS_ARCH_OPT && (target_mask >> TG & 1)) FAIL(MENOS_EINVAL, "OPT has no gate projection");
  CUDA_TRY(cudaSetDevice(s->device));
  int id = -1;
  for (size_t i = 0; i < s->clients.size(); ++i) if (!s->clients[i].used) { id = (int)i; break; }
  if (id < 0) FAIL(MENOS_ENOMEM, "client registry full (%d)", s->opts.max_clients);
  if (s->live_save > 0) {   // the slot tables may not move under a live SAVE batch (its problem lists point into them)
    int cnt0[NG] = {0, 0, 0, 0};
    for (int t = 0; t < NT; ++t) if (target_mask >> t & 1) cnt0[kTargetGroup[t]]++;
    for (int g = 0; g < NG; ++g)
      if (cnt0[g] && !s->cols[g].fits(cnt0[g] * (int)align_up(rank, 16)))
        FAIL(MENOS_ESTATE, "registration would grow the LoRA slot tables while %d SAVE batch(es) are alive; run their "
             "backward (or menos_batch_free) first", s->live_save);
  }
  const Dims& D = s->D;
  Client c;
  c.rank = rank; c.rs = (int)align_up(rank, 16); c.alpha = alpha; c.s = alpha / (float)rank; c.mask = target_mask;
  c.opt = opt ? *opt : menos_adamw_cfg{1e-4, 0.9, 0.999, 1e-8, 0.01};
  c.cut = cut_layer - s->first_layer;
  for (int t = 0; t < NT; ++t) c.sub[t] = -1;
  int cnt[NG] = {0, 0, 0, 0};
  for (int t = 0; t < NT; ++t)
    if (target_mask >> t & 1) { const int g = kTargetGroup[t]; c.sub[t] = cnt[g] * c.rs; cnt[g]++; }
  // slot columns per group
  for (int g = 0; g < NG; ++g) {
    c.width[g] = cnt[g] * c.rs;
    if (!c.width[g]) continue;
    int off = s->cols[g].alloc(c.width[g]);
    if (off < 0) {
      int rc = grow_group(s, g, s->cols[g].cap + c.width[g]);
      if (rc) return rc;
      off = s->cols[g].alloc(c.width[g]);
    }
    if (off < 0) FAIL(MENOS_ENOMEM, "slot allocation");
    c.col_off[g] = off;
  }
  // parameter layout
  c.offA.assign((size_t)s->n_layers * NT, -1);
  c.offB.assign((size_t)s->n_layers * NT, -1);
  // replicated tensors first (A of column-parallel targets, B of row-parallel ones), so that under tensor
  // parallelism their gradient partial sums are one contiguous all-reduce (menos_tp_cfg); with world 1 the
  // split is immaterial
  size_t n = 0;
  if (prefix) {   // [layer >= cut][k | v][P][Nkv]; no LoRA, nothing replicated
    c.n_prefix = rank;
    for (int l = c.cut; l < s->n_layers; ++l) n += (size_t)2 * rank * D.Nkv;
  }
  for (int pass = 0; pass < 2 && !prefix; ++pass) {
    for (int l = c.cut; l < s->n_layers; ++l)   // no adapters below the client's cut
      for (int t = 0; t < NT; ++t) {
        if (!(target_mask >> t & 1)) continue;
        if ((pass == 0) == D.a_rep[t]) { c.offA[l * NT + t] = (long long)n; n += (size_t)rank * D.K_t[t]; }
        else { c.offB[l * NT + t] = (long long)n; n += (size_t)D.N_t[t] * rank; }
      }
    if (pass == 0) c.n_rep = n;
  }
  c.n_params = n;
  if (cudaMalloc(&c.buf, 4 * n * sizeof(float)) != cudaSuccess) { cudaGetLastError(); FAIL(MENOS_ENOMEM, "adapter state"); }
  CUDA_TRY(cudaMemset(c.buf, 0, 4 * n * sizeof(float)));
  // init: A ~ U(-1/sqrt(K), 1/sqrt(K)) (PEFT kaiming-uniform a=sqrt(5)), B = 0
  std::vector<float> host(n, 0.f);
  uint64_t st = init_seed * 0x2545F4914F6CDD1Dull + 1;
  // the draw is over the GLOBAL [r, K] of every (layer, target) in the same order on every tensor-parallel
  // rank; a row-parallel rank keeps its column slice, so the shards assemble the world-1 A exactly
  for (int l = c.cut; l < s->n_layers; ++l)
    for (int t = 0; t < NT; ++t) {
      if (!(target_mask >> t & 1)) continue;
      const int Kg = D.K_glob[t], Kl = D.K_t[t];
      const int c0 = D.a_rep[t] ? 0 : D.tp_rank * Kl;
      const double bound = 1.0 / std::sqrt((double)Kg);
      const long long o = c.offA[l * NT + t];
      for (int i = 0; i < rank; ++i)
        for (int k = 0; k < Kg; ++k) {
          const double u = (double)(splitmix(st) >> 11) * (1.0 / 9007199254740992.0);
          if (k >= c0 && k < c0 + Kl) host[o + (long long)i * Kl + (k - c0)] = (float)((2.0 * u - 1.0) * bound);
        }
    }
  if (prefix) {   // prefix keys / values ~ N(0, 1) (PEFT's embedding init), Box-Muller on the same stream
    for (size_t i = 0; i < n; ++i) {
      const double u1 = ((double)(splitmix(st) >> 11) + 1.0) * (1.0 / 9007199254740993.0);
      const double u2 = (double)(splitmix(st) >> 11) * (1.0 / 9007199254740992.0);
      host[i] = (float)(std::sqrt(-2.0 * std::log(u1)) * std::cos(6.283185307179586 * u2));
    }
    if (cudaMalloc(&c.pfx, n * sizeof(bf16)) != cudaSuccess) { cudaGetLastError(); cudaFree(c.buf); FAIL(MENOS_ENOMEM, "prefix table"); }
  }
  CUDA_TRY(cudaMemcpy(c.buf, host.data(), n * sizeof(float), cudaMemcpyHostToDevice));
  c.used = true;
  s->clients[id] = c;
  int rc = run_adam(s, {id}, false, 0);
  if (rc) return rc;
  CUDA_TRY(cudaDeviceSynchronize());
  *client_id = id;
  return MENOS_OK;
}

extern "C" int menos_unregister_client(menos_server* s, int32_t id) {
  if (!s) FAIL(MENOS_EINVAL, "null server");
  if (id < 0 || id >= (int)s->clients.size() || !s->clients[id].used) FAIL(MENOS_ENOCLIENT, "unknown client %d", id);
  if (s->batch_refs[id] > 0)
    FAIL(MENOS_ESTATE, "client %d is in %d live batch(es); run their backward (or menos_batch_free) first", id,
         s->batch_refs[id]);
  CUDA_TRY(cudaSetDevice(s->device));
  CUDA_TRY(cudaDeviceSynchronize());
  Client& c = s->clients[id];
  const Dims& D = s->D;
  for (int g = 0; g < NG; ++g) {
    if (!c.width[g]) continue;
    for (int l = 0; l < s->n_layers; ++l) {
      CUDA_TRY(cudaMemset2D(s->Bcat[g][l] + c.col_off[g], (size_t)s->cols[g].cap * 2, 0, (size_t)c.width[g] * 2, D.N_g[g]));
      CUDA_TRY(cudaMemset(s->Acat[g][l] + (size_t)c.col_off[g] * D.ldK_g[g], 0, (size_t)c.width[g] * D.ldK_g[g] * 2));
    }
    s->cols[g].release(c.col_off[g], c.width[g]);
  }
  CUDA_TRY(cudaFree(c.buf));
  if (c.pfx) CUDA_TRY(cudaFree(c.pfx));
  s->clients[id] = Client();
  CUDA_TRY(cudaDeviceSynchronize());
  return MENOS_OK;
}

// saved bytes per token per layer in SAVE mode (excluding the LoRA U share)
static size_t saved_bytes_per_token_layer(const Dims& D, bool save_a) {
  size_t b = 0;
  b += (size_t)D.d * 4 * 2;        // x, h (fp32 residual stream)
  b += (size_t)D.d * 2 * 2;        // xn, hn
  b += (size_t)D.Nqkv * 2;         // qkv
  b += (size_t)D.Nq * 2;           // O
  b += (size_t)D.gu_cols * 2;      // gu (OPT: relu(fc1))
  if (save_a) b += (size_t)D.fpad * 2;
  b += 4 * 2 + (size_t)D.H * 4;    // rstd1, rstd2, lse
  return b;
}
static size_t scratch_bytes_per_token(const Dims& D, int R_sum) {
  size_t b = 0;
  b += (size_t)D.d * 4 * 4;          // dyf, dxf, dhf, xout (fp32)
  b += (size_t)D.d * 2 * 5;          // dyb, dxb, dhb, dhn, io staging (bf16)
  b += (size_t)D.Nq * 2;             // dO
  b += (size_t)D.Nqkv * 2;           // dqkv
  b += (size_t)D.gu_cols * 2;        // dgu
  b += (size_t)D.fpad * 2;           // a (when not saved)
  b += (size_t)D.H * 4;              // D rowsums
  b += (size_t)R_sum * 2;            // dU
  b += 64;                           // alignment slack
  return b;
}

extern "C" int menos_client_memory(menos_server* s, int32_t id, int n_tokens, size_t* persistent, size_t* fwd_bytes,
                                   size_t* bwd_bytes) {
  if (!s) FAIL(MENOS_EINVAL, "null server");
  if (id < 0 || id >= (int)s->clients.size() || !s->clients[id].used) FAIL(MENOS_ENOCLIENT, "unknown client %d", id);
  if (n_tokens < 0) FAIL(MENOS_EINVAL, "n_tokens < 0");
  const Client& c = s->clients[id];
  const Dims& D = s->D;
  // A + O: fp32 p, g, m, v + the bf16 slot-table copy (Acat rows + Bcat columns incl. rank padding)
  size_t slots = 0;
  for (int g = 0; g < NG; ++g) slots += (size_t)c.width[g] * (D.N_g[g] + D.ldK_g[g]) * 2 * s->n_layers;
  if (c.pfx) slots += 2 * c.n_params;   // prefix tuning: the bf16 copy of the prefix table
  if (persistent) *persistent = 16 * c.n_params + slots;
  const bool save_a = ((c.mask >> TD) & 1) && D.arch != MENOS_ARCH_OPT;
  size_t ush = 0;
  for (int g = 0; g < NG; ++g) ush += (size_t)c.width[g] * 2;
  const size_t T = (size_t)n_tokens;
  if (fwd_bytes) *fwd_bytes = T * ((saved_bytes_per_token_layer(D, save_a) + ush) * s->n_layers);
  int rsum = 0;
  for (int g = 0; g < NG; ++g) rsum += c.width[g];
  if (bwd_bytes) *bwd_bytes = T * scratch_bytes_per_token(D, rsum);
  return MENOS_OK;
}

static size_t slab_bytes_of(const Dims& D, int Ls, int T, const int R_used[NG], bool save_a, bool save, int Text);
static size_t scratch_bytes_of(const Dims& D, int T, const int R_used[NG], bool nograd_set, int Text, long long ds_tiles);
static long long ds_tiles_bound(const menos_server* s, long long T);
static size_t meta_bytes_bound(int T, int Ls, int n_clients);

// The dS-stored attention backward (testing mode bit 6 with bit 3, the default) runs for head_dim 128 / 64 batches
// without prefix-tuning clients
static bool ds_path_on(const menos_server* s) {
  return (g_attn_tc & 72) == 72 && !(g_attn_tc & 32) && (s->D.hd == 128 || s->D.hd == 64);
}
// H * sum over sequences of attn_ds_tiles(L) <= H * T * (1 + max_seq_len / 16384) for any split of T tokens into
// sequences of at most max_seq_len (attn_ds_tiles(L) <= L + L^2 / 16384), capped by the chunk budget
static long long ds_tiles_bound(const menos_server* s, long long T) {
  if (!ds_path_on(s) || T <= 0) return 0;
  const double per = 1.0 + s->opts.max_seq_len / 16384.0;
  return std::min(g_attn_ds_cap_tiles, (long long)std::ceil((double)s->D.H * (double)T * per));
}

extern "C" int menos_batch_memory(menos_server* s, int n_clients, const int32_t* ids, const int32_t* n_tokens,
                                  int flags, size_t* fwd_bytes, size_t* bwd_bytes) {
  if (!s || n_clients < 0 || (n_clients > 0 && (!ids || !n_tokens))) FAIL(MENOS_EINVAL, "bad arguments");
  const Dims& D = s->D;
  if (flags & ~(MENOS_FWD_NOGRAD | MENOS_MEM_BOUND)) FAIL(MENOS_EINVAL, "bad flags %d", flags);
  int R[NG] = {0, 0, 0, 0};
  bool save_a = false;
  long long T = 0, Text = 0;   // prefix clients: bound on the extension, assuming one-token sequences
  if (flags & MENOS_MEM_BOUND) {   // additive bound: the registry-wide slot span and saved-tensor set
    for (const Client& c : s->clients) {
      if (!c.used) continue;
      for (int g = 0; g < NG; ++g) if (c.width[g]) R[g] = std::max(R[g], c.col_off[g] + c.width[g]);
      if ((c.mask >> TD & 1) && D.arch != MENOS_ARCH_OPT) save_a = true;
    }
  }
  for (int i = 0; i < n_clients; ++i) {
    const int id = ids[i];
    if (id < 0 || id >= (int)s->clients.size() || !s->clients[id].used) FAIL(MENOS_ENOCLIENT, "unknown client %d", id);
    if (n_tokens[i] < 0) FAIL(MENOS_EINVAL, "n_tokens < 0");
    const Client& c = s->clients[id];
    for (int g = 0; g < NG; ++g) if (c.width[g]) R[g] = std::max(R[g], c.col_off[g] + c.width[g]);
    if ((c.mask >> TD & 1) && D.arch != MENOS_ARCH_OPT) save_a = true;
    T += n_tokens[i];
    Text += (long long)n_tokens[i] * (1 + c.n_prefix);
  }
  if (T > (1ll << 30)) FAIL(MENOS_EINVAL, "too many tokens");
  for (int g = 0; g < NG; ++g) R[g] = (int)align_up(R[g], 64);
  const bool nograd = flags & MENOS_FWD_NOGRAD;
  const size_t meta = meta_bytes_bound((int)(T + Text), s->n_layers, n_clients);
  // forward: scratch (+ the NOGRAD layer set) + slab (+ meta); backward of a NOGRAD batch re-forwards with SAVE
  if (Text > (1ll << 30)) FAIL(MENOS_EINVAL, "too many tokens");
  const int Tx = (int)Text;
  // dS-stored attention backward (no prefix clients): a bound on the chunk buffer without the sequence lengths
  bool pfx = false;
  for (int i = 0; i < n_clients; ++i) pfx = pfx || s->clients[ids[i]].n_prefix > 0;
  const long long dst = pfx ? 0 : ds_tiles_bound(s, T);
  const size_t fwd = scratch_bytes_of(D, (int)T, R, nograd, Tx, dst) + slab_bytes_of(D, s->n_layers, (int)T, R, save_a, !nograd, Tx) + meta;
  const size_t bwd = scratch_bytes_of(D, (int)T, R, nograd, Tx, dst) + slab_bytes_of(D, s->n_layers, (int)T, R, save_a, true, Tx) +
                     (nograd ? slab_bytes_of(D, s->n_layers, (int)T, R, save_a, false, Tx) : 0) + 2 * meta;
  if (fwd_bytes) *fwd_bytes = fwd;
  if (bwd_bytes) *bwd_bytes = bwd;
  return MENOS_OK;
}

extern "C" int menos_adapter_shape(menos_server* s, int32_t id, int target, int* rows, int* cols) {
  if (!s || !rows || !cols) FAIL(MENOS_EINVAL, "null argument");
  if (id < 0 || id >= (int)s->clients.size() || !s->clients[id].used) FAIL(MENOS_ENOCLIENT, "unknown client %d", id);
  if (target < 0 || target > TPFX) FAIL(MENOS_EINVAL, "bad target");
  const Client& c = s->clients[id];
  if (!(c.mask >> target & 1)) FAIL(MENOS_EINVAL, "target %d not in client mask", target);
  if (target == TPFX) {   // prefix keys (A) and values (B): [P, Nkv] each
    rows[0] = rows[1] = c.n_prefix; cols[0] = cols[1] = s->D.Nkv;
    return MENOS_OK;
  }
  rows[0] = c.rank; cols[0] = s->D.K_t[target];   // A [r, K]
  rows[1] = s->D.N_t[target]; cols[1] = c.rank;   // B [N, r]
  return MENOS_OK;
}

static int adapter_ptr(menos_server* s, int32_t id, int layer, int target, int which, float** p, size_t* n,
                       Client** cp) {
  if (!s) FAIL(MENOS_EINVAL, "null server");
  if (id < 0 || id >= (int)s->clients.size() || !s->clients[id].used) FAIL(MENOS_ENOCLIENT, "unknown client %d", id);
  if (layer < 0 || layer >= s->n_layers || target < 0 || target > TPFX || which < 0 || which > 7)
    FAIL(MENOS_EINVAL, "bad layer/target/which");
  Client& c = s->clients[id];
  if (!(c.mask >> target & 1)) FAIL(MENOS_EINVAL, "target %d not in client mask", target);
  if (layer < c.cut) FAIL(MENOS_EINVAL, "layer %d is below client %d's cut (no adapter there)", layer, id);
  const bool isB = which & 1;
  if (target == TPFX) {   // A = prefix keys, B = prefix values, [P, Nkv] each
    const long long off = ((long long)(layer - c.cut) * 2 + (isB ? 1 : 0)) * c.n_prefix * s->D.Nkv;
    *n = (size_t)c.n_prefix * s->D.Nkv;
    float* base = which < 2 ? c.P() : which < 4 ? c.G() : which < 6 ? c.M() : c.V();
    *p = base + off;
    *cp = &c;
    return MENOS_OK;
  }
  const long long off = isB ? c.offB[layer * NT + target] : c.offA[layer * NT + target];
  *n = (size_t)c.rank * (isB ? s->D.N_t[target] : s->D.K_t[target]);
  float* base = which < 2 ? c.P() : which < 4 ? c.G() : which < 6 ? c.M() : c.V();
  *p = base + off;
  *cp = &c;
  return MENOS_OK;
}

extern "C" int menos_get_adapter(menos_server* s, int32_t id, int layer, int target, int which, float* host_out) {
  float* p; size_t n; Client* c;
  int rc = adapter_ptr(s, id, layer, target, which, &p, &n, &c);
  if (rc) return rc;
  if (!host_out) FAIL(MENOS_EINVAL, "null output");
  CUDA_TRY(cudaSetDevice(s->device));
  CUDA_TRY(cudaDeviceSynchronize());
  CUDA_TRY(cudaMemcpy(host_out, p, n * sizeof(float), cudaMemcpyDeviceToHost));
  return MENOS_OK;
}

extern "C" int menos_set_adapter(menos_server* s, int32_t id, int layer, int target, int which, const float* host_in) {
  if (which > 1) FAIL(MENOS_EINVAL, "set_adapter: which must be 0 (A) or 1 (B)");
  float* p; size_t n; Client* c;
  int rc = adapter_ptr(s, id, layer, target, which, &p, &n, &c);
  if (rc) return rc;
  if (!host_in) FAIL(MENOS_EINVAL, "null input");
  CUDA_TRY(cudaSetDevice(s->device));
  CUDA_TRY(cudaDeviceSynchronize());
  CUDA_TRY(cudaMemcpy(p, host_in, n * sizeof(float), cudaMemcpyHostToDevice));
  std::vector<AdamSeg> all, one;
  client_segments(s, *c, 0, all);
  for (auto& sg : all) {
    const long long want = target == TPFX ? (long long)(p - c->P())
                                          : which ? c->offB[layer * NT + target] : c->offA[layer * NT + target];
    if (sg.p_off == want) one.push_back(sg);
  }
  rc = run_adam(s, {id}, false, 0, &one);
  if (rc) return rc;
  CUDA_TRY(cudaDeviceSynchronize());
  return MENOS_OK;
}

extern "C" int menos_adapter_step(menos_server* s, int n, const int32_t* ids, void* stream) {
  if (!s || n < 0 || (n > 0 && !ids)) FAIL(MENOS_EINVAL, "bad arguments");
  std::vector<int> v;
  for (int i = 0; i < n; ++i) {
    if (ids[i] < 0 || ids[i] >= (int)s->clients.size() || !s->clients[ids[i]].used) FAIL(MENOS_ENOCLIENT, "unknown client %d", ids[i]);
    for (int x : v) if (x == ids[i]) FAIL(MENOS_EINVAL, "client %d listed twice", ids[i]);
    v.push_back(ids[i]);
  }
  CUDA_TRY(cudaSetDevice(s->device));
  if (int rc0 = bind_stream(s, (cudaStream_t)stream)) return rc0;
  return run_adam(s, v, true, (cudaStream_t)stream);
}

extern "C" int menos_get_stats(menos_server* s, menos_stats* o) {
  if (!s || !o) FAIL(MENOS_EINVAL, "null argument");
  memset(o, 0, sizeof *o);
  o->base_bytes = s->wbytes;
  size_t ad = 0;
  for (auto& c : s->clients) if (c.used) { ad += 16 * c.n_params; o->n_clients++; }
  for (int g = 0; g < NG; ++g) ad += (size_t)s->cols[g].cap * (s->D.N_g[g] + s->D.ldK_g[g]) * 2 * s->n_layers;
  o->adapters_bytes = ad;
  o->arena_bytes = s->arena.cap; o->arena_used = s->arena.used; o->arena_peak = s->arena.peak;
  o->num_sms = s->num_sms;
  return MENOS_OK;
}

extern "C" unsigned long long menos_launch_count(void) { return g_launch_count; }

extern "C" int menos_profile_enable(int on) {
  g_prof_on = on != 0;
  g_prof.clear();
  g_ev_used = 0;
  return MENOS_OK;
}

extern "C" int menos_profile_read(menos_kernel_stat* out, int max_n, int* n_out) {
  if (!out || !n_out || max_n < PC_N) FAIL(MENOS_EINVAL, "need room for %d classes", (int)PC_N);
  CUDA_TRY(cudaDeviceSynchronize());
  for (int c = 0; c < PC_N; ++c) {
    memset(&out[c], 0, sizeof out[c]);
    snprintf(out[c].name, sizeof out[c].name, "%s", kProfName[c]);
  }
  for (auto& r : g_prof) {
    float ms = 0.f;
    CUDA_TRY(cudaEventElapsedTime(&ms, r.a, r.b));
    out[r.cls].launches += 1; out[r.cls].ms += ms; out[r.cls].flops += r.flops; out[r.cls].bytes += r.bytes;
  }
  *n_out = PC_N;
  g_prof.clear();
  g_ev_used = 0;
  return MENOS_OK;
}

extern "C" int menos_sync(menos_server* s) {
  if (!s) FAIL(MENOS_EINVAL, "null server");
  CUDA_TRY(cudaSetDevice(s->device));
  CUDA_TRY(cudaDeviceSynchronize());
  CUDA_TRY(cudaGetLastError());
  return MENOS_OK;
}

extern "C" const char* menos_last_error(void) { return tl_err.c_str(); }

extern "C" int menos_tp_stats(menos_server* s, long long* calls, double* bytes) {
  if (!s || !calls || !bytes) FAIL(MENOS_EINVAL, "null argument");
  *calls = s->comm.calls; *bytes = s->comm.bytes;
  return MENOS_OK;
}

// =====================================================================================================
// batch construction (BatchPacker)
// =====================================================================================================
struct Scratch {
  float *dyf, *dxf, *dhf, *xout;     // fp32 residual streams (gradient ping-pong, dh, forward output); local rows
  bf16 *dyb, *dxb, *dhb;             // bf16 copies (A operands of the dX GEMMs, LoRA dY); local rows
  bf16 *dhn, *dO, *dqkv, *dgu, *a, *io;  // io: bf16 staging of x_c / x_s / g_c / g_s ([Tpad, d])
  bf16 *gath, *rsout;                // sequence parallel: all-gathered dy / dh [Tpad, d]; reduce-scatter output [Tloc, d]
  bf16 *qkv_x, *O_x, *dO_x, *dqkv_x; // prefix-tuning extension [Text, .] (nullptr without prefix clients)
  float *D_x, *dqacc_x;
  float* Dsum;
  float* wsp;                        // fused dU + dB: per-slab fp32 dU partials (one group at a time)
  bf16* ds;                          // dS-stored attention backward: bf16 dS^T tiles of one chunk (or nullptr)
  bf16* dU[NG];
};

static int build_batch(menos_server* s, int n_seqs, const int32_t* seq_client, const int32_t* seq_len, bool nograd,
                       std::unique_ptr<menos_batch>& out) {
  const Dims& D = s->D;
  std::unique_ptr<menos_batch> b(new menos_batch());
  b->n_seqs = n_seqs; b->nograd = nograd;
  b->cu.push_back(0);
  for (int i = 0; i < n_seqs; ++i) {
    const int c = seq_client[i], L = seq_len[i];
    if (c < 0 || c >= (int)s->clients.size() || !s->clients[c].used) FAIL(MENOS_ENOCLIENT, "sequence %d: unknown client %d", i, c);
    if (L < 1 || L > s->opts.max_seq_len) FAIL(MENOS_EINVAL, "sequence %d: length %d outside [1, %d]", i, L, s->opts.max_seq_len);
    if (i > 0 && c != seq_client[i - 1]) {
      for (int x : b->bclients) if (x == c) FAIL(MENOS_EINVAL, "client %d's sequences are not contiguous", c);
    }
    if (b->bclients.empty() || b->bclients.back() != c) { b->bclients.push_back(c); b->btok_off.push_back(b->cu.back()); b->btok_n.push_back(0); }
    b->btok_n.back() += L;
    b->seq_client.push_back(c); b->seq_len.push_back(L);
    b->cu.push_back(b->cu.back() + L);
    for (int p = 0; p < L; ++p) b->pos.push_back(p);
    b->pairs += 0.5 * (double)L * (L + 1);
  }
  b->T = b->cu.back();
  const int T = b->T;
  // prefix tuning: the extension's sequence lengths
  b->ext_len.resize(n_seqs);
  b->Text = 0;
  for (int i = 0; i < n_seqs; ++i) {
    const Client& c = s->clients[b->seq_client[i]];
    if (c.n_prefix) b->has_pfx = true;
    b->ext_len[i] = c.n_prefix + b->seq_len[i];
    b->Text += b->ext_len[i];
    b->pairs_ext += 0.5 * (double)b->ext_len[i] * (b->ext_len[i] + 1);
  }
  b->ds_tiles = (ds_path_on(s) && !b->has_pfx)
                    ? std::min(g_attn_ds_cap_tiles, attn_ds_total_tiles(b->seq_len.data(), n_seqs, D.H)) : 0;
  if (b->has_pfx) {
    if (D.sp) FAIL(MENOS_EINVAL, "prefix tuning is not supported with tensor parallelism");
    for (int c : b->bclients)
      if (s->clients[c].cut != 0) FAIL(MENOS_EINVAL, "a batch with prefix-tuning clients cannot mix cut points");
    for (int i = 0; i < n_seqs; ++i)
      if (b->ext_len[i] > s->opts.max_seq_len)
        FAIL(MENOS_EINVAL, "sequence %d: prefix + length %d exceeds max_seq_len %d", i, b->ext_len[i], s->opts.max_seq_len);
  }
  // per-client cuts: clients must come in non-decreasing cut order; layer l sees the prefix of clients with cut <= l
  b->Tl.assign(s->n_layers, 0);
  b->nseq_l.assign(s->n_layers, 0);
  for (size_t k = 0; k < b->bclients.size(); ++k) {
    const int cut = s->clients[b->bclients[k]].cut;
    if (k > 0 && cut < s->clients[b->bclients[k - 1]].cut)
      FAIL(MENOS_EINVAL, "clients must be ordered by non-decreasing cut layer (client %d)", b->bclients[k]);
  }
  if (D.sp)
    for (int c : b->bclients)
      if (s->clients[c].cut != 0) FAIL(MENOS_EINVAL, "per-client cut points are not supported with tensor parallelism");
  for (int i = 0; i < n_seqs; ++i) {
    const int cut = s->clients[b->seq_client[i]].cut;
    for (int l = cut; l < s->n_layers; ++l) { b->Tl[l] = b->cu[i + 1]; b->nseq_l[l] = i + 1; }
  }
  // LoRA groups active in this batch and their used slot width
  for (int c : b->bclients) {
    const Client& cl = s->clients[c];
    for (int g = 0; g < NG; ++g)
      if (cl.width[g]) { b->g_active[g] = true; b->R_used[g] = std::max(b->R_used[g], cl.col_off[g] + cl.width[g]); }
    if ((cl.mask >> TD & 1) && D.arch != MENOS_ARCH_OPT) b->save_a = true;
  }
  for (int g = 0; g < NG; ++g) b->R_used[g] = (int)align_up(b->R_used[g], 64);
  b->n_mt = ceil_div(T, 128);
  (void)D;
  // small-GEMM problem lists are filled later (need layer buffers); reserve host vectors here
  b->sg_fwd.resize((size_t)s->n_layers * NG);
  b->sg_shk.assign((size_t)s->n_layers * NG, menos_batch::ShkList());
  b->dub_bufs.assign((size_t)s->n_layers * NG, menos_batch::DubBufs());
  b->da_tc.assign((size_t)s->n_layers * NG, menos_batch::DaTc());
  b->sg_dub.resize((size_t)s->n_layers * NG);
  b->sg_da.resize((size_t)s->n_layers * NG);

  out = std::move(b);
  return MENOS_OK;
}

// Allocate the slab (saved activations or x_c copy) and upload all metadata incl. small-GEMM problem lists.
// arena bytes of a batch's slab: the SAVE activations of every layer (I in Eq.3), or under NOGRAD
// only the x_c copy; R_used = the batch's block-diagonal LoRA slot widths per group (0 = inactive)
// Text: rows of the prefix-tuning extension (== T without prefix clients); lse is kept for the extension
static size_t slab_bytes_of(const Dims& D, int Ls, int T, const int R_used[NG], bool save_a, bool save, int Text) {
  const Rows R = rows_of(D, T);   // sequence parallel: x, h, rstd local; xn, hn all-gathered
  if (!save) return align_up((size_t)R.Tloc * D.d * 4, 256);
  size_t per_layer = 0;
  auto A = [&](size_t n) { per_layer += align_up(n, 256); };
  A((size_t)R.Tloc * D.d * 4); A((size_t)R.Tpad * D.d * 2); A((size_t)R.Tloc * 4);   // x (fp32), xn, rstd1
  A((size_t)T * D.Nqkv * 2); A((size_t)T * D.Nq * 2); A((size_t)D.H * std::max(T, Text) * 4 + kLsePad);   // qkv, O, lse
  A((size_t)R.Tloc * D.d * 4); A((size_t)R.Tpad * D.d * 2); A((size_t)R.Tloc * 4);   // h (fp32), hn, rstd2
  A((size_t)T * D.gu_cols * 2);                                             // gu
  if (save_a) A((size_t)T * D.fpad * 2);
  for (int g = 0; g < NG; ++g) if (R_used[g]) A((size_t)T * R_used[g] * 2);
  return per_layer * Ls;
}
// arena bytes of the per-call scratch block (see get_scratch)
// slab width of a fused dU + dB problem (see finalize_batch); MENOS_LORA_DUB_MT=128 forces 128 (A/B), and
// MENOS_LORA_DUB_MMA=1 puts every problem on the mma.sync kernel (128)
static bool dub_env_mma() {
  static const bool v = [] { const char* e = getenv("MENOS_LORA_DUB_MMA"); return e && atoi(e) == 1; }();
  return v;
}
static int dub_mts(const LoraDUBProblem& q) {
  static const int force = [] { const char* e = getenv("MENOS_LORA_DUB_MT"); return e ? atoi(e) : 0; }();
  if (dub_env_mma() || q.rank > 16 || force == 128) return 128;
  return q.Nt >= 8192 ? 256 : 128;
}

// fused dU + dB partials of one group's problems: sum over clients and targets of ceil(N_t/128) * T_c * rank * 4 B,
// bounded per token by (max over the group's targets of ceil(N_t/128)) * (slot span R_used[g]) * 4 B
static size_t wsp_bytes_of(const Dims& D, int T, const int R_used[NG]) {
  size_t w = 0;
  for (int g = 0; g < NG; ++g) {
    if (!R_used[g]) continue;
    int ms = 0;
    for (int t = 0; t < NT; ++t)
      if (kTargetGroup[t] == g) ms = std::max(ms, (D.N_t[t] + LORA_DUB_MT - 1) / LORA_DUB_MT);
    w = std::max(w, (size_t)ms * R_used[g] * 4);
  }
  return w * (size_t)T;
}

static size_t scratch_bytes_of(const Dims& D, int T, const int R_used[NG], bool nograd_set, int Text, long long ds_tiles) {
  size_t need = 0;
  auto A = [&](size_t n) { need += align_up(n, 256); };
  const Rows Rw = rows_of(D, T);
  const size_t df = (size_t)Rw.Tloc * D.d * 4, db = (size_t)Rw.Tloc * D.d * 2, dp = (size_t)Rw.Tpad * D.d * 2;
  A(df); A(df); A(df); A(df);                                                 // dyf, dxf, dhf, xout (local rows)
  A(db); A(db); A(db); A(dp); A(dp);                                          // dyb, dxb, dhb (local), dhn, io
  if (D.sp) { A(dp); A(db); }                                                 // gathered dy / dh, reduce-scatter out
  if (Text > T) {   // prefix-tuning extension: qkv, O, dO, dqkv, D (fp32), the one-pass backward's dQ sums (fp32)
    A((size_t)Text * D.Nqkv * 2); A((size_t)Text * D.Nq * 2); A((size_t)Text * D.Nq * 2);
    A((size_t)Text * D.Nqkv * 2); A((size_t)D.H * Text * 4 + kLsePad); A((size_t)Text * D.Nq * 4);
  }
  A((size_t)T * D.Nq * 2); A((size_t)T * D.Nqkv * 2); A((size_t)T * D.gu_cols * 2); A((size_t)T * D.fpad * 2);
  A((size_t)D.H * T * 4 + kLsePad);                                           // Dsum
  A(wsp_bytes_of(D, T, R_used));                                              // dU partials
  for (int g = 0; g < NG; ++g) A((size_t)T * R_used[g] * 2);
  // NOGRAD forward layer set (x ping-pong = xout/dxf; intermediates reuse the grad buffers where free)
  if (nograd_set) {
    A(dp); A(df); A((size_t)T * D.Nqkv * 2); A((size_t)T * D.Nq * 2);
    A((size_t)T * D.gu_cols * 2); A((size_t)D.H * std::max(T, Text) * 4 + kLsePad); A((size_t)Rw.Tloc * 8); A(dp);
    for (int g = 0; g < NG; ++g) A((size_t)T * R_used[g] * 2);
  }
  A((size_t)ds_tiles * kDsTileBytes);   // dS-stored attention backward: the chunk buffer, last
  return need;
}
// generous bound of a batch's metadata block (segment tables, positions, tile maps, LoRA problem lists)
static size_t meta_bytes_bound(int T, int Ls, int n_clients) {
  return (size_t)64 * T + (size_t)Ls * (64 << 10) + (size_t)n_clients * Ls * 4096 + (1 << 20);
}

static int finalize_batch(menos_server* s, menos_batch* b, Scratch& sc, const LayerSave* ng, cudaStream_t st) {
  const Dims& D = s->D;
  const int T = b->T, Ls = s->n_layers;
  // ---- sizes
  const bool save = !b->nograd;
  int R_act[NG];
  for (int g = 0; g < NG; ++g) R_act[g] = b->g_active[g] ? b->R_used[g] : 0;
  const size_t slab_bytes = slab_bytes_of(D, Ls, T, R_act, b->save_a, save, b->Text);
  // ---- metadata blob
  std::vector<uint8_t> blob;
  auto put = [&](const void* p, size_t n) {
    size_t o = align_up(blob.size(), 256); blob.resize(o + n); if (n) memcpy(blob.data() + o, p, n); return o; };
  std::vector<int2> blocks;
  for (int i = 0; i < b->n_seqs; ++i)
    for (int q = 0; q < b->seq_len[i]; q += 64) blocks.push_back(make_int2(i, q));
  b->n_blocks = (int)blocks.size();
  std::vector<int2> blocks128;   // 128-row q blocks of the tcgen05 attention forward
  for (int i = 0; i < b->n_seqs; ++i)
    for (int q = 0; q < b->seq_len[i]; q += 128) blocks128.push_back(make_int2(i, q));
  b->n_blocks128 = (int)blocks128.size();
  // one attention view (work lists over the first n sequences) per distinct active prefix
  b->views.clear();
  b->view_of.assign(Ls, -1);
  std::vector<std::vector<int4>> v_items, v_items_kv, v_items_q, v_items_seq;
  std::vector<AttnDsPlan> v_ds;
  for (int l = 0; l < Ls; ++l) {
    const int ns = b->nseq_l[l];
    if (ns == 0) continue;
    if (!b->views.empty() && b->views.back().n_seqs == ns) { b->view_of[l] = (int)b->views.size() - 1; continue; }
    menos_batch::AttnView v;
    v.n_seqs = ns;
    for (int i = 0; i < ns; ++i) {
      v.n_blocks += ceil_div(b->seq_len[i], 64);
      v.n_blocks128 += ceil_div(b->seq_len[i], 128);
      v.pairs += 0.5 * (double)b->seq_len[i] * (b->seq_len[i] + 1);
    }
    v_items.emplace_back(); v_items_kv.emplace_back(); v_items_q.emplace_back();
    attn_ws_items(b->seq_len.data(), ns, D.H, v_items.back(), g_attn_order ? 1 : 0, s->num_sms);
    attn_ws_items(b->seq_len.data(), ns, D.Hkv, v_items_kv.back(), g_attn_order ? 2 : 0, s->num_sms);
    v_items_seq.emplace_back();
    attn_seq_items(b->seq_len.data(), ns, D.Hkv, v_items_seq.back());
    attn_ws_items(b->seq_len.data(), ns, D.H, v_items_q.back(), g_attn_order ? 1 : 0, s->num_sms);
    v.n_items = (int)v_items.back().size();
    v.n_items_kv = (int)v_items_kv.back().size();
    v.n_items_seq = (int)v_items_seq.back().size();
    v_ds.emplace_back();
    if (b->ds_tiles > 0) {
      v.ds_ok = attn_ds_plan(b->seq_len.data(), ns, D.H, D.Hkv, b->ds_tiles, v_ds.back(), s->num_sms);
      if (v.ds_ok) v.ds_chunks = v_ds.back().chunks;
    }
    b->views.push_back(v);
    b->view_of[l] = (int)b->views.size() - 1;
  }
  std::vector<int2> mt((size_t)NG * b->n_mt, make_int2(0, 0));
  for (int g = 0; g < NG; ++g) {
    if (!b->g_active[g]) continue;
    for (int m = 0; m < b->n_mt; ++m) {
      const int r0 = m * 128, r1 = std::min(T, r0 + 128);
      int lo = 1 << 30, hi = -1;
      for (size_t k = 0; k < b->bclients.size(); ++k) {
        const int a0 = b->btok_off[k], a1 = a0 + b->btok_n[k];
        if (a1 <= r0 || a0 >= r1) continue;
        const Client& cl = s->clients[b->bclients[k]];
        if (!cl.width[g]) continue;
        lo = std::min(lo, cl.col_off[g]); hi = std::max(hi, cl.col_off[g] + cl.width[g]);
      }
      if (hi > lo) mt[(size_t)g * b->n_mt + m] = make_int2(lo, (hi - lo) / 16);
    }
  }
  const int n_nt = ceil_div(D.Nqkv, 256);
  std::vector<uint8_t> ntq(n_nt, 0);
  for (int c : b->bclients) {
    const Client& cl = s->clients[c];
    const int lo[3] = {0, D.Nq, D.Nq + D.Nkv}, hi[3] = {D.Nq, D.Nq + D.Nkv, D.Nqkv};
    for (int t = 0; t < 3; ++t)
      if (cl.mask >> t & 1)
        for (int n = lo[t] / 256; n <= (hi[t] - 1) / 256; ++n) ntq[n] = 1;
  }
  const size_t o_cu = put(b->cu.data(), b->cu.size() * 4);
  const size_t o_pos = put(b->pos.data(), b->pos.size() * 4);
  const size_t o_blk = put(blocks.data(), blocks.size() * sizeof(int2));
  const size_t o_blk128 = put(blocks128.data(), blocks128.size() * sizeof(int2));
  for (size_t v = 0; v < b->views.size(); ++v) {
    b->views[v].o_items = put(v_items[v].data(), v_items[v].size() * sizeof(int4));
    b->views[v].o_items_kv = put(v_items_kv[v].data(), v_items_kv[v].size() * sizeof(int4));
    b->views[v].o_items_q = put(v_items_q[v].data(), v_items_q[v].size() * sizeof(int4));
    b->views[v].o_items_seq = put(v_items_seq[v].data(), v_items_seq[v].size() * sizeof(int4));
    if (b->views[v].ds_ok) {
      b->views[v].o_ds_kv = put(v_ds[v].items_kv.data(), v_ds[v].items_kv.size() * sizeof(int4));
      b->views[v].o_ds_q = put(v_ds[v].items_q.data(), v_ds[v].items_q.size() * sizeof(int4));
      b->views[v].o_ds_base = put(v_ds[v].base.data(), v_ds[v].base.size() * sizeof(int));
    }
  }
  // prefix tuning: the extended batch's segment tables, row maps and attention work lists (one view)
  size_t o_xcu = 0, o_xblk = 0, o_xblk128 = 0, o_xsrc = 0, o_xtok = 0, o_tokx = 0, o_seqx = 0, o_pc = 0, o_seqsh = 0;
  size_t o_xit = 0, o_xitkv = 0, o_xitq = 0, o_xitseq = 0;
  if (b->has_pfx) {
    const std::vector<int>& xl = b->ext_len;
    std::vector<int> xcu(1, 0), xtok, tokx(T), seqx(b->n_seqs), seqsh(b->n_seqs);
    std::vector<int2> xsrc, xb64, xb128;
    std::vector<PrefixClient> pcs;
    std::vector<int> slot_of(s->clients.size(), -1);
    for (size_t k = 0; k < b->bclients.size(); ++k) {
      const Client& c = s->clients[b->bclients[k]];
      if (!c.n_prefix) continue;
      PrefixClient pc{};
      pc.table = c.pfx; pc.grad = c.G(); pc.n = c.n_prefix; pc.first_layer = c.cut;
      pc.seq0 = pc.seq1 = -1;
      slot_of[b->bclients[k]] = (int)pcs.size();
      pcs.push_back(pc);
    }
    for (int i = 0; i < b->n_seqs; ++i) {
      const int cid = b->seq_client[i], P = s->clients[cid].n_prefix;
      seqx[i] = xcu.back();
      seqsh[i] = P;
      if (P) {
        PrefixClient& pc = pcs[slot_of[cid]];
        if (pc.seq0 < 0) pc.seq0 = i;
        pc.seq1 = i + 1;
      }
      for (int p = 0; p < P; ++p) { xsrc.push_back(make_int2(-1, slot_of[cid] << 16 | p)); xtok.push_back(-1); }
      for (int t = b->cu[i]; t < b->cu[i + 1]; ++t) { tokx[t] = (int)xsrc.size(); xsrc.push_back(make_int2(t, 0)); xtok.push_back(t); }
      xcu.push_back(xcu.back() + xl[i]);
      for (int q = 0; q < xl[i]; q += 64) xb64.push_back(make_int2(i, q));
      for (int q = 0; q < xl[i]; q += 128) xb128.push_back(make_int2(i, q));
    }
    b->n_pc = (int)pcs.size();
    b->pc_rows = 0;
    for (auto& pc : pcs) b->pc_rows += pc.n;
    std::vector<int4> xi, xikv, xiq, xiseq;
    attn_ws_items(xl.data(), b->n_seqs, D.H, xi, g_attn_order ? 1 : 0, s->num_sms);
    attn_ws_items(xl.data(), b->n_seqs, D.Hkv, xikv, g_attn_order ? 2 : 0, s->num_sms);
    attn_ws_items(xl.data(), b->n_seqs, D.H, xiq, g_attn_order ? 1 : 0, s->num_sms);
    attn_seq_items(xl.data(), b->n_seqs, D.Hkv, xiseq);
    menos_batch::AttnView& xv = b->xview;
    xv.n_seqs = b->n_seqs; xv.n_blocks = (int)xb64.size(); xv.n_blocks128 = (int)xb128.size(); xv.pairs = b->pairs_ext;
    xv.n_items = (int)xi.size(); xv.n_items_kv = (int)xikv.size(); xv.n_items_seq = (int)xiseq.size();
    o_xcu = put(xcu.data(), xcu.size() * 4); o_xblk = put(xb64.data(), xb64.size() * sizeof(int2));
    o_xblk128 = put(xb128.data(), xb128.size() * sizeof(int2)); o_xsrc = put(xsrc.data(), xsrc.size() * sizeof(int2));
    o_xtok = put(xtok.data(), xtok.size() * 4); o_tokx = put(tokx.data(), tokx.size() * 4);
    o_seqx = put(seqx.data(), seqx.size() * 4); o_pc = put(pcs.data(), pcs.size() * sizeof(PrefixClient));
    o_seqsh = put(seqsh.data(), seqsh.size() * 4);
    o_xit = put(xi.data(), xi.size() * sizeof(int4)); o_xitkv = put(xikv.data(), xikv.size() * sizeof(int4));
    o_xitq = put(xiq.data(), xiq.size() * sizeof(int4)); o_xitseq = put(xiseq.data(), xiseq.size() * sizeof(int4));
  }
  const size_t o_mt = put(mt.data(), mt.size() * sizeof(int2));
  const size_t o_nt = put(ntq.data(), ntq.size());

  // ---- slab
  uint8_t* slab = (uint8_t*)s->arena.alloc(slab_bytes);
  if (!slab) FAIL(MENOS_ENOMEM, "arena: batch needs %zu B, %zu of %zu B in use", slab_bytes, s->arena.used, s->arena.cap);
  b->slab = slab;
  b->L.assign(Ls, LayerSave{});
  const Rows Rw = rows_of(D, T);
  if (save) {
    uint8_t* p = slab;
    auto take = [&](size_t n) { uint8_t* r = p; p += align_up(n, 256); return r; };
    for (int l = 0; l < Ls; ++l) {
      LayerSave& S = b->L[l];
      S.x = (float*)take((size_t)Rw.Tloc * D.d * 4); S.xn = (bf16*)take((size_t)Rw.Tpad * D.d * 2);
      S.rstd1 = (float*)take((size_t)Rw.Tloc * 4);
      S.qkv = (bf16*)take((size_t)T * D.Nqkv * 2); S.O = (bf16*)take((size_t)T * D.Nq * 2);
      S.lse = (float*)take((size_t)D.H * std::max(T, b->Text) * 4 + kLsePad);
      S.h = (float*)take((size_t)Rw.Tloc * D.d * 4); S.hn = (bf16*)take((size_t)Rw.Tpad * D.d * 2);
      S.rstd2 = (float*)take((size_t)Rw.Tloc * 4);
      S.gu = (bf16*)take((size_t)T * D.gu_cols * 2);
      S.a = D.arch == MENOS_ARCH_OPT ? S.gu : b->save_a ? (bf16*)take((size_t)T * D.fpad * 2) : sc.a;
      for (int g = 0; g < NG; ++g) S.U[g] = b->g_active[g] ? (bf16*)take((size_t)T * b->R_used[g] * 2) : nullptr;
    }
  } else {
    b->L[0].x = (float*)slab;  // x_c copy (only the forward input is cached)
  }

  // ---- LoRA side-contraction problem lists (need buffer pointers: SAVE layout, or the NOGRAD layer set)
  std::vector<LoraRowsProblem> rprobs;
  std::vector<int2> rtiles;
  std::vector<LoraTokRedProblem> tprobs;
  std::vector<int4> ttiles;
  std::vector<LoraDUBProblem> dprobs;
  std::vector<LoraShrinkProblem> sprobs;
  std::vector<LoraTokRedProblem> daprobs;
  std::vector<int2> stiles;
  auto add_rows = [&](SGList& L, const std::vector<LoraRowsProblem>& ps) {
    L.probs_off = (int)rprobs.size(); L.n_probs = (int)ps.size(); L.tiles_off = (int)rtiles.size();
    std::vector<int2> tl;
    lora_rows_tiles(ps.data(), (int)ps.size(), tl);
    for (auto& x : tl) x.x += L.probs_off;
    for (const auto& pp : ps) { L.flops += 2.0 * pp.M * pp.N * pp.K; L.max_n = std::max(L.max_n, pp.N); }
    L.n_tiles = (int)tl.size();
    rprobs.insert(rprobs.end(), ps.begin(), ps.end());
    rtiles.insert(rtiles.end(), tl.begin(), tl.end());
  };
  auto add_tokred = [&](SGList& L, const std::vector<LoraTokRedProblem>& ps, int mt, int nt) {
    L.probs_off = (int)tprobs.size(); L.n_probs = (int)ps.size(); L.tiles_off = (int)ttiles.size();
    std::vector<int4> tl;
    lora_tokred_tiles(ps.data(), (int)ps.size(), mt, nt, tl);
    for (auto& x : tl) x.x += L.probs_off;
    for (const auto& pp : ps) L.flops += 2.0 * pp.M * pp.N * pp.T;
    L.n_tiles = (int)tl.size(); L.max_n = mt; L.tile_n = nt;
    tprobs.insert(tprobs.end(), ps.begin(), ps.end());
    ttiles.insert(ttiles.end(), tl.begin(), tl.end());
  };
  for (int l = 0; l < Ls; ++l) {
    const LayerSave& S = save ? b->L[l] : *ng;
    // bf16 copy of layer l's incoming gradient (sequence parallel: its all-gather, which also holds dh later)
    bf16* dyl = D.sp ? sc.gath : ((Ls - 1 - l) % 2 == 0) ? sc.dyb : sc.dxb;
    for (int g = 0; g < NG; ++g) {
      if (!b->g_active[g]) continue;
      const int R = b->R_used[g];
      // group input (X) and its leading dim; output-grad (dY) and its leading dim
      const bf16* X = nullptr; int ldx = 0;
      const bf16* dY = nullptr; int ldy = 0;
      bf16* U = S.U[g];
      switch (g) {
        case GQKV: X = S.xn; ldx = D.d; dY = sc.dqkv; ldy = D.Nqkv; break;
        case GO: X = S.O; ldx = D.Nq; dY = D.sp ? sc.gath : sc.dhb; ldy = D.d; break;
        case GGU: X = S.hn; ldx = D.d; dY = sc.dgu; ldy = D.gu_cols; break;
        case GD: X = S.a; ldx = D.fpad; dY = dyl; ldy = D.d; break;
      }
      std::vector<LoraRowsProblem> f;
      std::vector<LoraShrinkProblem> shk;
      std::vector<LoraDUBProblem> dub;
      std::vector<LoraTokRedProblem> da;
      size_t woff = 0;   // fp32 offset of the next problem's dU partials in sc.wsp (the group's lists run in turn)
      int da_w = 0;
      for (size_t k = 0; k < b->bclients.size(); ++k) {
        const Client& c = s->clients[b->bclients[k]];
        if (!c.width[g] || c.cut > l) continue;   // not yet in the segment at this layer
        const int t0 = b->btok_off[k], Tc = b->btok_n[k];
        for (int j0 = 0; j0 < c.width[g]; j0 += 128) {
          const int w = std::min(128, c.width[g] - j0);
          const int col = c.col_off[g] + j0;
          // shrink: U[t, col..col+w) = s * X_c Acat[col.., :]^T
          LoraRowsProblem p{};
          p.A = X + (size_t)t0 * ldx; p.lda = ldx;
          p.B = s->Acat[g][l] + (size_t)col * D.ldK_g[g]; p.ldb = D.ldK_g[g]; p.b_kn = 0;
          p.C = U + (size_t)t0 * R + col; p.ldc = R;
          p.M = Tc; p.N = w; p.K = D.K_g[g]; p.scale = c.s;
          f.push_back(p);
          shk.push_back(LoraShrinkProblem{t0, Tc, col, w, c.s});
        }
        // per target, ONE pass over its dY columns: dB = dY_t^T (s U_t) and dU_t = s dY_t B_t (per-slab partials,
        // then a fixed-order slab sum); targets own contiguous (gate/up: 128-interleaved) row ranges of Bcat
        LoraTokRedProblem pa{};
        int nseg = 0;
        for (int t = 0; t < NT; ++t) {
          if (kTargetGroup[t] != g || !(c.mask >> t & 1)) continue;
          LoraDUBProblem q{};
          q.dY = dY + (size_t)t0 * ldy + D.rb_base[t]; q.ldy = ldy;
          q.p_blk = D.rb_blk[t]; q.p_blk_stride = D.rb_stride[t];
          q.U = U + (size_t)t0 * R + c.col_off[g] + c.sub[t]; q.ldu = R;
          q.B = s->Bcat[g][l] + (size_t)D.rb_base[t] * s->cols[g].cap + c.col_off[g] + c.sub[t];
          q.ldb = s->cols[g].cap;
          q.dB = c.G() + c.offB[l * NT + t];
          q.dU = sc.dU[g] + (size_t)t0 * R + c.col_off[g] + c.sub[t]; q.lddu = R;
          q.Nt = D.N_t[t]; q.rank = c.rank; q.rs = c.rs; q.T = Tc; q.scale = c.s;
          // slab width from the target's own shape and rank (never from the batch: bitwise batched == alone):
          // 256 columns for the wide targets (N_t >= 8192: half the fp32 dU partials), 128 otherwise / on mma.sync
          q.n_slabs = (q.Nt + dub_mts(q) - 1) / dub_mts(q);
          q.W = sc.wsp + woff;
          q.t0 = t0; q.ycol0 = D.rb_base[t]; q.ucol0 = c.col_off[g] + c.sub[t];
          if (q.p_blk % LORA_DUB_MT) FAIL(MENOS_EINVAL, "LoRA row block %d not a multiple of %d", q.p_blk, LORA_DUB_MT);
          woff += (size_t)q.n_slabs * Tc * c.rank;
          dub.push_back(q);
          // dA of every target of the group in one pass over X: dU columns [sub_t, sub_t + rank) -> dA_t rows
          float* Ct = c.G() + c.offA[l * NT + t];
          if (nseg == 0) pa.C = Ct; else if (nseg == 1) pa.C1 = Ct; else pa.C2 = Ct;
          pa.N = D.K_t[t]; pa.ldc = D.K_t[t];
          ++nseg;
        }
        pa.P = sc.dU[g] + (size_t)t0 * R + c.col_off[g]; pa.ldp = R;
        pa.p_blk = 1 << 30; pa.p_blk_stride = 0;
        pa.Q = X + (size_t)t0 * ldx; pa.ldq = ldx;
        pa.M = c.width[g]; pa.T = Tc; pa.scale = 1.f;
        pa.m_seg = c.rs; pa.m_valid = c.rank;
        pa.t0 = t0; pa.pcol0 = c.col_off[g];
        da.push_back(pa);
        da_w = std::max(da_w, c.width[g]);
      }
      const size_t li = (size_t)l * NG + g;
      add_rows(b->sg_fwd[li], f);
      {
        menos_batch::ShkList& H = b->sg_shk[li];
        H = menos_batch::ShkList();
        H.X = X; H.x_rows = T; H.ldx = ldx; H.A = s->Acat[g][l]; H.a_rows = s->cols[g].cap; H.lda = D.ldK_g[g];
        H.K = D.K_g[g]; H.U = U; H.ldu = R;
        H.probs_off = (int)sprobs.size(); H.tiles_off = (int)stiles.size();
        std::vector<int2> tl;
        lora_shrink_tiles(shk.data(), (int)shk.size(), tl);
        for (auto& x : tl) x.x += H.probs_off;
        for (const auto& q : shk) { H.max_w = std::max(H.max_w, q.w); H.flops += 2.0 * q.T * q.w * H.K; }
        H.n_tiles = (int)tl.size();
        sprobs.insert(sprobs.end(), shk.begin(), shk.end());
        stiles.insert(stiles.end(), tl.begin(), tl.end());
      }
      b->dub_bufs[li] = menos_batch::DubBufs{dY, ldy, U, R, T};
      // rank <= 16 first (tcgen05 kernel), larger ranks after (mma.sync kernel): the kernel a client's problem
      // takes depends on its own rank only, never on who shares the batch
      std::stable_partition(dub.begin(), dub.end(), [](const LoraDUBProblem& q) { return q.rank <= 16; });
      std::stable_partition(dub.begin(), dub.end(), [](const LoraDUBProblem& q) { return dub_mts(q) == 256; });
      {
        SGList& Ld = b->sg_dub[li];
        Ld = SGList();
        for (const auto& q : dub) { Ld.n_small += q.rank <= 16 && !dub_env_mma(); Ld.n_wide += dub_mts(q) == 256; }
        Ld.probs_off = (int)dprobs.size(); Ld.n_probs = (int)dub.size();
        for (const auto& q : dub) {
          Ld.flops += 4.0 * q.Nt * q.rank * q.T;
          Ld.max_n = std::max(Ld.max_n, q.n_slabs);
          Ld.max_rank = std::max(Ld.max_rank, q.rank);
          Ld.max_elems = std::max(Ld.max_elems, (long long)q.T * q.rs);
        }
        dprobs.insert(dprobs.end(), dub.begin(), dub.end());
      }
      const int da_mt = da_w <= 16 ? 16 : da_w <= 32 ? 32 : 64;
      // slots <= 32 wide: tcgen05 (per client: the kernel never depends on who shares the batch); wider: mma.sync
      // with 128-column tiles (64-column ones, twice the CTAs at cfg1, measured slower: 33.6 vs 28.6 us, r2bf)
      {
        static const bool da_mma = [] { const char* e = getenv("MENOS_LORA_DA_MMA"); return e && atoi(e) == 1; }();
        std::vector<LoraTokRedProblem> da_big;
        menos_batch::DaTc& Dt = b->da_tc[li];
        Dt = menos_batch::DaTc();   // lists are rebuilt when a NOGRAD batch re-forwards
        Dt.probs_off = (int)daprobs.size(); Dt.X = X; Dt.rows = T; Dt.ldx = ldx; Dt.dU = sc.dU[g]; Dt.lddu = R;
        for (const auto& pa : da) {
          if (!da_mma && pa.M <= 32) {   // wider slots: the per-stage transpose of 48-64 dU columns makes the
                                           // tcgen05 kernel slower than the token reduction (r2bh: 150 vs 119 us)
            daprobs.push_back(pa); ++Dt.n;
            Dt.max_w = std::max(Dt.max_w, pa.M); Dt.max_n = std::max(Dt.max_n, pa.N);
            Dt.flops += 2.0 * pa.M * pa.N * pa.T;
          } else {
            da_big.push_back(pa);
          }
        }
        int big_w = 0;
        for (const auto& pa : da_big) big_w = std::max(big_w, pa.M);
        add_tokred(b->sg_da[li], da_big, big_w <= 16 ? 16 : big_w <= 32 ? 32 : 64, 128);
      }
    }
  }
  const size_t o_rp = put(rprobs.data(), rprobs.size() * sizeof(LoraRowsProblem));
  const size_t o_rt = put(rtiles.data(), rtiles.size() * sizeof(int2));
  const size_t o_tp = put(tprobs.data(), tprobs.size() * sizeof(LoraTokRedProblem));
  const size_t o_tt = put(ttiles.data(), ttiles.size() * sizeof(int4));
  const size_t o_dp = put(dprobs.data(), dprobs.size() * sizeof(LoraDUBProblem));
  const size_t o_sp = put(sprobs.data(), sprobs.size() * sizeof(LoraShrinkProblem));
  const size_t o_dap = put(daprobs.data(), daprobs.size() * sizeof(LoraTokRedProblem));
  const size_t o_st = put(stiles.data(), stiles.size() * sizeof(int2));
  uint8_t* meta = (uint8_t*)s->arena.alloc(blob.size());
  if (!meta) { s->arena.release(slab); b->slab = nullptr; FAIL(MENOS_ENOMEM, "arena: batch metadata"); }
  b->meta = meta;
  int rc = upload(s, meta, blob.data(), blob.size(), st);
  if (rc) return rc;
  b->d_cu = (int*)(meta + o_cu); b->d_pos = (int*)(meta + o_pos); b->d_blocks = (int2*)(meta + o_blk);
  if (b->has_pfx) {
    b->d_cu_ext = (int*)(meta + o_xcu); b->d_blocks_ext = (int2*)(meta + o_xblk);
    b->d_blocks128_ext = (int2*)(meta + o_xblk128); b->d_ext_src = (int2*)(meta + o_xsrc);
    b->d_ext_tok = (int*)(meta + o_xtok); b->d_tok_ext = (int*)(meta + o_tokx); b->d_seq_ext0 = (int*)(meta + o_seqx);
    b->d_pc = (PrefixClient*)(meta + o_pc);
    b->d_seq_shift = (int*)(meta + o_seqsh);
    b->xview.items = (int4*)(meta + o_xit); b->xview.items_kv = (int4*)(meta + o_xitkv);
    b->xview.items_q = (int4*)(meta + o_xitq); b->xview.items_seq = (int4*)(meta + o_xitseq);
  }
  b->d_blocks128 = (int2*)(meta + o_blk128);
  for (auto& v : b->views) {
    v.items = (int4*)(meta + v.o_items);
    v.items_kv = (int4*)(meta + v.o_items_kv);
    v.items_q = (int4*)(meta + v.o_items_q);
    v.items_seq = (int4*)(meta + v.o_items_seq);
    if (v.ds_ok) {
      v.ds_kv = (int4*)(meta + v.o_ds_kv); v.ds_q = (int4*)(meta + v.o_ds_q); v.ds_base = (int*)(meta + v.o_ds_base);
    }
  }
  for (int g = 0; g < NG; ++g) b->d_mtile[g] = (int2*)(meta + o_mt) + (size_t)g * b->n_mt;
  b->d_ntile_qkv = meta + o_nt;
  b->d_rprobs = (LoraRowsProblem*)(meta + o_rp);
  b->h_rprobs = std::move(rprobs);
  b->h_tprobs = std::move(tprobs);
  b->scratch_base = s->scratch; b->scratch_span = s->scratch_bytes;
  b->d_rtiles = (int2*)(meta + o_rt);
  b->d_tprobs = (LoraTokRedProblem*)(meta + o_tp);
  b->d_ttiles = (int4*)(meta + o_tt);
  b->d_dprobs = (LoraDUBProblem*)(meta + o_dp);
  b->d_sprobs = (LoraShrinkProblem*)(meta + o_sp);
  b->d_daprobs = (LoraTokRedProblem*)(meta + o_dap);
  b->h_daprobs = std::move(daprobs);
  b->d_stiles = (int2*)(meta + o_st);
  b->h_dprobs = std::move(dprobs);
  return MENOS_OK;
}

// scratch (per server, grown to the largest batch; used only inside one call)
// nograd_set: also reserve the NOGRAD forward's layer buffers (only a MENOS_FWD_NOGRAD forward needs them; the
// backward's re-forward writes into the batch's SAVE slab), so SAVE batches use exactly scratch_bytes_per_token
static int get_scratch(menos_server* s, int T, const int R_used[NG], Scratch& sc, bool nograd_set, int Text,
                       long long ds_tiles) {
  const Dims& D = s->D;
  const size_t need = scratch_bytes_of(D, T, R_used, nograd_set, Text, ds_tiles);
  const Rows Rw = rows_of(D, T);
  const size_t df = (size_t)Rw.Tloc * D.d * 4, db = (size_t)Rw.Tloc * D.d * 2, dp = (size_t)Rw.Tpad * D.d * 2;
  if (need != s->scratch_bytes) {   // shrink-to-fit too: a stale large block must not outlive the call that needed it
    if (s->scratch) s->arena.release(s->scratch);
    s->scratch = (uint8_t*)s->arena.alloc(need);
    if (!s->scratch) { s->scratch_bytes = 0; FAIL(MENOS_ENOMEM, "arena: scratch needs %zu B", need); }
    s->scratch_bytes = need;
  }
  uint8_t* p = s->scratch;
  auto take = [&](size_t n) { uint8_t* r = p; p += align_up(n, 256); return r; };
  sc.dyf = (float*)take(df); sc.dxf = (float*)take(df); sc.dhf = (float*)take(df); sc.xout = (float*)take(df);
  sc.dyb = (bf16*)take(db); sc.dxb = (bf16*)take(db); sc.dhb = (bf16*)take(db); sc.dhn = (bf16*)take(dp);
  sc.io = (bf16*)take(dp);
  sc.gath = sc.rsout = nullptr;
  if (D.sp) { sc.gath = (bf16*)take(dp); sc.rsout = (bf16*)take(db); }
  sc.qkv_x = sc.O_x = sc.dO_x = sc.dqkv_x = nullptr; sc.D_x = sc.dqacc_x = nullptr;
  if (Text > T) {
    sc.qkv_x = (bf16*)take((size_t)Text * D.Nqkv * 2); sc.O_x = (bf16*)take((size_t)Text * D.Nq * 2);
    sc.dO_x = (bf16*)take((size_t)Text * D.Nq * 2); sc.dqkv_x = (bf16*)take((size_t)Text * D.Nqkv * 2);
    sc.D_x = (float*)take((size_t)D.H * Text * 4 + kLsePad); sc.dqacc_x = (float*)take((size_t)Text * D.Nq * 4);
  }
  sc.dO = (bf16*)take((size_t)T * D.Nq * 2); sc.dqkv = (bf16*)take((size_t)T * D.Nqkv * 2);
  sc.dgu = (bf16*)take((size_t)T * D.gu_cols * 2); sc.a = (bf16*)take((size_t)T * D.fpad * 2);
  sc.Dsum = (float*)take((size_t)D.H * T * 4 + kLsePad);
  sc.wsp = (float*)take(wsp_bytes_of(D, T, R_used));
  for (int g = 0; g < NG; ++g) sc.dU[g] = (bf16*)take((size_t)T * R_used[g] * 2);
  sc.ds = ds_tiles > 0 ? (bf16*)(s->scratch + need - align_up((size_t)ds_tiles * kDsTileBytes, 256)) : nullptr;
  return MENOS_OK;
}

// NOGRAD layer buffers carved after the regular scratch (same arena block)
static void nograd_layer(menos_server* s, int T, const int R_used[NG], const Scratch& sc, LayerSave& S, int Text) {
  const Dims& D = s->D;
  const Rows Rw = rows_of(D, T);
  uint8_t* p = (uint8_t*)(sc.dU[NG - 1]) + align_up((size_t)T * R_used[NG - 1] * 2, 256);
  auto take = [&](size_t n) { uint8_t* r = p; p += align_up(n, 256); return r; };
  S.xn = (bf16*)take((size_t)Rw.Tpad * D.d * 2); S.h = (float*)take((size_t)Rw.Tloc * D.d * 4);
  S.qkv = (bf16*)take((size_t)T * D.Nqkv * 2); S.O = (bf16*)take((size_t)T * D.Nq * 2);
  S.gu = (bf16*)take((size_t)T * D.gu_cols * 2); S.lse = (float*)take((size_t)D.H * std::max(T, Text) * 4 + kLsePad);
  S.rstd1 = (float*)take((size_t)Rw.Tloc * 8); S.rstd2 = S.rstd1 + Rw.Tloc;
  S.hn = (bf16*)take((size_t)Rw.Tpad * D.d * 2);
  S.a = D.arch == MENOS_ARCH_OPT ? S.gu : sc.a;   // OPT: the down projection's input is relu(fc1), kept in gu
  for (int g = 0; g < NG; ++g) S.U[g] = (bf16*)take((size_t)T * R_used[g] * 2);
}

// =====================================================================================================
// per-layer schedules
// =====================================================================================================
// forward shrink U = s X A^T of one group's clients (tcgen05; MENOS_LORA_SHRINK_MMA=1: the mma.sync rows kernel)
static int run_shrink(menos_batch* b, size_t li, cudaStream_t st) {
  static const bool mma = [] { const char* e = getenv("MENOS_LORA_SHRINK_MMA"); return e && atoi(e) == 1; }();
  const menos_batch::ShkList& H = b->sg_shk[li];
  if (H.n_tiles == 0) return 0;
  if (mma || H.max_w > 128) {
    const SGList& L = b->sg_fwd[li];
    if (L.n_tiles == 0) return 0;
    ProfScope ps(PC_LORA, L.flops, 0, st);
    return lora_rows_run(b->d_rprobs, b->d_rtiles + L.tiles_off, L.n_tiles, L.max_n, st);
  }
  ProfScope ps(PC_LORA, H.flops, 0, st);
  return lora_shrink_tc_run(H.X, H.x_rows, H.ldx, H.A, H.a_rows, H.lda, H.K, b->d_sprobs, b->d_stiles + H.tiles_off,
                            H.n_tiles, H.max_w, H.U, H.ldu, st);
}
static int run_rows(menos_batch* b, const SGList& L, cudaStream_t st) {
  if (L.n_tiles == 0) return 0;
  ProfScope ps(PC_LORA, L.flops, 0, st);
  return lora_rows_run(b->d_rprobs, b->d_rtiles + L.tiles_off, L.n_tiles, L.max_n, st);
}
// fused dU + dB (one pass over each target's dY), then the fixed-order slab sum into the bf16 dU slot columns
// (tcgen05 for rank <= 16; MENOS_LORA_DUB_MMA=1 or larger ranks: the mma.sync kernel)
static int run_dub(menos_batch* b, size_t li, cudaStream_t st) {
  const SGList& L = b->sg_dub[li];
  if (L.n_probs == 0) return 0;
  ProfScope ps(PC_LORA, L.flops, 0, st);
  const menos_batch::DubBufs& Bf = b->dub_bufs[li];
  // [0, n_wide): tcgen05 with 256-column slabs; [n_wide, n_small): tcgen05, 128; the rest: mma.sync, 128
  int rc = lora_dub_tc_run(b->d_dprobs + L.probs_off, L.n_wide, L.max_n, Bf.Y, Bf.rows, Bf.ldy, Bf.U, Bf.ldu, 256, st);
  if (!rc)
    rc = lora_dub_tc_run(b->d_dprobs + L.probs_off + L.n_wide, L.n_small - L.n_wide, L.max_n, Bf.Y, Bf.rows, Bf.ldy, Bf.U,
                         Bf.ldu, 128, st);
  if (!rc && L.n_probs > L.n_small)
    rc = lora_dub_run(b->d_dprobs + L.probs_off + L.n_small, L.n_probs - L.n_small, L.max_n, L.max_rank, st);
  if (rc) return rc;
  return lora_du_reduce_run(b->d_dprobs + L.probs_off, L.n_probs, L.max_elems, st);
}
// dA of every client's group: tcgen05 for slots <= 32 wide, the mma.sync token reduction for wider ones
static int run_da(menos_batch* b, size_t li, cudaStream_t st);
static int run_tokred(menos_batch* b, const SGList& L, cudaStream_t st) {
  if (L.n_tiles == 0) return 0;
  ProfScope ps(PC_LORA, L.flops, 0, st);
  return lora_tokred_run(b->d_tprobs, b->d_ttiles + L.tiles_off, L.n_tiles, L.max_n, L.tile_n, st);
}
static int run_da(menos_batch* b, size_t li, cudaStream_t st) {
  const menos_batch::DaTc& Dt = b->da_tc[li];
  if (Dt.n > 0) {
    ProfScope ps(PC_LORA, Dt.flops, 0, st);
    int rc = lora_da_tc_run(b->d_daprobs + Dt.probs_off, Dt.n, Dt.max_n, Dt.max_w, Dt.X, Dt.rows, Dt.ldx, Dt.dU,
                            Dt.lddu, st);
    if (rc) return rc;
  }
  return run_tokred(b, b->sg_da[li], st);
}

// tensor-parallel all-reduce (sum, in place, stream-ordered) through the caller's callback (menos_tp_cfg)
static int tp_allreduce(menos_server* s, void* buf, size_t count, int dtype, cudaStream_t st) {
  if (s->tp.world <= 1 || count == 0) return MENOS_OK;
  return s->comm.run(MENOS_COLL_ALLREDUCE, buf, buf, count, dtype, st);
}
static inline bool tp_on(const menos_server* s) { return s->tp.world > 1; }

// sequence parallel (A16): all-gather of the rank's [Tloc, d] rows (already in place at buf + row0 d) into [Tpad, d]
static int sp_gather(menos_server* s, const Rows& R, bf16* buf, cudaStream_t st) {
  return s->comm.run(MENOS_COLL_ALLGATHER, buf + (size_t)R.row0 * s->D.d, buf, (size_t)R.Tloc * s->D.d, MENOS_DT_BF16, st);
}
// reduce-scatter of a [Tpad, d] partial sum (rows past T zeroed) into the rank's [Tloc, d] rows
static int sp_scatter(menos_server* s, const Rows& R, bf16* part, bf16* out, cudaStream_t st) {
  if (R.Tpad > R.T) CUDA_TRY(cudaMemsetAsync(part + (size_t)R.T * s->D.d, 0, (size_t)(R.Tpad - R.T) * s->D.d * 2, st));
  return s->comm.run(MENOS_COLL_REDUCE_SCATTER, part, out, (size_t)R.Tloc * s->D.d, MENOS_DT_BF16, st);
}

static GemmArgs gemm_base(menos_server* s) {
  GemmArgs a;
  memset(&a, 0, sizeof a);
  a.num_sms = s->num_sms;
  return a;
}

// forward of layer l: x -> y; S holds the destinations of every intermediate
// x, y: the layer's fp32 residual stream in / out (sequence parallel: the rank's Tloc rows)
static int layer_forward(menos_server* s, menos_batch* b, int l, const float* x, float* y, const LayerSave& S,
                         const Scratch& sc, bool use_lists, cudaStream_t st) {
  const Dims& D = s->D;
  const auto& W = s->W[l];
  const int T = b->Tl[l];
  if (T == 0) return MENOS_OK;
  const Rows R = rows_of(D, T);
  const menos_batch::AttnView& V = b->views[b->view_of[l]];
  const bool opt = D.arch == MENOS_ARCH_OPT;
  // A1: RMSNorm1 (OPT: LayerNorm1) (fp32 residual in, bf16 GEMM operand out); sequence parallel: on the rank's rows,
  // written in place into the all-gather buffer
  {
    ProfScope ps(PC_NORM, 0, (double)R.Tloc * (6.0 * D.d + 4), st);
    bf16* xn = S.xn + (size_t)R.row0 * D.d;
    if (opt) K_TRY(layernorm_fwd(x, W.g1, W.be1, xn, S.rstd1, R.Tloc, D.d, D.eps, st));
    else K_TRY(rmsnorm_fwd(x, W.g1, xn, S.rstd1, R.Tloc, D.d, D.eps, st));
  }
  if (D.sp) { int rc = sp_gather(s, R, S.xn, st); if (rc) return rc; }   // A16: every token's xn for the QKV GEMM
  // A2: QKV GEMM (+ segmented LoRA q/k/v expand, + RoPE epilogue)
  if (b->g_active[GQKV]) {
    CUDA_TRY(cudaMemsetAsync(S.U[GQKV], 0, (size_t)T * b->R_used[GQKV] * 2, st));
    if (use_lists) K_TRY(run_shrink(b, (size_t)l * NG + GQKV, st));
  }
  {
    GemmArgs a = gemm_base(s);
    a.M = T; a.N = D.Nqkv; a.K = D.d; a.b_mn_major = 0;
    a.A = S.xn; a.lda = D.d; a.B = W.wqkv; a.ldb = D.d;
    if (b->g_active[GQKV]) {
      a.R = b->R_used[GQKV]; a.A2 = S.U[GQKV]; a.lda2 = a.R; a.B2 = s->Bcat[GQKV][l]; a.ldb2 = s->cols[GQKV].cap;
      a.mtile_extra = b->d_mtile[GQKV]; a.ntile_extra = b->d_ntile_qkv;
    }
    a.epi = EPI_ROPE; a.out = S.qkv; a.ldo = D.Nqkv;
    a.rope_cs = s->rope; a.pos = b->d_pos; a.head_dim = D.hd; a.rope_cols = D.Nq + D.Nkv;
    if (opt) { a.epi = EPI_STORE; a.bias = W.bqkv; }   // OPT: biases, no RoPE (learned positions are client-side)
    { ProfScope ps(PC_GEMM, 2.0 * a.M * a.N * a.K, 0, st); K_TRY(gemm_run(a, st)); }
  }
  // A3: varlen causal flash attention (prefix tuning, NEXT-3: on the extension -- every prefix client's sequence is
  // preceded by its P prefix rows, so causal attention over it is "the whole prefix plus the causal keys", R28)
  {
    const bool xp = b->has_pfx;
    const menos_batch::AttnView& AV = xp ? b->xview : V;
    if (xp)
      K_TRY(prefix_gather(S.qkv, D.Nqkv, b->d_ext_src, b->Text, b->d_pc, l, D.Nq, D.Nkv, sc.qkv_x, st));
    AttnArgs a;
    memset(&a, 0, sizeof a);
    a.qkv = xp ? sc.qkv_x : S.qkv; a.ld_qkv = D.Nqkv; a.O = xp ? sc.O_x : S.O; a.ld_o = D.Nq; a.lse = S.lse;
    a.cu_seqlens = xp ? b->d_cu_ext : b->d_cu;
    const int2* blk64 = xp ? b->d_blocks_ext : b->d_blocks;
    a.qblocks = blk64; a.n_qblocks = AV.n_blocks; a.kvblocks = blk64; a.n_kvblocks = AV.n_blocks;
    a.T = xp ? b->Text : T; a.H = D.H; a.Hkv = D.Hkv; a.hd = D.hd; a.scale = 1.f / std::sqrt((float)D.hd);
    {
      ProfScope ps(PC_ATTN_FWD, 4.0 * D.hd * D.H * AV.pairs, 0, st);
      if ((D.hd == 128 || D.hd == 64) && (g_attn_tc & 4)) K_TRY(attn_fwd_ws(a, AV.items, AV.n_items, s->num_sms, st));
      else K_TRY(attn_fwd(a, st));
    }
    if (xp) K_TRY(rows_map(sc.O_x, D.Nq, b->d_tok_ext, T, D.Nq, S.O, D.Nq, st));   // drop the prefix rows' outputs
  }
  // A4: O GEMM (+ LoRA o) + residual
  if (b->g_active[GO]) {
    CUDA_TRY(cudaMemsetAsync(S.U[GO], 0, (size_t)T * b->R_used[GO] * 2, st));
    if (use_lists) K_TRY(run_shrink(b, (size_t)l * NG + GO, st));
  }
  {
    GemmArgs a = gemm_base(s);
    a.M = T; a.N = D.d; a.K = D.Nq; a.A = S.O; a.lda = D.Nq; a.B = W.wo; a.ldb = D.Nq;
    if (b->g_active[GO]) {
      a.R = b->R_used[GO]; a.A2 = S.U[GO]; a.lda2 = a.R; a.B2 = s->Bcat[GO][l]; a.ldb2 = s->cols[GO].cap;
      a.mtile_extra = b->d_mtile[GO];
    }
    a.epi = EPI_RESID; a.outf = S.h; a.ldo = D.d; a.resid = x; a.ldr = D.d;
    if (opt) a.bias = W.bo;
    if (D.sp) { a.epi = EPI_STORE; a.out = sc.dhn; a.outf = nullptr; a.resid = nullptr; }   // row-parallel partial
    { ProfScope ps(PC_GEMM, 2.0 * a.M * a.N * a.K, 0, st); K_TRY(gemm_run(a, st)); }
    if (D.sp) {   // A16: reduce-scatter of the o-proj partial sums, then the residual add on the rank's rows
      int rc = sp_scatter(s, R, sc.dhn, sc.rsout, st);
      if (rc) return rc;
      K_TRY(add_bf16_to_f32(x, sc.rsout, S.h, (long long)R.Tloc * D.d, st));
    }
  }
  // A5: RMSNorm2 (OPT: LayerNorm2)
  {
    ProfScope ps(PC_NORM, 0, (double)R.Tloc * (6.0 * D.d + 4), st);
    bf16* hn = S.hn + (size_t)R.row0 * D.d;
    if (opt) K_TRY(layernorm_fwd(S.h, W.g2, W.be2, hn, S.rstd2, R.Tloc, D.d, D.eps, st));
    else K_TRY(rmsnorm_fwd(S.h, W.g2, hn, S.rstd2, R.Tloc, D.d, D.eps, st));
  }
  if (D.sp) { int rc = sp_gather(s, R, S.hn, st); if (rc) return rc; }   // A16: every token's hn for gate|up
  // A6: gate/up GEMM (+ LoRA gate/up) + SwiGLU epilogue
  if (b->g_active[GGU]) {
    CUDA_TRY(cudaMemsetAsync(S.U[GGU], 0, (size_t)T * b->R_used[GGU] * 2, st));
    if (use_lists) K_TRY(run_shrink(b, (size_t)l * NG + GGU, st));
  }
  {
    GemmArgs a = gemm_base(s);
    a.M = T; a.N = 2 * D.fpad; a.K = D.d; a.A = S.hn; a.lda = D.d; a.B = W.wgu; a.ldb = D.d;
    if (b->g_active[GGU]) {
      a.R = b->R_used[GGU]; a.A2 = S.U[GGU]; a.lda2 = a.R; a.B2 = s->Bcat[GGU][l]; a.ldb2 = s->cols[GGU].cap;
      a.mtile_extra = b->d_mtile[GGU];
    }
    a.epi = EPI_SWIGLU_FWD; a.out = S.gu; a.ldo = 2 * D.fpad; a.out2 = S.a; a.ldo2 = D.fpad;
    if (opt) { a.N = D.fpad; a.epi = EPI_RELU_FWD; a.ldo = D.fpad; a.bias = W.bu; }   // OPT: a = relu(fc1(hn))
    { ProfScope ps(PC_GEMM, 2.0 * a.M * a.N * a.K, 0, st); K_TRY(gemm_run(a, st)); }
  }
  // A7: down GEMM (+ LoRA down) + residual
  if (b->g_active[GD]) {
    CUDA_TRY(cudaMemsetAsync(S.U[GD], 0, (size_t)T * b->R_used[GD] * 2, st));
    if (use_lists) K_TRY(run_shrink(b, (size_t)l * NG + GD, st));
  }
  {
    GemmArgs a = gemm_base(s);
    a.M = T; a.N = D.d; a.K = D.fpad; a.A = S.a; a.lda = D.fpad; a.B = W.wd; a.ldb = D.fpad;
    if (b->g_active[GD]) {
      a.R = b->R_used[GD]; a.A2 = S.U[GD]; a.lda2 = a.R; a.B2 = s->Bcat[GD][l]; a.ldb2 = s->cols[GD].cap;
      a.mtile_extra = b->d_mtile[GD];
    }
    a.epi = EPI_RESID; a.outf = y; a.ldo = D.d; a.resid = S.h; a.ldr = D.d;
    if (opt) a.bias = W.bd;
    if (D.sp) { a.epi = EPI_STORE; a.out = sc.dhn; a.outf = nullptr; a.resid = nullptr; }
    { ProfScope ps(PC_GEMM, 2.0 * a.M * a.N * a.K, 0, st); K_TRY(gemm_run(a, st)); }
    if (D.sp) {   // A16: reduce-scatter of the down-proj partial sums, residual add on the rank's rows
      int rc = sp_scatter(s, R, sc.dhn, sc.rsout, st);
      if (rc) return rc;
      K_TRY(add_bf16_to_f32(S.h, sc.rsout, y, (long long)R.Tloc * D.d, st));
    }
  }
  return MENOS_OK;
}

// backward of layer l: dy -> dx (LoRA grads of layer l written into each client's G)
// dyf/dy: the incoming gradient (fp32 residual stream + its bf16 copy); dxf/dxb: the outgoing one
static int layer_backward(menos_server* s, menos_batch* b, int l, const float* dyf, const bf16* dy, float* dxf,
                          bf16* dxb, const Scratch& sc, cudaStream_t st) {
  const Dims& D = s->D;
  const auto& W = s->W[l];
  const LayerSave& S = b->L[l];
  const int T = b->Tl[l];
  if (T == 0) return MENOS_OK;
  const menos_batch::AttnView& V = b->views[b->view_of[l]];
  const bool opt = D.arch == MENOS_ARCH_OPT;
  const Rows R = rows_of(D, T);
  if (D.sp) {   // A16: every token's incoming gradient for the row-parallel down-dX GEMM (and LoRA down)
    CUDA_TRY(cudaMemcpyAsync(sc.gath + (size_t)R.row0 * D.d, dy, (size_t)R.Tloc * D.d * 2, cudaMemcpyDeviceToDevice, st));
    int rc = sp_gather(s, R, sc.gath, st);
    if (rc) return rc;
    dy = sc.gath;
  }
  // A8: down dX (+ LoRA down) with SwiGLU backward epilogue -> dgu
  if (b->g_active[GD]) K_TRY(run_dub(b, (size_t)l * NG + GD, st));
  {
    GemmArgs a = gemm_base(s);
    a.M = T; a.N = D.fpad; a.K = D.d; a.b_mn_major = 1;
    a.A = dy; a.lda = D.d; a.B = W.wd; a.ldb = D.fpad;
    if (b->g_active[GD]) {
      a.R = b->R_used[GD]; a.A2 = sc.dU[GD]; a.lda2 = a.R; a.B2 = s->Acat[GD][l]; a.ldb2 = D.ldK_g[GD];
      a.mtile_extra = b->d_mtile[GD];
    }
    a.epi = EPI_SWIGLU_BWD; a.out = sc.dgu; a.ldo = 2 * D.fpad; a.aux = S.gu; a.ldaux = 2 * D.fpad;
    if (opt) { a.epi = EPI_RELU_BWD; a.ldo = D.fpad; a.ldaux = D.fpad; }   // dz = da * (relu(z) > 0)
    { ProfScope ps(PC_GEMM, 2.0 * a.M * a.N * a.K, 0, st); K_TRY(gemm_run(a, st)); }
  }
  if (b->g_active[GD]) K_TRY(run_da(b, (size_t)l * NG + GD, st));
  // A9: gate/up dX (+ LoRA) -> dhn; RMSNorm2 backward + residual -> dh
  if (b->g_active[GGU]) K_TRY(run_dub(b, (size_t)l * NG + GGU, st));
  {
    GemmArgs a = gemm_base(s);
    a.M = T; a.N = D.d; a.K = D.gu_cols; a.b_mn_major = 1;
    a.A = sc.dgu; a.lda = D.gu_cols; a.B = W.wgu; a.ldb = D.d;
    if (b->g_active[GGU]) {
      a.R = b->R_used[GGU]; a.A2 = sc.dU[GGU]; a.lda2 = a.R; a.B2 = s->Acat[GGU][l]; a.ldb2 = D.ldK_g[GGU];
      a.mtile_extra = b->d_mtile[GGU];
    }
    a.epi = EPI_STORE; a.out = sc.dhn; a.ldo = D.d;
    { ProfScope ps(PC_GEMM, 2.0 * a.M * a.N * a.K, 0, st); K_TRY(gemm_run(a, st)); }
    if (D.sp) { int rc = sp_scatter(s, R, sc.dhn, sc.rsout, st); if (rc) return rc; }   // A16: gate|up-dX partials
  }
  if (b->g_active[GGU]) K_TRY(run_da(b, (size_t)l * NG + GGU, st));
  {
    ProfScope ps(PC_NORM, 0, (double)R.Tloc * (16.0 * D.d + 4), st);
    const bf16* dhn = D.sp ? sc.rsout : sc.dhn;
    if (opt) K_TRY(layernorm_bwd(dhn, S.h, W.g2, dyf, sc.dhf, sc.dhb, R.Tloc, D.d, D.eps, st));
    else K_TRY(rmsnorm_bwd(dhn, S.h, W.g2, S.rstd2, dyf, sc.dhf, sc.dhb, R.Tloc, D.d, st));
  }
  bf16* dh_all = sc.dhb;   // the O-dX GEMM's A operand: every token's dh
  if (D.sp) {               // A16
    CUDA_TRY(cudaMemcpyAsync(sc.gath + (size_t)R.row0 * D.d, sc.dhb, (size_t)R.Tloc * D.d * 2, cudaMemcpyDeviceToDevice, st));
    int rc = sp_gather(s, R, sc.gath, st);
    if (rc) return rc;
    dh_all = sc.gath;
  }
  // A10: O dX (+ LoRA o) -> dO (and, for head_dim % 32 == 0, the attention backward's row sums D)
  const bool fuse_dsum = D.hd % 32 == 0 && 128 % D.hd == 0;
  if (b->g_active[GO]) K_TRY(run_dub(b, (size_t)l * NG + GO, st));
  {
    GemmArgs a = gemm_base(s);
    a.M = T; a.N = D.Nq; a.K = D.d; a.b_mn_major = 1;
    a.A = dh_all; a.lda = D.d; a.B = W.wo; a.ldb = D.Nq;
    if (b->g_active[GO]) {
      a.R = b->R_used[GO]; a.A2 = sc.dU[GO]; a.lda2 = a.R; a.B2 = s->Acat[GO][l]; a.ldb2 = D.ldK_g[GO];
      a.mtile_extra = b->d_mtile[GO];
    }
    a.epi = EPI_STORE; a.out = sc.dO; a.ldo = D.Nq;
    if (fuse_dsum) {   // A11 prologue fused: D = rowsum(dO . O) per head from the epilogue's bf16 dO
      a.epi = EPI_STORE_DSUM; a.aux = S.O; a.ldaux = D.Nq; a.dsum = sc.Dsum; a.dsum_ld = T; a.dsum_hd = D.hd;
    }
    { ProfScope ps(PC_GEMM, 2.0 * a.M * a.N * a.K, 0, st); K_TRY(gemm_run(a, st)); }
  }
  if (b->g_active[GO]) K_TRY(run_da(b, (size_t)l * NG + GO, st));
  // A11: attention backward (+ RoPE backward) -> dqkv
  if (!fuse_dsum) {
    ProfScope ps(PC_ATTN_PREP, 0, (double)T * (4.0 * D.Nq + 4 * D.H), st);
    K_TRY(attn_bwd_prep(sc.dO, S.O, sc.Dsum, T, D.H, D.hd, st));
  }
  {
    // prefix tuning (NEXT-3): the backward runs on the extension too -- dO and D are zero on the prefix rows (their
    // outputs were dropped), the kernels skip the RoPE backward (prefix keys are not rotated, R28) and it is applied
    // when the sequence rows are copied back; the prefix rows' dk, dv become the prefix gradients
    const bool xp = b->has_pfx;
    const menos_batch::AttnView& AV = xp ? b->xview : V;
    if (xp) {
      K_TRY(rows_map(sc.dO, D.Nq, b->d_ext_tok, b->Text, D.Nq, sc.dO_x, D.Nq, st));
      K_TRY(lse_map(sc.Dsum, T, b->d_ext_tok, b->Text, D.H, sc.D_x, st));
      K_TRY(prefix_gather(S.qkv, D.Nqkv, b->d_ext_src, b->Text, b->d_pc, l, D.Nq, D.Nkv, sc.qkv_x, st));
    }
    AttnArgs a;
    memset(&a, 0, sizeof a);
    a.qkv = xp ? sc.qkv_x : S.qkv; a.ld_qkv = D.Nqkv; a.O = S.O; a.ld_o = D.Nq; a.lse = S.lse;
    a.cu_seqlens = xp ? b->d_cu_ext : b->d_cu;
    const int2* blk64 = xp ? b->d_blocks_ext : b->d_blocks;
    a.qblocks = blk64; a.n_qblocks = AV.n_blocks; a.kvblocks = blk64; a.n_kvblocks = AV.n_blocks;
    a.T = xp ? b->Text : T; a.H = D.H; a.Hkv = D.Hkv; a.hd = D.hd; a.scale = 1.f / std::sqrt((float)D.hd);
    a.dO = xp ? sc.dO_x : sc.dO; a.ld_do = D.Nq; a.D = xp ? sc.D_x : sc.Dsum;
    a.dqkv = xp ? sc.dqkv_x : sc.dqkv; a.ld_dqkv = D.Nqkv;
    a.rope_cs = opt ? nullptr : s->rope;   // OPT: no RoPE backward
    a.pos_shift = xp ? b->d_seq_shift : nullptr;   // extension: positions shifted back by the prefix, prefix rows unrotated
    // one-pass backward: dQ accumulates in fp32 in the forward-output buffer (free during the backward: Nq <= d)
    a.dq_acc = xp ? sc.dqacc_x : sc.xout;
    {
      ProfScope ps(PC_ATTN_BWD, 8.0 * D.hd * D.H * AV.pairs, 0, st);
      if (!xp && AV.ds_ok && sc.ds) {   // S, P, dP once per pair: dK/dV (+ dS^T tiles), then dQ from the tiles
        for (const int4& c : AV.ds_chunks)
          K_TRY(attn_bwd_ws_ds(a, AV.ds_kv + c.x, c.y, AV.ds_q + c.z, c.w, sc.ds, b->ds_tiles, AV.ds_base,
                               s->num_sms, st));
      } else if (D.hd == 128 && (g_attn_tc & 32))
        K_TRY(attn_bwd_fused(a, AV.items_seq, AV.n_items_seq, s->num_sms, st));
      else if ((D.hd == 128 || D.hd == 64) && (g_attn_tc & 8))
        K_TRY(attn_bwd_ws(a, AV.items_kv, AV.n_items_kv, AV.items_q, AV.n_items, s->num_sms, st));
      else K_TRY(attn_bwd(a, st));
    }
    if (xp) {
      // the kernels applied the RoPE backward at the true positions: the sequence rows are copied back as they are
      // (the same kernel epilogue as without prefix clients, so a LoRA client's results do not depend on them)
      K_TRY(dqkv_from_ext(sc.dqkv_x, b->d_tok_ext, T, D.H, D.Hkv, D.hd, nullptr, b->d_pos, sc.dqkv, st));
      K_TRY(prefix_grad(sc.dqkv_x, D.Nq, D.Nkv, b->d_pc, b->n_pc, b->pc_rows, b->d_seq_ext0, l, st));
    }
  }
  // A12: QKV dX (+ LoRA q/k/v) -> dxn; RMSNorm1 backward + residual -> dx
  if (b->g_active[GQKV]) K_TRY(run_dub(b, (size_t)l * NG + GQKV, st));
  {
    GemmArgs a = gemm_base(s);
    a.M = T; a.N = D.d; a.K = D.Nqkv; a.b_mn_major = 1;
    a.A = sc.dqkv; a.lda = D.Nqkv; a.B = W.wqkv; a.ldb = D.d;
    if (b->g_active[GQKV]) {
      a.R = b->R_used[GQKV]; a.A2 = sc.dU[GQKV]; a.lda2 = a.R; a.B2 = s->Acat[GQKV][l]; a.ldb2 = D.ldK_g[GQKV];
      a.mtile_extra = b->d_mtile[GQKV];
    }
    a.epi = EPI_STORE; a.out = sc.dhn; a.ldo = D.d;
    { ProfScope ps(PC_GEMM, 2.0 * a.M * a.N * a.K, 0, st); K_TRY(gemm_run(a, st)); }
    if (D.sp) { int rc = sp_scatter(s, R, sc.dhn, sc.rsout, st); if (rc) return rc; }   // A16: qkv-dX partials
  }
  if (b->g_active[GQKV]) K_TRY(run_da(b, (size_t)l * NG + GQKV, st));
  {
    ProfScope ps(PC_NORM, 0, (double)R.Tloc * (16.0 * D.d + 4), st);
    const bf16* dxn = D.sp ? sc.rsout : sc.dhn;
    if (opt) K_TRY(layernorm_bwd(dxn, S.x, W.g1, sc.dhf, dxf, dxb, R.Tloc, D.d, D.eps, st));
    else K_TRY(rmsnorm_bwd(dxn, S.x, W.g1, S.rstd1, sc.dhf, dxf, dxb, R.Tloc, D.d, st));
  }
  return MENOS_OK;
}

// NEXT-3: the clients whose cut is layer l enter there -- their x_c rows [Tl[l-1], Tl[l]) (kept in
// the fp32 copy L[0].x of the whole batch input) join the residual stream x that layer l reads
static int join_rows(menos_server* s, menos_batch* b, int l, float* x, cudaStream_t st) {
  if (l <= 0 || l >= s->n_layers) return MENOS_OK;
  const int lo = b->Tl[l - 1], hi = b->Tl[l];
  if (hi == lo || x == b->L[0].x) return MENOS_OK;
  const size_t d = (size_t)s->D.d;
  CUDA_TRY(cudaMemcpyAsync(x + lo * d, b->L[0].x + lo * d, (size_t)(hi - lo) * d * 4, cudaMemcpyDeviceToDevice, st));
  return MENOS_OK;
}

// full SAVE forward over all layers: X[0] = b->L[0].x (already filled), output -> xout (fp32)
static int forward_save(menos_server* s, menos_batch* b, const Scratch& sc, float* xout, cudaStream_t st) {
  for (int l = 0; l < s->n_layers; ++l) {
    float* y = (l + 1 < s->n_layers) ? b->L[l + 1].x : xout;
    int rc = layer_forward(s, b, l, b->L[l].x, y, b->L[l], sc, true, st);
    if (rc) return rc;
    rc = join_rows(s, b, l + 1, y, st);
    if (rc) return rc;
  }
  return MENOS_OK;
}

// =====================================================================================================
// C-ABI: forward / backward
// =====================================================================================================
extern "C" int menos_forward(menos_server* s, int n_seqs, const int32_t* seq_client, const int32_t* seq_len,
                             const void* x_c, void* x_s, int flags, void* stream, menos_batch** batch) {
  if (!s || n_seqs <= 0 || !seq_client || !seq_len || !x_c || !x_s) FAIL(MENOS_EINVAL, "bad arguments");
  if (flags != MENOS_FWD_SAVE && flags != MENOS_FWD_NOGRAD) FAIL(MENOS_EINVAL, "bad flags %d", flags);
  if (!batch && flags != MENOS_FWD_NOGRAD) FAIL(MENOS_EINVAL, "batch == NULL requires MENOS_FWD_NOGRAD");
  if (batch) *batch = nullptr;
  for (int l = 0; l < s->n_layers; ++l) if (!s->loaded[l]) FAIL(MENOS_ESTATE, "layer %d weights not loaded", l);
  CUDA_TRY(cudaSetDevice(s->device));
  cudaStream_t st = (cudaStream_t)stream;
  if (int rc0 = bind_stream(s, st)) return rc0;
  std::unique_ptr<menos_batch> b;
  int rc = build_batch(s, n_seqs, seq_client, seq_len, flags == MENOS_FWD_NOGRAD, b);
  if (rc) return rc;
  const Dims& D = s->D;
  const int T = b->T;
  Scratch sc;
  rc = get_scratch(s, T, b->R_used, sc, b->nograd, b->Text, b->ds_tiles);
  if (rc) return rc;
  LayerSave ng{};
  if (b->nograd) nograd_layer(s, T, b->R_used, sc, ng, b->Text);
  rc = finalize_batch(s, b.get(), sc, &ng, st);
  if (rc) return rc;
  auto fail_free = [&](int code) {
    if (b->slab) s->arena.release(b->slab);
    if (b->meta) s->arena.release(b->meta);
    return code;
  };
  // x_c (bf16, host or device) -> staging -> the fp32 residual stream X[0] (sequence parallel: the rank's rows;
  // padding rows zero)
  const Rows R = rows_of(D, T);
  if (R.Tpad > T) CUDA_TRY(cudaMemsetAsync(sc.io + (size_t)T * D.d, 0, (size_t)(R.Tpad - T) * D.d * 2, st));
  if (cudaMemcpyAsync(sc.io, x_c, (size_t)T * D.d * 2, cudaMemcpyDefault, st) != cudaSuccess ||
      convert_bf16_to_f32_vec(sc.io + (size_t)R.row0 * D.d, b->L[0].x, (long long)R.Tloc * D.d, st) != 0) {
    set_err("copy of x_c failed");
    return fail_free(MENOS_ECUDA);
  }
  if (!b->nograd) {
    rc = forward_save(s, b.get(), sc, sc.xout, st);
    if (rc) return fail_free(rc);
  } else {
    // Alg.1 L6: forward without caching activations; only x_c is kept
    const float* x = b->L[0].x;
    for (int l = 0; l < s->n_layers; ++l) {
      float* y = ((s->n_layers - 1 - l) % 2 == 0) ? sc.xout : sc.dxf;
      rc = layer_forward(s, b.get(), l, x, y, ng, sc, true, st);
      if (rc) return fail_free(rc);
      rc = join_rows(s, b.get(), l + 1, y, st);
      if (rc) return fail_free(rc);
      x = y;
    }
  }
  if (convert_f32_to_bf16(sc.xout, sc.io + (size_t)R.row0 * D.d, (long long)R.Tloc * D.d, st) != 0) {
    set_err("conversion of x_s failed");
    return fail_free(MENOS_ECUDA);
  }
  if (D.sp) { rc = sp_gather(s, R, sc.io, st); if (rc) return fail_free(rc); }   // every rank returns all of x_s
  if (cudaMemcpyAsync(x_s, sc.io, (size_t)T * D.d * 2, cudaMemcpyDefault, st) != cudaSuccess) {
    set_err("copy of x_s failed");
    return fail_free(MENOS_ECUDA);
  }
  cudaPointerAttributes pa;
  if (cudaPointerGetAttributes(&pa, x_s) == cudaSuccess && pa.type != cudaMemoryTypeDevice &&
      pa.type != cudaMemoryTypeManaged)
    CUDA_TRY(cudaStreamSynchronize(st));
  cudaGetLastError();
  if (!batch) {   // NOGRAD, nothing retained (Alg.1 L7): later arena allocations are stream-ordered after this call
    fail_free(MENOS_OK);
    return MENOS_OK;
  }
  b->counted = true;
  for (int c : b->bclients) s->batch_refs[c]++;
  if (!b->nograd) { b->counted_save = true; s->live_save++; }
  *batch = b.release();
  return MENOS_OK;
}

extern "C" int menos_batch_free(menos_server* s, menos_batch* b) {
  if (!s || !b) FAIL(MENOS_EINVAL, "null argument");
  if (b->counted) for (int c : b->bclients) s->batch_refs[c]--;
  if (b->counted_save) s->live_save--;
  if (b->slab) s->arena.release(b->slab);
  if (b->meta) s->arena.release(b->meta);
  delete b;
  return MENOS_OK;
}

// Shift every problem-list pointer into the batch's forward-time scratch block to the current block (same T and
// slot widths => same internal offsets, get_scratch) and re-upload the lists (stream-ordered, pinned ring).
static int relocate_scratch_refs(menos_server* s, menos_batch* b, cudaStream_t st) {
  if (b->scratch_base == s->scratch || b->scratch_base == nullptr) return MENOS_OK;
  const uint8_t* lo = b->scratch_base;
  const uint8_t* hi = lo + b->scratch_span;
  const ptrdiff_t delta = s->scratch - b->scratch_base;
  auto mv = [&](auto*& p) {
    const uint8_t* q = reinterpret_cast<const uint8_t*>(p);
    if (q >= lo && q < hi) p = reinterpret_cast<std::remove_reference_t<decltype(p)>>(const_cast<uint8_t*>(q) + delta);
  };
  for (auto& p : b->h_rprobs) { mv(p.A); mv(p.B); mv(p.C); }
  for (auto& p : b->h_tprobs) { mv(p.P); mv(p.Q); mv(p.C); mv(p.C1); mv(p.C2); }
  for (auto& p : b->h_dprobs) { mv(p.dY); mv(p.U); mv(p.B); mv(p.dB); mv(p.W); mv(p.dU); }
  for (auto& d : b->dub_bufs) { mv(d.Y); mv(d.U); }
  for (auto& d : b->da_tc) { mv(d.X); mv(d.dU); }
  int rc = 0;
  if (!b->h_rprobs.empty()) rc = upload(s, b->d_rprobs, b->h_rprobs.data(), b->h_rprobs.size() * sizeof(LoraRowsProblem), st);
  if (!rc && !b->h_tprobs.empty())
    rc = upload(s, b->d_tprobs, b->h_tprobs.data(), b->h_tprobs.size() * sizeof(LoraTokRedProblem), st);
  if (!rc && !b->h_dprobs.empty())
    rc = upload(s, b->d_dprobs, b->h_dprobs.data(), b->h_dprobs.size() * sizeof(LoraDUBProblem), st);
  if (rc) return rc;
  b->scratch_base = s->scratch; b->scratch_span = s->scratch_bytes;
  return MENOS_OK;
}

extern "C" int menos_backward(menos_server* s, menos_batch* b, const void* g_c, void* g_s, void* stream) {
  if (!s || !b || !g_c || !g_s) FAIL(MENOS_EINVAL, "bad arguments");
  for (int c : b->bclients) if (!s->clients[c].used) FAIL(MENOS_ESTATE, "client %d unregistered since forward", c);
  CUDA_TRY(cudaSetDevice(s->device));
  cudaStream_t st = (cudaStream_t)stream;
  if (int rc0 = bind_stream(s, st)) return rc0;
  const Dims& D = s->D;
  const int T = b->T;
  const Rows R = rows_of(D, T);
  Scratch sc;
  int rc = get_scratch(s, T, b->R_used, sc, false, b->Text, b->ds_tiles);
  if (rc) return rc;
  if (b->nograd) {
    // Alg.1 L10: re-forward with gradient preparation from the cached x_c; the SAVE slab is
    // allocated only now (on-demand allocation)
    float* xc = b->L[0].x;
    uint8_t* old_slab = b->slab;
    uint8_t* old_meta = b->meta;
    b->slab = nullptr; b->meta = nullptr;
    b->nograd = false;
    rc = finalize_batch(s, b, sc, nullptr, st);
    if (rc) { b->nograd = true; b->slab = old_slab; b->meta = old_meta; return rc; }
    CUDA_TRY(cudaMemcpyAsync(b->L[0].x, xc, (size_t)R.Tloc * D.d * 4, cudaMemcpyDeviceToDevice, st));
    s->arena.release(old_meta);   // stream-ordered reuse: later users run after these copies
    s->arena.release(old_slab);
    rc = forward_save(s, b, sc, sc.xout, st);
    if (rc) return rc;
  } else {
    rc = relocate_scratch_refs(s, b, st);
    if (rc) return rc;
  }
  // g_c (bf16) -> the bf16 copy of the incoming gradient and the fp32 gradient residual stream (sequence parallel:
  // the rank's rows, padding rows zero)
  if (D.sp) {
    if (R.Tpad > T) CUDA_TRY(cudaMemsetAsync(sc.io + (size_t)T * D.d, 0, (size_t)(R.Tpad - T) * D.d * 2, st));
    CUDA_TRY(cudaMemcpyAsync(sc.io, g_c, (size_t)T * D.d * 2, cudaMemcpyDefault, st));
    CUDA_TRY(cudaMemcpyAsync(sc.dyb, sc.io + (size_t)R.row0 * D.d, (size_t)R.Tloc * D.d * 2, cudaMemcpyDeviceToDevice, st));
  } else {
    CUDA_TRY(cudaMemcpyAsync(sc.dyb, g_c, (size_t)T * D.d * 2, cudaMemcpyDefault, st));
  }
  K_TRY(convert_bf16_to_f32_vec(sc.dyb, sc.dyf, (long long)R.Tloc * D.d, st));
  // the block-diagonal dU scratch: zero once (a batch's slot positions are the same in every layer)
  for (int g = 0; g < NG; ++g)
    if (b->g_active[g]) CUDA_TRY(cudaMemsetAsync(sc.dU[g], 0, (size_t)T * b->R_used[g] * 2, st));
  float* dyf = sc.dyf; bf16* dyb = sc.dyb;
  float* dxf = sc.dxf; bf16* dxb = sc.dxb;
  const bool mixed_cuts = b->Tl[0] != T;
  for (int l = s->n_layers - 1; l >= 0; --l) {
    rc = layer_backward(s, b, l, dyf, dyb, dxf, dxb, sc, st);
    if (rc) return rc;
    std::swap(dyf, dxf);
    std::swap(dyb, dxb);
    if (mixed_cuts) {   // NEXT-3: the clients whose cut is layer l leave here; dx rows [Tl[l-1], Tl[l]) are their g_s
      const int lo = l > 0 ? b->Tl[l - 1] : 0, hi = b->Tl[l];
      if (hi > lo)
        CUDA_TRY(cudaMemcpyAsync(sc.io + (size_t)lo * D.d, dyb + (size_t)lo * D.d, (size_t)(hi - lo) * D.d * 2,
                                 cudaMemcpyDeviceToDevice, st));
    }
  }
  // A16: the replicated adapters' gradients (dA of column-parallel, dB of row-parallel targets) are partial
  // sums over the ranks' shards; one contiguous fp32 all-reduce per client
  if (tp_on(s))
    for (int c : b->bclients) {
      rc = tp_allreduce(s, s->clients[c].G(), s->clients[c].n_rep, MENOS_DT_F32, st);
      if (rc) return rc;
    }
  if (D.sp) {   // every rank returns all of g_s
    CUDA_TRY(cudaMemcpyAsync(sc.io + (size_t)R.row0 * D.d, dyb, (size_t)R.Tloc * D.d * 2, cudaMemcpyDeviceToDevice, st));
    rc = sp_gather(s, R, sc.io, st);
    if (rc) return rc;
  }
  CUDA_TRY(cudaMemcpyAsync(g_s, (mixed_cuts || D.sp) ? sc.io : dyb, (size_t)T * D.d * 2, cudaMemcpyDefault, st));
  cudaPointerAttributes pa;
  if (cudaPointerGetAttributes(&pa, g_s) == cudaSuccess && pa.type != cudaMemoryTypeDevice &&
      pa.type != cudaMemoryTypeManaged)
    CUDA_TRY(cudaStreamSynchronize(st));
  cudaGetLastError();
  // Release I after the backward (Fig.3(b); Alg.1 L13): the slab returns to the arena; stream
  // order guarantees later users run after this backward's kernels.
  return menos_batch_free(s, b);
}

// =====================================================================================================
// white-box test hooks (include/menos_testing.h)
// =====================================================================================================
extern "C" int menos_test_batch_tensor(menos_server* s, menos_batch* b, int layer, int which, void* host_out,
                                       size_t* bytes) {
  if (!s || !b || !bytes || layer < 0 || layer >= s->n_layers || b->nograd) FAIL(MENOS_EINVAL, "bad arguments");
  const Dims& D = s->D;
  const LayerSave& S = b->L[layer];
  const size_t T = b->T;
  const Rows R = rows_of(D, b->T);   // sequence parallel: x, h are the rank's rows; xn, hn all-gathered (padded)
  const void* src = nullptr;
  size_t n = 0;
  switch (which) {
    case 0: src = S.x; n = (size_t)R.Tloc * D.d * 4; break;
    case 1: src = S.xn; n = T * D.d * 2; break;
    case 2: src = S.qkv; n = T * D.Nqkv * 2; break;
    case 3: src = S.O; n = T * D.Nq * 2; break;
    case 4: src = S.h; n = (size_t)R.Tloc * D.d * 4; break;
    case 5: src = S.hn; n = T * D.d * 2; break;
    case 6: src = S.gu; n = T * D.gu_cols * 2; break;
    case 7: src = S.a; n = T * D.fpad * 2; break;
    case 8: case 9: case 10: case 11: src = S.U[which - 8]; n = src ? T * b->R_used[which - 8] * 2 : 0; break;
    case 12: src = S.lse; n = (size_t)D.H * std::max<size_t>(T, b->Text) * 4; break;   // prefix: [H, Text]
    default: FAIL(MENOS_EINVAL, "bad which");
  }
  *bytes = n;
  if (host_out && n) {
    CUDA_TRY(cudaDeviceSynchronize());
    CUDA_TRY(cudaMemcpy(host_out, src, n, cudaMemcpyDeviceToHost));
  }
  return MENOS_OK;
}
