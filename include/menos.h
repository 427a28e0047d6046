/*
 * menos.h -- C-ABI of the Menos server segment on B200 (sm_100a).
 *
 * Menos (Hu & Li, MIDDLEWARE '24) splits a Llama-2 model between clients and a server.  The server runs
 * the middle segment f_s (decoder layers [cut, L)) for many clients at once over ONE shared frozen base
 * copy (spatial sharing, §3.1), each client with its own LoRA adapters phi_s
 * (§2.1; §5.1).  This header is the boundary the paper's problem statement
 * implies:
 *
 *   server cycle (§2.2, Alg.1):
 *     menos_forward   : x_s = f_s(x_c; theta_s, phi_s)                  (Step 2 / Alg.1 L6, L10)
 *     menos_backward  : g_s = dL/dx_c from g_c = dL/dx_s, plus dphi_s   (Step 4 / Alg.1 L11)
 *     menos_adapter_step : AdamW on phi_s only                          (Alg.1 L12; Eq.1)
 *   client join / profiling (§3.3): menos_register_client, menos_client_memory.
 *   OOM avoidance (§4.1): MENOS_ENOMEM is RETURNED, never a crash.
 *
 * Conventions (all functions):
 *   - Return an int status (menos_status); 0 = OK.  Argument / shape / state errors return synchronously
 *     and launch nothing.  Asynchronous device errors are sticky and surface from the next call or from
 *     menos_sync().  menos_last_error() gives a thread-local message for the last failure.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *   - Activation buffers (x_c, x_s, g_c, g_s) are bf16, token-major row-major [T, d_model], client-major
 *     then sequence-major packing.  They may be HOST or DEVICE pointers (detected with
 *     cudaPointerGetAttributes): host buffers are staged through pinned memory inside the call, and the call
 *     synchronises `stream` before returning when it wrote to a host buffer.
 *   - No torch types, no C++ types.  The library never frees caller memory; the caller never frees
 *     library memory except through the destroy / free calls below.
 *   - Every kernel runs on the GPU (sm_100a); there is no CPU fallback.  If no sm_100 device is present,
 *     menos_server_create returns MENOS_ECUDA.
 */
#ifndef MENOS_H_
#define MENOS_H_

#include <stddef.h>
#include <stdint.h>

#ifndef MENOS_API
#define MENOS_API __attribute__((visibility("default")))
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  MENOS_OK = 0,
  MENOS_EINVAL = -1,    /* bad argument, shape or layout                                        */
  MENOS_ENOMEM = -2,    /* arena / registry / device memory cannot hold the request */
  MENOS_ENOCLIENT = -3, /* unknown client id                                                     */
  MENOS_ESTATE = -4,    /* e.g. backward on a batch without a live forward, weights not loaded    */
  MENOS_ECUDA = -5,     /* CUDA error (sticky until menos_sync)                                   */
  MENOS_ENCCL = -6      /* tensor-parallel all-reduce callback failed (menos_tp_cfg)             */
} menos_status;

typedef struct menos_server menos_server;
typedef struct menos_batch menos_batch;

/* Llama-2 decoder-layer dimensions (PAPER.md:292 names Llama 2 [32]; dims are Llama-2's). */
typedef struct {
  int d_model;     /* d                                  */
  int n_heads;     /* H                                  */
  int n_kv_heads;  /* H_kv (GQA when < H)                 */
  int d_ff;        /* f (SwiGLU inner size)               */
  float rms_eps;   /* RMSNorm epsilon (1e-5); LayerNorm epsilon for OPT */
  float rope_theta;/* RoPE base (1e4); unused for OPT      */
  int arch;        /* MENOS_ARCH_LLAMA (0, default) or MENOS_ARCH_OPT (1)  */
} menos_model_cfg;

/* Model families (SURVEY.md §8(f) NEXT-4; PAPER.md:292, :294 evaluate Llama 2 and OPT):
 *   LLAMA: pre-RMSNorm, RoPE, no biases, SwiGLU MLP (gate, up, down), GQA allowed.
 *   OPT  : pre-LayerNorm (do_layer_norm_before, OPT-1.3B and up) with gain and bias, learned positions (on the
 *          client: the embedding layer is client-side), biases on q, k, v, o, fc1, fc2, ReLU MLP
 *          y = h + fc2(relu(fc1(LN2(h)))).  n_kv_heads must equal n_heads.  LoRA targets q, k, v, o, up (= fc1)
 *          and down (= fc2); gate does not exist (EINVAL). */
enum { MENOS_ARCH_LLAMA = 0, MENOS_ARCH_OPT = 1 };

/* One decoder layer's frozen base weights, natural (HF) layouts, bf16 row-major, host or device.
 * The library COPIES them into its single device copy (WeightStore); the caller may free them after the
 * call returns.  hd = d_model / n_heads.  Under tensor parallelism (opts->tp.world = W > 1) every projection
 * is the rank's SHARD with H, H_kv, f replaced by H/W, H_kv/W, f/W in the shapes below (wo and wdown keep
 * their d rows and hold the rank's columns); g1, g2 are full. */
typedef struct {
  const void* wq;    /* [H*hd, d]     */
  const void* wk;    /* [H_kv*hd, d]  */
  const void* wv;    /* [H_kv*hd, d]  */
  const void* wo;    /* [d, H*hd]     */
  const void* wgate; /* [f, d]        */
  const void* wup;   /* [f, d]        */
  const void* wdown; /* [d, f]        */
  const void* g1;    /* [d] input RMSNorm gain          (OPT: self_attn_layer_norm weight) */
  const void* g2;    /* [d] post-attention RMSNorm gain (OPT: final_layer_norm weight)     */
  /* OPT only (NULL for Llama): biases and LayerNorm biases, bf16.  wgate is NULL for OPT; wup = fc1 [f, d],
   * wdown = fc2 [d, f]. */
  const void* bq;    /* [H*hd] */
  const void* bk;    /* [H*hd] */
  const void* bv;    /* [H*hd] */
  const void* bo;    /* [d]    */
  const void* bup;   /* [f]  fc1 bias */
  const void* bdown; /* [d]  fc2 bias */
  const void* b1;    /* [d]  self_attn_layer_norm bias */
  const void* b2;    /* [d]  final_layer_norm bias     */
} menos_layer_weights;

/* LoRA target projections (bit mask).  PAPER.md:294 uses q,v.
 * MENOS_T_PREFIX: prefix tuning instead of LoRA (SURVEY.md §8(f) NEXT-3; PAPER.md:59 §2.1, :121 §3.1; Li & Liang [16]):
 * the client holds, per server layer, P = `rank` learned key and value vectors per KV head which every query of its
 * sequences attends to in addition to its causal keys (one softmax over both; the prefix keys are used as given, no
 * RoPE; sequence positions stay 0-based -- DESIGN.md R28).  It must be the client's only target (alpha is ignored);
 * not available with tensor parallelism, and a batch holding a prefix client cannot mix cut points.  Init
 * N(0, 1).  get/set_adapter target index 7: which A = prefix keys [P, H_kv*hd], B = prefix values [P, H_kv*hd]
 * (dA / dB their gradients, summed over the client's tokens). */
enum {
  MENOS_T_Q = 1, MENOS_T_K = 2, MENOS_T_V = 4, MENOS_T_O = 8,
  MENOS_T_GATE = 16, MENOS_T_UP = 32, MENOS_T_DOWN = 64, MENOS_T_PREFIX = 128
};
/* target index (0..7) used by get/set_adapter: q, k, v, o, gate, up, down, prefix */

typedef struct {
  double lr, beta1, beta2, eps, weight_decay; /* torch.optim.AdamW semantics (scalars in double, as torch forms them) */
} menos_adamw_cfg;

/* Tensor parallelism (Llama-2-70B, BASELINE.json configs[4]).
 * Megatron split of every server layer over `world` ranks, one process and one server object per GPU, with
 * SEQUENCE PARALLELISM for everything outside the split GEMMs:
 *   column-parallel: Wq, Wk, Wv (rank r holds heads [r*H/world, (r+1)*H/world) and the matching KV heads),
 *                    W_gate, W_up (rows [r*f/world, (r+1)*f/world));
 *   row-parallel:    Wo (columns of rank r's heads), W_down (columns [r*f/world, (r+1)*f/world));
 *   token-parallel:  the residual streams (x, h forward; dy, dh backward), RMSNorm forward / backward and their
 *                    saved statistics: rank r owns token rows [r*Tl, (r+1)*Tl), Tl = ceil(T / world) (the last rank's
 *                    rows past T are padding and never read).
 * Exchanges per layer, all bf16 [*, d] (the payload of one all-reduce split into its two halves):
 *   forward : all-gather of RMSNorm1's and RMSNorm2's outputs (the column-parallel GEMMs read every token);
 *             reduce-scatter of the o-proj and down-proj partial sums (the residual add then runs on the rank's rows);
 *   backward: all-gather of the incoming gradient dy and of dh (the row-parallel dX GEMMs read every token);
 *             reduce-scatter of the gate|up-dX and qkv-dX partial sums (RMSNorm backward runs on the rank's rows).
 * x_c / g_c are read at the rank's own rows; x_s / g_s are all-gathered so every rank returns the whole [T, d].
 * LoRA: column-parallel targets keep A [r, d] replicated and B [N/world, r] sharded; row-parallel targets keep
 * A [r, K/world] sharded and B [d, r] replicated.  Row-parallel adapters fold into the reduce-scatter by linearity;
 * the gradients of the replicated tensors (dA of q,k,v,gate,up; dB of o,down) are partial sums and are all-reduced
 * (fp32) once per backward per client over a contiguous region.  No other exchange.
 * Transport: if `nccl_id` is non-NULL (128 bytes from menos_tp_unique_id on rank 0, broadcast by the caller) the
 * library creates an NCCL communicator and issues the collectives itself on the call's stream (NCCL over NVLink /
 * NVSwitch; `collective` is ignored).  Otherwise `collective` is called (e.g. torch.distributed over gloo); it must
 * be stream-ordered w.r.t. `stream` and leave identical bytes on every rank.  Nonzero return: MENOS_ENCCL.
 * world <= 1 and nccl_id == NULL: no tensor parallelism (replica).  world == 1 with nccl_id: the sequence-parallel
 * schedule on one rank (test vehicle for the NCCL transport). */
enum { MENOS_DT_F32 = 0, MENOS_DT_BF16 = 1 };
enum { MENOS_COLL_ALLREDUCE = 0, MENOS_COLL_ALLGATHER = 1, MENOS_COLL_REDUCE_SCATTER = 2 };
/* ALLREDUCE: in-place sum of `count` elements (send == recv).  ALLGATHER: send holds `count` elements, recv
 * world * count (rank-major).  REDUCE_SCATTER: send holds world * count, recv gets this rank's `count` of the sum. */
typedef int (*menos_collective_fn)(int op, const void* send, void* recv, size_t count, int dtype, void* stream,
                                   void* user);
typedef struct {
  int rank, world;                /* 0 <= rank < world; H, H_kv and d_ff divisible by world               */
  menos_collective_fn collective; /* caller transport (used when nccl_id == NULL)                          */
  void* user;                     /* passed back to collective                                             */
  const void* nccl_id;            /* 128-byte ncclUniqueId, or NULL                                        */
} menos_tp_cfg;
/* 128-byte NCCL unique id for menos_tp_cfg.nccl_id (call on one rank, broadcast to the others).  ENCCL if NCCL is
 * not loadable. */
MENOS_API int menos_tp_unique_id(void* out128);
/* Collectives this server has issued on the tensor-parallel path and their payload bytes (an all-reduce counts its
 * buffer, an all-gather / reduce-scatter world x one rank's share). */
MENOS_API int menos_tp_stats(menos_server* s, long long* calls, double* bytes);

typedef struct {
  int max_clients;     /* registry capacity (default 64)                                     */
  int max_rank;        /* largest LoRA rank accepted (default 64)                             */
  int max_seq_len;     /* longest sequence (RoPE table rows; default 4096)                   */
  size_t arena_bytes;  /* activation arena I (Eq.3); 0 = free memory - 8 GiB    */
  int num_sms;         /* persistent-grid width; 0 = device SM count                          */
  menos_tp_cfg tp;     /* tensor parallelism; zero-initialised = none                          */
} menos_server_opts;

/* forward flags */
enum {
  MENOS_FWD_SAVE = 0,   /* keep the intermediates I for the backward                                   */
  MENOS_FWD_NOGRAD = 1  /* Menos on-demand mode (Alg.1 L6): keep only x_c; backward
                           re-forwards with SAVE, then runs backward (Alg.1 L10-11)                     */
};

/* Create a server for decoder layers [first_layer, first_layer + n_layers) on CUDA device `device`.
 * `w` = n_layers entries (or NULL: load each layer with menos_server_load_layer before forward).
 * opts may be NULL (defaults).  Errors: EINVAL (dims), ECUDA (no sm_100 device), ENOMEM. */
MENOS_API int menos_server_create(const menos_model_cfg* cfg, int first_layer, int n_layers, const menos_layer_weights* w,
                        int device, const menos_server_opts* opts, menos_server** out);
MENOS_API int menos_server_load_layer(menos_server* s, int layer /* 0..n_layers-1 */, const menos_layer_weights* w);
MENOS_API void menos_server_destroy(menos_server* s);

/* Client join: allocates A, B (fp32 master + bf16 copy in the shared slot tables), dA,
 * dB, AdamW m, v.  Init: A ~ U(-1/sqrt(K), 1/sqrt(K)) from init_seed, B = 0 (PEFT default).
 * rank 1..max_rank; alpha > 0; target_mask != 0.  Returns ENOMEM when the registry is full. */
MENOS_API int menos_register_client(menos_server* s, int rank, float alpha, uint32_t target_mask, const menos_adamw_cfg* opt,
                          uint64_t init_seed, int32_t* client_id);
/* Per-client cut point (clients choose how many layers they keep): the client
 * holds layers [0, cut_layer) itself and its tokens enter the server segment at ABSOLUTE layer cut_layer
 * (first_layer <= cut_layer < first_layer + n_layers); menos_register_client == cut_layer = first_layer.  The
 * client has adapters only for layers >= cut_layer (get/set_adapter below it: EINVAL); its x_c is the input of
 * layer cut_layer and its g_s the gradient there.  In a batch, clients must come in non-decreasing cut order
 * (EINVAL otherwise): layer l then runs on the prefix of tokens whose client has cut <= l. */
MENOS_API int menos_register_client_at(menos_server* s, int cut_layer, int rank, float alpha, uint32_t target_mask,
                                       const menos_adamw_cfg* opt, uint64_t init_seed, int32_t* client_id);
MENOS_API int menos_unregister_client(menos_server* s, int32_t client_id);

/* Closed-form memory demands (Alg.2 L2): persistent A+O bytes of the client, and the arena
 * bytes of a SAVE forward (M_f) and of the backward (M_b) for n_tokens tokens of that client. */
MENOS_API int menos_client_memory(menos_server* s, int32_t client_id, int n_tokens, size_t* persistent, size_t* fwd_bytes,
                        size_t* bwd_bytes);

/* Exact arena demand of ONE batched call over these clients (n_tokens[i] tokens of client ids[i]): the peak arena
 * bytes the forward (*fwd_bytes) and the backward (*bwd_bytes) of that batch need, including the per-call scratch
 * block and the block-diagonal LoRA slot columns the batch spans (which depend on the set of clients, so a sum of
 * per-client menos_client_memory figures is not exact).  flags as in menos_forward.  Used to form waves / admit
 * clients (Alg.2) without ever hitting MENOS_ENOMEM. */
MENOS_API int menos_batch_memory(menos_server* s, int n_clients, const int32_t* ids, const int32_t* n_tokens, int flags,
                       size_t* fwd_bytes, size_t* bwd_bytes);
/* flags bit for menos_batch_memory: figures are ADDITIVE UPPER BOUNDS -- computed with the LoRA slot span and the
 * saved-tensor set of every registered client instead of the batch's own, so for any partition of a batch into
 * parts P_k, sum_k demand(P_k, MENOS_MEM_BOUND) >= demand(batch): every term is linear in tokens plus a nonnegative
 * constant, and 256-byte rounding is subadditive.  The Alg.2 scheduler (menos_sched_*) ADDS per-client demands
 * (PAPER.md:238-263); this keeps its accounting safe when the granted requests run as one batched call. */
enum { MENOS_MEM_BOUND = 2 };

/* Stream rule: every forward / backward / adapter_step of one server must be issued on ONE stream (the first such
 * call binds it; a different stream later returns MENOS_EINVAL).  Arena slabs and the scratch block are released on
 * the host as soon as their last kernel is enqueued and reused in stream order, which is only safe on one stream.
 * Live batches: a SAVE batch (or a retained NOGRAD batch) returned by menos_forward is "live" until menos_backward or
 * menos_batch_free.  While any SAVE batch is live, a registration that would grow the LoRA slot tables returns
 * MENOS_ESTATE (the batch's precomputed LoRA problem lists point into them); a client that belongs to a live batch
 * cannot be unregistered (MENOS_ESTATE), so its id cannot be reused under the batch either. */

/* Step 2: x_s = f_s(x_c).  n_seqs sequences; seq_client[i] (host) is the client of sequence i and
 * seq_len[i] (host) its length (>= 1, <= max_seq_len).  Sequences of one client must be contiguous
 * (client-major packing).  T = sum(seq_len).  x_c, x_s: [T, d] bf16 (host or device).
 * On success *batch is a handle that owns the saved activations (or the x_c copy under NOGRAD) until
 * menos_backward or menos_batch_free.  ENOMEM if the arena cannot hold them (form smaller waves).
 * NOGRAD with batch == NULL: nothing is retained after the call (Alg.1 L6-7: compute x_s without caching, then
 * release GPU memory); the caller keeps x_c for the later re-forward ("we just need to cache the
 * forward activations for the re-forward computation") and runs it as a SAVE forward + backward.  This is the
 * mode the Alg.2 scheduler loop uses: a backward wave may group clients whose forwards ran in different waves.
 * SAVE requires batch != NULL. */
MENOS_API int menos_forward(menos_server* s, int n_seqs, const int32_t* seq_client, const int32_t* seq_len, const void* x_c,
                  void* x_s, int flags, void* stream, menos_batch** batch);

/* Step 4: g_s = dL/dx_c from g_c = dL/dx_s ([T, d] bf16, host or device).  OVERWRITES every participating
 * client's dA, dB (summed over its tokens).  Frees the batch's arena slab; the handle is consumed. */
MENOS_API int menos_backward(menos_server* s, menos_batch* batch, const void* g_c, void* g_s, void* stream);
MENOS_API int menos_batch_free(menos_server* s, menos_batch* batch);

/* Alg.1 L12: one fused AdamW launch over the n clients' adapters (torch.optim.AdamW semantics, per-client
 * step count); consumes and zeroes their dA, dB and refreshes the bf16 copies used by the kernels. */
MENOS_API int menos_adapter_step(menos_server* s, int n, const int32_t* client_ids, void* stream);

/* Host copies of one adapter tensor (fp32).  which: 0 = A [r, K], 1 = B [N, r], 2 = dA, 3 = dB,
 * (under tensor parallelism K and N are the rank's local extents: see menos_tp_cfg; adapter_shape reports them)
 * 4 = m_A, 5 = m_B, 6 = v_A, 7 = v_B.  layer in 0..n_layers-1, target 0..6 (must be in the client's mask).
 * set_adapter accepts which 0..1 (A, B) and refreshes the bf16 copy.  Both synchronise the device. */
MENOS_API int menos_adapter_shape(menos_server* s, int32_t id, int target, int* rows, int* cols);
MENOS_API int menos_get_adapter(menos_server* s, int32_t id, int layer, int target, int which, float* host_out);
MENOS_API int menos_set_adapter(menos_server* s, int32_t id, int layer, int target, int which, const float* host_in);

/* Statistics: bytes of the shared base copy (M), of all clients' A+O, arena capacity and in-use bytes. */
typedef struct {
  size_t base_bytes, adapters_bytes, arena_bytes, arena_used, arena_peak;
  int n_clients;
  int num_sms;
} menos_stats;
MENOS_API int menos_get_stats(menos_server* s, menos_stats* out);

/* Per-kernel-class device time, measured with CUDA events recorded on the launching stream around every
 * launch while profiling is enabled (bench.py's live roofline).  enable(1) clears the counters; read
 * synchronises the device, fills one entry per class (max_n >= 8) and clears the counters.
 * flops / bytes are the ALGORITHMIC work of the launches (DESIGN.md §"Roofline accounting"). */
typedef struct {
  char name[32];
  int launches;
  double ms, flops, bytes;
} menos_kernel_stat;
MENOS_API int menos_profile_enable(int on);
MENOS_API int menos_profile_read(menos_kernel_stat* out, int max_n, int* n_out);

/* Number of kernels this library has launched since load (evidence for bench.py's gpu_launches). */
MENOS_API unsigned long long menos_launch_count(void);

MENOS_API int menos_sync(menos_server* s);
MENOS_API const char* menos_last_error(void);

/* ---------------------------------------------------------------------------------------------------------------
 * Task scheduler: Algorithm 2 of PAPER.md:235-263 (§4.2), FCFS + backfilling over GPU memory (SURVEY.md §8(f)
 * NEXT-2).  Host-only (no CUDA; usable without a GPU).  It decides which waiting requests enter the batched
 * menos_forward / menos_backward calls: every SCHEDULE (one per event) returns a list of grants, and the caller
 * runs the FWD grants of that list as one batched NOGRAD menos_forward (Alg.1 L6) and the BWD grants as one
 * batched re-forward + menos_backward + menos_adapter_step (Alg.1 L10-12), then reports each client's completion.
 *
 *   menos_sched_create(M_avail)          Alg.2 L1, L3, L4 (M_avail = bytes the scheduler may hand out)
 *   menos_sched_set_demand(i, M_f, M_b)  Alg.2 L2 (e.g. menos_batch_memory(..., MENOS_MEM_BOUND) of client i
 *                                        alone: those figures are additive, so a batch of granted requests
 *                                        never exceeds the memory the grants reserved)
 *   menos_sched_arrive(i, kind)          Alg.2 L7-9: x_c (kind FWD) or g_c (kind BWD) of client i arrived
 *   menos_sched_complete(i)              Alg.2 L10-13: client i's task finished and released A[i]
 * Grants are written to out[0..*n_out) in the order they were made: the FCFS head first (L16-22), then the
 * backfilled requests in waiting-list order (L23-24).  out must hold max_clients entries (max_out >= max_clients;
 * EINVAL otherwise, checked before anything changes).  Errors: ENOCLIENT (id out of range / no demands), ESTATE (the client
 * already has a request waiting or running, or complete() without a running task), ENOMEM (a demand larger than
 * M_avail at create: it could never be granted and would block the FCFS head forever; nothing is enqueued).
 * Not thread-safe: one event at a time (the paper's scheduler is one event loop, Alg.2 L5-6). */
typedef struct menos_sched menos_sched;
enum { MENOS_REQ_FWD = 0, MENOS_REQ_BWD = 1 };
typedef struct {
  int32_t client;  /* serving process S_i                                 */
  int32_t kind;    /* MENOS_REQ_FWD / MENOS_REQ_BWD                        */
  size_t bytes;    /* memory reserved for it: M_f[i] or M_b[i] (A[i])     */
} menos_sched_grant;
MENOS_API int menos_sched_create(size_t m_avail, int max_clients, menos_sched** out);
MENOS_API void menos_sched_destroy(menos_sched* s);
MENOS_API int menos_sched_set_demand(menos_sched* s, int32_t client, size_t m_f, size_t m_b);
MENOS_API int menos_sched_arrive(menos_sched* s, int32_t client, int kind, menos_sched_grant* out, int max_out,
                                 int* n_out);
MENOS_API int menos_sched_complete(menos_sched* s, int32_t client, menos_sched_grant* out, int max_out, int* n_out);
/* current M_avail, |W|, number of running tasks, and the first max_waiting entries of W (may be NULL) */
MENOS_API int menos_sched_state(menos_sched* s, size_t* m_avail, int* n_waiting, int* n_running, int32_t* waiting,
                                int max_waiting);
/* decision latency of SCHEDULE ("less than 0.1 milliseconds"): count, mean and max in ns */
MENOS_API int menos_sched_timing(menos_sched* s, long long* decisions, double* mean_ns, double* max_ns);

#ifdef __cplusplus
}
#endif
#endif /* MENOS_H_ */
