/*
 * occu.h — C ABI of the B200-native DNN-occu GNN hot path.
 *
 * The method (Mei et al., "GPU Occupancy Prediction of Deep Learning Models
 * Using Graph Neural Network"; PAPER.md = /root/reference/PAPER.md, "P<n>" =
 * its line n) maps a DL model's computation DAG (P49, P139) with Table I
 * node/edge features (P97-P133) to one GPU-occupancy scalar (P81, P85-P91):
 * ANEE message-passing rounds (P139-P151), a per-graph readout and an MLP head
 * (P125), trained with MSE (P209-P213) and Adam (P273).  Readings of garbled or
 * silent passages are DESIGN.md §3 R1-R22.
 *
 * Conventions (all entry points)
 *  - Every call returns an occu_status; no C++ exception crosses the ABI.  On a
 *    non-OK status nothing is written to caller outputs and occu_last_error()
 *    returns a message for that ctx (or the thread's last ctx-less error).
 *  - Ownership: the caller owns every input array and output buffer; the
 *    library borrows them for the duration of the call only.  The library owns
 *    weights, Adam state, workspace and the NCCL communicator (freed by
 *    occu_destroy).  occu_csr_batch objects are owned by the library and freed
 *    with occu_batch_free.
 *  - Memory space: feature/target/output pointers may be host or device
 *    (detected with cudaPointerGetAttributes); node_feat, edge_feat and out_occ
 *    of one call must be in the same space.  Host pointers => the call is
 *    synchronous.  Device pointers => the call is stream-ordered on the ctx
 *    stream and returns before completion.
 *  - Layout: row-major, little-endian float32, 16-byte aligned rows are NOT
 *    required (F_n = 80, F_e = 4 give 320 B / 16 B rows anyway).
 *  - Determinism: same inputs + same world size + same precision => bitwise
 *    identical outputs (no atomics on any reduction; fixed reduction orders).
 *  - Thread safety: one ctx per host thread.
 */
#ifndef OCCU_H_
#define OCCU_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define OCCU_ABI_VERSION 1

typedef struct occu_ctx occu_ctx;

typedef enum {
  OCCU_OK = 0,
  OCCU_EINVAL = 1,    /* bad argument: sizes, ids out of range, self-loop, config mismatch */
  OCCU_ENOMEM = 2,    /* host or device allocation failed */
  OCCU_ECUDA = 3,     /* CUDA runtime error (message in occu_last_error) */
  OCCU_EFORMAT = 4,   /* weights/state file malformed or checksum mismatch */
  OCCU_ENOTREADY = 5, /* weights not initialised / nothing computed yet */
  OCCU_ENCCL = 6      /* NCCL error */
} occu_status;

typedef enum { OCCU_AGGR_SUM = 0, OCCU_AGGR_MEAN = 1 } occu_aggr;            /* P149 Σ; MEAN option */
typedef enum { OCCU_MSG_CHANNEL_SOFTMAX = 0, OCCU_MSG_NEIGHBOR_SOFTMAX = 1 } occu_msg; /* R4 */
typedef enum { OCCU_FP32 = 0, OCCU_BF16 = 1 } occu_precision;

typedef enum { OCCU_READOUT_MEAN = 0, OCCU_READOUT_SET_DECODER = 1 } occu_readout;

/* Model configuration.  L ANEE rounds of width d (64, 128 or 256); d = 256 is the paper's
 * hidden width (P273) and runs on the CTA-pair tensor-core path: OCCU_FP32 or
 * OCCU_BF16 (BF16: F_e <= 16), msg = OCCU_MSG_CHANNEL_SOFTMAX, readout MEAN, graphormer = 0,
 * F_n <= 256, inference only (occu_train_step / occu_grads return OCCU_EINVAL; any other d,
 * or d = 256 with another mode, fails occu_create with OCCU_EINVAL).  Raw feature
 * widths F_n (node, Table I) and F_e (edge); head hidden width d_h; LeakyReLU slope (R7,
 * 0.01); F_n, F_e multiples of 4.  msg = OCCU_MSG_NEIGHBOR_SOFTMAX (reading B, NEXT-1):
 * kernel path 0; OCCU_FP32 forward + training, OCCU_BF16 forward (training with OCCU_BF16
 * returns OCCU_EINVAL: DESIGN.md R40).  readout: OCCU_READOUT_MEAN (a7, the north_star's segmented
 * mean; default when the trailing fields are zero) or OCCU_READOUT_SET_DECODER (P159-P205,
 * NEXT-2: Decoder(H) = FFN(SAB(PMA_k(H))) per graph, k seeds, `heads` attention heads, the
 * head reading the flattened k·d output; kernel path 0; training in OCCU_FP32 (R46;
 * with OCCU_BF16 training returns OCCU_EINVAL and inference runs the decoder in FP32 on the
 * BF16-stored h_L, R41);
 * k in [1, 8], heads in {1, 2, 4, 8}, k·heads <= 16.
 * graphormer: number of Graphormer layers (P153-P157, NEXT-3; R35-R37) between the
 * last ANEE round and the readout, h̄ = MHA(LN(h)) + h, h' = FFN(LN(h̄)) + h̄ with
 * self-attention over each graph's own node set, `heads` heads (d / heads in {16, 32, 64});
 * 0 = none (default).  Kernel path 0; training in OCCU_FP32 (R47); with OCCU_BF16 inference
 * runs the layers in FP32 on the BF16-stored h_L (R41) and training returns OCCU_EINVAL;
 * graphormer in [0, 4]. */
typedef struct {
  int32_t L, F_n, F_e, d, d_h;
  int32_t aggr;      /* occu_aggr */
  int32_t msg;       /* occu_msg */
  int32_t prec;      /* occu_precision */
  float slope;
  int32_t readout;   /* occu_readout */
  int32_t k, heads;  /* decoder seeds; decoder / Graphormer attention heads */
  int32_t graphormer; /* Graphormer layers (NEXT-3), 0 = none */
} occu_config;

/* One caller-owned input graph (host memory), local node ids. */
typedef struct {
  int32_t num_nodes;          /* >= 1 */
  int32_t num_edges;          /* >= 0 */
  const int32_t *src, *dst;   /* [num_edges], ids in [0, num_nodes), src != dst */
} occu_graph_view;

/* Packed batch.  Graphs concatenated in caller order; global
 * id = node_off[b] + local id; global input edge id = edge_off[b] + j.
 *   in-CSR : edges sorted by key (dst, src, eid); in_ptr[v] = #{edges with dst < v}
 *   out-CSR: edges sorted by key (src, dst, eid); out_pos[j] = in-CSR position
 *            of the j-th out-ordered edge; out_ptr[v] = #{edges with src < v}
 * All int32.  on_device = 0: host arrays (occu_pack); 1: device arrays
 * (occu_batch_to_device).  Library-owned; free with occu_batch_free. */
typedef struct {
  int32_t num_graphs, num_nodes, num_edges;
  int32_t *node_off, *edge_off;           /* [B+1] */
  int32_t *in_ptr;                        /* [N+1] */
  int32_t *in_src, *in_dst, *in_eid;      /* [E]   */
  int32_t *out_ptr;                       /* [N+1] */
  int32_t *out_pos;                       /* [E]   */
  int32_t *node_graph;                    /* [N]   */
  int32_t on_device;
  int32_t max_in_degree;                  /* max_v (in_ptr[v+1] - in_ptr[v]); -1 = unknown.  Set
                                             by occu_pack / occu_synthesize, kept by
                                             occu_batch_to_device; selects the aggregation's
                                             hub path (in-degree > 256, see occu_predict) */
  void *priv;                             /* library-private (device schedule) */
} occu_csr_batch;

/* Training batch: packed CSR + features (same conventions as occu_predict);
 * global_num_graphs = B summed over all DP ranks (loss scale 1/B_glob, R15). */
typedef struct {
  const occu_csr_batch *csr;
  const float *node_feat;     /* [N][F_n] graph-concatenated order */
  const float *edge_feat;     /* [E][F_e] graph-concatenated INPUT edge order */
  int32_t global_num_graphs;
} occu_batch;

/* ---- lifecycle ------------------------------------------------------------ */
/* Create a context on CUDA device `cuda_device`, launching on `cuda_stream`
 * (a cudaStream_t; NULL = the legacy default stream).  Validates cfg. */
occu_status occu_create(occu_ctx **out, const occu_config *cfg, int cuda_device, void *cuda_stream);
occu_status occu_destroy(occu_ctx *ctx);
/* Rebind the launch stream (e.g. torch's current stream). */
occu_status occu_set_stream(occu_ctx *ctx, void *cuda_stream);
size_t occu_num_params(const occu_config *cfg);

/* ---- weights (SURVEY §8(b) file format "OCCUW001") ------------------------ */
/* Deterministic init: element j of the flat parameter vector (file order) =
 * float((2u_j - 1) / sqrt(fan_in)), u_j = splitmix64 uniform #j for seed (R21). */
occu_status occu_init_weights(occu_ctx *ctx, uint64_t seed);
occu_status occu_load_weights(occu_ctx *ctx, const char *path);    /* EFORMAT on mismatch */
occu_status occu_save_weights(const occu_ctx *ctx, const char *path);
/* Flat float32 parameter vector in file order, host memory, n = occu_num_params. */
occu_status occu_set_params(occu_ctx *ctx, const float *host_flat, size_t n);
occu_status occu_get_params(const occu_ctx *ctx, float *host_flat, size_t n);

/* ---- packing (host, C++; a0) ---------------------------------------------- */
/* EINVAL: num_graphs < 1, num_nodes < 1, id out of range, self-loop,
 * N or E >= 2^31.  Acyclicity is not checked (the math is a fixed number of
 * rounds).  Threaded over graphs; output is bit-identical to oracle.pack. */
occu_status occu_pack(const occu_graph_view *graphs, int32_t num_graphs, occu_csr_batch **out);
/* Device copy (+ kernel schedule) of a host batch, on the ctx stream. */
occu_status occu_batch_to_device(occu_ctx *ctx, const occu_csr_batch *host, occu_csr_batch **dev_out);
void occu_batch_free(occu_csr_batch *b);

/* ---- forward (P139-P151, P125) -------------------------------------------- */
/* out_occ[B] <- ŷ for each graph.  csr_batch host or device. */
occu_status occu_predict(occu_ctx *ctx, const occu_csr_batch *csr_batch,
                         const float *node_feat, const float *edge_feat, float *out_occ);

/* Pipelined variant for a stream of host batches: returns at once.  The batch's CSR and
 * features are copied on an internal copy stream into one of two device staging slots while
 * the previous batch still computes on the ctx stream; the forward waits for its copy, and
 * out_occ (host, pinned for overlap) is written by an async D2H on the ctx stream.  The call
 * blocks only until the previous call's copy has landed, so the caller keeps csr_batch,
 * node_feat and edge_feat alive and unmodified until the next occu_predict_async (or
 * occu_wait) returns, and reads out_occ after occu_wait.  EINVAL for device pointers or a device
 * batch (use occu_predict, which is already stream-ordered for those). */
occu_status occu_predict_async(occu_ctx *ctx, const occu_csr_batch *csr_batch,
                               const float *node_feat, const float *edge_feat, float *out_occ);
/* Blocks until every occu_predict_async / occu_train_step_async issued on ctx has completed. */
occu_status occu_wait(occu_ctx *ctx);

/* ---- training (P209-P213, P273) ------------------------------------------- */
/* Forward with saved activations, MSE loss scaled by 1/global_num_graphs,
 * backward, NCCL allreduce of the flat gradient (if occu_dist_init was
 * called), Adam(lr, wd = 1e-4, β = (0.9, 0.999), ε = 1e-8).  targets[B] in
 * the features' memory space; out_loss (nullable, host) = global mean loss. */
occu_status occu_train_step(occu_ctx *ctx, const occu_batch *batch, const float *targets,
                            float lr, float *out_loss);
/* Pipelined occu_train_step: a HOST batch (occu_pack) with pinned host features / targets;
 * the copies run on a copy stream into one of two staging slots and the step is enqueued on
 * the ctx stream behind them, so the host can pack the next batch and its copies overlap this
 * step.  Blocks only until the previous call's copies have landed: keep batch, features and
 * targets alive and unmodified until the next occu_train_step_async (or occu_wait) returns.
 * out_loss (nullable, pinned host float) receives the global mean loss — read it after
 * occu_wait.  Same arithmetic as occu_train_step (bitwise-identical parameters). */
occu_status occu_train_step_async(occu_ctx *ctx, const occu_batch *batch, const float *targets,
                                  float lr, float *out_loss);
/* Forward + backward only (no allreduce, no Adam): grads left in the ctx. */
occu_status occu_compute_grads(occu_ctx *ctx, const occu_batch *batch, const float *targets,
                               float *out_loss);
occu_status occu_get_grads(const occu_ctx *ctx, float *host_flat, size_t n);
occu_status occu_set_weight_decay(occu_ctx *ctx, float wd);

/* ---- NEXT-4: on-device feature synthesis (R39) ---------
 * A DL-model family's training DAG has one topology for all its hyperparameter variants
 * (P237), so a batch of variants is built on the GPU from per-family templates plus four
 * numbers per graph, instead of copying ~350 B of Table I features per node over PCIe.
 * occu_template_create uploads one family (device memory of ctx's device, owned by the
 * template): graph = the family's DAG (host, local ids; validated like occu_pack);
 * node_static [n][80] = the hyperparameter-independent Table I columns (operator one-hot, role
 * bits, runtime GPU constants; zeros in columns 42-75); node_coef [n][22][12] = the 22
 * hyperparameter-dependent quantities of each node (16 operator hyperparameters -> columns
 * 42-57, 4 tensor sizes -> 66-69 and, times 4 bytes, 70-73, FLOPs -> 74, temporary size -> 75)
 * as tensor-product Newton coefficients on the nodes batch {4, 8}, cin {1, 2}, seq {16, 32, 48}
 * (coefficient 6i + 3j + k of Nb_i Nc_j Ns_k, Nb = (1, b-4), Nc = (1, c-1),
 * Ns = (1, s-16, (s-16)(s-32)); occu_gen/templates.py builds them); edge_static [m][4] (column
 * 2 zero) and edge_coef [m][12] (bytes carried -> column 2), both in input edge order.
 * occu_synthesize builds a device batch of num_graphs graphs, graph b = templates[b] at
 * hp[b] = (batch, cin, seq, hw) (host [B][4], finite, >= 0): the CSR (bit-identical to
 * occu_pack of the same graphs), node_feat [N][80] and edge_feat [E][4] (input edge order),
 * each quantity evaluated in float64 and encoded log2(1 + x) / 40 (configuration columns
 * 58-61 = the encoded hp, 62-65 = 0).  Stream-ordered on the ctx stream.  The returned arrays
 * live in ctx-owned device memory, valid until the next occu_synthesize on ctx; free the
 * returned batch struct with occu_batch_free (it does not free the arrays).  Errors:
 * OCCU_EINVAL (NULL, num_graphs < 1, a template of another device, bad hp, F_n != 80 or
 * F_e != 4 in the ctx config, N or E >= 2^31), OCCU_ENOMEM, OCCU_ECUDA. */
typedef struct occu_template occu_template;
occu_status occu_template_create(occu_ctx *ctx, const occu_graph_view *graph,
                                 const float *node_static, const double *node_coef,
                                 const float *edge_static, const double *edge_coef,
                                 occu_template **out);
void occu_template_destroy(occu_template *t);
occu_status occu_synthesize(occu_ctx *ctx, const occu_template *const *templates,
                            int32_t num_graphs, const float *hp, occu_csr_batch **csr_out,
                            float **node_feat, float **edge_feat);

/* ---- NEXT-4 consumer: occu-packing (P390-P392; R38) ------------------
 * Host-side first-fit bin packing of jobs by predicted occupancy (the output of
 * occu_predict), the paper's co-location policy: "the cumulative GPU occupancy of the DL
 * load not exceeding 100%" (P392).  Jobs are taken in array order; job j goes to the
 * lowest-numbered GPU slot b with load_b + occ_j <= capacity (float64, occ widened from
 * float32, predictions < 0 counted as 0), else a new slot opens (a job larger than the
 * capacity gets a slot of its own).  occ: host [num_jobs]; slot_of_job: host [num_jobs]
 * (caller-allocated, written); slot_load: nullable host [num_jobs] (the first *num_slots
 * entries are written); *num_slots = slots opened.  O(num_jobs log num_jobs).  Errors:
 * OCCU_EINVAL for NULL pointers, num_jobs < 0, capacity not finite and > 0, or a NaN / Inf
 * prediction (message via occu_last_error(NULL)); nothing is written then. */
occu_status occu_pack_jobs(const float *occ, int32_t num_jobs, double capacity,
                           int32_t *slot_of_job, double *slot_load, int32_t *num_slots);

/* ---- data parallel (north_star: NCCL gradient allreduce over NVLink) ------ */
/* One process per GPU.  occu_nccl_unique_id: rank 0 creates the 128-byte id, the caller
 * broadcasts it (e.g. torch.distributed); every rank then calls occu_dist_init with its rank and
 * the world size (world >= 1; world = 1 runs the same NCCL data plane on one GPU).  The
 * communicator is created non-blocking; occu_train_step then sums the flat gradient (+ the
 * loss) with ncclAllReduce over NVLink on the ctx stream before Adam, so every rank applies the
 * same update (replicas stay bitwise equal).  Errors: OCCU_EINVAL (NULL, bad rank / world),
 * OCCU_ENCCL (NCCL failure, or no progress within the timeout: the communicator is then
 * aborted with ncclCommAbort and every later collective call fails with OCCU_ENCCL until
 * occu_dist_init is called again). */
occu_status occu_nccl_unique_id(void *out_128_bytes);
occu_status occu_dist_init(occu_ctx *ctx, int rank, int world, const void *nccl_unique_id);
/* Watchdog timeout in seconds for communicator setup and for every blocking wait on a step that
 * contains a collective (default 600; 0 disables).  OCCU_EINVAL if seconds < 0. */
occu_status occu_dist_set_timeout(occu_ctx *ctx, double seconds);
/* Abort the communicator (ncclCommAbort), e.g. from a host watchdog after a peer died; safe to
 * call from another host thread while a step is waiting. */
occu_status occu_dist_abort(occu_ctx *ctx);
/* Wait (host) until everything enqueued on the ctx stream has completed, polling NCCL for
 * asynchronous errors; OCCU_ENCCL + abort on error or timeout. */
occu_status occu_dist_sync(occu_ctx *ctx);

/* ---- optimizer state (Adam m, v, t) --------------------------------------- */
occu_status occu_save_state(const occu_ctx *ctx, const char *path);
occu_status occu_load_state(occu_ctx *ctx, const char *path);

/* ---- introspection for parity tests --------------------------------------- */
typedef enum {
  OCCU_T_HBAR = 0,   /* [N][d]  layer l */
  OCCU_T_P = 1,      /* [N]     layer l */
  OCCU_T_Q = 2,      /* [N]     layer l */
  OCCU_T_E = 3,      /* [E][d]  layer l, in-CSR edge order */
  OCCU_T_H = 4,      /* [N][d]  layer l */
  OCCU_T_R = 5,      /* [B][d]  readout ([B][k·d] flattened decoder output with the decoder) */
  OCCU_T_YHAT = 6,   /* [B] */
  OCCU_T_GPH = 7     /* [N][d]  output of Graphormer layer l (NEXT-3) */
} occu_tensor;
/* Kernel path: 0 (default) = tcgen05 tensor cores (fp16x2-split GEMMs with
 * per-row power-of-two scaling, FP32 accumulation in TMEM) + CUDA-core
 * gather/segmented sum; 2 = as 0 with the gate, message and segmented sum fused
 * into one tensor-core kernel; 1 = CUDA-core FP32 (SIMT) everywhere.  All meet
 * the FP32 tolerance. */
occu_status occu_set_kernel_path(occu_ctx *ctx, int path);
/* Single-CTA forward for tiny batches (CFG1: <= 64 nodes, <= 128 edges, OCCU_FP32, reading
 * A, mean readout, shared-memory budget permitting; kernels_small.cu): the whole inference
 * forward in one launch with every activation in shared memory.  On by default (enable = 0
 * turns it off): on a B200 it takes 40 us for CFG1 against 45 us for the regular
 * 9-kernel path (both 39 us replayed from a CUDA graph), see DESIGN.md.  Per-layer tensors
 * are then not stored (occu_get_tensor returns OCCU_ENOTREADY for them unless
 * occu_set_keep_intermediates is set, which selects the regular path); training never uses it. */
occu_status occu_set_small_batch_kernel(occu_ctx *ctx, int enable);
/* Keep every intermediate of the next forward (costs memory/bandwidth).  Without
 * it, the last layer's e and (kernel path 0) h are not stored: path 0 folds the
 * readout's node sums into the last aggregation, and occu_get_tensor returns
 * OCCU_ENOTREADY for them. */
occu_status occu_set_keep_intermediates(occu_ctx *ctx, int keep);
/* Copy an intermediate of the last forward into host memory (float32; BF16
 * precision stores are widened).  bytes must equal the tensor size. */
occu_status occu_get_tensor(occu_ctx *ctx, int32_t which, int32_t layer, void *host_dst, size_t bytes);
/* Test hook for the weight-gradient GEMM of the backward (SURVEY §8(c) step BW: dW_m = DVᵀE',
 * dW_e = DZᵀE_in, dW_u = dPᵀH_in): out[a][b] = Σ_{r<R} X[r][a]·Y[r][b] with the library's own
 * kernels (deterministic split-K, fixed-order reduction), exactly as occu_train_step calls them.
 * X: device FP32 [R][A]; Y: device [R][Bn], FP32, or BF16 when y_bf16 != 0 (OCCU_BF16
 * training's stored activations; then A, Bn in {32..128}, multiples of 32 / 16); out: device
 * FP32 [A][Bn].  Stream-ordered on the ctx stream.  EINVAL on NULL pointers or unsupported
 * shapes; the ctx needs no weights. */
occu_status occu_test_wgrad(occu_ctx *ctx, const float *X, int32_t A, const void *Y, int32_t Bn,
                            int64_t R, int32_t y_bf16, float *out);
/* Number of kernel launches issued by the last predict/train call. */
int64_t occu_last_launch_count(const occu_ctx *ctx);

/* ---- per-kernel timing (CUDA events recorded on the ctx stream) ---------- */
/* enable != 0: every kernel launch is bracketed by a pair of cudaEvents on the
 * launch stream; occu_profile_query(idx) returns the idx-th kernel name, the
 * summed device time (ms) and the launch count since the last reset
 * (synchronises the stream).  EINVAL when idx is out of range. */
occu_status occu_set_profiling(occu_ctx *ctx, int enable);
occu_status occu_profile_reset(occu_ctx *ctx);
occu_status occu_profile_query(occu_ctx *ctx, int32_t idx, const char **name, double *total_ms,
                               int64_t *launches);

const char *occu_last_error(const occu_ctx *ctx);

#ifdef __cplusplus
}
#endif
#endif /* OCCU_H_ */
