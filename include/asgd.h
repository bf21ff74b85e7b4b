/*
 * asgd.h -- C ABI of libasgd.so, the B200 (sm_100a) hot path of Adaptive SGD
 * (Ma, Rusu, Wu, Sim, "Adaptive Optimization for Sparse Data on Heterogeneous
 * GPUs", IPDPSW 2022).  "P:a-b" cites lines a..b of the paper's text
 * (/root/reference/PAPER.md); "Qn" cites a reading listed in DESIGN.md.
 *
 * Conventions (all entry points):
 *  - Every call returns int status: ASGD_OK (0) or one of ASGD_E_*.  The
 *    message of the last failure on the calling thread is asgd_last_error().
 *    No C++ exception crosses this boundary and the library never aborts.
 *  - Device pointers ("_dev" / documented as device) must be CUDA device
 *    memory of the ctx's device; host pointers ("_host") are host memory.
 *    Float/int arrays must be aligned to 16 bytes.
 *  - The CALLER owns all device memory (dataset, params, w, d, outputs and
 *    the workspace sized by asgd_workspace_bytes).  The library allocates only
 *    the host-side ctx / scheduler structs.
 *  - All device work is enqueued on the ctx's cudaStream_t (passed as void*);
 *    calls are asynchronous unless documented "synchronous".  Asynchronous
 *    CUDA / device-side errors are sticky: the next call on the ctx (or
 *    asgd_sync) reports them as ASGD_E_CUDA.
 *  - One ctx per GPU (per replica), driven by one thread at a time.  The
 *    host-pure functions (asgd_merge_weights, asgd_scale_batches,
 *    asgd_route_*, asgd_precision_at_k) are reentrant.
 *  - There is no CPU fallback: without an sm_100 device every device call
 *    fails with ASGD_E_CUDA / ASGD_E_UNSUPPORTED.
 *
 * Model (§V-A; D3): a 3-layer MLP  X (B x F, CSR) -> ReLU hidden
 * (H) -> softmax over L labels, cross-entropy loss with the uniform target
 * T_nj = 1/|Y_n| on the true labels (Q3), batch-mean reduction (Q4); or, with
 * loss = ASGD_LOSS_SIGMOID, per-label sigmoid binary cross-entropy with 0/1
 * targets summed over the L labels, batch mean (north_star "softmax/sigmoid
 * cross-entropy"; reading R11).  The
 * parameters are ONE flat fp32 vector of P = F*H + H + L*H + L entries, in
 * order W1 (F x H row-major, feature-major), b1 (H), W2 (L x H row-major,
 * label-major), b2 (L), so that one all-reduce covers the whole replica.
 */
#ifndef ASGD_H_
#define ASGD_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ASGD_OK 0
#define ASGD_E_ARG 1          /* null / misaligned pointer, bad scalar        */
#define ASGD_E_SHAPE 2        /* sizes inconsistent with the model / data     */
#define ASGD_E_CUDA 3         /* CUDA runtime / device-side error (sticky)    */
#define ASGD_E_STATE 4        /* call out of order (e.g. no data registered)  */
#define ASGD_E_UNSUPPORTED 5  /* configuration not supported by this build    */

/* Arithmetic of the dense output-layer contractions (Q28).
 * ASGD_PREC_FP32: fp32 CUDA-core FFMA contractions (tolerance 1e-4 vs fp64).
 * ASGD_PREC_BF16: tcgen05 tensor-core GEMMs, bf16 operands, fp32 accumulate
 *                 (tolerance 2e-2).  Master weights are fp32 in both. */
#define ASGD_PREC_FP32 0
#define ASGD_PREC_BF16 1

/* Output-layer loss (a5).
 * ASGD_LOSS_SOFTMAX: loss_n = lse(Z_n) - sum_j T_nj Z_nj, T_nj = 1/|Y_n| on Y_n;
 *                    dZ = (softmax(Z) - T) / B                      (Q3, Q4).
 * ASGD_LOSS_SIGMOID: loss_n = sum_j [softplus(Z_nj) - Y_nj Z_nj], Y_nj in {0,1};
 *                    dZ = (sigmoid(Z) - Y) / B                       (R11). */
#define ASGD_LOSS_SOFTMAX 0
#define ASGD_LOSS_SIGMOID 1

typedef struct asgd_ctx asgd_ctx;
typedef struct asgd_sched asgd_sched;

typedef struct {
  int64_t F;              /* input features                                 */
  int64_t L;              /* labels (output units)                          */
  int64_t H;              /* hidden units; one of 64, 128, 256, 512 (bf16:
                             <= 256, ASGD_E_UNSUPPORTED otherwise)          */
  int32_t precision;      /* ASGD_PREC_*                                    */
  int32_t b_max;          /* max rows of one local step (<= 2048)           */
  int64_t max_step_nnz;   /* max feature nnz of one step's rows             */
  int64_t max_step_labels;/* max label entries of one step's rows           */
  int32_t loss;           /* ASGD_LOSS_* (0 = softmax-CE, the paper's)      */
  int32_t reserved;       /* must be 0                                      */
} asgd_model_desc;

/* A CSR split: features (row_ptr, col, val) and labels (lab_ptr, lab).
 * row_ptr/lab_ptr: int64[n_rows+1], monotone, row_ptr[0] = lab_ptr[0] = 0;
 * col: int32[nnz] in [0, F), strictly increasing within a row; val: fp32[nnz];
 * lab: int32[n_lab] in [0, L), strictly increasing within a row, >= 1 label
 * per row (Table I; D1, D2). */
typedef struct {
  const int64_t* row_ptr;
  const int32_t* col;
  const float* val;
  const int64_t* lab_ptr;
  const int32_t* lab;
  int64_t n_rows;
  int64_t nnz;
  int64_t n_lab;
} asgd_csr;

/* ---------------------------------------------------------------- replica */

/* Bytes of device workspace one ctx needs for this model (>= 0; 0 = bad desc). */
size_t asgd_workspace_bytes(const asgd_model_desc* desc);

/* Create the replica context of one GPU (S2: the "GPU manager").
 * params: fp32[P] device, the replica w_i; w: fp32[P] device, the global
 * model; d: fp32[P] device, w - w_p (Q19: caller zero-fills before the first
 * merge).  ws: device workspace of ws_bytes >= asgd_workspace_bytes(desc).
 * stream: cudaStream_t (NULL = legacy default stream).  Synchronous.
 * Sets u = 0.  Errors: ASGD_E_ARG, ASGD_E_SHAPE, ASGD_E_UNSUPPORTED
 * (H not supported, device is not sm_100), ASGD_E_CUDA. */
int asgd_replica_init(asgd_ctx** out, const asgd_model_desc* desc, int device,
                      void* stream, float* params, float* w, float* d, void* ws,
                      size_t ws_bytes);

/* Free the host-side ctx (device memory belongs to the caller). */
int asgd_replica_destroy(asgd_ctx* ctx);

/* Switch the stream later calls enqueue on. */
int asgd_set_stream(asgd_ctx* ctx, void* stream);

/* The caller changed params outside the library (e.g. copied w into it at a
 * mega-batch start): refresh derived copies (bf16 shadow of W2).
 * Asynchronous. */
int asgd_params_changed(asgd_ctx* ctx);

/* Register the (device-resident, read-only) training split the local steps
 * index into.  Validates the CSR invariants once on the device (monotone
 * pointers, ids in range, strictly increasing within rows, >= 1 label per
 * row).  Synchronous.  ASGD_E_SHAPE if an invariant fails. */
int asgd_data_register(asgd_ctx* ctx, const asgd_csr* dev_csr);

/* Copy a HOST split (pinned memory for asynchronous copies) into caller-owned
 * device arrays dev_dst (same sizes) on the ctx stream and register it without
 * re-validation (the e2e path: host buffers -> device -> local steps).
 * Asynchronous. */
int asgd_data_upload(asgd_ctx* ctx, const asgd_csr* host_src, const asgd_csr* dev_dst);

/* asgd_data_upload in two halves, so that the next split's H2D copies overlap the current
 * split's local steps (the e2e path with two device staging buffers):
 *   asgd_data_stage: the copies host_src -> dev_dst (same sizes as asgd_data_upload) on
 *     `stream` (cudaStream_t, NULL = the ctx stream); nothing is registered.  The caller
 *     must not stage into a buffer that enqueued steps may still read.
 *   asgd_data_use: registers dev (its nnz / n_lab = the staged split's counts; no
 *     re-validation) for the steps enqueued after it; the ctx stream first waits for the
 *     copies last staged into that buffer.  Step graphs are cached per dataset (pointers
 *     and row count), so alternating buffers are not re-captured.
 * Both asynchronous; asgd_data_upload = stage on the ctx stream + use. */
int asgd_data_stage(asgd_ctx* ctx, const asgd_csr* host_src, const asgd_csr* dev_dst, void* stream);
int asgd_data_use(asgd_ctx* ctx, const asgd_csr* dev);

/* One local minibatch SGD step on the replica (A1; rows a2-a8 of
 * DESIGN.md §Path): rows_dev: int32[n_rows] device, sample ids of the batch
 * (a slice of the pass permutation, Q31), 1 <= n_rows <= b_max; lr: this
 * replica's learning rate lr_i.  Computes, all on the device:
 *   K-0 batch CSR view + touched-feature set (sorted unique cols, segments);
 *   K-1 A1 = X W1 + b1, H1 = ReLU(A1);   G1 Z = H1 W2^T + b2;
 *   softmax-CE: per-row lse, loss, dZ = (softmax(Z) - T)/B  (or, for
 *   ASGD_LOSS_SIGMOID, dZ = (sigmoid(Z) - Y)/B and the BCE row loss, fused
 *   into G1's epilogue on the bf16 path);
 *   G2 dH1 = dZ W2 (pre-step W2), dA1 = dH1 * [A1 > 0], b1 -= lr 1^T dA1;
 *   G3 W2 -= lr dZ^T H1, b2 -= lr 1^T dZ;
 *   K-5 W1[f,:] -= lr sum_{n: X_nf != 0} X_nf dA1[n,:] on touched f only.
 * loss_dev: nullable fp32 device scalar, receives the step's mean loss (Q33).
 * u += 1 (a truncated batch counts, Q9).  Asynchronous. */
int asgd_local_step(asgd_ctx* ctx, const int32_t* rows_dev, int32_t n_rows,
                    float lr, float* loss_dev);

/* Number of local steps since the last asgd_merge_finish (u_i). */
int asgd_updates(const asgd_ctx* ctx, int64_t* u_out);

/* Debug/parity: when grad_dev (fp32[P] device) is non-null, the next local
 * steps also write their full gradient there (zero outside touched W1 rows).
 * The fused kernels never materialise it otherwise.  NULL turns it off. */
int asgd_set_debug_grads(asgd_ctx* ctx, float* grad_dev);

/* Step trace (per-rank step log): with tracing on, every local step
 * records a pair of CUDA timing events around its enqueue on the ctx stream.
 *   asgd_trace_enable(ctx, 1): (re)starts the trace, its time origin is now.
 *   asgd_trace_read: synchronous; out: int64[4*cap] rows of (stream start of the
 *     step's batch -- the ticket's start in asgd_run_tickets / asgd_run_static, -1
 *     for a direct asgd_local_step --, rows, t0_ns, t1_ns) since the origin, in
 *     step order; *n_out = steps; clears the trace.  ASGD_E_SHAPE if cap is short.
 * The events add ~2 us of host work per step: leave tracing off for timing. */
int asgd_trace_enable(asgd_ctx* ctx, int32_t on);
int asgd_trace_read(asgd_ctx* ctx, int64_t* out_host, int64_t cap, int64_t* n_out);

/* Kernel timeline (diagnostic, process-wide, current device): with buf_dev non-null
 * every kernel of the library records, per kernel class k (TL_* order: touched, spmm,
 * g1, softmax, g2, dh, b1, g3, scatter, g1b, merge, other, then 8 in-kernel phase
 * marks ph0..ph7), buf_dev[3k] = min CTA arrival, buf_dev[3k+1] = min return from its
 * wait on the predecessor kernel, buf_dev[3k+2] = max CTA end (phase marks: only this
 * slot), as %globaltimer ns (uint64[60] device, caller-owned;
 * the caller fills the min slots with ~0 and the max slots with 0 before a step).
 * NULL turns it off.  ASGD_E_UNSUPPORTED unless libasgd was built with
 * -DASGD_TIMELINE (the probes are compiled out of the default build). */
int asgd_timeline_set(void* buf_dev);

/* Debug/parity: the sorted unique feature ids of the last local step
 * (touched W1 rows).  out_dev: int32[cap] device; *n_out_host = count.
 * Synchronous. ASGD_E_SHAPE if cap is too small. */
int asgd_last_touched(asgd_ctx* ctx, int32_t* out_dev, int64_t cap, int64_t* n_out_host);

/* ------------------------------------------------------------------ merge */

/* sum_k params[k]^2 in fp64 (deterministic order) for Alg. 2 line 4's
 * ||w_i||_2 / |w| (Q16).  out_dev: fp64 device scalar.  Asynchronous. */
int asgd_replica_sqnorm(asgd_ctx* ctx, double* out_dev);

/* Alg. 2 lines 1-7, host, pure.  u, b: int64[n]; nu: fp64[n]
 * norms per parameter ||w_i||_2 / P.  Ties: key (u_i, b_i), lowest index,
 * perturbation skipped when key(r) == key(s) (Q17); no renormalisation unless
 * flags has ASGD_MERGE_RENORM (Q18, Q34).  With ASGD_MERGE_NORM_UB line 3
 * becomes alpha_i = u_i b_i / sum_j u_j b_j ("normalize based on
 * the product between the number of updates and the batch size", reading
 * R12); line 2 is unchanged.  Other bits: ASGD_E_ARG.  alpha_out: fp64[n];
 * r_out, s_out, perturbed_out: nullable. */
#define ASGD_MERGE_RENORM 1   /* divide alpha by sum(alpha) after line 6    */
#define ASGD_MERGE_NORM_UB 2  /* line 3 normalises u_i * b_i (R12)          */
int asgd_merge_weights(int32_t n, const int64_t* u, const int64_t* b,
                       const double* nu, double pert_thr, double delta,
                       int32_t flags, double* alpha_out, int32_t* r_out,
                       int32_t* s_out, int32_t* perturbed_out);

/* Alg. 2 line 4's norm per parameter (reading Q16):
 * nu_i = sqrt(sqnorm_i) / P, fp64, from the squared norms asgd_replica_sqnorm
 * produced (all-gathered across ranks).  Host, pure.  sqnorm: fp64[n];
 * nu_out: fp64[n].  ASGD_E_ARG if n < 1, P < 1 or a sqnorm is negative/NaN. */
int asgd_norm_per_param(int32_t n, const double* sqnorm, int64_t P, double* nu_out);

/* Elastic SGD's merge weights (elastic model averaging; reading
 * R10): alpha_i = 1/N for the N = n replicas.  Host, pure.  alpha_out: fp64[n]. */
int asgd_elastic_weights(int32_t n, double* alpha_out);

/* params <- alpha * params (Alg. 2 line 8's alpha_i w_i, K-6).  Asynchronous.
 * After it the caller sums the prescaled replicas (one NCCL all-reduce SUM
 * over NVLink, or asgd_replicas_weighted_sum on one device). */
int asgd_merge_prescale(asgd_ctx* ctx, double alpha);

/* Alg. 2 lines 8-9 epilogue (K-7), params holding S = sum_i alpha_i w_i:
 * w' = S + gamma d;  d <- w' - w;  w <- w';  params <- w' (Q20, Q21);
 * refreshes derived copies; u <- 0.  Asynchronous. */
int asgd_merge_finish(asgd_ctx* ctx, float gamma);

/* Single-device stand-in for the all-reduce (simulated replicas):
 * out[k] = sum_i alpha_i * replicas[i][k] for k < P, alpha in fp64, summed in
 * replica order.  replicas_dev: device array of n device pointers.
 * Enqueued on ctx's stream. */
int asgd_replicas_weighted_sum(asgd_ctx* ctx, const float* const* replicas_dev,
                               const double* alpha_dev, int32_t n, float* out_dev);

/* Fused peer-memory merge (Alg. 2 lines 8-9 over NVLink
 * in one kernel instead of prescale + all-reduce + epilogue).  One process per
 * GPU, N <= 8 ranks on one node.
 *   asgd_peer_export: writes this replica's CUDA IPC handle (replica and
 *     workspace allocations) into out[ASGD_PEER_HANDLE_BYTES] (host).
 *   asgd_peer_open: maps the N ranks' handles (host array of
 *     N * ASGD_PEER_HANDLE_BYTES, in rank order; entry `rank` is ignored).
 *     Synchronous; call once after asgd_replica_init on every rank.
 *   asgd_merge_fused: rank r computes, for its shard of the parameters,
 *     S = sum_j alpha[j] w_j (fp64, j = 0..N-1) reading every replica over
 *     P2P, w' = S + gamma d, d <- w' - w, w <- w' on that shard, and stores w'
 *     into every replica; the stream then waits until all N ranks delivered
 *     their shards (system-scope counters).  alpha: host fp64[N] (Alg. 2 lines
 *     1-7, identical on all ranks).  The caller must ensure every rank
 *     finished its local steps first (the statistics all-gather does).  w and d
 *     are kept up to date on this rank's shard only.  u <- 0.  Asynchronous. */
#define ASGD_PEER_HANDLE_BYTES 160
int asgd_peer_export(asgd_ctx* ctx, void* out_host);
int asgd_peer_open(asgd_ctx* ctx, int32_t rank, int32_t world, const void* handles_host);
/* Close the peer mappings asgd_peer_open made (synchronises the ctx stream);
 * asgd_merge_fused then fails with ASGD_E_STATE until the next asgd_peer_open.
 * A rank that opened its peers but must fall back to the NCCL merge because
 * another rank could not calls this. */
int asgd_peer_close(asgd_ctx* ctx);
int asgd_merge_fused(asgd_ctx* ctx, const double* alpha_host, float gamma);

/* ---------------------------------------------------------------- scaling */

/* Alg. 1, host, pure, exact integers: increments
 * beta (u_i - mu~) = beta (N u_i - sum u)/N truncated toward zero (Q12); a
 * violated bound leaves b_i unchanged (Q13); lr_i = lr_max * b_i / b_max (Q14).
 * b_inout: int64[n]; lr_out: fp64[n] (nullable). */
int asgd_scale_batches(int32_t n, const int64_t* u, int64_t* b_inout,
                       double* lr_out, int64_t b_min, int64_t b_max,
                       int64_t beta, double lr_max);

/* Adaptive Alg. 1 frequency ("if stability is achieved or the system enters an
 * oscillatory state, the frequency at which scaling is performed can be [reduced]";
 * reading R17): after an Alg. 1 invocation moved b_before -> b_after (int64[n]), with
 * d_i = sign(b_after_i - b_before_i): when every d_i is 0 (stable) or some d_i is
 * opposite to rank i's previous non-zero move (oscillating), the interval to the next
 * invocation doubles up to max_interval, otherwise it returns to 1.  last_sign:
 * int32[n] in/out (the last non-zero move per rank, start at 0).  Host, pure. */
int asgd_scale_frequency(int32_t n, const int64_t* b_before, const int64_t* b_after,
                         int32_t* last_sign, int32_t interval, int32_t max_interval,
                         int32_t* interval_out);

/* -------------------------------------------------------------- routing */

/* Dynamic scheduler (S3): a ticket counter in POSIX
 * shared memory `shm_name` shared by the n_ranks processes of one node.
 * Rank 0 creates (create != 0), the others attach.  Each mega-batch holds M
 * samples (Q8). */
int asgd_sched_open(const char* shm_name, int32_t n_ranks, int64_t M,
                    int32_t create, asgd_sched** out);
/* Next batch for `rank` with batch size b_i: on success *start, *len are the
 * range [c, min(c + b_i, M)) of the mega-batch and the return is 1; 0 when
 * the mega-batch is exhausted (c >= M); < 0 on error (negated ASGD_E_*).
 * Lock-free (atomic fetch-add); appends (ticket, rank, start, len) to the log. */
int asgd_sched_next(asgd_sched* s, int32_t rank, int64_t b_i, int64_t* start,
                    int64_t* len);
/* Copy the log of the current mega-batch: out: int64[4*cap] rows of
 * (ticket, rank, start, len) in ticket order; *n_out = entries. */
int asgd_sched_log(asgd_sched* s, int64_t* out, int64_t cap, int64_t* n_out);
/* Start mega-batch `mb` (rank 0 only, after every rank is done with mb - 1):
 * cursor <- 0, then publishes mb (release). */
int asgd_sched_reset(asgd_sched* s, int64_t mb);
/* Block until mega-batch `mb` (or a later one) is published by
 * asgd_sched_reset, at most timeout_ms; ASGD_E_STATE on timeout. */
int asgd_sched_wait(asgd_sched* s, int64_t mb, int64_t timeout_ms);
int asgd_sched_close(asgd_sched* s, int32_t unlink_shm);

/* Rank `rank`'s share of the current mega-batch (the dynamic routing loop,
 * P:631-636, Fig. 2), run natively: until the scheduler is exhausted, take a
 * ticket [start, start + len) of b_i samples and enqueue
 * asgd_local_step(ctx, stream_rows_dev + start, len, lr, losses_dev + k) on the
 * ctx stream for the k-th ticket.  At most `inflight` (1..8) of the rank's
 * steps are outstanding when a ticket is taken: 1 = ask only when the previous
 * step finished (paper-faithful), 2 = ask while one step still runs (Q32).
 * stream_rows_dev: int32[M] device sample ids of the mega-batch (owned by the
 * caller); losses_dev: nullable fp32 device[losses_cap] (a step k >= losses_cap
 * gets no loss).  *n_steps = tickets taken (u_i of this mega-batch).  Returns
 * when the last step is enqueued (asynchronous); errors as asgd_local_step. */
int asgd_run_tickets(asgd_ctx* ctx, asgd_sched* s, int32_t rank, int64_t b_i,
                     const int32_t* stream_rows_dev, float lr, float* losses_dev,
                     int64_t losses_cap, int32_t inflight, int64_t* n_steps);

/* Elastic SGD's static schedule (elastic model averaging; SURVEY
 * NEXT-2): the mega-batch of M samples is cut into batches of b samples and
 * batch k goes to rank k mod world, so every rank processes the same number
 * of batches (+-1 when world does not divide the batch count, reading R10).
 * Enqueues this rank's steps exactly like asgd_run_tickets (same inflight,
 * losses and n_steps semantics), without the shared counter. */
int asgd_run_static(asgd_ctx* ctx, int32_t rank, int32_t world, int64_t b,
                    const int32_t* stream_rows_dev, int64_t M, float lr,
                    float* losses_dev, int64_t losses_cap, int32_t inflight,
                    int64_t* n_steps);

/* Replay (parity): ranks in ticket order -> routes (rank, start, len) with the
 * batch sizes b[rank] (host int64[n_ranks]), stopping at M.  out: int64[3*cap].
 * ASGD_E_ARG if an order entry is outside [0, n_ranks). */
int asgd_route_replay(int32_t n_ranks, int32_t n_tickets, const int32_t* order,
                      const int64_t* b, int64_t M, int64_t* out, int64_t cap,
                      int64_t* n_out);
/* Elastic SGD's static routes (R10): the M samples cut into
 * batches of b, batch k -> rank k mod n; out: int64[3*cap] (rank, start, len). */
int asgd_route_static(int32_t n, int64_t b, int64_t M, int64_t* out, int64_t cap, int64_t* n_out);

/* Simulated clock (Q10): every rank free at t = 0; the rank free first (ties:
 * lowest id) takes the next batch; it stays busy
 * cost_factor[r] * (nnz(batch) + per_row * len).  row_nnz: int64[M] nnz of the
 * mega-batch's samples in stream order.  out: int64[3*cap]. */
int asgd_route_simulate(int32_t n, const int64_t* b, int64_t M,
                        const double* cost_factor, double per_row,
                        const int64_t* row_nnz, int64_t* out, int64_t cap,
                        int64_t* n_out);

/* ------------------------------------------------------------- evaluate */

/* Top-k labels of the replica's model for test rows (a13):
 * rows_dev: int32[n] ids into test_dev (device CSR, validated on first use);
 * topk_dev: int32[n*k] device, per row the k highest-scoring labels, ties to
 * the lower id (Q23); 1 <= k <= 8.  Asynchronous.  Untimed. */
int asgd_eval_topk(asgd_ctx* ctx, const asgd_csr* test_dev, const int32_t* rows_dev,
                   int32_t n, int32_t k, int32_t* topk_dev);

/* Host, pure: hits = sum_n |topk_n[:k] cap Y_n| for P@k = hits / (k n). */
int asgd_precision_at_k(const int32_t* topk_host, const int64_t* lab_ptr,
                        const int32_t* lab, int32_t n, int32_t k, int64_t* hits_out);

/* --------------------------------------------------------------- misc */

/* Wait for the ctx's stream; report sticky asynchronous errors. */
int asgd_sync(asgd_ctx* ctx);

/* Number of kernels this ctx launched so far (for the bench's gpu_launches). */
int asgd_kernel_launches(const asgd_ctx* ctx, int64_t* out);

/* Live per-kernel timing with CUDA events recorded on the launching stream
 * around every launch of the kernel classes in class_mask (bit k = class k,
 * ASGD_PROF_ALL = all; 0 = off) -- for the bench's roofline.  Starting resets
 * the counters; asgd_profile_read is synchronous and returns per class the
 * summed milliseconds and the number of timed launches.  K-0 (class
 * ASGD_K_TOUCHED) runs on the ctx's internal side stream, overlapped with
 * K-1..G3, and is joined back before K-5. */
#define ASGD_PROF_ALL 0x3ff
#define ASGD_K_TOUCHED 0   /* K-0: batch scan, count, scan, place, segment sort */
#define ASGD_K_SPMM 1      /* K-1: X W1 + b1, ReLU                              */
#define ASGD_K_G1 2        /* Z = H1 W2^T + b2                                  */
#define ASGD_K_SOFTMAX 3   /* lse, loss, dZ                                     */
#define ASGD_K_G2 4        /* dH1 = dZ W2 (split-K)                             */
#define ASGD_K_DH 5        /* split-K reduce, ReLU', b1 update                  */
#define ASGD_K_B2 6        /* b2 update                                         */
#define ASGD_K_G3 7        /* W2 -= lr dZ^T H1                                  */
#define ASGD_K_SCATTER 8   /* K-5 scatter-SGD on touched W1 rows                */
#define ASGD_K_MERGE 9     /* K-6 / K-7: sqnorm, prescale, momentum epilogue    */
#define ASGD_PROF_N 10
int asgd_profile(asgd_ctx* ctx, int32_t class_mask);
int asgd_profile_read(asgd_ctx* ctx, double* ms_out, int64_t* count_out);

/* Async copy device -> host (pinned) on the ctx stream (e2e result read). */
int asgd_copy_to_host(asgd_ctx* ctx, void* dst_host, const void* src_dev, size_t bytes);

const char* asgd_last_error(void);

/* Build identification, e.g. "asgd sm_100a <git-ish>". */
const char* asgd_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ASGD_H_ */
