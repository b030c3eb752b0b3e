/*
 * astra.h — C ABI of the B200-native Astra custom-RNN training hot path.
 *
 * What the library computes.  One training step — forward and backward through time — of a
 * long-tail recurrent cell that cuDNN does not cover ("MI-LSTM [36], LSTM with
 * Attention [35], SC-RNN [22], RHN [39]"), plus the online, work-conserving variant
 * exploration that picks how that step runs (§4).  Because every mini-batch
 * runs the same computation on the same shapes, the library measures candidate
 * variants on real steps with cudaEvent pairs, indexes the timings under mangled
 * keys and keeps the fastest.  All variants are value-preserving
 * (P:447): they produce bitwise-identical numbers within one precision path.
 *
 * Cell equations are readings of the cited works (the paper only cites them); they are
 * written out in DESIGN.md "Readings" and in the fp64 oracle (oracle/cells.py).
 *
 * Conventions (every entry point):
 *   - Layouts are time-major and row-major: x [T][B][I], y [T][B][Hout], states [B][H].
 *   - Row-vector maths, y = x·W with W stored [in][out]; gate blocks in (i, f, g, o) order.
 *   - Parameters and gradients are ONE flat fp32 vector each, laid out as astra_param_info
 *     reports (each tensor row-major at its offset).
 *   - Precision paths: ASTRA_BF16 — bf16 GEMM operands (x, y, dy, dx are bf16), fp32
 *     accumulate, fp32 states, saved projections, master weights and gradients;
 *     ASTRA_FP32 — everything fp32 (the parity path).
 *   - Memory: the CALLER allocates all device memory (params, grads, workspace, I/O).  The
 *     library owns only its host handle, tuner state, CUDA events, and the NCCL communicator.
 *     `saved` must stay untouched between astra_step_fwd and the matching astra_step_bwd.
 *   - Pointers marked "device" are CUDA device pointers on the handle's device; "host" are
 *     host pointers.  No torch type appears anywhere in this ABI.
 *   - Errors: every call returns astra_status.  Argument/state errors are detected before any
 *     side effect.  CUDA faults are sticky and surface as ASTRA_E_CUDA; NCCL failures as
 *     ASTRA_E_NCCL.  astra_last_error() returns a thread-local detail string.  The library
 *     never aborts the process.
 *   - Threading: one handle per host thread at a time.  All work is asynchronous on the
 *     streams given by astra_set_streams (default: the legacy default stream).
 */
#ifndef ASTRA_H_
#define ASTRA_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct astra_cell_s* astra_cell;
typedef struct astra_lm_s* astra_lm;
typedef int astra_status;
typedef void* astra_stream;  /* a cudaStream_t */

enum astra_cell_type {
  ASTRA_LSTM = 0,       /* textbook LSTM (reduction base; PAPER P:352 stacked LSTM)        */
  ASTRA_MILSTM = 1,     /* multiplicative-integration LSTM [36]           */
  ASTRA_SCRNN = 2,      /* structurally-constrained RNN [22]              */
  ASTRA_RHN = 3,        /* recurrent highway network [39], coupled carry             */
  ASTRA_LSTM_ATTN = 4,  /* LSTM encoder + attentive LSTM decoder, reduced GNMT [35] */
  ASTRA_SUBLSTM = 5     /* subtractive LSTM [8]                                 */
};
enum astra_dtype { ASTRA_BF16 = 0, ASTRA_FP32 = 1 };
enum astra_status_code {
  ASTRA_OK = 0,
  ASTRA_E_ARG = 1,
  ASTRA_E_UNSUPPORTED = 2,
  ASTRA_E_STATE = 3,
  ASTRA_E_CUDA = 4,
  ASTRA_E_NCCL = 5,
  ASTRA_E_WORKSPACE = 6
};
enum astra_tune { ASTRA_TUNE_OFF = 0, ASTRA_TUNE_ON = 1, ASTRA_TUNE_FROZEN = 2 };
enum astra_tune_state { ASTRA_TUNE_IDLE = 0, ASTRA_TUNE_EXPLORING = 1, ASTRA_TUNE_CONVERGED = 2 };

/* Full description of a cell.  Zero-valued optional fields take the defaults shown. */
typedef struct {
  int cell_type;     /* enum astra_cell_type                                      */
  int hidden;        /* H > 0                                                      */
  int input;         /* I > 0                                                      */
  int batch;         /* B > 0 (per rank)                                           */
  int seq;           /* T > 0 (decoder length Tt for ASTRA_LSTM_ATTN)              */
  int dtype;         /* enum astra_dtype                                           */
  int device;        /* CUDA device ordinal                                        */
  int depth;         /* RHN recurrence depth L (default 10)                        */
  int context;       /* SCRN context size S (default H)                            */
  float scrn_alpha;  /* SCRN fixed context decay α (default 0.95; reading R5)      */
  int src_seq;       /* attention source length Ts (default = seq)                 */
  int attn_dim;      /* attention size A (default = H)                             */
} astra_cell_desc;

/* ---- lifetime ------------------------------------------------------------------------- */
/* North-star signature: bf16 path, all optional fields at their defaults.                   */
astra_status astra_cell_create(astra_cell* out, int cell_type, int hidden, int input, int batch, int seq);
astra_status astra_cell_create_ex(astra_cell* out, const astra_cell_desc* d);
astra_status astra_cell_destroy(astra_cell c);

/* ---- parameters and workspace --------------------------------------------------------- */
/* Length (in fp32 elements) of the flat parameter (= gradient) vector.                      */
astra_status astra_param_count(astra_cell c, size_t* n_params);
/* Tensor idx (0-based): its name (static string), element offset in the flat vector and
 * its 2-D shape (vectors: rows = 1).  Returns ASTRA_E_ARG past the last tensor.            */
astra_status astra_param_info(astra_cell c, int idx, const char** name, size_t* offset, int* rows, int* cols);
/* Device bytes the caller must provide: `saved` (live from step_fwd to step_bwd) and
 * `scratch` (may be reused between calls).  Maximum over every enumerated variant.          */
astra_status astra_workspace_size(astra_cell c, size_t* saved_bytes, size_t* scratch_bytes);
/* Attach caller memory (all device, 256-byte aligned).  params/grads: flat fp32 vectors.    */
astra_status astra_bind(astra_cell c, float* params, float* grads, void* saved, void* scratch);
/* Streams: `main` carries the step; `side` (optional, n_side ≥ 0) and `comm` (optional,
 * may be NULL) enable stream-assignment variants and overlapped gradient sync.              */
astra_status astra_set_streams(astra_cell c, astra_stream main, const astra_stream* side, int n_side, astra_stream comm);

/* ---- one training step ------------------------------------------------------------------ */
/* Forward through time.  x: device [T][B][I] (bf16 or fp32 by path; attention: xe [Ts][B][I]
 * followed contiguously by xd [T][B][I]); h0, c0: device fp32 [B][H] (SCRN: c0 carries s0
 * [B][S]; RHN ignores c0; NULL = zeros); y: device [T][B][Hout] (Hout = H; SCRN H+S;
 * attention 2H); hT, cT: device fp32 [B][H] final states (may be NULL).                    */
astra_status astra_step_fwd(astra_cell c, const void* x, const float* h0, const float* c0,
                            void* y, float* hT, float* cT);
/* Backward through time of L = Σ dy⊙y + Σ dhT⊙hT + Σ dcT⊙cT for the LAST step_fwd.
 * dy: device like y; dhT, dcT: device fp32 (NULL = zeros).  OVERWRITES grads (no
 * accumulation); dx: device like x (may be NULL); dh0, dc0: device fp32 (may be NULL).
 * If astra_comm_init was called with world > 1, the gradient sum over ranks is launched on
 * the comm stream and joined before the call's work completes on `main`.                    */
astra_status astra_step_bwd(astra_cell c, const void* dy, const float* dhT, const float* dcT,
                            void* dx, float* dh0, float* dc0);
/* Plain SGD on the bound params, θ ← θ − lr·g (reading R15).                    */
astra_status astra_sgd(astra_cell c, float lr);

/* ---- the online tuner (PAPER §4.3-§4.7) -------------------------------------- */
/* Call once per step after step_bwd.  Harvests the previous steps' event pairs without
 * blocking (cudaEventQuery), updates the profile index, iterates the update tree and binds
 * the next variant.  *state ← enum astra_tune_state.                                        */
astra_status astra_tune_next(astra_cell c, int* state);
/* mode: ASTRA_TUNE_OFF (default variant), ASTRA_TUNE_ON (explore), ASTRA_TUNE_FROZEN
 * (use `forced_variant`, a string from astra_tune_report's "variant" field, or the best
 * found so far when NULL).                                                                  */
astra_status astra_tune_mode(astra_cell c, int mode, const char* forced_variant);
/* Region events (cudaEvent pairs around the step phases).  on = 1 (default): the
 * always-on level — the step region every step, the phase regions (a1, chains, head, SE4,
 * dU / dW / dX) only while the tuner explores or races; on = 2: the phase regions every step
 * (diagnostics: astra_region_times); on = 0: none.  The tuner harvests them, so on = 0 is refused
 * with E_STATE while the mode is ASTRA_TUNE_ON; off is for measuring the profiling overhead
 * (< 0.5 %).  Other values: E_ARG.                                                   */
astra_status astra_set_profiling(astra_cell c, int on);
/* JSON report (current variant, #configs explored, index size, trials).  Writes at most
 * len bytes including the NUL; *needed ← required length.                                  */
astra_status astra_tune_report(astra_cell c, char* buf, size_t len, size_t* needed);

/* ---- data parallelism -------------------------------------------------- */
/* nccl_unique_id: host pointer to the 128-byte ncclUniqueId broadcast by the caller.       */
astra_status astra_comm_init(astra_cell c, const void* nccl_unique_id, int rank, int world);
/* The same for an LM: ONE communicator shared by every layer of the (stacked) LM, so the head,
 * embedding and every layer's buckets are reduced.  A world > 1 LM step whose layers lack a
 * common communicator (NCCL or K11p) fails with ASTRA_E_STATE instead of silently diverging.   */
astra_status astra_lm_comm_init(astra_lm m, const void* nccl_unique_id, int rank, int world);
/* Write a fresh ncclUniqueId (128 bytes) to host memory `out` (call on rank 0).           */
astra_status astra_comm_unique_id(void* out, size_t len);

/* Deterministic peer-memory backend (K11p; SURVEY §8(e) "backend 2", the semantics of §8(c.3)
 * item 8: g = (1/N)·Σ_r g_r over contiguous batch shards).  Replaces the NCCL gradient all-reduce
 * and the SGD of a world > 1 step by kernels that work directly on every rank's memory over
 * NVLink / NVSwitch (CUDA IPC mappings):
 *   - each gradient bucket [off, off+n) is cut into `world` contiguous shards (boundaries rounded
 *     to 4 floats); rank r sums shard r of all ranks' gradients in rank order 0..N-1, scales by
 *     1/N and stores it into its OWN gradients.  The sum is bitwise independent of bucketing and
 *     timing, and identical on every N-rank run;
 *   - SGD updates the owned shards (θ − lr·g, the rounding of astra_sgd) and stores the new values
 *     into every rank's parameters (the all-gather), so all ranks hold identical parameters.
 * After a step_bwd / lm_train_step the gradients hold the global mean only on this rank's owned
 * shards (other elements: this rank's shard-mean gradient).
 * Protocol: after bind, each rank calls *_comm_peer_handle (ASTRA_PEER_HANDLE_BYTES of host
 * memory out), the caller all-gathers the handles over its process group (rank order), then each
 * rank calls *_comm_peer_init with the world × ASTRA_PEER_HANDLE_BYTES array.  The params/grads
 * vectors must be cudaMalloc memory (torch's default allocator is) and must not be rebound.  Up
 * to 8 ranks; ranks may share one device (tests).  Every rank must issue the same sequence of
 * steps.  Exploration (ASTRA_TUNE_ON) with world > 1 also needs astra_comm_init (the tuner's
 * cross-rank max, reading R29).  A rank that waits more than ASTRA_PEER_TIMEOUT_S (default 60)
 * seconds for a peer traps the device (sticky ASTRA_E_CUDA), it never hangs.
 * The library owns the IPC mappings and a 4 KB signal array per rank.                         */
#define ASTRA_PEER_HANDLE_BYTES 256
astra_status astra_comm_peer_handle(astra_cell c, void* out, size_t len);
astra_status astra_comm_peer_init(astra_cell c, const void* handles, int rank, int world);
/* The same for an LM: the window is the LM's flat params / grads; every layer uses it.         */
astra_status astra_lm_comm_peer_handle(astra_lm m, void* out, size_t len);
astra_status astra_lm_comm_peer_init(astra_lm m, const void* handles, int rank, int world);

/* ---- language-model wrapper (embedding → cell → linear head → mean CE) ----------------- */
/* Adds E [V][I], W_o [Hout][V], b_o [V] after the cell's parameters in one flat vector.    */
astra_status astra_lm_create(astra_lm* out, astra_cell c, int vocab);
/* Stacked LM (the paper's PTB stacked LSTM, Table 5): cells[0] is
 * the bottom layer (fed by the embedding), cells[n-1] the top (read by the head); layer l+1's
 * input size must equal layer l's output size, all layers share batch, seq and dtype, and outputs
 * must be single-segment (LSTM family, RHN; not SCRN).  Parameters: each layer's block with its
 * names prefixed "L<l>.", then E, W_o, b_o.  The cells stay owned by the caller and must outlive
 * the LM; astra_lm_set_state takes the layers' states concatenated in layer order.  Each cell
 * keeps its own tuner (call astra_tune_next on every layer after a step).  E_ARG on a shape
 * mismatch, E_UNSUPPORTED for a cell type without an LM form.                                 */
astra_status astra_lm_create_stacked(astra_lm* out, const astra_cell* cells, int n_layers, int vocab);
astra_status astra_lm_destroy(astra_lm m);
astra_status astra_lm_param_count(astra_lm m, size_t* n_params);
astra_status astra_lm_param_info(astra_lm m, int idx, const char** name, size_t* offset, int* rows, int* cols);
astra_status astra_lm_workspace_size(astra_lm m, size_t* bytes);
/* params/grads: device flat fp32 [lm_param_count]; workspace: device [lm_workspace_size].  */
astra_status astra_lm_bind(astra_lm m, float* params, float* grads, void* workspace);
/* Recurrent state carried across steps (truncated BPTT; reading R13).  h, c: device fp32
 * [B][H] (c: SCRN [B][S]; ignored for RHN); NULL = zeros.                                   */
astra_status astra_lm_set_state(astra_lm m, const float* h, const float* c);
/* One full training step: tokens device int32 [T+1][B]; forward, loss, backward, gradient
 * sync (world > 1), SGD with learning rate lr.  loss_dev: device fp32 scalar (mean CE of
 * this rank's shard) or NULL.  Gradients of the step stay in the bound grads vector.       */
astra_status astra_lm_train_step(astra_lm m, const int32_t* tokens, float lr, float* loss_dev);
/* Same step without the SGD update (for parity tests of the gradients).                   */
astra_status astra_lm_fwd_bwd(astra_lm m, const int32_t* tokens, float* loss_dev);
/* ---- bucketed profiling for variable-length mini-batches (§5.5; Table 8,
 *      P:395-404) ------------------------------------------------------------------ */
/* Bucket sizes (ascending, each in [1, seq]; the paper's PTB calibration is 13, 18, 24, 30, 83).
 * n = 0 removes the buckets.  Each bucket explores its own update tree and its profile-index keys
 * carry the bucket ("b=<T_b>"); the workspace stays the one of the largest size (seq).         */
astra_status astra_lm_set_buckets(astra_lm m, const int* sizes, int n);
/* One training step on a mini-batch of length len (1 <= len <= seq): tokens device int32
 * [len+1][B].  The step runs at the smallest bucket T_b >= len (seq if none) on right-padded
 * tokens; the mean CE is over the first len·B positions only, so loss and gradients equal those
 * of an unpadded length-len step (padding contributes exact zeros).  Sentence-level semantics:
 * the initial state is zero and no state is carried to the next step.  E_ARG: len out of range. */
astra_status astra_lm_train_step_len(astra_lm m, const int32_t* tokens, int len, float lr, float* loss_dev);
astra_status astra_lm_fwd_bwd_len(astra_lm m, const int32_t* tokens, int len, float* loss_dev);
/* CUDA-graph replay of frozen / untuned bf16 LM steps (default on; ASTRA_GRAPH=0 turns the default
 * off).  on = 0: every step is enqueued kernel by kernel; results are bitwise identical either way.  */
astra_status astra_lm_set_graph(astra_lm m, int on);

/* ---- K1 as a plain library GEMM (tests, microbenchmarks of the paper's Table 1 shapes,
 *      P:107-112, and the fusion example P:122) ------------------------------------------ */
/* C[m][n] (fp32, row stride ldc) = Σ_k A(m,k)·B(k,n), bf16 operands, fp32 accumulate, on the
 * tcgen05 path.  A (device bf16): a_mn = 0 → stored [M][lda] (K contiguous); a_mn = 1 → stored
 * [K][lda] (M contiguous).  B (device bf16): b_mn = 0 → stored [N][ldb]; b_mn = 1 → stored
 * [K][ldb].  lda/ldb in elements, multiples of 8; pointers 16-byte aligned.  bn ∈ {64, 128,
 * 256} is the CTA tile width and cm, cn ∈ {1, 2, 4} (cm·cn ≤ 8) the thread-block-cluster shape
 * for TMA multicast of B (along M) and A (along N) — tuner variables; the result does not
 * depend on them (bitwise).                                                                 */
astra_status astra_gemm_bf16(int M, int N, int K, const void* A, int a_mn, long lda, const void* B, int b_mn,
                             long ldb, float* C, long ldc, int bn, int cm, int cn, astra_stream stream);
/* Extended form.  cta_group = 2 runs the CTA-pair kernel: two CTAs of a cluster share one
 * 256 x bn tile (each holds half of A's rows and half of B's columns in shared memory; requires
 * bn ∈ {128, 256} and cm = cn = 1); the result is bitwise identical to cta_group = 1.
 * ksplit > 1 is the fixed split-K form (the BPTT GEMM's canonical numerics): K is cut into
 * ksplit chunks of ceil(ceil(K/64)/ksplit)·64 elements; chunk s writes its fp32 partial
 * Σ_{k in chunk s} A·B to C + s·M·ldc (C holds ksplit·M rows of ldc floats; a chunk past K writes
 * nothing) and the caller sums the partials in chunk order.  ksplit ∈ [1, 16]; ksplit > 1
 * requires cm = cn = 1.                                                                      */
astra_status astra_gemm_bf16_ex(int M, int N, int K, const void* A, int a_mn, long lda, const void* B, int b_mn,
                                long ldb, float* C, long ldc, int bn, int cm, int cn, int cta_group, int ksplit,
                                astra_stream stream);

/* ---- diagnostics ----------------------------------------------------------------------- */
const char* astra_status_string(astra_status s);
const char* astra_last_error(void);
/* Device times (ms, from the library's cudaEvent pairs) of the regions of the LAST
 * completed step, in this order: a1 hoisted GEMM, forward chain, LM head, BPTT chain, dU, dW,
 * dX, weight-gradient section, whole step.  Unused regions read 0.  Synchronises on the step's
 * end event.  out: host double[cap]; *n ← number written.                                  */
astra_status astra_region_times(astra_cell c, double* out, int cap, int* n);
/* Number of kernels this library has launched since load (all handles).                    */
uint64_t astra_kernel_launch_count(void);

/* ---- day-1 microbenchmarks: floors of the latency-bound chains.  Each call
 *      enqueues its kernels on `stream` and returns; the caller times them with events. -------- */
/* Read `bytes` (multiple of 16) of device memory `buf` `passes` times with 16-byte L2-cached
 * loads from 4 CTAs per SM; sink: device float, written only for a sentinel sum (never in
 * practice).  Bandwidth by size separates L2-resident from HBM streaming (the per-step
 * weight-stream time of U / R_l).                                                            */
astra_status astra_micro_stream_read(const void* buf, size_t bytes, int passes, float* sink, astra_stream stream);
/* One CTA per SM runs `iters` grid-wide flag barriers (release add / acquire spin on *counter,
 * a device unsigned the call zeroes first): the per-step floor of a persistent fused chain.   */
astra_status astra_micro_grid_barrier(unsigned* counter, int iters, astra_stream stream);
/* n dependent empty kernels of `blocks` CTAs, launched with programmatic dependent launch
 * (pdl = 1, as the chain kernels are) or plainly: the per-step floor of a launched chain.     */
/* TMA read throughput: `ctas` CTAs each stream `nbox` boxes {64, box_rows} of the bf16 [rows][64·kb]
 * device buffer through a `stages`-deep shared-memory ring; same = 1: all CTAs read the same boxes. */
/* Per-MMA issue time of a tcgen05.mma chain (the serial MMA chain of a small-batch recurrent step,
 * DESIGN §6c): `ctas` CTAs each issue `iters` dependent M x N x 16 bf16 MMAs (M ∈ {64, 128}, N a
 * multiple of 16 ≤ 256) from shared memory into TMEM; cycles (device int64[ctas]) ← clock64 from
 * the first issue to completion.  mode (bits, per group of 4 MMAs = one k-block, as a k loop
 * does): 1 an mbarrier wait on an already completed phase, 2 tcgen05.fence::after_thread_sync,
 * 4 a tcgen05.commit to an mbarrier.  dump (device fp32[128][N], or null): with iters = 1, CTA
 * 0's 128 TMEM lanes × N columns.  Errors: bad arguments → ASTRA_ERR_ARG.                      */
astra_status astra_micro_mma_chain(int M, int N, int iters, int ctas, int mode, long long* cycles, float* dump,
                                   astra_stream stream);
astra_status astra_micro_tma_read(const void* buf, long rows, int kb, int box_rows, int ctas, int stages, int nbox,
                                  int same, astra_stream stream);
astra_status astra_micro_launch_chain(int n, int pdl, int blocks, astra_stream stream);
/* K11p's rank-ordered reduce kernel for `world` simulated ranks on one device: bufs[r] (device
 * fp32 [n]) is rank r's gradient buffer, sigs[r] a zeroed device array of 4096 bytes (the signal
 * slots), streams[r] its stream.  Each of `reps` rounds launches rank r's kernel on streams[r] with
 * sequence number seq0 + round (must exceed every value used before on these sigs): rank r writes
 * (Σ_q bufs[q][i]) / world, q in rank order, into bufs[r][i] for its shard.  The production kernel
 * and barrier protocol, reading local HBM instead of NVLink (a measure of the kernel itself).     */
astra_status astra_micro_peer_reduce(float* const* bufs, unsigned* const* sigs, int world, size_t n, int reps,
                                     unsigned seq0, const astra_stream* streams);
/* Diagnostic phase traces (globaltimer stamps, ns) written by instrumented kernels into a caller
 * device buffer; NULL turns a trace off (the default).  kind 0: the forward pointwise kernel of the
 * LSTM family, per CTA [2 + 2·16] stamps (entry, grid-dependency wait done, then per row: operands
 * ready, row done); kind 1: the persistent fused RHN forward, per CTA and micro-step [12] stamps
 * (scratch/trace_fwdpw.py, scratch/trace_rhn.py read them).  The buffer must be large enough for
 * the next launch of that kernel; E_ARG for an unknown kind.                                     */
astra_status astra_debug_set_trace(int kind, void* device_buffer);

/* ---- host-only test hooks (no GPU) ------------------------------------------------------ */
/* Drive the tuner's update tree on a fake clock.  `tree` is an s-expression, e.g.
 *   (par (exh g0 (leaf f0 3 g0) (leaf k0 2 g0)) (pre (leaf e0 2 ep0) (leaf e1 3 ep1)))
 *   (fork (leaf alloc 2 step) step (par (leaf fuse 3 gemm 1 3) (leaf kern 2 kern)))
 * where (leaf NAME N METRIC [n_ctx0 n_ctx1 ...]).  `cost` is called once per trial with the
 * configuration (one option index per AV, in the order the AVs appear in the tree) and
 * must write the metric values in `out` (metric names in order of first appearance).
 * trials_out: host int array of capacity max_trials × n_avs; final_out: n_avs ints.       */
typedef void (*astra_fake_cost_fn)(const int* config, int n_avs, double* out, int n_metrics, void* user);
astra_status astra_tuner_selftest(const char* tree, astra_fake_cost_fn cost, void* user,
                                  int* trials_out, int max_trials, int* n_trials,
                                  int* final_out, int* n_avs);

#ifdef __cplusplus
}
#endif
#endif /* ASTRA_H_ */
