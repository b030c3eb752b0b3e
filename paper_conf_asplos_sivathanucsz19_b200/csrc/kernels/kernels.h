// Host launch wrappers of the non-GEMM kernels (K2/K4 unfused pointwise halves, K5 reductions,
// K6 embedding, K7 cross-entropy, K9 SGD + operand mirrors).  Every wrapper launches on `st`.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../common.h"

namespace astra {

// Diagnostic phase traces (astra_debug_set_trace): device buffers of globaltimer stamps written by
// instrumented kernels when set; null (the default) disables the stamps.
enum TraceKind { TRACE_FWD_PW = 0, TRACE_RHN_FWD = 1, TRACE_SB_FWD = 2, TRACE_SB_BWD = 3, TRACE_KINDS };
unsigned long long* trace_buffer(int kind);
void set_trace_buffer(int kind, unsigned long long* buf);

struct GateParams {          // external-layout fp32 vectors of length 4H (may be null for LSTM)
  const float* b = nullptr;
  const float* alpha = nullptr;
  const float* beta1 = nullptr;
  const float* beta2 = nullptr;
};

// ---- mirrors (K9): fp32 params → operand-type copies in the internal layout
// dst[gcol_u(g, j, gu)][k] = src[k][g*H + j] for the gate-blocked [K][4H] matrix `src`
// (dst rows = 4*Hp, row stride ldd ≥ K; padding rows/cols zero).  gu: the internal gate layout of
// the `alloc` fork — 64 (GATE_U, gate-interleaved, the default) or Hp (gate-blocked), cell_math.cuh.
void mirror_gates_T(OT ot, const float* src, int K, int H, int Hp, void* dst, long ldd, cudaStream_t st,
                    long kcols = -1, int gu = 64);
// dst[n][k] = src[k][n] (plain transpose), dst [Np][ldd], padding zero.
void mirror_T(OT ot, const float* src, int K, int N, int Np, int Kp, void* dst, long ldd, cudaStream_t st);
// Operand copy of an external [rows][cols] (OT or fp32 `src_ot`) into [rows][ldd] of type `ot`.
// dcols (default ldd): number of destination columns written (the rest of the row is left as is).
void copy_pad(OT ot, const void* src, OT src_ot, long rows, int cols, long lds, void* dst, long ldd, cudaStream_t st,
              long dcols = -1);
// dst fp32 [rows][ldd] ← src fp32 [rows][lds] (cols), zero padding; src null → zeros.
void copy_f32_pad(const float* src, long rows, int cols, long lds, float* dst, long ldd, int dcols, cudaStream_t st);

// ---- LSTM-family pointwise halves (cell kind: 0 LSTM, 1 MI-LSTM, 5 subLSTM)
// h_op: operand copy of h_t, row stride ldh (≥ Hp); y (type y_ot, row stride ldy) optional.
void lstm_fwd_pointwise(int kind, OT ot, int B, int H, int Hp, const float* WX, const float* UH, GateParams gp,
                        const float* c_prev, float* c_new, void* h_op, long ldh, void* y, long ldy, OT y_ot,
                        float* hT, float* cT, cudaStream_t st, int gu = 64);
// dy: row stride ldy of type dy_ot (or fp32); dh_rec: [B][ld_dh] fp32 or null (zeros).
// dh_rec: nsplit fp32 partials (split-K) at stride split_stride elements, summed in order.
void lstm_bwd_pointwise(int kind, OT ot, int B, int H, int Hp, const void* dy, long ldy, OT dy_ot, bool dy_f32,
                        const float* dh_rec, long ld_dh, int nsplit, long split_stride, float* dc, const float* WX, const float* UH,
                        const float* c_new, const float* c_prev, GateParams gp, void* D_uh, void* D_wx,
                        float* partials, int nq, bool first, cudaStream_t st, int form = 0, int gu = 64);
// form (AV "bwd_pw", bitwise interchangeable): 0 the row-lane kernel (thread = unit, rows walked 4
// lanes x 8), 1 the wide kernel (thread = row x 4 units, all rows of a 32-row chunk in flight), 2 the
// wide kernel with its operand tiles landed in shared memory by TMA (fp32 dy and split dh_rec partials
// only, not at the first step; otherwise it runs form 1).
int lstm_bwd_row_chunks(int B);
constexpr int BWD_ROW_CHUNK = 32;   // rows per column-partial chunk of the backward pointwise kernels (R5)
// grads_q[e] = Σ_chunk partials[chunk][q][gcol(e)] for q < nq (external e < 4H).
void reduce_gate_partials(const float* partials, int nchunk, int nq, int H, int Hp, float* const* grads_q,
                          cudaStream_t st, int gu = 64);

// ---- SCRN [22] / RHN [39] pointwise and scan halves (scrn_rhn_kernels.cu)
int pw_row_chunks(int B);
void scrn_scan_fwd(OT ot, int B, int S, int Sp, int T, float alpha, const float* XB, long ldxb, const float* s0,
                   float* Sf, void* HSs, long ldhs, void* y, long ldy, float* sT, cudaStream_t st);
// Z / dh: nsplit fp32 partials at split_stride elements (the chain GEMM's split-K, reading R33), summed in order.
void scrn_fwd_pw(OT ot, int B, int H, int Hp, const float* Q, long ldq, const float* Z, int nsplit, long split_stride,
                 const float* bh, float* Hf, void* HSh, long ldhs, void* y, long ldy, float* hT, cudaStream_t st);
void scrn_bwd_pw(OT ot, int B, int H, int Hp, const void* dy, long ldy, bool dy_f32, const float* dh, long ld_dh,
                 int nsplit, long split_stride, const float* Hf, void* DZ, long ldz, float* part, bool first,
                 cudaStream_t st);
void scrn_scan_bwd(OT ot, int B, int S, int Sp, int T, float alpha, const void* dys, long ldy, bool dy_f32,
                   const float* DSP, long ldsp, const float* dsT, void* DSa, long ldsa, float* ds0, cudaStream_t st);
// a = (Σ_k Zpart[k] in k order, or Z when Zpart is null) + b (+ WX at ℓ = 1), written to Z (saved pre-activations)
void rhn_fwd_pw(OT ot, int B, int H, int Hp, float* Z, const float* Zpart, int nsplit, long split_stride,
                const float* WX, const float* bl, const float* s_prev, float* s_next, void* s_next_op, void* y,
                long ldy, float* sT, cudaStream_t st);
// ds = ds_in (the carry ds·(1−τ) of the micro-step above) + Σ_k ds_part[k] in k order (the BPTT GEMM's
// split-K partials, reading R33; null at the first micro-step) (+ dy at the top micro-layer).
void rhn_bwd_pw(OT ot, int B, int H, int Hp, const float* ds_in, const float* ds_part, int nsplit, long split_stride,
                const void* dy, long ldy, bool dy_f32, const float* Apre, const float* s_prev, void* DA,
                float* ds_out, float* part, bool first, cudaStream_t st);
void reduce_blocked_partials(const float* part, int nchunk, int nq, int H, int Hp, float* out, cudaStream_t st);
void mirror_blocked_T(OT ot, const float* src, int K, int G, int H, int Hp, void* dst, long ldd, cudaStream_t st);

// ---- K3 attention step (attn_kernels.cu): q [B][Ap], keys/enc [Ts][B][Ap|Hp] fp32, pr [B][Ts]
// escratch / dpscratch: [B][Ts] fp32 (the scores / dp_j between the step's two kernels)
void attn_fwd(OT ot, int B, int Ts, int H, int Hp, int A, int Ap, const float* q, const float* keys, const float* v,
              const float* enc, float* pr, float* escratch, void* ctx_op, long ldc, void* y_ctx, long ldy,
              cudaStream_t st);
// dctx_save: [B][Hp], de_save: [B][Ts] — this step's rows for attn_acc
void attn_bwd(OT ot, int B, int Ts, int H, int Hp, int A, int Ap, const void* dy_ctx, long ldy, bool dy_f32,
              const float* dctx_rec, long ldr, const float* pr, float* dpscratch, const float* q, const float* keys,
              const float* v, const float* enc, void* dq_op, float* dctx_save, float* de_save, float* dvb, bool first,
              cudaStream_t st, int ns = 1, long ss = 0);   // dctx_rec: ns split-K partials at stride ss
// denc / dk ([Ts][B][Hp] / [Ts][B][Ap], overwritten) from the T steps' saved p, de, dctx and q
void attn_acc(OT ot, int T, int B, int Ts, int Hp, int A, int Ap, const float* pr, const float* de_save,
              const float* dctx_save, const float* q, const float* keys, const float* v, float* denc, float* dk,
              cudaStream_t st);

// ---- LM pieces
// dst[b][c][r] = src[b][r][c] for nb bf16 matrices of rows x cols (the RHN BPTT's K-major R copy)
void transpose_bf16(const void* src, int nb, int rows, int cols, void* dst, cudaStream_t st);
void embed_gather(OT ot, const int32_t* tok, long n, const float* E, int I, void* X, long ldx, cudaStream_t st);
// rowloss[r] = lse - logit[target]; dlog (ot) and dlog32 = (softmax - onehot) * inv_n.
void ce_fwd_bwd(OT ot, const float* logits, long ldl, int V, const int32_t* targets, long n, float inv_n,
                float* rowloss, void* dlog, long ldd, float* dlog32, cudaStream_t st, const int* nvp = nullptr,
                long row0 = 0);
// out[i] = Σ_{k < ks} part[k·n + i] in k order (split-K partials, R25/R28).
// out[i] += Σ_k part[k·n + i] (partials summed in k order first)
void add_split_partials(float* out, const float* part, int ks, long n, cudaStream_t st);
void sum_split_partials(const float* part, int ks, long n, float* out, cudaStream_t st);
void sum_rows_to_scalar(const float* v, long n, float scale, float* out, cudaStream_t st, const int* nvp = nullptr);
// *p = v (a one-thread kernel: device-side scalars that captured CUDA graphs read)
void set_i32(int* p, int v, cudaStream_t st);
// out[c] = Σ_r in[r][c] over rows in fixed order (two-level); scratch ≥ colsum_scratch(rows, cols)
size_t colsum_scratch_floats(long rows, int cols);
void colsum(const float* in, long rows, int cols, long ld, float* scratch, float* out, cudaStream_t st);
// Deterministic embedding backward: dE[v] = Σ_{rows with tok=v} dX[row] in ascending row order.
size_t embed_bwd_scratch_bytes(long n, int V);
size_t embed_bwd_partial_floats(long n, int V, int I);
void embed_bwd(const int32_t* tok, long n, int V, const float* dX, long ldx, int I, float* dE, void* scratch,
               size_t scratch_bytes, float* partials, cudaStream_t st);

// ---- SGD (K9): p -= lr * g over n elements
void sgd(float* p, const float* g, size_t n, float lr, cudaStream_t st);
void scale_inplace(float* p, size_t n, float s, cudaStream_t st);

}  // namespace astra
