// Host interface of the fused recurrent kernels (rec_fused.cu), LSTM family, bf16 path.
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>

#include "kernels.h"

namespace astra {

struct RecFwdArgs {
  int B, H, Hp, NG, T;      // T: total steps of the sequence (for hT / cT)
  int t0, t1;               // steps run by this launch
  int num_m, num_n;         // tiles: ceil(B/128) x NG/256
  int stages, nk, persistent;
  uint32_t idesc;           // instruction descriptor of the 128x256 bf16 MMA
  const float* WX;          // [T·B][NG] hoisted projection
  float* UH;                // [T·B][NG] recurrent projection (saved)
  float* C;                 // [(T+1)·B][Hp] cell state
  __nv_bfloat16* Hb;        // [(T+1)·B][Hp] h operand (TMA map A reads it)
  void* y;                  // optional output
  long ldy;
  int y_kind;               // 0 none, 1 bf16 external [T·B][ldy], 2 fp32 [T·B][ldy]
  float* hT;
  float* cT;
  GateParams gp;
  unsigned* flags;          // [num_m] row-block counters (zeroed before a persistent launch)
  int K = 0;                // contraction length of the recurrent GEMM (0: Hp; the attentive decoder's
                            // K-concatenated [h | ctx]·[U_d; C_d] has K = 2Hp)
  long ldh = 0;             // row stride of Hb (0: Hp; the decoder's [h | ctx] operand rows: 2Hp)
};

// CTA-pair fused forward step (rec_fused2.cu): one launch per step t.
struct RecFwd2Args {
  int B, H, Hp, NG, T, t;
  int num_mp, num_n;        // pair tiles: ceil(B/256) x NG/256
  int stages, nk;
  uint32_t idesc;           // M = 256, N = 256 bf16 MMA (cta_group::2)
  int y_kind;               // 0 none, 1 bf16 [T][B][H] via TMA, 2 the same with element stores (H % 8 != 0)
  void* y;
  float* hT;
  float* cT;
  GateParams gp;
};
struct RecFwd2Maps {
  CUtensorMap A;    // Hb [(T+1)][B][Hp] bf16, K-major, box {64, 128} (z = t)
  CUtensorMap B;    // U mirror [NG][Hp] bf16, box {64, 128}
  CUtensorMap WX;   // [T][B][NG] fp32, box {32, 32}, SWIZZLE_128B
  CUtensorMap UH;   // [T][B][NG] fp32, box {32, 32}, SWIZZLE_128B
  CUtensorMap C;    // [(T+1)][B][Hp] fp32, box {32, 32}, SWIZZLE_128B
  CUtensorMap H;    // [(T+1)][B][Hp] bf16, box {32, 32}, SWIZZLE_64B
  CUtensorMap Y;    // [T][B][H] bf16, box {32, 32}, SWIZZLE_64B (unused when y_kind = 0)
};
void lstm_fwd_pair_launch(int kind, const RecFwd2Maps& m, RecFwd2Args a, cudaStream_t st);

// mapA: Hb as a 3-D K-major map (inner Hp, rows B, z = T+1), box {64, 128};
// mapB: the U mirror [NG][Hp] K-major, box {64, 256}.
void lstm_rec_fwd_launch(int kind, const CUtensorMap& mapA, const CUtensorMap& mapB, RecFwdArgs a, cudaStream_t st);

// Fused BPTT step (bptt_fused.cu): dh_rec = D_uh_{t+1}·Uᵀ (canonical split-K kept as nsplit TMEM
// accumulators) + the cell backward of step t; one launch per step t < T-1.
struct BpttFusedArgs {
  int B, H, Hp, NG, t;
  int nk, kper, nsplit;     // k-blocks of K = NG, k-blocks per split-K chunk, chunks (reading R25)
  int stages;
  uint32_t idesc;           // M = 128, N = 64, A K-major, B MN-major bf16 MMA
  int nq;                   // column-sum quantities (4 MI-LSTM: b, α, β1, β2; else 1)
  GateParams gp;
  void* D_uh;               // bf16 [T·B][NG] (base; the kernel writes step t's slice)
  void* D_wx;
  float* dc;                // [B][Hp]
  float* partials;          // [chunks][nq][NG]
};
struct BpttFusedMaps {
  CUtensorMap A;    // D_uh [T][B][NG] bf16, K-major, box {64, 128} (z = t+1)
  CUtensorMap B;    // U mirror [NG][Hp] bf16 as MN-major B, box {64, 64}
  CUtensorMap WX;   // [T][B][NG] fp32, box {256, 16}
  CUtensorMap UH;   // [T][B][NG] fp32, box {256, 16}
  CUtensorMap C;    // [T+1][B][Hp] fp32, box {64, 16}
  CUtensorMap DC;   // [1][B][Hp] fp32, box {64, 16}
  CUtensorMap DY;   // dy [T][B][ld] fp32 (LM internal, ld = Hp) or bf16 (external, ld = H), box {64, 16}
};
// Persistent fused RHN forward chain (rhn_fused.cu): all T·L micro-steps of [t0, t1) in one
// cooperative launch; tiles of 128 rows × 32 units (their H and T columns), split-K chunks of the
// canonical R33 split kept as TMEM accumulators, the whole K of a micro-step resident when it fits.
struct RhnFwdArgs {
  int B, H, Hp, T, L, t0, t1;
  int nsplit;               // canonical split-K chunks of K = Hp (RhnCell::fwd_ksplit)
  int num_m, num_n, stages, nk, kper, tmem_cols;   // set by the launcher
  int a_rows;               // rows of the A box: 64 when B <= 64 (the MMA's rows 64..127 are never read), else 128
  uint32_t idesc;           // M = 128, N = 128 bf16 MMA, both operands K-major
  const float* WX;          // [T·B][2Hp] hoisted x·W (added at ℓ = 1)
  const float* b;           // [L][2H] external biases
  float* Apre;              // [L][T][B][2Hp] pre-activations (saved for BPTT)
  float* Sf;                // fp32 states, RhnCell::slot layout
  __nv_bfloat16* Sop;       // bf16 operand states (mapA reads them), same layout
  __nv_bfloat16* y;         // optional [T][B][ldy]
  long ldy;
  float* sT;                // optional [B][H]
  unsigned* flags;          // [num_m] row-block counters, zeroed before the launch
  unsigned long long* trace;   // optional (astra_debug_set_trace): [grid][T·L][12] globaltimer stamps
};
bool rhn_rec_fwd_supported(int B, int Hp, int nsplit);
// mapA: the bf16 state operands as a 3-D K-major map (inner Hp, rows B, z = L·(T+1)), box {64, a_rows};
// mapB: the R mirrors [L][2Hp][Hp] K-major, box {64, 32}; both SWIZZLE_128B.
void rhn_rec_fwd_launch(const CUtensorMap& mapA, const CUtensorMap& mapB, RhnFwdArgs a, cudaStream_t st);

// Small-batch persistent forward chain (rec_persist.cu, fwd_mode 3): all steps [t0, t1) in one
// cooperative launch of Hp/16 CTAs (16 units each, their U slice resident in shared memory as far as
// it fits), B ≤ 128, fused gate epilogue, one grid-wide counter per step.
struct RecPersistArgs {
  int B, H, Hp, NG, T, t0, t1;
  int nk, resident, sa, sb, a_rows, a_bytes, ka, kbs;   // set by the launcher (ka / kbs: k-blocks per A / B stage)
  uint32_t idesc;
  const float* WX;          // [T·B][NG]
  float* UH;                // [T·B][NG] saved for BPTT, or null (recompute context)
  float* C;                 // [(T+1)·B][Hp]
  __nv_bfloat16* Hb;        // [(T+1)·B][Hp]
  void* y;
  long ldy;
  int y_kind;               // 0 none, 1 bf16 [T·B][ldy], 2 fp32 [T·B][ldy]
  float* hT;
  float* cT;
  GateParams gp;
  unsigned* flags;          // one counter, zeroed before the launch
  unsigned long long* trace;   // optional (astra_debug_set_trace kind 2): [grid][t1-t0][6] globaltimer stamps
  int K = 0;                // contraction length (0: Hp); the attentive decoder's [h | ctx]·[U_d; C_d]: 2Hp.
                            // Hb rows and U-mirror rows then have stride K
  long ldh = 0;             // row stride of Hb (0: K; set by the launcher)
  int max_resident = -1;    // cap on the resident U k-blocks (-1: as many as fit); a one-step launch
                            // streams its whole U slice through the ring (0) so the MMAs start at once
  int b_old = 0;            // 1: the U mirror was written ≥ 2 launches back (PDL launch): the B producer
                            // starts before the grid dependency resolves
};
bool lstm_fwd_persist_supported(int B, int Hp);
// Hb: [(Tmax+1)][B][Hp] bf16 h operands; Um: the U mirror [NG][Hp] (tensor maps built per launch).
void lstm_fwd_persist_launch(int kind, const void* Hb, const void* Um, int Tmax, RecPersistArgs a, cudaStream_t st);

// SC-RNN persistent forward h-chain (scrn_persist.cu, ScrnCell fwd_mode 1): all steps [t0, t1) in one
// cooperative launch of Hp/16 CTAs, B ≤ 128, the R slice resident, the R33 split kept as TMEM
// accumulators, h_t = σ(Q_t + Σ partials + b_h) fused.
struct ScrnPersistArgs {
  int B, H, Hp, T, t0, t1, nsplit;
  int nk, kper, ka, a_rows, a_bytes;   // set by the launcher
  uint32_t idesc;
  const float* Q;           // [T·B][ldq] hoisted x·A + s·P
  long ldq;
  const float* bh;          // [H]
  float* Hf;                // [(T+1)·B][Hp] fp32 h
  __nv_bfloat16* HS;        // [(T+1)·B][ldhs] bf16 [h | s] operand rows (h part written)
  long ldhs;
  __nv_bfloat16* y;         // optional [T·B][ldy] external y (h part)
  long ldy;
  float* hT;
  unsigned* flags;          // one counter, zeroed before the launch
};
bool scrn_fwd_persist_supported(int B, int Hp, int nsplit);
// SC-RNN persistent BPTT h-chain (ScrnCell bwd_mode 1): t = T−1 … 0 in one cooperative launch;
// dh_rec = dz_{t+1}·Rᵀ with the R33 split as TMEM accumulators (R resident as a K-major copy),
// dz_t = (dy^h + dh_rec)·h(1−h) fused, db_h partials in the row-lane order of scrn_bwd_pw_kernel.
struct ScrnBpttArgs {
  int B, H, Hp, T, nsplit;
  int nk, kper, ka, a_rows, a_bytes;   // set by the launcher
  uint32_t idesc;
  const void* dy;           // h part of dy: fp32 [T·B][ldy] (LM) or bf16 [T·B][ldy] (external)
  long ldy;
  const float* dhT;         // optional [B][H]
  const float* Hf;          // [(T+1)·B][Hp] fp32 h
  __nv_bfloat16* DZ;        // [T·B][lddz] dz operand rows (dz part written)
  long lddz;
  float* part;              // [ceil(B/32)][Hp] db_h partials (written at the end)
  unsigned* flags;          // one counter, zeroed before the launch
};
bool scrn_bwd_persist_supported(int B, int Hp, int nsplit, int T);
void scrn_bwd_persist_launch(const void* DZ, long lddz, const void* Rk, int T, bool dy_f32, ScrnBpttArgs a,
                             cudaStream_t st);
void scrn_fwd_persist_launch(const void* HS, long ldhs, const void* MR, int Tmax, ScrnPersistArgs a, cudaStream_t st);

// Small-batch persistent BPTT chain (bptt_persist.cu, LSTM-family bwd_mode 2/3): t = T−1 … 0 in one
// cooperative launch of Hp/16 CTAs in clusters of 4 (the R25 split-K chunks), 64 units per cluster,
// the chunk partials of dh_rec summed in chunk order over distributed shared memory, the cell
// backward fused, one counter per K chunk.  B ≤ 128, bf16 path, Hp % 256 == 0, nsplit == 4.
struct BpttPersistArgs {
  int B, H, Hp, NG, T;
  int kper, resident, sa, sb, a_rows, a_bytes, ka, kbs;   // set by the launcher
  uint32_t idesc;
  int nq;                   // column-sum quantities (4 MI-LSTM, else 1)
  GateParams gp;
  const void* dy;           // fp32 [T·B][ldy] (LM, ldy = Hp) or bf16 [T·B][ldy] (external, ldy = H)
  long ldy;
  const float* dhT;         // optional [B][H]
  const float* WX;          // [T·B][NG]
  const float* UH;          // [T·B][NG]
  const float* C;           // [(T+1)·B][Hp]
  float* dc;                // [B][Hp]: dc_T in, dc_0 out
  __nv_bfloat16* D_uh;      // [T·B][NG]
  __nv_bfloat16* D_wx;      // [T·B][NG] (MI-LSTM)
  float* partials;          // [ceil(B/32)][nq][NG], written at the end
  unsigned* flags;          // [4] per-chunk counters, zeroed before the launch
  unsigned long long spin;  // diagnostics: give up a wait after this many probes (0: never)
  unsigned long long* trace;   // optional (astra_debug_set_trace kind 3): [grid][T][8] globaltimer stamps
};
bool lstm_bptt_persist_supported(int B, int Hp, int nsplit);
// true when the clusters of the launch are co-resident on this device (checked once per shape)
bool lstm_bptt_persist_fits(int kind, int B, int Hp, int NG);
void lstm_bptt_persist_launch(int kind, bool dy_f32, const void* Duh, const void* Um, int Tmax, BpttPersistArgs a,
                              cudaStream_t st);

// Persistent RHN BPTT chain (rhn_bptt_persist.cu, RhnCell bwd_mode 1): all T·L backward micro-steps in
// one cooperative launch of clusters of 4 CTAs (the R33 chunks), 32 units per cluster, the chunk
// partials exchanged over distributed shared memory; B ≤ 64, nsplit == 4.
struct RhnBpttArgs {
  int B, H, Hp, T, L, nsplit, nchunk;
  int nk, kper;             // set by the launcher
  uint32_t idesc;
  const void* dy;           // fp32 [T·B][ldy] (LM, ldy = Hp) or bf16 [T·B][ldy] (external, ldy = H)
  long ldy;
  const float* Apre;        // [L][T][B][2Hp]
  const float* Sf;          // fp32 states, RhnCell::slot layout
  __nv_bfloat16* DA;        // [L][T][B][2Hp]
  float* dS;                // [B][Hp]: ds_T in, ds of s^0_0 out
  float* part;              // [L][nchunk][2][Hp] db partials
  unsigned* flags;          // one counter, zeroed before the launch
};
bool rhn_bptt_persist_supported(int B, int Hp, int nsplit, int L);
bool rhn_bptt_persist_fits(int B, int Hp, int nsplit, int L);
// DA: the DA base; RK: the K-major R copy [L][Hp][2Hp] (rows = units)
void rhn_bptt_persist_launch(bool dy_f32, const void* DA, const void* RK, RhnBpttArgs a, cudaStream_t st);

bool lstm_bptt_fused_supported(int B, int Hp, int nsplit);
void lstm_bptt_fused_launch(int kind, bool dy_bf16, const BpttFusedMaps& m, BpttFusedArgs a, cudaStream_t st);

}  // namespace astra
