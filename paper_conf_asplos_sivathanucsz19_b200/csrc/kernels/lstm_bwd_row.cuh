// The per-(row, unit) LSTM-family cell backward and the fixed-order column reduction, shared by the
// unfused backward pointwise kernel (cell_kernels.cu) and the fused BPTT kernel (bptt_fused.cu), so
// the two K4 variants produce the same bits (reading R17).
//
// Reduction order of the bias / α / β column partial sums (R5): a chunk is BWD_RB = 32 consecutive
// batch rows; thread (tx, ty) owns unit u0 + tx and rows ty, ty + 4, ..., ty + 28 of the chunk, and
// accumulates its quantities in registers in ascending row order; the 4 row lanes are then combined
// in ty order (((s0 + s1) + s2) + s3) and folded into partials[chunk][q][col] step after step.
#pragma once
#include "cell_math.cuh"

namespace astra {

constexpr int BWD_RB = 32;  // rows per partial chunk
constexpr int BWD_UX = 64;  // units per CTA (one gate group); thread tx owns unit u0 + tx
constexpr int BWD_RY = 4;   // row lanes (threadIdx.y)
template <int KIND>
struct BwdNV { static constexpr int value = KIND == K_MILSTM ? 16 : 4; };   // quantities per unit: q*4 + gate

// Cell backward of one (row, unit), split in two so a kernel may run the row arithmetic and the
// column-sum accumulation in different threads (lstm_bwd_pw2_kernel) with the same operations:
//   lstm_bwd_da:  pre-activations from (w, h) = (WX, UH) and the gate parameters, cell_bwd → da,
//                 and the gate gradients D_uh / D_wx (bf16 or fp32) returned in duh / dwx;
//   lstm_bwd_acc: the quantities accumulated for the column sums, in this order:
//                 q0 da (→ db), q1 da·wx·uh (→ dα), q2 da·uh (→ dβ1), q3 da·wx (→ dβ2).
template <int KIND, bool F>
__device__ __forceinline__ void lstm_bwd_da(const float (&w)[4], const float (&h)[4], float dh, float& dcv, float cp,
                                            float cn, const float (&bb)[4], const float (&al)[4],
                                            const float (&be1)[4], const float (&be2)[4], float (&da)[4],
                                            float (&duh)[4], float (&dwx)[4]) {
  float a[4];
#pragma unroll
  for (int g = 0; g < 4; ++g) a[g] = preact<KIND, F>(w[g], h[g], bb[g], al[g], be1[g], be2[g]);
  cell_bwd<KIND, F>(a, cp, cn, dh, dcv, da);
#pragma unroll
  for (int g = 0; g < 4; ++g) {
    if (KIND == K_MILSTM) {
      const float gu = F ? __fmaf_rn(al[g], w[g], be1[g]) : __fadd_rn(__fmul_rn(al[g], w[g]), be1[g]);
      const float gw = F ? __fmaf_rn(al[g], h[g], be2[g]) : __fadd_rn(__fmul_rn(al[g], h[g]), be2[g]);
      duh[g] = __fmul_rn(da[g], gu);
      dwx[g] = __fmul_rn(da[g], gw);
    } else {
      duh[g] = da[g];
      dwx[g] = da[g];
    }
  }
}

template <int KIND, bool F>
__device__ __forceinline__ void lstm_bwd_acc(float (&acc)[BwdNV<KIND>::value], int g, float da, float w, float h) {
  constexpr int NV = BwdNV<KIND>::value;
  acc[g] = __fadd_rn(acc[g], da);
  if (KIND == K_MILSTM) {
    const float dw = __fmul_rn(da, w);
    float& r4 = acc[(NV > 4 ? 4 : 0) + g];
    r4 = F ? __fmaf_rn(dw, h, r4) : __fadd_rn(r4, __fmul_rn(dw, h));
    float& r8 = acc[(NV > 8 ? 8 : 0) + g];
    r8 = F ? __fmaf_rn(da, h, r8) : __fadd_rn(r8, __fmul_rn(da, h));
    float& r12 = acc[(NV > 12 ? 12 : 0) + g];
    r12 = __fadd_rn(r12, dw);
  }
}

// Both halves for one (row, unit) with the accumulation in this thread (the unfused kernel's and the
// fused BPTT kernel's form): D_uh / D_wx stored at gate stride gs (GATE_U, or Hp gate-blocked).
template <int KIND, typename T>
__device__ __forceinline__ void lstm_bwd_row(const float (&w)[4], const float (&h)[4], float dh, float& dcv, float cp,
                                             float cn, const float (&bb)[4], const float (&al)[4],
                                             const float (&be1)[4], const float (&be2)[4],
                                             float (&acc)[BwdNV<KIND>::value], T* duhp, T* dwxp, int gs = GATE_U) {
  constexpr bool F = FastMath<T>::value;   // bf16 path: fused multiply-adds (reading R27)
  float da[4], duh[4], dwx[4];
  lstm_bwd_da<KIND, F>(w, h, dh, dcv, cp, cn, bb, al, be1, be2, da, duh, dwx);
#pragma unroll
  for (int g = 0; g < 4; ++g) {
    lstm_bwd_acc<KIND, F>(acc, g, da[g], w[g], h[g]);
    duhp[g * gs] = from_f<T>(duh[g]);
    if (KIND == K_MILSTM) __stcs(dwxp + g * gs, from_f<T>(dwx[g]));
  }
}

// After every thread of the chunk has stored red[ty][i][tx] = acc[i] and the caller synchronised:
// thread (tx, ty) finalises quantities i = ty, ty + 4, ... for unit column `col` (gate g at col +
// g·gs) into the chunk's partials p[q·NG + ...].
// pre (optional): the old partials p[...] of these items, loaded earlier by the caller (pre[i][tx]).
template <int NV>
__device__ __forceinline__ void bwd_chunk_finalize(const float (*red)[NV][BWD_UX], int tx, int ty, float* p, long NG,
                                                   int col0, int nq, int first, int gs = GATE_U,
                                                   const float (*pre)[BWD_UX] = nullptr) {
  for (int i = ty; i < NV; i += BWD_RY) {
    float v = 0.f;
#pragma unroll
    for (int y = 0; y < BWD_RY; ++y) v = __fadd_rn(v, red[y][i][tx]);
    const int q = i / 4, g = i % 4;
    if (q >= nq) continue;
    float* pp = p + (long)q * NG + col0 + g * gs;
    *pp = first ? v : __fadd_rn(pre ? pre[i][tx] : *pp, v);
  }
}

}  // namespace astra
