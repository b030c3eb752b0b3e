// Per-element cell arithmetic shared by every kernel variant of a precision path:
// the unfused pointwise kernels and the fused GEMM epilogues call exactly these functions, written
// with explicit round-to-nearest intrinsics so no variant can be contracted differently.
#pragma once
#include <cuda_bf16.h>

namespace astra {

// Internal gate-interleaved column order (the `alloc` layout, unit block u = 64):
// internal column of (gate g, unit j) = (j / 64)·256 + g·64 + (j % 64).
constexpr int GATE_U = 64;
__host__ __device__ __forceinline__ int gcol(int g, int j) { return (j / GATE_U) * (4 * GATE_U) + g * GATE_U + (j % GATE_U); }
// The same order for a general unit block gu (a multiple of 64): gu = GATE_U is the interleaved layout
// above, gu = Hp the gate-blocked one (column g·Hp + j) — the two layouts of the `alloc` fork (R38).
// The gate stride of a unit's four columns is gu.
__host__ __device__ __forceinline__ int gcol_u(int g, int j, int gu) { return (j / gu) * (4 * gu) + g * gu + (j % gu); }

// Transcendentals.  fp32 path (F = false): IEEE-accurate expf / tanhf (the 1e-4 parity bar).  bf16
// path (F = true, reading R3): the MUFU tanh.approx.f32 (rel. error ≈ 2^-11), σ(x) = ½·tanh(x/2) + ½ —
// far below the 2e-2 bar and shared by every bf16 kernel variant, so variants stay bitwise equal.
__device__ __forceinline__ float tanh_approx(float x) {
  float y;
  asm("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
template <bool F = false>
__device__ __forceinline__ float sigm(float x) {
  if (F) return __fmaf_rn(0.5f, tanh_approx(__fmul_rn(0.5f, x)), 0.5f);
  return __frcp_rn(__fadd_rn(1.f, expf(-x)));
}
template <bool F = false>
__device__ __forceinline__ float tanh_(float x) {
  if (F) return tanh_approx(x);
  return tanhf(x);
}
template <typename T> struct FastMath { static constexpr bool value = false; };
template <> struct FastMath<__nv_bfloat16> { static constexpr bool value = true; };

template <typename T> __device__ __forceinline__ float to_f(T v);
template <> __device__ __forceinline__ float to_f<float>(float v) { return v; }
template <> __device__ __forceinline__ float to_f<__nv_bfloat16>(__nv_bfloat16 v) { return __bfloat162float(v); }
template <typename T> __device__ __forceinline__ T from_f(float v);
template <> __device__ __forceinline__ float from_f<float>(float v) { return v; }
template <> __device__ __forceinline__ __nv_bfloat16 from_f<__nv_bfloat16>(float v) { return __float2bfloat16_rn(v); }

// p[0] + p[s] + ... + p[(n−1)·s] summed in chunk order (the R25 / R33 split-K partials).  The loads
// of the first SPLIT_MAX partials are issued together (predicated) before the ordered adds, so a row
// waits one memory latency instead of n dependent ones; the sum and its rounding order are unchanged.
constexpr int SPLIT_MAX = 4;   // R25 and R33 never split further
__device__ __forceinline__ float sum_split(const float* __restrict__ p, int n, long s) {
  float v[SPLIT_MAX];
#pragma unroll
  for (int k = 0; k < SPLIT_MAX; ++k) v[k] = k < n ? p[k * s] : 0.f;
  float r = v[0];
#pragma unroll
  for (int k = 1; k < SPLIT_MAX; ++k)
    if (k < n) r = __fadd_rn(r, v[k]);
  for (int k = SPLIT_MAX; k < n; ++k) r = __fadd_rn(r, p[k * s]);
  return r;
}

// The same sum with the chunk count fixed at compile time (NS > 0; NS = 0: sum_split): the loads
// are unpredicated and the adds in the same order.
template <int NS>
__device__ __forceinline__ float sum_split_n(const float* __restrict__ p, int n, long s) {
  if constexpr (NS == 0) {
    return sum_split(p, n, s);
  } else {
    float v[NS];
#pragma unroll
    for (int k = 0; k < NS; ++k) v[k] = p[k * s];
    float r = v[0];
#pragma unroll
    for (int k = 1; k < NS; ++k) r = __fadd_rn(r, v[k]);
    return r;
  }
}

enum CellKind { K_LSTM = 0, K_MILSTM = 1, K_SUBLSTM = 5 };

// Pre-activation of one gate.  LSTM/subLSTM: a = wx + uh + b.
// MI-LSTM [36]: a = α·wx·uh + β1·uh + β2·wx + b  (reading R3/R4).  fp32 path: evaluated left to
// right with separate roundings; bf16 path (F): the same sum as a fixed chain of fused multiply-adds
// a = fma(α·wx, uh, fma(β1, uh, fma(β2, wx, b))) — fewer instructions, identical in every bf16 kernel.
template <int KIND, bool F = false>
__device__ __forceinline__ float preact(float wx, float uh, float b, float al, float b1, float b2) {
  if (KIND == K_MILSTM) {
    if (F) return __fmaf_rn(__fmul_rn(al, wx), uh, __fmaf_rn(b1, uh, __fmaf_rn(b2, wx, b)));
    float a = __fmul_rn(__fmul_rn(al, wx), uh);
    a = __fadd_rn(a, __fmul_rn(b1, uh));
    a = __fadd_rn(a, __fmul_rn(b2, wx));
    return __fadd_rn(a, b);
  } else {
    return __fadd_rn(__fadd_rn(wx, uh), b);
  }
}

// Forward cell update from the four pre-activations.  Returns (c_new, h_new).
template <int KIND, bool F = false>
__device__ __forceinline__ void cell_fwd(const float (&a)[4], float c_prev, float& c_new, float& h_new) {
  if (KIND == K_SUBLSTM) {
    const float i = sigm<F>(a[0]), f = sigm<F>(a[1]), z = sigm<F>(a[2]), o = sigm<F>(a[3]);
    c_new = F ? __fsub_rn(__fmaf_rn(f, c_prev, z), i) : __fsub_rn(__fadd_rn(__fmul_rn(f, c_prev), z), i);
    h_new = __fsub_rn(sigm<F>(c_new), o);
  } else {
    const float i = sigm<F>(a[0]), f = sigm<F>(a[1]), g = tanh_<F>(a[2]), o = sigm<F>(a[3]);
    c_new = F ? __fmaf_rn(f, c_prev, __fmul_rn(i, g)) : __fadd_rn(__fmul_rn(f, c_prev), __fmul_rn(i, g));
    h_new = __fmul_rn(o, tanh_<F>(c_new));
  }
}

// Backward of one cell update.  dh = dL/dh_t, dc = dL/dc_t from step t+1 (in/out: becomes
// dL/dc_{t-1}).  da[4] = dL/da for the four gates.  x·(1−x) and 1−x² as fused forms in the bf16
// path (F), separate roundings in the fp32 path.
template <int KIND, bool F = false>
__device__ __forceinline__ void cell_bwd(const float (&a)[4], float c_prev, float c_new, float dh, float& dc,
                                         float (&da)[4]) {
  auto dsig = [](float s) { return F ? __fmaf_rn(-s, s, s) : __fmul_rn(s, __fsub_rn(1.f, s)); };
  auto dtnh = [](float t) { return F ? __fmaf_rn(-t, t, 1.f) : __fsub_rn(1.f, __fmul_rn(t, t)); };
  if (KIND == K_SUBLSTM) {
    const float i = sigm<F>(a[0]), f = sigm<F>(a[1]), z = sigm<F>(a[2]), o = sigm<F>(a[3]);
    const float sc = sigm<F>(c_new);
    const float dcc = F ? __fmaf_rn(dh, dsig(sc), dc) : __fadd_rn(dc, __fmul_rn(dh, dsig(sc)));
    da[0] = __fmul_rn(-dcc, dsig(i));
    da[1] = __fmul_rn(__fmul_rn(dcc, c_prev), dsig(f));
    da[2] = __fmul_rn(dcc, dsig(z));
    da[3] = __fmul_rn(-dh, dsig(o));
    dc = __fmul_rn(dcc, f);
  } else {
    const float i = sigm<F>(a[0]), f = sigm<F>(a[1]), g = tanh_<F>(a[2]), o = sigm<F>(a[3]);
    const float tau = tanh_<F>(c_new);
    const float dcc = F ? __fmaf_rn(__fmul_rn(dh, o), dtnh(tau), dc)
                        : __fadd_rn(dc, __fmul_rn(__fmul_rn(dh, o), dtnh(tau)));
    da[0] = __fmul_rn(__fmul_rn(dcc, g), dsig(i));
    da[1] = __fmul_rn(__fmul_rn(dcc, c_prev), dsig(f));
    da[2] = __fmul_rn(__fmul_rn(dcc, i), dtnh(g));
    da[3] = __fmul_rn(__fmul_rn(dh, tau), dsig(o));
    dc = __fmul_rn(dcc, f);
  }
}

}  // namespace astra
