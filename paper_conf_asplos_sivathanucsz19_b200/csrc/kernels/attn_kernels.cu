// K3: additive attention step of the reduced GNMT decoder [35] (PAPER.md P:37, P:352, P:372-382,
// P:410 "mostly covered by cuDNN except the Attention module"; reading R10).
//
//   e_j = vᵀ tanh(q + k_j),  p = softmax_j(e),  ctx = Σ_j p_j enc_j          (one decoder step, per b)
//
// Each direction is two kernels over many CTAs (round 1 ran one CTA per batch row: 128 CTAs doing
// the whole step serially, 60-130 µs per decoder step at cfg4): forward = scores (one warp per
// (b, j)) then softmax + context (B × ⌈Hp/256⌉ CTAs); backward = dp_j (one warp per (b, j)) then
// de, denc, dq, dk, dv (B × ⌈max(Hp, Ap)/256⌉ CTAs).  Every reduction has a fixed order (a warp's
// lanes take float4 quads in ascending order + a fixed xor tree; the softmax and Σ p dp by warp 0
// over lane-strided j; the context, dq, dv and the denc / dk accumulators in ascending j), so the
// result is independent of launch timing (R5).  fp32 throughout (ALU/MUFU-bound).
#include <algorithm>

#include "cell_math.cuh"
#include "kernels.h"
#include "pdl.cuh"

namespace astra {

constexpr int ATT_THREADS = 256;

// Scores, one warp per (b, j) over a grid of B × ⌈Ts/8⌉ CTAs: lane l takes the float4 quads
// c = l, l + 32, … of the attention width in ascending order (tanh per element, then the products
// added in element order), then a fixed xor tree over the lanes.  Rows b of the q / keys buffers
// hold Ap floats (A ≤ Ap, the pad columns are ignored).
template <typename T>
__global__ void __launch_bounds__(ATT_THREADS)
    attn_score_kernel(int B, int Ts, int A, int Ap, const float* __restrict__ q, const float* __restrict__ keys,
                      const float* __restrict__ v, float* __restrict__ e) {
  pdl_wait();   // chain kernel: launched with PDL (pdl.cuh)
  pdl_trigger();
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  const int b = blockIdx.y, j = blockIdx.x * (ATT_THREADS / 32) + w;
  if (j >= Ts) return;
  const float4* qb = reinterpret_cast<const float4*>(q + (long)b * Ap);
  const float4* kj = reinterpret_cast<const float4*>(keys + ((long)j * B + b) * Ap);
  const float4* v4 = reinterpret_cast<const float4*>(v);
  constexpr bool F = FastMath<T>::value;
  float s = 0.f;
  const int nq = (A + 3) / 4;
  for (int c = l; c < nq; c += 32) {
    const float4 qa = qb[c], ka = __ldcs(kj + c), va = v4[c];
    const int a0 = 4 * c;
    s = __fadd_rn(s, __fmul_rn(va.x, tanh_<F>(__fadd_rn(qa.x, ka.x))));
    if (a0 + 1 < A) s = __fadd_rn(s, __fmul_rn(va.y, tanh_<F>(__fadd_rn(qa.y, ka.y))));
    if (a0 + 2 < A) s = __fadd_rn(s, __fmul_rn(va.z, tanh_<F>(__fadd_rn(qa.z, ka.z))));
    if (a0 + 3 < A) s = __fadd_rn(s, __fmul_rn(va.w, tanh_<F>(__fadd_rn(qa.w, ka.w))));
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
  if (l == 0) e[(long)b * Ts + j] = s;
}

// Softmax over j (every CTA of row b recomputes it from the scores: warp 0, lane-strided max / sum,
// fixed xor trees), then ctx_h = Σ_j p_j enc_j,h in ascending j for the CTA's 256 hidden units;
// the blockIdx.x == 0 CTA of each row stores p (saved for the backward).
template <typename T, typename TY>
__global__ void __launch_bounds__(ATT_THREADS)
    attn_ctx_kernel(int B, int Ts, int H, int Hp, const float* __restrict__ escore, const float* __restrict__ enc,
                    float* __restrict__ pr, T* __restrict__ ctx_op, long ldc, TY* __restrict__ y_ctx, long ldy) {
  pdl_wait();
  pdl_trigger();
  extern __shared__ float sh[];
  float* e = sh;            // [Ts]
  const int b = blockIdx.y;
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  for (int j = threadIdx.x; j < Ts; j += ATT_THREADS) e[j] = escore[(long)b * Ts + j];
  __syncthreads();
  if (w == 0) {
    float m = -INFINITY;
    for (int j = l; j < Ts; j += 32) m = fmaxf(m, e[j]);
#pragma unroll
    for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    float s = 0.f;
    for (int j = l; j < Ts; j += 32) {
      e[j] = expf(__fsub_rn(e[j], m));
      s = __fadd_rn(s, e[j]);
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
    __syncwarp();
    for (int j = l; j < Ts; j += 32) e[j] = __fdiv_rn(e[j], s);
  }
  __syncthreads();
  if (blockIdx.x == 0)
    for (int j = threadIdx.x; j < Ts; j += ATT_THREADS) pr[(long)b * Ts + j] = e[j];
  const int h = blockIdx.x * ATT_THREADS + threadIdx.x;
  if (h >= Hp) return;
  float c = 0.f;
  if (h < H) {
    constexpr int JG = 10;   // loads of a group issued before its adds (the sum order is unchanged)
    for (int j0 = 0; j0 < Ts; j0 += JG) {
      float x[JG];
#pragma unroll
      for (int k = 0; k < JG; ++k) x[k] = j0 + k < Ts ? enc[((long)(j0 + k) * B + b) * Hp + h] : 0.f;
#pragma unroll
      for (int k = 0; k < JG; ++k)
        if (j0 + k < Ts) c = __fadd_rn(c, __fmul_rn(e[j0 + k], x[k]));
    }
  }
  ctx_op[(long)b * ldc + h] = from_f<T>(c);
  if (y_ctx && h < H) y_ctx[(long)b * ldy + h] = from_f<TY>(c);
}

void attn_fwd(OT ot, int B, int Ts, int H, int Hp, int A, int Ap, const float* q, const float* keys, const float* v,
              const float* enc, float* pr, float* escratch, void* ctx_op, long ldc, void* y_ctx, long ldy,
              cudaStream_t st) {
  ASTRA_CHECK_ARG(Ap % 4 == 0 && ((uintptr_t)q & 15) == 0 && ((uintptr_t)keys & 15) == 0 && ((uintptr_t)v & 15) == 0,
                  "attn_fwd: q / keys / v rows must be 16-byte aligned float4 rows");
  const dim3 gs(cdiv(Ts, ATT_THREADS / 32), B), gc(cdiv(Hp, ATT_THREADS), B);
  const size_t sm = (Ts + 8) * sizeof(float);
  if (ot == OT::BF16) {
    launch_pdl(attn_score_kernel<__nv_bfloat16>, gs, dim3(ATT_THREADS), 0, st, 1, B, Ts, A, Ap, q, keys, v, escratch);
    LAUNCH_CHECK();
    launch_pdl(attn_ctx_kernel<__nv_bfloat16, __nv_bfloat16>, gc, dim3(ATT_THREADS), sm, st, 1, B, Ts, H, Hp,
               (const float*)escratch, enc, pr, (__nv_bfloat16*)ctx_op, ldc, (__nv_bfloat16*)y_ctx, ldy);
  } else {
    launch_pdl(attn_score_kernel<float>, gs, dim3(ATT_THREADS), 0, st, 1, B, Ts, A, Ap, q, keys, v, escratch);
    LAUNCH_CHECK();
    launch_pdl(attn_ctx_kernel<float, float>, gc, dim3(ATT_THREADS), sm, st, 1, B, Ts, H, Hp, (const float*)escratch,
               enc, pr, (float*)ctx_op, ldc, (float*)y_ctx, ldy);
  }
  LAUNCH_CHECK();
}

// Backward of one attention step (oracle/cells.py attn_backward):
//   dctx = dy_ctx + dctx_rec;  dp_j = dctx·enc_j;  de_j = p_j (dp_j − Σ p dp);  denc_j += p_j dctx;
//   u_j = tanh(q + k_j);  du_j = de_j v (1 − u_j²);  dq = Σ_j du_j;  dk_j += du_j;  dv_b += Σ_j de_j u_j
// dctx_h of row b = dy_ctx + dctx_rec (0 past H); dctx_rec may be the ns split-K partials of the
// decoder's BPTT GEMM at stride ss (reading R42), summed in chunk order first
template <typename TDY>
__device__ __forceinline__ float attn_dctx(const TDY* __restrict__ dy_ctx, long ldy, const float* __restrict__ dctx_rec,
                                           long ldr, int ns, long ss, int b, int h, int H) {
  if (h >= H) return 0.f;
  float d = dy_ctx ? to_f<TDY>(dy_ctx[(long)b * ldy + h]) : 0.f;
  if (dctx_rec) d = __fadd_rn(d, sum_split(dctx_rec + (long)b * ldr + h, ns, ss));
  return d;
}

// dp_j = dctx·enc_j, one warp per (b, j): lane l takes the hidden quads c = l, l + 32, … in
// ascending order, then a fixed xor tree.
template <typename TDY>
__global__ void __launch_bounds__(ATT_THREADS)
    attn_dp_kernel(int B, int Ts, int H, int Hp, const TDY* __restrict__ dy_ctx, long ldy,
                   const float* __restrict__ dctx_rec, long ldr, int ns, long ss, const float* __restrict__ enc, float* __restrict__ dp) {
  extern __shared__ float sdctx[];   // [Hp]: row b's dctx, formed once per CTA (its warps share b)
  pdl_wait();
  pdl_trigger();
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  const int b = blockIdx.y, j = blockIdx.x * (ATT_THREADS / 32) + w;
  for (int h = threadIdx.x; h < Hp; h += ATT_THREADS) sdctx[h] = attn_dctx(dy_ctx, ldy, dctx_rec, ldr, ns, ss, b, h, H);
  __syncthreads();
  if (j >= Ts) return;
  const float4* ej = reinterpret_cast<const float4*>(enc + ((long)j * B + b) * Hp);
  float s = 0.f;
  for (int c = l; 4 * c < H; c += 32) {
    const float4 x = ej[c];
    const int h = 4 * c;
    s = __fadd_rn(s, __fmul_rn(sdctx[h], x.x));
    s = __fadd_rn(s, __fmul_rn(sdctx[h + 1], x.y));
    s = __fadd_rn(s, __fmul_rn(sdctx[h + 2], x.z));
    s = __fadd_rn(s, __fmul_rn(sdctx[h + 3], x.w));
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
  if (l == 0) dp[(long)b * Ts + j] = s;
}

// The rest of one attention step's backward, grid ⌈max(Hp, Ap)/256⌉ × B: every CTA of row b forms
// de_j = p_j (dp_j − Σ p dp) (warp 0, lane-strided j, fixed xor tree), then thread index x does
//   hidden unit x:  saves dctx (the step's dctx row) for the deferred denc accumulation;
//   width x:        u_j = tanh(q + k_j), du_j = de_j v (1 − u_j²), dq = Σ_j du_j, dv_b += Σ_j de_j u_j
//                   (ascending j);
// and the row's de is saved for the deferred dk accumulation (attn_acc_kernel).
template <typename T, typename TDY>
__global__ void __launch_bounds__(ATT_THREADS)
    attn_bwd_kernel(int B, int Ts, int H, int Hp, int A, int Ap, const TDY* __restrict__ dy_ctx, long ldy,
                    const float* __restrict__ dctx_rec, long ldr, int ns, long ss, const float* __restrict__ pr,
                    const float* __restrict__ dpv, const float* __restrict__ q, const float* __restrict__ keys,
                    const float* __restrict__ v, T* __restrict__ dq_op, float* __restrict__ dctx_save,
                    float* __restrict__ de_save, float* __restrict__ dvb, int first) {
  pdl_wait();   // chain kernel: launched with PDL (pdl.cuh)
  pdl_trigger();
  extern __shared__ float sh[];
  float* de = sh;                // [Ts]
  const int b = blockIdx.y;
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  for (int j = threadIdx.x; j < Ts; j += ATT_THREADS) de[j] = dpv[(long)b * Ts + j];
  __syncthreads();
  if (w == 0) {   // de_j = p_j (dp_j − Σ p dp), the sum by a fixed xor tree over lane-strided partials
    float s = 0.f;
    for (int j = l; j < Ts; j += 32) s = __fadd_rn(s, __fmul_rn(pr[(long)b * Ts + j], de[j]));
#pragma unroll
    for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
    __syncwarp();
    for (int j = l; j < Ts; j += 32) de[j] = __fmul_rn(pr[(long)b * Ts + j], __fsub_rn(de[j], s));
  }
  __syncthreads();
  if (blockIdx.x == 0)
    for (int j = threadIdx.x; j < Ts; j += ATT_THREADS) de_save[(long)b * Ts + j] = de[j];
  const int x = blockIdx.x * ATT_THREADS + threadIdx.x;
  if (x < Hp) dctx_save[(long)b * Hp + x] = attn_dctx(dy_ctx, ldy, dctx_rec, ldr, ns, ss, b, x, H);
  if (x < Ap) {   // attention-width terms
    constexpr int JG = 10;
    const int a = x;
    const float* qb = q + (long)b * Ap;
    float dq = 0.f, dva = 0.f;
    const bool valid = a < A;
    const float qa = valid ? qb[a] : 0.f, va = valid ? v[a] : 0.f;
    if (valid) {
      for (int j0 = 0; j0 < Ts; j0 += JG) {
        float kk[JG];
#pragma unroll
        for (int k = 0; k < JG; ++k) kk[k] = j0 + k < Ts ? keys[((long)(j0 + k) * B + b) * Ap + a] : 0.f;
#pragma unroll
        for (int k = 0; k < JG; ++k) {
          const int j = j0 + k;
          if (j >= Ts) break;
          const float u = tanh_<FastMath<T>::value>(__fadd_rn(qa, kk[k]));
          const float du = __fmul_rn(__fmul_rn(de[j], va), __fsub_rn(1.f, __fmul_rn(u, u)));
          dq = __fadd_rn(dq, du);
          dva = __fadd_rn(dva, __fmul_rn(de[j], u));
        }
      }
    }
    dq_op[(long)b * Ap + a] = from_f<T>(dq);
    float* dv = dvb + (long)b * Ap + a;
    *dv = first ? dva : __fadd_rn(*dv, dva);
  }
}

// The encoder-side accumulators over the T decoder steps, after the BPTT loop, in the loop's order
// (step T−1 first, then T−2, …, 0 — the order the round-1 per-step read-modify-write used):
//   denc_j,h = Σ_i p_i,j · dctx_i,h               (blockIdx.z == 0, thread per hidden unit h)
//   dk_j,a   = Σ_i de_i,j · v_a · (1 − u_ij,a²),   u_ij,a = tanh(q_i,a + k_j,a)   (blockIdx.z == 1, per a)
// Grid ⌈max(Hp, Ap)/256⌉ × B × 2; the row's p / de of every step are staged in shared memory.
template <typename T>
__global__ void __launch_bounds__(ATT_THREADS)
    attn_acc_kernel(int T_, int B, int Ts, int Hp, int A, int Ap, const float* __restrict__ pr,
                    const float* __restrict__ de_save, const float* __restrict__ dctx_save,
                    const float* __restrict__ q, const float* __restrict__ keys, const float* __restrict__ v,
                    float* __restrict__ denc, float* __restrict__ dk) {
  extern __shared__ float sh[];   // [T][Ts] p (z = 0) or de (z = 1) of row b, then [T][256] per-thread columns
  const int b = blockIdx.y, z = blockIdx.z;
  const float* src = z == 0 ? pr : de_save;
  for (int k = threadIdx.x; k < T_ * Ts; k += ATT_THREADS) {
    const int i = k / Ts, j = k % Ts;
    sh[k] = src[((long)i * B + b) * Ts + j];
  }
  float* col = sh + T_ * Ts;      // col[i·256 + thread]: this thread's dctx_i (z = 0) or q_i (z = 1)
  const int x = blockIdx.x * ATT_THREADS + threadIdx.x;
  const int n = z == 0 ? Hp : Ap;
  if (x < n)
    for (int i = 0; i < T_; ++i)
      col[i * ATT_THREADS + threadIdx.x] =
          z == 0 ? dctx_save[((long)i * B + b) * Hp + x] : q[((long)i * B + b) * Ap + x];
  __syncthreads();
  if (x >= n) return;
  const float* cx = col + threadIdx.x;
  // four source positions j at a time: four independent accumulators (instruction-level
  // parallelism, q_i / dctx_i read once for the four), each still summed over i in the loop's order
  constexpr int JB = 4;
  if (z == 0) {
    for (int j0 = 0; j0 < Ts; j0 += JB) {
      float acc[JB];
#pragma unroll
      for (int jj = 0; jj < JB; ++jj) acc[jj] = 0.f;
      for (int i = T_ - 1; i >= 0; --i) {
        const float c = cx[i * ATT_THREADS];
#pragma unroll
        for (int jj = 0; jj < JB; ++jj) {
          if (j0 + jj >= Ts) break;
          const float add = __fmul_rn(sh[i * Ts + j0 + jj], c);
          acc[jj] = i == T_ - 1 ? add : __fadd_rn(acc[jj], add);
        }
      }
#pragma unroll
      for (int jj = 0; jj < JB; ++jj)
        if (j0 + jj < Ts) denc[((long)(j0 + jj) * B + b) * Hp + x] = acc[jj];
    }
  } else {
    const bool valid = x < A;
    const float va = valid ? v[x] : 0.f;
    for (int j0 = 0; j0 < Ts; j0 += JB) {
      float kj[JB], acc[JB];
#pragma unroll
      for (int jj = 0; jj < JB; ++jj) {
        kj[jj] = (valid && j0 + jj < Ts) ? keys[((long)(j0 + jj) * B + b) * Ap + x] : 0.f;
        acc[jj] = 0.f;
      }
      for (int i = T_ - 1; i >= 0; --i) {
        const float qi = cx[i * ATT_THREADS];
#pragma unroll
        for (int jj = 0; jj < JB; ++jj) {
          if (j0 + jj >= Ts) break;
          float du = 0.f;
          if (valid) {
            const float u = tanh_<FastMath<T>::value>(__fadd_rn(qi, kj[jj]));
            du = __fmul_rn(__fmul_rn(sh[i * Ts + j0 + jj], va), __fsub_rn(1.f, __fmul_rn(u, u)));
          }
          acc[jj] = i == T_ - 1 ? du : __fadd_rn(acc[jj], du);
        }
      }
#pragma unroll
      for (int jj = 0; jj < JB; ++jj)
        if (j0 + jj < Ts) dk[((long)(j0 + jj) * B + b) * Ap + x] = acc[jj];
    }
  }
}

void attn_acc(OT ot, int T, int B, int Ts, int Hp, int A, int Ap, const float* pr, const float* de_save,
              const float* dctx_save, const float* q, const float* keys, const float* v, float* denc, float* dk,
              cudaStream_t st) {
  const dim3 grid(cdiv(std::max(Hp, Ap), ATT_THREADS), B, 2);
  const size_t sm = (size_t)T * (Ts + ATT_THREADS) * sizeof(float);
  ASTRA_CHECK_ARG(sm <= 200 * 1024, "attn_acc: too many decoder steps for the shared-memory staging");
  if (ot == OT::BF16) {
    CUDA_TRY(cudaFuncSetAttribute(attn_acc_kernel<__nv_bfloat16>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
    attn_acc_kernel<__nv_bfloat16><<<grid, ATT_THREADS, sm, st>>>(T, B, Ts, Hp, A, Ap, pr, de_save, dctx_save, q, keys,
                                                                  v, denc, dk);
  } else {
    CUDA_TRY(cudaFuncSetAttribute(attn_acc_kernel<float>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
    attn_acc_kernel<float><<<grid, ATT_THREADS, sm, st>>>(T, B, Ts, Hp, A, Ap, pr, de_save, dctx_save, q, keys, v, denc,
                                                          dk);
  }
  LAUNCH_CHECK();
}

template <typename T, typename TDY>
static void attn_bwd_launch(int B, int Ts, int H, int Hp, int A, int Ap, const TDY* dy_ctx, long ldy,
                            const float* dctx_rec, long ldr, int ns, long ss, const float* pr, float* dp, const float* q,
                            const float* keys, const float* v, const float* enc, T* dq_op, float* dctx_save,
                            float* de_save, float* dvb, bool first, cudaStream_t st) {
  launch_pdl(attn_dp_kernel<TDY>, dim3(cdiv(Ts, ATT_THREADS / 32), B), dim3(ATT_THREADS), (size_t)Hp * sizeof(float), st, 1, B, Ts, H, Hp,
             dy_ctx, ldy, dctx_rec, ldr, ns, ss, enc, dp);
  LAUNCH_CHECK();
  launch_pdl(attn_bwd_kernel<T, TDY>, dim3(cdiv(std::max(Hp, Ap), ATT_THREADS), B), dim3(ATT_THREADS),
             (Ts + 8) * sizeof(float), st, 1, B, Ts, H, Hp, A, Ap, dy_ctx, ldy, dctx_rec, ldr, ns, ss, pr, (const float*)dp, q,
             keys, v, dq_op, dctx_save, de_save, dvb, (int)first);
  LAUNCH_CHECK();
}

void attn_bwd(OT ot, int B, int Ts, int H, int Hp, int A, int Ap, const void* dy_ctx, long ldy, bool dy_f32,
              const float* dctx_rec, long ldr, const float* pr, float* dpscratch, const float* q, const float* keys,
              const float* v, const float* enc, void* dq_op, float* dctx_save, float* de_save, float* dvb, bool first,
              cudaStream_t st, int ns, long ss) {
  ASTRA_CHECK_ARG(ns >= 1, "attn_bwd: ns must be >= 1");
  ASTRA_CHECK_ARG((size_t)Hp * sizeof(float) <= 48 * 1024, "attn_bwd: Hp too large for the staged dctx row");
  ASTRA_CHECK_ARG(Hp % 4 == 0 && ((uintptr_t)enc & 15) == 0, "attn_bwd: enc rows must be 16-byte aligned");
  if (ot == OT::BF16) {
    if (dy_f32 || !dy_ctx)
      attn_bwd_launch<__nv_bfloat16, float>(B, Ts, H, Hp, A, Ap, (const float*)dy_ctx, ldy, dctx_rec, ldr, ns, ss, pr,
                                            dpscratch, q, keys, v, enc, (__nv_bfloat16*)dq_op, dctx_save, de_save, dvb,
                                            first, st);
    else
      attn_bwd_launch<__nv_bfloat16, __nv_bfloat16>(B, Ts, H, Hp, A, Ap, (const __nv_bfloat16*)dy_ctx, ldy, dctx_rec,
                                                    ldr, ns, ss, pr, dpscratch, q, keys, v, enc, (__nv_bfloat16*)dq_op,
                                                    dctx_save, de_save, dvb, first, st);
  } else {
    attn_bwd_launch<float, float>(B, Ts, H, Hp, A, Ap, (const float*)dy_ctx, ldy, dctx_rec, ldr, ns, ss, pr, dpscratch, q,
                                  keys, v, enc, (float*)dq_op, dctx_save, de_save, dvb, first, st);
  }
}

}  // namespace astra
