// K3: additive attention step of the reduced GNMT decoder [35] (PAPER.md P:37, P:352, P:372-382,
// P:410 "mostly covered by cuDNN except the Attention module"; reading R10).
//
//   e_j = vᵀ tanh(q + k_j),  p = softmax_j(e),  ctx = Σ_j p_j enc_j          (one decoder step, per b)
//
// One CTA per batch row b; every reduction (over the attention width A for e_j and the hidden units
// for dp_j: one warp per source position, lane-strided partials + a fixed xor tree; over j for the
// softmax: warp 0, the same tree) has a fixed order, so the result is independent of launch timing (R5).  fp32 throughout (ALU/MUFU-bound).
#include "cell_math.cuh"
#include "kernels.h"
#include "pdl.cuh"

namespace astra {

constexpr int ATT_THREADS = 256;

// Fixed-order block sum of one value per thread (ATT_THREADS threads); result broadcast to all.
__device__ __forceinline__ float block_sum(float v, float* red) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, o));
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  __syncthreads();
  if (l == 0) red[w] = v;
  __syncthreads();
  float s = 0.f;
  if (threadIdx.x < 32) {
    s = threadIdx.x < ATT_THREADS / 32 ? red[threadIdx.x] : 0.f;
#pragma unroll
    for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
    if (threadIdx.x == 0) red[32] = s;
  }
  __syncthreads();
  return red[32];
}

template <typename T, typename TY>
__global__ void __launch_bounds__(ATT_THREADS)
    attn_fwd_kernel(int B, int Ts, int H, int Hp, int A, int Ap, const float* __restrict__ q,
                    const float* __restrict__ keys, const float* __restrict__ v, const float* __restrict__ enc,
                    float* __restrict__ pr, T* __restrict__ ctx_op, long ldc, TY* __restrict__ y_ctx, long ldy) {
  pdl_wait();   // chain kernel: launched with PDL (pdl.cuh)
  pdl_trigger();
  extern __shared__ float sh[];
  float* e = sh;            // [Ts]
  float* red = sh + Ts;     // [33]
  (void)red;
  const int b = blockIdx.x;
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  const float* qb = q + (long)b * Ap;
  // e_j: one warp per source position j; lane l sums a = l, l + 32, ... in order, then a fixed
  // xor-butterfly over the lanes (no block-wide barrier per j)
  for (int j = w; j < Ts; j += ATT_THREADS / 32) {
    const float* kj = keys + ((long)j * B + b) * Ap;
    float s = 0.f;
    for (int a = l; a < A; a += 32) s = __fadd_rn(s, __fmul_rn(v[a], tanh_<FastMath<T>::value>(__fadd_rn(qb[a], kj[a]))));
#pragma unroll
    for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
    if (l == 0) e[j] = s;
  }
  __syncthreads();
  if (w == 0) {   // softmax over j by warp 0: lane-strided max / sum, fixed xor trees
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
  for (int j = threadIdx.x; j < Ts; j += ATT_THREADS) pr[(long)b * Ts + j] = e[j];
  for (int h = threadIdx.x; h < Hp; h += ATT_THREADS) {
    float c = 0.f;
    if (h < H)
      for (int j = 0; j < Ts; ++j) c = __fadd_rn(c, __fmul_rn(e[j], enc[((long)j * B + b) * Hp + h]));
    ctx_op[(long)b * ldc + h] = from_f<T>(c);
    if (y_ctx && h < H) y_ctx[(long)b * ldy + h] = from_f<TY>(c);
  }
}

void attn_fwd(OT ot, int B, int Ts, int H, int Hp, int A, int Ap, const float* q, const float* keys, const float* v,
              const float* enc, float* pr, void* ctx_op, long ldc, void* y_ctx, long ldy, cudaStream_t st) {
  const size_t sm = (Ts + 40) * sizeof(float);
  if (ot == OT::BF16)
    launch_pdl(attn_fwd_kernel<__nv_bfloat16, __nv_bfloat16>, dim3(B), dim3(ATT_THREADS), sm, st, 1, 
        B, Ts, H, Hp, A, Ap, q, keys, v, enc, pr, (__nv_bfloat16*)ctx_op, ldc, (__nv_bfloat16*)y_ctx, ldy);
  else
    launch_pdl(attn_fwd_kernel<float, float>, dim3(B), dim3(ATT_THREADS), sm, st, 1, B, Ts, H, Hp, A, Ap, q, keys, v, enc, pr,
                                                              (float*)ctx_op, ldc, (float*)y_ctx, ldy);
  LAUNCH_CHECK();
}

// Backward of one attention step (oracle/cells.py attn_backward):
//   dctx = dy_ctx + dctx_rec;  dp_j = dctx·enc_j;  de_j = p_j (dp_j − Σ p dp);  denc_j += p_j dctx;
//   u_j = tanh(q + k_j);  du_j = de_j v (1 − u_j²);  dq = Σ_j du_j;  dk_j += du_j;  dv_b += Σ_j de_j u_j
template <typename T, typename TDY>
__global__ void __launch_bounds__(ATT_THREADS)
    attn_bwd_kernel(int B, int Ts, int H, int Hp, int A, int Ap, const TDY* __restrict__ dy_ctx, long ldy,
                    const float* __restrict__ dctx_rec, long ldr, const float* __restrict__ pr,
                    const float* __restrict__ q, const float* __restrict__ keys, const float* __restrict__ v,
                    const float* __restrict__ enc, T* __restrict__ dq_op, float* __restrict__ denc,
                    float* __restrict__ dk, float* __restrict__ dvb, int first) {
  pdl_wait();   // chain kernel: launched with PDL (pdl.cuh)
  pdl_trigger();
  extern __shared__ float sh[];
  float* dctx = sh;              // [Hp]
  float* de = sh + Hp;           // [Ts]
  float* red = de + Ts;          // [33]
  const int b = blockIdx.x;
  for (int h = threadIdx.x; h < Hp; h += ATT_THREADS) {
    float d = 0.f;
    if (h < H) {
      d = dy_ctx ? to_f<TDY>(dy_ctx[(long)b * ldy + h]) : 0.f;
      if (dctx_rec) d = __fadd_rn(d, dctx_rec[(long)b * ldr + h]);
    }
    dctx[h] = d;
  }
  __syncthreads();
  (void)red;
  const int w = threadIdx.x / 32, l = threadIdx.x % 32;
  for (int j = w; j < Ts; j += ATT_THREADS / 32) {   // dp_j: one warp per j, lane-strided h, xor tree
    const float* ej = enc + ((long)j * B + b) * Hp;
    float s = 0.f;
    for (int h = l; h < H; h += 32) s = __fadd_rn(s, __fmul_rn(dctx[h], ej[h]));
#pragma unroll
    for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
    if (l == 0) de[j] = s;   // dp_j for now
  }
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
  // denc_j += p_j dctx.  The accumulators (L2-resident) are read-modified-written in groups of
  // ATT_JG source positions with every load of a group issued before its stores, so a thread keeps
  // ATT_JG requests in flight instead of one dependent round trip per j.
  constexpr int ATT_JG = 10;
  for (int h = threadIdx.x; h < Hp; h += ATT_THREADS) {
    const float dc = dctx[h];
    for (int j0 = 0; j0 < Ts; j0 += ATT_JG) {
      float old[ATT_JG];
#pragma unroll
      for (int k = 0; k < ATT_JG; ++k)
        old[k] = (!first && j0 + k < Ts) ? denc[((long)(j0 + k) * B + b) * Hp + h] : 0.f;
#pragma unroll
      for (int k = 0; k < ATT_JG; ++k) {
        if (j0 + k >= Ts) break;
        const float add = __fmul_rn(pr[(long)b * Ts + j0 + k], dc);
        denc[((long)(j0 + k) * B + b) * Hp + h] = first ? add : __fadd_rn(old[k], add);
      }
    }
  }
  // attention-width terms (dq and dv accumulated in ascending j, dk_j read-modify-written in groups)
  const float* qb = q + (long)b * Ap;
  for (int a = threadIdx.x; a < Ap; a += ATT_THREADS) {
    float dq = 0.f, dva = 0.f;
    const bool valid = a < A;
    const float qa = valid ? qb[a] : 0.f, va = valid ? v[a] : 0.f;
    for (int j0 = 0; j0 < Ts; j0 += ATT_JG) {
      float old[ATT_JG], kk[ATT_JG];
#pragma unroll
      for (int k = 0; k < ATT_JG; ++k) {
        const bool in = j0 + k < Ts;
        old[k] = (!first && in) ? dk[((long)(j0 + k) * B + b) * Ap + a] : 0.f;
        kk[k] = (valid && in) ? keys[((long)(j0 + k) * B + b) * Ap + a] : 0.f;
      }
#pragma unroll
      for (int k = 0; k < ATT_JG; ++k) {
        const int j = j0 + k;
        if (j >= Ts) break;
        float du = 0.f;
        if (valid) {
          const float u = tanh_<FastMath<T>::value>(__fadd_rn(qa, kk[k]));
          du = __fmul_rn(__fmul_rn(de[j], va), __fsub_rn(1.f, __fmul_rn(u, u)));
          dq = __fadd_rn(dq, du);
          dva = __fadd_rn(dva, __fmul_rn(de[j], u));
        }
        dk[((long)j * B + b) * Ap + a] = first ? du : __fadd_rn(old[k], du);
      }
    }
    dq_op[(long)b * Ap + a] = from_f<T>(dq);
    float* dv = dvb + (long)b * Ap + a;
    *dv = first ? dva : __fadd_rn(*dv, dva);
  }
}

void attn_bwd(OT ot, int B, int Ts, int H, int Hp, int A, int Ap, const void* dy_ctx, long ldy, bool dy_f32,
              const float* dctx_rec, long ldr, const float* pr, const float* q, const float* keys, const float* v,
              const float* enc, void* dq_op, float* denc, float* dk, float* dvb, bool first, cudaStream_t st) {
  const size_t sm = (Hp + Ts + 40) * sizeof(float);
  if (ot == OT::BF16) {
    if (dy_f32 || !dy_ctx)
      launch_pdl(attn_bwd_kernel<__nv_bfloat16, float>, dim3(B), dim3(ATT_THREADS), sm, st, 1, B, Ts, H, Hp, A, Ap, (const float*)dy_ctx, ldy,
                                                                        dctx_rec, ldr, pr, q, keys, v, enc,
                                                                        (__nv_bfloat16*)dq_op, denc, dk, dvb, first);
    else
      launch_pdl(attn_bwd_kernel<__nv_bfloat16, __nv_bfloat16>, dim3(B), dim3(ATT_THREADS), sm, st, 1, 
          B, Ts, H, Hp, A, Ap, (const __nv_bfloat16*)dy_ctx, ldy, dctx_rec, ldr, pr, q, keys, v, enc,
          (__nv_bfloat16*)dq_op, denc, dk, dvb, first);
  } else {
    launch_pdl(attn_bwd_kernel<float, float>, dim3(B), dim3(ATT_THREADS), sm, st, 1, B, Ts, H, Hp, A, Ap, (const float*)dy_ctx, ldy,
                                                              dctx_rec, ldr, pr, q, keys, v, enc, (float*)dq_op, denc,
                                                              dk, dvb, first);
  }
  LAUNCH_CHECK();
}

}  // namespace astra
