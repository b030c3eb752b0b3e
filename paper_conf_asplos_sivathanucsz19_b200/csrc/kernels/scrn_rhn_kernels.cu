// Pointwise / scan kernels of the SCRN [22] and RHN [39] steps (
// equations: DESIGN.md readings R5-R9, oracle/cells.py).  The GEMM halves run on K1 (bf16 path) or
// K10 (fp32 path); these kernels are the elementwise halves.  Column partial sums (bias gradients)
// follow the fixed-order scheme of the LSTM backward kernel (R5).
#include "cell_math.cuh"
#include "kernels.h"
#include "pdl.cuh"

namespace astra {

constexpr int PW_UX = 32;  // units per CTA (a warp = 32 consecutive units of one row lane; the sums are per unit, so the CTA width never changes a bit)
constexpr int PW_RY = 8;   // row lanes per CTA
constexpr int PW_RB = 32;  // rows per CTA
int pw_row_chunks(int B) { return cdiv(B, PW_RB); }

template <typename T>
__device__ __forceinline__ float ldv(const void* p, long i) { return to_f<T>(reinterpret_cast<const T*>(p)[i]); }

// ---------------------------------------------------------------------------------- SCRN
// s_t = (1−α)·xb_t + α·s_{t−1}: one thread per (b, s), sequential over t (K8).
template <typename T, typename TY>
__global__ void scrn_scan_fwd_kernel(int B, int S, int T_, float alpha, const float* __restrict__ XB, long ldxb,
                                     const float* __restrict__ s0, float* __restrict__ Sf, int Sp,
                                     T* __restrict__ HSs, long ldhs, TY* __restrict__ y, long ldy,
                                     float* __restrict__ sT) {
  const int s = blockIdx.x * blockDim.x + threadIdx.x;
  const int b = blockIdx.y;
  if (s >= Sp) return;
  const bool valid = s < S;
  const float oma = __fsub_rn(1.f, alpha);
  float cur = (valid && s0) ? s0[(long)b * S + s] : 0.f;
  Sf[(long)b * Sp + s] = cur;
  HSs[(long)b * ldhs + s] = from_f<T>(cur);
  for (int t = 0; t < T_; ++t) {
    const long r = (long)t * B + b;
    if (valid) cur = __fadd_rn(__fmul_rn(oma, XB[r * ldxb + s]), __fmul_rn(alpha, cur));
    Sf[(r + B) * Sp + s] = cur;
    HSs[(r + B) * ldhs + s] = from_f<T>(cur);
    if (y && valid) y[r * ldy + s] = from_f<TY>(cur);
  }
  if (sT && valid) sT[(long)b * S + s] = cur;
}

void scrn_scan_fwd(OT ot, int B, int S, int Sp, int T, float alpha, const float* XB, long ldxb, const float* s0,
                   float* Sf, void* HSs, long ldhs, void* y, long ldy, float* sT, cudaStream_t st) {
  dim3 grid(cdiv(Sp, 128), B);
  if (ot == OT::BF16)
    scrn_scan_fwd_kernel<__nv_bfloat16, __nv_bfloat16><<<grid, 128, 0, st>>>(
        B, S, T, alpha, XB, ldxb, s0, Sf, Sp, (__nv_bfloat16*)HSs, ldhs, (__nv_bfloat16*)y, ldy, sT);
  else
    scrn_scan_fwd_kernel<float, float><<<grid, 128, 0, st>>>(B, S, T, alpha, XB, ldxb, s0, Sf, Sp, (float*)HSs, ldhs,
                                                             (float*)y, ldy, sT);
  LAUNCH_CHECK();
}

// h_t = σ((q_t + z_t) + b_h)   (q_t = x_t·A + s_t·P, the hoisted ladder; z_t = h_{t−1}·R)
template <typename T, typename TY>
__global__ void scrn_fwd_pw_kernel(int B, int H, int Hp, const float* __restrict__ Q, long ldq,
                                   const float* __restrict__ Z, int nsplit, long split_stride,
                                   const float* __restrict__ bh, float* __restrict__ Hf,
                                   T* __restrict__ HSh, long ldhs, TY* __restrict__ y, long ldy,
                                   float* __restrict__ hT) {
  pdl_wait();   // chain kernel: launched with PDL (pdl.cuh)
  pdl_trigger();
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  const int b = blockIdx.y;
  if (j >= Hp) return;
  float h = 0.f;
  if (j < H) {
    const float z = sum_split(Z + (long)b * Hp + j, nsplit, split_stride);   // reading R33: chunk order
    h = sigm<FastMath<T>::value>(__fadd_rn(__fadd_rn(Q[(long)b * ldq + j], z), bh[j]));
  }
  Hf[(long)b * Hp + j] = h;
  HSh[(long)b * ldhs + j] = from_f<T>(h);
  if (j < H) {
    if (y) y[(long)b * ldy + j] = from_f<TY>(h);
    if (hT) hT[(long)b * H + j] = h;
  }
}

void scrn_fwd_pw(OT ot, int B, int H, int Hp, const float* Q, long ldq, const float* Z, int nsplit, long split_stride,
                 const float* bh, float* Hf, void* HSh, long ldhs, void* y, long ldy, float* hT, cudaStream_t st) {
  dim3 grid(cdiv(Hp, 128), B);
  if (ot == OT::BF16)
    launch_pdl(scrn_fwd_pw_kernel<__nv_bfloat16, __nv_bfloat16>, dim3(grid), dim3(128), 0, st, 1, 
        B, H, Hp, Q, ldq, Z, nsplit, split_stride, bh, Hf, (__nv_bfloat16*)HSh, ldhs, (__nv_bfloat16*)y, ldy, hT);
  else
    launch_pdl(scrn_fwd_pw_kernel<float, float>, dim3(grid), dim3(128), 0, st, 1, B, H, Hp, Q, ldq, Z, nsplit, split_stride, bh, Hf, (float*)HSh, ldhs, (float*)y,
                                                           ldy, hT);
  LAUNCH_CHECK();
}

// dz_t = (dy^h_t + dh_rec)·h_t·(1 − h_t); db_h partials over rows (fixed order)
template <typename T, typename TDY>
__global__ void __launch_bounds__(PW_UX * PW_RY)
    scrn_bwd_pw_kernel(int B, int H, int Hp, const TDY* __restrict__ dy, long ldy, const float* __restrict__ dh,
                       long ld_dh, int nsplit, long split_stride, const float* __restrict__ Hf, T* __restrict__ DZ,
                       long ldz,
                       float* __restrict__ part, int first) {
  __shared__ float red[PW_RY][PW_UX];
  const int ux = threadIdx.x, ty = threadIdx.y;
  const int j = blockIdx.x * PW_UX + ux;
  const int chunk = blockIdx.y;
  // the chunk's old db_h partial (the previous step's kernel, 2 launches back): loaded before the
  // grid dependency so the final fold does not wait on a load
  const float pold = (!first && ty == 0 && j < Hp) ? part[(long)chunk * Hp + j] : 0.f;
  pdl_wait();   // chain kernel: launched with PDL (pdl.cuh)
  pdl_trigger();
  const int b0 = chunk * PW_RB, b1 = min(B, b0 + PW_RB);
  float sacc = 0.f;
  if (j < Hp) {
    for (int b = b0 + ty; b < b1; b += PW_RY) {
      float dz = 0.f;
      if (j < H) {
        float g = to_f<TDY>(dy[(long)b * ldy + j]);
        if (dh) {   // reading R33: split-K partials of dz·Rᵀ summed in chunk order, then added to dy
          g = __fadd_rn(g, sum_split(dh + (long)b * ld_dh + j, nsplit, split_stride));
        }
        const float h = Hf[(long)b * Hp + j];
        dz = __fmul_rn(__fmul_rn(g, h), __fsub_rn(1.f, h));
      }
      DZ[(long)b * ldz + j] = from_f<T>(dz);
      sacc = __fadd_rn(sacc, dz);
    }
  }
  red[ty][ux] = sacc;
  __syncthreads();
  if (ty == 0 && j < Hp) {
    float v = 0.f;
#pragma unroll
    for (int y = 0; y < PW_RY; ++y) v = __fadd_rn(v, red[y][ux]);
    part[(long)chunk * Hp + j] = first ? v : __fadd_rn(pold, v);
  }
}

void scrn_bwd_pw(OT ot, int B, int H, int Hp, const void* dy, long ldy, bool dy_f32, const float* dh, long ld_dh,
                 int nsplit, long split_stride, const float* Hf, void* DZ, long ldz, float* part, bool first,
                 cudaStream_t st) {
  dim3 grid(cdiv(Hp, PW_UX), pw_row_chunks(B)), block(PW_UX, PW_RY);
  if (ot == OT::BF16) {
    if (dy_f32)
      launch_pdl(scrn_bwd_pw_kernel<__nv_bfloat16, float>, dim3(grid), dim3(block), 0, st, 1, B, H, Hp, (const float*)dy, ldy, dh, ld_dh, nsplit, split_stride,
                                                                       Hf, (__nv_bfloat16*)DZ, ldz, part, first);
    else
      launch_pdl(scrn_bwd_pw_kernel<__nv_bfloat16, __nv_bfloat16>, dim3(grid), dim3(block), 0, st, 1, 
          B, H, Hp, (const __nv_bfloat16*)dy, ldy, dh, ld_dh, nsplit, split_stride, Hf, (__nv_bfloat16*)DZ, ldz, part, first);
  } else {
    launch_pdl(scrn_bwd_pw_kernel<float, float>, dim3(grid), dim3(block), 0, st, 1, B, H, Hp, (const float*)dy, ldy, dh, ld_dh, nsplit, split_stride, Hf,
                                                             (float*)DZ, ldz, part, first);
  }
  LAUNCH_CHECK();
}

// Reverse scan (K8): ds_t = dy^s_t + (dz_t·Pᵀ) + [t = T−1 ? ds_T : α·ds_{t+1}]; writes (1−α)·ds_t as
// the operand of dBm and dx, and ds0 = α·ds_1.
template <typename T, typename TDY>
__global__ void scrn_scan_bwd_kernel(int B, int S, int Sp, int T_, float alpha, const TDY* __restrict__ dys,
                                     long ldy, const float* __restrict__ DSP, long ldsp, const float* __restrict__ dsT,
                                     T* __restrict__ DSa, long ldsa, float* __restrict__ ds0) {
  const int s = blockIdx.x * blockDim.x + threadIdx.x;
  const int b = blockIdx.y;
  if (s >= Sp) return;
  const bool valid = s < S;
  const float oma = __fsub_rn(1.f, alpha);
  float ds = 0.f;
  for (int t = T_ - 1; t >= 0; --t) {
    const long r = (long)t * B + b;
    float v = 0.f;
    if (valid) {
      v = __fadd_rn(to_f<TDY>(dys[r * ldy + s]), DSP[r * ldsp + s]);
      const float carry = (t == T_ - 1) ? (dsT ? dsT[(long)b * S + s] : 0.f) : __fmul_rn(alpha, ds);
      v = __fadd_rn(v, carry);
    }
    ds = v;
    DSa[r * ldsa + s] = from_f<T>(__fmul_rn(oma, ds));
  }
  if (ds0 && valid) ds0[(long)b * S + s] = __fmul_rn(alpha, ds);
}

void scrn_scan_bwd(OT ot, int B, int S, int Sp, int T, float alpha, const void* dys, long ldy, bool dy_f32,
                   const float* DSP, long ldsp, const float* dsT, void* DSa, long ldsa, float* ds0, cudaStream_t st) {
  dim3 grid(cdiv(Sp, 128), B);
  if (ot == OT::BF16) {
    if (dy_f32)
      scrn_scan_bwd_kernel<__nv_bfloat16, float><<<grid, 128, 0, st>>>(B, S, Sp, T, alpha, (const float*)dys, ldy, DSP,
                                                                       ldsp, dsT, (__nv_bfloat16*)DSa, ldsa, ds0);
    else
      scrn_scan_bwd_kernel<__nv_bfloat16, __nv_bfloat16><<<grid, 128, 0, st>>>(
          B, S, Sp, T, alpha, (const __nv_bfloat16*)dys, ldy, DSP, ldsp, dsT, (__nv_bfloat16*)DSa, ldsa, ds0);
  } else {
    scrn_scan_bwd_kernel<float, float><<<grid, 128, 0, st>>>(B, S, Sp, T, alpha, (const float*)dys, ldy, DSP, ldsp,
                                                             dsT, (float*)DSa, ldsa, ds0);
  }
  LAUNCH_CHECK();
}

// ---------------------------------------------------------------------------------- RHN
// Micro-step ℓ of time t (coupled carry): a = z + b_ℓ (+ wx_t at ℓ = 0), stored back as the saved
// pre-activation; h = tanh a_H, τ = σ(a_T); s' = h·τ + s·(1 − τ).  Internal columns: g·Hp + j.
template <typename T, typename TY>
__global__ void rhn_fwd_pw_kernel(int B, int H, int Hp, float* __restrict__ Z, const float* __restrict__ Zpart,
                                  int nsplit, long split_stride, const float* __restrict__ WX,
                                  const float* __restrict__ bl, const float* __restrict__ s_prev,
                                  float* __restrict__ s_next, T* __restrict__ s_next_op, TY* __restrict__ y, long ldy,
                                  float* __restrict__ sT) {
  pdl_wait();   // chain kernel: launched with PDL (pdl.cuh)
  pdl_trigger();
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  const int b = blockIdx.y;
  if (j >= Hp) return;
  const long rz = (long)b * 2 * Hp;
  float s_new = 0.f;
  if (j < H) {
    float zH, zT;
    if (Zpart) {   // reading R33: the recurrent GEMM's split-K partials summed in chunk order
      zH = sum_split(Zpart + rz + j, nsplit, split_stride);
      zT = sum_split(Zpart + rz + Hp + j, nsplit, split_stride);
    } else {
      zH = Z[rz + j];
      zT = Z[rz + Hp + j];
    }
    float aH = __fadd_rn(zH, bl[j]);
    float aT = __fadd_rn(zT, bl[H + j]);
    if (WX) {
      aH = __fadd_rn(aH, WX[rz + j]);
      aT = __fadd_rn(aT, WX[rz + Hp + j]);
    }
    Z[rz + j] = aH;
    Z[rz + Hp + j] = aT;
    const float h = tanh_<FastMath<T>::value>(aH), tau = sigm<FastMath<T>::value>(aT);
    const float s = s_prev[(long)b * Hp + j];
    s_new = __fadd_rn(__fmul_rn(h, tau), __fmul_rn(s, __fsub_rn(1.f, tau)));
    if (y) y[(long)b * ldy + j] = from_f<TY>(s_new);
    if (sT) sT[(long)b * H + j] = s_new;
  }
  s_next[(long)b * Hp + j] = s_new;
  s_next_op[(long)b * Hp + j] = from_f<T>(s_new);
}

void rhn_fwd_pw(OT ot, int B, int H, int Hp, float* Z, const float* Zpart, int nsplit, long split_stride,
                const float* WX, const float* bl, const float* s_prev, float* s_next, void* s_next_op, void* y,
                long ldy, float* sT, cudaStream_t st) {
  dim3 grid(cdiv(Hp, 128), B);
  if (ot == OT::BF16)
    launch_pdl(rhn_fwd_pw_kernel<__nv_bfloat16, __nv_bfloat16>, dim3(grid), dim3(128), 0, st, 1, 
        B, H, Hp, Z, Zpart, nsplit, split_stride, WX, bl, s_prev, s_next, (__nv_bfloat16*)s_next_op, (__nv_bfloat16*)y, ldy, sT);
  else
    launch_pdl(rhn_fwd_pw_kernel<float, float>, dim3(grid), dim3(128), 0, st, 1, B, H, Hp, Z, Zpart, nsplit, split_stride, WX, bl, s_prev, s_next, (float*)s_next_op,
                                                          (float*)y, ldy, sT);
  LAUNCH_CHECK();
}

// Backward of micro-step ℓ:  ds = ds_in (+ dy_t at ℓ = L−1); dh = ds·τ; dτ = ds·(h − s_prev);
// da_H = dh·(1 − h²); da_T = dτ·τ·(1 − τ); ds_out = ds·(1 − τ) (the BPTT GEMM then adds da·R_ℓᵀ).
template <typename T, typename TDY>
__global__ void __launch_bounds__(PW_UX * PW_RY)
    rhn_bwd_pw_kernel(int B, int H, int Hp, const float* __restrict__ ds_in, const float* __restrict__ ds_part,
                      int nsplit, long split_stride, const TDY* __restrict__ dy, long ldy,
                      const float* __restrict__ Apre, const float* __restrict__ s_prev, T* __restrict__ DA,
                      float* __restrict__ ds_out, float* __restrict__ part, int first) {
  constexpr int NR = PW_RB / PW_RY;   // rows per thread: b0 + ty, b0 + ty + PW_RY, … (in this order)
  __shared__ float red[PW_RY][2][PW_UX];
  const int ux = threadIdx.x, ty = threadIdx.y;
  const int j = blockIdx.x * PW_UX + ux;
  const int chunk = blockIdx.y;
  const int b0 = chunk * PW_RB, b1 = min(B, b0 + PW_RB);
  const bool unit = j < H;
  // every operand of the thread's rows is loaded before the arithmetic (one memory latency, not NR);
  // the saved forward tensors, dy and the carry are older than the grid dependency: loaded before
  // it, except at the first micro-step (ds_part == null), whose predecessor initialised the carry
  float aH[NR], aT[NR], sp[NR], dsv[NR], dyv[NR];
  auto load_old = [&] {
#pragma unroll
    for (int k = 0; k < NR; ++k) {
      const int b = b0 + ty + k * PW_RY;
      const bool ok = unit && b < b1;
      const long rz = (long)b * 2 * Hp;
      aH[k] = ok ? Apre[rz + j] : 0.f;
      aT[k] = ok ? Apre[rz + Hp + j] : 0.f;
      sp[k] = ok ? s_prev[(long)b * Hp + j] : 0.f;
      dsv[k] = ok ? ds_in[(long)b * Hp + j] : 0.f;
      dyv[k] = (ok && dy) ? to_f<TDY>(dy[(long)b * ldy + j]) : 0.f;
    }
  };
  const bool early = ds_part != nullptr;
  if (early) load_old();
  // this chunk's old db partial (written by an earlier micro-step's kernel, ≥ 2 launches back):
  // loaded now so the final fold does not wait on a load
  float pold = 0.f;
  if (!first && ty < 2 && j < Hp) pold = part[(long)chunk * 2 * Hp + ty * Hp + j];
  pdl_wait();   // chain kernel: launched with PDL (pdl.cuh)
  pdl_trigger();
  if (!early) load_old();
  float pz[NR];   // the BPTT GEMM's split-K partials (this launch's dependency), summed in chunk order
#pragma unroll
  for (int k = 0; k < NR; ++k) {
    const int b = b0 + ty + k * PW_RY;
    pz[k] = (ds_part && unit && b < b1) ? sum_split(ds_part + (long)b * Hp + j, nsplit, split_stride) : 0.f;
  }
  float sH = 0.f, sT_ = 0.f;
  if (j < Hp) {
#pragma unroll
    for (int k = 0; k < NR; ++k) {
      const int b = b0 + ty + k * PW_RY;
      if (b >= b1) break;
      const long rz = (long)b * 2 * Hp;
      float daH = 0.f, daT = 0.f, dso = 0.f;
      if (unit) {
        float ds = dsv[k];
        if (ds_part) ds = __fadd_rn(ds, pz[k]);   // reading R33: carry + the partials in chunk order
        if (dy) ds = __fadd_rn(dyv[k], ds);
        const float h = tanh_<FastMath<T>::value>(aH[k]), tau = sigm<FastMath<T>::value>(aT[k]);
        const float dh = __fmul_rn(ds, tau);
        const float dtau = __fmul_rn(ds, __fsub_rn(h, sp[k]));
        daH = __fmul_rn(dh, __fsub_rn(1.f, __fmul_rn(h, h)));
        daT = __fmul_rn(__fmul_rn(dtau, tau), __fsub_rn(1.f, tau));
        dso = __fmul_rn(ds, __fsub_rn(1.f, tau));
      }
      DA[rz + j] = from_f<T>(daH);
      DA[rz + Hp + j] = from_f<T>(daT);
      ds_out[(long)b * Hp + j] = dso;
      sH = __fadd_rn(sH, daH);
      sT_ = __fadd_rn(sT_, daT);
    }
  }
  red[ty][0][ux] = sH;
  red[ty][1][ux] = sT_;
  __syncthreads();
  if (ty < 2 && j < Hp) {
    float v = 0.f;
#pragma unroll
    for (int y = 0; y < PW_RY; ++y) v = __fadd_rn(v, red[y][ty][ux]);
    part[(long)chunk * 2 * Hp + ty * Hp + j] = first ? v : __fadd_rn(pold, v);
  }
}

void rhn_bwd_pw(OT ot, int B, int H, int Hp, const float* ds_in, const float* ds_part, int nsplit, long split_stride,
                const void* dy, long ldy, bool dy_f32, const float* Apre, const float* s_prev, void* DA,
                float* ds_out, float* part, bool first, cudaStream_t st) {
  dim3 grid(cdiv(Hp, PW_UX), pw_row_chunks(B)), block(PW_UX, PW_RY);
  if (ot == OT::BF16) {
    if (dy_f32 || !dy)
      launch_pdl(rhn_bwd_pw_kernel<__nv_bfloat16, float>, dim3(grid), dim3(block), 0, st, 1, B, H, Hp, ds_in, ds_part, nsplit, split_stride, (const float*)dy, ldy, Apre,
                                                                      s_prev, (__nv_bfloat16*)DA, ds_out, part, first);
    else
      launch_pdl(rhn_bwd_pw_kernel<__nv_bfloat16, __nv_bfloat16>, dim3(grid), dim3(block), 0, st, 1, 
          B, H, Hp, ds_in, ds_part, nsplit, split_stride, (const __nv_bfloat16*)dy, ldy, Apre, s_prev,
          (__nv_bfloat16*)DA, ds_out, part, first);
  } else {
    launch_pdl(rhn_bwd_pw_kernel<float, float>, dim3(grid), dim3(block), 0, st, 1, B, H, Hp, ds_in, ds_part, nsplit, split_stride, (const float*)dy, ldy, Apre, s_prev,
                                                            (float*)DA, ds_out, part, first);
  }
  LAUNCH_CHECK();
}

// out[q·Hq + j] (external, j < H) = Σ_chunk part[chunk][q·Hp_ + j] in chunk order, for q < nq blocks.
__global__ void reduce_blocked_partials_kernel(const float* __restrict__ part, int nchunk, int nq, int H, int Hp_,
                                               float* __restrict__ out) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= nq * H) return;
  const int q = e / H, j = e % H;
  float s = 0.f;
  for (int c = 0; c < nchunk; ++c) s = __fadd_rn(s, part[(long)c * nq * Hp_ + q * Hp_ + j]);
  out[e] = s;
}

void reduce_blocked_partials(const float* part, int nchunk, int nq, int H, int Hp, float* out, cudaStream_t st) {
  reduce_blocked_partials_kernel<<<cdiv((long)nq * H, 256), 256, 0, st>>>(part, nchunk, nq, H, Hp, out);
  LAUNCH_CHECK();
}

// dst[g·Hp + j][k] = src[k][g·H + j] for a gate-blocked [K][G·H] matrix (mirror rows, padding zero).
template <typename T>
__global__ void mirror_blocked_T_kernel(const float* __restrict__ src, int K, int G, int H, int Hp,
                                        T* __restrict__ dst, long ldd) {
  __shared__ float tile[32][33];
  const int r0 = blockIdx.x * 32, k0 = blockIdx.y * 32;
  const int tx = threadIdx.x, ty = threadIdx.y;
  for (int i = ty; i < 32; i += 8) {
    const int k = k0 + i, r = r0 + tx;
    const int g = r / Hp, j = r % Hp;
    tile[i][tx] = (k < K && g < G && j < H) ? src[(long)k * G * H + g * H + j] : 0.f;
  }
  __syncthreads();
  for (int i = ty; i < 32; i += 8) {
    const int r = r0 + i, k = k0 + tx;
    if (r < G * Hp && k < ldd) dst[(long)r * ldd + k] = from_f<T>(tile[tx][i]);
  }
}

void mirror_blocked_T(OT ot, const float* src, int K, int G, int H, int Hp, void* dst, long ldd, cudaStream_t st) {
  dim3 grid(cdiv((long)G * Hp, 32), cdiv(ldd, 32)), block(32, 8);
  if (ot == OT::BF16)
    mirror_blocked_T_kernel<__nv_bfloat16><<<grid, block, 0, st>>>(src, K, G, H, Hp, (__nv_bfloat16*)dst, ldd);
  else
    mirror_blocked_T_kernel<float><<<grid, block, 0, st>>>(src, K, G, H, Hp, (float*)dst, ldd);
  LAUNCH_CHECK();
}

}  // namespace astra
