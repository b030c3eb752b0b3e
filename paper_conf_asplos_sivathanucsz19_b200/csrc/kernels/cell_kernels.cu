// Pointwise cell kernels (unfused halves of K2/K4), K5 fixed-order reductions, K6 embedding,
// K7 cross-entropy, K9 SGD and operand mirrors.
#include "cell_math.cuh"
#include "lstm_bwd_row.cuh"
#include "kernels.h"
#include "pdl.cuh"
#include "gemm.h"
#include "sm100.cuh"
#include <algorithm>
#include <cstdlib>
#include <map>
#include <mutex>
#include <tuple>

namespace astra {

// two adjacent elements in one store (float2 / bf16 pair)
template <typename T>
__device__ __forceinline__ void store2(T* p, float a, float b);
template <>
__device__ __forceinline__ void store2<float>(float* p, float a, float b) {
  *reinterpret_cast<float2*>(p) = make_float2(a, b);
}
template <>
__device__ __forceinline__ void store2<__nv_bfloat16>(__nv_bfloat16* p, float a, float b) {
  *reinterpret_cast<__nv_bfloat162*>(p) = __floats2bfloat162_rn(a, b);
}

// ============================================================================ mirrors
template <typename T>
__global__ void mirror_gates_T_kernel(const float* __restrict__ src, int K, int H, int Hp, T* __restrict__ dst,
                                      long ldd, long kcols, int gu) {
  // tile 32 (k) x 32 (internal rows r); dst[r][k] = src[k][ext(r)]
  __shared__ float tile[32][33];
  const int r0 = blockIdx.x * 32, k0 = blockIdx.y * 32;
  const int tx = threadIdx.x, ty = threadIdx.y;  // 32 x 8
  for (int i = ty; i < 32; i += 8) {
    const int k = k0 + i, r = r0 + tx;
    const int tileu = r / (4 * gu), g = (r % (4 * gu)) / gu, j = tileu * gu + r % gu;
    float v = 0.f;
    if (k < K && j < H) v = src[(long)k * 4 * H + g * H + j];
    tile[i][tx] = v;
  }
  __syncthreads();
  for (int i = ty; i < 32; i += 8) {
    const int r = r0 + i, k = k0 + tx;
    if (r < 4 * Hp && k < kcols) dst[(long)r * ldd + k] = from_f<T>(tile[tx][i]);
  }
}

// Same mapping, tile 32 internal rows x 64 k: a thread stores two adjacent k (one 4-byte bf16 pair,
// a warp one 128-byte run of a dst row) instead of one 2-byte element.  Same per-element rounding.
template <typename T>
__global__ void mirror_gates_T2_kernel(const float* __restrict__ src, int K, int H, int Hp, T* __restrict__ dst,
                                       long ldd, long kcols, int gu) {
  __shared__ float tile[64][33];
  const int r0 = blockIdx.x * 32, k0 = blockIdx.y * 64;
  const int tx = threadIdx.x, ty = threadIdx.y;  // 32 x 8
  const int r = r0 + tx;
  const int tileu = r / (4 * gu), g = (r % (4 * gu)) / gu, j = tileu * gu + r % gu;
  for (int i = ty; i < 64; i += 8) {
    const int k = k0 + i;
    tile[i][tx] = (k < K && j < H) ? src[(long)k * 4 * H + g * H + j] : 0.f;
  }
  __syncthreads();
  for (int i = ty; i < 32; i += 8) {
    const int rr = r0 + i, k = k0 + 2 * tx;
    if (rr < 4 * Hp && k < kcols) store2<T>(dst + (long)rr * ldd + k, tile[2 * tx][i], tile[2 * tx + 1][i]);
  }
}

// Same mapping, tile = one 64-unit gate block (64 internal rows) x 64 k: float4 loads of the 64
// consecutive source columns g·H + j0 … (H % 4 == 0), 4 consecutive k per thread on the store side.
template <typename T>
__global__ void __launch_bounds__(256) mirror_gates_T4_kernel(const float* __restrict__ src, int K, int H, int Hp,
                                                              T* __restrict__ dst, long ldd, long kcols, int gu) {
  __shared__ float tile[64][65];
  const int rb = blockIdx.x, k0 = blockIdx.y * 64, tid = threadIdx.x;
  // a 64-row block lies inside one gate of one unit block (gu is a multiple of 64)
  const int r0 = rb * 64, g = (r0 % (4 * gu)) / gu, j0 = (r0 / (4 * gu)) * gu + r0 % gu;
#pragma unroll
  for (int jj = 0; jj < 4; ++jj) {
    const int kl = tid / 16 + 16 * jj, q = tid % 16, k = k0 + kl, j = j0 + 4 * q;
    float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
    if (k < K && j < H) x = *reinterpret_cast<const float4*>(src + (long)k * 4 * H + (long)g * H + j);
    tile[kl][4 * q] = x.x;
    tile[kl][4 * q + 1] = x.y;
    tile[kl][4 * q + 2] = x.z;
    tile[kl][4 * q + 3] = x.w;
  }
  __syncthreads();
#pragma unroll
  for (int jj = 0; jj < 4; ++jj) {
    const int nl = tid / 16 + 16 * jj, q = tid % 16, r = r0 + nl, k = k0 + 4 * q;
    if (r >= 4 * Hp || k >= kcols) continue;
    T* d = dst + (long)r * ldd + k;
    if (k + 4 <= kcols) {
      if constexpr (sizeof(T) == 2) {
        __nv_bfloat162 lo = __floats2bfloat162_rn(tile[4 * q][nl], tile[4 * q + 1][nl]);
        __nv_bfloat162 hi = __floats2bfloat162_rn(tile[4 * q + 2][nl], tile[4 * q + 3][nl]);
        uint2 u;
        u.x = *reinterpret_cast<uint32_t*>(&lo);
        u.y = *reinterpret_cast<uint32_t*>(&hi);
        *reinterpret_cast<uint2*>(d) = u;
      } else {
        *reinterpret_cast<float4*>(d) =
            make_float4(tile[4 * q][nl], tile[4 * q + 1][nl], tile[4 * q + 2][nl], tile[4 * q + 3][nl]);
      }
    } else {
      for (int i = 0; k + i < kcols; ++i) d[i] = from_f<T>(tile[4 * q + i][nl]);
    }
  }
}

void mirror_gates_T(OT ot, const float* src, int K, int H, int Hp, void* dst, long ldd, cudaStream_t st, long kcols,
                    int gu) {
  if (kcols < 0) kcols = ldd;
  ASTRA_CHECK_ARG(gu % 64 == 0 && gu > 0 && (gu == GATE_U || gu == Hp), "mirror_gates_T: gate layout must be GATE_U or Hp");
  const size_t e = ot == OT::BF16 ? 2 : 4;
  if (H % 4 == 0 && ldd % 4 == 0 && Hp % GATE_U == 0 && ((uintptr_t)src & 15) == 0 &&
      ((uintptr_t)dst & (4 * e - 1)) == 0) {
    dim3 grid(4 * Hp / 64, cdiv(kcols, 64));
    if (ot == OT::BF16)
      mirror_gates_T4_kernel<__nv_bfloat16><<<grid, 256, 0, st>>>(src, K, H, Hp, (__nv_bfloat16*)dst, ldd, kcols, gu);
    else
      mirror_gates_T4_kernel<float><<<grid, 256, 0, st>>>(src, K, H, Hp, (float*)dst, ldd, kcols, gu);
    LAUNCH_CHECK();
    return;
  }
  if (kcols % 2 == 0 && ldd % 2 == 0) {
    dim3 grid(cdiv(4L * Hp, 32), cdiv(kcols, 64)), block(32, 8);
    if (ot == OT::BF16)
      mirror_gates_T2_kernel<__nv_bfloat16><<<grid, block, 0, st>>>(src, K, H, Hp, (__nv_bfloat16*)dst, ldd, kcols, gu);
    else
      mirror_gates_T2_kernel<float><<<grid, block, 0, st>>>(src, K, H, Hp, (float*)dst, ldd, kcols, gu);
    LAUNCH_CHECK();
    return;
  }
  dim3 grid(cdiv(4L * Hp, 32), cdiv(kcols, 32)), block(32, 8);
  if (ot == OT::BF16)
    mirror_gates_T_kernel<__nv_bfloat16><<<grid, block, 0, st>>>(src, K, H, Hp, (__nv_bfloat16*)dst, ldd, kcols, gu);
  else
    mirror_gates_T_kernel<float><<<grid, block, 0, st>>>(src, K, H, Hp, (float*)dst, ldd, kcols, gu);
  LAUNCH_CHECK();
}

template <typename T>
__global__ void mirror_T_kernel(const float* __restrict__ src, int K, int N, int Np, int Kp, T* __restrict__ dst,
                                long ldd) {
  __shared__ float tile[32][33];
  const int n0 = blockIdx.x * 32, k0 = blockIdx.y * 32;
  const int tx = threadIdx.x, ty = threadIdx.y;
  for (int i = ty; i < 32; i += 8) {
    const int k = k0 + i, n = n0 + tx;
    tile[i][tx] = (k < K && n < N) ? src[(long)k * N + n] : 0.f;
  }
  __syncthreads();
  for (int i = ty; i < 32; i += 8) {
    const int n = n0 + i, k = k0 + tx;
    if (n < Np && k < Kp) dst[(long)n * ldd + k] = from_f<T>(tile[tx][i]);
  }
}

// 64×64 tiles, float4 loads (N % 4 == 0), 4 consecutive k per thread on the store side
template <typename T>
__global__ void __launch_bounds__(256) mirror_T4_kernel(const float* __restrict__ src, int K, int N, int Np, int Kp,
                                                        T* __restrict__ dst, long ldd) {
  __shared__ float tile[64][65];
  const int n0 = blockIdx.x * 64, k0 = blockIdx.y * 64, tid = threadIdx.x;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int kl = tid / 16 + 16 * j, q = tid % 16, k = k0 + kl, n = n0 + 4 * q;
    float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
    if (k < K && n < N) x = *reinterpret_cast<const float4*>(src + (long)k * N + n);
    tile[kl][4 * q] = x.x;
    tile[kl][4 * q + 1] = x.y;
    tile[kl][4 * q + 2] = x.z;
    tile[kl][4 * q + 3] = x.w;
  }
  __syncthreads();
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int nl = tid / 16 + 16 * j, q = tid % 16, n = n0 + nl, k = k0 + 4 * q;
    if (n >= Np || k >= Kp) continue;
    T* d = dst + (long)n * ldd + k;
    if (k + 4 <= Kp) {
      if constexpr (sizeof(T) == 2) {
        __nv_bfloat162 lo = __floats2bfloat162_rn(tile[4 * q][nl], tile[4 * q + 1][nl]);
        __nv_bfloat162 hi = __floats2bfloat162_rn(tile[4 * q + 2][nl], tile[4 * q + 3][nl]);
        uint2 u;
        u.x = *reinterpret_cast<uint32_t*>(&lo);
        u.y = *reinterpret_cast<uint32_t*>(&hi);
        *reinterpret_cast<uint2*>(d) = u;
      } else {
        *reinterpret_cast<float4*>(d) =
            make_float4(tile[4 * q][nl], tile[4 * q + 1][nl], tile[4 * q + 2][nl], tile[4 * q + 3][nl]);
      }
    } else {
      for (int i = 0; k + i < Kp; ++i) d[i] = from_f<T>(tile[4 * q + i][nl]);
    }
  }
}

void mirror_T(OT ot, const float* src, int K, int N, int Np, int Kp, void* dst, long ldd, cudaStream_t st) {
  const size_t e = ot == OT::BF16 ? 2 : 4;
  if (N % 4 == 0 && ldd % 4 == 0 && ((uintptr_t)src & 15) == 0 && ((uintptr_t)dst & (4 * e - 1)) == 0) {
    dim3 grid(cdiv(Np, 64), cdiv(Kp, 64));
    if (ot == OT::BF16)
      mirror_T4_kernel<__nv_bfloat16><<<grid, 256, 0, st>>>(src, K, N, Np, Kp, (__nv_bfloat16*)dst, ldd);
    else
      mirror_T4_kernel<float><<<grid, 256, 0, st>>>(src, K, N, Np, Kp, (float*)dst, ldd);
    LAUNCH_CHECK();
    return;
  }
  dim3 grid(cdiv(Np, 32), cdiv(Kp, 32)), block(32, 8);
  if (ot == OT::BF16)
    mirror_T_kernel<__nv_bfloat16><<<grid, block, 0, st>>>(src, K, N, Np, Kp, (__nv_bfloat16*)dst, ldd);
  else
    mirror_T_kernel<float><<<grid, block, 0, st>>>(src, K, N, Np, Kp, (float*)dst, ldd);
  LAUNCH_CHECK();
}

__global__ void transpose_bf16_kernel(const __nv_bfloat16* __restrict__ src, int rows, int cols,
                                      __nv_bfloat16* __restrict__ dst) {
  __shared__ __nv_bfloat16 tile[32][34];
  const long base = (long)blockIdx.z * rows * cols;
  const int c0 = blockIdx.x * 32, r0 = blockIdx.y * 32, tx = threadIdx.x, ty = threadIdx.y;
  for (int i = ty; i < 32; i += 8) {
    const int r = r0 + i, c = c0 + tx;
    tile[i][tx] = (r < rows && c < cols) ? src[base + (long)r * cols + c] : __float2bfloat16_rn(0.f);
  }
  __syncthreads();
  for (int i = ty; i < 32; i += 8) {
    const int c = c0 + i, r = r0 + tx;
    if (c < cols && r < rows) dst[base + (long)c * rows + r] = tile[tx][i];
  }
}

void transpose_bf16(const void* src, int nb, int rows, int cols, void* dst, cudaStream_t st) {
  dim3 grid(cdiv(cols, 32), cdiv(rows, 32), nb), block(32, 8);
  transpose_bf16_kernel<<<grid, block, 0, st>>>((const __nv_bfloat16*)src, rows, cols, (__nv_bfloat16*)dst);
  LAUNCH_CHECK();
}

template <typename TD, typename TS>
__global__ void copy_pad_kernel(const TS* __restrict__ src, long rows, int cols, long lds, TD* __restrict__ dst,
                                long ldd, long dcols) {
  const long r = blockIdx.y;
  for (long c = blockIdx.x * blockDim.x + threadIdx.x; c < dcols; c += (long)gridDim.x * blockDim.x) {
    float v = (c < cols && src) ? to_f<TS>(src[r * lds + c]) : 0.f;
    dst[r * ldd + c] = from_f<TD>(v);
  }
}

void copy_pad(OT ot, const void* src, OT src_ot, long rows, int cols, long lds, void* dst, long ldd, cudaStream_t st,
              long dcols) {
  if (rows == 0) return;
  if (dcols < 0) dcols = ldd;
  ASTRA_CHECK_ARG(rows < 65536L * 32768L, "copy_pad: too many rows");
  // grid.y is limited to 65535: fold rows into chunks
  const long ychunk = 65535;
  for (long r0 = 0; r0 < rows; r0 += ychunk) {
    const long nr = rows - r0 < ychunk ? rows - r0 : ychunk;
    dim3 grid(cdiv(dcols, 256) < 8 ? cdiv(dcols, 256) : 8, (unsigned)nr);
    const size_t es = ot_size(src_ot), ed = ot_size(ot);
    const char* s = (const char*)src + (src ? r0 * lds * es : 0);
    char* d = (char*)dst + r0 * ldd * ed;
    if (ot == OT::BF16 && src_ot == OT::BF16)
      copy_pad_kernel<__nv_bfloat16, __nv_bfloat16><<<grid, 256, 0, st>>>((const __nv_bfloat16*)(src ? s : nullptr), nr, cols, lds, (__nv_bfloat16*)d, ldd, dcols);
    else if (ot == OT::BF16)
      copy_pad_kernel<__nv_bfloat16, float><<<grid, 256, 0, st>>>((const float*)(src ? s : nullptr), nr, cols, lds, (__nv_bfloat16*)d, ldd, dcols);
    else if (src_ot == OT::BF16)
      copy_pad_kernel<float, __nv_bfloat16><<<grid, 256, 0, st>>>((const __nv_bfloat16*)(src ? s : nullptr), nr, cols, lds, (float*)d, ldd, dcols);
    else
      copy_pad_kernel<float, float><<<grid, 256, 0, st>>>((const float*)(src ? s : nullptr), nr, cols, lds, (float*)d, ldd, dcols);
    LAUNCH_CHECK();
  }
}

void copy_f32_pad(const float* src, long rows, int cols, long lds, float* dst, long ldd, int dcols, cudaStream_t st) {
  // dst has `dcols` used columns (≤ ldd); columns ≥ cols are zero
  (void)dcols;
  copy_pad(OT::F32, src, OT::F32, rows, cols, lds, dst, ldd, st);
}

// ============================================================================ LSTM-family pointwise
// K2 forward half, streamed through shared memory by the TMA engine.  Work item = one batch row
// x one block of FB_UB hidden units: its gate pre-activations WX and UH (gate-interleaved, so the
// block is one contiguous FB_UB·4-float run of each) and c_{t-1} are fetched with three 1-D bulk
// copies into a FB_STAGES-deep ring, so every SM keeps ~100 KB of loads in flight with a handful
// of instructions; the 256 threads then read their 2 units per gate from shared memory.  Each CTA
// keeps one unit block (its gate parameters staged once in shared memory) and walks rows
// b_first, b_first + rstep, ...  Arithmetic per element is the same as the plain kernel.
template <typename T>
__device__ __forceinline__ void store2cs(T* p, float a, float b);
template <>
__device__ __forceinline__ void store2cs<float>(float* p, float a, float b) {
  __stcs(reinterpret_cast<float2*>(p), make_float2(a, b));
}
template <>
__device__ __forceinline__ void store2cs<__nv_bfloat16>(__nv_bfloat16* p, float a, float b) {
  __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
  __stcs(reinterpret_cast<unsigned int*>(p), *reinterpret_cast<unsigned int*>(&v));
}

constexpr int FB_UB = 512;
constexpr int FB_THREADS = 256;
constexpr int FB_STAGES = 4;
constexpr int FB_SW = FB_UB * 4 * 4;           // bytes of one row block of WX (or UH)
constexpr int FB_STAGE = 2 * FB_SW + FB_UB * 4;

struct FwdPwArgs {
  int B, H, Hp, nub, rstep;
  int gu;                      // gate layout (cell_math.cuh gcol_u): GATE_U interleaved, Hp gate-blocked
  const float* WX;
  const float* UH;
  GateParams gp;
  const float* c_prev;
  float* c_new;
  void* h_op;
  long ldh;
  void* y;
  long ldy;
  float* hT;
  float* cT;
  unsigned long long* trace;   // diagnostics (astra_debug_set_trace): [grid][2 + 2·16] globaltimer stamps
};

__device__ __forceinline__ unsigned long long gtime_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

template <typename T>
__device__ __forceinline__ void store_pair(T* p, bool vec, float a, float b, bool ok1) {
  if (vec) {
    store2<T>(p, a, b);
  } else {
    p[0] = from_f<T>(a);
    if (ok1) p[1] = from_f<T>(b);
  }
}

template <int KIND, typename T, typename TY, bool BLK>
__global__ void __launch_bounds__(FB_THREADS, 3) lstm_fwd_pw_kernel(const FwdPwArgs a) {
  constexpr int NP = KIND == K_MILSTM ? 4 : 1;
  extern __shared__ __align__(128) uint8_t sm[];
  uint64_t* full = reinterpret_cast<uint64_t*>(sm + FB_STAGES * FB_STAGE);
  const int tid = threadIdx.x;
  const int ub = blockIdx.x % a.nub, b_first = blockIdx.x / a.nub;
  const int u0 = ub * FB_UB, nu = min(FB_UB, a.Hp - u0);   // nu: multiple of 64
  const long NG = 4L * a.Hp;
  const int nitems = b_first < a.B ? (a.B - b_first + a.rstep - 1) / a.rstep : 0;
  const uint32_t wbytes = (uint32_t)nu * 16, cbytes = (uint32_t)nu * 4;
  // WX_t (the a1 GEMM's output) and c_{t-1} (the previous pointwise kernel's, complete before the
  // GEMM of this step released us) are older than the grid dependency: their copies for the first
  // stages go out before griddepcontrol.wait; UH_t (the GEMM's output) after it.
  // interleaved layout: the CTA's units' four gates are one contiguous run of 4·nu columns; gate-
  // blocked: four runs of nu columns (g·Hp + u0), landed at gate offsets g·FB_UB of the stage
  constexpr bool blk = BLK;   // the `alloc` layout at compile time (interleaved: folded offsets)
  auto load_gates = [&](uint32_t dst, const float* row, uint64_t* bar) {
    if (!blk) {
      sm100::bulk_load(dst, row + (long)u0 * 4, wbytes, bar);
    } else {
#pragma unroll
      for (int g = 0; g < 4; ++g) sm100::bulk_load(dst + g * FB_UB * 4, row + (long)g * a.Hp + u0, cbytes, bar);
    }
  };
  auto issue_old = [&](int k) {
    const int s = k % FB_STAGES;
    const long b = b_first + (long)k * a.rstep;
    uint8_t* st = sm + s * FB_STAGE;
    sm100::mbar_arrive_expect_tx(&full[s], 2 * wbytes + cbytes);
    load_gates(sm100::smem_u32(st), a.WX + b * NG, &full[s]);
    sm100::bulk_load(sm100::smem_u32(st + 2 * FB_SW), a.c_prev + b * a.Hp + u0, cbytes, &full[s]);
  };
  auto issue_new = [&](int k) {
    const int s = k % FB_STAGES;
    const long b = b_first + (long)k * a.rstep;
    load_gates(sm100::smem_u32(sm + s * FB_STAGE + FB_SW), a.UH + b * NG, &full[s]);
  };
  unsigned long long* tr = a.trace ? a.trace + (size_t)blockIdx.x * 34 : nullptr;
  if (tr && tid == 0) tr[0] = gtime_ns();
  if (tid == 0) {
    for (int s = 0; s < FB_STAGES; ++s) sm100::mbar_init(&full[s], 1);
    sm100::fence_barrier_init();
    for (int k = 0; k < FB_STAGES && k < nitems; ++k) issue_old(k);
  }
  pdl_wait();
  pdl_trigger();
  if (tr && tid == 0) tr[1] = gtime_ns();
  if (tid == 0)
    for (int k = 0; k < FB_STAGES && k < nitems; ++k) issue_new(k);
  __syncthreads();   // the ring's barriers are initialised
  const int ul = 2 * tid;
  const bool act = ul < nu;
  const int base = blk ? ul : (ul / 64) * 256 + ul % 64;
  const int gstride = blk ? FB_UB : 64;   // stage offset between a unit's gates
  const bool vh = (a.ldh & 1) == 0, vy = (a.ldy & 1) == 0;
  // this thread's units keep their gate parameters in registers for all its rows (loaded straight
  // from the external vectors: no shared staging, so three CTAs fit on an SM)
  float pb[2][4], pal[2][4], pb1[2][4], pb2[2][4];
#pragma unroll
  for (int u = 0; u < 2; ++u)
#pragma unroll
    for (int g = 0; g < 4; ++g) {
      const int j = u0 + ul + u, e = g * a.H + j;
      const bool ok = act && j < a.H;
      pb[u][g] = ok ? a.gp.b[e] : 0.f;
      pal[u][g] = (ok && KIND == K_MILSTM) ? a.gp.alpha[e] : 0.f;
      pb1[u][g] = (ok && KIND == K_MILSTM) ? a.gp.beta1[e] : 0.f;
      pb2[u][g] = (ok && KIND == K_MILSTM) ? a.gp.beta2[e] : 0.f;
    }
  for (int k = 0; k < nitems; ++k) {
    const int s = k % FB_STAGES;
    sm100::mbar_wait(&full[s], (uint32_t)((k / FB_STAGES) & 1));
    if (tr && tid == 0 && k < 16) tr[2 + 2 * k] = gtime_ns();
    const long b = b_first + (long)k * a.rstep;
    if (act) {
      const float* sw = reinterpret_cast<const float*>(sm + s * FB_STAGE);
      const float* su = sw + FB_UB * 4;
      const float* sc = su + FB_UB * 4;
      float2 wx[4], uh[4];
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        wx[g] = *reinterpret_cast<const float2*>(sw + base + g * gstride);
        uh[g] = *reinterpret_cast<const float2*>(su + base + g * gstride);
      }
      const float2 cp = *reinterpret_cast<const float2*>(sc + ul);
      float cv[2], hv[2];
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        const int j = u0 + ul + u;
        if (j < a.H) {
          float pa[4];
#pragma unroll
          for (int g = 0; g < 4; ++g)
            pa[g] = preact<KIND, FastMath<T>::value>(u ? wx[g].y : wx[g].x, u ? uh[g].y : uh[g].x, pb[u][g], pal[u][g], pb1[u][g],
                                 pb2[u][g]);
          cell_fwd<KIND, FastMath<T>::value>(pa, u ? cp.y : cp.x, cv[u], hv[u]);
        } else {   // padding units stay exactly zero
          cv[u] = 0.f;
          hv[u] = 0.f;
        }
      }
      const int j = u0 + ul;
      const int bi = (int)b;   // one step's rows: B·max(Hp, ldh, ldy) < 2^31 (checked by the launcher)
      *reinterpret_cast<float2*>(a.c_new + (bi * a.Hp + j)) = make_float2(cv[0], cv[1]);
      store_pair<T>(reinterpret_cast<T*>(a.h_op) + (bi * (int)a.ldh + j), vh, hv[0], hv[1], true);
      if (a.y) {
        const bool ok0 = j < a.H || a.ldy >= a.Hp, ok1 = j + 1 < a.H || a.ldy >= a.Hp;
        if (ok0) store_pair<TY>(reinterpret_cast<TY*>(a.y) + (bi * (int)a.ldy + j), vy && ok1, hv[0], hv[1], ok1);
      }
      if (a.hT || a.cT) {   // the last step only
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          if (j + u >= a.H) break;
          if (a.hT) a.hT[(long)b * a.H + j + u] = hv[u];
          if (a.cT) a.cT[(long)b * a.H + j + u] = cv[u];
        }
      }
    }
    __syncthreads();   // stage s fully consumed
    if (tr && tid == 0 && k < 16) tr[3 + 2 * k] = gtime_ns();
    if (tid == 0 && k + FB_STAGES < nitems) {
      sm100::fence_proxy_async_smem();
      issue_old(k + FB_STAGES);
      issue_new(k + FB_STAGES);
    }
  }
}

template <int KIND, typename T>
static void fwd_pw_launch(OT y_ot, int B, int H, int Hp, const float* WX, const float* UH, GateParams gp,
                          const float* c_prev, float* c_new, void* h_op, long ldh, void* y, long ldy, float* hT,
                          float* cT, cudaStream_t st, int gu) {
  FwdPwArgs a;
  a.B = B; a.H = H; a.Hp = Hp;
  ASTRA_CHECK_ARG(gu == GATE_U || gu == Hp, "lstm_fwd_pointwise: gate layout must be GATE_U or Hp");
  a.gu = gu;
  ASTRA_CHECK_ARG((long)B * std::max({(long)Hp, ldh, ldy}) < (1L << 31), "lstm_fwd_pointwise: one step's rows must have < 2^31 elements");
  const bool blk = gu != GATE_U;
  a.nub = cdiv(Hp, FB_UB);
  static const int cap = [] {   // A/B knob: CTAs of one launch (row_streams experiments)
    const char* e = std::getenv("ASTRA_FWDPW_CTAS");
    return e ? std::atoi(e) : 0;
  }();
  a.rstep = std::max(1, std::min(B, (cap > 0 ? cap : 3 * num_sms()) / a.nub));
  a.WX = WX; a.UH = UH; a.gp = gp; a.c_prev = c_prev; a.c_new = c_new;
  a.h_op = h_op; a.ldh = ldh; a.y = y; a.ldy = ldy; a.hT = hT; a.cT = cT;
  a.trace = trace_buffer(TRACE_FWD_PW);   // diagnostics only (null: no stamps)
  const int np = KIND == K_MILSTM ? 4 : 1;
  (void)np;
  const size_t smem = (size_t)FB_STAGES * FB_STAGE + FB_STAGES * 8;
  const dim3 grid(a.nub * a.rstep);
  if (y_ot == OT::BF16) {
    auto k = blk ? lstm_fwd_pw_kernel<KIND, T, __nv_bfloat16, true> : lstm_fwd_pw_kernel<KIND, T, __nv_bfloat16, false>;
    static bool attr[2] = {false, false};
    if (!attr[blk]) { CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)); attr[blk] = true; }
    launch_pdl(k, grid, dim3(FB_THREADS), smem, st, 1, a);
  } else {
    auto k = blk ? lstm_fwd_pw_kernel<KIND, T, float, true> : lstm_fwd_pw_kernel<KIND, T, float, false>;
    static bool attr[2] = {false, false};
    if (!attr[blk]) { CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)); attr[blk] = true; }
    launch_pdl(k, grid, dim3(FB_THREADS), smem, st, 1, a);
  }
  LAUNCH_CHECK();
}

void lstm_fwd_pointwise(int kind, OT ot, int B, int H, int Hp, const float* WX, const float* UH, GateParams gp,
                        const float* c_prev, float* c_new, void* h_op, long ldh, void* y, long ldy, OT y_ot,
                        float* hT, float* cT, cudaStream_t st, int gu) {
#define FWD_CASE(K)                                                                                          \
  if (kind == K) {                                                                                           \
    if (ot == OT::BF16)                                                                                      \
      fwd_pw_launch<K, __nv_bfloat16>(y_ot, B, H, Hp, WX, UH, gp, c_prev, c_new, h_op, ldh, y, ldy, hT, cT, st, gu); \
    else                                                                                                     \
      fwd_pw_launch<K, float>(y_ot, B, H, Hp, WX, UH, gp, c_prev, c_new, h_op, ldh, y, ldy, hT, cT, st, gu);      \
    return;                                                                                                  \
  }
  FWD_CASE(K_LSTM)
  FWD_CASE(K_MILSTM)
  FWD_CASE(K_SUBLSTM)
#undef FWD_CASE
  throw Error(ASTRA_E_UNSUPPORTED, "lstm_fwd_pointwise: kind");
}

static unsigned long long* g_trace[TRACE_KINDS] = {nullptr, nullptr, nullptr, nullptr};
unsigned long long* trace_buffer(int kind) { return kind >= 0 && kind < TRACE_KINDS ? g_trace[kind] : nullptr; }
void set_trace_buffer(int kind, unsigned long long* buf) {
  ASTRA_CHECK_ARG(kind >= 0 && kind < TRACE_KINDS, "debug_set_trace: unknown kind");
  g_trace[kind] = buf;
}

int lstm_bwd_row_chunks(int B) { return cdiv(B, BWD_RB); }

// K4 backward half + K5 column partials (unfused variant).  CTA = 64 hidden units (all four gates)
// x 32 batch rows; thread (tx, ty) owns unit u0 + tx (its 4 gates' parameters in registers) for
// rows b0 + ty, b0 + ty + 4, ...; a warp reads 128-byte runs of every gate's pre-activations.  The
// row arithmetic and the column-sum order are lstm_bwd_row.cuh's, shared with the fused BPTT kernel.
// 256-thread CTAs at <= 64 registers: one resident wave at B = 512.
template <int KIND, typename T, typename TDY, bool BLK, int NS>
__global__ void __launch_bounds__(BWD_UX * BWD_RY, 4)
    lstm_bwd_pw_kernel(int B, int H, int Hp, const TDY* __restrict__ dy, long ldy, const float* __restrict__ dh_rec,
                       long ld_dh, int nsplit, long split_stride, float* __restrict__ dc,
                       const float* __restrict__ WX, const float* __restrict__ UH, const float* __restrict__ c_new,
                       const float* __restrict__ c_prev, GateParams gp, T* __restrict__ D_uh,
                       T* __restrict__ D_wx, float* __restrict__ partials, int nq, int first, int gu) {
  constexpr int NV = BwdNV<KIND>::value;
  constexpr int NP = KIND == K_MILSTM ? 4 : 1;   // gate parameter sets: b (and α, β1, β2)
  __shared__ float red[BWD_RY][NV][BWD_UX];
  __shared__ float sgp[NP][4][BWD_UX];   // staged once; re-read per row so they hold no registers
  __shared__ float spre[NV][BWD_UX];     // the chunk's old column-sum partials (prefetched)
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int j = blockIdx.x * BWD_UX + tx;
  if (ty < NP) {   // parameters are not written by the chain: staged before the grid dependency
    const float* src = ty == 0 ? gp.b : ty == 1 ? gp.alpha : ty == 2 ? gp.beta1 : gp.beta2;
#pragma unroll
    for (int g = 0; g < 4; ++g) sgp[ty][g][tx] = j < H ? src[g * H + j] : 0.f;
  }
  const int chunk = blockIdx.y;
  const int NG = 4 * Hp;
  const int b0 = chunk * BWD_RB, b1 = min(B, b0 + BWD_RB);
  // gate stride of the `alloc` layout: the interleaved one is a compile-time 64 (folded into the
  // address offsets), the gate-blocked one Hp
  const int gs = BLK ? gu : GATE_U;
  const int c0 = BLK ? j : gcol(0, j);   // gate g of unit j at column c0 + g·gs
  // the previous step's partials of this chunk (written two launches back: complete) — loaded now,
  // so the final fold does not wait on a load after the row loop
  if (!first && j < Hp)
    for (int i = ty; i < NV; i += BWD_RY)
      if (i / 4 < nq) spre[i][tx] = partials[(long)chunk * nq * NG + (long)(i / 4) * NG + c0 + (i % 4) * gs];
  // Per-thread 32-bit element offsets of the first row (one step's tensors: B·4Hp < 2^31, checked by
  // the launcher), advanced by BWD_RY rows per iteration: the row loop's address arithmetic is an
  // add per operand instead of fresh 64-bit products, without holding nine 64-bit pointers
  const int bf = b0 + ty;
  int o_ng = bf * NG + c0, o_hp = bf * Hp + j, o_dy = bf * (int)ldy + j, o_dh = bf * (int)ld_dh + j;
  const int st_ng = BWD_RY * NG, st_hp = BWD_RY * Hp, st_dy = BWD_RY * (int)ldy, st_dh = BWD_RY * (int)ld_dh;
  // Operands of one row.  Only dh_rec is produced by the predecessor (the BPTT GEMM); WX, UH, the
  // cell states and dy are older, and dc was written by the pointwise kernel two launches back
  // (complete: the GEMM waits on it before triggering this launch).  So the first row is loaded
  // before the grid dependency resolves — by the CTAs already resident beside the GEMM.  Not at the
  // first step (`first`): its predecessor may be the kernel that initialised dc or produced dy.
  const bool early = !first;
  float w[4], h[4], dcv = 0.f, cp = 0.f, cn = 0.f, dyv = 0.f;
  auto load_row = [&] {
#pragma unroll
    for (int g = 0; g < 4; ++g) {
      w[g] = __ldcs(WX + o_ng + g * gs);
      h[g] = __ldcs(UH + o_ng + g * gs);
    }
    dcv = dc[o_hp];
    cp = c_prev[o_hp];
    cn = c_new[o_hp];
    dyv = to_f<TDY>(dy[o_dy]);
  };
  if (early && j < H && bf < b1) load_row();
  pdl_wait();
  pdl_trigger();
  __syncthreads();
  float acc[NV];
#pragma unroll
  for (int i = 0; i < NV; ++i) acc[i] = 0.f;
  if (j < H) {
#pragma unroll 1
    for (int b = bf; b < b1; b += BWD_RY) {
      // every operand of the row is loaded before any arithmetic: one memory latency per row
      if (!early || b != bf) load_row();
      float dh = dyv;
      if (dh_rec)   // split-K partials of dh_rec summed in chunk order, then added to dy
        dh = __fadd_rn(dh, sum_split_n<NS>(dh_rec + o_dh, nsplit, split_stride));
      float bb[4], al[4], be1[4], be2[4];
      const volatile float* sg = &sgp[0][0][tx];   // volatile: re-read each row, not hoisted into registers
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        bb[g] = sg[g * BWD_UX];
        al[g] = KIND == K_MILSTM ? sg[(NP > 1 ? 4 : 0) * BWD_UX + g * BWD_UX] : 0.f;
        be1[g] = KIND == K_MILSTM ? sg[(NP > 2 ? 8 : 0) * BWD_UX + g * BWD_UX] : 0.f;
        be2[g] = KIND == K_MILSTM ? sg[(NP > 3 ? 12 : 0) * BWD_UX + g * BWD_UX] : 0.f;
      }
      lstm_bwd_row<KIND, T>(w, h, dh, dcv, cp, cn, bb, al, be1, be2, acc, D_uh + o_ng, D_wx + o_ng, gs);
      dc[o_hp] = dcv;
      o_ng += st_ng; o_hp += st_hp; o_dy += st_dy; o_dh += st_dh;
    }
  } else if (j < Hp) {  // padding units: keep their gradients exactly zero
    for (int b = bf; b < b1; b += BWD_RY) {
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        D_uh[(long)b * NG + c0 + g * gs] = from_f<T>(0.f);
        if (KIND == K_MILSTM) D_wx[(long)b * NG + c0 + g * gs] = from_f<T>(0.f);
      }
      dc[(long)b * Hp + j] = 0.f;
    }
  }
#pragma unroll
  for (int i = 0; i < NV; ++i) red[ty][i][tx] = acc[i];
  __syncthreads();
  if (j >= Hp) return;
  bwd_chunk_finalize<NV>(red, tx, ty, partials + (long)chunk * nq * NG, NG, c0, nq, first, gs, spre);
}

// K4 backward half, wide form (AV bwd_pw = 1; measured faster at small batch — B = 64: BPTT chain
// 2.37 → 1.96 ms at cfg5 shapes — and slower at B = 512, where the row-lane kernel above fills the
// GPU in one wave).  Same row
// arithmetic and the same R5 column-sum order, different work split: CTA = one 32-row partial chunk
// x 32 units, thread = (row, 4 consecutive units), so every operand of a row is one 16-byte load per
// gate (float4 WX / UH / dh partials / dc / c) and all 32 rows of the chunk are in flight at once
// (the row-per-thread-lane kernel walks 8 rows one after another and is memory-latency bound).
// The per-row contributions (da, and for MI-LSTM wx, uh) go to shared memory; then thread (unit,
// gate, lane y) runs lane y's fixed-order accumulation over rows y, y+4, ..., y+28 exactly as the
// other kernel's thread (tx = unit, ty = y) does, and the lanes are combined in y order.
constexpr int BW2_UB = 32;                   // units per CTA
constexpr int BW2_THREADS = BWD_RB * BW2_UB / 4;   // 256: 32 rows x 8 unit quads

template <typename TDY>
__device__ __forceinline__ void load4_dy(const TDY* p, bool vec, float (&v)[4], int nvalid);
template <>
__device__ __forceinline__ void load4_dy<float>(const float* p, bool vec, float (&v)[4], int nvalid) {
  if (vec) {
    const float4 x = __ldcs(reinterpret_cast<const float4*>(p));
    v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
  } else {
#pragma unroll
    for (int u = 0; u < 4; ++u) v[u] = u < nvalid ? p[u] : 0.f;
  }
}
template <>
__device__ __forceinline__ void load4_dy<__nv_bfloat16>(const __nv_bfloat16* p, bool vec, float (&v)[4], int nvalid) {
  if (vec) {
    const uint2 x = *reinterpret_cast<const uint2*>(p);
    const __nv_bfloat162 a = *reinterpret_cast<const __nv_bfloat162*>(&x.x), b = *reinterpret_cast<const __nv_bfloat162*>(&x.y);
    v[0] = __low2float(a); v[1] = __high2float(a); v[2] = __low2float(b); v[3] = __high2float(b);
  } else {
#pragma unroll
    for (int u = 0; u < 4; ++u) v[u] = u < nvalid ? __bfloat162float(p[u]) : 0.f;
  }
}
__device__ __forceinline__ float4 ld4(const float* p) { return *reinterpret_cast<const float4*>(p); }
__device__ __forceinline__ float4 ld4cs(const float* p) { return __ldcs(reinterpret_cast<const float4*>(p)); }
__device__ __forceinline__ float f4(const float4& v, int u) { return u == 0 ? v.x : u == 1 ? v.y : u == 2 ? v.z : v.w; }
template <typename T>
__device__ __forceinline__ void store4(T* p, const float (&v)[4]);
template <>
__device__ __forceinline__ void store4<float>(float* p, const float (&v)[4]) {
  *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
}
template <>
__device__ __forceinline__ void store4<__nv_bfloat16>(__nv_bfloat16* p, const float (&v)[4]) {
  __nv_bfloat162 a = __floats2bfloat162_rn(v[0], v[1]), b = __floats2bfloat162_rn(v[2], v[3]);
  uint2 x;
  x.x = *reinterpret_cast<uint32_t*>(&a);
  x.y = *reinterpret_cast<uint32_t*>(&b);
  *reinterpret_cast<uint2*>(p) = x;
}

template <int KIND, typename T, typename TDY>
__global__ void __launch_bounds__(BW2_THREADS, 2)
    lstm_bwd_pw2_kernel(int B, int H, int Hp, const TDY* __restrict__ dy, long ldy, const float* __restrict__ dh_rec,
                        long ld_dh, int nsplit, long split_stride, float* __restrict__ dc,
                        const float* __restrict__ WX, const float* __restrict__ UH, const float* __restrict__ c_new,
                        const float* __restrict__ c_prev, GateParams gp, T* __restrict__ D_uh,
                        T* __restrict__ D_wx, float* __restrict__ partials, int nq, int first, int gu) {
  constexpr int NV = BwdNV<KIND>::value;
  constexpr int NP = KIND == K_MILSTM ? 4 : 1;
  constexpr int NC = KIND == K_MILSTM ? 3 : 1;    // per (row, unit, gate): da (, wx, uh)
  constexpr bool F = FastMath<T>::value;
  extern __shared__ float smf[];
  float* con = smf;                                // [NC][4][32 rows][BW2_UB]; later red [4][NV][BW2_UB]
  float* sgp = smf + NC * 4 * BWD_RB * BW2_UB;     // [NP][4][BW2_UB]
  const int tid = threadIdx.x;
  const int qd = tid % (BW2_UB / 4), r = tid / (BW2_UB / 4);
  const int u0 = blockIdx.x * BW2_UB, ul = 4 * qd, j0 = u0 + ul;
  const int chunk = blockIdx.y, b0 = chunk * BWD_RB, b = b0 + r;
  const long NG = 4L * Hp;
  for (int i = tid; i < NP * 4 * BW2_UB; i += BW2_THREADS) {   // parameters: not written by the chain
    const int pi = i / (4 * BW2_UB), g = (i / BW2_UB) % 4, u = i % BW2_UB, j = u0 + u;
    const float* src = pi == 0 ? gp.b : pi == 1 ? gp.alpha : pi == 2 ? gp.beta1 : gp.beta2;
    sgp[i] = j < H ? src[g * H + j] : 0.f;
  }
  const bool rowok = b < B;
  const int nvalid = min(4, H - j0);            // units of this quad that exist (≤ 0: padding only)
  const int c0 = gcol_u(0, j0, gu);   // gate g of the quad's units at c0 + g·gu
  const long ro = (long)b * Hp + j0;
  // everything except the GEMM's dh_rec is older than the grid dependency: loaded before the wait
  // (not at the first step, whose predecessor may have produced dy or initialised dc)
  float4 w4[4], h4[4], dc4, cp4, cn4;
  float dyv[4];
  auto load_old = [&] {
#pragma unroll
    for (int g = 0; g < 4; ++g) {
      w4[g] = ld4cs(WX + (long)b * NG + c0 + g * gu);
      h4[g] = ld4cs(UH + (long)b * NG + c0 + g * gu);
    }
    dc4 = ld4(dc + ro);
    cp4 = ld4cs(c_prev + ro);
    cn4 = ld4cs(c_new + ro);
    load4_dy<TDY>(dy + (long)b * ldy + j0, (ldy % 4 == 0) && nvalid == 4 && ((uintptr_t)dy % (4 * sizeof(TDY))) == 0,
                  dyv, nvalid);
  };
  const bool early = !first;
  if (early && rowok && nvalid > 0) load_old();
  pdl_wait();
  pdl_trigger();
  if (!early && rowok && nvalid > 0) load_old();
  __syncthreads();   // parameters staged
  if (rowok) {
    float duh4[4][4], dwx4[4][4], dcn[4];   // [unit][gate]
    auto put = [&](int u, int g, float da, float w, float h) {   // this row's column-sum contribution
      con[((0 * 4 + g) * BWD_RB + r) * BW2_UB + ul + u] = da;
      if (KIND == K_MILSTM) {
        con[((1 * 4 + g) * BWD_RB + r) * BW2_UB + ul + u] = w;
        con[((2 * 4 + g) * BWD_RB + r) * BW2_UB + ul + u] = h;
      }
    };
    if (nvalid > 0) {
      float dh[4];
      if (dh_rec) {   // split-K partials of dh_rec summed in chunk order, then added to dy
        const bool vec = nvalid == 4 && (ld_dh % 4) == 0 && (split_stride % 4) == 0 && ((uintptr_t)dh_rec & 15) == 0;
        if (vec) {
          float4 pv[SPLIT_MAX];
#pragma unroll
          for (int k = 0; k < SPLIT_MAX; ++k) pv[k] = k < nsplit ? ld4(dh_rec + (long)b * ld_dh + j0 + k * split_stride) : make_float4(0, 0, 0, 0);
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            float s = f4(pv[0], u);
#pragma unroll
            for (int k = 1; k < SPLIT_MAX; ++k)
              if (k < nsplit) s = __fadd_rn(s, f4(pv[k], u));
            for (int k = SPLIT_MAX; k < nsplit; ++k) s = __fadd_rn(s, dh_rec[(long)b * ld_dh + j0 + u + k * split_stride]);
            dh[u] = __fadd_rn(dyv[u], s);
          }
        } else {
#pragma unroll
          for (int u = 0; u < 4; ++u)
            dh[u] = u < nvalid ? __fadd_rn(dyv[u], sum_split(dh_rec + (long)b * ld_dh + j0 + u, nsplit, split_stride)) : 0.f;
        }
      } else {
#pragma unroll
        for (int u = 0; u < 4; ++u) dh[u] = dyv[u];
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        float w[4], h[4], bb[4], al[4], be1[4], be2[4], da[4], duh[4], dwx[4];
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          w[g] = f4(w4[g], u);
          h[g] = f4(h4[g], u);
          bb[g] = sgp[g * BW2_UB + ul + u];
          al[g] = KIND == K_MILSTM ? sgp[(NP > 1 ? 1 : 0) * 4 * BW2_UB + g * BW2_UB + ul + u] : 0.f;
          be1[g] = KIND == K_MILSTM ? sgp[(NP > 2 ? 2 : 0) * 4 * BW2_UB + g * BW2_UB + ul + u] : 0.f;
          be2[g] = KIND == K_MILSTM ? sgp[(NP > 3 ? 3 : 0) * 4 * BW2_UB + g * BW2_UB + ul + u] : 0.f;
        }
        float dcv = f4(dc4, u);
        if (u < nvalid) {
          lstm_bwd_da<KIND, F>(w, h, dh[u], dcv, f4(cp4, u), f4(cn4, u), bb, al, be1, be2, da, duh, dwx);
        } else {   // padding units: exact zeros everywhere (gradients, contributions, dc)
#pragma unroll
          for (int g = 0; g < 4; ++g) { da[g] = 0.f; duh[g] = 0.f; dwx[g] = 0.f; w[g] = 0.f; h[g] = 0.f; }
          dcv = 0.f;
        }
        dcn[u] = dcv;
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          put(u, g, da[g], w[g], h[g]);
          duh4[u][g] = duh[g]; dwx4[u][g] = dwx[g];
        }
      }
    } else {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        dcn[u] = 0.f;
#pragma unroll
        for (int g = 0; g < 4; ++g) { put(u, g, 0.f, 0.f, 0.f); duh4[u][g] = 0.f; dwx4[u][g] = 0.f; }
      }
    }
    // outputs: D_uh / D_wx per gate (4 units = one 8- or 16-byte store), dc
#pragma unroll
    for (int g = 0; g < 4; ++g) {
      float v[4] = {duh4[0][g], duh4[1][g], duh4[2][g], duh4[3][g]};
      store4<T>(D_uh + (long)b * NG + c0 + g * gu, v);
      if (KIND == K_MILSTM) {
        float x[4] = {dwx4[0][g], dwx4[1][g], dwx4[2][g], dwx4[3][g]};
        store4<T>(D_wx + (long)b * NG + c0 + g * gu, x);
      }
    }
    *reinterpret_cast<float4*>(dc + ro) = make_float4(dcn[0], dcn[1], dcn[2], dcn[3]);
  }
  __syncthreads();
  // lane sums: thread (u, y) accumulates rows y, y+4, ... of the chunk in ascending order, every gate
  const int nrows = min(BWD_RB, B - b0);
  float acc[NV];
#pragma unroll
  for (int i = 0; i < NV; ++i) acc[i] = 0.f;
  const int su = tid % BW2_UB, sy = tid / BW2_UB;   // tid < 4·BW2_UB = 128 do the sums
  if (tid < BWD_RY * BW2_UB) {
    for (int rr = sy; rr < nrows; rr += BWD_RY) {
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        const float da = con[((0 * 4 + g) * BWD_RB + rr) * BW2_UB + su];
        const float w = KIND == K_MILSTM ? con[((1 * 4 + g) * BWD_RB + rr) * BW2_UB + su] : 0.f;
        const float h = KIND == K_MILSTM ? con[((2 * 4 + g) * BWD_RB + rr) * BW2_UB + su] : 0.f;
        lstm_bwd_acc<KIND, F>(acc, g, da, w, h);
      }
    }
  }
  __syncthreads();   // contributions consumed: the same memory holds the lane sums
  float* red = con;  // [4 lanes][NV][BW2_UB]
  if (tid < BWD_RY * BW2_UB) {
#pragma unroll
    for (int i = 0; i < NV; ++i) red[(sy * NV + i) * BW2_UB + su] = acc[i];
  }
  __syncthreads();
  // lanes combined in y order and folded into the chunk's partials (bwd_chunk_finalize's order)
  for (int item = tid; item < NV * BW2_UB; item += BW2_THREADS) {
    const int u = item % BW2_UB, i = item / BW2_UB, j = u0 + u;
    const int q = i / 4, g = i % 4;
    if (q >= nq || j >= Hp) continue;
    float v = 0.f;
#pragma unroll
    for (int y = 0; y < BWD_RY; ++y) v = __fadd_rn(v, red[(y * NV + i) * BW2_UB + u]);
    float* pp = partials + (long)chunk * nq * NG + (long)q * NG + gcol_u(g, j, gu);
    *pp = first ? v : __fadd_rn(*pp, v);
  }
}

// K4 backward half, TMA-tiled form (AV bwd_pw = 2; large batch).  The wide form's work split (CTA =
// one 32-row partial chunk x 32 units, thread = row x 4 units) and arithmetic (lstm_bwd_da, then the
// R5 column sums replayed in the row-lane kernel's order: the same bits), but every operand tile is
// landed in shared memory by the copy engine — WX_t / UH_t (4 gate boxes each), c_t, c_{t-1}, dc,
// dy (boxes of 32 rows x 32 units, fp32) and the nsplit dh_rec partials — so no register holds a
// load in flight: 2 CTAs per SM, each CTA's whole tile (64 KB at cfg5) requested at once, all the
// older operands (and the chunk's column-sum partials) before the grid dependency resolves.  The
// replay reads w, h from the operand tiles (only da is staged).
struct Bw3Maps {
  CUtensorMap wx, uh, p, dc, cp, cn, dy;   // fp32 [rows][cols] boxes {32, 32}; p: z = split chunk
};
constexpr int BW3_TILE = BWD_RB * BW2_UB;   // floats of one [32 rows][32 units] box
constexpr int BW3_FLOATS = (4 + 4 + SPLIT_MAX + 4 + 4) * BW3_TILE + 4 * 4 * BW2_UB;   // + params
constexpr size_t BW3_SMEM = (size_t)BW3_FLOATS * 4 + 128 + 64;

template <int KIND, typename T>
__global__ void __launch_bounds__(BW2_THREADS, 2)
    lstm_bwd_pw3_kernel(const __grid_constant__ Bw3Maps m, int B, int H, int Hp, int nsplit, int gu,
                        float* __restrict__ dc, GateParams gp, T* __restrict__ D_uh, T* __restrict__ D_wx,
                        float* __restrict__ partials, int nq, int first) {
  constexpr int NV = BwdNV<KIND>::value;
  constexpr int NP = KIND == K_MILSTM ? 4 : 1;
  constexpr bool F = FastMath<T>::value;
  extern __shared__ uint8_t sm3_raw[];
  float* smf = reinterpret_cast<float*>((reinterpret_cast<uintptr_t>(sm3_raw) + 127) & ~uintptr_t(127));
  float* sWX = smf;                          // [4 gates][32 rows][32 units]
  float* sUH = sWX + 4 * BW3_TILE;
  float* sP = sUH + 4 * BW3_TILE;            // [nsplit][32][32]
  float* sDC = sP + SPLIT_MAX * BW3_TILE;
  float* sCP = sDC + BW3_TILE;
  float* sCN = sCP + BW3_TILE;
  float* sDY = sCN + BW3_TILE;
  float* sDA = sDY + BW3_TILE;               // [4 gates][32][32] da; later the lane sums
  float* sgp = sDA + 4 * BW3_TILE;           // [NP][4][32]
  uint64_t* bar = reinterpret_cast<uint64_t*>(sgp + 4 * 4 * BW2_UB);   // [0] older operands, [1] dh_rec
  const int tid = threadIdx.x;
  const int qd = tid % (BW2_UB / 4), r = tid / (BW2_UB / 4);
  const int u0 = blockIdx.x * BW2_UB, ul = 4 * qd, j0 = u0 + ul;
  const int chunk = blockIdx.y, b0 = chunk * BWD_RB, b = b0 + r;
  const long NG = 4L * Hp;
  const int cg0 = gcol_u(0, u0, gu);         // gate g of the tile's 32 units: columns cg0 + g·gu ..
  constexpr uint32_t BOX = BW3_TILE * 4;
  auto issue_old = [&] {
    sm100::mbar_arrive_expect_tx(&bar[0], 12 * BOX);
#pragma unroll
    for (int g = 0; g < 4; ++g) {
      sm100::tma_load_3d(sWX + g * BW3_TILE, &m.wx, &bar[0], cg0 + g * gu, b0, 0);
      sm100::tma_load_3d(sUH + g * BW3_TILE, &m.uh, &bar[0], cg0 + g * gu, b0, 0);
    }
    sm100::tma_load_3d(sDC, &m.dc, &bar[0], u0, b0, 0);
    sm100::tma_load_3d(sCP, &m.cp, &bar[0], u0, b0, 0);
    sm100::tma_load_3d(sCN, &m.cn, &bar[0], u0, b0, 0);
    sm100::tma_load_3d(sDY, &m.dy, &bar[0], u0, b0, 0);
  };
  if (tid == 0) {
    sm100::mbar_init(&bar[0], 1);
    sm100::mbar_init(&bar[1], 1);
    sm100::fence_barrier_init();
    sm100::tma_prefetch(&m.wx); sm100::tma_prefetch(&m.uh); sm100::tma_prefetch(&m.p);
  }
  __syncthreads();
  // the previous step's column-sum partials of this chunk (written two launches back: complete)
  float pre[2] = {0.f, 0.f};
  for (int k = 0, item = tid; item < NV * BW2_UB; item += BW2_THREADS, ++k) {
    const int u = item % BW2_UB, i = item / BW2_UB, j = u0 + u, q = i / 4, g = i % 4;
    if (!first && q < nq && j < Hp) pre[k] = partials[(long)chunk * nq * NG + (long)q * NG + gcol_u(g, j, gu)];
  }
  // operands older than the grid dependency: all but dh_rec (not at the first step, whose
  // predecessor may have produced dy or initialised dc)
  if (tid == 0 && !first) issue_old();
  for (int i = tid; i < NP * 4 * BW2_UB; i += BW2_THREADS) {   // parameters: not written by the chain
    const int pi = i / (4 * BW2_UB), g = (i / BW2_UB) % 4, u = i % BW2_UB, j = u0 + u;
    const float* src = pi == 0 ? gp.b : pi == 1 ? gp.alpha : pi == 2 ? gp.beta1 : gp.beta2;
    sgp[i] = j < H ? src[g * H + j] : 0.f;
  }
  pdl_wait();
  pdl_trigger();
  if (tid == 0) {
    if (first) issue_old();
    sm100::mbar_arrive_expect_tx(&bar[1], (uint32_t)nsplit * BOX);
    for (int k = 0; k < nsplit; ++k) sm100::tma_load_3d(sP + k * BW3_TILE, &m.p, &bar[1], u0, b0, k);
  }
  __syncthreads();   // parameters staged
  sm100::mbar_wait(&bar[0], 0);
  sm100::mbar_wait(&bar[1], 0);
  const bool rowok = b < B;
  const int nvalid = min(4, H - j0);
  const int c0 = gcol_u(0, j0, gu);
  const long ro = (long)b * Hp + j0;
  const int so = r * BW2_UB + ul;            // this thread's offset in a [32][32] tile
  if (rowok) {
    float duh4[4][4], dwx4[4][4], dcn[4];
    if (nvalid > 0) {
      float4 w4[4], h4[4];
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        w4[g] = *reinterpret_cast<const float4*>(sWX + g * BW3_TILE + so);
        h4[g] = *reinterpret_cast<const float4*>(sUH + g * BW3_TILE + so);
      }
      const float4 dc4 = *reinterpret_cast<const float4*>(sDC + so);
      const float4 cp4 = *reinterpret_cast<const float4*>(sCP + so);
      const float4 cn4 = *reinterpret_cast<const float4*>(sCN + so);
      const float4 dy4 = *reinterpret_cast<const float4*>(sDY + so);
      float4 pv[SPLIT_MAX];
#pragma unroll
      for (int k = 0; k < SPLIT_MAX; ++k)
        pv[k] = k < nsplit ? *reinterpret_cast<const float4*>(sP + k * BW3_TILE + so) : make_float4(0, 0, 0, 0);
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        // split-K partials of dh_rec summed in chunk order, then added to dy (the other forms' order)
        float sacc = f4(pv[0], u);
#pragma unroll
        for (int k = 1; k < SPLIT_MAX; ++k)
          if (k < nsplit) sacc = __fadd_rn(sacc, f4(pv[k], u));
        const float dh = __fadd_rn(f4(dy4, u), sacc);
        float w[4], h[4], bb[4], al[4], be1[4], be2[4], da[4], duh[4], dwx[4];
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          w[g] = f4(w4[g], u);
          h[g] = f4(h4[g], u);
          bb[g] = sgp[g * BW2_UB + ul + u];
          al[g] = KIND == K_MILSTM ? sgp[(NP > 1 ? 1 : 0) * 4 * BW2_UB + g * BW2_UB + ul + u] : 0.f;
          be1[g] = KIND == K_MILSTM ? sgp[(NP > 2 ? 2 : 0) * 4 * BW2_UB + g * BW2_UB + ul + u] : 0.f;
          be2[g] = KIND == K_MILSTM ? sgp[(NP > 3 ? 3 : 0) * 4 * BW2_UB + g * BW2_UB + ul + u] : 0.f;
        }
        float dcv = f4(dc4, u);
        if (u < nvalid) {
          lstm_bwd_da<KIND, F>(w, h, dh, dcv, f4(cp4, u), f4(cn4, u), bb, al, be1, be2, da, duh, dwx);
        } else {   // padding units: exact zeros everywhere
#pragma unroll
          for (int g = 0; g < 4; ++g) { da[g] = 0.f; duh[g] = 0.f; dwx[g] = 0.f; }
          dcv = 0.f;
        }
        dcn[u] = dcv;
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          sDA[g * BW3_TILE + so + u] = da[g];
          duh4[u][g] = duh[g]; dwx4[u][g] = dwx[g];
        }
      }
    } else {
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        dcn[u] = 0.f;
#pragma unroll
        for (int g = 0; g < 4; ++g) { sDA[g * BW3_TILE + so + u] = 0.f; duh4[u][g] = 0.f; dwx4[u][g] = 0.f; }
      }
    }
#pragma unroll
    for (int g = 0; g < 4; ++g) {
      float v[4] = {duh4[0][g], duh4[1][g], duh4[2][g], duh4[3][g]};
      store4<T>(D_uh + (long)b * NG + c0 + g * gu, v);
      if (KIND == K_MILSTM) {
        float x[4] = {dwx4[0][g], dwx4[1][g], dwx4[2][g], dwx4[3][g]};
        store4<T>(D_wx + (long)b * NG + c0 + g * gu, x);
      }
    }
    *reinterpret_cast<float4*>(dc + ro) = make_float4(dcn[0], dcn[1], dcn[2], dcn[3]);
  }
  __syncthreads();
  // lane sums: thread (u, y) accumulates rows y, y+4, ... of the chunk in ascending order, every gate
  // (lstm_bwd_pw2_kernel's replay; w, h of padding units are zero there, so here too)
  const int nrows = min(BWD_RB, B - b0);
  float acc[NV];
#pragma unroll
  for (int i = 0; i < NV; ++i) acc[i] = 0.f;
  const int su = tid % BW2_UB, sy = tid / BW2_UB;
  const bool uvalid = u0 + su < H;
  if (tid < BWD_RY * BW2_UB) {
    for (int rr = sy; rr < nrows; rr += BWD_RY) {
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        const int o = g * BW3_TILE + rr * BW2_UB + su;
        const float da = sDA[o];
        const float w = (KIND == K_MILSTM && uvalid) ? sWX[o] : 0.f;
        const float h = (KIND == K_MILSTM && uvalid) ? sUH[o] : 0.f;
        lstm_bwd_acc<KIND, F>(acc, g, da, w, h);
      }
    }
  }
  __syncthreads();   // contributions consumed: the same memory holds the lane sums
  float* red = sDA;  // [4 lanes][NV][BW2_UB]
  if (tid < BWD_RY * BW2_UB) {
#pragma unroll
    for (int i = 0; i < NV; ++i) red[(sy * NV + i) * BW2_UB + su] = acc[i];
  }
  __syncthreads();
  for (int k = 0, item = tid; item < NV * BW2_UB; item += BW2_THREADS, ++k) {
    const int u = item % BW2_UB, i = item / BW2_UB, j = u0 + u;
    const int q = i / 4, g = i % 4;
    if (q >= nq || j >= Hp) continue;
    float v = 0.f;
#pragma unroll
    for (int y = 0; y < BWD_RY; ++y) v = __fadd_rn(v, red[(y * NV + i) * BW2_UB + u]);
    partials[(long)chunk * nq * NG + (long)q * NG + gcol_u(g, j, gu)] = first ? v : __fadd_rn(pre[k], v);
  }
}

// fp32 tile maps of the TMA-tiled form, cached by (pointer, shape): the per-step operand pointers
// repeat every training step, so each map is encoded once
static CUtensorMap bw3_map(const void* ptr, long inner, long rows, long z, long ld, long zstride) {
  using Key = std::tuple<const void*, long, long, long, long, long>;
  static std::map<Key, CUtensorMap> cache;
  static std::mutex mu;   // cells may enqueue from several host threads
  std::lock_guard<std::mutex> lock(mu);
  const Key k{ptr, inner, rows, z, ld, zstride};
  auto it = cache.find(k);
  if (it != cache.end()) return it->second;
  if (cache.size() > 16384) cache.clear();
  CUtensorMap mm;
  make_tile_map(&mm, ptr, false, inner, rows, z, ld, zstride, 32, 32, 0);
  return cache.emplace(k, mm).first->second;
}

template <int KIND, typename T>
static void bwd_pw_launch(int B, int H, int Hp, const void* dy, long ldy, OT dy_ot, bool dy_f32, const float* dh_rec,
                          long ld_dh, int nsplit, long split_stride, float* dc, const float* WX, const float* UH, const float* c_new,
                          const float* c_prev, GateParams gp, void* D_uh, void* D_wx, float* partials, int nq,
                          bool first, cudaStream_t st, int form, int gu) {
  // the TMA-tiled form needs fp32 dy (the LM's internal dY), split partials of dh_rec, 16-byte rows
  if (form == 2) {
    const bool ok = !first && dh_rec && nsplit >= 1 && nsplit <= SPLIT_MAX && (dy_f32 || dy_ot == OT::F32) && ld_dh % 4 == 0 &&
                    split_stride % 4 == 0 && ldy % 4 == 0 && Hp % BW2_UB == 0 && ((uintptr_t)dh_rec & 15) == 0 &&
                    ((uintptr_t)dy & 15) == 0 && ((uintptr_t)WX & 15) == 0 && ((uintptr_t)UH & 15) == 0 &&
                    ((uintptr_t)c_new & 15) == 0 && ((uintptr_t)c_prev & 15) == 0 && ((uintptr_t)dc & 15) == 0;
    if (!ok && !first && std::getenv("ASTRA_BPW2_STRICT"))   // tests: prove the tiled form runs
      throw Error(ASTRA_E_UNSUPPORTED, "lstm_bwd_pointwise: the TMA-tiled form cannot run this step");
    if (!ok) form = 1;
  }
  if (form == 2) {
    const long NG = 4L * Hp;
    Bw3Maps m;
    m.wx = bw3_map(WX, NG, B, 1, NG, 0);
    m.uh = bw3_map(UH, NG, B, 1, NG, 0);
    m.p = bw3_map(dh_rec, Hp, B, nsplit, ld_dh, split_stride);
    m.dc = bw3_map(dc, Hp, B, 1, Hp, 0);
    m.cp = bw3_map(c_prev, Hp, B, 1, Hp, 0);
    m.cn = bw3_map(c_new, Hp, B, 1, Hp, 0);
    m.dy = bw3_map(dy, Hp, B, 1, ldy, 0);
    auto k = lstm_bwd_pw3_kernel<KIND, T>;
    static bool attr = false;
    if (!attr) { CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)BW3_SMEM)); attr = true; }
    dim3 grid3(Hp / BW2_UB, lstm_bwd_row_chunks(B));
    launch_pdl(k, grid3, dim3(BW2_THREADS), BW3_SMEM, st, 1, m, B, H, Hp, nsplit, gu, dc, gp, (T*)D_uh, (T*)D_wx,
               partials, nq, (int)first);
    LAUNCH_CHECK();
    return;
  }
  if (form == 1) {
    constexpr int NC = KIND == K_MILSTM ? 3 : 1, NP = KIND == K_MILSTM ? 4 : 1;
    const size_t smem = (size_t)(NC * 4 * BWD_RB * BW2_UB + NP * 4 * BW2_UB) * 4;
    dim3 grid2(cdiv(Hp, BW2_UB), lstm_bwd_row_chunks(B));
    if (dy_f32 || dy_ot == OT::F32) {
      auto k = lstm_bwd_pw2_kernel<KIND, T, float>;
      static bool attr = false;
      if (!attr) { CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)); attr = true; }
      launch_pdl(k, grid2, dim3(BW2_THREADS), smem, st, 1, B, H, Hp, (const float*)dy, ldy, dh_rec, ld_dh, nsplit,
                 split_stride, dc, WX, UH, c_new, c_prev, gp, (T*)D_uh, (T*)D_wx, partials, nq, (int)first, gu);
    } else {
      auto k = lstm_bwd_pw2_kernel<KIND, T, __nv_bfloat16>;
      static bool attr = false;
      if (!attr) { CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)); attr = true; }
      launch_pdl(k, grid2, dim3(BW2_THREADS), smem, st, 1, B, H, Hp, (const __nv_bfloat16*)dy, ldy, dh_rec, ld_dh,
                 nsplit, split_stride, dc, WX, UH, c_new, c_prev, gp, (T*)D_uh, (T*)D_wx, partials, nq, (int)first, gu);
    }
    LAUNCH_CHECK();
    return;
  }
  dim3 grid(cdiv(Hp, BWD_UX), lstm_bwd_row_chunks(B));
  dim3 block(BWD_UX, BWD_RY);
  const bool blk = gu != GATE_U;
  ASTRA_CHECK_ARG((long)B * 4 * Hp < (1L << 31) && (long)B * ldy < (1L << 31) && (long)B * ld_dh < (1L << 31),
                  "lstm_bwd_pointwise: one step's tensors must have < 2^31 elements");
  // compile-time split count for the R25 splits the chains use (4 at cfg5, 2, 1), else generic
  const int ns = !dh_rec ? 1 : (nsplit == 4 || nsplit == 2 || nsplit == 1) ? nsplit : 0;
  auto pick = [&](auto tdy) {
    using TD = decltype(tdy);
    void (*k)(int, int, int, const TD*, long, const float*, long, int, long, float*, const float*, const float*,
              const float*, const float*, GateParams, T*, T*, float*, int, int, int) = nullptr;
#define BWD_NS(N) \
    if (ns == N) k = blk ? lstm_bwd_pw_kernel<KIND, T, TD, true, N> : lstm_bwd_pw_kernel<KIND, T, TD, false, N>;
    BWD_NS(0) BWD_NS(1) BWD_NS(2) BWD_NS(4)
#undef BWD_NS
    launch_pdl(k, grid, block, 0, st, 1, B, H, Hp, (const TD*)dy, ldy, dh_rec, ld_dh, nsplit, split_stride, dc, WX, UH,
               c_new, c_prev, gp, (T*)D_uh, (T*)D_wx, partials, nq, (int)first, gu);
  };
  if (dy_f32 || dy_ot == OT::F32) pick(float{});
  else pick(__nv_bfloat16{});
  LAUNCH_CHECK();
}

void lstm_bwd_pointwise(int kind, OT ot, int B, int H, int Hp, const void* dy, long ldy, OT dy_ot, bool dy_f32,
                        const float* dh_rec, long ld_dh, int nsplit, long split_stride, float* dc, const float* WX, const float* UH,
                        const float* c_new, const float* c_prev, GateParams gp, void* D_uh, void* D_wx,
                        float* partials, int nq, bool first, cudaStream_t st, int form, int gu) {
  ASTRA_CHECK_ARG(gu == GATE_U || gu == Hp, "lstm_bwd_pointwise: gate layout must be GATE_U or Hp");
#define BWD_CASE(K)                                                                                            \
  if (kind == K) {                                                                                             \
    if (ot == OT::BF16)                                                                                        \
      bwd_pw_launch<K, __nv_bfloat16>(B, H, Hp, dy, ldy, dy_ot, dy_f32, dh_rec, ld_dh, nsplit, split_stride, dc, WX, UH, c_new, c_prev, \
                                      gp, D_uh, D_wx, partials, nq, first, st, form, gu);                          \
    else                                                                                                       \
      bwd_pw_launch<K, float>(B, H, Hp, dy, ldy, dy_ot, dy_f32, dh_rec, ld_dh, nsplit, split_stride, dc, WX, UH, c_new, c_prev, gp,  \
                              D_uh, D_wx, partials, nq, first, st, form, gu);                                      \
    return;                                                                                                    \
  }
  BWD_CASE(K_LSTM)
  BWD_CASE(K_MILSTM)
  BWD_CASE(K_SUBLSTM)
#undef BWD_CASE
  throw Error(ASTRA_E_UNSUPPORTED, "lstm_bwd_pointwise: kind");
}

struct GradPtrs { float* p[4]; };

__global__ void reduce_gate_partials_kernel(const float* __restrict__ partials, int nchunk, int nq, int H, int Hp,
                                            GradPtrs out, int gu) {
  const int e = blockIdx.x * blockDim.x + threadIdx.x;
  const int q = blockIdx.y;
  if (e >= 4 * H) return;
  const int g = e / H, j = e % H;
  const long NG = 4L * Hp;
  const int col = gcol_u(g, j, gu);
  float s = 0.f;
  for (int c = 0; c < nchunk; ++c) s = __fadd_rn(s, partials[((long)c * nq + q) * NG + col]);
  out.p[q][e] = s;
}

void reduce_gate_partials(const float* partials, int nchunk, int nq, int H, int Hp, float* const* grads_q,
                          cudaStream_t st, int gu) {
  GradPtrs gp{};
  for (int q = 0; q < nq; ++q) gp.p[q] = grads_q[q];
  dim3 grid(cdiv(4L * H, 256), nq);
  reduce_gate_partials_kernel<<<grid, 256, 0, st>>>(partials, nchunk, nq, H, Hp, gp, gu);
  LAUNCH_CHECK();
}

// ============================================================================ LM pieces
template <typename T>
__global__ void embed_gather_kernel(const int32_t* __restrict__ tok, long n, const float* __restrict__ E, int I,
                                    T* __restrict__ X, long ldx) {
  const long r = blockIdx.x;
  const long src = (long)tok[r] * I;
  for (int c = threadIdx.x; c < ldx; c += blockDim.x) X[r * ldx + c] = from_f<T>(c < I ? E[src + c] : 0.f);
}

// bf16 output, I and ldx multiples of 8: one thread converts 8 columns (two 16-byte loads, one
// 16-byte store) — the same per-element rounding as embed_gather_kernel.
__global__ void embed_gather8_kernel(const int32_t* __restrict__ tok, const float* __restrict__ E, int I,
                                     __nv_bfloat16* __restrict__ X, long ldx) {
  const long r = blockIdx.y;
  const long c = ((long)blockIdx.x * blockDim.x + threadIdx.x) * 8;
  if (c >= ldx) return;
  float v[8];
  if (c < I) {
    const float4* src = reinterpret_cast<const float4*>(E + (long)tok[r] * I + c);
    const float4 p = __ldg(src), q = __ldg(src + 1);
    v[0] = p.x; v[1] = p.y; v[2] = p.z; v[3] = p.w; v[4] = q.x; v[5] = q.y; v[6] = q.z; v[7] = q.w;
  } else {
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = 0.f;
  }
  uint4 o;
  __nv_bfloat162* ob = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
  for (int i = 0; i < 4; ++i) ob[i] = __halves2bfloat162(__float2bfloat16_rn(v[2 * i]), __float2bfloat16_rn(v[2 * i + 1]));
  __stcs(reinterpret_cast<uint4*>(X + r * ldx + c), o);
}

void embed_gather(OT ot, const int32_t* tok, long n, const float* E, int I, void* X, long ldx, cudaStream_t st) {
  if (n == 0) return;
  if (ot == OT::BF16 && I % 8 == 0 && ldx % 8 == 0) {
    for (long r0 = 0; r0 < n; r0 += 65535) {   // grid.y ≤ 65535 rows per launch
      const long nr = n - r0 < 65535 ? n - r0 : 65535;
      dim3 grid((unsigned)cdiv(ldx / 8, 128), (unsigned)nr);
      embed_gather8_kernel<<<grid, 128, 0, st>>>(tok + r0, E, I, (__nv_bfloat16*)X + r0 * ldx, ldx);
      LAUNCH_CHECK();
    }
    return;
  }
  if (ot == OT::BF16)
    embed_gather_kernel<__nv_bfloat16><<<(unsigned)n, 256, 0, st>>>(tok, n, E, I, (__nv_bfloat16*)X, ldx);
  else
    embed_gather_kernel<float><<<(unsigned)n, 256, 0, st>>>(tok, n, E, I, (float*)X, ldx);
  LAUNCH_CHECK();
}

// one warp per row; fixed-order warp-shuffle trees
template <typename T>
__global__ void ce_kernel(const float* __restrict__ logits, long ldl, int V, const int32_t* __restrict__ targets,
                          long n, float inv_n, const int* __restrict__ nvp, long row0, float* __restrict__ rowloss,
                          T* __restrict__ dlog, long ldd, float* __restrict__ dlog32) {
  const long r = (long)blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32;
  const int lane = threadIdx.x % 32;
  if (r >= n) return;
  if (nvp) {   // rows ≥ *nvp are padding (bucketed steps): no loss, zero gradient; mean over *nvp rows
    const long nv = *nvp;
    inv_n = __fdiv_rn(1.f, (float)nv);
    if (row0 + r >= nv) {
      if (lane == 0) rowloss[r] = 0.f;
      for (int c = lane; c < ldd; c += 32) dlog[r * ldd + c] = from_f<T>(0.f);
      for (int c = lane; c < V; c += 32) dlog32[r * V + c] = 0.f;
      return;
    }
  }
  const float* row = logits + r * ldl;
  float m = -INFINITY;
  for (int c = lane; c < V; c += 32) m = fmaxf(m, row[c]);
#pragma unroll
  for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  float s = 0.f;
  for (int c = lane; c < V; c += 32) s = __fadd_rn(s, expf(__fsub_rn(row[c], m)));
#pragma unroll
  for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
  const float lse = __fadd_rn(m, logf(s));
  const int tgt = targets[r];
  if (lane == 0) rowloss[r] = __fsub_rn(lse, row[tgt]);
  const float rs = __frcp_rn(s);
  for (int c = lane; c < V; c += 32) {
    float p = __fmul_rn(expf(__fsub_rn(row[c], m)), rs);
    if (c == tgt) p = __fsub_rn(p, 1.f);
    const float d = __fmul_rn(p, inv_n);
    dlog[r * ldd + c] = from_f<T>(d);
    dlog32[r * V + c] = d;
  }
  for (int c = V + lane; c < ldd; c += 32) dlog[r * ldd + c] = from_f<T>(0.f);
}

// One 256-thread CTA per row, float4 loads/stores (V % 4 == 0): thread t takes the quads t, t+256,
// … in ascending order, then a warp xor tree and the 8 warp sums in warp order — a fixed order for
// every row, so the row's bits do not depend on how the rows are chunked or launched.
constexpr int CE_T = 256;
template <typename T> __device__ __forceinline__ void ce_store4(T* p, float a, float b, float c, float d);
template <> __device__ __forceinline__ void ce_store4<float>(float* p, float a, float b, float c, float d) {
  *reinterpret_cast<float4*>(p) = make_float4(a, b, c, d);
}
template <> __device__ __forceinline__ void ce_store4<__nv_bfloat16>(__nv_bfloat16* p, float a, float b, float c,
                                                                      float d) {
  __nv_bfloat162 lo = __floats2bfloat162_rn(a, b), hi = __floats2bfloat162_rn(c, d);
  uint2 u;
  u.x = *reinterpret_cast<uint32_t*>(&lo);
  u.y = *reinterpret_cast<uint32_t*>(&hi);
  *reinterpret_cast<uint2*>(p) = u;
}

template <typename T>
__global__ void __launch_bounds__(CE_T) ce_row_kernel(const float* __restrict__ logits, long ldl, int V,
                                                      const int32_t* __restrict__ targets, long n, float inv_n,
                                                      const int* __restrict__ nvp, long row0,
                                                      float* __restrict__ rowloss, T* __restrict__ dlog, long ldd,
                                                      float* __restrict__ dlog32) {
  __shared__ float red[CE_T / 32];
  const long r = blockIdx.x;
  const int tid = threadIdx.x, lane = tid % 32, w = tid / 32;
  const int V4 = V / 4;
  T* drow = dlog + r * ldd;
  float* d32 = dlog32 + r * V;
  if (nvp) {   // rows ≥ *nvp are padding (bucketed steps): no loss, zero gradient; mean over *nvp rows
    const long nv = *nvp;
    inv_n = __fdiv_rn(1.f, (float)nv);
    if (row0 + r >= nv) {
      if (tid == 0) rowloss[r] = 0.f;
      for (int q = tid; q < V4; q += CE_T) {
        ce_store4<T>(drow + 4 * q, 0.f, 0.f, 0.f, 0.f);
        ce_store4<float>(d32 + 4 * q, 0.f, 0.f, 0.f, 0.f);
      }
      for (int c = V + tid; c < ldd; c += CE_T) drow[c] = from_f<T>(0.f);
      return;
    }
  }
  const float4* row = reinterpret_cast<const float4*>(logits + r * ldl);
  float m = -INFINITY;
  for (int q = tid; q < V4; q += CE_T) {
    const float4 x = row[q];
    m = fmaxf(fmaxf(m, fmaxf(x.x, x.y)), fmaxf(x.z, x.w));
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
  if (lane == 0) red[w] = m;
  __syncthreads();
  m = red[0];
#pragma unroll
  for (int k = 1; k < CE_T / 32; ++k) m = fmaxf(m, red[k]);
  __syncthreads();
  float s = 0.f;
  for (int q = tid; q < V4; q += CE_T) {
    const float4 x = row[q];
    s = __fadd_rn(s, expf(__fsub_rn(x.x, m)));
    s = __fadd_rn(s, expf(__fsub_rn(x.y, m)));
    s = __fadd_rn(s, expf(__fsub_rn(x.z, m)));
    s = __fadd_rn(s, expf(__fsub_rn(x.w, m)));
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) s = __fadd_rn(s, __shfl_xor_sync(0xffffffffu, s, o));
  if (lane == 0) red[w] = s;
  __syncthreads();
  s = red[0];
#pragma unroll
  for (int k = 1; k < CE_T / 32; ++k) s = __fadd_rn(s, red[k]);
  const float lse = __fadd_rn(m, logf(s));
  const int tgt = targets[r];
  if (tid == 0) rowloss[r] = __fsub_rn(lse, logits[r * ldl + tgt]);
  const float rs = __frcp_rn(s);
  for (int q = tid; q < V4; q += CE_T) {
    const float4 x = row[q];
    float p[4] = {__fmul_rn(expf(__fsub_rn(x.x, m)), rs), __fmul_rn(expf(__fsub_rn(x.y, m)), rs),
                  __fmul_rn(expf(__fsub_rn(x.z, m)), rs), __fmul_rn(expf(__fsub_rn(x.w, m)), rs)};
    if ((tgt >> 2) == q) p[tgt & 3] = __fsub_rn(p[tgt & 3], 1.f);
#pragma unroll
    for (int k = 0; k < 4; ++k) p[k] = __fmul_rn(p[k], inv_n);
    ce_store4<T>(drow + 4 * q, p[0], p[1], p[2], p[3]);
    ce_store4<float>(d32 + 4 * q, p[0], p[1], p[2], p[3]);
  }
  for (int c = V + tid; c < ldd; c += CE_T) drow[c] = from_f<T>(0.f);
}

void ce_fwd_bwd(OT ot, const float* logits, long ldl, int V, const int32_t* targets, long n, float inv_n,
                float* rowloss, void* dlog, long ldd, float* dlog32, cudaStream_t st, const int* nvp, long row0) {
  if (n == 0) return;
  const size_t e = ot == OT::BF16 ? 2 : 4;
  // one CTA per row pays off for wide rows only (cfg2/cfg3, V = 10k: 75 -> 25 µs per chunk); at V = 256
  // (cfg5) most of its threads would idle and a warp per row is faster (33 vs 112 µs per step)
  const bool vec = V >= 2048 && V % 4 == 0 && ldl % 4 == 0 && ldd % 4 == 0 && ((uintptr_t)logits & 15) == 0 &&
                   ((uintptr_t)dlog & (4 * e - 1)) == 0 && ((uintptr_t)dlog32 & 15) == 0;
  if (vec) {
    ASTRA_CHECK_ARG(n < (1L << 31), "ce_fwd_bwd: too many rows");
    if (ot == OT::BF16)
      ce_row_kernel<__nv_bfloat16><<<(unsigned)n, CE_T, 0, st>>>(logits, ldl, V, targets, n, inv_n, nvp, row0, rowloss,
                                                                 (__nv_bfloat16*)dlog, ldd, dlog32);
    else
      ce_row_kernel<float><<<(unsigned)n, CE_T, 0, st>>>(logits, ldl, V, targets, n, inv_n, nvp, row0, rowloss,
                                                         (float*)dlog, ldd, dlog32);
    LAUNCH_CHECK();
    return;
  }
  const int rows_per = 8;
  dim3 grid(cdiv(n, rows_per));
  if (ot == OT::BF16)
    ce_kernel<__nv_bfloat16><<<grid, 32 * rows_per, 0, st>>>(logits, ldl, V, targets, n, inv_n, nvp, row0, rowloss,
                                                             (__nv_bfloat16*)dlog, ldd, dlog32);
  else
    ce_kernel<float><<<grid, 32 * rows_per, 0, st>>>(logits, ldl, V, targets, n, inv_n, nvp, row0, rowloss, (float*)dlog,
                                                     ldd, dlog32);
  LAUNCH_CHECK();
}

// s + p[0] + p[stride] + ... + p[(n−1)·stride], added in ascending order (the fixed order of every
// reduction below); the loads are issued 8 at a time, so a thread waits one memory latency per 8
// terms instead of one per term.  Same bits as the one-term-at-a-time loop.
// (NB terms ahead: 8 for wide grids; 32 for the few-block final reductions, whose threads are few.)
template <int NB = 8>
__device__ __forceinline__ float ordered_sum(const float* __restrict__ p, long n, long stride, float s = 0.f) {
  long i = 0;
  for (; i + NB <= n; i += NB) {
    float v[NB];
#pragma unroll
    for (int k = 0; k < NB; ++k) v[k] = p[(i + k) * stride];
#pragma unroll
    for (int k = 0; k < NB; ++k) s = __fadd_rn(s, v[k]);
  }
  for (; i < n; ++i) s = __fadd_rn(s, p[i * stride]);
  return s;
}

__global__ void sum_scalar_kernel(const float* __restrict__ v, long n, float scale, const int* __restrict__ nvp,
                                  float* __restrict__ out) {
  __shared__ float sh[1024];
  if (nvp) scale = __fdiv_rn(1.f, (float)*nvp);   // mean over the valid rows (the rest are exact zeros)
  const long nt = n > (long)threadIdx.x ? (n - threadIdx.x + blockDim.x - 1) / blockDim.x : 0;
  sh[threadIdx.x] = ordered_sum<32>(v + threadIdx.x, nt, blockDim.x);
  __syncthreads();
  for (int w = blockDim.x / 2; w > 0; w >>= 1) {
    if (threadIdx.x < w) sh[threadIdx.x] = __fadd_rn(sh[threadIdx.x], sh[threadIdx.x + w]);
    __syncthreads();
  }
  if (threadIdx.x == 0) *out = __fmul_rn(sh[0], scale);
}

void sum_rows_to_scalar(const float* v, long n, float scale, float* out, cudaStream_t st, const int* nvp) {
  sum_scalar_kernel<<<1, 1024, 0, st>>>(v, n, scale, nvp, out);
  LAUNCH_CHECK();
}

__global__ void set_i32_kernel(int* p, int v) { *p = v; }
void set_i32(int* p, int v, cudaStream_t st) {
  set_i32_kernel<<<1, 1, 0, st>>>(p, v);
  LAUNCH_CHECK();
}

constexpr int COLSUM_RB = 256;
size_t colsum_scratch_floats(long rows, int cols) { return (size_t)cdiv(rows, COLSUM_RB) * cols; }

__global__ void colsum_partial_kernel(const float* __restrict__ in, long rows, int cols, long ld,
                                      float* __restrict__ part) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  const long r0 = (long)blockIdx.y * COLSUM_RB;
  if (c >= cols) return;
  const long r1 = min(rows, r0 + COLSUM_RB);
  part[(long)blockIdx.y * cols + c] = ordered_sum(in + r0 * ld + c, r1 - r0, ld);
}
__global__ void colsum_final_kernel(const float* __restrict__ part, int nchunk, int cols, float* __restrict__ out) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= cols) return;
  out[c] = ordered_sum<32>(part + c, nchunk, cols);
}

void colsum(const float* in, long rows, int cols, long ld, float* scratch, float* out, cudaStream_t st) {
  const int nchunk = cdiv(rows, COLSUM_RB);
  colsum_partial_kernel<<<dim3(cdiv(cols, 128), nchunk), 128, 0, st>>>(in, rows, cols, ld, scratch);
  LAUNCH_CHECK();
  colsum_final_kernel<<<cdiv(cols, 128), 128, 0, st>>>(scratch, nchunk, cols, out);
  LAUNCH_CHECK();
}

// ---- embedding backward: stable counting sort of (token, row) then ordered segment sums
// Segmented, deterministic embedding backward.  A stable counting sort of (token, row) — hand-written:
// per-block token histograms, a parallel scan, and a one-warp-per-block stable scatter — puts the rows
// of token v in the sorted range [lo_v, lo_v + n_v) in ascending row order.  That range is cut into
// segments of EMB_SEG rows (so a hot Zipf token does not serialise onto one CTA); segment partial
// sums are taken in row order and the segments of a token are then added in order.  (The block
// size only changes how the sort is computed, never the sorted order: the bits do not depend on it.)
constexpr int EMB_SEG = 64;

// rows per counting block: ~2 blocks per SM, at least 128 rows, a multiple of 32
static long emb_blk(long n) {
  long b = (n + 295) / 296;
  b = (b + 31) / 32 * 32;
  return b < 128 ? 128 : b;
}
static long emb_blocks(long n) { return n > 0 ? (n + emb_blk(n) - 1) / emb_blk(n) : 0; }

size_t embed_bwd_scratch_bytes(long n, int V) {
  const size_t nb = round_up(n * 4, 256), vb = round_up((V + 1) * 4L, 256);
  const size_t cb = round_up((size_t)emb_blocks(n) * V * 4, 256);
  return cb + 2 * nb + 3 * vb;
}

// cnt[b][v] = rows of block b with token v (integer atomics: the counts do not depend on the order)
__global__ void emb_count_kernel(const int32_t* __restrict__ tok, long n, long blk, int V, int32_t* __restrict__ cnt) {
  const long b = blockIdx.x;
  const long r0 = b * blk, r1 = min(n, r0 + blk);
  for (long i = r0 + threadIdx.x; i < r1; i += blockDim.x) {
    const int v = tok[i];
    if (v >= 0 && v < V) atomicAdd(&cnt[b * V + v], 1);
  }
}

// tot[v] = Σ_b cnt[b][v]; nseg[v] = ⌈tot[v] / EMB_SEG⌉ (written to lo / segoff, scanned next).
// One warp per token: lanes take 32 consecutive blocks at a time (integer sums: exact in any order).
__global__ void emb_total_kernel(const int32_t* __restrict__ cnt, long nblk, int V, int32_t* __restrict__ lo,
                                 int32_t* __restrict__ segoff) {
  const int v = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (v >= V) return;
  int tot = 0;
  for (long b = lane; b < nblk; b += 32) tot += cnt[b * V + v];
#pragma unroll
  for (int o = 16; o; o >>= 1) tot += __shfl_xor_sync(0xffffffffu, tot, o);
  if (lane == 0) {
    lo[v] = tot;
    segoff[v] = (tot + EMB_SEG - 1) / EMB_SEG;
  }
}

// One CTA: in-place exclusive scans of lo[0..V) and segoff[0..V), totals into lo[V] / segoff[V];
// tiles of 4·1024 entries, 4 consecutive per thread, carried across tiles.
__global__ void __launch_bounds__(1024) emb_scan_kernel(int V, int32_t* __restrict__ lo, int32_t* __restrict__ segoff) {
  __shared__ int32_t wsum[2][32];
  __shared__ int32_t carry[2];
  const int tid = threadIdx.x, lane = tid % 32, w = tid / 32;
  if (tid == 0) { carry[0] = 0; carry[1] = 0; }
  __syncthreads();
  for (int t0 = 0; t0 < V; t0 += 4 * 1024) {
    int a[4], s[4], ta = 0, ts = 0;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int v = t0 + tid * 4 + k;
      a[k] = v < V ? lo[v] : 0;
      s[k] = v < V ? segoff[v] : 0;
      ta += a[k];
      ts += s[k];
    }
    int it = ta, is = ts;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int x = __shfl_up_sync(0xffffffffu, it, d), y = __shfl_up_sync(0xffffffffu, is, d);
      if (lane >= d) { it += x; is += y; }
    }
    if (lane == 31) { wsum[0][w] = it; wsum[1][w] = is; }
    __syncthreads();
    if (w == 0) {
      int x = wsum[0][lane], y = wsum[1][lane];
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const int p = __shfl_up_sync(0xffffffffu, x, d), q = __shfl_up_sync(0xffffffffu, y, d);
        if (lane >= d) { x += p; y += q; }
      }
      wsum[0][lane] = x;
      wsum[1][lane] = y;
    }
    __syncthreads();
    int ra = carry[0] + (it - ta) + (w > 0 ? wsum[0][w - 1] : 0);
    int rs = carry[1] + (is - ts) + (w > 0 ? wsum[1][w - 1] : 0);
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const int v = t0 + tid * 4 + k;
      if (v < V) { lo[v] = ra; segoff[v] = rs; }
      ra += a[k];
      rs += s[k];
    }
    __syncthreads();   // everyone has read carry
    if (tid == 1023) { carry[0] = ra; carry[1] = rs; }
    __syncthreads();
  }
  if (tid == 0) { lo[V] = carry[0]; segoff[V] = carry[1]; }
}

// cnt[b][v] ← lo_v + Σ_{b' < b} cnt[b'][v]: the first sorted position of block b's rows of token v.
// One warp per token: an exclusive warp scan over 32 consecutive blocks at a time, carried.
__global__ void emb_cursor_kernel(int32_t* __restrict__ cnt, long nblk, int V, const int32_t* __restrict__ lo) {
  const int v = blockIdx.x * (blockDim.x / 32) + threadIdx.x / 32, lane = threadIdx.x % 32;
  if (v >= V) return;
  int run = lo[v];
  for (long b0 = 0; b0 < nblk; b0 += 32) {
    const long b = b0 + lane;
    const int c = b < nblk ? cnt[b * V + v] : 0;
    int incl = c;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int x = __shfl_up_sync(0xffffffffu, incl, d);
      if (lane >= d) incl += x;
    }
    if (b < nblk) cnt[b * V + v] = run + incl - c;
    run += __shfl_sync(0xffffffffu, incl, 31);
  }
}

// Stable scatter: one warp per block walks its rows 32 at a time in ascending order; lanes with the
// same token rank themselves by lane (match.any), the lowest of them advances the token's cursor.
__global__ void __launch_bounds__(32) emb_scatter_kernel(const int32_t* __restrict__ tok, long n, long blk, int V,
                                                         int32_t* __restrict__ cnt, int32_t* __restrict__ srows) {
  const long b = blockIdx.x;
  const int lane = threadIdx.x;
  const long r0 = b * blk, r1 = min(n, r0 + blk);
  int32_t* cur = cnt + b * V;   // this block's cursors (first positions, from emb_cursor_kernel)
  for (long base = r0; base < r1; base += 32) {
    const long i = base + lane;
    const bool ok = i < r1;
    const int v = ok ? tok[i] : -1 - lane;   // unique dummy keys for the tail lanes
    const bool valid = ok && v >= 0 && v < V;
    const unsigned peers = __match_any_sync(0xffffffffu, v);
    const int rank = __popc(peers & ((1u << lane) - 1u));
    const int leader = __ffs(peers) - 1;
    int pos = 0;
    if (valid && lane == leader) pos = cur[v];
    pos = __shfl_sync(0xffffffffu, pos, leader) + rank;
    __syncwarp();
    if (valid) {
      srows[pos] = (int32_t)i;
      if (lane == leader) cur[v] = pos - rank + __popc(peers);
    }
    __syncwarp();
  }
}

// W consecutive columns per thread (4 where I and the row stride allow float4, else 1)
template <int W> struct emb_vec;
template <> struct emb_vec<4> { using t = float4; };
template <> struct emb_vec<1> { using t = float; };
__device__ __forceinline__ void emb_acc(float4& a, const float4& x) {
  a.x = __fadd_rn(a.x, x.x); a.y = __fadd_rn(a.y, x.y); a.z = __fadd_rn(a.z, x.z); a.w = __fadd_rn(a.w, x.w);
}
__device__ __forceinline__ void emb_acc(float& a, const float& x) { a = __fadd_rn(a, x); }
template <int W> __device__ __forceinline__ typename emb_vec<W>::t emb_zero() {
  if constexpr (W == 4) return make_float4(0.f, 0.f, 0.f, 0.f); else return 0.f;
}

// partial[s][c] = Σ rows of segment s (ascending); the owning token is found from segoff.  A
// grid-stride loop over the segments actually present (segoff[V]).
template <int W>
__global__ void __launch_bounds__(256) emb_seg_partial_kernel(const int32_t* __restrict__ srows, int V,
                                                              const int32_t* __restrict__ lo,
                                                              const int32_t* __restrict__ segoff,
                                                              const float* __restrict__ dX, long ldx, int I,
                                                              float* __restrict__ part) {
  using VT = typename emb_vec<W>::t;
  const int total = segoff[V];
  const int c = (blockIdx.x * blockDim.x + threadIdx.x) * W;
  if (c >= I) return;
  for (int s = blockIdx.y; s < total; s += gridDim.y) {
    // token v: last v with segoff[v] <= s
    int a = 0, b = V;  // invariant segoff[a] <= s < segoff[b]
    while (b - a > 1) {
      const int m = (a + b) / 2;
      if (segoff[m] <= s) a = m; else b = m;
    }
    const long r0 = lo[a] + (long)(s - segoff[a]) * EMB_SEG;
    const long r1 = min((long)lo[a + 1], r0 + EMB_SEG);
    VT acc = emb_zero<W>();
    long k = r0;
    for (; k + 8 <= r1; k += 8) {
      VT x[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) x[j] = *reinterpret_cast<const VT*>(dX + (long)srows[k + j] * ldx + c);
#pragma unroll
      for (int j = 0; j < 8; ++j) emb_acc(acc, x[j]);
    }
    for (; k < r1; ++k) emb_acc(acc, *reinterpret_cast<const VT*>(dX + (long)srows[k] * ldx + c));
    *reinterpret_cast<VT*>(part + (long)s * I + c) = acc;
  }
}

// dE[v][c] = Σ_s part[s][c] over token v's segments in order (0 for an absent token); W columns
// per thread, one flat grid over V·I/W.
template <int W>
__global__ void emb_seg_final_kernel(int V, const int32_t* __restrict__ segoff, const float* __restrict__ part, int I,
                                     float* __restrict__ dE) {
  using VT = typename emb_vec<W>::t;
  const long q = (long)blockIdx.x * blockDim.x + threadIdx.x;
  const int iw = I / W;
  if (q >= (long)V * iw) return;
  const int v = (int)(q / iw), c = (int)(q % iw) * W;
  const int s0 = segoff[v], s1 = segoff[v + 1];
  VT acc = emb_zero<W>();
  int s = s0;
  for (; s + 8 <= s1; s += 8) {   // 8 loads in flight, then the ordered adds (same sum)
    VT x[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) x[k] = *reinterpret_cast<const VT*>(part + (long)(s + k) * I + c);
#pragma unroll
    for (int k = 0; k < 8; ++k) emb_acc(acc, x[k]);
  }
  for (; s < s1; ++s) emb_acc(acc, *reinterpret_cast<const VT*>(part + (long)s * I + c));
  *reinterpret_cast<VT*>(dE + (long)v * I + c) = acc;
}

size_t embed_bwd_partial_floats(long n, int V, int I) {
  return (size_t)(n / EMB_SEG + (n < V ? n : V) + 1) * I;   // segments ≤ n/EMB_SEG + distinct tokens
}

void embed_bwd(const int32_t* tok, long n, int V, const float* dX, long ldx, int I, float* dE, void* scratch,
               size_t scratch_bytes, float* part, cudaStream_t st) {
  if (n == 0) {
    CUDA_TRY(cudaMemsetAsync(dE, 0, (size_t)V * I * 4, st));
    return;
  }
  const long blk = emb_blk(n), nblk = emb_blocks(n);
  const size_t nb = round_up(n * 4, 256), vb = round_up((V + 1) * 4L, 256);
  const size_t cb = round_up((size_t)nblk * V * 4, 256);
  ASTRA_CHECK_ARG(scratch_bytes >= cb + 2 * nb + 3 * vb, "embed_bwd: scratch too small");
  char* base = (char*)scratch;
  int32_t* cnt = (int32_t*)base;
  int32_t* srows = (int32_t*)(base + cb + nb);
  int32_t* lo = (int32_t*)(base + cb + 2 * nb);
  int32_t* segoff = (int32_t*)(base + cb + 2 * nb + vb);
  CUDA_TRY(cudaMemsetAsync(cnt, 0, (size_t)nblk * V * 4, st));
  emb_count_kernel<<<(unsigned)nblk, 256, 0, st>>>(tok, n, blk, V, cnt);
  LAUNCH_CHECK();
  emb_total_kernel<<<cdiv(V, 8), 256, 0, st>>>(cnt, nblk, V, lo, segoff);
  LAUNCH_CHECK();
  emb_scan_kernel<<<1, 1024, 0, st>>>(V, lo, segoff);
  LAUNCH_CHECK();
  emb_cursor_kernel<<<cdiv(V, 8), 256, 0, st>>>(cnt, nblk, V, lo);
  LAUNCH_CHECK();
  emb_scatter_kernel<<<(unsigned)nblk, 32, 0, st>>>(tok, n, blk, V, cnt, srows);
  LAUNCH_CHECK();
  const long max_seg = n / EMB_SEG + (n < V ? n : V);
  const bool vec = I % 4 == 0 && ldx % 4 == 0 && ((uintptr_t)dX & 15) == 0 && ((uintptr_t)dE & 15) == 0 &&
                   ((uintptr_t)part & 15) == 0;
  const int W = vec ? 4 : 1;
  const int gx = cdiv(I, 256 * W);
  const long gy = std::min<long>(max_seg, 148L * 16 / gx + 1);
  const unsigned gf = (unsigned)cdiv((long)V * (I / W), 256);
  if (vec) {
    emb_seg_partial_kernel<4><<<dim3(gx, (unsigned)gy), 256, 0, st>>>(srows, V, lo, segoff, dX, ldx, I, part);
    LAUNCH_CHECK();
    emb_seg_final_kernel<4><<<gf, 256, 0, st>>>(V, segoff, part, I, dE);
  } else {
    emb_seg_partial_kernel<1><<<dim3(gx, (unsigned)gy), 256, 0, st>>>(srows, V, lo, segoff, dX, ldx, I, part);
    LAUNCH_CHECK();
    emb_seg_final_kernel<1><<<gf, 256, 0, st>>>(V, segoff, part, I, dE);
  }
  LAUNCH_CHECK();
}

// ============================================================================ split-K partial sums
// out[i] = Σ_k part[k][i] in ascending k (the fixed chunk order of R25 / R28).
__global__ void sum_split_partials_kernel(const float4* __restrict__ part, int ks, long n4, float4* __restrict__ out) {
  const long i = (long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n4) return;
  float4 v = part[i];
  for (int k = 1; k < ks; ++k) {
    const float4 q = part[(long)k * n4 + i];
    v.x = __fadd_rn(v.x, q.x); v.y = __fadd_rn(v.y, q.y); v.z = __fadd_rn(v.z, q.z); v.w = __fadd_rn(v.w, q.w);
  }
  out[i] = v;
}
__global__ void sum_split_partials1_kernel(const float* __restrict__ part, int ks, long n, float* __restrict__ out) {
  const long i = (long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  float v = part[i];
  for (int k = 1; k < ks; ++k) v = __fadd_rn(v, part[(long)k * n + i]);
  out[i] = v;
}
__global__ void add_split_partials_kernel(float* __restrict__ out, const float* __restrict__ part, int ks, long n) {
  const long i = (long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  float v = part[i];
  for (int k = 1; k < ks; ++k) v = __fadd_rn(v, part[(long)k * n + i]);
  out[i] = __fadd_rn(out[i], v);
}
void add_split_partials(float* out, const float* part, int ks, long n, cudaStream_t st) {
  add_split_partials_kernel<<<(unsigned)cdiv(n, 256), 256, 0, st>>>(out, part, ks, n);
  LAUNCH_CHECK();
}

void sum_split_partials(const float* part, int ks, long n, float* out, cudaStream_t st) {
  if ((n & 3) == 0 && (((uintptr_t)part | (uintptr_t)out) & 15) == 0)
    sum_split_partials_kernel<<<(unsigned)cdiv(n / 4, 256), 256, 0, st>>>((const float4*)part, ks, n / 4, (float4*)out);
  else
    sum_split_partials1_kernel<<<(unsigned)cdiv(n, 256), 256, 0, st>>>(part, ks, n, out);
  LAUNCH_CHECK();
}

// ============================================================================ SGD
__global__ void sgd_kernel(float* __restrict__ p, const float* __restrict__ g, size_t n, float lr) {
  const size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  const size_t n4 = n / 4;
  if (i < n4) {
    float4 a = reinterpret_cast<float4*>(p)[i];
    const float4 b = reinterpret_cast<const float4*>(g)[i];
    a.x = __fsub_rn(a.x, __fmul_rn(lr, b.x));
    a.y = __fsub_rn(a.y, __fmul_rn(lr, b.y));
    a.z = __fsub_rn(a.z, __fmul_rn(lr, b.z));
    a.w = __fsub_rn(a.w, __fmul_rn(lr, b.w));
    reinterpret_cast<float4*>(p)[i] = a;
  }
  if (i < n - n4 * 4) {
    const size_t k = n4 * 4 + i;
    p[k] = __fsub_rn(p[k], __fmul_rn(lr, g[k]));
  }
}

void sgd(float* p, const float* g, size_t n, float lr, cudaStream_t st) {
  if (!n) return;
  const size_t n4 = n / 4 > 0 ? n / 4 : 1;
  sgd_kernel<<<(unsigned)cdiv((long)n4, 256), 256, 0, st>>>(p, g, n, lr);
  LAUNCH_CHECK();
}

__global__ void scale_kernel(float* p, size_t n, float s) {
  const size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) p[i] = __fmul_rn(p[i], s);
}
void scale_inplace(float* p, size_t n, float s, cudaStream_t st) {
  if (!n) return;
  scale_kernel<<<(unsigned)cdiv((long)n, 256), 256, 0, st>>>(p, n, s);
  LAUNCH_CHECK();
}

}  // namespace astra
