// K2 / K4: fused recurrent kernels of the LSTM family on the bf16 path.
//
// One CTA owns one output tile for the whole chain.  Per step the tcgen05 main loop computes the
// recurrent product into TMEM and the epilogue warps apply the cell arithmetic directly from TMEM
// (the "fused gate epilogue" of the north star): no UH round trip through a separate kernel and no
// kernel boundary per step.
//
//   forward  (lstm_rec_fwd_kernel): tile = 128 batch rows × 256 gate columns (64 units, 4 gates,
//            gate-interleaved layout) of  UH_t = h_{t−1}·U;  epilogue → c_t, h_t (bf16 operand of
//            step t+1), UH_t (saved), y_t.
//   backward (lstm_rec_bwd_kernel): tile = 128 rows × 64 units of  dh_rec = D_uh_{t+1}·Uᵀ;  epilogue
//            → da, D_uh_t / D_wx_t (bf16 operands of step t−1 and of the weight gradients), dc, and
//            the bias / α / β column partial sums (fixed butterfly tree over the tile's 128 rows).
//
// Modes: persistent = 1 runs steps [t0, t1) in one cooperative launch; CTAs of the same row block
// exchange "h_t complete" through a release/acquire counter per row block (the next step's TMA
// reads the other CTAs' stores: writer fence.proxy.async + release, reader acquire +
// fence.proxy.async).  The weight operand of the next step does not depend on the recurrence, so
// the producer prefetches its first stages before waiting on the counter.  persistent = 0 is one
// launch per step (stream order replaces the counter).  Both modes execute identical arithmetic,
// so they are bitwise interchangeable (R17).
#include <cooperative_groups.h>

#include "cell_math.cuh"
#include "gemm_tc.cuh"
#include "kernels.h"
#include "rec_fused.h"

namespace astra {

constexpr int RF_EPI_WARPS = 8;
constexpr int RF_THREADS = 64 + 32 * RF_EPI_WARPS;  // warp 0 TMA, warp 1 MMA, 8 epilogue warps

__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}
__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void wait_flag(const unsigned* p, unsigned target) {
  while (ld_acquire(p) < target) __nanosleep(64);
}
__device__ __forceinline__ void epi_bar() {  // named barrier over the epilogue warps only
  asm volatile("bar.sync 1, %0;" ::"n"(32 * RF_EPI_WARPS) : "memory");
}

// ============================================================================== forward
template <int KIND>
__global__ void __launch_bounds__(RF_THREADS, 1)
    lstm_rec_fwd_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                        const RecFwdArgs a) {
  constexpr int BN = 256;
  using S = TcSmem<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int stages = a.stages;
  float* prm = reinterpret_cast<float*>(smem + stages * S::STAGE_BYTES);  // [4][256]: b, α, β1, β2
  uint64_t* full = reinterpret_cast<uint64_t*>(prm + 4 * BN);
  uint64_t* empty = full + stages;
  uint64_t* tfull = empty + stages;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int m_blk = blockIdx.x % a.num_m, n_blk = blockIdx.x / a.num_m;
  const int m0 = m_blk * TC_BM, n0 = n_blk * BN, u0 = n_blk * 64;
  const int nk = a.nk;

  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      sm100::mbar_init(&full[s], 1);
      sm100::mbar_init(&empty[s], 1);
    }
    for (int q = 0; q < 2; ++q) {
      sm100::mbar_init(&tfull[q], 1);
      sm100::mbar_init(&tempty[q], 32 * RF_EPI_WARPS);
    }
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, 512);
  for (int c = threadIdx.x; c < BN; c += RF_THREADS) {   // this tile's per-gate-column parameters
    const int g = c / 64, unit = u0 + c % 64, e = g * a.H + unit;
    const bool ok = unit < a.H;
    prm[c] = ok ? a.gp.b[e] : 0.f;
    prm[BN + c] = (ok && KIND == K_MILSTM) ? a.gp.alpha[e] : 0.f;
    prm[2 * BN + c] = (ok && KIND == K_MILSTM) ? a.gp.beta1[e] : 0.f;
    prm[3 * BN + c] = (ok && KIND == K_MILSTM) ? a.gp.beta2[e] : 0.f;
  }
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      long it = 0;
      const uint64_t pol = sm100::l2_policy_evict_last();
      for (int t = a.t0; t < a.t1; ++t) {
        const int pre = nk < stages ? nk : stages;
        for (int kb = 0; kb < pre; ++kb) {   // weight tiles do not depend on the recurrence
          const long i = it + kb;
          const int s = (int)(i % stages);
          sm100::mbar_wait(&empty[s], (uint32_t)((i / stages) & 1) ^ 1);
          sm100::mbar_arrive_expect_tx(&full[s], S::STAGE_BYTES);
          sm100::tma_load_3d_hint(smem + s * S::STAGE_BYTES + S::A_BYTES, &mapB, &full[s], kb * TC_BK, n0, 0, pol);
        }
        if (a.persistent && t > a.t0) {
          wait_flag(a.flags + m_blk, (unsigned)(a.num_n * (t - a.t0)));
          fence_proxy_async_global();
        }
        for (int kb = 0; kb < pre; ++kb) {
          const int s = (int)((it + kb) % stages);
          sm100::tma_load_3d(smem + s * S::STAGE_BYTES, &mapA, &full[s], kb * TC_BK, m0, t);
        }
        for (int kb = pre; kb < nk; ++kb) {
          const long i = it + kb;
          const int s = (int)(i % stages);
          sm100::mbar_wait(&empty[s], (uint32_t)((i / stages) & 1) ^ 1);
          sm100::mbar_arrive_expect_tx(&full[s], S::STAGE_BYTES);
          sm100::tma_load_3d(smem + s * S::STAGE_BYTES, &mapA, &full[s], kb * TC_BK, m0, t);
          sm100::tma_load_3d_hint(smem + s * S::STAGE_BYTES + S::A_BYTES, &mapB, &full[s], kb * TC_BK, n0, 0, pol);
        }
        it += nk;
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    {   // whole warp (umma_*_warp elect the issuing lane); lean loop: descriptors advanced by (bytes >> 4)
      const uint32_t sa0 = sm100::smem_u32(smem);
      const uint64_t dA0 = sm100::smem_desc_sw128(sa0, 16, 1024);
      const uint64_t dB0 = sm100::smem_desc_sw128(sa0 + S::A_BYTES, 16, 1024);
      const uint32_t idesc = a.idesc;
      int s = 0;
      uint32_t ph = 0;
      int local = 0;
      for (int t = a.t0; t < a.t1; ++t, ++local) {
        const int acc = local & 1;
        sm100::mbar_wait(&tempty[acc], (uint32_t)((local >> 1) & 1) ^ 1);
        sm100::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = 0; kb < nk; ++kb) {
          sm100::mbar_wait(&full[s], ph);
          sm100::tc_fence_after();
          const uint64_t ad = dA0 + (uint64_t)(s * (S::STAGE_BYTES >> 4)), bd = dB0 + (uint64_t)(s * (S::STAGE_BYTES >> 4));
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk)
            sm100::umma_bf16_warp(d_tmem, ad + 2 * kk, bd + 2 * kk, idesc, (kb | kk) != 0);
          sm100::umma_commit_warp(&empty[s]);
          if (++s == stages) { s = 0; ph ^= 1; }
        }
        sm100::umma_commit_warp(&tfull[acc]);
      }
    }
  } else {
    // ------------------------------------------------------------ fused gate epilogue (8 warps)
    const int ew = warp - 2;
    const int quarter = warp & 3;            // TMEM lane quarter of this warp
    const int half = ew / 4;                 // which 32 of the tile's 64 units
    const int row = quarter * 32 + lane;
    const int m = m0 + row;
    const bool valid = m < a.B;
    const long NG = a.NG;
    int local = 0;
    for (int t = a.t0; t < a.t1; ++t, ++local) {
      const int acc = local & 1;
      sm100::mbar_wait(&tfull[acc], (uint32_t)((local >> 1) & 1));
      sm100::tc_fence_after();
      const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * BN;
      const long r = (long)t * a.B + m;      // row of step t in [T·B] buffers
#pragma unroll 1
      for (int uc = 0; uc < 2; ++uc) {
        const int ul = half * 32 + uc * 16;  // first local unit of this chunk
        float z[4][16];
#pragma unroll
        for (int g = 0; g < 4; ++g) sm100::tmem_ld16(taddr + g * 64 + ul, z[g]);
        if (valid) {
          const float* wxr = a.WX + r * NG + n0;
          float* uhr = a.UH + r * NG + n0;
          float wx[4][16];
#pragma unroll
          for (int g = 0; g < 4; ++g) {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const float4 v = reinterpret_cast<const float4*>(wxr + g * 64 + ul)[q];
              wx[g][4 * q] = v.x; wx[g][4 * q + 1] = v.y; wx[g][4 * q + 2] = v.z; wx[g][4 * q + 3] = v.w;
              reinterpret_cast<float4*>(uhr + g * 64 + ul)[q] =
                  make_float4(z[g][4 * q], z[g][4 * q + 1], z[g][4 * q + 2], z[g][4 * q + 3]);
            }
          }
          const float* cp = a.C + r * a.Hp + u0 + ul;
          float* cn = a.C + (r + a.B) * a.Hp + u0 + ul;
          __nv_bfloat16* hn = a.Hb + (r + a.B) * (a.ldh ? a.ldh : (long)a.Hp) + u0 + ul;
          float cv[16], hv[16];
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            const int unit = u0 + ul + i;
            float pa[4];
#pragma unroll
            for (int g = 0; g < 4; ++g) {
              const int c = g * 64 + ul + i;
              pa[g] = preact<KIND, true>(wx[g][i], z[g][i], prm[c], prm[BN + c], prm[2 * BN + c], prm[3 * BN + c]);
            }
            float c_, h_;
            cell_fwd<KIND, true>(pa, cp[i], c_, h_);
            if (unit >= a.H) { c_ = 0.f; h_ = 0.f; }
            cv[i] = c_;
            hv[i] = h_;
          }
#pragma unroll
          for (int q = 0; q < 4; ++q)
            reinterpret_cast<float4*>(cn)[q] = make_float4(cv[4 * q], cv[4 * q + 1], cv[4 * q + 2], cv[4 * q + 3]);
          uint4 pk[2];
          uint32_t* pu = reinterpret_cast<uint32_t*>(pk);
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            __nv_bfloat162 b2 = __floats2bfloat162_rn(hv[2 * i], hv[2 * i + 1]);
            pu[i] = *reinterpret_cast<uint32_t*>(&b2);
          }
          reinterpret_cast<uint4*>(hn)[0] = pk[0];
          reinterpret_cast<uint4*>(hn)[1] = pk[1];
          const bool last = t == a.T - 1;
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            const int unit = u0 + ul + i;
            if (unit >= a.H) continue;
            if (a.y_kind == 1)
              reinterpret_cast<__nv_bfloat16*>(a.y)[r * a.ldy + unit] = __float2bfloat16_rn(hv[i]);
            else if (a.y_kind == 2)
              reinterpret_cast<float*>(a.y)[r * a.ldy + unit] = hv[i];
            if (last && a.hT) a.hT[(long)m * a.H + unit] = hv[i];
            if (last && a.cT) a.cT[(long)m * a.H + unit] = cv[i];
          }
        }
      }
      sm100::tc_fence_before();
      sm100::mbar_arrive(&tempty[acc]);
      if (a.persistent && t + 1 < a.t1) {     // publish h_t of this tile to the row block
        fence_proxy_async_global();
        __threadfence();
        epi_bar();
        if (ew == 0 && lane == 0) atomicAdd(a.flags + m_blk, 1u);
      }
    }
  }
  __syncthreads();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, 512);
  }
}

static int rf_smem_bytes(int stages, int stage_bytes, int prm_floats) {
  return 1024 + stages * stage_bytes + prm_floats * 4 + 256;
}

void lstm_rec_fwd_launch(int kind, const CUtensorMap& mapA, const CUtensorMap& mapB, RecFwdArgs a, cudaStream_t st) {
  using S = TcSmem<256>;
  int dev = 0, maxs = 0, nsm = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  CUDA_TRY(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  int stages = (maxs - 1024 - 256 - 4 * 256 * 4) / S::STAGE_BYTES;
  if (stages > 4) stages = 4;
  a.stages = stages;
  a.nk = cdiv(a.K ? a.K : a.Hp, TC_BK);
  const int smem = rf_smem_bytes(stages, S::STAGE_BYTES, 4 * 256);
  const int grid = a.num_m * a.num_n;
  ASTRA_CHECK_ARG(!a.persistent || grid <= nsm, "fused recurrent kernel: persistent mode needs one CTA per SM");
  void (*fn)(CUtensorMap, CUtensorMap, RecFwdArgs) = nullptr;
  switch (kind) {
    case K_LSTM: fn = lstm_rec_fwd_kernel<K_LSTM>; break;
    case K_MILSTM: fn = lstm_rec_fwd_kernel<K_MILSTM>; break;
    default: fn = lstm_rec_fwd_kernel<K_SUBLSTM>; break;
  }
  CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(RF_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = a.persistent ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  CUDA_TRY(cudaLaunchKernelEx(&cfg, fn, mapA, mapB, a));
  LAUNCH_CHECK();
}

}  // namespace astra
