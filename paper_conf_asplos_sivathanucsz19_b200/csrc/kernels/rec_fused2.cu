// K2 fused, CTA-pair form: one launch per step computes UH_t = h_{t-1}·U on the tcgen05 CTA-pair
// main loop (tc_gemm2_kernel's pipeline) and applies the LSTM-family cell update in the epilogue —
// the "fused gate epilogue" of the north star — without the UH round trip
// through a separate pointwise kernel.
//
// Tile: a CTA pair owns 256 batch rows x 256 gate-interleaved columns (64 units x 4 gates); each
// CTA's TMEM holds its 128 rows x 256 columns.  One tile per CTA (grid = 2 x tiles <= #SMs), so
// when the accumulator is complete the main-loop stage buffers are free and the epilogue reuses
// them: each of the 8 epilogue warps (32 rows x 32 units: TMEM lane quarter x unit half) pulls its
// WX_t slice (4 gates x 32 x 32 fp32) and c_{t-1} slice with TMA tensor loads into 128-byte-
// swizzled tiles, computes c_t and h_t per (row, unit) with cell_math.cuh (the same arithmetic as
// the unfused kernels: bitwise-identical results, tests/test_gpu_cell.py::test_fused_forward_modes),
// writes UH_t over the consumed WX slots, c_t over c_{t-1}, h_t (bf16) into a 64-byte-swizzled
// tile, and hands them to TMA tensor stores (UH_t saved for the backward pass, c_t, h_t as the next
// step's GEMM operand, y_t).  Rows >= B and units >= H are clipped by the copy engine.
#include "cell_math.cuh"
#include "gemm.h"
#include "kernels.h"
#include "pdl.cuh"
#include "rec_fused.h"
#include "sm100.cuh"

namespace astra {

constexpr int R2_EPI_WARPS = 8;
constexpr int R2_THREADS = 64 + 32 * R2_EPI_WARPS;
constexpr int R2_BN = 256;                       // pair tile width (64 units x 4 gates)
constexpr int R2_WARP_IN = 4 * 4096 + 4096;      // per epilogue warp: WX 4 gates x 4 KB + c 4 KB
constexpr int R2_HTILE = 32 * 32 * 2;            // per epilogue warp: h tile, 32 rows x 32 units bf16

template <int KIND>
__global__ void __launch_bounds__(R2_THREADS, 1)
    lstm_fwd_pair_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                         const __grid_constant__ CUtensorMap mapWX, const __grid_constant__ CUtensorMap mapUH,
                         const __grid_constant__ CUtensorMap mapC, const __grid_constant__ CUtensorMap mapH,
                         const __grid_constant__ CUtensorMap mapY, const RecFwd2Args a) {
  using S = TcSmem<R2_BN / 2>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int stages = a.stages;
  float4* prm = reinterpret_cast<float4*>(smem + stages * S::STAGE_BYTES);          // [4 gates][64 units]
  uint8_t* htiles = reinterpret_cast<uint8_t*>(prm + 4 * 64);                        // 8 x 2 KB, 512-aligned
  uint64_t* full = reinterpret_cast<uint64_t*>(htiles + R2_EPI_WARPS * R2_HTILE);
  uint64_t* empty = full + stages;
  uint64_t* tfull = empty + stages;
  uint64_t* ebar = tfull + 1;                                                        // [8] epilogue loads
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(ebar + R2_EPI_WARPS);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int rank = (int)sm100::cluster_ctarank();
  const int pair = blockIdx.x / 2;
  const int mp = pair % a.num_mp, nt = pair / a.num_mp;
  const int m0 = mp * 256 + rank * 128;        // this CTA's first batch row
  const int n0 = nt * R2_BN;                   // first gate-interleaved column of the pair tile
  const int u0 = nt * 64;                      // first hidden unit
  const int t = a.t;
  if (threadIdx.x == 0) GEMM_TRACE(0);

  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      sm100::mbar_init(&full[s], 1);
      sm100::mbar_init(&empty[s], 1);
    }
    sm100::mbar_init(tfull, 1);
    for (int w = 0; w < R2_EPI_WARPS; ++w) sm100::mbar_init(&ebar[w], 1);
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
  }
  if (warp == 1) sm100::tmem_alloc_cg2(tmem_slot, R2_BN);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::cluster_sync();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  if (threadIdx.x == 0) {
    // WX_t (written by the a1 GEMM long before) → L2 while the main loop runs
#pragma unroll 1
    for (int w = 0; w < R2_EPI_WARPS; ++w)
      for (int g = 0; g < 4; ++g)
        sm100::tma_prefetch_l2_box(&mapWX, n0 + g * 64 + (w / 4) * 32, m0 + ((w + 2) & 3) * 32, t);
  }
  if (warp == 0 && lane == 0) {
    // the U mirror (weights, written at the start of the step) for the first stages before the grid
    // dependency resolves; h_{t-1} (A) after it
    const uint64_t pol = sm100::l2_policy_evict_last();
    const int pre = a.nk < stages ? a.nk : stages;
    for (int kb = 0; kb < pre; ++kb) {
      uint8_t* sa = smem + kb * S::STAGE_BYTES;
      if (rank == 0) sm100::mbar_arrive_expect_tx(&full[kb], 2 * S::STAGE_BYTES);
      sm100::tma_load_3d_cg2_hint(sa + S::A_BYTES, &mapB, sm100::mapa_shared(sm100::smem_u32(&full[kb]), 0),
                                  kb * TC_BK, n0 + rank * (R2_BN / 2), 0, pol);
    }
  }
  pdl_wait();
  pdl_trigger();
  for (int i = threadIdx.x; i < 4 * 64; i += R2_THREADS) {   // per-(gate, unit) parameters
    const int g = i / 64, j = u0 + i % 64, e = g * a.H + j;
    const bool ok = j < a.H;
    prm[i] = make_float4(ok ? a.gp.b[e] : 0.f, (ok && KIND == K_MILSTM) ? a.gp.alpha[e] : 0.f,
                         (ok && KIND == K_MILSTM) ? a.gp.beta1[e] : 0.f, (ok && KIND == K_MILSTM) ? a.gp.beta2[e] : 0.f);
  }
  __syncthreads();
  if (threadIdx.x == 0) GEMM_TRACE(1);

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer (both CTAs)
    if (lane == 0) {
      const uint64_t pol = sm100::l2_policy_evict_last();
      const uint32_t bar0 = sm100::mapa_shared(sm100::smem_u32(&full[0]), 0);
      const int pre = a.nk < stages ? a.nk : stages;
      for (int kb = 0; kb < a.nk; ++kb) {
        const int s = kb % stages;
        if (kb >= pre) sm100::mbar_wait(&empty[s], (uint32_t)((kb / stages) & 1) ^ 1);
        uint8_t* sa = smem + s * S::STAGE_BYTES;
        if (kb >= pre && rank == 0) sm100::mbar_arrive_expect_tx(&full[s], 2 * S::STAGE_BYTES);
        const uint32_t bar = bar0 + (uint32_t)s * 8;
        sm100::tma_load_3d_cg2(sa, &mapA, bar, kb * TC_BK, m0, t);
        if (kb >= pre)
          sm100::tma_load_3d_cg2_hint(sa + S::A_BYTES, &mapB, bar, kb * TC_BK, n0 + rank * (R2_BN / 2), 0, pol);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer (pair leader)
    if (rank == 0) {   // whole warp (umma_*_warp elect the issuing lane); lean loop: descriptors advanced by (bytes >> 4)
      const uint32_t sa0 = sm100::smem_u32(smem);
      const uint64_t dA0 = sm100::smem_desc_sw128(sa0, 16, 1024);
      const uint64_t dB0 = sm100::smem_desc_sw128(sa0 + S::A_BYTES, 16, 1024);
      const uint32_t idesc = a.idesc;
      int s = 0;
      uint32_t ph = 0;
      for (int kb = 0; kb < a.nk; ++kb) {
        sm100::mbar_wait(&full[s], ph);
        if (kb == 0) GEMM_TRACE(3);
        sm100::tc_fence_after();
        const uint64_t ad = dA0 + (uint64_t)(s * (S::STAGE_BYTES >> 4)), bd = dB0 + (uint64_t)(s * (S::STAGE_BYTES >> 4));
#pragma unroll
        for (int kk = 0; kk < TC_BK / 16; ++kk)
          sm100::umma_bf16_cg2_warp(tmem_base, ad + 2 * kk, bd + 2 * kk, idesc, (kb | kk) != 0);
        sm100::umma_commit_cg2_mc_warp(&empty[s], 0x3);
        if (++s == stages) { s = 0; ph ^= 1; }
      }
      sm100::umma_commit_cg2_mc_warp(tfull, 0x3);
      GEMM_TRACE(4);
    }
  } else {
    // ------------------------------------------------------------ fused gate epilogue (8 warps)
    const int ew = warp - 2;
    const int quarter = warp & 3;            // TMEM lanes (rows) quarter·32 .. +31
    const int half = ew / 4;                 // units half·32 .. +31 of the tile's 64
    const int mq = m0 + quarter * 32;        // first batch row of this warp
    const int uc = u0 + half * 32;           // first unit of this warp
    uint8_t* wbuf = smem + ew * R2_WARP_IN;  // reuses the (drained) main-loop stages
    const uint32_t wx_s = sm100::smem_u32(wbuf), c_s = wx_s + 4 * 4096;
    const uint32_t h_s = sm100::smem_u32(htiles + ew * R2_HTILE);
    sm100::mbar_wait(tfull, 0);              // accumulator complete ⇒ every stage buffer consumed
    if (ew == 0 && lane == 0) GEMM_TRACE(5);
    sm100::tc_fence_after();
    if (lane == 0) {
      sm100::mbar_arrive_expect_tx(&ebar[ew], R2_WARP_IN);
#pragma unroll
      for (int g = 0; g < 4; ++g) sm100::tma_load_box(wx_s + g * 4096, &mapWX, &ebar[ew], n0 + g * 64 + half * 32, mq, t);
      sm100::tma_load_box(c_s, &mapC, &ebar[ew], uc, mq, t);
    }
    sm100::mbar_wait(&ebar[ew], 0);
    if (ew == 0 && lane == 0) GEMM_TRACE(6);
    const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16);
    const int r = lane;                       // this thread's row within the warp's 32
    const bool last = t == a.T - 1;
#pragma unroll 1
    for (int sc = 0; sc < 4; ++sc) {          // 8 units per sub-chunk
      uint32_t zr[4][8];
#pragma unroll
      for (int g = 0; g < 4; ++g) sm100::tmem_ld8_nowait(taddr + g * 64 + half * 32 + sc * 8, zr[g]);
      sm100::tmem_wait_ld();
      // 16-byte chunks 2sc, 2sc+1 of this row in the 128-byte-swizzled tiles
      const uint32_t o0 = (uint32_t)r * 128 + (uint32_t)(((2 * sc) ^ (r & 7)) * 16);
      const uint32_t o1 = (uint32_t)r * 128 + (uint32_t)(((2 * sc + 1) ^ (r & 7)) * 16);
      float wx[4][8], cp[8];
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        const float4 v0 = sm100::lds_v4(wx_s + g * 4096 + o0), v1 = sm100::lds_v4(wx_s + g * 4096 + o1);
        wx[g][0] = v0.x; wx[g][1] = v0.y; wx[g][2] = v0.z; wx[g][3] = v0.w;
        wx[g][4] = v1.x; wx[g][5] = v1.y; wx[g][6] = v1.z; wx[g][7] = v1.w;
      }
      {
        const float4 v0 = sm100::lds_v4(c_s + o0), v1 = sm100::lds_v4(c_s + o1);
        cp[0] = v0.x; cp[1] = v0.y; cp[2] = v0.z; cp[3] = v0.w; cp[4] = v1.x; cp[5] = v1.y; cp[6] = v1.z; cp[7] = v1.w;
      }
      float cv[8], hv[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const int ul = half * 32 + sc * 8 + i;   // unit within the tile
        const int j = u0 + ul;
        if (j < a.H) {
          float pa[4];
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            const float4 p = prm[g * 64 + ul];
            pa[g] = preact<KIND, true>(wx[g][i], __uint_as_float(zr[g][i]), p.x, p.y, p.z, p.w);
          }
          cell_fwd<KIND, FastMath<__nv_bfloat16>::value>(pa, cp[i], cv[i], hv[i]);
        } else {
          cv[i] = 0.f;
          hv[i] = 0.f;
        }
      }
      // UH over the consumed WX slots, c_t over c_{t-1}, h_t into the 64-byte-swizzled h tile
#pragma unroll
      for (int g = 0; g < 4; ++g) {
        sm100::sts_v4(wx_s + g * 4096 + o0, __uint_as_float(zr[g][0]), __uint_as_float(zr[g][1]),
                      __uint_as_float(zr[g][2]), __uint_as_float(zr[g][3]));
        sm100::sts_v4(wx_s + g * 4096 + o1, __uint_as_float(zr[g][4]), __uint_as_float(zr[g][5]),
                      __uint_as_float(zr[g][6]), __uint_as_float(zr[g][7]));
      }
      sm100::sts_v4(c_s + o0, cv[0], cv[1], cv[2], cv[3]);
      sm100::sts_v4(c_s + o1, cv[4], cv[5], cv[6], cv[7]);
      {
        uint32_t u[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          __nv_bfloat162 b2 = __floats2bfloat162_rn(hv[2 * i], hv[2 * i + 1]);
          u[i] = *reinterpret_cast<uint32_t*>(&b2);
        }
        sm100::sts_v4(h_s + (uint32_t)r * 64 + (uint32_t)((sc ^ ((r >> 1) & 3)) * 16), __uint_as_float(u[0]),
                      __uint_as_float(u[1]), __uint_as_float(u[2]), __uint_as_float(u[3]));
      }
      if (a.y_kind == 2 && mq + r < a.B) {  // y rows not TMA-mappable (odd H): element stores
        __nv_bfloat16* yr = reinterpret_cast<__nv_bfloat16*>(a.y) + ((long)t * a.B + mq + r) * a.H;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int j = uc + sc * 8 + i;
          if (j < a.H) yr[j] = __float2bfloat16_rn(hv[i]);
        }
      }
      if (last && mq + r < a.B) {            // final state (external [B][H] fp32)
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int j = uc + sc * 8 + i;
          if (j >= a.H) break;
          if (a.hT) a.hT[(long)(mq + r) * a.H + j] = hv[i];
          if (a.cT) a.cT[(long)(mq + r) * a.H + j] = cv[i];
        }
      }
    }
    if (ew == 0 && lane == 0) GEMM_TRACE(7);
    sm100::tc_fence_before();
    sm100::fence_proxy_async_smem();
    __syncwarp();
    if (lane == 0) {
#pragma unroll
      for (int g = 0; g < 4; ++g) sm100::tma_store_3d(&mapUH, wx_s + g * 4096, n0 + g * 64 + half * 32, mq, t);
      sm100::tma_store_3d(&mapC, c_s, uc, mq, t + 1);
      sm100::tma_store_3d(&mapH, h_s, uc, mq, t + 1);
      if (a.y_kind == 1) sm100::tma_store_3d(&mapY, h_s, uc, mq, t);
      sm100::bulk_commit();
      sm100::bulk_wait_read<0>();
      if (ew == 0) GEMM_TRACE(8);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) GEMM_TRACE(9);
  sm100::cluster_sync();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc_cg2(tmem_base, R2_BN);
  }
}

int lstm_fwd_pair_smem(int stages) {
  using S = TcSmem<R2_BN / 2>;
  return 1024 + stages * S::STAGE_BYTES + 4 * 64 * 16 + R2_EPI_WARPS * R2_HTILE + 256;
}

void lstm_fwd_pair_launch(int kind, const RecFwd2Maps& m, RecFwd2Args a, cudaStream_t st) {
  using S = TcSmem<R2_BN / 2>;
  int dev = 0, maxs = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  int stages = (maxs - lstm_fwd_pair_smem(0)) / S::STAGE_BYTES;
  if (stages > 8) stages = 8;
  ASTRA_CHECK_STATE(stages * S::STAGE_BYTES >= R2_EPI_WARPS * R2_WARP_IN, "fused forward: shared memory too small");
  a.stages = stages;
  a.nk = cdiv(a.Hp, TC_BK);
  const int smem = lstm_fwd_pair_smem(stages);
  void (*fn)(CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap,
             RecFwd2Args) = nullptr;
  switch (kind) {
    case K_LSTM: fn = lstm_fwd_pair_kernel<K_LSTM>; break;
    case K_MILSTM: fn = lstm_fwd_pair_kernel<K_MILSTM>; break;
    default: fn = lstm_fwd_pair_kernel<K_SUBLSTM>; break;
  }
  static int attr_bytes[8] = {0};
  if (attr_bytes[kind & 7] < smem) {
    CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    attr_bytes[kind & 7] = smem;
  }
  launch_pdl(fn, dim3(2 * a.num_mp * a.num_n), dim3(R2_THREADS), smem, st, 2, m.A, m.B, m.WX, m.UH, m.C, m.H, m.Y,
             a);
  LAUNCH_CHECK();
}

}  // namespace astra
