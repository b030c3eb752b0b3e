// K2 for SC-RNN [22] (SURVEY §8(a) row a3 "SC-RNN's context blend", §8(a.9) `fwd_kernel`): the whole
// h-chain of the forward in ONE cooperative launch for B ≤ 128 — the SCRN counterpart of the LSTM
// family's small-batch persistent forward (rec_persist.cu).
//
// Per step t the chain computes  h_t = σ(Q_t + h_{t−1}·R + b_h)  where Q_t = x_t·A + s_t·P is the
// context blend, hoisted before the chain (the s-scan and the [X|S]·[A;P] ladder, rows a1/a2).  Each
// CTA owns 16 hidden units: its R slice (16 rows of the R mirror, K = Hp) is resident in shared
// memory for the whole chain (32 KB at H = 1024); h_{t−1} streams in through a TMA ring (4-D boxes of
// 4 k-blocks); one thread issues the tcgen05 MMAs (M = 128 rows, N = 16 units); the canonical split
// of reading R33 (s fixed K chunks, each accumulated from zero) is kept as s TMEM accumulators; the
// 8 epilogue warps sum them in chunk order, add Q_t and b_h, apply σ and store h_t (bf16 operand,
// fp32 copy, y); one grid-wide release/acquire counter per step publishes h_t.
//
// Numerics (R1, R3, R17, R33): every chunk partial is the launched chain's tc_gemm partial (one
// fp32 accumulation from zero over the chunk's k-blocks in ascending order), the partials are
// summed in chunk order exactly as sum_split, and σ((Q + z) + b) is scrn_fwd_pw_kernel's expression
// with the same fast-math sigmoid (bf16 path) — bitwise equal to GEMM + pointwise.
#include "cell_math.cuh"
#include "gemm.h"
#include "gemm_tc.cuh"
#include "kernels.h"
#include "pdl.cuh"
#include "rec_fused.h"

namespace astra {

constexpr int SP_UC = 16;                  // hidden units per CTA = MMA N
constexpr int SP_BT = SP_UC * TC_BK * 2;   // bytes of one B k-block (16 rows x 128 B)
constexpr int SP_EPI_WARPS = 8;
constexpr int SP_THREADS = 32 * (2 + SP_EPI_WARPS);   // warp 0 producer, 1 MMA, 2..9 epilogue
constexpr int SP_KA = 4;                   // k-blocks per A stage
constexpr int SP_SA = 4;                   // A stages

__device__ __forceinline__ void sp_fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ unsigned sp_ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void sp_epi_bar() { asm volatile("bar.sync 1, %0;" ::"n"(32 * SP_EPI_WARPS) : "memory"); }

__global__ void __launch_bounds__(SP_THREADS, 1)
    scrn_fwd_persist_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                            const ScrnPersistArgs a) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int nk = a.nk, ka = a.ka, SA = SP_SA;
  const int stage_bytes = ka * a.a_bytes;
  // [A ring][resident R slice][b_h][barriers]; the A ring first (the MMA reads 128 rows of a
  // 64-row k-block tile: the rows past the tile stay inside the allocation)
  uint8_t* sA = smem;
  uint8_t* sRes = sA + SA * stage_bytes;
  float* prm = reinterpret_cast<float*>(sRes + nk * SP_BT);
  uint64_t* fullA = reinterpret_cast<uint64_t*>(prm + SP_UC);
  uint64_t* emptyA = fullA + SA;
  uint64_t* resbar = emptyA + SA;
  uint64_t* tfull = resbar + 1;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int u0 = blockIdx.x * SP_UC;
  const unsigned nct = gridDim.x;
  const int ns = a.nsplit, kper = a.kper;
  const int acc_cols = ns * SP_UC;   // one accumulator set: ns chunk partials x 16 units

  if (threadIdx.x == 0) {
    for (int s = 0; s < SA; ++s) {
      sm100::mbar_init(&fullA[s], 1);
      sm100::mbar_init(&emptyA[s], 1);
    }
    sm100::mbar_init(resbar, 1);
    for (int q = 0; q < 2; ++q) {
      sm100::mbar_init(&tfull[q], 1);
      sm100::mbar_init(&tempty[q], 32 * SP_EPI_WARPS);
    }
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, 128);
  for (int c = threadIdx.x; c < SP_UC; c += SP_THREADS) prm[c] = u0 + c < a.H ? a.bh[u0 + c] : 0.f;
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ producer: R slice once, then h_{t−1}
    {   // whole warp: the *_warp TMA / arrive forms elect the issuing lane
      const uint64_t pol = sm100::l2_policy_evict_last();
      pdl_wait();
      sm100::mbar_arrive_expect_tx_warp(resbar, (uint32_t)(nk * SP_BT));
      for (int kb = 0; kb < nk; kb += 8) {
        const int n = nk - kb < 8 ? nk - kb : 8;
        for (int j = 0; j < n; ++j)   // 3-D box {64, 16 units, 1 k-block}
          sm100::tma_load_3d_hint_warp(sRes + (kb + j) * SP_BT, &mapB, resbar, 0, u0, kb + j, pol);
      }
      int s = 0;
      uint32_t ph = 0;
      for (int t = a.t0; t < a.t1; ++t) {
        if (t > a.t0) {   // every CTA has published h_{t−1}
          while (sp_ld_acquire(a.flags) < nct * (unsigned)(t - a.t0)) __nanosleep(32);
          sp_fence_proxy_async_global();
        }
        for (int kb = 0; kb < nk; kb += ka) {
          sm100::mbar_wait(&emptyA[s], ph ^ 1);
          sm100::mbar_arrive_expect_tx_warp(&fullA[s], (uint32_t)stage_bytes);
          sm100::tma_load_4d_warp(sA + s * stage_bytes, &mapA, &fullA[s], 0, 0, kb, t);
          if (++s == SA) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer (lean loop, see rec_persist.cu)
    {   // whole warp: umma_*_warp elect the issuing lane
      sm100::mbar_wait(resbar, 0);
      sm100::tc_fence_after();
      const uint32_t idesc = a.idesc;
      const uint64_t dA0 = sm100::smem_desc_sw128(sm100::smem_u32(sA), 16, 1024);
      const uint64_t dR0 = sm100::smem_desc_sw128(sm100::smem_u32(sRes), 16, 1024);
      const uint32_t a_kb = (uint32_t)a.a_bytes >> 4, a_st = (uint32_t)stage_bytes >> 4, b_kb = SP_BT >> 4;
      int sa = 0;
      uint32_t pa = 0;
      int local = 0;
      for (int t = a.t0; t < a.t1; ++t, ++local) {
        const int acc = local & 1;
        sm100::mbar_wait(&tempty[acc], (uint32_t)((local >> 1) & 1) ^ 1);
        sm100::tc_fence_after();
        int ja = ka, jk = 0, q = 0;   // ja: k-blocks used of the A stage; jk: of the chunk q
        uint64_t adesc = 0;
        for (int kb = 0; kb < nk; ++kb) {
          if (ja == ka) {
            sm100::mbar_wait(&fullA[sa], pa);
            sm100::tc_fence_after();
            adesc = dA0 + (uint64_t)(sa * a_st);
            ja = 0;
          }
          const uint32_t d_tmem = tmem_base + acc * acc_cols + q * SP_UC;
          const uint64_t bd = dR0 + (uint64_t)(kb * b_kb);
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk)
            sm100::umma_bf16_warp(d_tmem, adesc + 2 * kk, bd + 2 * kk, idesc, (jk | kk) != 0);
          adesc += a_kb;
          if (++ja == ka) {
            sm100::umma_commit_warp(&emptyA[sa]);
            if (++sa == SA) { sa = 0; pa ^= 1; }
          }
          if (++jk == kper) { jk = 0; ++q; }   // next canonical split-K chunk (R33): a fresh accumulator
        }
        sm100::umma_commit_warp(&tfull[acc]);
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue (8 warps)
    const int ew = warp - 2;
    const int quarter = warp & 3;
    const int half = ew >> 2;                 // units [8·half, 8·half + 8)
    const int row = quarter * 32 + lane;
    const bool valid = row < a.B;
    const int ul0 = half * 8, unit0 = u0 + ul0;
    pdl_wait();
    int local = 0;
    for (int t = a.t0; t < a.t1; ++t, ++local) {
      const int acc = local & 1;
      const long r = (long)t * a.B + row;
      float qv[8];   // Q_t (hoisted context blend): old data, loaded while the MMAs run
      if (valid) {
        const float4* qp = reinterpret_cast<const float4*>(a.Q + r * a.ldq + unit0);
        const float4 q0 = __ldcs(qp), q1 = __ldcs(qp + 1);
        qv[0] = q0.x; qv[1] = q0.y; qv[2] = q0.z; qv[3] = q0.w;
        qv[4] = q1.x; qv[5] = q1.y; qv[6] = q1.z; qv[7] = q1.w;
      }
      sm100::mbar_wait(&tfull[acc], (uint32_t)((local >> 1) & 1));
      sm100::tc_fence_after();
      const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * acc_cols + ul0;
      float z[8];
      {
        uint32_t zr[8];
        sm100::tmem_ld8_nowait(taddr, zr);
        sm100::tmem_wait_ld();
#pragma unroll
        for (int i = 0; i < 8; ++i) z[i] = __uint_as_float(zr[i]);
        for (int c = 1; c < ns; ++c) {   // partials summed in chunk order (sum_split)
          sm100::tmem_ld8_nowait(taddr + c * SP_UC, zr);
          sm100::tmem_wait_ld();
#pragma unroll
          for (int i = 0; i < 8; ++i) z[i] = __fadd_rn(z[i], __uint_as_float(zr[i]));
        }
      }
      sm100::tc_fence_before();
      sm100::mbar_arrive(&tempty[acc]);
      float hv[8];
      uint4 hp;
      if (valid) {
#pragma unroll
        for (int i = 0; i < 8; ++i)
          hv[i] = unit0 + i < a.H ? sigm<true>(__fadd_rn(__fadd_rn(qv[i], z[i]), prm[ul0 + i])) : 0.f;
        uint32_t* hw = reinterpret_cast<uint32_t*>(&hp);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          __nv_bfloat162 b2 = __floats2bfloat162_rn(hv[2 * i], hv[2 * i + 1]);
          hw[i] = *reinterpret_cast<uint32_t*>(&b2);
        }
        *reinterpret_cast<uint4*>(a.HS + (r + a.B) * a.ldhs + unit0) = hp;   // next step's operand
      }
      if (t + 1 < a.t1) {   // publish h_t (generic-proxy stores → the other CTAs' TMA reads)
        sp_fence_proxy_async_global();
        __threadfence();
        sp_epi_bar();
        if (ew == 0 && lane == 0) atomicAdd(a.flags, 1u);
      }
      if (valid) {   // the stores no other CTA reads this step
        float4* hf = reinterpret_cast<float4*>(a.Hf + (r + a.B) * a.Hp + unit0);
        hf[0] = make_float4(hv[0], hv[1], hv[2], hv[3]);
        hf[1] = make_float4(hv[4], hv[5], hv[6], hv[7]);
        if (a.y) {
          __nv_bfloat16* yp = a.y + r * a.ldy + unit0;
#pragma unroll
          for (int i = 0; i < 8; ++i)
            if (unit0 + i < a.H) yp[i] = __float2bfloat16_rn(hv[i]);
        }
        if (t == a.T - 1 && a.hT) {
#pragma unroll
          for (int i = 0; i < 8; ++i)
            if (unit0 + i < a.H) a.hT[(long)row * a.H + unit0 + i] = hv[i];
        }
      }
    }
  }
  __syncthreads();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, 128);
  }
}

// ============================================================================ BPTT (bwd_mode 1)
// The SC-RNN h-chain backward in one cooperative launch (SURVEY §8(a) row a5 for a non-LSTM cell):
//   dh_rec_t = dz_{t+1}·Rᵀ (R33 split kept as TMEM accumulators, R resident as a K-major copy);
//   dz_t = (dy^h_t + Σ partials)·h_t·(1 − h_t) (scrn_bwd_pw_kernel's expression and rounding);
//   db_h partials: 32-row chunks, 8 row lanes each summing rows y, y+8, … in ascending order, lanes
//   combined in y order, folded into the running partial step after step (its fixed order, R5).
// dz_t (bf16) is the next step's A operand: written, fenced, released through one grid counter.
constexpr int SPB_RB = 32, SPB_RY = 8;   // scrn_bwd_pw_kernel's PW_RB / PW_RY

template <typename TDY>
__global__ void __launch_bounds__(SP_THREADS, 1)
    scrn_bwd_persist_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                            const ScrnBpttArgs a) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int nk = a.nk, ka = a.ka, SA = SP_SA;
  const int stage_bytes = ka * a.a_bytes;
  const int nch = (a.B + SPB_RB - 1) / SPB_RB;   // db_h row chunks
  uint8_t* sA = smem;
  uint8_t* sRes = sA + SA * stage_bytes;
  float* sdz = reinterpret_cast<float*>(sRes + nk * SP_BT);    // [128 rows][16 units] this step's dz
  float* slane = sdz + 128 * SP_UC;                            // [4 chunks][8 lanes][16 units]
  float* spart = slane + 4 * SPB_RY * SP_UC;                   // [4 chunks][16 units] running partials
  uint64_t* fullA = reinterpret_cast<uint64_t*>(spart + 4 * SP_UC);
  uint64_t* emptyA = fullA + SA;
  uint64_t* resbar = emptyA + SA;
  uint64_t* tfull = resbar + 1;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int u0 = blockIdx.x * SP_UC;
  const unsigned nct = gridDim.x;
  const int ns = a.nsplit, kper = a.kper;
  const int acc_cols = ns * SP_UC;
  const int T = a.T;

  if (threadIdx.x == 0) {
    for (int s = 0; s < SA; ++s) {
      sm100::mbar_init(&fullA[s], 1);
      sm100::mbar_init(&emptyA[s], 1);
    }
    sm100::mbar_init(resbar, 1);
    for (int q = 0; q < 2; ++q) {
      sm100::mbar_init(&tfull[q], 1);
      sm100::mbar_init(&tempty[q], 32 * SP_EPI_WARPS);
    }
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, 128);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ producer: R once, then dz_{t+1}
    {   // whole warp: the *_warp TMA / arrive forms elect the issuing lane
      const uint64_t pol = sm100::l2_policy_evict_last();
      pdl_wait();
      sm100::mbar_arrive_expect_tx_warp(resbar, (uint32_t)(nk * SP_BT));
      for (int kb = 0; kb < nk; ++kb) sm100::tma_load_3d_hint_warp(sRes + kb * SP_BT, &mapB, resbar, 0, u0, kb, pol);
      int s = 0;
      uint32_t ph = 0;
      for (int t = T - 2; t >= 0; --t) {
        // every CTA has published dz_{t+1} (step t+1 is the (T−2−t)-th release)
        while (sp_ld_acquire(a.flags) < nct * (unsigned)(T - 1 - t)) __nanosleep(32);
        sp_fence_proxy_async_global();
        for (int kb = 0; kb < nk; kb += ka) {
          sm100::mbar_wait(&emptyA[s], ph ^ 1);
          sm100::mbar_arrive_expect_tx_warp(&fullA[s], (uint32_t)stage_bytes);
          sm100::tma_load_4d_warp(sA + s * stage_bytes, &mapA, &fullA[s], 0, 0, kb, t + 1);
          if (++s == SA) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    {   // whole warp: umma_*_warp elect the issuing lane
      sm100::mbar_wait(resbar, 0);
      sm100::tc_fence_after();
      const uint32_t idesc = a.idesc;
      const uint64_t dA0 = sm100::smem_desc_sw128(sm100::smem_u32(sA), 16, 1024);
      const uint64_t dR0 = sm100::smem_desc_sw128(sm100::smem_u32(sRes), 16, 1024);
      const uint32_t a_kb = (uint32_t)a.a_bytes >> 4, a_st = (uint32_t)stage_bytes >> 4, b_kb = SP_BT >> 4;
      int sa = 0;
      uint32_t pa = 0;
      int local = 0;
      for (int t = T - 2; t >= 0; --t, ++local) {
        const int acc = local & 1;
        sm100::mbar_wait(&tempty[acc], (uint32_t)((local >> 1) & 1) ^ 1);
        sm100::tc_fence_after();
        int ja = ka, jk = 0, q = 0;
        uint64_t adesc = 0;
        for (int kb = 0; kb < nk; ++kb) {
          if (ja == ka) {
            sm100::mbar_wait(&fullA[sa], pa);
            sm100::tc_fence_after();
            adesc = dA0 + (uint64_t)(sa * a_st);
            ja = 0;
          }
          const uint32_t d_tmem = tmem_base + acc * acc_cols + q * SP_UC;
          const uint64_t bd = dR0 + (uint64_t)(kb * b_kb);
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk)
            sm100::umma_bf16_warp(d_tmem, adesc + 2 * kk, bd + 2 * kk, idesc, (jk | kk) != 0);
          adesc += a_kb;
          if (++ja == ka) {
            sm100::umma_commit_warp(&emptyA[sa]);
            if (++sa == SA) { sa = 0; pa ^= 1; }
          }
          if (++jk == kper) { jk = 0; ++q; }
        }
        sm100::umma_commit_warp(&tfull[acc]);
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue (8 warps)
    const int ew = warp - 2;
    const int quarter = warp & 3;
    const int half = ew >> 2;
    const int row = quarter * 32 + lane;
    const bool valid = row < a.B;
    const int ul0 = half * 8, unit0 = u0 + ul0;
    const int etid = ew * 32 + lane;   // 0..255
    pdl_wait();
    int local = 0;
    for (int t = T - 1; t >= 0; --t) {
      const long r = (long)t * a.B + row;
      float gv[8], hv[8];   // dy^h_t and h_t: older than the chain, loaded before the MMAs finish
      if (valid) {
        const TDY* dp = reinterpret_cast<const TDY*>(a.dy) + r * a.ldy + unit0;
#pragma unroll
        for (int i = 0; i < 8; ++i) gv[i] = unit0 + i < a.H ? to_f<TDY>(dp[i]) : 0.f;
        const float4* hp = reinterpret_cast<const float4*>(a.Hf + (r + a.B) * a.Hp + unit0);
        const float4 h0 = hp[0], h1 = hp[1];
        hv[0] = h0.x; hv[1] = h0.y; hv[2] = h0.z; hv[3] = h0.w;
        hv[4] = h1.x; hv[5] = h1.y; hv[6] = h1.z; hv[7] = h1.w;
      }
      if (t < T - 1) {
        const int acc = local & 1;
        sm100::mbar_wait(&tfull[acc], (uint32_t)((local >> 1) & 1));
        sm100::tc_fence_after();
        const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * acc_cols + ul0;
        float z[8];
        uint32_t zr[8];
        sm100::tmem_ld8_nowait(taddr, zr);
        sm100::tmem_wait_ld();
#pragma unroll
        for (int i = 0; i < 8; ++i) z[i] = __uint_as_float(zr[i]);
        for (int c = 1; c < ns; ++c) {   // partials summed in chunk order (sum_split)
          sm100::tmem_ld8_nowait(taddr + c * SP_UC, zr);
          sm100::tmem_wait_ld();
#pragma unroll
          for (int i = 0; i < 8; ++i) z[i] = __fadd_rn(z[i], __uint_as_float(zr[i]));
        }
        sm100::tc_fence_before();
        sm100::mbar_arrive(&tempty[acc]);
        ++local;
#pragma unroll
        for (int i = 0; i < 8; ++i) gv[i] = __fadd_rn(gv[i], z[i]);
      } else if (a.dhT && valid) {   // t = T − 1: the caller's dhT (one "partial")
#pragma unroll
        for (int i = 0; i < 8; ++i)
          if (unit0 + i < a.H) gv[i] = __fadd_rn(gv[i], a.dhT[(long)row * a.H + unit0 + i]);
      }
      float dz[8];
#pragma unroll
      for (int i = 0; i < 8; ++i)
        dz[i] = (valid && unit0 + i < a.H) ? __fmul_rn(__fmul_rn(gv[i], hv[i]), __fsub_rn(1.f, hv[i])) : 0.f;
      if (valid) {
        uint4 pk;
        uint32_t* pw = reinterpret_cast<uint32_t*>(&pk);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          __nv_bfloat162 b2 = __floats2bfloat162_rn(dz[2 * i], dz[2 * i + 1]);
          pw[i] = *reinterpret_cast<uint32_t*>(&b2);
        }
        *reinterpret_cast<uint4*>(a.DZ + r * a.lddz + unit0) = pk;   // the next step's operand
      }
      if (t > 0) {   // publish dz_t
        sp_fence_proxy_async_global();
        __threadfence();
        sp_epi_bar();
        if (ew == 0 && lane == 0) atomicAdd(a.flags, 1u);
      }
      // db_h column partials in scrn_bwd_pw_kernel's order
#pragma unroll
      for (int i = 0; i < 8; ++i) sdz[row * SP_UC + ul0 + i] = dz[i];
      sp_epi_bar();
      for (int it = etid; it < nch * SPB_RY * SP_UC; it += 32 * SP_EPI_WARPS) {
        const int u = it % SP_UC, y = (it / SP_UC) % SPB_RY, c = it / (SP_UC * SPB_RY);
        float sacc = 0.f;
        for (int rr = y; rr < SPB_RB && c * SPB_RB + rr < a.B; rr += SPB_RY)
          sacc = __fadd_rn(sacc, sdz[(c * SPB_RB + rr) * SP_UC + u]);
        slane[(c * SPB_RY + y) * SP_UC + u] = sacc;
      }
      sp_epi_bar();
      for (int it = etid; it < nch * SP_UC; it += 32 * SP_EPI_WARPS) {
        const int u = it % SP_UC, c = it / SP_UC;
        float v = 0.f;
#pragma unroll
        for (int y = 0; y < SPB_RY; ++y) v = __fadd_rn(v, slane[(c * SPB_RY + y) * SP_UC + u]);
        spart[c * SP_UC + u] = t == T - 1 ? v : __fadd_rn(spart[c * SP_UC + u], v);
      }
      sp_epi_bar();
    }
    for (int it = etid; it < nch * SP_UC; it += 32 * SP_EPI_WARPS) {
      const int u = it % SP_UC, c = it / SP_UC;
      if (u0 + u < a.Hp) a.part[(long)c * a.Hp + u0 + u] = spart[c * SP_UC + u];
    }
  }
  __syncthreads();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, 128);
  }
}

bool scrn_bwd_persist_supported(int B, int Hp, int nsplit, int T) {
  return T >= 2 && scrn_fwd_persist_supported(B, Hp, nsplit);
}

void scrn_bwd_persist_launch(const void* DZ, long lddz, const void* Rk, int T, bool dy_f32, ScrnBpttArgs a,
                             cudaStream_t st) {
  ASTRA_CHECK_ARG(scrn_bwd_persist_supported(a.B, a.Hp, a.nsplit, T), "persistent SCRN BPTT: unsupported shape");
  a.T = T;
  a.nk = a.Hp / TC_BK;
  a.kper = (a.nk + a.nsplit - 1) / a.nsplit;
  a.a_rows = a.B <= 64 ? 64 : 128;
  a.a_bytes = a.a_rows * TC_BK * 2;
  a.ka = 1;
  for (int c = SP_KA; c > 1; --c)
    if (a.nk % c == 0) { a.ka = c; break; }
  a.idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(SP_UC >> 3) << 17) | ((uint32_t)(TC_BM >> 4) << 24);
  CUtensorMap mA, mB;
  {   // dz part of the [dz | (1−α)ds] rows: {64 k, rows B, k-block (stride 128 B), t}
    const long dims[4] = {64, a.B, a.nk, T};
    const long str[3] = {lddz * 2, 128, (long)a.B * lddz * 2};
    const int box[4] = {64, a.a_rows, a.ka, 1};
    make_map_nd(&mA, DZ, 4, dims, str, box, 128);
  }
  {   // R (not transposed) rows k: {64 j, row k, k-block (stride 128 B)}
    const long dims[3] = {64, a.Hp, a.nk};
    const long str[2] = {(long)a.Hp * 2, 128};
    const int box[3] = {64, SP_UC, 1};
    make_map_nd(&mB, Rk, 3, dims, str, box, 128);
  }
  const int bars = (2 * SP_SA + 1 + 4) * 8 + 16;
  const int smem = 1024 + SP_SA * a.ka * a.a_bytes + a.nk * SP_BT + (128 * SP_UC + 4 * SPB_RY * SP_UC + 4 * SP_UC) * 4 + bars;
  int dev = 0, maxs = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  ASTRA_CHECK_ARG(smem <= maxs, "persistent SCRN BPTT: the R slice does not fit in shared memory");
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(a.Hp / SP_UC);
  cfg.blockDim = dim3(SP_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  if (dy_f32) {
    auto k = scrn_bwd_persist_kernel<float>;
    CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    CUDA_TRY(cudaLaunchKernelEx(&cfg, k, mA, mB, a));
  } else {
    auto k = scrn_bwd_persist_kernel<__nv_bfloat16>;
    CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    CUDA_TRY(cudaLaunchKernelEx(&cfg, k, mA, mB, a));
  }
  LAUNCH_CHECK();
}

bool scrn_fwd_persist_supported(int B, int Hp, int nsplit) {
  return B >= 1 && B <= 128 && Hp % SP_UC == 0 && Hp / SP_UC <= num_sms() && nsplit >= 1 && nsplit <= 4 &&
         2 * nsplit * SP_UC <= 128;
}

void scrn_fwd_persist_launch(const void* HS, long ldhs, const void* MR, int Tmax, ScrnPersistArgs a, cudaStream_t st) {
  ASTRA_CHECK_ARG(scrn_fwd_persist_supported(a.B, a.Hp, a.nsplit), "persistent SCRN forward: unsupported shape");
  a.nk = a.Hp / TC_BK;
  a.kper = (a.nk + a.nsplit - 1) / a.nsplit;
  a.a_rows = a.B <= 64 ? 64 : 128;
  a.a_bytes = a.a_rows * TC_BK * 2;
  a.ka = 1;
  for (int c = SP_KA; c > 1; --c)
    if (a.nk % c == 0) { a.ka = c; break; }
  a.idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(SP_UC >> 3) << 17) | ((uint32_t)(TC_BM >> 4) << 24);
  CUtensorMap mA, mB;
  {   // h part of the [h | s] operand rows: {64 k, rows B, k-block (stride 128 B), t}
    const long dims[4] = {64, a.B, a.nk, Tmax + 1};
    const long str[3] = {ldhs * 2, 128, (long)a.B * ldhs * 2};
    const int box[4] = {64, a.a_rows, a.ka, 1};
    make_map_nd(&mA, HS, 4, dims, str, box, 128);
  }
  {   // R mirror rows (output units): {64 k, unit row, k-block (stride 128 B)}
    const long dims[3] = {64, a.Hp, a.nk};
    const long str[2] = {(long)a.Hp * 2, 128};
    const int box[3] = {64, SP_UC, 1};
    make_map_nd(&mB, MR, 3, dims, str, box, 128);
  }
  const int bars = (2 * SP_SA + 1 + 4) * 8 + 16;
  const int smem = 1024 + SP_SA * a.ka * a.a_bytes + a.nk * SP_BT + SP_UC * 4 + bars;
  int dev = 0, maxs = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  ASTRA_CHECK_ARG(smem <= maxs, "persistent SCRN forward: the R slice does not fit in shared memory");
  CUDA_TRY(cudaFuncSetAttribute(scrn_fwd_persist_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(a.Hp / SP_UC);
  cfg.blockDim = dim3(SP_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  CUDA_TRY(cudaLaunchKernelEx(&cfg, scrn_fwd_persist_kernel, mA, mB, a));
  LAUNCH_CHECK();
}

}  // namespace astra
