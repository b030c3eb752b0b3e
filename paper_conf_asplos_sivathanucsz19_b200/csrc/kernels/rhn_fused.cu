// K2 persistent fused forward of the RHN chain (SURVEY §8(a) row a3 for cfg3; §8(a.9) `fwd_kernel`
// "persistent" and `fwd_epilogue` "RHN micro-layers per launch {1, L}"; the cfg3 chain sat
// 7.5× above its launch-latency floor with one GEMM + one pointwise launch per micro-step).
//
// One cooperative launch runs all T·L micro-steps.  CTA (m_blk, n_blk) owns batch rows
// [128·m_blk, +128) and hidden units [32·n_blk, +32): its B tile is the 32 H-columns and the
// matching 32 T-columns of R_ℓ's gate-blocked mirror (two 32-row TMA boxes stacked into one
// 64-wide operand), so the highway epilogue has both pre-activations of its units in TMEM.  When
// it fits (cfg3: 13 k-blocks of 16 KB) the whole K of a micro-step is resident: R_{ℓ+1} is loaded
// while micro-step ℓ finishes, and after the row block's counter only A crosses L2, in one round.
// Per micro-step: TMA (A = s^{ℓ−1} bf16 operand, B = R_ℓ slice) → tcgen05 MMA into the canonical
// split-K chunk accumulators (reading R33: chunk c accumulated from zero in its own TMEM columns,
// exactly the chunks of the unfused GEMM) → epilogue warps sum the chunks in chunk order, add b_ℓ
// (and x_t·W at ℓ = 1), store the pre-activations (for BPTT), apply the highway update and write
// s^ℓ (fp32 + bf16 operand) → release/acquire counter per row block → the next micro-step's TMA
// reads the other CTAs' s^ℓ.  R_{ℓ+1} tiles are prefetched while the counter is awaited.  The
// arithmetic is rhn_fwd_pw_kernel's, operation for operation, so the result is bitwise identical
// to the unfused chain (tests/test_gpu_cell.py::test_rhn_fused_forward_bitwise).
#include <algorithm>

#include "cell_math.cuh"
#include "gemm.h"
#include "gemm_tc.cuh"
#include "kernels.h"
#include "rec_fused.h"

namespace astra {

namespace {

constexpr int RH_EPI_WARPS = 16;
constexpr int RH_THREADS = 64 + 32 * RH_EPI_WARPS;   // warp 0 TMA, warp 1 MMA, 16 epilogue warps (four per
                                                      // TMEM lane quarter, one per 8-unit quarter of the tile)
constexpr int RH_UW = 32 * 4 / (RH_EPI_WARPS);        // units per epilogue thread (8)
constexpr int RH_UB = 32;                             // hidden units per tile
constexpr int RH_BN = 2 * RH_UB;                      // MMA N: the units' H-columns then their T-columns
constexpr int RH_SP = RH_UB + 1;                      // row strides of the per-thread (row) shared buffers,
constexpr int RH_ZP = RH_BN + 1;                      // padded: a warp's 32 rows hit 32 different banks

__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t global_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// a row block that never completes (a co-residency or protocol fault) traps after 20 s instead of
// hanging the device: sticky CUDA error, ASTRA_E_CUDA on the next call
__device__ __forceinline__ void wait_flag(const unsigned* p, unsigned target) {
  const uint64_t t0 = global_ns();
  while (ld_acquire(p) < target) {
    __nanosleep(64);
    if (global_ns() - t0 > 20ull * 1000 * 1000 * 1000) __trap();
  }
}
__device__ __forceinline__ void red_release_gpu(unsigned* p, unsigned v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// mbarrier wait with back-off: the producer and MMA warps wait microseconds per micro-step for the
// epilogue; a hot try_wait loop would take issue slots from the epilogue warps sharing their scheduler
__device__ __forceinline__ bool mbar_try(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, P1;\n\t}"
      : "=r"(ok)
      : "r"(sm100::smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait_idle(uint64_t* bar, uint32_t parity) {
  while (!mbar_try(bar, parity)) __nanosleep(64);
}
__device__ __forceinline__ void epi_bar() { asm volatile("bar.sync 1, %0;" ::"n"(32 * RH_EPI_WARPS) : "memory"); }

__global__ void __launch_bounds__(RH_THREADS, 1)
    rhn_rec_fwd_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                       const RhnFwdArgs a) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int stages = a.stages;
  const int a_bytes = a.a_rows * TC_BK * 2, stage_bytes = a_bytes + RH_BN * TC_BK * 2;
  // s^{ℓ−1} of this CTA's rows and units stays on chip between micro-steps (the tile's own epilogue
  // produced it); the biases of every micro-layer for the tile's units are staged once
  float* sprev = reinterpret_cast<float*>(smem + stages * stage_bytes);   // [a_rows][RH_SP]
  float* bls = sprev + a.a_rows * RH_SP;                                  // [L][RH_BN]: b_H | b_T
  float* zst = bls + a.L * RH_BN;   // [a_rows][RH_ZP] pre-activations staged until after the publish
  uint64_t* full = reinterpret_cast<uint64_t*>(zst + ((a.a_rows * RH_ZP + 1) & ~1));
  uint64_t* empty = full + stages;
  uint64_t* tfull = empty + stages;
  uint64_t* tempty = tfull + 1;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int m_blk = blockIdx.x % a.num_m, n_blk = blockIdx.x / a.num_m;
  const int m0 = m_blk * TC_BM, u0 = n_blk * RH_UB;
  const int nk = a.nk, kper = a.kper;
  const int L = a.L;
  const int nsteps = (a.t1 - a.t0) * L;

  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      sm100::mbar_init(&full[s], 1);
      sm100::mbar_init(&empty[s], 1);
    }
    sm100::mbar_init(tfull, 1);
    sm100::mbar_init(tempty, 32 * RH_EPI_WARPS);
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, a.tmem_cols);
  for (int i = threadIdx.x; i < a.L * RH_BN; i += blockDim.x) {
    const int l = i / RH_BN, c = i % RH_BN, j = u0 + c % RH_UB;
    bls[i] = j < a.H ? a.b[(size_t)l * 2 * a.H + (c < RH_UB ? 0 : a.H) + j] : 0.f;
  }
  for (int i = threadIdx.x; i < a.a_rows * RH_UB; i += blockDim.x) {   // initial state s^0 at t0
    const int r = i / RH_UB, m = m0 + r;
    sprev[r * RH_SP + i % RH_UB] = m < a.B ? a.Sf[((size_t)a.t0 * a.B + m) * a.Hp + u0 + i % RH_UB] : 0.f;
  }
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    {   // whole warp: the *_warp TMA / arrive forms elect the issuing lane
      long it = 0;
      const uint64_t pol = sm100::l2_policy_evict_last();
      const int pre = nk < stages ? nk : stages;
      for (int q = 0; q < nsteps; ++q) {
        const int t = a.t0 + q / L, l = q % L;
        const int az = l * (a.T + 1) + t;   // the slot of s^{ℓ−1} at time t (RhnCell::slot)
        auto load_b = [&](int s, int kb) {
          uint8_t* sb = smem + s * stage_bytes + a_bytes;
          sm100::tma_load_3d_hint_warp(sb, &mapB, &full[s], kb * TC_BK, u0, l, pol);                        // H columns
          sm100::tma_load_3d_hint_warp(sb + RH_UB * 128, &mapB, &full[s], kb * TC_BK, a.Hp + u0, l, pol);  // T columns
        };
        for (int kb = 0; kb < pre; ++kb) {   // R_ℓ tiles do not depend on the recurrence
          const long i = it + kb;
          const int s = (int)(i % stages);
          mbar_wait_idle(&empty[s], (uint32_t)((i / stages) & 1) ^ 1);
          sm100::mbar_arrive_expect_tx_warp(&full[s], (uint32_t)stage_bytes);
          load_b(s, kb);
        }
        if (q > 0) {   // every CTA of the row block has stored s^{ℓ−1}
          wait_flag(a.flags + m_blk, (unsigned)(a.num_n * q));
          fence_proxy_async_global();
        }
        if (a.trace) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 0] = global_ns();
        for (int kb = 0; kb < pre; ++kb) {
          const int s = (int)((it + kb) % stages);
          sm100::tma_load_3d_warp(smem + s * stage_bytes, &mapA, &full[s], kb * TC_BK, m0, az);
        }
        for (int kb = pre; kb < nk; ++kb) {
          const long i = it + kb;
          const int s = (int)(i % stages);
          mbar_wait_idle(&empty[s], (uint32_t)((i / stages) & 1) ^ 1);
          sm100::mbar_arrive_expect_tx_warp(&full[s], (uint32_t)stage_bytes);
          sm100::tma_load_3d_warp(smem + s * stage_bytes, &mapA, &full[s], kb * TC_BK, m0, az);
          load_b(s, kb);
        }
        it += nk;
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    // Lean issue loop (round 2, cf. rec_persist.cu): stage bookkeeping by counters and shared-memory
    // descriptors advanced by adding (bytes >> 4) — the per-k-block scalar work (long divisions,
    // descriptor rebuilds) otherwise paced the k loop, not the operands' arrival.
    {   // whole warp: umma_*_warp elect the issuing lane
      const uint64_t dA0 = sm100::smem_desc_sw128(sm100::smem_u32(smem), 16, 1024);
      const uint64_t dB0 = sm100::smem_desc_sw128(sm100::smem_u32(smem) + a_bytes, 16, 1024);
      const uint32_t st_step = (uint32_t)stage_bytes >> 4;
      const uint32_t idesc = a.idesc;
      int s = 0;
      uint32_t ph = 0;
      for (int q = 0; q < nsteps; ++q) {
        mbar_wait_idle(tempty, (uint32_t)(q & 1) ^ 1);
        sm100::tc_fence_after();
        int c = 0, jk = 0;   // canonical split-K chunk (R33) and k-block within it
        for (int kb = 0; kb < nk; ++kb) {
          sm100::mbar_wait(&full[s], ph);
          sm100::tc_fence_after();
          if (a.trace && kb == 0) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 1] = global_ns();
          if (a.trace && kb == nk - 1) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 2] = global_ns();
          // a_rows = 64: the M = 128 MMA's rows 64..127 read the B tile's bytes — garbage rows of
          // TMEM that the epilogue never reads (rows ≥ B)
          const uint64_t ad = dA0 + (uint64_t)(s * st_step), bd = dB0 + (uint64_t)(s * st_step);
          const uint32_t d_tmem = tmem_base + c * RH_BN;
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk)
            sm100::umma_bf16_warp(d_tmem, ad + 2 * kk, bd + 2 * kk, idesc, (jk | kk) != 0);
          sm100::umma_commit_warp(&empty[s]);
          if (++s == stages) { s = 0; ph ^= 1; }
          if (++jk == kper) { jk = 0; ++c; }
        }
        sm100::umma_commit_warp(tfull);
      }
    }
  } else {
    // ------------------------------------------------------------ highway epilogue (16 warps)
    const int quarter = warp & 3;            // TMEM lane quarter of this warp
    const int uc = (warp - 2) / 4;           // the RH_UW-unit part of the tile this warp applies: at B ≤ 64
                                             // only the warps of lane quarters 0 / 1 have rows, so the
                                             // units are spread over four of them per quarter
    const int row = quarter * 32 + lane;
    const int m = m0 + row;
    const bool valid = m < a.B;
    const long G2 = 2L * a.Hp;
    for (int q = 0; q < nsteps; ++q) {
      const int t = a.t0 + q / L, l = q % L;
      const bool last = l == L - 1;
      sm100::mbar_wait(tfull, (uint32_t)(q & 1));
      sm100::tc_fence_after();
      if (a.trace && warp == 2 && lane == 0) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 3] = global_ns();
      const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16);
      const float* bl = bls + l * RH_BN;
      const size_t slot_out = last ? (size_t)(t + 1) * a.B * a.Hp : ((size_t)(l + 1) * (a.T + 1) + t) * a.B * a.Hp;
      float* Z = a.Apre + ((size_t)l * a.T + t) * a.B * G2 + (size_t)m * G2;   // row m
      const float* wx = a.WX + ((size_t)t * a.B + m) * G2;
      float* spr = sprev + row * RH_SP;   // valid rows only (m < B ≤ a_rows when a_rows = 64)
      float* zr = zst + row * RH_ZP;
      {
        const int ul = uc * RH_UW;
        float xh[RH_UW], xt[RH_UW];
        if (l == 0 && valid) {   // x_t·W (ℓ = 1 only): independent of the MMA, issued first
#pragma unroll
          for (int q4 = 0; q4 < RH_UW / 4; ++q4) {
            const float4 h4 = reinterpret_cast<const float4*>(wx + u0 + ul)[q4];
            const float4 t4 = reinterpret_cast<const float4*>(wx + a.Hp + u0 + ul)[q4];
            xh[4 * q4] = h4.x; xh[4 * q4 + 1] = h4.y; xh[4 * q4 + 2] = h4.z; xh[4 * q4 + 3] = h4.w;
            xt[4 * q4] = t4.x; xt[4 * q4 + 1] = t4.y; xt[4 * q4 + 2] = t4.z; xt[4 * q4 + 3] = t4.w;
          }
        }
        float zh[RH_UW], zt[RH_UW];
        {
          uint32_t rh[RH_UW], rt[RH_UW];
          sm100::tmem_ld8_nowait(taddr + ul, rh);
          sm100::tmem_ld8_nowait(taddr + RH_UB + ul, rt);
          sm100::tmem_wait_ld();
#pragma unroll
          for (int i = 0; i < RH_UW; ++i) {
            zh[i] = __uint_as_float(rh[i]);
            zt[i] = __uint_as_float(rt[i]);
          }
        }
        for (int c = 1; c < a.nsplit; ++c) {   // chunk partials summed in chunk order (rhn_fwd_pw)
          uint32_t ph[RH_UW], pt[RH_UW];
          sm100::tmem_ld8_nowait(taddr + c * RH_BN + ul, ph);
          sm100::tmem_ld8_nowait(taddr + c * RH_BN + RH_UB + ul, pt);
          sm100::tmem_wait_ld();
#pragma unroll
          for (int i = 0; i < RH_UW; ++i) {
            zh[i] = __fadd_rn(zh[i], __uint_as_float(ph[i]));
            zt[i] = __fadd_rn(zt[i], __uint_as_float(pt[i]));
          }
        }
        if (a.trace && warp == 4 && lane == 0) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + (uc == 0 ? 5 : 11)] = global_ns();
        if (valid) {
        __nv_bfloat16* so = a.Sop + slot_out + (size_t)m * a.Hp + u0 + ul;
        // every shared-memory operand into registers first, results out after: the buffers share
        // one base, so interleaved loads and stores would serialise the 16 units' dependency chains
        float sv[RH_UW], bh[RH_UW], bt[RH_UW];
#pragma unroll
        for (int i = 0; i < RH_UW; ++i) {
          sv[i] = spr[ul + i];
          bh[i] = bl[ul + i];
          bt[i] = bl[RH_UB + ul + i];
        }
        float snew[RH_UW];
#pragma unroll
        for (int i = 0; i < RH_UW; ++i) {
          const int j = u0 + ul + i;
          float s_new = 0.f, aH = 0.f, aT = 0.f;
          if (j < a.H) {
            aH = __fadd_rn(zh[i], bh[i]);
            aT = __fadd_rn(zt[i], bt[i]);
            if (l == 0) {
              aH = __fadd_rn(aH, xh[i]);
              aT = __fadd_rn(aT, xt[i]);
            }
            const float h = tanh_<true>(aH), tau = sigm<true>(aT);
            s_new = __fadd_rn(__fmul_rn(h, tau), __fmul_rn(sv[i], __fsub_rn(1.f, tau)));
          }
          zh[i] = aH;   // pre-activations for BPTT (padding units: 0), stored after the publish
          zt[i] = aT;
          snew[i] = s_new;
        }
#pragma unroll
        for (int i = 0; i < RH_UW; ++i) {
          spr[ul + i] = snew[i];   // s^ℓ: the next micro-step's s^{ℓ−1} of this row and unit
          zr[ul + i] = zh[i];
          zr[RH_UB + ul + i] = zt[i];
        }
        if (last) {
#pragma unroll
          for (int i = 0; i < RH_UW; ++i) {
            const int j = u0 + ul + i;
            if (j >= a.H) break;
            if (a.y) a.y[((size_t)t * a.B + m) * a.ldy + j] = __float2bfloat16_rn(snew[i]);
            if (t == a.T - 1 && a.sT) a.sT[(size_t)m * a.H + j] = snew[i];
          }
        }
        if (a.trace && warp == 4 && lane == 0 && uc == 0) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 9] = global_ns();
        uint4 pk[RH_UW / 8];
        uint32_t* pu = reinterpret_cast<uint32_t*>(pk);
#pragma unroll
        for (int i = 0; i < RH_UW / 2; ++i) {
          __nv_bfloat162 b2 = __floats2bfloat162_rn(snew[2 * i], snew[2 * i + 1]);
          pu[i] = *reinterpret_cast<uint32_t*>(&b2);
        }
#pragma unroll
        for (int i = 0; i < RH_UW / 8; ++i) reinterpret_cast<uint4*>(so)[i] = pk[i];
        if (a.trace && warp == 4 && lane == 0 && uc == 0) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 10] = global_ns();
        }
      }
      sm100::tc_fence_before();
      sm100::mbar_arrive(tempty);
      if (a.trace && warp == 4 && lane == 0) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 6] = global_ns();
      if (q + 1 < nsteps) {   // publish s^ℓ of this tile to the row block: every writer orders its
        fence_proxy_async_global();   // stores before the readers' TMA (async proxy); the CTA barrier
        if (a.trace && warp == 4 && lane == 0) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 7] = global_ns();
        epi_bar();                    // and one release add (cumulative) publish them at gpu scope
        if (a.trace && warp == 4 && lane == 0) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 8] = global_ns();
        if (warp == 2 && lane == 0) {
          red_release_gpu(a.flags + m_blk, 1u);
          if (a.trace) a.trace[((size_t)blockIdx.x * nsteps + q) * 12 + 4] = global_ns();
        }
      }
      // off the critical path: the fp32 state and the pre-activations, read only by the backward
      if (valid) {
        float* sn = a.Sf + slot_out + (size_t)m * a.Hp + u0;
#pragma unroll
        for (int q4 = (RH_UW / 4) * uc; q4 < (RH_UW / 4) * (uc + 1); ++q4) {   // this warp's units
          const int o = 4 * q4;
          reinterpret_cast<float4*>(sn)[q4] = make_float4(spr[o], spr[o + 1], spr[o + 2], spr[o + 3]);
          reinterpret_cast<float4*>(Z + u0)[q4] = make_float4(zr[o], zr[o + 1], zr[o + 2], zr[o + 3]);
          reinterpret_cast<float4*>(Z + a.Hp + u0)[q4] =
              make_float4(zr[RH_UB + o], zr[RH_UB + o + 1], zr[RH_UB + o + 2], zr[RH_UB + o + 3]);
        }
      }
    }
  }
  __syncthreads();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, a.tmem_cols);
  }
}

}  // namespace

bool rhn_rec_fwd_supported(int B, int Hp, int nsplit) {
  return nsplit >= 1 && nsplit <= 4 && Hp % RH_UB == 0 && cdiv(B, TC_BM) * (Hp / RH_UB) <= num_sms();
}

void rhn_rec_fwd_launch(const CUtensorMap& mapA, const CUtensorMap& mapB, RhnFwdArgs a, cudaStream_t st) {
  int dev = 0, maxs = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  ASTRA_CHECK_ARG(rhn_rec_fwd_supported(a.B, a.Hp, a.nsplit), "rhn fused forward: unsupported shape");
  ASTRA_CHECK_ARG(a.a_rows == TC_BM || (a.a_rows == 64 && a.B <= 64), "rhn fused forward: bad A box");
  a.nk = cdiv(a.Hp, TC_BK);
  a.kper = cdiv(a.nk, a.nsplit);
  a.num_m = cdiv(a.B, TC_BM);
  a.num_n = a.Hp / RH_UB;
  a.tmem_cols = a.nsplit <= 1 ? 64 : a.nsplit <= 2 ? 128 : 256;
  const int stage_bytes = a.a_rows * TC_BK * 2 + RH_BN * TC_BK * 2;
  const int extra = a.a_rows * RH_SP * 4 + a.L * RH_BN * 4 + ((a.a_rows * RH_ZP + 1) & ~1) * 4;   // state, biases, staging
  int stages = (maxs - 1024 - 256 - extra) / stage_bytes;
  if (stages > a.nk) stages = a.nk;   // the whole K of a micro-step resident when it fits
  ASTRA_CHECK_ARG(stages >= std::min(2, a.nk), "rhn fused forward: depth too large for shared memory");
  a.stages = stages;
  const int smem = 1024 + stages * stage_bytes + extra + 256;
  CUDA_TRY(cudaFuncSetAttribute(rhn_rec_fwd_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(a.num_m * a.num_n);
  cfg.blockDim = dim3(RH_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  CUDA_TRY(cudaLaunchKernelEx(&cfg, rhn_rec_fwd_kernel, mapA, mapB, a));
  LAUNCH_CHECK();
}

}  // namespace astra
