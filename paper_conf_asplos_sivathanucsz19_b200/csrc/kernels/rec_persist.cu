// K2 small-batch form (SURVEY §8(a) row a3, §8(a.9) `fwd_kernel` "persistent, weight-resident"):
// the whole forward chain of an LSTM-family cell in ONE cooperative launch, for B ≤ 128.
//
// Why: at small batch the per-step recurrent GEMM  UH_t = h_{t−1}·U  ([B, Hp] × [Hp, 4Hp]) is far
// too small to fill the GPU per launch ("individual operations are too small to keep the GPU
// occupied"; P:88 launch costs), and the launched chain pays a GEMM launch, a pointwise launch and
// the fp32 UH round trip per step.  Here every CTA owns SB_UC = 16 hidden units for all T steps:
//   - its slice of U (the 4 gates × 16 units = 64 gate columns, K = Hp) stays in shared memory for
//     as many k-blocks as fit (the rest streams from L2 every step, evict_last);
//   - per step it streams h_{t−1} (A, [B ≤ 128 rows × Hp], bf16) through a TMA ring, runs the
//     tcgen05 MMAs (M = 128, N = 64, one fp32 TMEM accumulator over the whole K), and its 8
//     epilogue warps apply the gate arithmetic straight from TMEM (the fused gate epilogue);
//   - one grid-wide release/acquire counter per step publishes h_t (the next step's A).
// The B tile holds the CTA's 64 gate columns as four 16-row strips (gate g of units u0..u0+15 at
// internal columns gcol(g, u0..u0+15)), loaded by four TMA boxes per k-block.
//
// Numerics (R1, R3, R17): every UH element is one fp32 accumulation from zero over K in ascending
// 64-wide k-blocks of 16-wide MMAs — exactly the launched chain's tc_gemm (tile shapes are bitwise
// interchangeable, tests/test_gpu_gemm.py) — and the epilogue is cell_math.cuh's preact / cell_fwd
// with the same roundings as lstm_fwd_pw_kernel, so this variant is bitwise equal to GEMM + pointwise.
#include <cstdlib>

#include "cell_math.cuh"
#include "gemm.h"
#include "gemm_tc.cuh"
#include "kernels.h"
#include "pdl.cuh"
#include "rec_fused.h"

namespace astra {

constexpr int SB_UC = 16;                  // hidden units per CTA
constexpr int SB_N = 4 * SB_UC;            // gate columns per CTA = MMA N
constexpr int SB_BT = SB_N * TC_BK * 2;    // bytes of one B k-block (64 rows x 128 B)
constexpr int SB_EPI_WARPS = 8;
constexpr int SB_THREADS = 32 * (3 + SB_EPI_WARPS);   // warp 0 A producer, 1 MMA, 2 B producer, 3..10 epilogue
constexpr int SB_PRM = 4 * SB_N;           // b, α, β1, β2 of the 64 gate columns

__device__ __forceinline__ void sb_fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ unsigned sb_ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long sb_gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void sb_epi_bar() {
  asm volatile("bar.sync 1, %0;" ::"n"(32 * SB_EPI_WARPS) : "memory");
}

template <int KIND>
__global__ void __launch_bounds__(SB_THREADS, 1)
    lstm_fwd_persist_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                            const __grid_constant__ CUtensorMap mapBr, const __grid_constant__ CUtensorMap mapB1,
                            const RecPersistArgs a) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int R = a.resident, SA = a.sa, SB = a.sb, nk = a.nk;
  // [A ring][resident B][B ring][params][barriers]: the A ring comes first so the MMA's rows
  // a_rows..127 of its last stage (a_rows = 64: never stored, never read back) stay inside the
  // allocation
  uint8_t* sA = smem;
  uint8_t* sRes = sA + SA * a.ka * a.a_bytes;
  uint8_t* sB = sRes + R * SB_BT;
  float* prm = reinterpret_cast<float*>(sB + SB * a.kbs * SB_BT);
  uint64_t* fullA = reinterpret_cast<uint64_t*>(prm + SB_PRM);
  uint64_t* emptyA = fullA + SA;
  uint64_t* fullB = emptyA + SA;
  uint64_t* emptyB = fullB + SB;
  uint64_t* resbar = emptyB + SB;
  uint64_t* tfull = resbar + 1;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int u0 = blockIdx.x * SB_UC;
  const int col0 = (u0 / GATE_U) * (4 * GATE_U) + (u0 % GATE_U);   // gcol(0, u0); gate g at + g·GATE_U
  const unsigned nct = gridDim.x;

  if (threadIdx.x == 0) {
    for (int s = 0; s < SA; ++s) {
      sm100::mbar_init(&fullA[s], 1);
      sm100::mbar_init(&emptyA[s], 1);
    }
    for (int s = 0; s < SB; ++s) {
      sm100::mbar_init(&fullB[s], 1);
      sm100::mbar_init(&emptyB[s], 1);
    }
    sm100::mbar_init(resbar, 1);
    for (int q = 0; q < 2; ++q) {
      sm100::mbar_init(&tfull[q], 1);
      sm100::mbar_init(&tempty[q], 32 * SB_EPI_WARPS);
    }
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
    sm100::tma_prefetch(&mapBr);
    sm100::tma_prefetch(&mapB1);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, 128);
  for (int c = threadIdx.x; c < SB_N; c += SB_THREADS) {   // this CTA's gate-column parameters
    const int g = c / SB_UC, unit = u0 + c % SB_UC, e = g * a.H + unit;
    const bool ok = unit < a.H;
    prm[c] = ok ? a.gp.b[e] : 0.f;
    prm[SB_N + c] = (ok && KIND == K_MILSTM) ? a.gp.alpha[e] : 0.f;
    prm[2 * SB_N + c] = (ok && KIND == K_MILSTM) ? a.gp.beta1[e] : 0.f;
    prm[3 * SB_N + c] = (ok && KIND == K_MILSTM) ? a.gp.beta2[e] : 0.f;
  }
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ A producer: h_{t−1}, KA k-blocks per box
    // One 4-D TMA box {64, a_rows, KA, 1} lands KA consecutive k-block tiles (the k-block dimension
    // has a 128-byte stride in the map): the per-box issue cost, not bandwidth, bounds small boxes.
    {   // whole warp: the *_warp TMA forms elect the issuing lane
      pdl_wait();
      int s = 0;
      uint32_t ph = 0;
      const uint32_t stage_bytes = (uint32_t)(a.ka * a.a_bytes);
      for (int t = a.t0; t < a.t1; ++t) {
        if (t > a.t0) {   // every CTA has published h_{t−1}
          while (sb_ld_acquire(a.flags) < nct * (unsigned)(t - a.t0)) __nanosleep(32);
          sb_fence_proxy_async_global();
        }
        if (a.trace) a.trace[((size_t)blockIdx.x * (a.t1 - a.t0) + (t - a.t0)) * 6 + 0] = sb_gtime();
        for (int kb = 0; kb < nk; kb += a.ka) {
          sm100::mbar_wait(&emptyA[s], ph ^ 1);
          sm100::mbar_arrive_expect_tx_warp(&fullA[s], stage_bytes);
          sm100::tma_load_4d_warp(sA + s * stage_bytes, &mapA, &fullA[s], 0, 0, kb, t);
          if (a.trace && blockIdx.x == 0 && t == a.t0 + (a.t1 - a.t0) / 2)
            a.trace[(size_t)gridDim.x * (a.t1 - a.t0) * 6 + kb / a.ka] = clock64();
          if (++s == SA) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 2) {
    // ------------------------------------------------------------ B producer: the U slice
    // The U mirror is written by the forward's first kernels, complete before this launch starts
    // (stream order); it does not change during the chain, so the resident part is loaded once and
    // the streamed part runs ahead of the recurrence (its ring is paced by the MMAs only).  A 4-D box
    // {64, 16 units, 4 gates, k-blocks} lands the B tiles of several k-blocks in MMA order
    // ([k-block][gate strip][16 rows][64]).
    {   // whole warp: the *_warp TMA / arrive forms elect the issuing lane
      const uint64_t pol = sm100::l2_policy_evict_last();
      if (!a.b_old) pdl_wait();
      if (R > 0) {
        sm100::mbar_arrive_expect_tx_warp(resbar, (uint32_t)(R * SB_BT));
        for (int kb = 0; kb < R; kb += 8) {
          const int n = R - kb < 8 ? R - kb : 8;   // resmap box: 8 k-blocks (the last may be clipped below)
          if (n == 8)
            sm100::tma_load_4d_hint_warp(sRes + kb * SB_BT, &mapBr, resbar, 0, col0, 0, kb, pol);
          else
            for (int j = 0; j < n; ++j)
              sm100::tma_load_4d_hint_warp(sRes + (kb + j) * SB_BT, &mapB1, resbar, 0, col0, 0, kb + j, pol);
        }
      } else {
        sm100::mbar_arrive_warp(resbar);
      }
      if (R < nk) {
        int s = 0;
        uint32_t ph = 0;
        const uint32_t stage_bytes = (uint32_t)(a.kbs * SB_BT);
        for (int t = a.t0; t < a.t1; ++t)
          for (int kb = R; kb < nk; kb += a.kbs) {
            sm100::mbar_wait(&emptyB[s], ph ^ 1);
            sm100::mbar_arrive_expect_tx_warp(&fullB[s], stage_bytes);
            sm100::tma_load_4d_hint_warp(sB + s * stage_bytes, &mapB, &fullB[s], 0, col0, 0, kb, pol);
            if (a.trace && blockIdx.x == 0 && t == a.t0 + (a.t1 - a.t0) / 2)
              a.trace[(size_t)gridDim.x * (a.t1 - a.t0) * 6 + 32 + (kb - R) / a.kbs] = clock64();
            if (++s == SB) { s = 0; ph ^= 1; }
          }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    // A single thread issues every MMA: at N = 64 an MMA takes ~35 ns, so the loop's own scalar
    // work (divisions, descriptor rebuilds, constant loads) must stay well below that — shared-
    // memory descriptors are advanced by adding (bytes >> 4) to their address field (addresses
    // < 256 KB never carry out of the 14-bit field), stage bookkeeping is counter-based.
    {   // the whole warp runs the loop (warp-uniform operands); one elected lane issues (umma_*_warp)
      sm100::mbar_wait(resbar, 0);
      sm100::tc_fence_after();
      const uint32_t idesc = a.idesc;
      const uint64_t dA0 = sm100::smem_desc_sw128(sm100::smem_u32(sA), 16, 1024);
      const uint64_t dR0 = sm100::smem_desc_sw128(sm100::smem_u32(sRes), 16, 1024);
      const uint64_t dB0 = sm100::smem_desc_sw128(sm100::smem_u32(sB), 16, 1024);
      const uint32_t a_kb = (uint32_t)a.a_bytes >> 4, b_kb = SB_BT >> 4;
      const uint32_t a_st = (uint32_t)(a.ka * a.a_bytes) >> 4, b_st = (uint32_t)(a.kbs * SB_BT) >> 4;
      const int ka = a.ka, kbs = a.kbs;
      int sa = 0, sb = 0;
      uint32_t pa = 0, pb = 0;
      int local = 0;
      for (int t = a.t0; t < a.t1; ++t, ++local) {
        const int acc = local & 1;
        sm100::mbar_wait(&tempty[acc], (uint32_t)((local >> 1) & 1) ^ 1);
        sm100::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * SB_N;
        int ja = ka, jb = kbs;   // k-blocks left in the current A / B stage
        uint64_t adesc = 0, bdesc = 0;
        for (int kb = 0; kb < nk; ++kb) {
          bool waited = false;
          if (ja == ka) {
            sm100::mbar_wait(&fullA[sa], pa);
            waited = true;
            adesc = dA0 + (uint64_t)(sa * a_st);
            ja = 0;
          }
          uint64_t bd;
          if (kb < R) {
            bd = dR0 + (uint64_t)(kb * b_kb);
          } else {
            if (jb == kbs) {
              sm100::mbar_wait(&fullB[sb], pb);
              waited = true;
              bdesc = dB0 + (uint64_t)(sb * b_st);
              jb = 0;
            }
            bd = bdesc;
          }
          if (waited) sm100::tc_fence_after();   // only after a new barrier wait
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk)
            sm100::umma_bf16_warp(d_tmem, adesc + 2 * kk, bd + 2 * kk, idesc, (kb | kk) != 0);
          adesc += a_kb;
          if (++ja == ka) {
            sm100::umma_commit_warp(&emptyA[sa]);
            if (++sa == SA) { sa = 0; pa ^= 1; }
          }
          if (kb >= R) {
            bdesc += b_kb;
            if (++jb == kbs) {
              sm100::umma_commit_warp(&emptyB[sb]);
              if (++sb == SB) { sb = 0; pb ^= 1; }
            }
          }
        }
        sm100::umma_commit_warp(&tfull[acc]);
        if (a.trace && lane == 0) a.trace[((size_t)blockIdx.x * (a.t1 - a.t0) + (t - a.t0)) * 6 + 2] = sb_gtime();
      }
    }
  } else {
    // ------------------------------------------------------------ fused gate epilogue (8 warps)
    const int ew = warp - 3;
    const int quarter = warp & 3;             // TMEM lane quarter this warp may access
    const int half = ew >> 2;                 // units [8·half, 8·half + 8) of the CTA's 16
    const int row = quarter * 32 + lane;
    const bool valid = row < a.B;
    const int ul0 = half * 8;
    const int unit0 = u0 + ul0;
    const int cb = col0 + ul0;                // internal column of gate 0, first unit of this thread
    const long NG = a.NG;
    pdl_wait();
    // c_{t−1} of this thread's (row, 8 units) is the c_t it computed one step earlier: kept in
    // registers across steps (loaded from C only at the first step)
    float cp[8];
    if (valid) {
      const float4* cpp = reinterpret_cast<const float4*>(a.C + ((long)a.t0 * a.B + row) * a.Hp + unit0);
      const float4 c0v = cpp[0], c1v = cpp[1];
      cp[0] = c0v.x; cp[1] = c0v.y; cp[2] = c0v.z; cp[3] = c0v.w;
      cp[4] = c1v.x; cp[5] = c1v.y; cp[6] = c1v.z; cp[7] = c1v.w;
    }
    int local = 0;
    for (int t = a.t0; t < a.t1; ++t, ++local) {
      const int acc = local & 1;
      // WX_t (the hoisted projection, written before this launch) does not depend on the recurrence:
      // its loads are in flight while this step's MMAs run
      float wx[4][8];
      if (valid) {
        const long r = (long)t * a.B + row;
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          const float4* wp = reinterpret_cast<const float4*>(a.WX + r * NG + cb + g * GATE_U);
          const float4 w0 = __ldcs(wp), w1 = __ldcs(wp + 1);
          wx[g][0] = w0.x; wx[g][1] = w0.y; wx[g][2] = w0.z; wx[g][3] = w0.w;
          wx[g][4] = w1.x; wx[g][5] = w1.y; wx[g][6] = w1.z; wx[g][7] = w1.w;
        }
      }
      sm100::mbar_wait(&tfull[acc], (uint32_t)((local >> 1) & 1));
      sm100::tc_fence_after();
      unsigned long long* tr = (a.trace && ew == 1 && lane == 0)
                                   ? a.trace + ((size_t)blockIdx.x * (a.t1 - a.t0) + (t - a.t0)) * 6 : nullptr;
      if (tr) tr[3] = sb_gtime();
      const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * SB_N + ul0;
      uint32_t zr[4][8];
#pragma unroll
      for (int g = 0; g < 4; ++g) sm100::tmem_ld8_nowait(taddr + g * SB_UC, zr[g]);
      sm100::tmem_wait_ld();
      sm100::tc_fence_before();
      sm100::mbar_arrive(&tempty[acc]);       // the accumulator is in registers: free it
      float zs[4][8];      // UH_t of this thread (saved for BPTT unless the recompute context)
      float hv_keep[8];
      uint4 hpk;
      if (valid) {
        const long r = (long)t * a.B + row;   // row of step t in the [T·B] buffers
        float (&z)[4][8] = zs;
#pragma unroll
        for (int g = 0; g < 4; ++g)
#pragma unroll
          for (int i = 0; i < 8; ++i) z[g][i] = __uint_as_float(zr[g][i]);
        float cv[8], hv[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          float pa[4];
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            const int c = g * SB_UC + ul0 + i;
            pa[g] = preact<KIND, true>(wx[g][i], z[g][i], prm[c], prm[SB_N + c], prm[2 * SB_N + c], prm[3 * SB_N + c]);
          }
          cell_fwd<KIND, true>(pa, cp[i], cv[i], hv[i]);
          if (unit0 + i >= a.H) { cv[i] = 0.f; hv[i] = 0.f; }   // padding units stay exactly zero
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) cp[i] = cv[i];
        uint4 hp;
        uint32_t* hw = reinterpret_cast<uint32_t*>(&hp);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          __nv_bfloat162 b2 = __floats2bfloat162_rn(hv[2 * i], hv[2 * i + 1]);
          hw[i] = *reinterpret_cast<uint32_t*>(&b2);
        }
        *reinterpret_cast<uint4*>(a.Hb + (r + a.B) * a.ldh + unit0) = hp;
        hpk = hp;
#pragma unroll
        for (int i = 0; i < 8; ++i) hv_keep[i] = hv[i];
      }
      if (tr) tr[4] = sb_gtime();
      if (t + 1 < a.t1) {   // publish h_t (generic-proxy stores → the other CTAs' TMA reads)
        sb_fence_proxy_async_global();
        __threadfence();
        sb_epi_bar();
        if (ew == 0 && lane == 0) {
          atomicAdd(a.flags, 1u);
          if (a.trace) a.trace[((size_t)blockIdx.x * (a.t1 - a.t0) + (t - a.t0)) * 6 + 5] = sb_gtime();
        }
      }
      // the stores no other CTA reads this step (saved UH, c_t, y, final state) go out after the
      // publish, off the chain's critical path
      if (valid) {
        const long r = (long)t * a.B + row;
        const uint4 hp = hpk;
        const float* hv = hv_keep;
        const float* cv = cp;
        if (a.UH) {
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            float4* up = reinterpret_cast<float4*>(a.UH + r * NG + cb + g * GATE_U);
            up[0] = make_float4(zs[g][0], zs[g][1], zs[g][2], zs[g][3]);
            up[1] = make_float4(zs[g][4], zs[g][5], zs[g][6], zs[g][7]);
          }
        }
        float4* cn = reinterpret_cast<float4*>(a.C + (r + a.B) * a.Hp + unit0);
        cn[0] = make_float4(cv[0], cv[1], cv[2], cv[3]);
        cn[1] = make_float4(cv[4], cv[5], cv[6], cv[7]);
        if (a.y_kind == 1) {          // bf16 [T·B][ldy] (external y, ldy = H)
          __nv_bfloat16* yp = reinterpret_cast<__nv_bfloat16*>(a.y) + r * a.ldy + unit0;
          if ((a.ldy & 7) == 0 && unit0 + 8 <= a.H) {
            *reinterpret_cast<uint4*>(yp) = hp;
          } else {
#pragma unroll
            for (int i = 0; i < 8; ++i)
              if (unit0 + i < a.H) yp[i] = __float2bfloat16_rn(hv[i]);
          }
        } else if (a.y_kind == 2) {   // fp32 [T·B][ldy] (internal, ldy ≥ Hp: padding columns too)
          float* yp = reinterpret_cast<float*>(a.y) + r * a.ldy + unit0;
#pragma unroll
          for (int i = 0; i < 8; ++i)
            if (unit0 + i < a.H || a.ldy >= a.Hp) yp[i] = hv[i];
        }
        if (t == a.T - 1) {
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            if (unit0 + i >= a.H) break;
            if (a.hT) a.hT[(long)row * a.H + unit0 + i] = hv[i];
            if (a.cT) a.cT[(long)row * a.H + unit0 + i] = cv[i];
          }
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

bool lstm_fwd_persist_supported(int B, int Hp) {
  return B >= 1 && B <= 128 && Hp % SB_UC == 0 && Hp / SB_UC <= num_sms();
}

static int sb_smem_bytes(const RecPersistArgs& a) {
  const int bars = (2 * a.sa + 2 * a.sb + 1 + 4) * 8 + 16;
  return 1024 + a.sa * a.ka * a.a_bytes + a.resident * SB_BT + a.sb * a.kbs * SB_BT + SB_PRM * 4 + bars;
}

void lstm_fwd_persist_launch(int kind, const void* Hb, const void* Um, int Tmax, RecPersistArgs a, cudaStream_t st) {
  ASTRA_CHECK_ARG(lstm_fwd_persist_supported(a.B, a.Hp), "persistent small-batch forward: B <= 128 and Hp/16 <= #SMs");
  int dev = 0, maxs = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  auto knob = [](const char* n, int d) { const char* e = std::getenv(n); return e ? std::atoi(e) : d; };
  static const int k_ka = knob("ASTRA_SB_KA", 4), k_sa = knob("ASTRA_SB_SA", 3), k_kb = knob("ASTRA_SB_KB", 2),
                   k_sb = knob("ASTRA_SB_SB", 2), k_res = knob("ASTRA_SB_RES", -1);
  const long K = a.K ? a.K : a.Hp;   // U-mirror rows and h rows have stride K
  ASTRA_CHECK_ARG(K % TC_BK == 0, "persistent small-batch forward: K must be a multiple of 64");
  a.ldh = K;
  a.nk = (int)(K / TC_BK);
  a.a_rows = a.B <= 64 ? 64 : 128;
  a.a_bytes = a.a_rows * TC_BK * 2;
  a.ka = 1;
  for (int c = k_ka; c > 1; --c)
    if (a.nk % c == 0) { a.ka = c; break; }
  a.sa = std::max(2, k_sa);
  a.kbs = std::max(1, k_kb);
  a.sb = 0;
  a.resident = a.nk;
  // the rest of shared memory holds resident U k-blocks; the streamed ones go through the B ring in
  // stages of kbs k-blocks (the streamed count is a multiple of kbs)
  const int res_cap = a.max_resident >= 0 ? (k_res >= 0 ? std::min(k_res, a.max_resident) : a.max_resident) : k_res;
  while (sb_smem_bytes(a) > maxs || (res_cap >= 0 && a.resident > res_cap) || (a.nk - a.resident) % a.kbs != 0) {
    a.sb = std::max(1, k_sb);
    --a.resident;
    ASTRA_CHECK_ARG(a.resident >= 0, "persistent small-batch forward: shared memory too small");
  }
  if (a.max_resident == 0)   // streaming the whole slice: as deep a B ring as fits (≤ 8 stages)
    while (a.sb < 8) {
      ++a.sb;
      if (sb_smem_bytes(a) > maxs) { --a.sb; break; }
    }
  // instruction descriptor: D f32, A/B bf16 K-major, N = 64, M = 128
  a.idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(SB_N >> 3) << 17) | ((uint32_t)(TC_BM >> 4) << 24);
  // maps.  A: h as {64 k, rows B, k-block (stride 128 B), t}; B: U mirror rows as {64 k, unit row,
  // gate (stride GATE_U rows), k-block (stride 128 B)}
  CUtensorMap mA, mB, mBr, mB1;
  {
    const long dims[4] = {64, a.B, a.nk, Tmax + 1};
    const long str[3] = {K * 2, 128, (long)a.B * K * 2};
    const int box[4] = {64, a.a_rows, a.ka, 1};
    make_map_nd(&mA, Hb, 4, dims, str, box, 128);
  }
  {
    const long dims[4] = {64, a.NG, 4, a.nk};
    const long str[3] = {K * 2, (long)GATE_U * K * 2, 128};
    const int box[4] = {64, SB_UC, 4, a.kbs};
    make_map_nd(&mB, Um, 4, dims, str, box, 128);
    const int boxr[4] = {64, SB_UC, 4, 8};
    make_map_nd(&mBr, Um, 4, dims, str, boxr, 128);
    const int box1[4] = {64, SB_UC, 4, 1};
    make_map_nd(&mB1, Um, 4, dims, str, box1, 128);
  }
  const int smem = sb_smem_bytes(a);
  void (*fn)(CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap, RecPersistArgs) = nullptr;
  switch (kind) {
    case K_LSTM: fn = lstm_fwd_persist_kernel<K_LSTM>; break;
    case K_MILSTM: fn = lstm_fwd_persist_kernel<K_MILSTM>; break;
    default: fn = lstm_fwd_persist_kernel<K_SUBLSTM>; break;
  }
  CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(a.Hp / SB_UC);
  cfg.blockDim = dim3(SB_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  if (a.t1 - a.t0 > 1) {
    attr[0].id = cudaLaunchAttributeCooperative;   // every CTA resident: the per-step counter is a grid barrier
    attr[0].val.cooperative = 1;
  } else {   // one step (no grid barrier): a PDL launch whose prologue overlaps the predecessor —
             // h_{t−1} and U are read after pdl_wait, c_{t−1} / WX_t are ≥ 2 launches old
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  }
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  CUDA_TRY(cudaLaunchKernelEx(&cfg, fn, mA, mB, mBr, mB1, a));
  LAUNCH_CHECK();
}

}  // namespace astra
