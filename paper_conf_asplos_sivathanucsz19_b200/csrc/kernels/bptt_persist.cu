// K4 small-batch form (SURVEY §8(a) row a5, §8(a.9) `bwd_kernel` "persistent"): the whole BPTT
// chain of an LSTM-family cell in ONE cooperative launch of clusters, for B ≤ 128 and the canonical
// 4-chunk split of K = 4Hp (reading R25, H ≥ 2048).
//
// Why: at small batch the per-step BPTT GEMM  dh_rec = D_uh,{t+1}·Uᵀ  ([B, 4Hp] × [4Hp, Hp]) fills
// a few dozen SMs per launch and its fp32 split-K partials make a round trip through L2 to the
// pointwise kernel.  Here a cluster of 4 CTAs owns 64 hidden units for all steps:
//   - CTA c of the cluster computes split-K chunk c of the 64 units' dh_rec (K range = chunk c's
//     kper k-blocks: tcgen05 MMAs M = 128, N = 64, A = D_uh rows streamed by TMA, B = its Uᵀ slice,
//     resident in shared memory as far as it fits, the rest streamed from L2);
//   - the four fp32 partials meet in shared memory: CTA c reads the partials of ITS 16 units from
//     all four CTAs over distributed shared memory and adds them in chunk order 0, 1, 2, 3 — the
//     launched pointwise kernel's sum_split order — then runs the cell backward of those units
//     (lstm_bwd_da, the same function as lstm_bwd_pw_kernel / lstm_bwd_pw2_kernel);
//   - D_uh,t of the 16 units goes to global memory and one release/acquire counter per K chunk
//     (the kper CTAs whose units form that chunk) publishes it to the CTAs that read the chunk.
// The bias / α / β column sums follow R5 exactly: thread (unit, row lane y, 32-row chunk) walks rows
// y, y+4, … of its chunk in ascending order and accumulates lstm_bwd_acc per gate, the four lanes
// are combined in y order and folded into the chunk's partial step after step (T−1 down to 0).
// So the kernel is bitwise equal to the launched chain (BPTT GEMM with ksplit 4 + pointwise kernel).
#include <cstdio>
#include <cstdlib>
#include <map>
#include <tuple>

#include "cell_math.cuh"
#include "gemm.h"
#include "gemm_tc.cuh"
#include "kernels.h"
#include "lstm_bwd_row.cuh"
#include "pdl.cuh"
#include "rec_fused.h"

namespace astra {

constexpr int PB_CL = 4;                    // cluster size = the canonical split-K chunks
constexpr int PB_UG = 64;                   // units per cluster (the MMA's N)
constexpr int PB_UC = PB_UG / PB_CL;        // units finalised per CTA
constexpr int PB_BT = PB_UG * TC_BK * 2;    // bytes of one B k-block (64 k rows x 64 units)
constexpr int PB_EPI_WARPS = 8;
constexpr int PB_THREADS = 32 * (3 + PB_EPI_WARPS);   // warp 0 A producer, 1 MMA, 2 B producer, 3..10 epilogue
constexpr int PB_XS = 68;                   // fp32 row stride of the partial exchange buffer
constexpr int PB_RPT = BWD_RB / BWD_RY;     // rows per finalising thread (8: rows y, y+4, …, y+28)

__device__ __forceinline__ void pb_fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ unsigned pb_ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned long long pb_gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void pb_epi_bar() { asm volatile("bar.sync 1, %0;" ::"n"(32 * PB_EPI_WARPS) : "memory"); }
__device__ __forceinline__ bool pb_try_cluster(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, P1;\n\t}"
      : "=r"(ok) : "r"(sm100::smem_u32(bar)), "r"(parity) : "memory");
  return ok != 0;
}
__device__ __forceinline__ float pb_ld_cluster(uint32_t a) {
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(a) : "memory");
  return v;
}

__device__ __forceinline__ bool pb_try(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, P1;\n\t}"
      : "=r"(ok) : "r"(sm100::smem_u32(bar)), "r"(parity) : "memory");
  return ok != 0;
}
// Diagnostics (ASTRA_PB_SPIN > 0): every wait gives up after that many probes and prints where it
// was stuck, so a protocol error ends the kernel instead of hanging it.
#define PB_WAIT(probe, tag, step_)                                                                          \
  do {                                                                                                 \
    unsigned long long n_ = 0;                                                                         \
    while (!(probe)) {                                                                                 \
      if (a.spin && ++n_ > a.spin) {                                                                   \
        printf("pb stuck: %s cta %d thr %d step %d\n", tag, (int)blockIdx.x, (int)threadIdx.x, (int)(step_)); \
        break;                                                                                         \
      }                                                                                                \
    }                                                                                                  \
  } while (0)

template <int KIND, typename TDY>
__global__ void __launch_bounds__(PB_THREADS, 1)
    lstm_bptt_persist_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                             const __grid_constant__ CUtensorMap mapBr, const __grid_constant__ CUtensorMap mapB1,
                             const BpttPersistArgs a) {
  constexpr int NV = BwdNV<KIND>::value;
  constexpr bool F = true;   // bf16 path (reading R27)
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int R = a.resident, SA = a.sa, SB = a.sb, kper = a.kper;
  const int nch = (a.B + BWD_RB - 1) / BWD_RB;
  uint8_t* sA = smem;
  uint8_t* sRes = sA + SA * a.ka * a.a_bytes;
  uint8_t* sB = sRes + R * PB_BT;
  float* xbuf = reinterpret_cast<float*>(sB + SB * a.kbs * PB_BT);   // [2][a_rows][PB_XS]
  float* red = xbuf + 2 * a.a_rows * PB_XS;                           // [nch][BWD_RY][NV][PB_UC]
  float* cpart = red + nch * BWD_RY * NV * PB_UC;                     // [nch][NV][PB_UC]
  float* prm = cpart + nch * NV * PB_UC;                              // [4 (b, α, β1, β2)][4 gates][PB_UC]
  uint64_t* fullA = reinterpret_cast<uint64_t*>(prm + 16 * PB_UC);
  uint64_t* emptyA = fullA + SA;
  uint64_t* fullB = emptyA + SA;
  uint64_t* emptyB = fullB + SB;
  uint64_t* resbar = emptyB + SB;
  uint64_t* tfull = resbar + 1;
  uint64_t* tempty = tfull + 2;
  uint64_t* xready = tempty + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(xready + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int crank = (int)sm100::cluster_ctarank();      // = the split-K chunk this CTA computes
  const int grp = blockIdx.x / PB_CL;                    // unit group: units [64·grp, 64·grp + 64)
  const int kb0 = crank * kper;                          // first k-block of the chunk
  const int out_chunk = (grp * PB_UG * 4 / TC_BK) / kper;   // chunk whose A rows this group's units form
  const int T = a.T;
  const int nmm = T - 1;                                 // steps with a GEMM: t = T−2 … 0

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
      sm100::mbar_init(&tempty[q], 32 * PB_EPI_WARPS);
      sm100::mbar_init(&xready[q], PB_CL);
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
  const int ju0 = grp * PB_UG + crank * PB_UC;   // first unit this CTA finalises
  for (int i = threadIdx.x; i < 16 * PB_UC; i += PB_THREADS) {
    const int pi = i / (4 * PB_UC), g = (i / PB_UC) % 4, u = i % PB_UC, j = ju0 + u;
    const float* src = pi == 0 ? a.gp.b : pi == 1 ? a.gp.alpha : pi == 2 ? a.gp.beta1 : a.gp.beta2;
    prm[i] = (j < a.H && (pi == 0 || KIND == K_MILSTM)) ? src[g * a.H + j] : 0.f;
  }
  sm100::tc_fence_before();
  __syncthreads();
  sm100::cluster_sync();   // every CTA's barriers are initialised before any remote arrive
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ A producer: D_uh,{t+1} chunk rows
    {   // whole warp: the *_warp TMA / arrive forms elect the issuing lane
      pdl_wait();
      int s = 0;
      uint32_t ph = 0;
      const uint32_t stage_bytes = (uint32_t)(a.ka * a.a_bytes);
      for (int i = 0; i < nmm; ++i) {
        const int t = T - 2 - i;
        // the kper CTAs whose units make up this chunk have published D_uh,{t+1}
        PB_WAIT(pb_ld_acquire(a.flags + crank) >= (unsigned)(kper * (i + 1)), "flags", i);
        pb_fence_proxy_async_global();
        if (a.trace) a.trace[((size_t)blockIdx.x * T + t) * 8 + 0] = pb_gtime();
        for (int kb = 0; kb < kper; kb += a.ka) {
          PB_WAIT(pb_try(&emptyA[s], ph ^ 1), "emptyA", i);
          sm100::mbar_arrive_expect_tx_warp(&fullA[s], stage_bytes);
          sm100::tma_load_4d_warp(sA + s * stage_bytes, &mapA, &fullA[s], 0, 0, kb0 + kb, t + 1);
          if (++s == SA) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 2) {
    // ------------------------------------------------------------ B producer: the Uᵀ slice of the chunk
    // (the U mirror does not change during the chain: resident part once, streamed part paced by
    // the MMAs only)
    {   // whole warp: the *_warp TMA / arrive forms elect the issuing lane
      const uint64_t pol = sm100::l2_policy_evict_last();
      pdl_wait();
      const int n0 = grp * PB_UG;
      if (R > 0) {
        sm100::mbar_arrive_expect_tx_warp(resbar, (uint32_t)(R * PB_BT));
        for (int kb = 0; kb < R; kb += 8) {
          const int n = R - kb < 8 ? R - kb : 8;
          if (n == 8)
            sm100::tma_load_3d_hint_warp(sRes + kb * PB_BT, &mapBr, resbar, n0, 0, kb0 + kb, pol);
          else
            for (int j = 0; j < n; ++j)
              sm100::tma_load_3d_hint_warp(sRes + (kb + j) * PB_BT, &mapB1, resbar, n0, 0, kb0 + kb + j, pol);
        }
      } else {
        sm100::mbar_arrive_warp(resbar);
      }
      if (R < kper && nmm > 0) {
        int s = 0;
        uint32_t ph = 0;
        const uint32_t stage_bytes = (uint32_t)(a.kbs * PB_BT);
        for (int i = 0; i < nmm; ++i)
          for (int kb = R; kb < kper; kb += a.kbs) {
            PB_WAIT(pb_try(&emptyB[s], ph ^ 1), "emptyB", i);
            sm100::mbar_arrive_expect_tx_warp(&fullB[s], stage_bytes);
            sm100::tma_load_3d_hint_warp(sB + s * stage_bytes, &mapB, &fullB[s], n0, 0, kb0 + kb, pol);
            if (++s == SB) { s = 0; ph ^= 1; }
          }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer (lean loop, rec_persist.cu)
    {   // whole warp: umma_*_warp elect the issuing lane
      PB_WAIT(pb_try(resbar, 0), "resbar", 0);
      sm100::tc_fence_after();
      const uint32_t idesc = a.idesc;
      const uint64_t dA0 = sm100::smem_desc_sw128(sm100::smem_u32(sA), 16, 1024);
      const uint64_t dR0 = sm100::smem_desc_sw128(sm100::smem_u32(sRes), 8192, 1024);
      const uint64_t dB0 = sm100::smem_desc_sw128(sm100::smem_u32(sB), 8192, 1024);
      const uint32_t a_kb = (uint32_t)a.a_bytes >> 4, b_kb = PB_BT >> 4;
      const uint32_t a_st = (uint32_t)(a.ka * a.a_bytes) >> 4, b_st = (uint32_t)(a.kbs * PB_BT) >> 4;
      const int ka = a.ka, kbs = a.kbs;
      int sa = 0, sb = 0;
      uint32_t pa = 0, pb = 0;
      for (int i = 0; i < nmm; ++i) {
        const int acc = i & 1;
        PB_WAIT(pb_try(&tempty[acc], (uint32_t)((i >> 1) & 1) ^ 1), "tempty", i);
        sm100::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * PB_UG;
        int ja = ka, jb = kbs;
        uint64_t adesc = 0, bdesc = 0;
        for (int kb = 0; kb < kper; ++kb) {
          bool waited = false;
          if (ja == ka) {
            PB_WAIT(pb_try(&fullA[sa], pa), "fullA", i);
            if (a.trace && kb == 0) a.trace[((size_t)blockIdx.x * T + (T - 2 - i)) * 8 + 1] = pb_gtime();
            waited = true;
            adesc = dA0 + (uint64_t)(sa * a_st);
            ja = 0;
          }
          uint64_t bd;
          if (kb < R) {
            bd = dR0 + (uint64_t)(kb * b_kb);
          } else {
            if (jb == kbs) {
              PB_WAIT(pb_try(&fullB[sb], pb), "fullB", i);
              waited = true;
              bdesc = dB0 + (uint64_t)(sb * b_st);
              jb = 0;
            }
            bd = bdesc;
          }
          if (waited) sm100::tc_fence_after();
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk)   // A K-major: +32 B per K step; B MN-major: +2048 B
            sm100::umma_bf16_warp(d_tmem, adesc + 2 * kk, bd + 128 * kk, idesc, (kb | kk) != 0);
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
        if (a.trace) a.trace[((size_t)blockIdx.x * T + (T - 2 - i)) * 8 + 2] = pb_gtime();
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue + cell backward (8 warps)
    const int ew = warp - 3, et = threadIdx.x - 96;
    const int quarter = warp & 3, half = ew >> 2;   // TMEM lane quarter; columns [32·half, +32)
    // finalising thread: unit u of the CTA's 16, row lane y, 32-row chunk ch (rows ch·32 + y + 4i)
    const int u = et % PB_UC, y = (et / PB_UC) % BWD_RY, ch = et / (PB_UC * BWD_RY);
    const bool fin = ch < nch;
    const int j = ju0 + u;
    const bool unit_ok = j < a.H;
    const int jc = gcol(0, j);                        // internal column of gate 0 of unit j
    const long NG = a.NG;
    const uint32_t xb0 = sm100::smem_u32(xbuf);
    uint32_t xpeer[PB_CL];
#pragma unroll
    for (int k = 0; k < PB_CL; ++k) xpeer[k] = sm100::mapa_shared(xb0, (uint32_t)k);
    pdl_wait();
    float dcv[PB_RPT];
#pragma unroll
    for (int i = 0; i < PB_RPT; ++i) {
      const int r = ch * BWD_RB + y + BWD_RY * i;
      dcv[i] = (fin && r < a.B) ? a.dc[(long)r * a.Hp + j] : 0.f;
    }
    for (int t = T - 1; t >= 0; --t) {
      const int i = T - 2 - t;                // GEMM step index (t < T−1)
      const int xs = i & 1;
      // saved operands of step t (independent of the chain): in flight while the MMAs run
      float w[PB_RPT][4], h[PB_RPT][4], cp[PB_RPT], cn[PB_RPT], dyv[PB_RPT];
#pragma unroll
      for (int q = 0; q < PB_RPT; ++q) {
        const int r = ch * BWD_RB + y + BWD_RY * q;
        const bool ok = fin && r < a.B && unit_ok;
        const long rr = (long)t * a.B + r;
#pragma unroll
        for (int g = 0; g < 4; ++g) {
          w[q][g] = ok ? __ldcs(a.WX + rr * NG + jc + g * GATE_U) : 0.f;
          h[q][g] = ok ? __ldcs(a.UH + rr * NG + jc + g * GATE_U) : 0.f;
        }
        cn[q] = ok ? __ldcs(a.C + (rr + a.B) * a.Hp + j) : 0.f;
        cp[q] = ok ? __ldcs(a.C + rr * a.Hp + j) : 0.f;
        dyv[q] = ok ? to_f<TDY>(reinterpret_cast<const TDY*>(a.dy)[rr * a.ldy + j]) : 0.f;
      }
      float s[PB_RPT];
      bool have_s = false;
      if (t < T - 1) {
        // this CTA's chunk partial of the 64 units: TMEM → exchange buffer
        const int acc = i & 1;
        PB_WAIT(pb_try(&tfull[acc], (uint32_t)((i >> 1) & 1)), "tfull", i);
        sm100::tc_fence_after();
        if (a.trace && et == 0) a.trace[((size_t)blockIdx.x * T + t) * 8 + 3] = pb_gtime();
        if (quarter * 32 < a.B) {
          float v[32];
          sm100::tmem_ld32(tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * PB_UG + half * 32, v);
          const int row = quarter * 32 + lane;
          if (row < a.B) {
            float* xp = xbuf + ((size_t)xs * a.a_rows + row) * PB_XS + half * 32;
#pragma unroll
            for (int c = 0; c < 32; c += 4) *reinterpret_cast<float4*>(xp + c) = make_float4(v[c], v[c + 1], v[c + 2], v[c + 3]);
          }
        }
        sm100::tc_fence_before();
        sm100::mbar_arrive(&tempty[acc]);
        pb_epi_bar();   // the CTA's partial is complete
        if (et == 0) {
          if (a.trace) a.trace[((size_t)blockIdx.x * T + t) * 8 + 4] = pb_gtime();
#pragma unroll
          for (int k = 0; k < PB_CL; ++k)
            sm100::mbar_arrive_cluster(sm100::mapa_shared(sm100::smem_u32(&xready[xs]), (uint32_t)k));
        }
        PB_WAIT(pb_try_cluster(&xready[xs], (uint32_t)((i >> 1) & 1)), "xready", i);
        if (a.trace && et == 0) a.trace[((size_t)blockIdx.x * T + t) * 8 + 5] = pb_gtime();
        // dh_rec of (row, unit j): the four chunk partials in chunk order (sum_split's order), read
        // for four rows at a time (registers)
        if (fin) {
#pragma unroll
          for (int q0 = 0; q0 < PB_RPT; q0 += 4) {
            float pv[4][PB_CL];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int r = ch * BWD_RB + y + BWD_RY * (q0 + q);
              const uint32_t off = (uint32_t)((((size_t)xs * a.a_rows + (r < a.B ? r : 0)) * PB_XS + crank * PB_UC + u) * 4);
#pragma unroll
              for (int k = 0; k < PB_CL; ++k) pv[q][k] = pb_ld_cluster(xpeer[k] + off);
            }
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              float v = pv[q][0];
#pragma unroll
              for (int k = 1; k < PB_CL; ++k) v = __fadd_rn(v, pv[q][k]);
              s[q0 + q] = v;
            }
          }
        }
        have_s = true;
      } else if (a.dhT) {
#pragma unroll
        for (int q = 0; q < PB_RPT; ++q) {
          const int r = ch * BWD_RB + y + BWD_RY * q;
          s[q] = (fin && r < a.B && unit_ok) ? a.dhT[(long)r * a.H + j] : 0.f;
        }
        have_s = true;
      }
      // cell backward of the rows, column-sum contributions in ascending row order (R5)
      float acc[NV];
#pragma unroll
      for (int q = 0; q < NV; ++q) acc[q] = 0.f;
      if (fin) {
#pragma unroll
        for (int q = 0; q < PB_RPT; ++q) {
          const int r = ch * BWD_RB + y + BWD_RY * q;
          if (r >= a.B) break;
          const long rr = (long)t * a.B + r;
          float da[4], duh[4], dwx[4];
          if (unit_ok) {
            float bb[4], al[4], be1[4], be2[4];   // (from shared memory: registers are the limit here)
#pragma unroll
            for (int g = 0; g < 4; ++g) {
              bb[g] = prm[g * PB_UC + u];
              al[g] = prm[(4 + g) * PB_UC + u];
              be1[g] = prm[(8 + g) * PB_UC + u];
              be2[g] = prm[(12 + g) * PB_UC + u];
            }
            const float dh = have_s ? __fadd_rn(dyv[q], s[q]) : dyv[q];
            lstm_bwd_da<KIND, F>(w[q], h[q], dh, dcv[q], cp[q], cn[q], bb, al, be1, be2, da, duh, dwx);
          } else {   // padding units: exact zeros everywhere
#pragma unroll
            for (int g = 0; g < 4; ++g) { da[g] = 0.f; duh[g] = 0.f; dwx[g] = 0.f; }
            dcv[q] = 0.f;
          }
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            lstm_bwd_acc<KIND, F>(acc, g, da[g], w[q][g], h[q][g]);
            a.D_uh[rr * NG + jc + g * GATE_U] = __float2bfloat16_rn(duh[g]);
            if (KIND == K_MILSTM) a.D_wx[rr * NG + jc + g * GATE_U] = __float2bfloat16_rn(dwx[g]);
          }
        }
      }
      // publish D_uh,t to the CTAs that read its chunk (generic-proxy stores → their TMA reads)
      if (a.trace && et == 0) a.trace[((size_t)blockIdx.x * T + t) * 8 + 6] = pb_gtime();
      if (t > 0) {
        pb_fence_proxy_async_global();
        __threadfence();
      }
      if (fin) {
#pragma unroll
        for (int q = 0; q < NV; ++q) red[((ch * BWD_RY + y) * NV + q) * PB_UC + u] = acc[q];
      }
      pb_epi_bar();
      if (t > 0 && et == 0) {
        atomicAdd(a.flags + out_chunk, 1u);
        if (a.trace) a.trace[((size_t)blockIdx.x * T + t) * 8 + 7] = pb_gtime();
      }
      // row lanes combined in y order, folded into the chunk partials (first step: assigned)
      for (int it = et; it < nch * NV * PB_UC; it += 32 * PB_EPI_WARPS) {
        const int c2 = it / (NV * PB_UC), q = (it / PB_UC) % NV, uu = it % PB_UC;
        if (q / 4 >= a.nq) continue;
        float v = 0.f;
#pragma unroll
        for (int yy = 0; yy < BWD_RY; ++yy) v = __fadd_rn(v, red[((c2 * BWD_RY + yy) * NV + q) * PB_UC + uu]);
        float& cpv = cpart[(c2 * NV + q) * PB_UC + uu];
        cpv = t == T - 1 ? v : __fadd_rn(cpv, v);
      }
      pb_epi_bar();   // red reusable
    }
    // final state: dc_0, the column-sum partials in the launched kernels' layout
    if (fin) {
#pragma unroll
      for (int q = 0; q < PB_RPT; ++q) {
        const int r = ch * BWD_RB + y + BWD_RY * q;
        if (r < a.B) a.dc[(long)r * a.Hp + j] = dcv[q];
      }
    }
    for (int it = et; it < nch * NV * PB_UC; it += 32 * PB_EPI_WARPS) {
      const int c2 = it / (NV * PB_UC), q = (it / PB_UC) % NV, uu = it % PB_UC;
      const int qq = q / 4, g = q % 4, jj = ju0 + uu;
      if (qq >= a.nq || jj >= a.Hp) continue;
      a.partials[(long)c2 * a.nq * NG + (long)qq * NG + gcol(g, jj)] = cpart[(c2 * NV + q) * PB_UC + uu];
    }
  }
  __syncthreads();
  sm100::cluster_sync();   // no CTA exits while a peer may still read its exchange buffer
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, 128);
  }
}

bool lstm_bptt_persist_supported(int B, int Hp, int nsplit) {
  return B >= 1 && B <= 128 && nsplit == PB_CL && Hp % 256 == 0 && Hp / PB_UC <= num_sms();
}

static int pb_smem_bytes(const BpttPersistArgs& a, int nq_kind) {
  const int NV = nq_kind * 4;
  const int nch = (a.B + BWD_RB - 1) / BWD_RB;
  const int bars = (2 * a.sa + 2 * a.sb + 1 + 6) * 8 + 16;
  return 1024 + a.sa * a.ka * a.a_bytes + a.resident * PB_BT + a.sb * a.kbs * PB_BT + 2 * a.a_rows * PB_XS * 4 +
         (nch * BWD_RY * NV * PB_UC + nch * NV * PB_UC + 16 * PB_UC) * 4 + bars;
}

using PbFn = void (*)(CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap, BpttPersistArgs);
static PbFn pb_kernel(int kind, bool dy_f32) {
  switch (kind) {
    case K_LSTM: return dy_f32 ? lstm_bptt_persist_kernel<K_LSTM, float> : lstm_bptt_persist_kernel<K_LSTM, __nv_bfloat16>;
    case K_MILSTM: return dy_f32 ? lstm_bptt_persist_kernel<K_MILSTM, float> : lstm_bptt_persist_kernel<K_MILSTM, __nv_bfloat16>;
    default: return dy_f32 ? lstm_bptt_persist_kernel<K_SUBLSTM, float> : lstm_bptt_persist_kernel<K_SUBLSTM, __nv_bfloat16>;
  }
}

// stage / residency plan for a shape (fills the launcher-set fields of a)
// Stage / residency plan for a shape (fills the launcher-set fields of a); false if nothing fits.
// Measured at cfg5, B = 64 (profiles/r2_pb_sweep.jsonl): the k-loop is bound by the bytes in flight
// per CTA, so the default spends shared memory on deep A / B rings (4 k-blocks per stage) rather
// than on resident U k-blocks; the A ring shrinks first when 128-row A boxes (B > 64) do not fit.
static bool pb_plan(int kind, BpttPersistArgs& a, int maxs) {
  auto knob = [](const char* n, int d) { const char* e = std::getenv(n); return e ? std::atoi(e) : d; };
  static const int k_ka = knob("ASTRA_PB_KA", 4), k_sa = knob("ASTRA_PB_SA", 3), k_kb = knob("ASTRA_PB_KB", 4),
                   k_sb = knob("ASTRA_PB_SB", 2), k_res = knob("ASTRA_PB_RES", 0);
  static const unsigned long long k_spin = [] {
    const char* e = std::getenv("ASTRA_PB_SPIN");
    return e ? std::strtoull(e, nullptr, 10) : 0ull;
  }();
  a.spin = k_spin;
  const int nk = a.NG / TC_BK;
  a.kper = nk / PB_CL;
  a.a_rows = a.B <= 64 ? 64 : 128;
  a.a_bytes = a.a_rows * TC_BK * 2;
  const int nqk = kind == K_MILSTM ? 4 : 1;
  for (int ka = k_ka; ka >= 1; --ka) {
    if (a.kper % ka != 0) continue;
    for (int sa = std::max(2, k_sa); sa >= 2; --sa)
      for (int kbs = std::max(1, k_kb); kbs >= 1; --kbs) {
        a.ka = ka; a.sa = sa; a.kbs = kbs;
        a.sb = 0;
        a.resident = a.kper;
        while (a.resident >= 0 && (pb_smem_bytes(a, nqk) > maxs || (k_res >= 0 && a.resident > k_res) ||
                                   (a.kper - a.resident) % a.kbs != 0)) {
          a.sb = std::max(1, k_sb);
          --a.resident;
        }
        if (a.resident >= 0) return true;
      }
  }
  return false;
}

static cudaLaunchConfig_t pb_config(const BpttPersistArgs& a, int smem, cudaStream_t st, cudaLaunchAttribute (&attr)[2],
                                    int nattr) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(a.Hp / PB_UC);
  cfg.blockDim = dim3(PB_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = PB_CL;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeCooperative;   // every CTA resident: the chunk counters act as barriers
  attr[1].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = nattr;
  return cfg;
}

bool lstm_bptt_persist_fits(int kind, int B, int Hp, int NG) {
  if (!lstm_bptt_persist_supported(B, Hp, PB_CL) || NG != 4 * Hp) return false;
  static std::map<std::tuple<int, int, int>, bool> memo;
  const auto key = std::make_tuple(kind, B, Hp);
  auto it = memo.find(key);
  if (it != memo.end()) return it->second;
  int dev = 0, maxs = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return false;
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  BpttPersistArgs a{};
  a.B = B; a.Hp = Hp; a.NG = NG;
  if (!pb_plan(kind, a, maxs)) {
    memo[key] = false;
    return false;
  }
  const int smem = pb_smem_bytes(a, kind == K_MILSTM ? 4 : 1);
  bool ok = true;
  for (int f = 0; f < 2 && ok; ++f) {
    PbFn fn = pb_kernel(kind, f == 0);
    CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    cudaLaunchAttribute attr[2];
    cudaLaunchConfig_t cfg = pb_config(a, smem, nullptr, attr, 1);
    int nclusters = 0;
    CUDA_TRY(cudaOccupancyMaxActiveClusters(&nclusters, fn, &cfg));
    ok = nclusters * PB_CL >= (int)cfg.gridDim.x;
    if (std::getenv("ASTRA_PB_VERBOSE")) {
      std::fprintf(stderr, "bptt_persist fits: kind %d B %d Hp %d smem %d resident %d clusters %d grid %d\n", kind, B, Hp,
                   smem, a.resident, nclusters, (int)cfg.gridDim.x);
      int nb = -1;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, PB_THREADS, smem);
      std::fprintf(stderr, "  blocks/SM %d\n", nb);
    }
  }
  memo[key] = ok;
  return ok;
}

void lstm_bptt_persist_launch(int kind, bool dy_f32, const void* Duh, const void* Um, int Tmax, BpttPersistArgs a,
                              cudaStream_t st) {
  ASTRA_CHECK_ARG(lstm_bptt_persist_fits(kind, a.B, a.Hp, a.NG),
                  "persistent small-batch BPTT: needs B <= 128, Hp % 256 == 0, 4 K chunks and co-resident clusters");
  int dev = 0, maxs = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  ASTRA_CHECK_ARG(pb_plan(kind, a, maxs), "persistent small-batch BPTT: shared memory too small");
  const int nk = a.NG / TC_BK;
  const int nqk = kind == K_MILSTM ? 4 : 1;
  // D f32, A bf16 K-major, B bf16 MN-major, N = 64, M = 128
  a.idesc = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(PB_UG >> 3) << 17) |
            ((uint32_t)(TC_BM >> 4) << 24);
  CUtensorMap mA, mB, mBr, mB1;
  {   // D_uh as {64 k, rows B, k-block (stride 128 B), t}
    const long dims[4] = {64, a.B, nk, Tmax};
    const long str[3] = {(long)a.NG * 2, 128, (long)a.B * a.NG * 2};
    const int box[4] = {64, a.a_rows, a.ka, 1};
    make_map_nd(&mA, Duh, 4, dims, str, box, 128);
  }
  {   // the U mirror [NG][Hp] as MN-major B: {Hp (units), 64 k rows, k-block (stride 64 rows)}
    const long dims[3] = {a.Hp, 64, nk};
    const long str[2] = {(long)a.Hp * 2, (long)TC_BK * a.Hp * 2};
    const int box[3] = {64, 64, a.kbs};
    make_map_nd(&mB, Um, 3, dims, str, box, 128);
    const int boxr[3] = {64, 64, 8};
    make_map_nd(&mBr, Um, 3, dims, str, boxr, 128);
    const int box1[3] = {64, 64, 1};
    make_map_nd(&mB1, Um, 3, dims, str, box1, 128);
  }
  const int smem = pb_smem_bytes(a, nqk);
  PbFn fn = pb_kernel(kind, dy_f32);
  CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaLaunchAttribute attr[2];
  cudaLaunchConfig_t cfg = pb_config(a, smem, st, attr, 2);
  CUDA_TRY(cudaLaunchKernelEx(&cfg, fn, mA, mB, mBr, mB1, a));
  LAUNCH_CHECK();
}

}  // namespace astra
