// K4 persistent form of the RHN BPTT chain (SURVEY §8(a) row a5 for cfg3, §8(a.9) `bwd_kernel`
// "persistent"; round-1 VERDICT: "fused BPTT for SCRN, RHN and attention").
//
// One cooperative launch runs all T·L backward micro-steps.  Clusters of 4 CTAs = the canonical R33
// split-K chunks of the micro-step GEMM  ds_part = DA(ℓ,t)·R_ℓᵀ  (K = 2·Hp), 32 hidden units per
// cluster:
//   - CTA c computes chunk c of its 32 units' partial (tcgen05 M = 128, N = 32; A = the chunk's
//     columns of DA(ℓ,t), one 4-D TMA box; B = the chunk of R_ℓ's rows for the 32 units, read from a
//     K-major copy of the R mirror and prefetched one micro-step ahead);
//   - the four fp32 partials meet in shared memory: CTA c reads the partials of ITS 8 units from all
//     four CTAs over distributed shared memory and adds them in chunk order — rhn_bwd_pw_kernel's
//     sum_split order — onto the carry ds·(1 − τ) it keeps in registers, then runs the micro-step
//     backward of rhn_bwd_pw_kernel operation for operation (dy added at ℓ = L − 1) and writes
//     DA(ℓ',t') of its units;
//   - one grid-wide counter per micro-step publishes DA to the next micro-step's A loads.
// The db column sums follow R5 exactly: thread (unit, row lane y of 8, 32-row chunk) walks rows y,
// y+8, y+16, y+24 in ascending order, the 8 lanes are combined in y order and folded per micro-layer
// ℓ over t = T−1 … 0.  The last GEMM's partials finish ds of s^0_0 (add_split_partials' order).
// Bitwise equal to the launched chain (rhn_bwd_pw + K1 split-K GEMM per micro-step).
#include <cstdlib>
#include <map>
#include <tuple>

#include "cell_math.cuh"
#include "gemm.h"
#include "gemm_tc.cuh"
#include "kernels.h"
#include "pdl.cuh"
#include "rec_fused.h"

namespace astra {

namespace {

constexpr int RB_CL = 4;                  // cluster size = the R33 chunks
constexpr int RB_UG = 32;                 // units per cluster (MMA N)
constexpr int RB_UC = RB_UG / RB_CL;      // units finalised per CTA (8)
constexpr int RB_BT = RB_UG * TC_BK * 2;  // bytes of one B k-block (32 rows x 128 B)
constexpr int RB_EPI_WARPS = 8;
constexpr int RB_THREADS = 32 * (3 + RB_EPI_WARPS);
constexpr int RB_XS = RB_UG + 1;          // fp32 row stride of the exchange buffer
constexpr int RB_RY = 8;                  // row lanes of the column sums (rhn_bwd_pw_kernel's PW_RY)
constexpr int RB_RB = 32;                 // rows per column-sum chunk (PW_RB)
constexpr int RB_RPT = RB_RB / RB_RY;     // rows per finalising thread (4)

__device__ __forceinline__ void rb_fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__device__ __forceinline__ unsigned rb_ld_acquire(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void rb_epi_bar() { asm volatile("bar.sync 1, %0;" ::"n"(32 * RB_EPI_WARPS) : "memory"); }
__device__ __forceinline__ void rb_wait_cluster(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE_%=;\n\t"
      "bra WAIT_%=;\n"
      "DONE_%=:\n\t}" ::"r"(sm100::smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ float rb_ld_cluster(uint32_t a) {
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(a) : "memory");
  return v;
}

template <typename TDY>
__global__ void __launch_bounds__(RB_THREADS, 1)
    rhn_bptt_persist_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                            const RhnBpttArgs a) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int kper = a.kper, L = a.L, T = a.T, TL = T * L;
  const int a_bytes = 64 * TC_BK * 2;   // A tiles of 64 rows (B ≤ 64)
  uint8_t* sA = smem;                                   // [kper][64 rows][128 B]
  uint8_t* sB = sA + kper * a_bytes;                    // [2][kper][32 rows][128 B]
  float* xbuf = reinterpret_cast<float*>(sB + 2 * kper * RB_BT);   // [2][64][RB_XS]
  float* red = xbuf + 2 * 64 * RB_XS;                   // [2 chunks][RB_RY][2][RB_UC]
  float* cpart = red + 2 * RB_RY * 2 * RB_UC;           // [L][2 chunks][2][RB_UC]
  uint64_t* fullA = reinterpret_cast<uint64_t*>(cpart + L * 2 * 2 * RB_UC + 2);
  uint64_t* emptyA = fullA + 1;
  uint64_t* fullB = emptyA + 1;    // [2]
  uint64_t* emptyB = fullB + 2;    // [2]
  uint64_t* tfull = emptyB + 2;    // [2]
  uint64_t* tempty = tfull + 2;    // [2]
  uint64_t* xready = tempty + 2;   // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(xready + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int crank = (int)sm100::cluster_ctarank();      // = the chunk this CTA computes
  const int grp = blockIdx.x / RB_CL;                    // units [32·grp, +32)
  const int kb0 = crank * kper, nkc = min(a.nk - kb0, kper);   // the chunk's k-blocks
  const unsigned nct = gridDim.x;

  if (threadIdx.x == 0) {
    sm100::mbar_init(fullA, 1);
    sm100::mbar_init(emptyA, 1);
    for (int q = 0; q < 2; ++q) {
      sm100::mbar_init(&fullB[q], 1);
      sm100::mbar_init(&emptyB[q], 1);
      sm100::mbar_init(&tfull[q], 1);
      sm100::mbar_init(&tempty[q], 32 * RB_EPI_WARPS);
      sm100::mbar_init(&xready[q], RB_CL);
    }
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, 64);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::cluster_sync();   // every CTA's barriers are initialised before any remote arrive
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ A producer: DA(q) chunk columns
    if (lane == 0) {
      pdl_wait();
      for (int q = 0; q < TL; ++q) {
        const int t = T - 1 - q / L, l = L - 1 - q % L;
        while (rb_ld_acquire(a.flags) < nct * (unsigned)(q + 1)) __nanosleep(32);   // pw(q) published everywhere
        rb_fence_proxy_async_global();
        sm100::mbar_wait(emptyA, (uint32_t)(q & 1) ^ 1);
        sm100::mbar_arrive_expect_tx(fullA, (uint32_t)(kper * a_bytes));
        sm100::tma_load_4d(sA, &mapA, fullA, 0, 0, kb0, l * T + t);
      }
    }
  } else if (warp == 2) {
    // ------------------------------------------------------------ B producer: R_ℓ chunk rows (one ahead)
    if (lane == 0) {
      const uint64_t pol = sm100::l2_policy_evict_last();
      pdl_wait();
      for (int q = 0; q < TL; ++q) {
        const int l = L - 1 - q % L, bq = q & 1;
        sm100::mbar_wait(&emptyB[bq], (uint32_t)((q >> 1) & 1) ^ 1);
        sm100::mbar_arrive_expect_tx(&fullB[bq], (uint32_t)(kper * RB_BT));
        sm100::tma_load_4d_hint(sB + bq * kper * RB_BT, &mapB, &fullB[bq], 0, grp * RB_UG, kb0, l, pol);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer (whole warp)
    {
      const uint32_t idesc = a.idesc;
      const uint64_t dA0 = sm100::smem_desc_sw128(sm100::smem_u32(sA), 16, 1024);
      const uint64_t dB0 = sm100::smem_desc_sw128(sm100::smem_u32(sB), 16, 1024);
      const uint32_t a_kb = (uint32_t)a_bytes >> 4, b_kb = RB_BT >> 4, b_buf = (uint32_t)(kper * RB_BT) >> 4;
      for (int q = 0; q < TL; ++q) {
        const int acc = q & 1;
        sm100::mbar_wait(&tempty[acc], (uint32_t)((q >> 1) & 1) ^ 1);
        sm100::mbar_wait(fullA, (uint32_t)(q & 1));
        sm100::mbar_wait(&fullB[acc], (uint32_t)((q >> 1) & 1));
        sm100::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * RB_UG;
        const uint64_t bdb = dB0 + (uint64_t)(acc * b_buf);
        for (int kb = 0; kb < nkc; ++kb) {
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk)
            sm100::umma_bf16_warp(d_tmem, dA0 + kb * a_kb + 2 * kk, bdb + kb * b_kb + 2 * kk, idesc, (kb | kk) != 0);
        }
        sm100::umma_commit_warp(emptyA);
        sm100::umma_commit_warp(&emptyB[acc]);
        sm100::umma_commit_warp(&tfull[acc]);
      }
    }
  } else {
    // ------------------------------------------------------------ exchange + micro-step backward (8 warps)
    const int et = threadIdx.x - 96;
    const int quarter = warp & 3;
    // finalising thread (et < 128): unit u of the CTA's 8, row lane y of 8, 32-row chunk ch
    const int u = et % RB_UC, y = (et / RB_UC) % RB_RY, ch = et / (RB_UC * RB_RY);
    const bool fin = et < 2 * RB_RY * RB_UC && ch * RB_RB < a.B;
    const int j = grp * RB_UG + crank * RB_UC + u;
    const bool unit_ok = j < a.H;
    const long G2 = 2L * a.Hp;
    const uint32_t xb0 = sm100::smem_u32(xbuf);
    uint32_t xpeer[RB_CL];
#pragma unroll
    for (int k = 0; k < RB_CL; ++k) xpeer[k] = sm100::mapa_shared(xb0, (uint32_t)k);
    pdl_wait();
    float carry[RB_RPT];   // ds·(1 − τ) of the thread's rows (the launched chain's ds_out / ds_in)
#pragma unroll
    for (int k = 0; k < RB_RPT; ++k) {
      const int r = ch * RB_RB + y + RB_RY * k;
      carry[k] = (fin && r < a.B && unit_ok) ? a.dS[(long)r * a.Hp + j] : 0.f;
    }
    // pw(q) of micro-step q = (t, ℓ), with the partial sums z (have_z) of GEMM(q − 1)
    auto micro_step = [&](int q, bool have_z, const float (&z)[RB_RPT]) {
      const int t = T - 1 - q / L, l = L - 1 - q % L;
      const bool first = t == T - 1;
      const float* Ap = a.Apre + ((size_t)l * T + t) * a.B * G2;
      const float* Sp = a.Sf + ((size_t)l * (T + 1) + t) * a.B * a.Hp;
      __nv_bfloat16* DA = a.DA + ((size_t)l * T + t) * a.B * G2;
      const TDY* dyt = (l == L - 1) ? reinterpret_cast<const TDY*>(a.dy) + (size_t)t * a.B * a.ldy : nullptr;
      float sH = 0.f, sT = 0.f;
      if (fin) {
#pragma unroll
        for (int k = 0; k < RB_RPT; ++k) {
          const int r = ch * RB_RB + y + RB_RY * k;
          if (r >= a.B) break;
          float daH = 0.f, daT = 0.f, dso = 0.f;
          if (unit_ok) {
            float ds = carry[k];
            if (have_z) ds = __fadd_rn(ds, z[k]);
            if (dyt) ds = __fadd_rn(to_f<TDY>(dyt[(long)r * a.ldy + j]), ds);
            const float h = tanh_<true>(Ap[(long)r * G2 + j]), tau = sigm<true>(Ap[(long)r * G2 + a.Hp + j]);
            const float sp = Sp[(long)r * a.Hp + j];
            const float dh = __fmul_rn(ds, tau);
            const float dtau = __fmul_rn(ds, __fsub_rn(h, sp));
            daH = __fmul_rn(dh, __fsub_rn(1.f, __fmul_rn(h, h)));
            daT = __fmul_rn(__fmul_rn(dtau, tau), __fsub_rn(1.f, tau));
            dso = __fmul_rn(ds, __fsub_rn(1.f, tau));
          }
          DA[(long)r * G2 + j] = __float2bfloat16_rn(daH);
          DA[(long)r * G2 + a.Hp + j] = __float2bfloat16_rn(daT);
          carry[k] = dso;
          sH = __fadd_rn(sH, daH);
          sT = __fadd_rn(sT, daT);
        }
      }
      // publish DA(q) for GEMM(q) (generic-proxy stores → the TMA reads of every CTA)
      rb_fence_proxy_async_global();
      __threadfence();
      if (fin) {
        red[((ch * RB_RY + y) * 2 + 0) * RB_UC + u] = sH;
        red[((ch * RB_RY + y) * 2 + 1) * RB_UC + u] = sT;
      }
      rb_epi_bar();
      if (et == 0) atomicAdd(a.flags, 1u);
      if (et < 2 * 2 * RB_UC) {   // lanes combined in y order, folded per micro-layer (first step t = T−1)
        const int c2 = et / (2 * RB_UC), qq = (et / RB_UC) % 2, uu = et % RB_UC;
        if (c2 * RB_RB < a.B) {
          float v = 0.f;
#pragma unroll
          for (int yy = 0; yy < RB_RY; ++yy) v = __fadd_rn(v, red[((c2 * RB_RY + yy) * 2 + qq) * RB_UC + uu]);
          float& cp = cpart[((l * 2 + c2) * 2 + qq) * RB_UC + uu];
          cp = first ? v : __fadd_rn(cp, v);
        }
      }
      rb_epi_bar();   // red reusable
    };
    float z[RB_RPT];
#pragma unroll
    for (int k = 0; k < RB_RPT; ++k) z[k] = 0.f;
    micro_step(0, false, z);   // the first micro-step has no GEMM before it
    for (int q = 0; q < TL; ++q) {
      const int acc = q & 1, xs = q & 1;
      // GEMM(q)'s chunk partial of the 32 units: TMEM → exchange buffer (rows < B: lane quarters 0, 1)
      sm100::mbar_wait(&tfull[acc], (uint32_t)((q >> 1) & 1));
      sm100::tc_fence_after();
      if ((warp == 4 || warp == 5) && quarter * 32 < a.B) {
        float v[32];
        sm100::tmem_ld32(tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * RB_UG, v);
        const int row = quarter * 32 + lane;
        if (row < a.B) {
          float* xp = xbuf + ((size_t)xs * 64 + row) * RB_XS;
#pragma unroll
          for (int c = 0; c < RB_UG; ++c) xp[c] = v[c];
        }
      }
      sm100::tc_fence_before();
      sm100::mbar_arrive(&tempty[acc]);
      rb_epi_bar();
      if (et == 0) {
#pragma unroll
        for (int k = 0; k < RB_CL; ++k)
          sm100::mbar_arrive_cluster(sm100::mapa_shared(sm100::smem_u32(&xready[xs]), (uint32_t)k));
      }
      rb_wait_cluster(&xready[xs], (uint32_t)((q >> 1) & 1));
      // z = the four chunk partials of (row, unit j) in chunk order
      if (fin) {
        float pv[RB_RPT][RB_CL];
#pragma unroll
        for (int k = 0; k < RB_RPT; ++k) {
          const int r = ch * RB_RB + y + RB_RY * k;
          const uint32_t off = (uint32_t)((((size_t)xs * 64 + (r < a.B ? r : 0)) * RB_XS + crank * RB_UC + u) * 4);
#pragma unroll
          for (int c = 0; c < RB_CL; ++c) pv[k][c] = rb_ld_cluster(xpeer[c] + off);
        }
#pragma unroll
        for (int k = 0; k < RB_RPT; ++k) {
          float s = pv[k][0];
#pragma unroll
          for (int c = 1; c < RB_CL; ++c) s = __fadd_rn(s, pv[k][c]);
          z[k] = s;
        }
      }
      if (q + 1 < TL) {
        micro_step(q + 1, true, z);
      } else if (fin) {   // ds of s^0_0 = carry + partials (add_split_partials' order)
#pragma unroll
        for (int k = 0; k < RB_RPT; ++k) {
          const int r = ch * RB_RB + y + RB_RY * k;
          if (r < a.B) a.dS[(long)r * a.Hp + j] = unit_ok ? __fadd_rn(carry[k], z[k]) : 0.f;
        }
      }
    }
    // the db partials in the launched kernels' layout part[ℓ][chunk][H | T][Hp]
    for (int it = et; it < L * 2 * 2 * RB_UC; it += 32 * RB_EPI_WARPS) {
      const int uu = it % RB_UC, qq = (it / RB_UC) % 2, c2 = (it / (2 * RB_UC)) % 2, l = it / (4 * RB_UC);
      const int jj = grp * RB_UG + crank * RB_UC + uu;
      if (c2 * RB_RB >= a.B || jj >= a.Hp) continue;
      a.part[(size_t)l * a.nchunk * G2 + (size_t)c2 * G2 + (size_t)qq * a.Hp + jj] = cpart[((l * 2 + c2) * 2 + qq) * RB_UC + uu];
    }
  }
  __syncthreads();
  sm100::cluster_sync();   // no CTA exits while a peer may still read its exchange buffer
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, 64);
  }
}

int rb_smem_bytes(int kper, int L) {
  return 1024 + kper * 64 * TC_BK * 2 + 2 * kper * RB_BT + 2 * 64 * RB_XS * 4 + 2 * RB_RY * 2 * RB_UC * 4 +
         (L * 2 * 2 * RB_UC + 2) * 4 + 16 * 8 + 64;
}

}  // namespace

bool rhn_bptt_persist_supported(int B, int Hp, int nsplit, int L) {
  const int nk = cdiv(2 * Hp, TC_BK), kper = cdiv(nk, nsplit);
  return B >= 1 && B <= 64 && nsplit == RB_CL && Hp % RB_UG == 0 && Hp / RB_UG * RB_CL <= num_sms() &&
         rb_smem_bytes(kper, L) <= 200 * 1024;
}

bool rhn_bptt_persist_fits(int B, int Hp, int nsplit, int L) {
  if (!rhn_bptt_persist_supported(B, Hp, nsplit, L)) return false;
  static std::map<std::tuple<int, int, int>, bool> memo;
  const auto key = std::make_tuple(B, Hp, L);
  auto it = memo.find(key);
  if (it != memo.end()) return it->second;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return false;
  const int nk = cdiv(2 * Hp, TC_BK), kper = cdiv(nk, nsplit);
  const int smem = rb_smem_bytes(kper, L);
  bool ok = true;
  for (int f = 0; f < 2 && ok; ++f) {
    auto fn = f == 0 ? rhn_bptt_persist_kernel<float> : rhn_bptt_persist_kernel<__nv_bfloat16>;
    CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(Hp / RB_UG * RB_CL);
    cfg.blockDim = dim3(RB_THREADS);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = RB_CL;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    int nclusters = 0;
    CUDA_TRY(cudaOccupancyMaxActiveClusters(&nclusters, fn, &cfg));
    ok = nclusters * RB_CL >= (int)cfg.gridDim.x;
  }
  memo[key] = ok;
  return ok;
}

void rhn_bptt_persist_launch(bool dy_f32, const void* DA, const void* RK, RhnBpttArgs a, cudaStream_t st) {
  ASTRA_CHECK_ARG(rhn_bptt_persist_fits(a.B, a.Hp, a.nsplit, a.L), "persistent RHN BPTT: unsupported shape");
  a.nk = cdiv(2 * a.Hp, TC_BK);
  a.kper = cdiv(a.nk, a.nsplit);
  // D f32, A / B bf16 K-major, N = 32, M = 128
  a.idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(RB_UG >> 3) << 17) | ((uint32_t)(TC_BM >> 4) << 24);
  CUtensorMap mA, mB;
  {   // DA as {64 k, rows B, k-block (stride 128 B), (ℓ·T + t) slots}
    const long dims[4] = {64, a.B, a.nk, (long)a.L * a.T};
    const long str[3] = {2L * a.Hp * 2, 128, (long)a.B * 2 * a.Hp * 2};
    const int box[4] = {64, 64, a.kper, 1};
    make_map_nd(&mA, DA, 4, dims, str, box, 128);
  }
  {   // the K-major R copy RK[ℓ][Hp rows (units)][2·Hp]: {64 k, unit rows, k-block (stride 128 B), ℓ}
    const long dims[4] = {64, a.Hp, a.nk, a.L};
    const long str[3] = {2L * a.Hp * 2, 128, (long)a.Hp * 2 * a.Hp * 2};
    const int box[4] = {64, RB_UG, a.kper, 1};
    make_map_nd(&mB, RK, 4, dims, str, box, 128);
  }
  const int smem = rb_smem_bytes(a.kper, a.L);
  auto fn = dy_f32 ? rhn_bptt_persist_kernel<float> : rhn_bptt_persist_kernel<__nv_bfloat16>;
  CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(a.Hp / RB_UG * RB_CL);
  cfg.blockDim = dim3(RB_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = RB_CL;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeCooperative;   // every CTA resident: the counter is a grid barrier
  attr[1].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  CUDA_TRY(cudaLaunchKernelEx(&cfg, fn, mA, mB, a));
  LAUNCH_CHECK();
}

}  // namespace astra
