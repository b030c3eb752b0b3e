// K4 fused: one launch per BPTT step computes dh_rec = D_uh_{t+1}·Uᵀ on the tcgen05 main loop and
// runs the LSTM-family cell backward of step t in the same kernel — the fused BPTT step of the
// north star, the backward counterpart of the fused gate epilogue.
//
// Tile: one CTA owns 128 batch rows x 64 hidden units (the 256 gate-interleaved columns of those
// units in D_uh_t / D_wx_t).  Main loop: K = 4·Hp in k-blocks of 64; the canonical split-K of the
// BPTT GEMM (reading R25: s chunks accumulated from zero, summed in chunk order) is kept by giving
// each chunk its own TMEM accumulator (s x 64 columns), so no partial leaves the SM.
// Epilogue (8 warps): (1) TMEM → dh_rec = ((p0 + p1) + p2) + p3 per (row, unit) → shared memory
// (transposed to the unit-per-thread layout); (2) the cell backward with the thread mapping, row
// order and column-sum order of the unfused kernel (lstm_bwd_row.cuh), its inputs — WX_t, UH_t,
// c_t, c_{t-1}, dc, dy_t for 16 rows at a time — streamed by TMA tensor loads into the drained
// main-loop stages (3-deep ring).  The saved tensors are prefetched into L2 at kernel start (they
// are older than the grid dependency), so the epilogue's loads overlap the main loop.  Bitwise
// identical to GEMM + unfused pointwise kernel (tests/test_gpu_cell.py::test_fused_bwd_bitwise).
#include "cell_math.cuh"
#include "gemm_tc.cuh"
#include "kernels.h"
#include "lstm_bwd_row.cuh"
#include "pdl.cuh"
#include "rec_fused.h"
#include "sm100.cuh"

namespace astra {

constexpr int BF_EPI_WARPS = 8;                       // 64 units x 4 row lanes
constexpr int BF_THREADS = 64 + 32 * BF_EPI_WARPS;    // warp 0 TMA, warp 1 MMA, warps 2..9 epilogue
constexpr int BF_BN = 64;                             // units per tile (MMA N)
constexpr int BF_STAGE = TC_BM * TC_BK * 2 + BF_BN * TC_BK * 2;   // A 16 KB + B 8 KB
constexpr int BF_HR = 16;                             // rows per streamed epilogue half-chunk
constexpr int BF_NBUF = 3;                            // epilogue input ring depth
constexpr int BF_DHS_LD = 65;                         // padded row stride of the dh tile (floats)
constexpr int BF_DHS_BYTES = ((TC_BM * BF_DHS_LD * 4 + 1023) / 1024) * 1024;
// half-chunk buffer: WX [16][256] | UH [16][256] | c_t [16][64] | c_{t-1} [16][64] | dc [16][64] | dy [16][64]
constexpr int BF_O_UH = BF_HR * 256 * 4, BF_O_CN = 2 * BF_HR * 256 * 4, BF_O_CP = BF_O_CN + BF_HR * 64 * 4,
              BF_O_DC = BF_O_CP + BF_HR * 64 * 4, BF_O_DY = BF_O_DC + BF_HR * 64 * 4;
constexpr int BF_BUF = BF_O_DY + BF_HR * 64 * 4;      // 48 KB

__device__ __forceinline__ void bf_epi_bar() {   // named barrier over the epilogue warps only
  asm volatile("bar.sync 1, %0;" ::"n"(32 * BF_EPI_WARPS) : "memory");
}

template <int KIND, typename TDY>
__global__ void __launch_bounds__(BF_THREADS, 1)
    lstm_bptt_fused_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                           const __grid_constant__ CUtensorMap mapWX, const __grid_constant__ CUtensorMap mapUH,
                           const __grid_constant__ CUtensorMap mapC, const __grid_constant__ CUtensorMap mapDC,
                           const __grid_constant__ CUtensorMap mapDY, const BpttFusedArgs a) {
  using T = __nv_bfloat16;
  constexpr int NV = BwdNV<KIND>::value;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int stages = a.stages;
  float (*red)[NV][BWD_UX] = reinterpret_cast<float (*)[NV][BWD_UX]>(smem + stages * BF_STAGE);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + stages * BF_STAGE + BWD_RY * NV * BWD_UX * 4);
  uint64_t* empty = full + stages;
  uint64_t* tfull = empty + stages;
  uint64_t* ebar = tfull + 1;   // [BF_NBUF]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(ebar + BF_NBUF);
  float* dhs = reinterpret_cast<float*>(smem);            // after the main loop: [128][65] dh_rec
  uint8_t* ebuf = smem + BF_DHS_BYTES;                    // after the main loop: BF_NBUF x 48 KB

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int num_m = (a.B + TC_BM - 1) / TC_BM;
  const int m_blk = blockIdx.x % num_m, u_blk = blockIdx.x / num_m;
  const int m0 = m_blk * TC_BM, u0 = u_blk * BF_BN, n0 = u_blk * 4 * BF_BN;
  const int t = a.t;
  const int nhc = (min(a.B - m0, TC_BM) + BF_HR - 1) / BF_HR;   // half-chunks with at least one real row

  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      sm100::mbar_init(&full[s], 1);
      sm100::mbar_init(&empty[s], 1);
    }
    sm100::mbar_init(tfull, 1);
    for (int q = 0; q < BF_NBUF; ++q) sm100::mbar_init(&ebar[q], 1);
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, 256);
  if (warp == 2 && lane == 0) {
    // the saved tensors of step t (written long before this launch) → L2 while the main loop runs
    for (int hc = 0; hc < nhc; ++hc) {
      const int r = m0 + hc * BF_HR;
      sm100::tma_prefetch_l2_box(&mapWX, n0, r, t);
      sm100::tma_prefetch_l2_box(&mapUH, n0, r, t);
      sm100::tma_prefetch_l2_box(&mapC, u0, r, t + 1);
      sm100::tma_prefetch_l2_box(&mapC, u0, r, t);
      sm100::tma_prefetch_l2_box(&mapDY, u0, r, t);
    }
  }
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      const uint64_t pol = sm100::l2_policy_evict_last();
      const int pre = a.nk < stages ? a.nk : stages;
      for (int kb = 0; kb < pre; ++kb) {   // the U mirror (weights) before the grid dependency resolves
        sm100::mbar_arrive_expect_tx(&full[kb], BF_STAGE);
        sm100::tma_load_3d_hint(smem + kb * BF_STAGE + TC_BM * TC_BK * 2, &mapB, &full[kb], u0, kb * TC_BK, 0, pol);
      }
      pdl_wait();
      pdl_trigger();
      for (int kb = 0; kb < a.nk; ++kb) {
        const int s = kb % stages;
        if (kb >= pre) {
          sm100::mbar_wait(&empty[s], (uint32_t)((kb / stages) & 1) ^ 1);
          sm100::mbar_arrive_expect_tx(&full[s], BF_STAGE);
          sm100::tma_load_3d_hint(smem + s * BF_STAGE + TC_BM * TC_BK * 2, &mapB, &full[s], u0, kb * TC_BK, 0, pol);
        }
        sm100::tma_load_3d(smem + s * BF_STAGE, &mapA, &full[s], kb * TC_BK, m0, t + 1);
      }
    } else {
      pdl_wait();
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer: one accumulator per split-K chunk
    pdl_wait();
    {   // whole warp (umma_*_warp elect the issuing lane); lean loop: descriptors advanced by (bytes >> 4)
      const uint32_t sa0 = sm100::smem_u32(smem);
      const uint64_t dA0 = sm100::smem_desc_sw128(sa0, 16, 1024);
      const uint64_t dB0 = sm100::smem_desc_sw128(sa0 + TC_BM * TC_BK * 2, 8192, 1024);
      const uint32_t idesc = a.idesc, kper = (uint32_t)a.kper;
      int s = 0, c = 0;
      uint32_t ph = 0, jk = 0;
      for (int kb = 0; kb < a.nk; ++kb) {
        sm100::mbar_wait(&full[s], ph);
        sm100::tc_fence_after();
        const uint64_t ad = dA0 + (uint64_t)(s * (BF_STAGE >> 4)), bd = dB0 + (uint64_t)(s * (BF_STAGE >> 4));
#pragma unroll
        for (int kk = 0; kk < TC_BK / 16; ++kk)
          sm100::umma_bf16_warp(tmem_base + c * BF_BN, ad + 2 * kk, bd + 128 * kk, idesc, (jk | kk) != 0);
        sm100::umma_commit_warp(&empty[s]);
        if (++s == stages) { s = 0; ph ^= 1; }
        if (++jk == kper) { jk = 0; ++c; }
      }
      sm100::umma_commit_warp(tfull);
    }
  } else {
    // ------------------------------------------------------------ fused cell backward (8 warps)
    pdl_wait();
    const int et = threadIdx.x - 64;             // 0..255
    const int tx = et % BWD_UX, ty = et / BWD_UX;
    const int j = u0 + tx;
    const bool issuer = et == 0;
    const uint32_t ebytes = (uint32_t)(BF_O_DY + BF_HR * 64 * sizeof(TDY));
    auto issue = [&](int hc) {                   // inputs of rows m0 + 16·hc .. +15 into buffer hc % BF_NBUF
      const uint32_t b = sm100::smem_u32(ebuf + (hc % BF_NBUF) * BF_BUF);
      uint64_t* bar = &ebar[hc % BF_NBUF];
      const int r = m0 + hc * BF_HR;
      sm100::mbar_arrive_expect_tx(bar, ebytes);
      sm100::tma_load_box(b, &mapWX, bar, n0, r, t);
      sm100::tma_load_box(b + BF_O_UH, &mapUH, bar, n0, r, t);
      sm100::tma_load_box(b + BF_O_CN, &mapC, bar, u0, r, t + 1);
      sm100::tma_load_box(b + BF_O_CP, &mapC, bar, u0, r, t);
      sm100::tma_load_box(b + BF_O_DC, &mapDC, bar, u0, r, 0);
      sm100::tma_load_box(b + BF_O_DY, &mapDY, bar, u0, r, t);
    };
    // this thread's gate parameters (registers, as in the unfused kernel)
    float bb[4], al[4], be1[4], be2[4];
#pragma unroll
    for (int g = 0; g < 4; ++g) {
      const int e = g * a.H + j;
      const bool ok = j < a.H;
      bb[g] = ok ? a.gp.b[e] : 0.f;
      al[g] = (ok && KIND == K_MILSTM) ? a.gp.alpha[e] : 0.f;
      be1[g] = (ok && KIND == K_MILSTM) ? a.gp.beta1[e] : 0.f;
      be2[g] = (ok && KIND == K_MILSTM) ? a.gp.beta2[e] : 0.f;
    }
    sm100::mbar_wait(tfull, 0);                  // accumulators complete ⇒ every stage drained
    sm100::tc_fence_after();
    if (issuer)
      for (int hc = 0; hc < BF_NBUF && hc < nhc; ++hc) issue(hc);
    {   // (1) dh_rec = Σ_c p_c in chunk order, TMEM (lane = row) → shared memory [row][unit]
      const int quarter = warp & 3, half = (warp - 2) / 4;
      const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + half * 32;
      float r[32];
      sm100::tmem_ld32(taddr, r);
      for (int c = 1; c < a.nsplit; ++c) {
        float p[32];
        sm100::tmem_ld32(taddr + c * BF_BN, p);
#pragma unroll
        for (int u = 0; u < 32; ++u) r[u] = __fadd_rn(r[u], p[u]);
      }
      float* row = dhs + (quarter * 32 + lane) * BF_DHS_LD + half * 32;
#pragma unroll
      for (int u = 0; u < 32; ++u) row[u] = r[u];
    }
    sm100::tc_fence_before();
    bf_epi_bar();
    // (2) cell backward, 32-row chunks in two streamed halves; thread (tx, ty): rows ty + 4i
    const long NG = a.NG;
    T* D_uh = reinterpret_cast<T*>(a.D_uh) + (long)t * a.B * NG;   // step t's slice
    T* D_wx = reinterpret_cast<T*>(a.D_wx) + (long)t * a.B * NG;
    const int c0 = gcol(0, j);
    for (int cc = 0; cc < (nhc + 1) / 2; ++cc) {
      float acc[NV];
#pragma unroll
      for (int i = 0; i < NV; ++i) acc[i] = 0.f;
      for (int hb = 0; hb < 2; ++hb) {
        const int hc = 2 * cc + hb;
        if (hc < nhc) {
          sm100::mbar_wait(&ebar[hc % BF_NBUF], (uint32_t)((hc / BF_NBUF) & 1));
          const uint8_t* buf = ebuf + (hc % BF_NBUF) * BF_BUF;
          const float* sWX = reinterpret_cast<const float*>(buf);
          const float* sUH = reinterpret_cast<const float*>(buf + BF_O_UH);
          const float* sCN = reinterpret_cast<const float*>(buf + BF_O_CN);
          const float* sCP = reinterpret_cast<const float*>(buf + BF_O_CP);
          const float* sDC = reinterpret_cast<const float*>(buf + BF_O_DC);
          const TDY* sDY = reinterpret_cast<const TDY*>(buf + BF_O_DY);
#pragma unroll 1
          for (int i = 0; i < BF_HR / BWD_RY; ++i) {
            const int rl = ty + BWD_RY * i;        // row within the half-chunk
            const int rt = hc * BF_HR + rl;        // row within the tile
            const long b = m0 + rt;
            if (b >= a.B) break;
            if (j < a.H) {
              float w[4], h[4];
#pragma unroll
              for (int g = 0; g < 4; ++g) {
                w[g] = sWX[rl * 256 + g * GATE_U + tx];
                h[g] = sUH[rl * 256 + g * GATE_U + tx];
              }
              const float dh = __fadd_rn(to_f<TDY>(sDY[rl * 64 + tx]), dhs[rt * BF_DHS_LD + tx]);
              float dcv = sDC[rl * 64 + tx];
              lstm_bwd_row<KIND, T>(w, h, dh, dcv, sCP[rl * 64 + tx], sCN[rl * 64 + tx], bb, al, be1, be2, acc,
                                    D_uh + b * NG + c0, D_wx + b * NG + c0);
              a.dc[b * a.Hp + j] = dcv;
            } else if (j < a.Hp) {   // padding units: keep their gradients exactly zero
#pragma unroll
              for (int g = 0; g < 4; ++g) {
                D_uh[b * NG + c0 + g * GATE_U] = from_f<T>(0.f);
                if (KIND == K_MILSTM) D_wx[b * NG + c0 + g * GATE_U] = from_f<T>(0.f);
              }
              a.dc[b * a.Hp + j] = 0.f;
            }
          }
          bf_epi_bar();                            // buffer hc consumed by every thread
          if (issuer && hc + BF_NBUF < nhc) {
            sm100::fence_proxy_async_smem();
            issue(hc + BF_NBUF);
          }
        }
      }
#pragma unroll
      for (int i = 0; i < NV; ++i) red[ty][i][tx] = acc[i];
      bf_epi_bar();
      if (j < a.Hp)
        bwd_chunk_finalize<NV>(red, tx, ty, a.partials + (long)(m0 / BWD_RB + cc) * a.nq * NG, NG, c0, a.nq, 0);
      bf_epi_bar();
    }
  }
  __syncthreads();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, 256);
  }
}

int lstm_bptt_fused_smem(int stages, int kind) {
  const int nv = kind == K_MILSTM ? 16 : 4;
  return 1024 + stages * BF_STAGE + BWD_RY * nv * BWD_UX * 4 + 256;
}

bool lstm_bptt_fused_supported(int B, int Hp, int nsplit) {
  (void)B;
  return Hp % BF_BN == 0 && nsplit >= 1 && nsplit <= 4;
}

void lstm_bptt_fused_launch(int kind, bool dy_bf16, const BpttFusedMaps& m, BpttFusedArgs a, cudaStream_t st) {
  int dev = 0, maxs = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  int stages = (maxs - lstm_bptt_fused_smem(0, kind)) / BF_STAGE;
  if (stages > 8) stages = 8;
  ASTRA_CHECK_STATE(stages * BF_STAGE >= BF_DHS_BYTES + BF_NBUF * BF_BUF, "fused BPTT: shared memory too small");
  ASTRA_CHECK_ARG(a.nsplit >= 1 && a.nsplit <= 4 && a.kper * a.nsplit >= a.nk, "fused BPTT: bad split");
  a.stages = stages;
  const int smem = lstm_bptt_fused_smem(stages, kind);
  using Fn = void (*)(CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap, CUtensorMap,
                      BpttFusedArgs);
  Fn fn = nullptr;
#define BF_PICK(K)                                                                          \
  if (kind == K) fn = dy_bf16 ? (Fn)lstm_bptt_fused_kernel<K, __nv_bfloat16> : (Fn)lstm_bptt_fused_kernel<K, float>;
  BF_PICK(K_LSTM)
  BF_PICK(K_MILSTM)
  BF_PICK(K_SUBLSTM)
#undef BF_PICK
  ASTRA_CHECK_ARG(fn != nullptr, "fused BPTT: cell kind");
  static int attr_bytes[8][2] = {};
  int& ab = attr_bytes[kind & 7][dy_bf16 ? 1 : 0];
  if (ab < smem) {
    CUDA_TRY(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    ab = smem;
  }
  const int grid = cdiv(a.B, TC_BM) * (a.Hp / BF_BN);
  launch_pdl(fn, dim3(grid), dim3(BF_THREADS), smem, st, 1, m.A, m.B, m.WX, m.UH, m.C, m.DC, m.DY, a);
  LAUNCH_CHECK();
}

}  // namespace astra
