// K1: persistent, warp-specialised tcgen05 GEMM for sm_100a.
//
//   D[M,N] = A[M,K] · B[K,N], bf16 operands fed by TMA (SWIZZLE_128B) into a ring of shared-memory
//   stages, fp32 accumulation in TMEM (two accumulator buffers so the epilogue of tile i overlaps
//   the main loop of tile i+1), epilogue = tcgen05.ld → registers → a functor.
//
//   Warp roles (192 threads): warp 0 = TMA producer, warp 1 = TMEM allocator + single-thread
//   MMA issuer, warps 2..5 = epilogue (warp w reads TMEM lanes 32·(w%4) ..+31, i.e. tile rows).
//
//   Operands may be K-major (K contiguous) or MN-major (M resp. N contiguous); the latter lets
//   the weight-gradient GEMMs (dU = Hᵀ·dZ, dW = Xᵀ·dZ) and the dgrad GEMMs read the saved
//   activations and the weight mirrors in place, without transposes.
//
//   Numerics: every output element is accumulated from 0 over K in k-blocks
//   of 64 (4 MMAs of K=16) in ascending order, one CTA per element, no split-K — so the result
//   does not depend on the tile width BN, the raster order or the grid size (checked on B200 by
//   tests/test_gpu_gemm.py::test_tile_shapes_bitwise).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include "sm100.cuh"

namespace astra {

constexpr int TC_BM = 128;
constexpr int TC_BK = 64;          // one 128-byte swizzle atom of bf16 along K
constexpr int TC_THREADS = 192;

struct TcArgs {
  int M, N, K;
  int num_m, num_n;
  int az, bz;       // third tensor-map coordinate (time slice) of A and B
  int a_mn, b_mn;   // 1 = MN-major operand
  int stages;
  int cm, cn;       // cluster shape (CTAs sharing B along M, sharing A along N)
  int b_keep;       // 1: load B with an L2 evict_last policy (weights re-read every step)
  int ksplit;       // fixed split of K into ksplit chunks; chunk ks writes its fp32 partial to C + ks·split_stride
  uint32_t idesc;
};

template <int BN>
struct TcSmem {
  static constexpr int A_BYTES = TC_BM * TC_BK * 2;   // 16 KB
  static constexpr int B_BYTES = BN * TC_BK * 2;      // BN * 128 B
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int TMEM_COLS = (2 * BN <= 32) ? 32 : (2 * BN <= 64) ? 64 : (2 * BN <= 128) ? 128 : (2 * BN <= 256) ? 256 : 512;
  static int stages_for(int max_smem) {
    int s = (max_smem - 1024 - 256) / STAGE_BYTES;
    return s > 10 ? 10 : s;
  }
  static int bytes(int stages) { return 1024 + stages * STAGE_BYTES + 256; }
};

// Generic epilogue: store the fp32 accumulator (optionally + bias[n], optionally added onto the
// fp32 value already in C: out = C_old + acc) as fp32 or bf16 into a row-major [M][ldc] output.
// Output columns can be remapped from an internal gate layout to the external one:
//   perm_u  > 0: gate-interleaved tiles — internal n = tile·4u + g·u + j ↔ external g·perm_H + tile·u + j
//   perm_blk > 0: gate-blocked, padded  — internal n = g·perm_blk + j  ↔ external g·perm_H + j
// Rows ≥ Mv and invalid (padding) columns are dropped.
struct EpiStore {
  void* C;
  long ldc;
  int Mv, Nv;
  int out_bf16;
  const float* bias;  // indexed by internal column n, may be null
  int perm_u, perm_H; // 0 = identity mapping
  int perm_blk;
  int accumulate;
  long split_stride;  // elements between the partial outputs of a split-K GEMM

  __device__ __forceinline__ int map_col(int n, bool& ok) const {
    if (n >= Nv) {  // columns past the GEMM's N (tile overhang) are never stored
      ok = false;
      return 0;
    }
    if (perm_u) {
      const int q = 4 * perm_u;
      const int tile = n / q, g = (n % q) / perm_u, j = n % perm_u;
      const int unit = tile * perm_u + j;
      ok = unit < perm_H;
      return g * perm_H + unit;
    }
    if (perm_blk) {
      const int g = n / perm_blk, j = n % perm_blk;
      ok = j < perm_H;
      return g * perm_H + j;
    }
    ok = n < Nv;
    return n;
  }

  __device__ __forceinline__ void store16(int m, int n0, const float (&v)[16]) const {
    if (m >= Mv) return;
    bool ok0;
    const int e0 = map_col(n0, ok0);
    bool contiguous = n0 + 16 <= Nv;
    if (!contiguous) {
    } else if (perm_u) contiguous = ((n0 % perm_u) + 16 <= perm_u) && ((n0 / (4 * perm_u)) * perm_u + n0 % perm_u + 16 <= perm_H);
    else if (perm_blk) contiguous = (n0 % perm_blk) + 16 <= perm_H;
    float w[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) w[i] = v[i] + ((bias && n0 + i < Nv) ? bias[n0 + i] : 0.f);
    if (contiguous) {
      if (out_bf16) {
        __nv_bfloat16* p = reinterpret_cast<__nv_bfloat16*>(C) + (long)m * ldc + e0;
        if ((((uintptr_t)p) & 15) == 0) {
          uint4 pk[2];
          uint32_t* u = reinterpret_cast<uint32_t*>(pk);
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            __nv_bfloat162 b2 = __floats2bfloat162_rn(w[2 * i], w[2 * i + 1]);
            u[i] = *reinterpret_cast<uint32_t*>(&b2);
          }
          reinterpret_cast<uint4*>(p)[0] = pk[0];
          reinterpret_cast<uint4*>(p)[1] = pk[1];
        } else {
#pragma unroll
          for (int i = 0; i < 16; ++i) p[i] = __float2bfloat16_rn(w[i]);
        }
      } else {
        float* p = reinterpret_cast<float*>(C) + (long)m * ldc + e0;
        if ((((uintptr_t)p) & 15) == 0) {
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            float4 o = make_float4(w[4 * i], w[4 * i + 1], w[4 * i + 2], w[4 * i + 3]);
            if (accumulate) {
              const float4 c = reinterpret_cast<const float4*>(p)[i];
              o.x = __fadd_rn(c.x, o.x); o.y = __fadd_rn(c.y, o.y); o.z = __fadd_rn(c.z, o.z); o.w = __fadd_rn(c.w, o.w);
            }
            reinterpret_cast<float4*>(p)[i] = o;
          }
        } else {
#pragma unroll
          for (int i = 0; i < 16; ++i) p[i] = accumulate ? __fadd_rn(p[i], w[i]) : w[i];
        }
      }
      return;
    }
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      bool ok;
      const int e = map_col(n0 + i, ok);
      if (!ok) continue;
      if (out_bf16) {
        reinterpret_cast<__nv_bfloat16*>(C)[(long)m * ldc + e] = __float2bfloat16_rn(w[i]);
      } else {
        float* p = reinterpret_cast<float*>(C) + (long)m * ldc + e;
        *p = accumulate ? __fadd_rn(*p, w[i]) : w[i];
      }
    }
    (void)ok0;
  }

  template <int BN>
  __device__ __forceinline__ void run(uint32_t taddr, int m0, int n0, int row, int ks) const {
    EpiStore e = *this;
    if (ks) e.C = reinterpret_cast<char*>(C) + (size_t)ks * split_stride * (out_bf16 ? 2 : 4);
#pragma unroll 1
    for (int c = 0; c < BN; c += 16) {
      float v[16];
      sm100::tmem_ld16(taddr + c, v);
      e.store16(m0 + row, n0 + c, v);
    }
  }
};

// Cluster multicast (cm x cn CTAs per cluster, cluster rank r: rm = r % cm, rn = r / cm): the cn
// CTAs that share an A tile (same rm) each load 1/cn of it and multicast it to the others; the cm
// CTAs that share a B tile (same rn) do the same for B.  Every CTA's stage is therefore written by
// cm + cn − 1 CTAs, so its `empty` barrier expects that many MMA-commit arrivals (each MMA issuer
// commits to the `empty` barriers of all its neighbours).  Cuts L2→SMEM operand traffic by
// cm (B) and cn (A) without changing any accumulation order.
template <int BN, class Epi>
__global__ void __launch_bounds__(TC_THREADS, 1)
    tc_gemm_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                   const TcArgs args, const Epi epi) {
  using S = TcSmem<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int stages = args.stages;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + stages * S::STAGE_BYTES);
  uint64_t* empty = full + stages;
  uint64_t* tfull = empty + stages;   // [2]
  uint64_t* tempty = tfull + 2;       // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x / 32;
  const int lane = threadIdx.x % 32;
  const int cm = args.cm, cn = args.cn, cs = cm * cn;
  const int crank = cs > 1 ? (int)sm100::cluster_ctarank() : 0;
  const int rm = crank % cm, rn = crank / cm;
  const int ncm = (args.num_m + cm - 1) / cm, ncn = (args.num_n + cn - 1) / cn;
  const int num_ct1 = ncm * ncn;                 // cluster tiles of one K chunk
  const int num_ct = num_ct1 * args.ksplit;      // × fixed K chunks (split-K)
  const int cluster_id = blockIdx.x / cs, num_clusters = gridDim.x / cs;
  const int nk_all = (args.K + TC_BK - 1) / TC_BK;
  const int kper = (nk_all + args.ksplit - 1) / args.ksplit;
  uint16_t mask_a = 0, mask_b = 0;
  for (int j = 0; j < cn; ++j) mask_a |= (uint16_t)(1u << (rm + cm * j));
  for (int i = 0; i < cm; ++i) mask_b |= (uint16_t)(1u << (i + cm * rn));
  const uint16_t mask_nb = mask_a | mask_b;

  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      sm100::mbar_init(&full[s], 1);
      sm100::mbar_init(&empty[s], cm + cn - 1);
    }
    for (int a = 0; a < 2; ++a) {
      sm100::mbar_init(&tfull[a], 1);
      sm100::mbar_init(&tempty[a], 128);
    }
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, S::TMEM_COLS);
  sm100::tc_fence_before();
  __syncthreads();
  if (cs > 1) sm100::cluster_sync();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      const uint64_t pol = sm100::l2_policy_evict_last();
      // slices this CTA loads (and multicasts) of the shared A / B tiles
      const int a_rows = TC_BM / cn, b_rows = BN / cm;       // K-major: rows of the box
      const int a_krows = TC_BK / cn, b_krows = TC_BK / cm;  // MN-major: K rows of each 64-wide box
      for (int ct = cluster_id; ct < num_ct; ct += num_clusters) {
        const int ks = ct / num_ct1, c1 = ct % num_ct1;
        const int m0 = ((c1 % ncm) * cm + rm) * TC_BM;
        const int n0 = ((c1 / ncm) * cn + rn) * BN;
        const int kb0 = ks * kper, kb1 = min(nk_all, kb0 + kper);
        for (int kb = kb0; kb < kb1; ++kb) {
          sm100::mbar_wait(&empty[s], ph ^ 1);
          uint8_t* sa = smem + s * S::STAGE_BYTES;
          uint8_t* sb = sa + S::A_BYTES;
          sm100::mbar_arrive_expect_tx(&full[s], S::STAGE_BYTES);
          const int k0 = kb * TC_BK;
          if (cs == 1) {
            if (args.a_mn) {
              sm100::tma_load_3d(sa, &mapA, &full[s], m0, k0, args.az);
              sm100::tma_load_3d(sa + 8192, &mapA, &full[s], m0 + 64, k0, args.az);
            } else {
              sm100::tma_load_3d(sa, &mapA, &full[s], k0, m0, args.az);
            }
            if (args.b_mn) {
#pragma unroll
              for (int j = 0; j < BN / 64; ++j) {
                if (args.b_keep) sm100::tma_load_3d_hint(sb + j * 8192, &mapB, &full[s], n0 + 64 * j, k0, args.bz, pol);
                else sm100::tma_load_3d(sb + j * 8192, &mapB, &full[s], n0 + 64 * j, k0, args.bz);
              }
            } else {
              if (args.b_keep) sm100::tma_load_3d_hint(sb, &mapB, &full[s], k0, n0, args.bz, pol);
              else sm100::tma_load_3d(sb, &mapB, &full[s], k0, n0, args.bz);
            }
          } else {
            if (args.a_mn) {
              for (int j = 0; j < 2; ++j)
                sm100::tma_load_3d_mc(sa + j * 8192 + rn * a_krows * 128, &mapA, &full[s], m0 + 64 * j,
                                      k0 + rn * a_krows, args.az, mask_a);
            } else {
              sm100::tma_load_3d_mc(sa + rn * a_rows * 128, &mapA, &full[s], k0, m0 + rn * a_rows, args.az, mask_a);
            }
            if (args.b_mn) {
              for (int j = 0; j < BN / 64; ++j) {
                if (args.b_keep)
                  sm100::tma_load_3d_mc_hint(sb + j * 8192 + rm * b_krows * 128, &mapB, &full[s], n0 + 64 * j,
                                             k0 + rm * b_krows, args.bz, mask_b, pol);
                else
                  sm100::tma_load_3d_mc(sb + j * 8192 + rm * b_krows * 128, &mapB, &full[s], n0 + 64 * j,
                                        k0 + rm * b_krows, args.bz, mask_b);
              }
            } else {
              if (args.b_keep)
                sm100::tma_load_3d_mc_hint(sb + rm * b_rows * 128, &mapB, &full[s], k0, n0 + rm * b_rows, args.bz,
                                           mask_b, pol);
              else
                sm100::tma_load_3d_mc(sb + rm * b_rows * 128, &mapB, &full[s], k0, n0 + rm * b_rows, args.bz, mask_b);
            }
          }
          if (++s == stages) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      int local = 0;
      for (int ct = cluster_id; ct < num_ct; ct += num_clusters, ++local) {
        const int acc = local & 1;
        const uint32_t use = (uint32_t)(local >> 1);
        sm100::mbar_wait(&tempty[acc], (use & 1) ^ 1);
        sm100::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        const int kb0 = (ct / num_ct1) * kper, kb1 = min(nk_all, kb0 + kper);
        for (int kb = kb0; kb < kb1; ++kb) {
          sm100::mbar_wait(&full[s], ph);
          sm100::tc_fence_after();
          const uint32_t sa = sm100::smem_u32(smem + s * S::STAGE_BYTES);
          const uint32_t sb = sa + S::A_BYTES;
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk) {
            const uint64_t ad = args.a_mn ? sm100::smem_desc_sw128(sa + kk * 2048, 8192, 1024)
                                          : sm100::smem_desc_sw128(sa + kk * 32, 16, 1024);
            const uint64_t bd = args.b_mn ? sm100::smem_desc_sw128(sb + kk * 2048, 8192, 1024)
                                          : sm100::smem_desc_sw128(sb + kk * 32, 16, 1024);
            sm100::umma_bf16(d_tmem, ad, bd, args.idesc, (kb != kb0 || kk != 0) ? 1u : 0u);
          }
          if (cs == 1) sm100::umma_commit(&empty[s]);
          else sm100::umma_commit_mc(&empty[s], mask_nb);
          if (++s == stages) { s = 0; ph ^= 1; }
        }
        sm100::umma_commit(&tfull[acc]);
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue warps 2..5
    const int quarter = warp & 3;           // TMEM lane quarter this warp may access
    const int row = quarter * 32 + lane;    // tile row (= TMEM lane)
    int local = 0;
    for (int ct = cluster_id; ct < num_ct; ct += num_clusters, ++local) {
      const int acc = local & 1;
      const uint32_t use = (uint32_t)(local >> 1);
      const int ks = ct / num_ct1, c1 = ct % num_ct1;
      const int m0 = ((c1 % ncm) * cm + rm) * TC_BM;
      const int n0 = ((c1 / ncm) * cn + rn) * BN;
      sm100::mbar_wait(&tfull[acc], use & 1);
      sm100::tc_fence_after();
      const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * BN;
      if (m0 < args.M && n0 < args.N && ks * kper < nk_all) epi.template run<BN>(taddr, m0, n0, row, ks);
      sm100::tc_fence_before();
      sm100::mbar_arrive(&tempty[acc]);
    }
  }
  __syncthreads();
  if (cs > 1) sm100::cluster_sync();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, S::TMEM_COLS);
  }
}

}  // namespace astra
