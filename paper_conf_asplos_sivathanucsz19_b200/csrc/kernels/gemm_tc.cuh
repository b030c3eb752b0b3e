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

#include "pdl.cuh"
#include "sm100.cuh"

namespace astra {

#ifdef ASTRA_GEMM_TRACE   // phase timestamps of CTA 0 (scratch/gemm_trace.cu)
__device__ unsigned long long g_gemm_trace[16];
__device__ __forceinline__ void gemm_trace(int i) {
  if (blockIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_gemm_trace[i] = t;
  }
}
#define GEMM_TRACE(i) gemm_trace(i)
#else
#define GEMM_TRACE(i) do {} while (0)
#endif

constexpr int TC_BM = 128;
constexpr int TC_BK = 64;          // one 128-byte swizzle atom of bf16 along K
constexpr int TC_EPI_WARPS = 4;                    // epilogue warps (one per TMEM lane quarter)
constexpr int TC_THREADS = 64 + 32 * TC_EPI_WARPS;

// Up to four global byte ranges the GEMM pulls into L2 while it runs (reading R31): the saved
// tensors the next pointwise kernel of a recurrent chain will read, so that kernel finds them in
// L2 instead of waiting on HBM latency.  A prefetch never changes any value.
struct L2Pf {
  const void* p[4];
  unsigned long long n[4];
};

struct TcArgs {
  L2Pf pf;          // L2 prefetch ranges (n = 0: none)
  int M, N, K;
  int num_m, num_n;
  int az, bz;       // third tensor-map coordinate (time slice) of A and B
  int a_mn, b_mn;   // 1 = MN-major operand
  int stages;
  int cm, cn;       // cluster shape (CTAs sharing B along M, sharing A along N)
  int b_keep;       // 1: load B with an L2 evict_last policy (weights re-read every step)
  int ksplit;       // fixed split of K into ksplit chunks; chunk ks writes its fp32 partial to C + ks·split_stride
  int cg;           // 1: one CTA per 128 x BN tile; 2: CTA pair per 256 x BN tile (tc_gemm2_kernel)
  int gm;           // raster group: tiles walk gm M-tiles of one N column before the next column
  uint32_t idesc;
  // tc_gemm_kernel without a cluster: kb k-blocks per pipeline stage, loaded by ONE tensor-map box
  // per operand (K-major: a 4-D map whose k-block dimension has a 128-byte stride; MN-major: a box
  // 64·kb K-rows tall) — a CTA's TMA unit retires ~1 box per 128 ns however small it is
  // (profiles/r2_tma_micro.jsonl), which bounds the small-M chain GEMMs; a_rows: rows of the K-major
  // A box (64 when M ≤ 64: the MMA's rows 64..127 read stale shared memory and are never stored).
  // The pair kernel (tc_gemm2) ignores both (kb = 1, a_rows = 128).
  int kb;
  int a_rows;
  // k-block order (the `alloc` fork, reading R38): 0 = ascending; P > 0 = the contraction runs over
  // 4 gate blocks of P k-blocks each (a gate-blocked K = 4·Hp, P = Hp/64) in the canonical gate-
  // interleaved order — canonical k-block c reads physical k-block (c % 4)·P + c / 4 — so the
  // accumulation order, hence every bit, is the interleaved layout's.  Needs kb = 1.
  int kperm;
};
__device__ __forceinline__ int tc_kphys(int kb, int kperm) { return kperm ? (kb & 3) * kperm + (kb >> 2) : kb; }

// One warp of every CTA issues its slice of the prefetch ranges (cp.async.bulk.prefetch.L2, 16-byte
// granules): range bytes split evenly over gridDim.x × 32 lanes.
__device__ __forceinline__ void l2_prefetch_slices(const L2Pf& pf, int lane) {
  const unsigned long long nthr = (unsigned long long)gridDim.x * 32, id = (unsigned long long)blockIdx.x * 32 + lane;
#pragma unroll
  for (int r = 0; r < 4; ++r) {
    const unsigned long long n = pf.n[r] & ~15ull;
    if (!n) continue;
    const unsigned long long piece = ((n + nthr - 1) / nthr + 255) & ~255ull;
    const unsigned long long lo = id * piece;
    if (lo >= n) continue;
    const unsigned long long sz = n - lo < piece ? n - lo : piece;
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(reinterpret_cast<uint64_t>(pf.p[r]) + lo),
                 "r"((uint32_t)sz)
                 : "memory");
  }
}

// Grouped raster of the persistent tile loop: tile c1 → (mi, ni) walking `gm` consecutive M-tiles
// down one N column, then the next column, group after group.  The CTAs resident at any time then
// share a few A row panels and the B columns stay L2-resident, instead of every N column
// re-streaming all of A from HBM.  Pure scheduling: no effect on any output bit.
__device__ __forceinline__ void tile_raster(int c1, int nm, int nn, int gm, int& mi, int& ni) {
  const int per = gm * nn;
  const int grp = c1 / per, r = c1 % per;
  const int mb = grp * gm;
  const int gs = min(gm, nm - mb);
  mi = mb + r % gs;
  ni = r / gs;
}

template <int BN>
struct TcSmem {
  static constexpr int A_BYTES = TC_BM * TC_BK * 2;   // 16 KB
  static constexpr int B_BYTES = BN * TC_BK * 2;      // BN * 128 B
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int TMEM_COLS = (2 * BN <= 32) ? 32 : (2 * BN <= 64) ? 64 : (2 * BN <= 128) ? 128 : (2 * BN <= 256) ? 256 : 512;
  // epilogue transpose tiles: one 32 x 36 fp32 tile per epilogue warp (after the barriers)
  static constexpr int EPI_TILE = 32 * 32 * 4;                  // one 32-row x 32-col fp32 tile (swizzled)
  static constexpr int EPI_BYTES = TC_EPI_WARPS * 2 * EPI_TILE;   // double-buffered per warp
  // layout: [stages][epilogue tiles (1024-aligned)][barriers 256 B]
  static int stages_for(int max_smem) {
    int s = (max_smem - 1024 - 256 - EPI_BYTES) / STAGE_BYTES;
    return s > 10 ? 10 : s;
  }
  static int bytes(int stages) { return 1024 + stages * STAGE_BYTES + EPI_BYTES + 256; }
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
  int tma;            // 1: plain stores go through the C tensor map (set by tc_gemm_launch)

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

  // Scalar store of one element (mapping, bias, bf16 and accumulate handled per element).
  __device__ __forceinline__ void store1(char* Cb, int m, int n, float v) const {
    bool ok;
    const int e = map_col(n, ok);
    if (!ok) return;
    v += bias ? bias[n] : 0.f;
    const long off = (long)m * ldc + e;
    if (out_bf16) {
      reinterpret_cast<__nv_bfloat16*>(Cb)[off] = __float2bfloat16_rn(v);
    } else {
      float* p = reinterpret_cast<float*>(Cb) + off;
      *p = accumulate ? __fadd_rn(*p, v) : v;
    }
  }

  // Epilogue of one 128 x BN accumulator tile, called by each of the 4 epilogue warps for its 32
  // TMEM lanes (tile rows quarter·32 ..+31), in 32-column chunks: tcgen05.ld (thread = row) →
  // the thread's row of a 32 x 32 fp32 shared-memory tile (dense 128-byte rows, 16-byte chunks
  // XOR-swizzled by row % 8 = the TMA SWIZZLE_128B pattern, so the 16-byte stores of 8 rows hit
  // distinct banks; two tiles per warp, alternating) → global:
  //  * tma (plain store, identity column map): one lane issues a TMA tensor store of the tile —
  //    the copy engine writes it out asynchronously and clips rows ≥ Mv / columns ≥ Nv;
  //  * otherwise (accumulate, remapped columns, bf16 via the same path): transpose through the
  //    tile and store with 16-byte vector stores, 4 full row segments per warp instruction,
  //    element stores where a 4-column group is not contiguous and aligned.
  template <int BN>
  __device__ __forceinline__ void run(uint32_t taddr, int m0, int n0, int quarter, int lane, int ks,
                                      uint32_t stile, int& nbuf, const CUtensorMap* mapC) const {
    char* Cb = reinterpret_cast<char*>(C) + (ks ? (size_t)ks * split_stride * (out_bf16 ? 2 : 4) : 0);
    const int r0 = m0 + quarter * 32;
    const int rr = lane >> 3, c4 = (lane & 7) * 4;
    const bool ld_al = ((ldc * (out_bf16 ? 2 : 4)) & 15) == 0 && (((uintptr_t)Cb) & 15) == 0;
#pragma unroll 1
    for (int c = 0; c < BN; c += 32) {
      const uint32_t tile = stile + (uint32_t)(nbuf & 1) * (32 * 32 * 4);
      const int n = n0 + c;
      float v[32];
      sm100::tmem_ld32(taddr + c, v);
      if (tma) {
        if (n >= Nv) continue;
        if (bias) {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] += (n + i < Nv) ? bias[n + i] : 0.f;
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] += 0.f;
        }
        if (lane == 0) sm100::bulk_wait_read<1>();   // the store that last read this tile is done
        __syncwarp();
        if (out_bf16) {   // 64-byte rows, SWIZZLE_64B: 16-byte chunk i of row r at i ^ ((r >> 1) & 3)
          uint32_t u[16];
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            __nv_bfloat162 b2 = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
            u[i] = *reinterpret_cast<uint32_t*>(&b2);
          }
          const uint32_t row = tile + (uint32_t)lane * 64;
#pragma unroll
          for (int i = 0; i < 4; ++i)
            sm100::sts_v4(row + (uint32_t)((i ^ ((lane >> 1) & 3)) * 16), __uint_as_float(u[4 * i]),
                          __uint_as_float(u[4 * i + 1]), __uint_as_float(u[4 * i + 2]), __uint_as_float(u[4 * i + 3]));
        } else {          // 128-byte rows, SWIZZLE_128B: chunk i of row r at i ^ (r & 7)
          const uint32_t row = tile + (uint32_t)lane * 128;
#pragma unroll
          for (int i = 0; i < 8; ++i)
            sm100::sts_v4(row + (uint32_t)((i ^ (lane & 7)) * 16), v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
        }
        sm100::fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) {
          sm100::tma_store_3d(mapC, tile, n, r0, ks);
          sm100::bulk_commit();
        }
        ++nbuf;
        continue;
      }
#pragma unroll
      for (int i = 0; i < 8; ++i)
        sm100::sts_v4(tile + (uint32_t)lane * 128 + (uint32_t)((i ^ (lane & 7)) * 16), v[4 * i], v[4 * i + 1],
                      v[4 * i + 2], v[4 * i + 3]);
      __syncwarp();
      const int nc = n + c4;
      bool ok0, ok3;
      const int e0 = map_col(nc, ok0);
      const int e3 = map_col(nc + 3, ok3);
      const bool vec = ld_al && ok0 && ok3 && e3 == e0 + 3 && (e0 & 3) == 0;
      float b4[4] = {0.f, 0.f, 0.f, 0.f};
      if (vec && bias) {
#pragma unroll
        for (int i = 0; i < 4; ++i) b4[i] = bias[nc + i];
      }
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const int row = q * 4 + rr;
        float4 w = sm100::lds_v4(tile + (uint32_t)row * 128 + (uint32_t)((((c4 >> 2) ^ (row & 7))) * 16));
        const int m = r0 + row;
        if (m >= Mv) continue;
        if (vec) {
          w.x += b4[0]; w.y += b4[1]; w.z += b4[2]; w.w += b4[3];
          const long off = (long)m * ldc + e0;
          if (out_bf16) {
            __nv_bfloat162 lo = __floats2bfloat162_rn(w.x, w.y), hi = __floats2bfloat162_rn(w.z, w.w);
            uint2 u;
            u.x = *reinterpret_cast<uint32_t*>(&lo);
            u.y = *reinterpret_cast<uint32_t*>(&hi);
            *reinterpret_cast<uint2*>(reinterpret_cast<__nv_bfloat16*>(Cb) + off) = u;
          } else {
            float4* p = reinterpret_cast<float4*>(reinterpret_cast<float*>(Cb) + off);
            if (accumulate) {
              const float4 o = *p;
              w.x = __fadd_rn(o.x, w.x); w.y = __fadd_rn(o.y, w.y); w.z = __fadd_rn(o.z, w.z); w.w = __fadd_rn(o.w, w.w);
            }
            *p = w;
          }
        } else {
          store1(Cb, m, nc, w.x);
          store1(Cb, m, nc + 1, w.y);
          store1(Cb, m, nc + 2, w.z);
          store1(Cb, m, nc + 3, w.w);
        }
      }
      __syncwarp();
      ++nbuf;
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
                   const __grid_constant__ CUtensorMap mapC, const TcArgs args, const Epi epi) {
  using S = TcSmem<BN>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  if (threadIdx.x == 0) GEMM_TRACE(0);
  const int stages = args.stages;
  const int KB = args.kb;
  // per k-block: A tile (K-major: a_rows x 128 B; MN-major: two 64-wide halves x 64 K-rows), B tile
  const int a_kb_bytes = args.a_mn ? S::A_BYTES : args.a_rows * TC_BK * 2;
  const int stage_bytes = KB * (a_kb_bytes + S::B_BYTES);
  const uint32_t epi_tiles = sm100::smem_u32(smem + stages * stage_bytes);   // 1024-aligned
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + stages * stage_bytes + S::EPI_BYTES);
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
      sm100::mbar_init(&tempty[a], 32 * TC_EPI_WARPS);
    }
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
    if (epi.tma) sm100::tma_prefetch(&mapC);
  }
  if (warp == 1) sm100::tmem_alloc(tmem_slot, S::TMEM_COLS);
  sm100::tc_fence_before();
  __syncthreads();
  if (cs > 1) sm100::cluster_sync();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  if (warp == 2) l2_prefetch_slices(args.pf, lane);   // old data only: no grid dependency needed
  pdl_wait();      // operands / outputs may belong to the previous kernel in the stream
  pdl_trigger();
  if (threadIdx.x == 0) GEMM_TRACE(1);

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    {   // whole warp: the *_warp TMA forms elect the issuing lane
      int s = 0;
      uint32_t ph = 0;
      const uint64_t pol = sm100::l2_policy_evict_last();
      // slices this CTA loads (and multicasts) of the shared A / B tiles
      const int a_rows = TC_BM / cn, b_rows = BN / cm;       // K-major: rows of the box
      const int a_krows = TC_BK / cn, b_krows = TC_BK / cm;  // MN-major: K rows of each 64-wide box
      for (int ct = cluster_id; ct < num_ct; ct += num_clusters) {
        const int ks = ct / num_ct1, c1 = ct % num_ct1;
        int mi, ni;
        tile_raster(c1, ncm, ncn, args.gm, mi, ni);
        const int m0 = (mi * cm + rm) * TC_BM;
        const int n0 = (ni * cn + rn) * BN;
        const int kb0 = ks * kper, kb1 = min(nk_all, kb0 + kper);
        for (int kb = kb0; kb < kb1; kb += KB) {
          sm100::mbar_wait(&empty[s], ph ^ 1);
          uint8_t* sa = smem + s * stage_bytes;
          uint8_t* sb = sa + KB * a_kb_bytes;
          sm100::mbar_arrive_expect_tx_warp(&full[s], stage_bytes);
          const int k0 = tc_kphys(kb, args.kperm) * TC_BK;
          if (KB > 1) {   // (cs == 1) one box per operand for the KB k-blocks of the stage
            if (args.a_mn) {
              sm100::tma_load_3d_warp(sa, &mapA, &full[s], m0, k0, args.az);
              sm100::tma_load_3d_warp(sa + KB * 8192, &mapA, &full[s], m0 + 64, k0, args.az);
            } else {
              sm100::tma_load_4d_warp(sa, &mapA, &full[s], 0, m0, kb, args.az);
            }
            if (args.b_mn) {
#pragma unroll
              for (int j = 0; j < BN / 64; ++j) {
                if (args.b_keep) sm100::tma_load_3d_hint_warp(sb + j * KB * 8192, &mapB, &full[s], n0 + 64 * j, k0, args.bz, pol);
                else sm100::tma_load_3d_warp(sb + j * KB * 8192, &mapB, &full[s], n0 + 64 * j, k0, args.bz);
              }
            } else {
              if (args.b_keep) sm100::tma_load_4d_hint_warp(sb, &mapB, &full[s], 0, n0, kb, args.bz, pol);
              else sm100::tma_load_4d_warp(sb, &mapB, &full[s], 0, n0, kb, args.bz);
            }
          } else if (cs == 1) {
            if (args.a_mn) {
              sm100::tma_load_3d_warp(sa, &mapA, &full[s], m0, k0, args.az);
              sm100::tma_load_3d_warp(sa + 8192, &mapA, &full[s], m0 + 64, k0, args.az);
            } else {
              sm100::tma_load_3d_warp(sa, &mapA, &full[s], k0, m0, args.az);
            }
            if (args.b_mn) {
#pragma unroll
              for (int j = 0; j < BN / 64; ++j) {
                if (args.b_keep) sm100::tma_load_3d_hint_warp(sb + j * 8192, &mapB, &full[s], n0 + 64 * j, k0, args.bz, pol);
                else sm100::tma_load_3d_warp(sb + j * 8192, &mapB, &full[s], n0 + 64 * j, k0, args.bz);
              }
            } else {
              if (args.b_keep) sm100::tma_load_3d_hint_warp(sb, &mapB, &full[s], k0, n0, args.bz, pol);
              else sm100::tma_load_3d_warp(sb, &mapB, &full[s], k0, n0, args.bz);
            }
          } else {
            if (args.a_mn) {
              for (int j = 0; j < 2; ++j)
                sm100::tma_load_3d_mc_warp(sa + j * 8192 + rn * a_krows * 128, &mapA, &full[s], m0 + 64 * j,
                                      k0 + rn * a_krows, args.az, mask_a);
            } else {
              sm100::tma_load_3d_mc_warp(sa + rn * a_rows * 128, &mapA, &full[s], k0, m0 + rn * a_rows, args.az, mask_a);
            }
            if (args.b_mn) {
              for (int j = 0; j < BN / 64; ++j) {
                if (args.b_keep)
                  sm100::tma_load_3d_mc_hint_warp(sb + j * 8192 + rm * b_krows * 128, &mapB, &full[s], n0 + 64 * j,
                                             k0 + rm * b_krows, args.bz, mask_b, pol);
                else
                  sm100::tma_load_3d_mc_warp(sb + j * 8192 + rm * b_krows * 128, &mapB, &full[s], n0 + 64 * j,
                                        k0 + rm * b_krows, args.bz, mask_b);
              }
            } else {
              if (args.b_keep)
                sm100::tma_load_3d_mc_hint_warp(sb + rm * b_rows * 128, &mapB, &full[s], k0, n0 + rm * b_rows, args.bz,
                                           mask_b, pol);
              else
                sm100::tma_load_3d_mc_warp(sb + rm * b_rows * 128, &mapB, &full[s], k0, n0 + rm * b_rows, args.bz, mask_b);
            }
          }
          if (++s == stages) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    {   // whole warp: umma_*_warp elect the issuing lane
      int s = 0;
      uint32_t ph = 0;
      int local = 0;
      // shared-memory descriptors of stage 0, advanced by adding (bytes >> 4) to the address field
      // (no carry: addresses < 256 KB): the single issuing thread's scalar work per k-block stays
      // far below one MMA — at the small-N per-step GEMMs it otherwise bounds the k-loop
      const uint32_t sa0 = sm100::smem_u32(smem), sb0 = sa0 + KB * a_kb_bytes;
      // MN-major: the 64-wide halves of a stage's tile are KB·8 KB apart (LBO)
      const uint64_t dA0 = args.a_mn ? sm100::smem_desc_sw128(sa0, 8192 * KB, 1024) : sm100::smem_desc_sw128(sa0, 16, 1024);
      const uint64_t dB0 = args.b_mn ? sm100::smem_desc_sw128(sb0, 8192 * KB, 1024) : sm100::smem_desc_sw128(sb0, 16, 1024);
      const uint32_t a_kk = args.a_mn ? (2048 >> 4) : (32 >> 4), b_kk = args.b_mn ? (2048 >> 4) : (32 >> 4);
      // k-block j of a stage: K-major + j tiles; MN-major + j·64 K-rows (8 KB)
      const uint32_t a_j = (uint32_t)(args.a_mn ? 8192 : a_kb_bytes) >> 4, b_j = (uint32_t)(args.b_mn ? 8192 : S::B_BYTES) >> 4;
      const uint32_t idesc = args.idesc;
      for (int ct = cluster_id; ct < num_ct; ct += num_clusters, ++local) {
        const int acc = local & 1;
        const uint32_t use = (uint32_t)(local >> 1);
        sm100::mbar_wait(&tempty[acc], (use & 1) ^ 1);
        sm100::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        const int kb0 = (ct / num_ct1) * kper, kb1 = min(nk_all, kb0 + kper);
        for (int kb = kb0; kb < kb1; kb += KB) {
          sm100::mbar_wait(&full[s], ph);
          if (kb == kb0 && local == 0) GEMM_TRACE(3);
          sm100::tc_fence_after();
          const uint64_t ad0 = dA0 + (uint64_t)(s * (stage_bytes >> 4)), bd0 = dB0 + (uint64_t)(s * (stage_bytes >> 4));
          const int nj = kb1 - kb < KB ? kb1 - kb : KB;   // a chunk's last stage may be partial
          for (int j = 0; j < nj; ++j) {
            const uint64_t ad = ad0 + j * a_j, bd = bd0 + j * b_j;
#pragma unroll
            for (int kk = 0; kk < TC_BK / 16; ++kk)
              sm100::umma_bf16_warp(d_tmem, ad + kk * a_kk, bd + kk * b_kk, idesc, (kb + j != kb0 || kk != 0) ? 1u : 0u);
          }
          if (cs == 1) sm100::umma_commit_warp(&empty[s]);
          else sm100::umma_commit_mc_warp(&empty[s], mask_nb);
          if (++s == stages) { s = 0; ph ^= 1; }
        }
        sm100::umma_commit_warp(&tfull[acc]);
        GEMM_TRACE(4);
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue warps 2..5
    const int quarter = warp & 3;           // TMEM lane quarter this warp may access
    int nbuf = 0;                           // epilogue tiles used so far (alternating buffers)
    int local = 0;
    for (int ct = cluster_id; ct < num_ct; ct += num_clusters, ++local) {
      const int acc = local & 1;
      const uint32_t use = (uint32_t)(local >> 1);
      const int ks = ct / num_ct1, c1 = ct % num_ct1;
      int mi, ni;
      tile_raster(c1, ncm, ncn, args.gm, mi, ni);
      const int m0 = (mi * cm + rm) * TC_BM;
      const int n0 = (ni * cn + rn) * BN;
      sm100::mbar_wait(&tfull[acc], use & 1);
      if (warp == 2 && lane == 0) GEMM_TRACE(5);
      sm100::tc_fence_after();
      const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * BN;
      if (m0 < args.M && n0 < args.N && ks * kper < nk_all) epi.template run<BN>(taddr, m0, n0, quarter, lane, ks, epi_tiles + (uint32_t)(warp - 2) * 2 * S::EPI_TILE, nbuf,
                                                                                   &mapC);
      sm100::tc_fence_before();
      if (warp == 2 && lane == 0) GEMM_TRACE(6);
      sm100::mbar_arrive(&tempty[acc]);
    }
    sm100::bulk_wait_read<0>();   // the copy engine has read this thread's staged tiles
  }
  __syncthreads();
  if (cs > 1) sm100::cluster_sync();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tmem_base, S::TMEM_COLS);
  }
  if (threadIdx.x == 0) GEMM_TRACE(7);
}

// CTA-pair variant (cta_group::2).  A cluster of 2 CTAs on one TPC owns a 256 x BN output tile:
// CTA r holds rows 128r..128r+127 of A and columns r·BN/2 .. of B in its shared memory, the pair
// leader (rank 0) issues one M = 256 MMA per K16 that reads both halves, and each CTA's TMEM
// receives its own 128 rows x BN accumulator.  Every operand byte therefore crosses L2 → SM once
// per pair instead of once per CTA for B, cutting the per-SM operand traffic of a 128 x BN tile
// from (128 + BN)·K to (128 + BN/2)·K elements — the bound of the small-M per-step GEMMs.
// Barriers: both CTAs' TMA loads signal the leader's `full` barrier (the leader expects the
// pair's bytes); the leader's MMA commit arrives on `empty` and `tfull` of both CTAs (multicast);
// each CTA's 4 epilogue warps arrive on the leader's `tempty`.  Accumulation order per output
// element is unchanged (ascending K, one chain per element, split-K chunks as in tc_gemm_kernel),
// so results are bitwise identical to the single-CTA kernel.
template <int BN, class Epi>
__global__ void __launch_bounds__(TC_THREADS, 1)
    tc_gemm2_kernel(const __grid_constant__ CUtensorMap mapA, const __grid_constant__ CUtensorMap mapB,
                    const __grid_constant__ CUtensorMap mapC, const TcArgs args, const Epi epi) {
  constexpr int BH = BN / 2;          // B columns held by each CTA
  using S = TcSmem<BH>;
  constexpr int TMEM_COLS = 2 * BN <= 256 ? 256 : 512;   // two accumulator buffers of BN columns (power of 2)
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int stages = args.stages;
  const uint32_t epi_tiles = sm100::smem_u32(smem + stages * S::STAGE_BYTES);   // 1024-aligned
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + stages * S::STAGE_BYTES + S::EPI_BYTES);
  uint64_t* empty = full + stages;
  uint64_t* tfull = empty + stages;   // [2]
  uint64_t* tempty = tfull + 2;       // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x / 32;
  const int lane = threadIdx.x % 32;
  const int rank = (int)sm100::cluster_ctarank();
  const int num_mp = (args.M + 2 * TC_BM - 1) / (2 * TC_BM);
  const int num_pt1 = num_mp * args.num_n;
  const int num_pt = num_pt1 * args.ksplit;
  const int pair_id = blockIdx.x / 2, num_pairs = gridDim.x / 2;
  const int nk_all = (args.K + TC_BK - 1) / TC_BK;
  const int kper = (nk_all + args.ksplit - 1) / args.ksplit;

  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      sm100::mbar_init(&full[s], 1);
      sm100::mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      sm100::mbar_init(&tfull[a], 1);
      sm100::mbar_init(&tempty[a], 2 * TC_EPI_WARPS);
    }
    sm100::fence_barrier_init();
  }
  if (warp == 0 && lane == 0) {
    sm100::tma_prefetch(&mapA);
    sm100::tma_prefetch(&mapB);
    if (epi.tma) sm100::tma_prefetch(&mapC);
  }
  if (warp == 1) sm100::tmem_alloc_cg2(tmem_slot, TMEM_COLS);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::cluster_sync();
  sm100::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  if (warp == 2) l2_prefetch_slices(args.pf, lane);   // old data only: no grid dependency needed

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer (both CTAs)
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0;
      const uint64_t pol = sm100::l2_policy_evict_last();
      auto load_b = [&](uint8_t* sb, uint32_t bar, int n0, int k0) {
        if (args.b_mn) {
#pragma unroll
          for (int j = 0; j < BH / 64; ++j) {
            if (args.b_keep) sm100::tma_load_3d_cg2_hint(sb + j * 8192, &mapB, bar, n0 + 64 * j, k0, args.bz, pol);
            else sm100::tma_load_3d_cg2(sb + j * 8192, &mapB, bar, n0 + 64 * j, k0, args.bz);
          }
        } else {
          if (args.b_keep) sm100::tma_load_3d_cg2_hint(sb, &mapB, bar, k0, n0, args.bz, pol);
          else sm100::tma_load_3d_cg2(sb, &mapB, bar, k0, n0, args.bz);
        }
      };
      // A weight operand (b_keep: written long before this launch — every kernel of the chain waits
      // on its predecessor before triggering its successor, so kernels two launches back are
      // complete) is fetched for the first stages before the grid dependency resolves; the
      // activations (A) and all outputs wait for it.
      int pre = 0;
      if (args.b_keep && pair_id < num_pt) {
        const int ks = pair_id / num_pt1, c1 = pair_id % num_pt1;
        int mi, ni;
        tile_raster(c1, num_mp, args.num_n, args.gm, mi, ni);
        const int kb0 = ks * kper, kb1 = min(nk_all, kb0 + kper);
        pre = min(stages, max(0, kb1 - kb0));
        for (int i = 0; i < pre; ++i) {
          uint8_t* sa = smem + i * S::STAGE_BYTES;
          if (rank == 0) sm100::mbar_arrive_expect_tx(&full[i], 2 * S::STAGE_BYTES);
          load_b(sa + S::A_BYTES, sm100::mapa_shared(sm100::smem_u32(&full[i]), 0), ni * BN + rank * BH,
                 tc_kphys(kb0 + i, args.kperm) * TC_BK);
        }
      }
      pdl_wait();
      pdl_trigger();
      int issued = 0;
      for (int ct = pair_id; ct < num_pt; ct += num_pairs) {
        const int ks = ct / num_pt1, c1 = ct % num_pt1;
        int mi, ni;
        tile_raster(c1, num_mp, args.num_n, args.gm, mi, ni);
        const int m0 = mi * 2 * TC_BM + rank * TC_BM;
        const int n0 = ni * BN + rank * BH;
        const int kb0 = ks * kper, kb1 = min(nk_all, kb0 + kper);
        for (int kb = kb0; kb < kb1; ++kb, ++issued) {
          const bool early = issued < pre;          // B of this stage already in flight
          if (!early) sm100::mbar_wait(&empty[s], ph ^ 1);
          uint8_t* sa = smem + s * S::STAGE_BYTES;
          uint8_t* sb = sa + S::A_BYTES;
          if (!early && rank == 0) sm100::mbar_arrive_expect_tx(&full[s], 2 * S::STAGE_BYTES);
          const uint32_t bar = sm100::mapa_shared(sm100::smem_u32(&full[s]), 0);
          const int k0 = tc_kphys(kb, args.kperm) * TC_BK;
          if (args.a_mn) {
            sm100::tma_load_3d_cg2(sa, &mapA, bar, m0, k0, args.az);
            sm100::tma_load_3d_cg2(sa + 8192, &mapA, bar, m0 + 64, k0, args.az);
          } else {
            sm100::tma_load_3d_cg2(sa, &mapA, bar, k0, m0, args.az);
          }
          if (!early) load_b(sb, bar, n0, k0);
          if (++s == stages) { s = 0; ph ^= 1; }
        }
      }
    } else {
      pdl_wait();
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer (pair leader only)
    pdl_wait();
    if (rank == 0) {   // whole warp: umma_*_warp elect the issuing lane
      int s = 0;
      uint32_t ph = 0;
      int local = 0;
      const uint32_t sa0 = sm100::smem_u32(smem), sb0 = sa0 + S::A_BYTES;   // (see tc_gemm_kernel)
      const uint64_t dA0 = args.a_mn ? sm100::smem_desc_sw128(sa0, 8192, 1024) : sm100::smem_desc_sw128(sa0, 16, 1024);
      const uint64_t dB0 = args.b_mn ? sm100::smem_desc_sw128(sb0, 8192, 1024) : sm100::smem_desc_sw128(sb0, 16, 1024);
      const uint32_t a_kk = args.a_mn ? (2048 >> 4) : (32 >> 4), b_kk = args.b_mn ? (2048 >> 4) : (32 >> 4);
      const uint32_t idesc = args.idesc;
      for (int ct = pair_id; ct < num_pt; ct += num_pairs, ++local) {
        const int acc = local & 1;
        const uint32_t use = (uint32_t)(local >> 1);
        sm100::mbar_wait(&tempty[acc], (use & 1) ^ 1);
        sm100::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        const int kb0 = (ct / num_pt1) * kper, kb1 = min(nk_all, kb0 + kper);
        for (int kb = kb0; kb < kb1; ++kb) {
          sm100::mbar_wait(&full[s], ph);
          sm100::tc_fence_after();
          const uint64_t ad = dA0 + (uint64_t)(s * (S::STAGE_BYTES >> 4)), bd = dB0 + (uint64_t)(s * (S::STAGE_BYTES >> 4));
#pragma unroll
          for (int kk = 0; kk < TC_BK / 16; ++kk)
            sm100::umma_bf16_cg2_warp(d_tmem, ad + kk * a_kk, bd + kk * b_kk, idesc, (kb != kb0 || kk != 0) ? 1u : 0u);
          sm100::umma_commit_cg2_mc_warp(&empty[s], 0x3);
          if (++s == stages) { s = 0; ph ^= 1; }
        }
        sm100::umma_commit_cg2_mc_warp(&tfull[acc], 0x3);
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue warps 2..5 (both CTAs)
    pdl_wait();
    const int quarter = warp & 3;
    int nbuf = 0;
    const uint32_t tempty_cl[2] = {sm100::mapa_shared(sm100::smem_u32(&tempty[0]), 0),
                                   sm100::mapa_shared(sm100::smem_u32(&tempty[1]), 0)};
    int local = 0;
    for (int ct = pair_id; ct < num_pt; ct += num_pairs, ++local) {
      const int acc = local & 1;
      const uint32_t use = (uint32_t)(local >> 1);
      const int ks = ct / num_pt1, c1 = ct % num_pt1;
      int mi, ni;
      tile_raster(c1, num_mp, args.num_n, args.gm, mi, ni);
      const int m0 = mi * 2 * TC_BM + rank * TC_BM;
      const int n0 = ni * BN;
      sm100::mbar_wait(&tfull[acc], use & 1);
      sm100::tc_fence_after();
      const uint32_t taddr = tmem_base + ((uint32_t)(quarter * 32) << 16) + acc * BN;
      if (m0 < args.M && n0 < args.N && ks * kper < nk_all) epi.template run<BN>(taddr, m0, n0, quarter, lane, ks, epi_tiles + (uint32_t)(warp - 2) * 2 * S::EPI_TILE, nbuf,
                                                                                   &mapC);
      sm100::tc_fence_before();
      __syncwarp();
      if (lane == 0) sm100::mbar_arrive_cluster(tempty_cl[acc]);
    }
    sm100::bulk_wait_read<0>();
  }
  __syncthreads();
  sm100::cluster_sync();
  if (warp == 1) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc_cg2(tmem_base, TMEM_COLS);
  }
}

}  // namespace astra
