// Day-1 microbenchmarks of SURVEY §8(d.4b): the floors of the latency-bound recurrent chains that
// neither MEASURED_PEAKS.json nor the paper gives (§8(d.3) "chain latency ... against a measured
// floor (an empty grid-barrier step plus the weight-stream time)").
//   - streaming read of a buffer over `passes` passes: L2-resident vs HBM bandwidth by size (the
//     per-step weight-stream time of U / R_ℓ);
//   - a persistent one-CTA-per-SM kernel doing `iters` grid-wide flag barriers (the step floor of a
//     persistent fused chain);
//   - a chain of `n` dependent empty kernels launched as the library launches its chain kernels
//     (with programmatic dependent launch, or without) — the step floor of a launched chain.
#include <cuda.h>

#include "../common.h"
#include "gemm.h"
#include "sm100.cuh"
#include "pdl.cuh"
#include "peer.h"

namespace astra {

namespace {

__global__ void __launch_bounds__(512) stream_read_kernel(const float4* __restrict__ p, size_t n4, int passes,
                                                          float* sink) {
  float acc = 0.f;
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  for (int r = 0; r < passes; ++r)
    for (size_t i = tid; i < n4; i += nth) {
      const float4 v = __ldcg(p + i);
      acc += v.x + v.y + v.z + v.w;
    }
  if (acc == 1.2345e-30f) *sink = acc;   // keeps the loads; never true for the benchmark's data
}

__device__ __forceinline__ void red_release_gpu(unsigned* p, unsigned v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// counter[0] is zeroed by the host; barrier k completes when it reaches (k + 1) · gridDim.x
__global__ void grid_barrier_kernel(unsigned* counter, int iters) {
  for (int k = 0; k < iters; ++k) {
    __syncthreads();
    if (threadIdx.x == 0) {
      red_release_gpu(counter, 1u);
      const unsigned target = (unsigned)(k + 1) * gridDim.x;
      while (ld_acquire_gpu(counter) < target) {
      }
    }
    __syncthreads();
  }
}

// TMA read throughput per SM: one thread streams `nbox` boxes {64 elements, box_rows} of a bf16
// [rows][64·kb] tensor through a `stages`-deep shared-memory ring (consumed by a second thread that
// only waits and releases).  same = 1: every CTA reads the same boxes in the same order (the
// broadcast pattern of a recurrent chain's h operand); 0: each CTA its own rows.
__global__ void __launch_bounds__(64, 1) tma_read_kernel(const __grid_constant__ CUtensorMap m, int nbox, int box_rows,
                                                         int stages, int kb, int row_blocks, int same) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int box_bytes = box_rows * 128;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + stages * box_bytes);
  uint64_t* empty = full + stages;
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      sm100::mbar_init(&full[s], 1);
      sm100::mbar_init(&empty[s], 1);
    }
    sm100::fence_barrier_init();
  }
  __syncthreads();
  const int rb0 = (same & 1) ? 0 : (int)blockIdx.x % row_blocks;
  if ((same & 2) && threadIdx.x < 32) {   // whole-warp issue (tma_load_3d_warp)
    int s = 0, k = 0, rb = rb0;
    uint32_t ph = 0;
    for (int i = 0; i < nbox; ++i) {
      sm100::mbar_wait(&empty[s], ph ^ 1);
      sm100::mbar_arrive_expect_tx_warp(&full[s], (uint32_t)box_bytes);
      sm100::tma_load_3d_warp(smem + s * box_bytes, &m, &full[s], k * 64, rb * box_rows, 0);
      if (++s == stages) { s = 0; ph ^= 1; }
      if (++k == kb) { k = 0; if (++rb == row_blocks) rb = 0; }
    }
  } else if (!(same & 2) && threadIdx.x == 0) {
    int s = 0, k = 0, rb = rb0;
    uint32_t ph = 0;
    for (int i = 0; i < nbox; ++i) {
      sm100::mbar_wait(&empty[s], ph ^ 1);
      sm100::mbar_arrive_expect_tx(&full[s], (uint32_t)box_bytes);
      sm100::tma_load_3d(smem + s * box_bytes, &m, &full[s], k * 64, rb * box_rows, 0);
      if (++s == stages) { s = 0; ph ^= 1; }
      if (++k == kb) { k = 0; if (++rb == row_blocks) rb = 0; }
    }
  } else if (threadIdx.x == 32) {
    int s = 0;
    uint32_t ph = 0;
    for (int i = 0; i < nbox; ++i) {
      sm100::mbar_wait(&full[s], ph);
      sm100::mbar_arrive(&empty[s]);
      if (++s == stages) { s = 0; ph ^= 1; }
    }
  }
  __syncthreads();
}

// One tcgen05.mma chain per CTA: `iters` dependent MMAs (M x N x 16, bf16, both operands K-major
// SWIZZLE_128B in shared memory, the 4 K-steps of one 64-wide k-block in turn) — the per-MMA issue
// time of the small-batch chains as a function of M and N.  A[m][k] = ((3m + k) mod 7 − 3)/4,
// B[n][k] = ((5n + 2k) mod 5 − 2)/2 (exact in bf16).  cycles[cta] = clock64 from the first issue to
// the commit's mbarrier completing; with iters == 1 CTA 0 dumps all 128 TMEM lanes × N columns to
// dump[lane][col] (the accumulator layout for M = 64).
__global__ void __launch_bounds__(128, 1) mma_chain_kernel(int M, int N, int iters, int mode, uint32_t idesc,
                                                           long long* __restrict__ cycles, float* __restrict__ dump) {
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char* sm = (unsigned char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  unsigned char* sA = sm;               // 128 rows x 128 B
  unsigned char* sB = sm + 128 * 128;   // 256 rows x 128 B
  __shared__ uint64_t bar, done, cbar;
  __shared__ uint32_t tbase;
  const int tid = threadIdx.x;
  for (int i = tid; i < (128 + 256) * 64; i += blockDim.x) {
    const bool isA = i < 128 * 64;
    const int j = isA ? i : i - 128 * 64, r = j / 64, k = j % 64;
    const float v = isA ? (float)(((3 * r + k) % 7) - 3) * 0.25f : (float)(((5 * r + 2 * k) % 5) - 2) * 0.5f;
    unsigned char* base = isA ? sA : sB;
    const int chunk = (k / 8) ^ (r % 8);
    __nv_bfloat16* dst = (__nv_bfloat16*)(base + (r / 8) * 1024 + (r % 8) * 128 + chunk * 16) + (k % 8);
    *dst = __float2bfloat16_rn(v);
  }
  if (tid == 0) {
    sm100::mbar_init(&bar, 1);
    sm100::mbar_init(&done, 1);
    sm100::mbar_init(&cbar, (iters + 3) / 4);
    sm100::fence_barrier_init();
    sm100::mbar_arrive(&done);   // phase 0 complete: a wait on it returns at once (a k loop's landed stage)
  }
  if (tid < 32) sm100::tmem_alloc(&tbase, 256);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tmem = tbase;
  if ((mode & 8) && tid < 32) {   // whole-warp issue (umma_bf16_warp)
    const uint64_t a0 = sm100::smem_desc_sw128(sm100::smem_u32(sA), 16, 1024);
    const uint64_t b0 = sm100::smem_desc_sw128(sm100::smem_u32(sB), 16, 1024);
    const long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      if ((i & 3) == 0) {
        if (mode & 1) sm100::mbar_wait(&done, 0);
        if (mode & 2) sm100::tc_fence_after();
      }
      const uint64_t kk = (uint64_t)(i & 3) * 2;
      sm100::umma_bf16_warp(tmem, a0 + kk, b0 + kk, idesc, i > 0 ? 1u : 0u);
      if ((mode & 4) && (i & 3) == 3) sm100::umma_commit_warp(&cbar);
    }
    sm100::umma_commit_warp(&bar);
    sm100::mbar_wait(&bar, 0);
    const long long t1 = clock64();
    if (tid == 0) cycles[blockIdx.x] = t1 - t0;
  } else if (!(mode & 8) && tid == 0) {
    const uint64_t a0 = sm100::smem_desc_sw128(sm100::smem_u32(sA), 16, 1024);
    const uint64_t b0 = sm100::smem_desc_sw128(sm100::smem_u32(sB), 16, 1024);
    const long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      // mode bits, per k-block of 4 MMAs, as a k loop does: 1 = mbarrier wait (on a completed phase),
      // 2 = tcgen05.fence::after_thread_sync, 4 = tcgen05.commit to an mbarrier after the 4 MMAs
      if ((i & 3) == 0) {
        if (mode & 1) sm100::mbar_wait(&done, 0);
        if (mode & 2) sm100::tc_fence_after();
      }
      const uint64_t kk = (uint64_t)(i & 3) * 2;   // 32 B per K-step of 16 bf16
      sm100::umma_bf16(tmem, a0 + kk, b0 + kk, idesc, i > 0 ? 1u : 0u);
      if ((mode & 4) && (i & 3) == 3) sm100::umma_commit(&cbar);
    }
    sm100::umma_commit(&bar);
    sm100::mbar_wait(&bar, 0);
    const long long t1 = clock64();
    cycles[blockIdx.x] = t1 - t0;
  }
  __syncthreads();
  sm100::tc_fence_after();
  if (dump && blockIdx.x == 0) {
    const int w = tid / 32;
    for (int c0 = 0; c0 < N; c0 += 16) {
      float v[16];
      sm100::tmem_ld16(tmem + ((uint32_t)(w * 32) << 16) + c0, v);
      for (int j = 0; j < 16; ++j) dump[(long)tid * N + c0 + j] = v[j];
    }
  }
  sm100::tc_fence_before();
  __syncthreads();
  if (tid < 32) sm100::tmem_dealloc(tmem, 256);
}

__global__ void empty_pdl_kernel(int) {
  pdl_wait();
  pdl_trigger();
}

__global__ void empty_kernel(int) {}

}  // namespace

void micro_stream_read(const void* buf, size_t bytes, int passes, float* sink, cudaStream_t st) {
  const size_t n4 = bytes / 16;
  ASTRA_CHECK_ARG(buf && n4 > 0 && passes > 0 && sink, "micro_stream_read: bad arguments");
  stream_read_kernel<<<num_sms() * 4, 512, 0, st>>>(reinterpret_cast<const float4*>(buf), n4, passes, sink);
  LAUNCH_CHECK();
}

void micro_grid_barrier(unsigned* counter, int iters, cudaStream_t st) {
  ASTRA_CHECK_ARG(counter && iters > 0, "micro_grid_barrier: bad arguments");
  CUDA_TRY(cudaMemsetAsync(counter, 0, sizeof(unsigned), st));
  grid_barrier_kernel<<<num_sms(), 128, 0, st>>>(counter, iters);   // one CTA per SM: all co-resident
  LAUNCH_CHECK();
}

void micro_tma_read(const void* buf, long rows, int kb, int box_rows, int ctas, int stages, int nbox, int same,
                    cudaStream_t st) {
  ASTRA_CHECK_ARG(buf && rows >= box_rows && kb > 0 && ctas > 0 && stages >= 1 && nbox > 0 && box_rows >= 8 &&
                      box_rows <= 256 && box_rows % 8 == 0, "micro_tma_read: bad arguments");
  CUtensorMap m;
  make_tile_map(&m, buf, true, (long)kb * 64, rows, 1, (long)kb * 64, 0, 64, box_rows, 128);
  const int smem = 1024 + stages * box_rows * 128 + stages * 16;
  CUDA_TRY(cudaFuncSetAttribute(tma_read_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  tma_read_kernel<<<ctas, 64, smem, st>>>(m, nbox, box_rows, stages, kb, (int)(rows / box_rows), same);
  LAUNCH_CHECK();
}

void micro_mma_chain(int M, int N, int iters, int ctas, int mode, long long* cycles, float* dump, cudaStream_t st) {
  ASTRA_CHECK_ARG((M == 64 || M == 128) && N >= 16 && N <= 256 && N % 16 == 0 && iters >= 1 && ctas >= 1 && cycles,
                  "micro_mma_chain: bad arguments");
  uint32_t d = 0;
  d |= 1u << 4;                     // D F32
  d |= 1u << 7;                     // A BF16
  d |= 1u << 10;                    // B BF16
  d |= (uint32_t)(N >> 3) << 17;    // N >> 3
  d |= (uint32_t)(M >> 4) << 24;    // M >> 4
  const int smem = 1024 + (128 + 256) * 128;
  CUDA_TRY(cudaFuncSetAttribute(mma_chain_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  mma_chain_kernel<<<ctas, 128, smem, st>>>(M, N, iters, mode, d, cycles, dump);
  LAUNCH_CHECK();
}

void micro_launch_chain(int n, int pdl, int blocks, cudaStream_t st) {
  ASTRA_CHECK_ARG(n > 0 && blocks > 0, "micro_launch_chain: bad arguments");
  for (int i = 0; i < n; ++i) {
    if (pdl) launch_pdl(empty_pdl_kernel, dim3(blocks), dim3(128), 0, st, 1, i);
    else empty_kernel<<<blocks, 128, 0, st>>>(i);
    LAUNCH_CHECK();
  }
}

}  // namespace astra

// K11p's reduce kernel with `world` ranks simulated on one device: rank r's launch on streams[r]
// reads shard r of every rank's buffer (all local HBM here) and writes the rank-ordered mean into
// buffer r — the production kernel and barrier protocol, without NVLink.  Measures the kernel's
// own efficiency against the HBM roofline (the NVLink-bound case needs a multi-GPU box).
namespace astra {
void micro_peer_reduce(float* const* bufs, uint32_t* const* sigs, int world, size_t n, int reps, uint32_t seq0,
                       const cudaStream_t* streams) {
  ASTRA_CHECK_ARG(bufs && sigs && streams && world >= 1 && world <= PEER_MAX_WORLD && n > 0 && reps > 0,
                  "micro_peer_reduce: bad arguments");
  PeerPtrs a{};
  a.world = world;
  for (int q = 0; q < world; ++q) {
    a.g[q] = bufs[q];
    a.p[q] = bufs[q];
    a.sig[q] = sigs[q];
  }
  for (int it = 0; it < reps; ++it)
    for (int r = 0; r < world; ++r) {
      a.rank = r;
      size_t lo, hi;
      peer_shard(0, n, r, world, &lo, &hi);
      peer_reduce(a, lo, hi, seq0 + (uint32_t)it, 1.0f / (float)world, 32, 60LL * 1000 * 1000 * 1000, streams[r]);
    }
}

}  // namespace astra
