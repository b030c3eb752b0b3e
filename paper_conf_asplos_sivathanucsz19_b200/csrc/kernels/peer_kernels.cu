// K11p kernels: rank-ordered reduce-scatter of gradient buckets over NVLink peer memory and the
// fused SGD + parameter all-gather (SURVEY §8(e) backend 2; the semantics g = (1/N)·Σ_r g_r of
// §8(c.3) item 8).  See peer.h for the protocol.
#include "../common.h"
#include "peer.h"

namespace astra {

namespace {

__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t global_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Flag barrier across ranks for this CTA: publish `seq` into slot [blockIdx.x][rank] of every
// rank's signal array, then wait until every rank has published ≥ seq into ours.  The CTA's
// earlier global stores (local or remote) are ordered before the flag by the CTA barrier and the
// system-scope fence (cumulativity); the acquire orders the CTA's later loads after the peers'.
__device__ __forceinline__ void peer_barrier(const PeerPtrs& a, uint32_t seq, long long timeout_ns) {
  __syncthreads();
  const int q = threadIdx.x;
  if (q < a.world) {
    const int slot = blockIdx.x * PEER_MAX_WORLD;
    __threadfence_system();
    st_release_sys(a.sig[q] + slot + a.rank, seq);
    const uint32_t* mine = a.sig[a.rank] + slot + q;
    const uint64_t t0 = global_ns();
    while ((int32_t)(ld_acquire_sys(mine) - seq) < 0) {
      if ((long long)(global_ns() - t0) > timeout_ns) __trap();   // a peer never arrived
      __nanosleep(100);
    }
  }
  __syncthreads();
}

template <int W>
__device__ __forceinline__ float4 rank_sum4(const PeerPtrs& a, size_t i4, float scale) {
  float4 v[W];
#pragma unroll
  for (int q = 0; q < W; ++q) v[q] = reinterpret_cast<const float4*>(a.g[q])[i4];
  float4 s = v[0];
#pragma unroll
  for (int q = 1; q < W; ++q) {   // rank order 0..N-1: the canonical summation (§8(e))
    s.x = __fadd_rn(s.x, v[q].x);
    s.y = __fadd_rn(s.y, v[q].y);
    s.z = __fadd_rn(s.z, v[q].z);
    s.w = __fadd_rn(s.w, v[q].w);
  }
  s.x = __fmul_rn(s.x, scale);
  s.y = __fmul_rn(s.y, scale);
  s.z = __fmul_rn(s.z, scale);
  s.w = __fmul_rn(s.w, scale);
  return s;
}

template <int W>
__device__ __forceinline__ float rank_sum1(const PeerPtrs& a, size_t i, float scale) {
  float s = a.g[0][i];
#pragma unroll
  for (int q = 1; q < W; ++q) s = __fadd_rn(s, a.g[q][i]);
  return __fmul_rn(s, scale);
}

template <int W>
__global__ void __launch_bounds__(512) peer_reduce_kernel(PeerPtrs a, size_t lo, size_t hi, uint32_t seq,
                                                           float scale, long long timeout_ns) {
  peer_barrier(a, seq, timeout_ns);   // every rank has produced this bucket
  const size_t lo4 = (lo + 3) / 4, hi4 = hi / 4 > lo4 ? hi / 4 : lo4;   // float4 body [4·lo4, 4·hi4)
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  float4* out = reinterpret_cast<float4*>(a.g[a.rank]);
  for (size_t i = lo4 + tid; i < hi4; i += nth) out[i] = rank_sum4<W>(a, i, scale);
  if (blockIdx.x == 0) {   // unaligned ends of the shard
    const size_t b0 = 4 * lo4 < hi ? 4 * lo4 : hi, b1 = 4 * hi4 > lo ? 4 * hi4 : lo;
    for (size_t i = lo + threadIdx.x; i < b0; i += blockDim.x) a.g[a.rank][i] = rank_sum1<W>(a, i, scale);
    for (size_t i = (b1 > b0 ? b1 : b0) + threadIdx.x; i < hi; i += blockDim.x)
      a.g[a.rank][i] = rank_sum1<W>(a, i, scale);
  }
  // no closing barrier: a peer reads only its own shard of our gradients, which we never write;
  // our gradients are next overwritten after the SGD kernel's entry barrier (stream order)
}

__device__ __forceinline__ float sgd1(float p, float g, float lr) { return __fsub_rn(p, __fmul_rn(lr, g)); }

template <int W>
__global__ void __launch_bounds__(512) peer_sgd_kernel(PeerPtrs a, PeerSegs s, float lr, uint32_t seq,
                                                        long long timeout_ns) {
  peer_barrier(a, seq, timeout_ns);   // every rank finished the step: parameters may be rewritten
  const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x, nth = (size_t)gridDim.x * blockDim.x;
  const float* gl = a.g[a.rank];
  const float* pl = a.p[a.rank];
  for (int k = 0; k < s.n; ++k) {
    const size_t lo = s.lo[k], hi = s.hi[k];
    const size_t lo4 = (lo + 3) / 4, hi4 = hi / 4 > lo4 ? hi / 4 : lo4;
    for (size_t i = lo4 + tid; i < hi4; i += nth) {
      float4 p = reinterpret_cast<const float4*>(pl)[i];
      const float4 g = reinterpret_cast<const float4*>(gl)[i];
      p.x = sgd1(p.x, g.x, lr);
      p.y = sgd1(p.y, g.y, lr);
      p.z = sgd1(p.z, g.z, lr);
      p.w = sgd1(p.w, g.w, lr);
#pragma unroll
      for (int q = 0; q < W; ++q) reinterpret_cast<float4*>(a.p[q])[i] = p;   // all-gather
    }
    if (blockIdx.x == 0) {
      const size_t b0 = 4 * lo4 < hi ? 4 * lo4 : hi, b1 = 4 * hi4 > lo ? 4 * hi4 : lo;
      auto one = [&](size_t i) {
        const float v = sgd1(pl[i], gl[i], lr);
#pragma unroll
        for (int q = 0; q < W; ++q) a.p[q][i] = v;
      };
      for (size_t i = lo + threadIdx.x; i < b0; i += blockDim.x) one(i);
      for (size_t i = (b1 > b0 ? b1 : b0) + threadIdx.x; i < hi; i += blockDim.x) one(i);
    }
  }
  peer_barrier(a, seq + 1, timeout_ns);   // every rank's stores into our window have landed
}

}  // namespace

void peer_shard(size_t off, size_t n, int r, int world, size_t* lo, size_t* hi) {
  auto bound = [&](int k) -> size_t {
    if (k <= 0) return off;
    if (k >= world) return off + n;
    size_t b = (off + (size_t)((unsigned __int128)n * k / world) + 3) / 4 * 4;
    return b < off ? off : (b > off + n ? off + n : b);
  };
  *lo = bound(r);
  *hi = bound(r + 1);
}

#define PEER_SWITCH(W, ...)                                  \
  switch (W) {                                               \
    case 1: { constexpr int WW = 1; __VA_ARGS__; } break;    \
    case 2: { constexpr int WW = 2; __VA_ARGS__; } break;    \
    case 3: { constexpr int WW = 3; __VA_ARGS__; } break;    \
    case 4: { constexpr int WW = 4; __VA_ARGS__; } break;    \
    case 5: { constexpr int WW = 5; __VA_ARGS__; } break;    \
    case 6: { constexpr int WW = 6; __VA_ARGS__; } break;    \
    case 7: { constexpr int WW = 7; __VA_ARGS__; } break;    \
    case 8: { constexpr int WW = 8; __VA_ARGS__; } break;    \
    default: throw Error(ASTRA_E_ARG, "peer: world must be in [1, 8]"); \
  }

void peer_reduce(const PeerPtrs& a, size_t lo, size_t hi, uint32_t seq, float scale, int blocks,
                 long long timeout_ns, cudaStream_t st) {
  ASTRA_CHECK_ARG(blocks >= 1 && blocks <= PEER_MAX_BLOCKS, "peer_reduce: bad block count");
  PEER_SWITCH(a.world, peer_reduce_kernel<WW><<<blocks, 512, 0, st>>>(a, lo, hi, seq, scale, timeout_ns));
  LAUNCH_CHECK();
}

void peer_sgd(const PeerPtrs& a, const PeerSegs& s, float lr, uint32_t seq, int blocks, long long timeout_ns,
              cudaStream_t st) {
  ASTRA_CHECK_ARG(blocks >= 1 && blocks <= PEER_MAX_BLOCKS, "peer_sgd: bad block count");
  PEER_SWITCH(a.world, peer_sgd_kernel<WW><<<blocks, 512, 0, st>>>(a, s, lr, seq, timeout_ns));
  LAUNCH_CHECK();
}

}  // namespace astra
