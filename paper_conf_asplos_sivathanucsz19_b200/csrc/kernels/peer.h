// K11p: deterministic data-parallel gradient sum over NVLink peer memory (backend 2).
//
// Every rank maps the parameter / gradient window and the signal array of every other rank (CUDA
// IPC).  A bucket [off, off + n) of the flat fp32 gradient vector is split into `world` contiguous
// shards; rank r owns shard r.  Two kernels per step:
//   peer_reduce  (per bucket, comm stream): rank r reads shard r of every rank's gradients over
//                NVLink and writes g = (g_0 + g_1 + ... + g_{N-1}) · (1/N) — summed in rank order
//                0..N-1, so the result is bitwise independent of bucket boundaries, NCCL algorithm
//                and timing — into its own gradient shard;
//   peer_sgd     (once per step, main stream): θ ← θ − lr·g on every owned shard (the same rounded
//                operations as the single-GPU SGD kernel), stored into every rank's parameter
//                window (the all-gather of the updated master weights).
// Ordering between ranks is a flag barrier in the signal arrays (per-CTA slots, release/acquire at
// system scope, monotonically increasing sequence numbers).  A barrier that waits longer than the
// timeout traps (sticky CUDA error → ASTRA_E_CUDA), it never hangs the device.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

namespace astra {

constexpr int PEER_MAX_WORLD = 8;
constexpr int PEER_MAX_BLOCKS = 128;     // signal slots per rank: [block][source rank]
constexpr int PEER_MAX_SEGS = 64;        // owned shards per SGD launch
constexpr size_t PEER_SIG_BYTES = (size_t)PEER_MAX_BLOCKS * PEER_MAX_WORLD * sizeof(uint32_t);

struct PeerPtrs {
  float* p[PEER_MAX_WORLD];       // every rank's parameter window (element 0 = window start)
  float* g[PEER_MAX_WORLD];       // every rank's gradient window
  uint32_t* sig[PEER_MAX_WORLD];  // every rank's signal array
  int rank, world;
};

struct PeerSegs {                 // owned shards [lo, hi) of the step's buckets (window element indices)
  int n;
  size_t lo[PEER_MAX_SEGS], hi[PEER_MAX_SEGS];
};

// Shard r of the bucket [off, off + n) over `world` ranks, boundaries rounded to 4 elements.
void peer_shard(size_t off, size_t n, int r, int world, size_t* lo, size_t* hi);

void peer_reduce(const PeerPtrs& a, size_t lo, size_t hi, uint32_t seq, float scale, int blocks,
                 long long timeout_ns, cudaStream_t st);
void peer_sgd(const PeerPtrs& a, const PeerSegs& s, float lr, uint32_t seq, int blocks, long long timeout_ns,
              cudaStream_t st);

}  // namespace astra
