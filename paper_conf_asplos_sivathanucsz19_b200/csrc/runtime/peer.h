// Host side of K11p, the deterministic peer-memory DP backend (SURVEY §8(e) backend 2): the
// parameter / gradient window of this rank, the IPC mappings of every peer's window and signal
// array, the buckets of the current step and the launches of kernels/peer.h.
#pragma once
#include <cuda_runtime.h>

#include <utility>
#include <vector>

#include "../common.h"
#include "../kernels/peer.h"

namespace astra {

class PeerComm {
 public:
  PeerComm(int device, float* P, float* G, size_t n);
  ~PeerComm();
  PeerComm(const PeerComm&) = delete;
  PeerComm& operator=(const PeerComm&) = delete;

  int device;
  float* P;   // local parameter window (the flat vector SGD updates: the LM's, else the cell's)
  float* G;   // local gradient window
  size_t n;   // window length in floats
  int rank = 0, world = 1;
  bool ready = false;
  int dpb = -1;   // bucket cap choice of the LM's top layer (set per step by the LM); -1: the cell's own

  // ASTRA_PEER_HANDLE_BYTES of IPC handles + offsets of this rank's window and signal array
  void export_handle(void* out, size_t len) const;
  // handles: world × ASTRA_PEER_HANDLE_BYTES in rank order (this rank's own entry included)
  void import_handles(const void* handles, int rank, int world);

  void begin_step() { buckets.clear(); }
  // bucket [off, off + cnt) of the window is final on stream `st`: rank-ordered reduce of our shard
  void reduce(size_t off, size_t cnt, cudaStream_t st);
  // θ ← θ − lr·g on the owned shards of this step's buckets, all-gathered into every rank's window.
  // `cover`: parameter ranges that must lie inside the buckets (checked once)
  void sgd(float lr, cudaStream_t st, const std::vector<std::pair<size_t, size_t>>& cover);

 private:
  uint32_t* sig = nullptr;   // own signal array (PEER_SIG_BYTES, zeroed)
  PeerPtrs ptrs{};
  std::vector<void*> opened;  // IPC mappings to close
  std::vector<std::pair<size_t, size_t>> buckets;
  uint32_t seq = 0;
  int blocks_reduce = 32, blocks_sgd = 64;
  long long timeout_ns = 60LL * 1000 * 1000 * 1000;
  bool covered = false;
};

}  // namespace astra
