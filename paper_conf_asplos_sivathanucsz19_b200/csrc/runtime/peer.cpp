// K11p host side (SURVEY §8(e) backend 2): window export / import over CUDA IPC, per-step bucket
// bookkeeping and the launches of the rank-ordered reduce and the fused SGD + all-gather.
#include "peer.h"

#include <cuda.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <string>

namespace astra {

namespace {

constexpr uint32_t PEER_MAGIC = 0x41535450u;   // "ASTP"
constexpr uint32_t PEER_VERSION = 1;

struct PeerWire {
  uint32_t magic, version;
  int32_t device, world_hint;
  uint64_t n, off_p, off_g;
  cudaIpcMemHandle_t hp, hg, hs;
};
static_assert(sizeof(PeerWire) <= ASTRA_PEER_HANDLE_BYTES, "peer handle does not fit");

using PFN_range = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);

// Base of the cudaMalloc allocation holding `p` (IPC handles name whole allocations; a torch
// tensor is a sub-range of a caching-allocator segment).
void* alloc_base(const void* p) {
  static PFN_range fn = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      f = nullptr;
    return reinterpret_cast<PFN_range>(f);
  }();
  if (!fn) throw Error(ASTRA_E_CUDA, "cuMemGetAddressRange unavailable");
  CUdeviceptr base = 0;
  size_t sz = 0;
  if (fn(&base, &sz, (CUdeviceptr)p) != CUDA_SUCCESS) throw Error(ASTRA_E_ARG, "peer: window is not device memory");
  return (void*)base;
}

}  // namespace

PeerComm::PeerComm(int dev, float* P_, float* G_, size_t n_) : device(dev), P(P_), G(G_), n(n_) {
  ASTRA_CHECK_ARG(P && G && n > 0, "peer: window not bound");
  ASTRA_CHECK_ARG(((uintptr_t)P & 15) == 0 && ((uintptr_t)G & 15) == 0, "peer: window must be 16-byte aligned");
  CUDA_TRY(cudaSetDevice(device));
  CUDA_TRY(cudaMalloc(&sig, PEER_SIG_BYTES));
  CUDA_TRY(cudaMemset(sig, 0, PEER_SIG_BYTES));
  CUDA_TRY(cudaDeviceSynchronize());
  if (const char* e = std::getenv("ASTRA_PEER_TIMEOUT_S")) timeout_ns = (long long)(std::atof(e) * 1e9);
  if (const char* e = std::getenv("ASTRA_PEER_BLOCKS")) blocks_reduce = std::clamp(std::atoi(e), 1, PEER_MAX_BLOCKS);
}

PeerComm::~PeerComm() {
  cudaSetDevice(device);
  for (void* p : opened) cudaIpcCloseMemHandle(p);
  if (sig) cudaFree(sig);
}

void PeerComm::export_handle(void* out, size_t len) const {
  ASTRA_CHECK_ARG(out && len >= ASTRA_PEER_HANDLE_BYTES, "comm_peer_handle: buffer too small");
  CUDA_TRY(cudaSetDevice(device));
  PeerWire w;
  std::memset(&w, 0, sizeof(w));
  w.magic = PEER_MAGIC;
  w.version = PEER_VERSION;
  w.device = device;
  w.n = n;
  void* bp = alloc_base(P);
  void* bg = alloc_base(G);
  w.off_p = (uint64_t)((char*)P - (char*)bp);
  w.off_g = (uint64_t)((char*)G - (char*)bg);
  CUDA_TRY(cudaIpcGetMemHandle(&w.hp, bp));
  CUDA_TRY(cudaIpcGetMemHandle(&w.hg, bg));
  CUDA_TRY(cudaIpcGetMemHandle(&w.hs, sig));
  std::memset(out, 0, ASTRA_PEER_HANDLE_BYTES);
  std::memcpy(out, &w, sizeof(w));
}

void PeerComm::import_handles(const void* handles, int r, int wd) {
  ASTRA_CHECK_ARG(handles, "comm_peer_init: handles is null");
  ASTRA_CHECK_ARG(wd >= 1 && wd <= PEER_MAX_WORLD && r >= 0 && r < wd, "comm_peer_init: bad rank/world (world <= 8)");
  ASTRA_CHECK_STATE(!ready, "comm_peer_init: already initialised");
  std::vector<PeerWire> w(wd);
  for (int q = 0; q < wd; ++q) {
    std::memcpy(&w[q], (const char*)handles + (size_t)q * ASTRA_PEER_HANDLE_BYTES, sizeof(PeerWire));
    ASTRA_CHECK_ARG(w[q].magic == PEER_MAGIC && w[q].version == PEER_VERSION, "comm_peer_init: not a peer handle");
    ASTRA_CHECK_ARG(w[q].n == n, "comm_peer_init: ranks bound windows of different lengths");
  }
  CUDA_TRY(cudaSetDevice(device));
  PeerPtrs a{};
  a.rank = r;
  a.world = wd;
  // each distinct allocation of a peer is opened once (params and grads may share a segment)
  std::vector<std::pair<cudaIpcMemHandle_t, void*>> seen;
  auto open = [&](const cudaIpcMemHandle_t& h) -> void* {
    for (auto& s : seen)
      if (std::memcmp(&s.first, &h, sizeof(h)) == 0) return s.second;
    void* p = nullptr;
    CUDA_TRY(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
    opened.push_back(p);
    seen.push_back({h, p});
    return p;
  };
  for (int q = 0; q < wd; ++q) {
    if (q == r) {
      a.p[q] = P;
      a.g[q] = G;
      a.sig[q] = sig;
      continue;
    }
    a.p[q] = (float*)((char*)open(w[q].hp) + w[q].off_p);
    a.g[q] = (float*)((char*)open(w[q].hg) + w[q].off_g);
    a.sig[q] = (uint32_t*)open(w[q].hs);
  }
  ptrs = a;
  rank = r;
  world = wd;
  ready = true;
}

void PeerComm::reduce(size_t off, size_t cnt, cudaStream_t st) {
  ASTRA_CHECK_STATE(ready, "peer: not initialised");
  ASTRA_CHECK_ARG(off + cnt <= n, "peer: bucket outside the window");
  for (auto& b : buckets)
    ASTRA_CHECK_STATE(off + cnt <= b.first || b.first + b.second <= off, "peer: overlapping buckets in one step");
  buckets.push_back({off, cnt});
  size_t lo, hi;
  peer_shard(off, cnt, rank, world, &lo, &hi);
  peer_reduce(ptrs, lo, hi, ++seq, 1.0f / (float)world, blocks_reduce, timeout_ns, st);
}

void PeerComm::sgd(float lr, cudaStream_t st, const std::vector<std::pair<size_t, size_t>>& cover) {
  ASTRA_CHECK_STATE(ready, "peer: not initialised");
  ASTRA_CHECK_STATE(!buckets.empty(), "peer sgd: no gradient buckets in this step (call after the backward)");
  if (!covered) {   // every parameter must be reduced (and so owned by exactly one rank)
    for (auto& c : cover) {
      size_t lo = c.first;
      const size_t hi = c.first + c.second;
      bool progress = true;
      while (lo < hi && progress) {
        progress = false;
        for (auto& b : buckets)
          if (b.first <= lo && lo < b.first + b.second) {
            lo = b.first + b.second;
            progress = true;
          }
      }
      ASTRA_CHECK_STATE(lo >= hi, "peer sgd: a parameter range is outside every gradient bucket");
    }
    covered = true;
  }
  PeerSegs s{};
  for (auto& b : buckets) {
    size_t lo, hi;
    peer_shard(b.first, b.second, rank, world, &lo, &hi);
    if (hi <= lo) continue;
    ASTRA_CHECK_STATE(s.n < PEER_MAX_SEGS, "peer sgd: too many buckets");
    s.lo[s.n] = lo;
    s.hi[s.n] = hi;
    ++s.n;
  }
  peer_sgd(ptrs, s, lr, seq + 1, blocks_sgd, timeout_ns, st);
  seq += 2;
  buckets.clear();
}

}  // namespace astra
