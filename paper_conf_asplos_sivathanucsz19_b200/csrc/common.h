// Internal helpers shared by the library's translation units (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <atomic>
#include <string>
#include <stdexcept>

#include "../../include/astra.h"

namespace astra {

// Thread-local error detail (astra_last_error).
void set_error(const std::string& s);

// Exceptions never cross the ABI: capi.cpp converts them to status codes.
struct Error : std::runtime_error {
  astra_status code;
  Error(astra_status c, const std::string& m) : std::runtime_error(m), code(c) {}
};

#define ASTRA_CHECK_ARG(cond, msg) \
  do { if (!(cond)) throw ::astra::Error(ASTRA_E_ARG, msg); } while (0)
#define ASTRA_CHECK_STATE(cond, msg) \
  do { if (!(cond)) throw ::astra::Error(ASTRA_E_STATE, msg); } while (0)
#define CUDA_TRY(expr)                                                                   \
  do {                                                                                   \
    cudaError_t e_ = (expr);                                                             \
    if (e_ != cudaSuccess)                                                               \
      throw ::astra::Error(ASTRA_E_CUDA, std::string(#expr) + ": " + cudaGetErrorString(e_) \
                           + " @" + __FILE__ + ":" + std::to_string(__LINE__));          \
  } while (0)

// Count of kernels launched by this library (bench.py reports it as gpu_launches).
extern std::atomic<uint64_t> g_launches;
inline void count_launch(uint64_t n = 1) { g_launches.fetch_add(n, std::memory_order_relaxed); }
#define LAUNCH_CHECK() do { ::astra::count_launch(); CUDA_TRY(cudaGetLastError()); } while (0)

inline int cdiv(long a, long b) { return (int)((a + b - 1) / b); }
inline long round_up(long a, long b) { return (a + b - 1) / b * b; }

enum class OT { BF16 = 0, F32 = 1 };  // GEMM operand type of a precision path
inline size_t ot_size(OT t) { return t == OT::BF16 ? 2 : 4; }

}  // namespace astra
