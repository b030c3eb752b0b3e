// Host interface of the two GEMM engines:
//   K1  tcgen05/TMA/TMEM bf16 GEMM (bf16 path), persistent, tile width BN ∈ {64, 128, 256}.
//   K10 SIMT FFMA fp32 GEMM (fp32 parity path), sequential k order.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "gemm_tc.cuh"

namespace astra {

// A row-major (optionally batched along z) bf16 matrix in device memory, described by its
// storage: `outer` rows of `inner` contiguous elements at row stride `ld`; `z` slices at
// stride `zstride` (elements).
struct Mat2 {
  const void* ptr = nullptr;
  long inner = 0, outer = 0, z = 1;
  long ld = 0, zstride = 0;
};

// A prepared tcgen05 GEMM: tensor maps are built once (bind time) and reused every launch.
struct TcGemm {
  CUtensorMap mapA, mapB;
  TcArgs args;
  int BN = 256;
  int smem = 0;
  bool ready = false;
};

// D[M,N] = A·B.  A is [M,K]: K-major ⇒ storage rows = M, inner = K; MN-major ⇒ storage rows =
// K, inner = M.  B is [K,N]: K-major ⇒ storage rows = N, inner = K; MN-major ⇒ rows = K, inner = N.
// plain_maps: one-k-block tensor maps (TcArgs::kb = 1) — for callers that hand g.mapA / g.mapB to
// another kernel (the fused recurrent / BPTT kernels load single k-block boxes through them).
void tc_gemm_prepare(TcGemm& g, const Mat2& A, bool a_mn, const Mat2& B, bool b_mn, int M, int N, int K, int BN,
                     int cm = 1, int cn = 1, bool b_keep = false, int ksplit = 1, int cg = 1, int smem_cap = 0,
                     bool plain_maps = false, int kperm = 0);
// Launch with the given z-coordinates (time slices) and epilogue; grid ≤ #SMs (persistent).
void tc_gemm_launch(const TcGemm& g, const EpiStore& epi, int az, int bz, cudaStream_t st, int max_ctas = 0,
                    const L2Pf* pf = nullptr);

// fp32 SIMT GEMM with arbitrary element strides: A(m,k) = A[m*sam + k*sak],
// B(k,n) = B[k*sbk + n*sbn]; result stored through the same EpiStore rules (out_bf16 = 0).
void simt_gemm(const float* A, long sam, long sak, const float* B, long sbk, long sbn, int M, int N, int K,
               const EpiStore& epi, cudaStream_t st);

int num_sms();

// bf16 tensor map of rank 2..5 with arbitrary byte strides (dims[0] contiguous; strides_bytes[i] is
// the stride of dims[i+1]; strides may overlap, e.g. a k-block dimension of stride 128 B next to a
// row dimension) — lets one TMA box carry several k-block tiles of an MMA operand.
void make_map_nd(CUtensorMap* m, const void* ptr, int rank, const long* dims, const long* strides_bytes,
                 const int* box, int swizzle_bytes);

// 3-D tiled tensor map ([z][rows][inner], row stride ld, slice stride zstride, in elements) with a
// {box_inner, box_rows, 1} box and the given swizzle (0 / 32 / 64 / 128 bytes) — epilogue I/O maps.
void make_tile_map(CUtensorMap* m, const void* ptr, bool bf16, long inner, long rows, long z, long ld, long zstride,
                   int box_inner, int box_rows, int swizzle_bytes);

}  // namespace astra
