// Host side of K1 (tcgen05 GEMM) and K10 (SIMT fp32 GEMM).
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cstdlib>
#include <cstring>
#include <algorithm>
#include <mutex>
#include <tuple>
#include <map>

#include "../common.h"
#include "gemm.h"

namespace astra {

int num_sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev));
  }
  return n;
}

static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  if (!fn) throw Error(ASTRA_E_CUDA, "cuTensorMapEncodeTiled unavailable (driver too old?)");
  return fn;
}

static void make_map(CUtensorMap* m, const Mat2& t, int box_inner, int box_outer) {
  ASTRA_CHECK_ARG(t.ptr != nullptr, "tensor map: null pointer");
  ASTRA_CHECK_ARG(((uintptr_t)t.ptr & 15) == 0, "tensor map: base must be 16-byte aligned");
  ASTRA_CHECK_ARG((t.ld * 2) % 16 == 0, "tensor map: row stride must be a multiple of 16 bytes");
  ASTRA_CHECK_ARG(t.z == 1 || (t.zstride * 2) % 16 == 0, "tensor map: z stride must be a multiple of 16 bytes");
  cuuint64_t dims[3] = {(cuuint64_t)t.inner, (cuuint64_t)t.outer, (cuuint64_t)t.z};
  cuuint64_t strides[2] = {(cuuint64_t)(t.ld * 2), (cuuint64_t)((t.z > 1 ? t.zstride : t.ld * t.outer) * 2)};
  cuuint32_t box[3] = {(cuuint32_t)box_inner, (cuuint32_t)box_outer, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = encode_fn()(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(t.ptr), dims, strides, box,
                           estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(ASTRA_E_CUDA, "cuTensorMapEncodeTiled failed: " + std::to_string((int)r));
}

// Output tensor map of a plain (identity-mapped, non-accumulating) epilogue: [ksplit][Mv][Nv] of
// fp32 / bf16 at row stride ldc, box 32 x 32 (one epilogue warp's chunk), swizzled like the
// epilogue's shared-memory tile.  Cached by (pointer, shape): the step's output buffers repeat.
static bool epi_tma_map(const EpiStore& e, int ksplit, CUtensorMap* out) {
  const long esz = e.out_bf16 ? 2 : 4;
  if (e.perm_u || e.perm_blk || e.accumulate) return false;
  if (((uintptr_t)e.C & 15) || ((e.ldc * esz) & 15) || e.Mv <= 0 || e.Nv <= 0) return false;
  const long zs = ksplit > 1 ? e.split_stride : (long)e.Mv * e.ldc;
  if (ksplit > 1 && ((zs * esz) & 15)) return false;
  using Key = std::tuple<const void*, int, int, long, int, long, int>;
  static std::map<Key, CUtensorMap> cache;
  static std::mutex mu;
  const Key key{e.C, e.Mv, e.Nv, e.ldc, ksplit, zs, e.out_bf16};
  std::lock_guard<std::mutex> lk(mu);
  auto it = cache.find(key);
  if (it == cache.end()) {
    CUtensorMap m;
    cuuint64_t dims[3] = {(cuuint64_t)e.Nv, (cuuint64_t)e.Mv, (cuuint64_t)ksplit};
    cuuint64_t strides[2] = {(cuuint64_t)(e.ldc * esz), (cuuint64_t)(zs * esz)};
    cuuint32_t box[3] = {32, 32, 1};
    cuuint32_t estr[3] = {1, 1, 1};
    CUresult r = encode_fn()(&m, e.out_bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3,
                             e.C, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                             e.out_bf16 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B,
                             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return false;
    if (cache.size() > 65536) cache.clear();
    it = cache.emplace(key, m).first;
  }
  *out = it->second;
  return true;
}

void make_tile_map(CUtensorMap* m, const void* ptr, bool bf16, long inner, long rows, long z, long ld, long zstride,
                   int box_inner, int box_rows, int swizzle_bytes) {
  ASTRA_CHECK_ARG(ptr != nullptr && ((uintptr_t)ptr & 15) == 0, "tile map: base must be 16-byte aligned");
  const long esz = bf16 ? 2 : 4;
  ASTRA_CHECK_ARG((ld * esz) % 16 == 0 && (z == 1 || (zstride * esz) % 16 == 0), "tile map: strides must be 16-byte multiples");
  cuuint64_t dims[3] = {(cuuint64_t)inner, (cuuint64_t)rows, (cuuint64_t)z};
  cuuint64_t strides[2] = {(cuuint64_t)(ld * esz), (cuuint64_t)((z > 1 ? zstride : ld * rows) * esz)};
  cuuint32_t box[3] = {(cuuint32_t)box_inner, (cuuint32_t)box_rows, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  const CUtensorMapSwizzle sw = swizzle_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                : swizzle_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                : swizzle_bytes == 32 ? CU_TENSOR_MAP_SWIZZLE_32B : CU_TENSOR_MAP_SWIZZLE_NONE;
  CUresult r = encode_fn()(m, bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3,
                           const_cast<void*>(ptr), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(ASTRA_E_CUDA, "cuTensorMapEncodeTiled (tile map) failed: " + std::to_string((int)r));
}

void make_map_nd(CUtensorMap* m, const void* ptr, int rank, const long* dims, const long* strides_bytes,
                 const int* box, int swizzle_bytes) {
  ASTRA_CHECK_ARG(ptr != nullptr && ((uintptr_t)ptr & 15) == 0, "tensor map: base must be 16-byte aligned");
  ASTRA_CHECK_ARG(rank >= 2 && rank <= 5, "tensor map: rank must be 2..5");
  cuuint64_t d[5], st[4];
  cuuint32_t bx[5], es[5];
  for (int i = 0; i < rank; ++i) {
    d[i] = (cuuint64_t)dims[i];
    bx[i] = (cuuint32_t)box[i];
    es[i] = 1;
    if (i + 1 < rank) {
      ASTRA_CHECK_ARG(strides_bytes[i] % 16 == 0, "tensor map: strides must be 16-byte multiples");
      st[i] = (cuuint64_t)strides_bytes[i];
    }
  }
  const CUtensorMapSwizzle sw = swizzle_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                : swizzle_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                : swizzle_bytes == 32 ? CU_TENSOR_MAP_SWIZZLE_32B : CU_TENSOR_MAP_SWIZZLE_NONE;
  CUresult r = encode_fn()(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, rank, const_cast<void*>(ptr), d, st, bx, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                           CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(ASTRA_E_CUDA, "cuTensorMapEncodeTiled (nd map) failed: " + std::to_string((int)r));
}

static uint32_t make_idesc(int BN, bool a_mn, bool b_mn, int BM = TC_BM) {
  uint32_t d = 0;
  d |= 1u << 4;                      // D format: F32
  d |= 1u << 7;                      // A format: BF16
  d |= 1u << 10;                     // B format: BF16
  d |= (a_mn ? 1u : 0u) << 15;       // A major
  d |= (b_mn ? 1u : 0u) << 16;       // B major
  d |= (uint32_t)(BN >> 3) << 17;    // N >> 3
  d |= (uint32_t)(BM >> 4) << 24;    // M >> 4
  return d;
}

template <int BN>
static int smem_for(int& stages, int cap) {
  int dev = 0, maxs = 0;
  CUDA_TRY(cudaGetDevice(&dev));
  CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
  if (cap > 0 && cap < maxs) maxs = cap;   // leave room for co-resident kernels (fewer stages, same bits)
  stages = TcSmem<BN>::stages_for(maxs);
  ASTRA_CHECK_ARG(stages >= 2, "tc_gemm: shared-memory cap leaves fewer than 2 stages");
  return TcSmem<BN>::bytes(stages);
}

void tc_gemm_prepare(TcGemm& g, const Mat2& A, bool a_mn, const Mat2& B, bool b_mn, int M, int N, int K, int BN,
                     int cm, int cn, bool b_keep, int ksplit, int cg, int smem_cap, bool plain_maps, int kperm) {
  ASTRA_CHECK_ARG(kperm == 0 || (K == 4 * kperm * TC_BK), "tc_gemm: a gate-permuted K must be 4 gate blocks of kperm k-blocks");
  // BN = 224 (74 CTA pairs fill all 148 SMs on an 8192-column chain GEMM instead of 64 pairs of 256)
  // exists only for CTA pairs with a K-major B (each CTA holds 112 B rows); elsewhere the same tile
  // width is run as 256 — same bits (R1: every output element is one accumulation over K)
  if (BN == 224 && (cg != 2 || b_mn)) BN = 256;
  ASTRA_CHECK_ARG(cg == 1 || (cg == 2 && cm == 1 && cn == 1 && BN >= 128),
                  "tc_gemm: CTA pairs (cg = 2) need BN >= 128 and no extra cluster multicast");
  ASTRA_CHECK_ARG((cm == 1 || cm == 2 || cm == 4) && (cn == 1 || cn == 2 || cn == 4) && cm * cn <= 8,
                  "tc_gemm: cluster shape must be cm, cn in {1,2,4}, cm*cn <= 8");
  ASTRA_CHECK_ARG(BN == 64 || BN == 128 || BN == 256 || BN == 224, "tc_gemm: BN must be 64, 128, 224 or 256");
  ASTRA_CHECK_ARG(M > 0 && N > 0 && K > 0, "tc_gemm: empty problem");
  // multi-k-block stages (TcArgs::kb; tc_gemm_kernel without a cluster): the largest of 4 / 2 that
  // fits the per-chunk k-block count and still leaves >= 3 stages; K-major operands need K % 64 == 0
  // (their 4-D view reads whole 64-element k-blocks)
  int KB = 1;
  {
    static const int kb_env = [] {
      const char* e = std::getenv("ASTRA_GEMM_KB");   // A/B runs: 1 disables
      return e ? std::atoi(e) : 0;
    }();
    const int nk_all = cdiv(K, TC_BK), kper = cdiv(nk_all, ksplit);
    const bool kmaj_ok = (a_mn || K % TC_BK == 0) && (b_mn || K % TC_BK == 0);
    if (cg == 1 && cm * cn == 1 && kmaj_ok && kb_env != 1 && !plain_maps && kperm == 0) {
      int dev = 0, maxs = 0;
      CUDA_TRY(cudaGetDevice(&dev));
      CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
      if (smem_cap > 0 && smem_cap < maxs) maxs = smem_cap;
      for (int kb : {4, 2}) {
        if (kb_env > 1 && kb != kb_env) continue;
        const int a_kb = a_mn ? TC_BM * TC_BK * 2 : ((M <= 64 ? 64 : TC_BM) * TC_BK * 2);
        const int sb = kb * (a_kb + BN * TC_BK * 2);
        const int epi_bytes = TC_EPI_WARPS * 2 * 32 * 32 * 4;
        const int st = std::min(10, (maxs - 1024 - 256 - epi_bytes) / sb);
        // a chunk whose k-block count kb does not divide ends in a partial stage (the box still
        // lands kb tiles; the extra ones are never multiplied): allowed up to 25 % extra bytes
        const int waste = (kper + kb - 1) / kb * kb - kper;
        if (kper >= kb && 4 * waste <= kper && st >= 3) {
          KB = kb;
          break;
        }
      }
    }
  }
  const int a_rows = (KB > 1 && !a_mn && M <= 64) ? 64 : TC_BM;
  if (KB > 1) {
    if (a_mn) {
      make_map(&g.mapA, A, 64, 64 * KB);
    } else {
      const long dims[4] = {64, A.outer, A.inner / 64, A.z};
      const long str[3] = {A.ld * 2, 128, (A.z > 1 ? A.zstride : A.ld * A.outer) * 2};
      const int box[4] = {64, a_rows, KB, 1};
      make_map_nd(&g.mapA, A.ptr, 4, dims, str, box, 128);
    }
    if (b_mn) {
      make_map(&g.mapB, B, 64, 64 * KB);
    } else {
      const long dims[4] = {64, B.outer, B.inner / 64, B.z};
      const long str[3] = {B.ld * 2, 128, (B.z > 1 ? B.zstride : B.ld * B.outer) * 2};
      const int box[4] = {64, BN, KB, 1};
      make_map_nd(&g.mapB, B.ptr, 4, dims, str, box, 128);
    }
  } else {
    if (a_mn) make_map(&g.mapA, A, 64, 64 / cn); else make_map(&g.mapA, A, 64, TC_BM / cn);
    if (b_mn) make_map(&g.mapB, B, 64, 64 / cm); else make_map(&g.mapB, B, 64, BN / cm / cg);
  }
  g.args.kb = KB;
  g.args.a_rows = a_rows;
  g.args.kperm = kperm;
  g.args.pf = L2Pf{};
  g.args.cg = cg;
  static const int gm_env = [] {
    const char* e = std::getenv("ASTRA_GM");   // raster group override (A/B runs)
    return e ? std::max(1, std::atoi(e)) : 8;
  }();
  g.args.gm = gm_env;
  g.args.cm = cm;
  g.args.cn = cn;
  g.args.b_keep = b_keep ? 1 : 0;
  ASTRA_CHECK_ARG(ksplit >= 1 && (ksplit == 1 || cm * cn == 1), "tc_gemm: split-K needs a 1x1 cluster");
  g.args.ksplit = ksplit;
  g.BN = BN;
  g.args.M = M; g.args.N = N; g.args.K = K;
  g.args.num_m = cdiv(M, TC_BM);
  g.args.num_n = cdiv(N, BN);
  g.args.az = g.args.bz = 0;
  g.args.a_mn = a_mn; g.args.b_mn = b_mn;
  g.args.idesc = make_idesc(BN, a_mn, b_mn, TC_BM * cg);
  int stages = 0;
  switch (BN / cg) {
    case 64: g.smem = smem_for<64>(stages, smem_cap); break;
    case 112: g.smem = smem_for<112>(stages, smem_cap); break;
    case 128: g.smem = smem_for<128>(stages, smem_cap); break;
    default: g.smem = smem_for<256>(stages, smem_cap); break;
  }
  if (KB > 1) {   // stages of KB k-blocks (A tiles of a_rows rows)
    int dev = 0, maxs = 0;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&maxs, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
    if (smem_cap > 0 && smem_cap < maxs) maxs = smem_cap;
    const int a_kb = a_mn ? TC_BM * TC_BK * 2 : a_rows * TC_BK * 2;
    const int sb = KB * (a_kb + BN * TC_BK * 2);
    const int epi_bytes = TC_EPI_WARPS * 2 * 32 * 32 * 4;
    stages = std::min(10, (maxs - 1024 - 256 - epi_bytes) / sb);
    g.smem = 1024 + stages * sb + epi_bytes + 256;
  }
  g.args.stages = stages;
  g.ready = true;
}

template <int BN>
static void launch_pair(const TcGemm& g, const EpiStore& epi, int az, int bz, cudaStream_t st, int max_ctas,
                        const L2Pf* pf) {
  static int attr_bytes = 0;
  if (g.smem > attr_bytes) {
    CUDA_TRY(cudaFuncSetAttribute(tc_gemm2_kernel<BN, EpiStore>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  g.smem));
    attr_bytes = g.smem;
  }
  TcArgs a = g.args;
  a.az = az;
  a.bz = bz;
  if (pf) a.pf = *pf;
  CUtensorMap mapC;
  EpiStore e = epi;
  e.tma = epi_tma_map(epi, a.ksplit, &mapC) ? 1 : 0;
  if (!e.tma) memset(&mapC, 0, sizeof(mapC));
  const int ptiles = cdiv(a.M, 2 * TC_BM) * a.num_n * a.ksplit;
  int pairs = num_sms() / 2;
  if (max_ctas > 0 && max_ctas / 2 < pairs) pairs = max_ctas / 2 > 0 ? max_ctas / 2 : 1;
  if (ptiles < pairs) pairs = ptiles;
  launch_pdl(tc_gemm2_kernel<BN, EpiStore>, dim3(2 * pairs), dim3(TC_THREADS), g.smem, st, 2, g.mapA, g.mapB, mapC, a,
             e);
  LAUNCH_CHECK();
}

template <int BN>
static void launch_bn(const TcGemm& g, const EpiStore& epi, int az, int bz, cudaStream_t st, int max_ctas,
                        const L2Pf* pf) {
  static int attr_bytes = 0;
  if (g.smem > attr_bytes) {
    CUDA_TRY(cudaFuncSetAttribute(tc_gemm_kernel<BN, EpiStore>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  g.smem));
    attr_bytes = g.smem;
  }
  TcArgs a = g.args;
  a.az = az;
  a.bz = bz;
  if (pf) a.pf = *pf;
  CUtensorMap mapC;
  EpiStore e = epi;
  e.tma = epi_tma_map(epi, a.ksplit, &mapC) ? 1 : 0;
  if (!e.tma) memset(&mapC, 0, sizeof(mapC));
  const int cs = a.cm * a.cn;
  const int ctiles = cdiv(a.num_m, a.cm) * cdiv(a.num_n, a.cn) * a.ksplit;   // cluster tiles × K chunks
  int clusters = num_sms() / cs;
  if (max_ctas > 0 && max_ctas / cs < clusters) clusters = max_ctas / cs > 0 ? max_ctas / cs : 1;
  if (ctiles < clusters) clusters = ctiles;
  const int grid = clusters * cs;
  launch_pdl(tc_gemm_kernel<BN, EpiStore>, dim3(grid), dim3(TC_THREADS), g.smem, st, cs, g.mapA, g.mapB, mapC, a, e);
  LAUNCH_CHECK();
}

void tc_gemm_launch(const TcGemm& g, const EpiStore& epi, int az, int bz, cudaStream_t st, int max_ctas,
                    const L2Pf* pf) {
  ASTRA_CHECK_STATE(g.ready, "tc_gemm: not prepared");
  if (g.args.cg == 2) {
    if (g.BN == 128) launch_pair<128>(g, epi, az, bz, st, max_ctas, pf);
    else if (g.BN == 224) launch_pair<224>(g, epi, az, bz, st, max_ctas, pf);
    else launch_pair<256>(g, epi, az, bz, st, max_ctas, pf);
    return;
  }
  switch (g.BN) {
    case 64: launch_bn<64>(g, epi, az, bz, st, max_ctas, pf); break;
    case 128: launch_bn<128>(g, epi, az, bz, st, max_ctas, pf); break;
    default: launch_bn<256>(g, epi, az, bz, st, max_ctas, pf); break;
  }
}

// ------------------------------------------------------------------------------ K10 SIMT
// 64x64 output tile per 256-thread CTA, 4x4 per thread, k chunks of 16 staged in shared memory.
// Each output element is one fp32 FMA chain over k = 0..K-1 in ascending order (R1/R2).
__global__ void __launch_bounds__(256) simt_gemm_kernel(const float* __restrict__ A, long sam, long sak,
                                                        const float* __restrict__ B, long sbk, long sbn, int M,
                                                        int N, int K, EpiStore epi) {
  __shared__ float As[16][64 + 1];
  __shared__ float Bs[16][64 + 1];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int m0 = blockIdx.y * 64, n0 = blockIdx.x * 64;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += 16) {
    for (int i = threadIdx.x; i < 16 * 64; i += 256) {
      const int kk = i / 64, r = i % 64;
      const int m = m0 + r, n = n0 + r, k = k0 + kk;
      As[kk][r] = (m < M && k < K) ? A[(long)m * sam + (long)k * sak] : 0.f;
      Bs[kk][r] = (n < N && k < K) ? B[(long)k * sbk + (long)n * sbn] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = __fmaf_rn(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int m = m0 + ty * 4 + i;
    if (m >= M || m >= epi.Mv) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = n0 + tx * 4 + j;
      if (n >= N) continue;
      bool ok;
      const int e = epi.map_col(n, ok);
      if (!ok) continue;
      const float v = __fadd_rn(acc[i][j], (epi.bias && n < epi.Nv) ? epi.bias[n] : 0.f);
      float* p = reinterpret_cast<float*>(epi.C) + (long)m * epi.ldc + e;
      *p = epi.accumulate ? __fadd_rn(*p, v) : v;
    }
  }
}

void simt_gemm(const float* A, long sam, long sak, const float* B, long sbk, long sbn, int M, int N, int K,
               const EpiStore& epi, cudaStream_t st) {
  ASTRA_CHECK_ARG(!epi.out_bf16, "simt_gemm writes fp32");
  dim3 grid(cdiv(N, 64), cdiv(M, 64));
  simt_gemm_kernel<<<grid, 256, 0, st>>>(A, sam, sak, B, sbk, sbn, M, N, K, epi);
  LAUNCH_CHECK();
}

}  // namespace astra
