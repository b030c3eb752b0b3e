// Standalone K1 timing harness: nvcc -DASTRA_GEMM_TRACE ... ; prints event time and CTA-0 phases.
#include <cstdio>
#include <vector>
#include "../paper_conf_asplos_sivathanucsz19_b200/csrc/kernels/gemm.cu"
namespace astra {
std::atomic<uint64_t> g_launches{0};
void set_error(const std::string&) {}
}
using namespace astra;
int main(int argc, char** argv) {
  int M = atoi(argv[1]), N = atoi(argv[2]), K = atoi(argv[3]), BN = atoi(argv[4]), cg = argc > 5 ? atoi(argv[5]) : 1;
  int reps = argc > 6 ? atoi(argv[6]) : 20;
  void *A, *B; float* C;
  cudaMalloc(&A, (size_t)M * K * 2); cudaMalloc(&B, (size_t)N * K * 2); cudaMalloc(&C, (size_t)M * N * 4);
  cudaMemset(A, 0, (size_t)M * K * 2); cudaMemset(B, 0, (size_t)N * K * 2);
  Mat2 a, b;
  a.ptr = A; a.inner = K; a.outer = M; a.ld = K;
  b.ptr = B; b.inner = K; b.outer = N; b.ld = K;
  TcGemm g;
  tc_gemm_prepare(g, a, false, b, false, M, N, K, BN, 1, 1, false, 1, cg);
  EpiStore e; memset(&e, 0, sizeof(e)); e.C = C; e.ldc = N; e.Mv = M; e.Nv = N;
  cudaStream_t st; cudaStreamCreate(&st);
  for (int i = 0; i < 5; ++i) tc_gemm_launch(g, e, 0, 0, st);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  // graph of `reps` launches (no host overhead)
  cudaGraph_t gr; cudaGraphExec_t ge;
  cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < reps; ++i) tc_gemm_launch(g, e, 0, 0, st);
  cudaStreamEndCapture(st, &gr);
  cudaGraphInstantiate(&ge, gr, 0);
  cudaGraphLaunch(ge, st);
  cudaEventRecord(e0, st);
  cudaGraphLaunch(ge, st);
  cudaEventRecord(e1, st);
  cudaStreamSynchronize(st);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long t[16];
  cudaMemcpyFromSymbol(t, g_gemm_trace, sizeof(t));
  printf("M=%d N=%d K=%d BN=%d cg=%d: %.2f us/launch (graph of %d) | CTA0 phases (ns from entry): setup %lld first-full %lld mma-done %lld epi-start %lld epi-done %lld exit %lld  err=%s\n",
         M, N, K, BN, cg, ms * 1e3 / reps, reps, (long long)(t[1] - t[0]), (long long)(t[3] - t[0]), (long long)(t[4] - t[0]),
         (long long)(t[5] - t[0]), (long long)(t[6] - t[0]), (long long)(t[7] - t[0]), cudaGetErrorString(cudaGetLastError()));
  return 0;
}
