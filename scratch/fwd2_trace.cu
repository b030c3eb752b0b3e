// Standalone timing of the fused CTA-pair forward step: nvcc -DASTRA_GEMM_TRACE
#include <cstdio>
#include <vector>
#include "../paper_conf_asplos_sivathanucsz19_b200/csrc/kernels/gemm.cu"
#include "../paper_conf_asplos_sivathanucsz19_b200/csrc/kernels/rec_fused2.cu"
namespace astra {
std::atomic<uint64_t> g_launches{0};
void set_error(const std::string&) {}
}
using namespace astra;
int main(int argc, char** argv) {
  const int B = argc > 1 ? atoi(argv[1]) : 512, H = argc > 2 ? atoi(argv[2]) : 2048, T = 2;
  const int Hp = H, NG = 4 * Hp;
  void *Hb, *Um; float *WX, *UH, *C, *prm;
  cudaMalloc(&Hb, (size_t)(T + 1) * B * Hp * 2); cudaMalloc(&Um, (size_t)NG * Hp * 2);
  cudaMalloc(&WX, (size_t)T * B * NG * 4); cudaMalloc(&UH, (size_t)T * B * NG * 4);
  cudaMalloc(&C, (size_t)(T + 1) * B * Hp * 4); cudaMalloc(&prm, (size_t)4 * 4 * H * 4);
  cudaMemset(Hb, 0, (size_t)(T + 1) * B * Hp * 2); cudaMemset(Um, 0, (size_t)NG * Hp * 2);
  cudaMemset(WX, 0, (size_t)T * B * NG * 4); cudaMemset(C, 0, (size_t)(T + 1) * B * Hp * 4); cudaMemset(prm, 0, 64 * H);
  Mat2 a, b;
  a.ptr = Hb; a.inner = Hp; a.outer = B; a.ld = Hp; a.z = T + 1; a.zstride = (long)B * Hp;
  b.ptr = Um; b.inner = Hp; b.outer = NG; b.ld = Hp;
  TcGemm g;
  tc_gemm_prepare(g, a, false, b, false, B, NG, Hp, 256, 1, 1, true, 1, 2);
  RecFwd2Maps m;
  m.A = g.mapA; m.B = g.mapB;
  make_tile_map(&m.WX, WX, false, NG, B, T, NG, (long)B * NG, 32, 32, 128);
  make_tile_map(&m.UH, UH, false, NG, B, T, NG, (long)B * NG, 32, 32, 128);
  make_tile_map(&m.C, C, false, Hp, B, T + 1, Hp, (long)B * Hp, 32, 32, 128);
  make_tile_map(&m.H, Hb, true, Hp, B, T + 1, Hp, (long)B * Hp, 32, 32, 64);
  m.Y = m.H;
  RecFwd2Args ra;
  ra.B = B; ra.H = H; ra.Hp = Hp; ra.NG = NG; ra.T = T; ra.t = 0;
  ra.num_mp = cdiv(B, 256); ra.num_n = NG / 256; ra.idesc = g.args.idesc; ra.y_kind = 0; ra.y = nullptr;
  ra.hT = nullptr; ra.cT = nullptr;
  ra.gp.b = prm; ra.gp.alpha = prm + 4 * H; ra.gp.beta1 = prm + 8 * H; ra.gp.beta2 = prm + 12 * H;
  cudaStream_t st; cudaStreamCreate(&st);
  for (int i = 0; i < 3; ++i) lstm_fwd_pair_launch(K_MILSTM, m, ra, st);
  const int reps = 20;
  cudaGraph_t gr; cudaGraphExec_t ge;
  cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < reps; ++i) lstm_fwd_pair_launch(K_MILSTM, m, ra, st);
  cudaStreamEndCapture(st, &gr);
  cudaGraphInstantiate(&ge, gr, 0);
  cudaGraphLaunch(ge, st);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0, st); cudaGraphLaunch(ge, st); cudaEventRecord(e1, st);
  cudaStreamSynchronize(st);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long t[16];
  cudaMemcpyFromSymbol(t, g_gemm_trace, sizeof(t));
  auto d = [&](int i) { return (long long)(t[i] - t[0]); };
  printf("fused fwd B=%d H=%d: %.2f us/launch | setup %lld first-full %lld mma-done %lld epi-start %lld loads-in %lld compute-done %lld stores-done %lld exit %lld  err=%s\n",
         B, H, ms * 1e3 / reps, d(1), d(3), d(4), d(5), d(6), d(7), d(8), d(9), cudaGetErrorString(cudaGetLastError()));
  return 0;
}
