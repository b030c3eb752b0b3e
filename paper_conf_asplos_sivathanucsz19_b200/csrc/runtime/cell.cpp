// L1 runtime: workspace carving and the executor of one training step of the LSTM-family cells
// (LSTM, MI-LSTM [36], subLSTM [8]) on both precision paths, plus the LM wrapper.
//
// Step anatomy:
//   fwd : mirrors(K9) → x copy → state init → a1 hoisted GEMM WX = X·W (K1) →
//         for t: UH_t = h_{t-1}·U (K1) ; pointwise gate epilogue (K2 half)
//   bwd : for t desc: dh_rec = D_uh[t+1]·Uᵀ (K1) ; pointwise cell backward (K4 half, K5 partials)
//         → dh0 → wgrad dU = Hᵀ·D_uh, dW = Xᵀ·D_wx (K1) → dX = D_wx·Wᵀ (K1) → bias/α/β reductions (K5)
//         → gradient sum over ranks (K11) when world > 1.
#include "cell.h"
#include "../kernels/cell_math.cuh"

#include <nccl.h>

#include <algorithm>
#include <cstring>
#include <sstream>

namespace astra {

const char* const ROLE_NAMES[G_ROLES] = {"a1", "rec", "bptt", "du", "dw", "dx", "head"};

std::string Variant::str() const {
  std::ostringstream o;
  for (int r = 0; r < G_ROLES; ++r) o << ROLE_NAMES[r] << "=" << g[r].bn << "." << g[r].cm << "." << g[r].cn << ",";
  o << "wg_side=" << wg_side;
  return o.str();
}

Variant Variant::parse(const std::string& s) {
  Variant v;
  size_t p = 0;
  while (p < s.size()) {
    size_t q = s.find(',', p);
    if (q == std::string::npos) q = s.size();
    const std::string kv = s.substr(p, q - p);
    p = q + 1;
    if (kv.empty()) continue;
    const size_t eq = kv.find('=');
    ASTRA_CHECK_ARG(eq != std::string::npos, "variant: expected key=value, got '" + kv + "'");
    const std::string k = kv.substr(0, eq), val = kv.substr(eq + 1);
    if (k == "wg_side") {
      v.wg_side = std::stoi(val);
      ASTRA_CHECK_ARG(v.wg_side == 0 || v.wg_side == 1, "variant: wg_side must be 0 or 1");
      continue;
    }
    int r = -1;
    for (int i = 0; i < G_ROLES; ++i)
      if (k == ROLE_NAMES[i]) r = i;
    ASTRA_CHECK_ARG(r >= 0, "variant: unknown variable '" + k + "'");
    KCfg c;
    int n = std::sscanf(val.c_str(), "%d.%d.%d", &c.bn, &c.cm, &c.cn);
    ASTRA_CHECK_ARG(n >= 1, "variant: bad kernel choice '" + val + "'");
    if (n < 3) c.cn = 1;
    if (n < 2) c.cm = 1;
    ASTRA_CHECK_ARG((c.bn == 64 || c.bn == 128 || c.bn == 256) && (c.cm == 1 || c.cm == 2 || c.cm == 4) &&
                        (c.cn == 1 || c.cn == 2 || c.cn == 4) && c.cm * c.cn <= 8,
                    "variant: tile width must be 64/128/256 and cluster cm, cn in {1,2,4} with cm*cn <= 8");
    v.g[r] = c;
  }
  return v;
}

static size_t align_up(size_t v, size_t a) { return (v + a - 1) / a * a; }

Cell::Cell(const astra_cell_desc& dd) : d(dd) {
  ASTRA_CHECK_ARG(d.hidden > 0 && d.input > 0 && d.batch > 0 && d.seq > 0, "cell: sizes must be positive");
  ASTRA_CHECK_ARG(d.dtype == ASTRA_BF16 || d.dtype == ASTRA_FP32, "cell: dtype must be ASTRA_BF16 or ASTRA_FP32");
  if (d.cell_type == ASTRA_LSTM) kind = K_LSTM;
  else if (d.cell_type == ASTRA_MILSTM) kind = K_MILSTM;
  else if (d.cell_type == ASTRA_SUBLSTM) kind = K_SUBLSTM;
  else if (d.cell_type == ASTRA_SCRNN || d.cell_type == ASTRA_RHN || d.cell_type == ASTRA_LSTM_ATTN)
    throw Error(ASTRA_E_UNSUPPORTED, "cell: SCRN / RHN / LSTM-attention CUDA paths are not built yet");
  else
    throw Error(ASTRA_E_ARG, "cell: unknown cell_type");
  ot = d.dtype == ASTRA_BF16 ? OT::BF16 : OT::F32;
  H = d.hidden; I = d.input; B = d.batch; T = d.seq;
  Hp = (int)round_up(H, GATE_U);
  Ip = (int)round_up(I, 64);
  NG = 4 * Hp;
  Hout = H;
  ASTRA_CHECK_ARG((long)T * B < (1L << 31) / 64, "cell: T*B too large");

  // flat fp32 parameter vector, every tensor 256-byte aligned
  auto add = [&](const char* n, int r, int c) {
    params.push_back({n, n_params, r, c});
    n_params = align_up(n_params + (size_t)r * c, 64);
  };
  add("W", I, 4 * H);
  add("U", H, 4 * H);
  add("b", 1, 4 * H);
  if (kind == K_MILSTM) {
    add("alpha", 1, 4 * H);
    add("beta1", 1, 4 * H);
    add("beta2", 1, 4 * H);
  }

  const size_t e = esz();
  const size_t TB = (size_t)T * B;
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes, 256); return r; };
  off_X = take(TB * Ip * e);
  off_WX = take(TB * NG * 4);
  off_UH = take(TB * NG * 4);
  off_C = take((TB + B) * Hp * 4);
  off_H = take((TB + B) * Hp * e);
  off_Wm = take((size_t)NG * Ip * e);
  off_Um = take((size_t)NG * Hp * e);
  saved_bytes = o;
  nchunk = lstm_bwd_row_chunks(B);
  o = 0;
  off_Duh = take(TB * NG * e);
  off_Dwx = kind == K_MILSTM ? take(TB * NG * e) : off_Duh;
  off_dH = take((size_t)B * Hp * 4);
  off_dC = take((size_t)B * Hp * 4);
  off_part = take((size_t)nchunk * 4 * NG * 4);
  off_dXf = 0;
  scratch_bytes = o;
  for (int r = 0; r < R_COUNT; ++r) region_used[r] = false;
  std::memset(ev, 0, sizeof(ev));
}

Cell::~Cell() {
  for (int r = 0; r < R_COUNT; ++r)
    for (int w = 0; w < 2; ++w)
      if (ev[r][w]) cudaEventDestroy(ev[r][w]);
  if (ev_fork) cudaEventDestroy(ev_fork);
  if (ev_join) cudaEventDestroy(ev_join);
  if (nccl_comm) ncclCommDestroy((ncclComm_t)nccl_comm);
}

size_t Cell::find_param(const std::string& n) const {
  for (auto& p : params)
    if (p.name == n) return p.offset;
  throw Error(ASTRA_E_ARG, "no parameter " + n);
}

void Cell::bind(float* pp, float* gg, void* sv_p, void* sc_p) {
  ASTRA_CHECK_ARG(pp && gg && sv_p && sc_p, "bind: null pointer");
  ASTRA_CHECK_ARG(((uintptr_t)pp & 255) == 0 && ((uintptr_t)gg & 255) == 0 && ((uintptr_t)sv_p & 255) == 0 &&
                      ((uintptr_t)sc_p & 255) == 0,
                  "bind: pointers must be 256-byte aligned");
  CUDA_TRY(cudaSetDevice(d.device));
  P = pp; G = gg; saved = (char*)sv_p; scratch = (char*)sc_p;
  tc_cache.clear();
  if (!ev_fork) {
    CUDA_TRY(cudaEventCreateWithFlags(&ev_fork, cudaEventDisableTiming));
    CUDA_TRY(cudaEventCreateWithFlags(&ev_join, cudaEventDisableTiming));
    for (int r = 0; r < R_COUNT; ++r)
      for (int w = 0; w < 2; ++w) CUDA_TRY(cudaEventCreate(&ev[r][w]));
  }
  bound = true;
  fwd_done = false;
}

void Cell::mark(Region r, int which, cudaStream_t st) {
  if (!profiling) return;
  CUDA_TRY(cudaEventRecord(ev[r][which], st));
  if (which) region_used[r] = true;
}

void Cell::run_gemm(int id, const GemmSpec& s, const EpiStore& e, int az, int bz, const KCfg& k, cudaStream_t st) {
  if (ot == OT::BF16) {
    auto key = std::make_tuple(id, k.bn, k.cm, k.cn);
    auto it = tc_cache.find(key);
    if (it == tc_cache.end()) {
      TcGemm g;
      tc_gemm_prepare(g, s.A, s.a_mn, s.B, s.b_mn, s.M, s.N, s.K, k.bn, k.cm, k.cn);
      it = tc_cache.emplace(key, g).first;
    }
    tc_gemm_launch(it->second, e, az, bz, st);
  } else {
    const float* A = (const float*)s.A.ptr + (long)az * s.A.zstride;
    const float* Bm = (const float*)s.B.ptr + (long)bz * s.B.zstride;
    long sam, sak, sbk, sbn;
    if (!s.a_mn) { sam = s.A.ld; sak = 1; } else { sam = 1; sak = s.A.ld; }
    if (!s.b_mn) { sbk = 1; sbn = s.B.ld; } else { sbk = s.B.ld; sbn = 1; }
    simt_gemm(A, sam, sak, Bm, sbk, sbn, s.M, s.N, s.K, e, st);
  }
}

static Mat2 mat(const void* p, long inner, long outer, long ld, long z = 1, long zstride = 0) {
  Mat2 m;
  m.ptr = p; m.inner = inner; m.outer = outer; m.ld = ld; m.z = z; m.zstride = zstride;
  return m;
}
static EpiStore epi(void* C, long ldc, int Mv, int Nv, int out_bf16 = 0, const float* bias = nullptr, int perm_u = 0,
                    int perm_H = 0) {
  EpiStore e;
  e.C = C; e.ldc = ldc; e.Mv = Mv; e.Nv = Nv; e.out_bf16 = out_bf16; e.bias = bias; e.perm_u = perm_u;
  e.perm_H = perm_H;
  return e;
}

void Cell::forward(const void* x, const float* h0, const float* c0, void* y, float* hT, float* cT) {
  ASTRA_CHECK_STATE(bound, "step_fwd: call astra_bind first");
  ASTRA_CHECK_ARG(lm_mode || x, "step_fwd: x is null");
  cudaStream_t st = main_st;
  const long TB = (long)T * B;
  const size_t e = esz();
  void* X = sv<char>(off_X);
  void* Wm = sv<char>(off_Wm);
  void* Um = sv<char>(off_Um);
  float* WX = sv<float>(off_WX);
  float* UH = sv<float>(off_UH);
  float* Cb = sv<float>(off_C);

  mark(R_STEP, 0, st);
  // K9 second half: operand mirrors in the internal gate-interleaved layout
  mirror_gates_T(ot, p("W"), I, H, Hp, Wm, Ip, st);
  mirror_gates_T(ot, p("U"), H, H, Hp, Um, Hp, st);
  if (!lm_mode) copy_pad(ot, x, ot, TB, I, I, X, Ip, st);
  copy_pad(ot, h0, OT::F32, B, H, H, Hrow(0), Hp, st);
  copy_f32_pad(c0, B, H, H, Cb, Hp, H, st);

  GateParams gp;
  gp.b = p("b");
  if (kind == K_MILSTM) { gp.alpha = p("alpha"); gp.beta1 = p("beta1"); gp.beta2 = p("beta2"); }

  // a1: hoisted input projection for all timesteps
  mark(R_A1, 0, st);
  GemmSpec a1;
  a1.A = mat(X, I, TB, Ip);
  a1.B = mat(Wm, I, NG, Ip);
  a1.M = (int)TB; a1.N = NG; a1.K = I;
  run_gemm(0, a1, epi(WX, NG, (int)TB, NG), 0, 0, var.g[G_A1], st);
  mark(R_A1, 1, st);

  // a3: recurrent chain
  mark(R_FWD, 0, st);
  GemmSpec rec;
  rec.A = mat(Hrow(0), Hp, B, Hp, T + 1, (long)B * Hp);
  rec.B = mat(Um, Hp, NG, Hp);
  rec.M = B; rec.N = NG; rec.K = Hp;
  for (int t = 0; t < T; ++t) {
    float* UHt = UH + (long)t * B * NG;
    run_gemm(1, rec, epi(UHt, NG, B, NG), t, 0, var.g[G_REC], st);
    const bool last = t == T - 1;
    void* yt = y ? (char*)y + (size_t)t * B * H * e : nullptr;
    lstm_fwd_pointwise(kind, ot, B, H, Hp, WX + (long)t * B * NG, UHt, gp, Cb + (long)t * B * Hp,
                       Cb + (long)(t + 1) * B * Hp, Hrow(t + 1), yt, H, ot, last ? hT : nullptr,
                       last ? cT : nullptr, st);
  }
  mark(R_FWD, 1, st);
  fwd_done = true;
}

void Cell::backward(const void* dy, const float* dhT, const float* dcT, void* dx, float* dh0, float* dc0) {
  ASTRA_CHECK_STATE(bound && fwd_done, "step_bwd: needs a preceding step_fwd");
  ASTRA_CHECK_ARG(lm_mode || dy, "step_bwd: dy is null");
  cudaStream_t st = main_st;
  const long TB = (long)T * B;
  const size_t e = esz();
  void* X = sv<char>(off_X);
  void* Wm = sv<char>(off_Wm);
  void* Um = sv<char>(off_Um);
  float* WX = sv<float>(off_WX);
  float* UH = sv<float>(off_UH);
  float* Cb = sv<float>(off_C);
  char* Duh = sc<char>(off_Duh);
  char* Dwx = sc<char>(off_Dwx);
  float* dH = sc<float>(off_dH);
  float* dC = sc<float>(off_dC);
  float* part = sc<float>(off_part);
  const int nq = kind == K_MILSTM ? 4 : 1;

  GateParams gp;
  gp.b = p("b");
  if (kind == K_MILSTM) { gp.alpha = p("alpha"); gp.beta1 = p("beta1"); gp.beta2 = p("beta2"); }

  copy_f32_pad(dcT, B, H, H, dC, Hp, H, st);

  // a5: BPTT chain
  mark(R_BPTT, 0, st);
  GemmSpec bp;
  bp.A = mat(Duh, NG, B, NG, T, (long)B * NG);
  bp.B = mat(Um, Hp, NG, Hp);
  bp.b_mn = true;
  bp.M = B; bp.N = Hp; bp.K = NG;
  for (int t = T - 1; t >= 0; --t) {
    const float* dh_rec;
    long ld_dh;
    if (t == T - 1) {
      dh_rec = dhT;
      ld_dh = H;
    } else {
      run_gemm(2, bp, epi(dH, Hp, B, Hp), t + 1, 0, var.g[G_BPTT], st);
      dh_rec = dH;
      ld_dh = Hp;
    }
    const void* dyt;
    long ldy;
    bool dyf32;
    if (lm_mode) { dyt = lm_dy + (long)t * B * Hp; ldy = Hp; dyf32 = true; }
    else { dyt = (const char*)dy + (size_t)t * B * H * e; ldy = H; dyf32 = false; }
    lstm_bwd_pointwise(kind, ot, B, H, Hp, dyt, ldy, ot, dyf32, dh_rec, ld_dh, dC, WX + (long)t * B * NG,
                       UH + (long)t * B * NG, Cb + (long)(t + 1) * B * Hp, Cb + (long)t * B * Hp, gp,
                       Duh + (size_t)t * B * NG * e, Dwx + (size_t)t * B * NG * e, part, nq, t == T - 1, st);
  }
  if (dh0) run_gemm(2, bp, epi(dh0, H, B, H), 0, 0, var.g[G_BPTT], st);
  if (dc0) copy_pad(OT::F32, dC, OT::F32, B, H, Hp, dc0, H, st);
  mark(R_BPTT, 1, st);

  // a6: weight gradients and input dgrad
  mark(R_SE4, 0, st);
  cudaStream_t st_u = st;
  if (var.wg_side && !side.empty()) {
    CUDA_TRY(cudaEventRecord(ev_fork, st));
    CUDA_TRY(cudaStreamWaitEvent(side[0], ev_fork, 0));
    st_u = side[0];
  }
  GemmSpec gu;
  gu.A = mat(Hrow(0), Hp, TB, Hp);
  gu.a_mn = true;
  gu.B = mat(Duh, NG, TB, NG);
  gu.b_mn = true;
  gu.M = Hp; gu.N = NG; gu.K = (int)TB;
  if (st_u == st) mark(R_DU, 0, st);
  run_gemm(4, gu, epi(g("U"), 4L * H, H, NG, 0, nullptr, GATE_U, H), 0, 0, var.g[G_DU], st_u);
  if (st_u == st) mark(R_DU, 1, st);

  GemmSpec gw;
  gw.A = mat(X, I, TB, Ip);
  gw.a_mn = true;
  gw.B = mat(Dwx, NG, TB, NG);
  gw.b_mn = true;
  gw.M = I; gw.N = NG; gw.K = (int)TB;
  mark(R_DW, 0, st);
  run_gemm(5, gw, epi(g("W"), 4L * H, I, NG, 0, nullptr, GATE_U, H), 0, 0, var.g[G_DW], st);
  mark(R_DW, 1, st);

  if (dx) {
    GemmSpec gx;
    gx.A = mat(Dwx, NG, TB, NG);
    gx.B = mat(Wm, I, NG, Ip);
    gx.b_mn = true;
    gx.M = (int)TB; gx.N = I; gx.K = NG;
    mark(R_DX, 0, st);
    if (lm_mode)
      run_gemm(6, gx, epi(dx, Ip, (int)TB, I), 0, 0, var.g[G_DX], st);
    else
      run_gemm(6, gx, epi(dx, I, (int)TB, I, ot == OT::BF16), 0, 0, var.g[G_DX], st);
    mark(R_DX, 1, st);
  }
  float* gq[4] = {g("b"), nullptr, nullptr, nullptr};
  if (kind == K_MILSTM) { gq[1] = g("alpha"); gq[2] = g("beta1"); gq[3] = g("beta2"); }
  reduce_gate_partials(part, nchunk, nq, H, Hp, gq, st);
  if (st_u != st) {
    CUDA_TRY(cudaEventRecord(ev_join, st_u));
    CUDA_TRY(cudaStreamWaitEvent(st, ev_join, 0));
  }
  mark(R_SE4, 1, st);
  if (world > 1 && !lm_mode) allreduce_grads(G, n_params, st);
  if (!lm_mode) mark(R_STEP, 1, st);
}

void Cell::allreduce_grads(float* grads, size_t n, cudaStream_t after) {
  ASTRA_CHECK_STATE(nccl_comm, "allreduce: astra_comm_init not called");
  cudaStream_t cs = comm_st ? comm_st : after;
  if (cs != after) {
    CUDA_TRY(cudaEventRecord(ev_fork, after));
    CUDA_TRY(cudaStreamWaitEvent(cs, ev_fork, 0));
  }
  ncclResult_t r = ncclAllReduce(grads, grads, n, ncclFloat, ncclSum, (ncclComm_t)nccl_comm, cs);
  if (r != ncclSuccess) throw Error(ASTRA_E_NCCL, std::string("ncclAllReduce: ") + ncclGetErrorString(r));
  count_launch();
  scale_inplace(grads, n, 1.0f / (float)world, cs);
  if (cs != after) {
    CUDA_TRY(cudaEventRecord(ev_join, cs));
    CUDA_TRY(cudaStreamWaitEvent(after, ev_join, 0));
  }
}

void Cell::sgd_step(float lr) {
  ASTRA_CHECK_STATE(bound, "sgd: not bound");
  sgd(P, G, n_params, lr, main_st);
}

// ------------------------------------------------------------------------ tuner glue
// The enumerator's static pruning (A19): per GEMM role, the kernel choices whose tile
// and cluster shape fit the problem; the default (Variant()) first.
void Cell::role_shape(int role, int& M, int& N) const {
  const int TB = T * B;
  switch (role) {
    case G_A1: M = TB; N = NG; break;
    case G_REC: M = B; N = NG; break;
    case G_BPTT: M = B; N = Hp; break;
    case G_DU: M = Hp; N = NG; break;
    case G_DW: M = I; N = NG; break;
    case G_DX: M = TB; N = I; break;
    default: M = TB; N = lm_V > 0 ? lm_V : Hp; break;
  }
}

static const KCfg CANDIDATES[] = {{256, 1, 1}, {128, 1, 1}, {64, 1, 1}, {256, 2, 1}, {256, 4, 1}, {256, 2, 2},
                                  {256, 1, 2}, {128, 2, 1}, {128, 4, 1}, {128, 2, 2}, {128, 1, 2}, {64, 2, 1},
                                  {64, 4, 1}, {64, 2, 2}};

void Cell::tuner_setup() {
  const Variant def;
  std::string par;
  const char* metric[G_ROLES] = {"t_a1", "t_fwd", "t_bptt", "t_du", "t_dw", "t_dx", "t_head"};
  if (ot == OT::BF16) {
    for (int r = 0; r < G_ROLES; ++r) {
      if (r == G_HEAD && !lm_mode) continue;
      int M, N;
      role_shape(r, M, N);
      allowed[r].clear();
      allowed[r].push_back(def.g[r]);
      for (const KCfg& k : CANDIDATES) {
        if (k == def.g[r]) continue;
        const int num_m = cdiv(M, TC_BM), num_n = cdiv(N, k.bn);
        if (k.bn > 64 && N <= k.bn / 2) continue;                                     // tile wider than N
        if (k.cm > num_m || k.cn > num_n) continue;                                    // idle cluster ranks
        allowed[r].push_back(k);
      }
      par += std::string(" (leaf g_") + ROLE_NAMES[r] + " " + std::to_string(allowed[r].size()) + " " + metric[r] + ")";
    }
  }
  std::string t = par.empty() ? "" : "(par" + par + ")";
  if (!side.empty()) t = t.empty() ? "(leaf wg_side 2 t_se4)" : "(pre " + t + " (leaf wg_side 2 t_se4))";
  if (t.empty()) t = "(leaf none 1 t_step)";
  tree.reset(new tuner::Tree(tuner::parse(t)));
  wirer.reset(new tuner::Wirer(tree.get()));
  wirer->start();
  configs_seen.clear();
  tuner::Config c;
  if (wirer->propose(c)) apply_config(c);
  rep_i = 0;
}

void Cell::apply_config(const tuner::Config& c) {
  Variant v = var;
  for (size_t i = 0; i < tree->avs.size(); ++i) {
    const std::string& n = tree->avs[i];
    const int o = c[i];
    if (n == "wg_side") { v.wg_side = o; continue; }
    for (int r = 0; r < G_ROLES; ++r)
      if (n == std::string("g_") + ROLE_NAMES[r]) v.g[r] = allowed[r].at(o);
  }
  var = v;
  configs_seen.push_back(v);
}

static float elapsed(cudaEvent_t a, cudaEvent_t b) {
  float ms = 0.f;
  if (cudaEventElapsedTime(&ms, a, b) != cudaSuccess) {
    cudaGetLastError();
    return 1e30f;
  }
  return ms;
}

// One call per step (after the step's work is enqueued).  Per configuration: one warm-up step
// (absorbs lazy tensor-map creation), then tune_reps measured steps whose region times are min-
// reduced (reading R19: clocks float on B200 so k = 3 reps instead of the paper's pinned clocks,
// P:457).  Only the measured steps synchronise on their own end event.
int Cell::tune_next() {
  if (tune_mode != ASTRA_TUNE_ON) return tune_mode == ASTRA_TUNE_FROZEN ? ASTRA_TUNE_CONVERGED : ASTRA_TUNE_IDLE;
  if (!wirer) tuner_setup();
  if (wirer->converged()) return ASTRA_TUNE_CONVERGED;
  if (rep_i == 0) {  // warm-up step done
    rep_i = 1;
    return ASTRA_TUNE_EXPLORING;
  }
  CUDA_TRY(cudaEventSynchronize(ev[R_STEP][1]));
  tuner::Metrics m(tree->metrics.size(), 0.0);
  for (size_t i = 0; i < tree->metrics.size(); ++i) {
    const std::string& n = tree->metrics[i];
    double v = 0;
    if (n == "t_a1") v = elapsed(ev[R_A1][0], ev[R_A1][1]);
    else if (n == "t_fwd") v = elapsed(ev[R_FWD][0], ev[R_FWD][1]);
    else if (n == "t_bptt") v = elapsed(ev[R_BPTT][0], ev[R_BPTT][1]);
    else if (n == "t_du") v = region_used[R_DU] ? elapsed(ev[R_DU][0], ev[R_DU][1]) : 0;
    else if (n == "t_dw") v = region_used[R_DW] ? elapsed(ev[R_DW][0], ev[R_DW][1]) : 0;
    else if (n == "t_dx") v = region_used[R_DX] ? elapsed(ev[R_DX][0], ev[R_DX][1]) : 0;
    else if (n == "t_head") v = region_used[R_HEAD] ? elapsed(ev[R_HEAD][0], ev[R_HEAD][1]) : 0;
    else if (n == "t_se4") v = elapsed(ev[R_SE4][0], ev[R_SE4][1]);
    else v = elapsed(ev[R_STEP][0], ev[R_STEP][1]);
    m[i] = v;
  }
  if (rep_i == 1) rep_min = m;
  else
    for (size_t i = 0; i < m.size(); ++i) rep_min[i] = std::min(rep_min[i], m[i]);
  if (rep_i < tune_reps) {
    ++rep_i;
    return ASTRA_TUNE_EXPLORING;
  }
  wirer->feed(rep_min);
  rep_i = 0;
  tuner::Config c;
  if (wirer->propose(c)) {
    apply_config(c);
    return ASTRA_TUNE_EXPLORING;
  }
  apply_config(wirer->final_config());
  configs_seen.pop_back();
  return ASTRA_TUNE_CONVERGED;
}

std::string Cell::report() {
  std::ostringstream o;
  o << "{\"variant\": \"" << var.str() << "\", \"mode\": " << tune_mode;
  if (wirer) {
    o << ", \"converged\": " << (wirer->converged() ? "true" : "false") << ", \"configs_explored\": "
      << wirer->trials() << ", \"steps_per_config\": " << (1 + tune_reps) << ", \"index_entries\": "
      << wirer->index().d.size() << ", \"tree_avs\": [";
    for (size_t i = 0; i < tree->avs.size(); ++i) o << (i ? ", " : "") << "\"" << tree->avs[i] << "\"";
    o << "], \"index\": {";
    size_t k = 0;
    for (auto& kv : wirer->index().d) o << (k++ ? ", " : "") << "\"" << kv.first << "\": " << kv.second;
    o << "}";
  }
  o << "}";
  return o.str();
}

// ======================================================================== LM
LM::LM(Cell* c, int vocab) : cell(c), V(vocab) {
  ASTRA_CHECK_ARG(vocab > 1, "lm: vocab must be > 1");
  Vp = (int)round_up(V, 8);
  c->lm_V = V;
  params = c->params;
  n_cell = c->n_params;
  n_params = n_cell;
  auto add = [&](const char* n, int r, int cc) {
    params.push_back({n, n_params, r, cc});
    n_params = align_up(n_params + (size_t)r * cc, 64);
  };
  add("E", V, c->I);
  add("W_o", c->Hout, V);
  add("b_o", 1, V);
  const long TB = (long)c->T * c->B;
  const size_t e = c->esz();
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = align_up(o + bytes, 256); return r; };
  off_cellsaved = take(c->saved_bytes);
  off_cellscratch = take(c->scratch_bytes);
  off_logits = take((size_t)TB * V * 4);
  off_dlog = take((size_t)TB * Vp * e);
  off_dlog32 = take((size_t)TB * V * 4);
  off_rowloss = take((size_t)TB * 4);
  off_dY = take((size_t)TB * c->Hp * 4);
  off_Wo = take((size_t)round_up(V, 256) * c->Hp * e);
  off_colsum = take(colsum_scratch_floats(TB, V) * 4);
  sort_bytes = embed_bwd_scratch_bytes(TB, V);
  off_sort = take(sort_bytes);
  off_h = take((size_t)c->B * c->H * 4);
  off_c = take((size_t)c->B * c->H * 4);
  off_loss = take(256);
  // dX (fp32) for the embedding backward
  size_t off_dx = take((size_t)TB * c->Ip * 4);
  c->off_dXf = off_dx;  // offset within the LM workspace
  ws_bytes = o;
}

size_t LM::find(const std::string& n) const {
  for (auto& p : params)
    if (p.name == n) return p.offset;
  throw Error(ASTRA_E_ARG, "no parameter " + n);
}

void LM::bind(float* pp, float* gg, void* w) {
  ASTRA_CHECK_ARG(pp && gg && w, "lm_bind: null pointer");
  P = pp; G = gg; ws = (char*)w;
  cell->lm_mode = true;
  cell->bind(pp, gg, ws + off_cellsaved, ws + off_cellscratch);
  CUDA_TRY(cudaMemsetAsync(ws + off_h, 0, (size_t)cell->B * cell->H * 4, cell->main_st));
  CUDA_TRY(cudaMemsetAsync(ws + off_c, 0, (size_t)cell->B * cell->H * 4, cell->main_st));
  bound = true;
}

void LM::set_state(const float* h, const float* c) {
  ASTRA_CHECK_STATE(bound, "lm_set_state: not bound");
  const size_t n = (size_t)cell->B * cell->H * 4;
  cudaStream_t st = cell->main_st;
  if (h) CUDA_TRY(cudaMemcpyAsync(ws + off_h, h, n, cudaMemcpyDeviceToDevice, st));
  else CUDA_TRY(cudaMemsetAsync(ws + off_h, 0, n, st));
  if (c) CUDA_TRY(cudaMemcpyAsync(ws + off_c, c, n, cudaMemcpyDeviceToDevice, st));
  else CUDA_TRY(cudaMemsetAsync(ws + off_c, 0, n, st));
}

void LM::step(const int32_t* tokens, float lr, float* loss_dev, bool do_sgd) {
  ASTRA_CHECK_STATE(bound, "lm_train_step: not bound");
  ASTRA_CHECK_ARG(tokens, "lm_train_step: tokens is null");
  Cell& c = *cell;
  cudaStream_t st = c.main_st;
  const long TB = (long)c.T * c.B;
  const int Hp = c.Hp;
  float* hs = (float*)(ws + off_h);
  float* cs = (float*)(ws + off_c);
  float* logits = (float*)(ws + off_logits);
  void* dlog = ws + off_dlog;
  float* dlog32 = (float*)(ws + off_dlog32);
  float* rowloss = (float*)(ws + off_rowloss);
  float* dY = (float*)(ws + off_dY);
  void* Wom = ws + off_Wo;
  float* dX = (float*)(ws + c.off_dXf);
  float* lossp = loss_dev ? loss_dev : (float*)(ws + off_loss);

  // a0: embedding gather into the cell's operand buffer
  embed_gather(c.ot, tokens, TB, P + find("E"), c.I, c.sv<char>(c.off_X), c.Ip, st);
  // cell forward (SE1); final state carried for the next step (truncated BPTT)
  c.forward(nullptr, hs, cs, nullptr, hs, cs);

  // a4: head forward + CE + head backward (SE2)
  c.mark(R_HEAD, 0, st);
  mirror_T(c.ot, P + find("W_o"), c.H, V, (int)round_up(V, 256), Hp, Wom, Hp, st);
  GemmSpec hd;
  hd.A = mat(c.Hrow(1), Hp, TB, Hp);
  hd.B = mat(Wom, Hp, V, Hp);
  hd.M = (int)TB; hd.N = V; hd.K = Hp;
  c.run_gemm(7, hd, epi(logits, V, (int)TB, V, 0, P + find("b_o")), 0, 0, c.var.g[G_HEAD], st);
  ce_fwd_bwd(c.ot, logits, V, V, tokens + c.B, TB, 1.0f / (float)TB, rowloss, dlog, Vp, dlog32, st);
  sum_rows_to_scalar(rowloss, TB, 1.0f / (float)TB, lossp, st);
  GemmSpec dy;
  dy.A = mat(dlog, V, TB, Vp);
  dy.B = mat(Wom, Hp, V, Hp);
  dy.b_mn = true;
  dy.M = (int)TB; dy.N = Hp; dy.K = V;
  c.run_gemm(8, dy, epi(dY, Hp, (int)TB, Hp), 0, 0, c.var.g[G_HEAD], st);
  GemmSpec dwo;
  dwo.A = mat(c.Hrow(1), Hp, TB, Hp);
  dwo.a_mn = true;
  dwo.B = mat(dlog, V, TB, Vp);
  dwo.b_mn = true;
  dwo.M = Hp; dwo.N = V; dwo.K = (int)TB;
  c.run_gemm(9, dwo, epi(G + find("W_o"), V, c.H, V), 0, 0, c.var.g[G_HEAD], st);
  colsum(dlog32, TB, V, V, (float*)(ws + off_colsum), G + find("b_o"), st);
  c.mark(R_HEAD, 1, st);

  // cell backward (SE3 + SE4)
  c.lm_dy = dY;
  c.backward(nullptr, nullptr, nullptr, dX, nullptr, nullptr);
  embed_bwd(tokens, TB, V, dX, c.Ip, c.I, G + find("E"), ws + off_sort, sort_bytes, st);
  if (c.world > 1) c.allreduce_grads(G, n_params, st);
  if (do_sgd) sgd(P, G, n_params, lr, st);
  c.mark(R_STEP, 1, st);
}

}  // namespace astra
