// Recurrent highway network [39] with coupled carry (BASELINE configs[2]),
// both precision paths.  Reading R9: input only at micro-layer ℓ = 1, output s^L.
//
//   s^0_t = s^L_{t−1};  for ℓ = 1..L:  a = [ℓ=1]·x_t·W + s^{ℓ−1}·R_ℓ + b_ℓ;  h = tanh a_H, τ = σ(a_T);
//                                      s^ℓ = h⊙τ + s^{ℓ−1}⊙(1 − τ)
//
// Plan: a1 WX = X·W (K1) hoisted; the chain is T·L dependent micro-steps, each = one K1 GEMM
// (s·R_ℓ, N = 2H) + one pointwise kernel (a3); BPTT mirrors it with ds = ds(1−τ) + da·R_ℓᵀ
// (pointwise writes ds(1−τ), the GEMM accumulates da·R_ℓᵀ onto it); dR_ℓ = S_ℓᵀ·DA_ℓ per micro-layer.
// Internal gate layout: gate-blocked and padded, column g·Hp + j.
#include <algorithm>
#include <cstdlib>

#include "../kernels/rec_fused.h"
#include "cell.h"

namespace astra {

class RhnCell : public Cell {
 public:
  int L, G2, nchunk;
  size_t off_X, off_WX, off_Apre, off_Sf, off_Sop, off_MW, off_MR;
  size_t off_DA, off_dS, off_dSpart, off_Zpart, off_part, off_flags, off_RK;

  // Reading R33: the BPTT GEMM ds·R_ℓᵀ (K = 2·Hp, few output tiles at small batch) is split over K
  // into s fixed chunks, each accumulated from zero; the next pointwise kernel adds the partials in
  // chunk order to the carry ds·(1−τ).  Depends only on the shapes (every variant, both paths).
  int fwd_ksplit() const {   // the same rule for the recurrent GEMM s·R_ℓ (K = Hp, N = 2·Hp)
    const int tiles = cdiv(B, 128) * cdiv(2 * Hp, 64), nk = cdiv(Hp, 64);
    int s = std::max(1, std::min(4, 64 / std::max(1, tiles)));
    while (s > 1 && nk / s < 4) --s;
    return s;
  }
  int bptt_ksplit() const {
    const int tiles = cdiv(B, 128) * cdiv(Hp, 64), nk = cdiv(2 * Hp, 64);
    int s = std::max(1, std::min(4, 64 / std::max(1, tiles)));
    while (s > 1 && nk / s < 4) --s;
    return s;
  }

  explicit RhnCell(const astra_cell_desc& dd) : Cell(dd) {
    L = d.depth;
    ASTRA_CHECK_ARG(L >= 1 && L <= 64, "rhn: depth must be in 1..64");
    G2 = 2 * Hp;
    add_param("W", I, 2 * H);
    add_param("R", L * H, 2 * H);
    add_param("b", L, 2 * H);
    const size_t e = esz();
    const size_t TB = (size_t)T * B;
    Carve s;
    off_X = s.take(TB * Ip * e);
    off_WX = s.take(TB * G2 * 4);
    off_Apre = s.take((size_t)L * TB * G2 * 4);
    off_Sf = s.take((size_t)L * (TB + B) * Hp * 4);
    off_Sop = s.take((size_t)L * (TB + B) * Hp * e);
    off_MW = s.take((size_t)G2 * Ip * e);
    off_MR = s.take((size_t)L * G2 * Hp * e);
    saved_bytes = s.o;
    nchunk = pw_row_chunks(B);
    Carve c;
    off_DA = c.take((size_t)L * TB * G2 * e);
    off_dS = c.take((size_t)B * Hp * 4);
    off_dSpart = c.take((size_t)bptt_ksplit() * B * Hp * 4);
    off_Zpart = c.take((size_t)fwd_ksplit() * B * G2 * 4);
    off_part = c.take((size_t)L * nchunk * G2 * 4);
    off_flags = c.take(4096);
    off_RK = c.take((size_t)L * Hp * G2 * e);   // K-major R copy of the persistent BPTT (bwd_mode 1)
    scratch_bytes = c.o;
  }

  // state slot (ℓ, t): input of micro-step ℓ at time t; slot (0, t+1) = output of time t
  size_t slot(int l, int t) const { return ((size_t)l * (T + 1) + t) * B * Hp; }
  float* Sf(int l, int t) { return sv<float>(off_Sf) + slot(l, t); }
  char* Sop(int l, int t) { return saved + off_Sop + slot(l, t) * esz(); }
  float* Apre(int l, int t) { return sv<float>(off_Apre) + ((size_t)l * T + t) * B * G2; }
  char* DA(int l, int t) { return scratch + off_DA + ((size_t)l * T + t) * B * G2 * esz(); }

  // K2 choices (AV fuse_fwd): GEMM + pointwise launch per micro-step, or the persistent fused chain
  bool fused_fwd_ok() const { return ot == OT::BF16 && rhn_rec_fwd_supported(B, Hp, fwd_ksplit()); }
  int fwd_fusions() const override { return fused_fwd_ok() ? 2 : 1; }
  // K4 persistent BPTT (rhn_bptt_persist.cu, bwd=1): a frozen-variant option.  At cfg3 its chain is
  // faster than the launched one when both are enqueued eagerly (2.79 vs 2.94 ms) but not against the
  // CUDA-graph replay the LM steps run in (5.98 vs 5.93 ms per step, profiles/r2_cfg56.jsonl), and
  // the tuner explores eagerly — so it is not offered to the tuner.
  bool persist_bwd_ok() const {
    return ot == OT::BF16 && rhn_bptt_persist_supported(B, Hp, bptt_ksplit(), L) &&
           rhn_bptt_persist_fits(B, Hp, bptt_ksplit(), L);
  }

  void* x_operand() override { return sv<char>(off_X); }
  Mat2 y_operand() override { return mat(Sop(0, 1), Hp, (long)T * B, Hp); }
  int y_width() const override { return Hp; }
  std::vector<KSeg> y_segments() const override { return {{0, 0, H}}; }
  int c_width() const override { return 0; }
  void role_shape(int role, int& M, int& N) const override {
    const int TB = T * B;
    switch (role) {
      case G_A1: M = TB; N = G2; break;
      case G_REC: M = B; N = G2; break;
      case G_BPTT: M = B; N = Hp; break;
      case G_DU: M = Hp; N = G2; break;
      case G_DW: M = I; N = G2; break;
      case G_DX: M = TB; N = I; break;
      default: M = lm_mode ? TB : 0; N = lm_V; break;
    }
  }

  void forward(const void* x, const float* s0, const float*, void* y, float* sT, float*) override {
    ASTRA_CHECK_STATE(bound, "step_fwd: call astra_bind first");
    ASTRA_CHECK_ARG(lm_mode || x, "step_fwd: x is null");
    cudaStream_t st = main_st;
    const long TB = (long)T * B;
    const size_t e = esz();
    void* X = sv<char>(off_X);
    float* WX = sv<float>(off_WX);
    char* MW = sv<char>(off_MW);
    char* MR = sv<char>(off_MR);

    if (!lm_mode) mark(R_STEP, 0, st);   // an LM marks its step itself
    mirror_blocked_T(ot, p("W"), I, 2, H, Hp, MW, Ip, st);
    for (int l = 0; l < L; ++l)
      mirror_blocked_T(ot, p("R") + (size_t)l * H * 2 * H, H, 2, H, Hp, MR + (size_t)l * G2 * Hp * e, Hp, st);
    if (!lm_mode) copy_pad(ot, x, ot, TB, I, I, X, Ip, st);
    copy_pad(OT::F32, s0, OT::F32, B, H, H, Sf(0, 0), Hp, st);
    copy_pad(ot, s0, OT::F32, B, H, H, Sop(0, 0), Hp, st);

    mark(R_A1, 0, st);
    GemmSpec a1;
    a1.A = mat(X, I, TB, Ip);
    a1.B = mat(MW, I, G2, Ip);
    a1.M = (int)TB; a1.N = G2; a1.K = I;
    run_gemm(0, a1, epi(WX, G2, (int)TB, G2), 0, 0, var.g[G_A1], st);
    mark(R_A1, 1, st);

    mark(R_FWD, 0, st);
    GemmSpec rec;
    rec.A = mat(Sop(0, 0), Hp, B, Hp, (long)L * (T + 1), (long)B * Hp);
    rec.B = mat(MR, Hp, G2, Hp, L, (long)G2 * Hp);
    rec.M = B; rec.N = G2; rec.K = Hp;
    rec.b_keep = true;
    rec.ksplit = fwd_ksplit();
    float* Zpart = sc<float>(off_Zpart);
    EpiStore ez = epi(Zpart, G2, B, G2);
    ez.split_stride = (long)B * G2;
    if (var.fwd_mode >= 1 && fused_fwd_ok()) {   // persistent fused chain: one launch for all T·L micro-steps
      const TcGemm& g64 = tc_get(1, rec, KCfg{64, 1, 1}, true);   // for the M = 128, N = 64 instruction descriptor
      RhnFwdArgs ra{};
      ra.B = B; ra.H = H; ra.Hp = Hp; ra.T = T; ra.L = L; ra.t0 = 0; ra.t1 = T;
      ra.nsplit = rec.ksplit;
      ra.idesc = g64.args.idesc;
      ra.a_rows = B <= 64 ? 64 : TC_BM;
      CUtensorMap mA, mB;
      make_tile_map(&mA, Sop(0, 0), true, Hp, B, (long)L * (T + 1), Hp, (long)B * Hp, 64, ra.a_rows, 128);
      make_tile_map(&mB, MR, true, Hp, G2, L, Hp, (long)G2 * Hp, 64, 32, 128);
      ra.WX = WX; ra.b = p("b"); ra.Apre = Apre(0, 0); ra.Sf = Sf(0, 0); ra.Sop = (__nv_bfloat16*)Sop(0, 0);
      ra.y = (__nv_bfloat16*)y; ra.ldy = H; ra.sT = sT;
      ra.flags = sc<unsigned>(off_flags);
      CUDA_TRY(cudaMemsetAsync(ra.flags, 0, 4096, st));
      ra.trace = trace_buffer(TRACE_RHN_FWD);   // phase trace of the persistent chain (diagnostics)
      rhn_rec_fwd_launch(mA, mB, ra, st);
      for (int t = 0; t < T; ++t) fwd_step_done(t, st);
      mark(R_FWD, 1, st);
      fwd_done = true;
      return;
    }
    for (int t = 0; t < T; ++t) {
      for (int l = 0; l < L; ++l) {
        float* Z = Apre(l, t);
        if (rec.ksplit > 1) run_gemm(1, rec, ez, l * (T + 1) + t, l, var.g[G_REC], st);
        else run_gemm(1, rec, epi(Z, G2, B, G2), l * (T + 1) + t, l, var.g[G_REC], st);
        const bool last = l == L - 1;
        float* sn = last ? Sf(0, t + 1) : Sf(l + 1, t);
        char* sno = last ? Sop(0, t + 1) : Sop(l + 1, t);
        rhn_fwd_pw(ot, B, H, Hp, Z, rec.ksplit > 1 ? Zpart : nullptr, rec.ksplit, (long)B * G2,
                   l == 0 ? WX + (long)t * B * G2 : nullptr, p("b") + (size_t)l * 2 * H, Sf(l, t),
                   sn, sno, (last && y) ? (char*)y + (size_t)t * B * H * e : nullptr, H,
                   (last && t == T - 1) ? sT : nullptr, st);
      }
      fwd_step_done(t, st);
    }
    mark(R_FWD, 1, st);
    fwd_done = true;
  }

  void backward(const void* dy, const float* dsT, const float*, void* dx, float* ds0, float*) override {
    ASTRA_CHECK_STATE(bound && fwd_done, "step_bwd: needs a preceding step_fwd");
    ASTRA_CHECK_ARG(lm_mode || dy, "step_bwd: dy is null");
    cudaStream_t st = main_st;
    const long TB = (long)T * B;
    const size_t e = esz();
    void* X = sv<char>(off_X);
    char* MW = sv<char>(off_MW);
    char* MR = sv<char>(off_MR);
    float* dS = sc<float>(off_dS);
    float* part = sc<float>(off_part);
    const long ldy = lm_mode ? Hp : H;

    copy_pad(OT::F32, dsT, OT::F32, B, H, H, dS, Hp, st);
    mark(R_BPTT, 0, st);
    GemmSpec bp;
    bp.A = mat(scratch + off_DA, G2, B, G2, (long)L * T, (long)B * G2);
    bp.B = mat(MR, Hp, G2, Hp, L, (long)G2 * Hp);
    bp.b_mn = true;
    bp.M = B; bp.N = Hp; bp.K = G2;
    bp.b_keep = true;
    bp.ksplit = bptt_ksplit();
    float* dSpart = sc<float>(off_dSpart);
    EpiStore ep = epi(dSpart, Hp, B, Hp);
    ep.split_stride = (long)B * Hp;
    const bool persist = var.bwd_mode == 1 && persist_bwd_ok();
    if (persist) {   // the whole chain in one launch; R_ℓ as a K-major copy (rows = units)
      transpose_bf16(MR, L, G2, Hp, sc<char>(off_RK), st);
      RhnBpttArgs pa{};
      pa.B = B; pa.H = H; pa.Hp = Hp; pa.T = T; pa.L = L; pa.nsplit = bp.ksplit; pa.nchunk = nchunk;
      if (lm_mode) { pa.dy = lm_dy; pa.ldy = Hp; }
      else { pa.dy = dy; pa.ldy = H; }
      pa.Apre = Apre(0, 0); pa.Sf = Sf(0, 0); pa.DA = (__nv_bfloat16*)DA(0, 0); pa.dS = dS; pa.part = part;
      pa.flags = sc<unsigned>(off_flags);
      CUDA_TRY(cudaMemsetAsync(pa.flags, 0, 64, st));
      rhn_bptt_persist_launch(lm_mode, DA(0, 0), sc<char>(off_RK), pa, st);
    }
    for (int t = persist ? -1 : T - 1; t >= 0; --t) {
      for (int l = L - 1; l >= 0; --l) {
        const void* dyt = nullptr;
        if (l == L - 1)
          dyt = lm_mode ? (const void*)(lm_dy + (long)t * B * Hp) : (const char*)dy + (size_t)t * B * H * e;
        const bool top = t == T - 1 && l == L - 1;   // no GEMM before the first micro-step
        rhn_bwd_pw(ot, B, H, Hp, dS, top ? nullptr : dSpart, bp.ksplit, (long)B * Hp, dyt, ldy, lm_mode, Apre(l, t),
                   Sf(l, t), DA(l, t), dS, part + (size_t)l * nchunk * G2, t == T - 1, st);
        run_gemm(2, bp, ep, l * T + t, l, var.g[G_BPTT], st);
      }
    }
    if (!persist) add_split_partials(dS, dSpart, bp.ksplit, (long)B * Hp, st);   // ds of s^0_0
    if (ds0) copy_pad(OT::F32, dS, OT::F32, B, H, Hp, ds0, H, st);
    mark(R_BPTT, 1, st);

    mark(R_SE4, 0, st);
    // wg_side (B3 stream assignment): the L independent dR_ℓ GEMMs alternate between the
    // main and a side stream, so one GEMM's tail wave overlaps the next one's (outputs disjoint: same bits)
    cudaStream_t st_s = st;
    if (var.wg_side && !side.empty()) {
      CUDA_TRY(cudaEventRecord(ev_fork, st));
      CUDA_TRY(cudaStreamWaitEvent(side[0], ev_fork, 0));
      st_s = side[0];
    }
    if (st_s == st) mark(R_DU, 0, st);
    for (int l = 0; l < L; ++l) {
      GemmSpec gr;
      gr.A = mat(Sop(l, 0), Hp, TB, Hp); gr.a_mn = true;
      gr.B = mat(DA(l, 0), G2, TB, G2); gr.b_mn = true;
      gr.M = Hp; gr.N = G2; gr.K = (int)TB;
      run_gemm(20 + l, gr, epi_perm(g("R") + (size_t)l * H * 2 * H, 2L * H, H, G2, 0, Hp, H), 0, 0, var.g[G_DU],
               (l & 1) ? st_s : st);
    }
    if (st_s == st) mark(R_DU, 1, st);
    mark(R_DW, 0, st);
    GemmSpec gw;
    gw.A = mat(X, I, TB, Ip); gw.a_mn = true;
    gw.B = mat(DA(0, 0), G2, TB, G2); gw.b_mn = true;
    gw.M = I; gw.N = G2; gw.K = (int)TB;
    run_gemm(3, gw, epi_perm(g("W"), 2L * H, I, G2, 0, Hp, H), 0, 0, var.g[G_DW], st);
    mark(R_DW, 1, st);
    for (int l = 0; l < L; ++l)
      reduce_blocked_partials(part + (size_t)l * nchunk * G2, nchunk, 2, H, Hp, g("b") + (size_t)l * 2 * H, st);
    if (dx) {
      GemmSpec gx;
      gx.A = mat(DA(0, 0), G2, TB, G2);
      gx.B = mat(MW, I, G2, Ip); gx.b_mn = true;
      gx.M = (int)TB; gx.N = I; gx.K = G2;
      mark(R_DX, 0, st);
      if (lm_mode) run_gemm(4, gx, epi(dx, Ip, (int)TB, I), 0, 0, var.g[G_DX], st);
      else run_gemm(4, gx, epi(dx, I, (int)TB, I, ot == OT::BF16), 0, 0, var.g[G_DX], st);
      mark(R_DX, 1, st);
    }
    if (st_s != st) {   // the side stream's dR_ℓ GEMMs overlapped dW / dX
      CUDA_TRY(cudaEventRecord(ev_join, st_s));
      CUDA_TRY(cudaStreamWaitEvent(st, ev_join, 0));
    }
    mark(R_SE4, 1, st);
    grad_bucket(G, n_params, st);   // one bucket for the cell's parameters
    if (!lm_mode) grad_join(st);
    if (!lm_mode) mark(R_STEP, 1, st);
  }
};

std::unique_ptr<Cell> make_rhn_cell(const astra_cell_desc& d) { return std::unique_ptr<Cell>(new RhnCell(d)); }

}  // namespace astra
