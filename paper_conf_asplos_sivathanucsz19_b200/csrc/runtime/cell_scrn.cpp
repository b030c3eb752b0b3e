// SC-RNN / SCRN [22] (Fig. 1, Table 2), both precision paths.
//
//   s_t = (1−α)(x_t·Bm) + α s_{t−1};  h_t = σ(x_t·A + s_t·P + h_{t−1}·R + b_h);  y_t = [h_t | s_t]
//   (readings R5-R8: fixed α, S = H default, b_h present, dense embedding input).
//
// Plan:
//   a1   XAB = X·[A | Bm]                one N-fused GEMM (GEMMs sharing the argument X)
//   a2   s-scan (K8) over XB; then the ladder Q = XA + S·P as a GEMM accumulated onto XA
//   a3   for t: Z = h_{t−1}·R (K1); h_t = σ(Q_t + Z + b_h) (pointwise)
//   a5   for t desc: dh_rec = dz_{t+1}·Rᵀ; dz_t = (dy^h + dh_rec)·h(1−h); then DSP = DZ·Pᵀ and the reverse
//        ds scan; ds writes (1−α)·ds next to dz so that the input gradient is one K-concatenated GEMM
//        dx = [dz | (1−α)ds]·[Aᵀ; Bmᵀ]
//   a6   dR = Hᵀ·DZ, dA = Xᵀ·DZ, dP = Sᵀ·DZ, dBm = Xᵀ·(1−α)DS, db_h (fixed-order partials)
//
// Operand layout: HS [(T+1)·B][Hp + Sp] holds h (cols 0..Hp) and s (cols Hp..) side by side, so the
// LM head reads [h | s] as one K-concatenated operand; DZS [T·B][Hp + Sp] likewise holds dz and (1−α)ds.
#include <algorithm>

#include "../kernels/rec_fused.h"
#include "cell.h"

namespace astra {

class ScrnCell : public Cell {
 public:
  int S, Sp, Yw, nchunk;
  float alpha;
  size_t off_X, off_XAB, off_Sf, off_HS, off_Hf, off_MAB, off_MP, off_MR;
  size_t off_Z, off_dH, off_DZS, off_DSP, off_part, off_flags, off_Rk;

  // Reading R33: both chain GEMMs (h·R and dz·Rᵀ, K = Hp, N = Hp) split over K into s fixed chunks
  // when the batch gives few output tiles; the pointwise kernels sum the partials in chunk order.
  int chain_ksplit() const {
    const int tiles = cdiv(B, 128) * cdiv(Hp, 64), nk = cdiv(Hp, 64);
    int s = std::max(1, std::min(4, 64 / std::max(1, tiles)));
    while (s > 1 && nk / s < 4) --s;
    return s;
  }

  explicit ScrnCell(const astra_cell_desc& dd) : Cell(dd) {
    S = d.context;
    ASTRA_CHECK_ARG(S > 0, "scrn: context size must be positive");
    alpha = d.scrn_alpha;
    Sp = (int)round_up(S, 64);
    Yw = Hp + Sp;
    Hout = H + S;
    add_param("A", I, H);
    add_param("Bm", I, S);
    add_param("P", S, H);
    add_param("R", H, H);
    add_param("b_h", 1, H);
    const size_t e = esz();
    const size_t TB = (size_t)T * B;
    Carve s;
    off_X = s.take(TB * Ip * e);
    off_XAB = s.take(TB * Yw * 4);
    off_Sf = s.take((TB + B) * Sp * 4);
    off_HS = s.take((TB + B) * Yw * e);
    off_Hf = s.take((TB + B) * Hp * 4);
    off_MAB = s.take((size_t)Yw * Ip * e);
    off_MP = s.take((size_t)Hp * Sp * e);
    off_MR = s.take((size_t)Hp * Hp * e);
    saved_bytes = s.o;
    nchunk = pw_row_chunks(B);
    Carve c;
    off_Z = c.take((size_t)chain_ksplit() * B * Hp * 4);
    off_dH = c.take((size_t)chain_ksplit() * B * Hp * 4);
    off_DZS = c.take(TB * Yw * e);
    off_DSP = c.take(TB * Sp * 4);
    off_part = c.take((size_t)nchunk * Hp * 4);
    off_flags = c.take(4096);
    off_Rk = c.take((size_t)Hp * Hp * e);   // R (not transposed) bf16, K-major B of the persistent BPTT
    scratch_bytes = c.o;
  }

  char* HSrow(int t) { return saved + off_HS + (size_t)t * B * Yw * esz(); }
  // K2 fusion choices (AV fuse_fwd): 0 chain GEMM + pointwise per step, 1 the persistent fused
  // h-chain (scrn_persist.cu) when B ≤ 128
  int fwd_fusions() const override {
    return (ot == OT::BF16 && scrn_fwd_persist_supported(B, Hp, chain_ksplit())) ? 2 : 1;
  }
  // K4 fusion choices (AV fuse_bwd): 0 BPTT GEMM + pointwise per step, 1 the persistent fused h-chain
  // backward (scrn_persist.cu)
  int bwd_fusions() const override {
    return (ot == OT::BF16 && scrn_bwd_persist_supported(B, Hp, chain_ksplit(), T)) ? 2 : 1;
  }
  void* x_operand() override { return sv<char>(off_X); }
  Mat2 y_operand() override { return mat(HSrow(1), Yw, (long)T * B, Yw); }
  int y_width() const override { return Yw; }
  std::vector<KSeg> y_segments() const override { return {{0, 0, H}, {Hp, H, S}}; }
  int c_width() const override { return S; }
  void role_shape(int role, int& M, int& N) const override {
    const int TB = T * B;
    switch (role) {
      case G_A1: M = TB; N = Yw; break;
      case G_REC: M = B; N = Hp; break;
      case G_BPTT: M = B; N = Hp; break;
      case G_DU: M = Hp; N = Hp; break;
      case G_DW: M = I; N = Hp; break;
      case G_DX: M = TB; N = I; break;
      default: M = lm_mode ? TB : 0; N = lm_V; break;
    }
  }

  void forward(const void* x, const float* h0, const float* s0, void* y, float* hT, float* sT) override {
    ASTRA_CHECK_STATE(bound, "step_fwd: call astra_bind first");
    ASTRA_CHECK_ARG(lm_mode || x, "step_fwd: x is null");
    cudaStream_t st = main_st;
    const long TB = (long)T * B;
    const size_t e = esz();
    void* X = sv<char>(off_X);
    float* XAB = sv<float>(off_XAB);
    float* Sf = sv<float>(off_Sf);
    float* Hf = sv<float>(off_Hf);
    char* MAB = sv<char>(off_MAB);
    void* MP = sv<char>(off_MP);
    void* MR = sv<char>(off_MR);
    float* Z = sc<float>(off_Z);
    const long ldy = H + S;

    if (!lm_mode) mark(R_STEP, 0, st);   // an LM marks its step itself
    // operand mirrors: [A | Bm]ᵀ, Pᵀ (as [H][S]), Rᵀ
    mirror_T(ot, p("A"), I, H, Hp, Ip, MAB, Ip, st);
    mirror_T(ot, p("Bm"), I, S, Sp, Ip, MAB + (size_t)Hp * Ip * e, Ip, st);
    mirror_T(ot, p("P"), S, H, Hp, Sp, MP, Sp, st);
    mirror_T(ot, p("R"), H, H, Hp, Hp, MR, Hp, st);
    if (!lm_mode) copy_pad(ot, x, ot, TB, I, I, X, Ip, st);
    copy_pad(ot, h0, OT::F32, B, H, H, HSrow(0), Yw, st, Hp);
    copy_pad(OT::F32, h0, OT::F32, B, H, H, Hf, Hp, st);

    // a1: XAB = X·[A | Bm]
    mark(R_A1, 0, st);
    GemmSpec a1;
    a1.A = mat(X, I, TB, Ip);
    a1.B = mat(MAB, I, Yw, Ip);
    a1.M = (int)TB; a1.N = Yw; a1.K = I;
    run_gemm(0, a1, epi(XAB, Yw, (int)TB, Yw), 0, 0, var.g[G_A1], st);
    // a2: context scan, then the ladder Q = XA + S·P
    scrn_scan_fwd(ot, B, S, Sp, T, alpha, XAB + Hp, Yw, s0, Sf, HSrow(0) + (size_t)Hp * e, Yw,
                  y ? (char*)y + (size_t)H * e : nullptr, ldy, sT, st);
    GemmSpec sp;
    sp.A = mat(HSrow(1) + (size_t)Hp * e, S, TB, Yw);
    sp.B = mat(MP, S, Hp, Sp);
    sp.M = (int)TB; sp.N = Hp; sp.K = S;
    run_gemm(1, sp, accum(epi(XAB, Yw, (int)TB, Hp)), 0, 0, var.g[G_A1], st);
    mark(R_A1, 1, st);

    // a3: recurrent chain
    mark(R_FWD, 0, st);
    GemmSpec rec;
    rec.A = mat(HSrow(0), Hp, B, Yw, T + 1, (long)B * Yw);
    rec.B = mat(MR, Hp, Hp, Hp);
    rec.M = B; rec.N = Hp; rec.K = Hp;
    rec.b_keep = true;
    rec.ksplit = chain_ksplit();
    EpiStore ez = epi(Z, Hp, B, Hp);
    ez.split_stride = (long)B * Hp;
    if (var.fwd_mode == 1 && ot == OT::BF16 && scrn_fwd_persist_supported(B, Hp, rec.ksplit)) {
      ScrnPersistArgs pa{};
      pa.B = B; pa.H = H; pa.Hp = Hp; pa.T = T; pa.t0 = 0; pa.t1 = T; pa.nsplit = rec.ksplit;
      pa.Q = XAB; pa.ldq = Yw; pa.bh = p("b_h"); pa.Hf = Hf;
      pa.HS = (__nv_bfloat16*)HSrow(0); pa.ldhs = Yw;
      pa.y = y ? (__nv_bfloat16*)y : nullptr; pa.ldy = ldy; pa.hT = hT;
      pa.flags = sc<unsigned>(off_flags);
      CUDA_TRY(cudaMemsetAsync(pa.flags, 0, 4096, st));
      scrn_fwd_persist_launch(HSrow(0), Yw, MR, Tmax, pa, st);
      for (int t = 0; t < T; ++t) fwd_step_done(t, st);   // one kernel: every step is done at its end
      mark(R_FWD, 1, st);
      fwd_done = true;
      return;
    }
    for (int t = 0; t < T; ++t) {
      run_gemm(2, rec, ez, t, 0, var.g[G_REC], st);
      scrn_fwd_pw(ot, B, H, Hp, XAB + (long)t * B * Yw, Yw, Z, rec.ksplit, (long)B * Hp, p("b_h"),
                  Hf + (long)(t + 1) * B * Hp, HSrow(t + 1),
                  Yw, y ? (char*)y + (size_t)t * B * ldy * e : nullptr, ldy, t == T - 1 ? hT : nullptr, st);
      fwd_step_done(t, st);
    }
    mark(R_FWD, 1, st);
    fwd_done = true;
  }

  void backward(const void* dy, const float* dhT, const float* dsT, void* dx, float* dh0, float* ds0) override {
    ASTRA_CHECK_STATE(bound && fwd_done, "step_bwd: needs a preceding step_fwd");
    ASTRA_CHECK_ARG(lm_mode || dy, "step_bwd: dy is null");
    cudaStream_t st = main_st;
    const long TB = (long)T * B;
    const size_t e = esz();
    void* X = sv<char>(off_X);
    float* Hf = sv<float>(off_Hf);
    char* MAB = sv<char>(off_MAB);
    void* MP = sv<char>(off_MP);
    void* MR = sv<char>(off_MR);
    float* dH = sc<float>(off_dH);
    char* DZS = sc<char>(off_DZS);
    float* DSP = sc<float>(off_DSP);
    float* part = sc<float>(off_part);
    const long ldy = lm_mode ? Yw : H + S;

    // a5: h-chain BPTT
    mark(R_BPTT, 0, st);
    GemmSpec bp;
    bp.A = mat(DZS, Hp, B, Yw, T, (long)B * Yw);
    bp.B = mat(MR, Hp, Hp, Hp);
    bp.b_mn = true;
    bp.M = B; bp.N = Hp; bp.K = Hp;
    bp.b_keep = true;
    GemmSpec bp0 = bp;   // dh0 (once, no split)
    bp.ksplit = chain_ksplit();
    const bool fused = var.bwd_mode == 1 && ot == OT::BF16 && scrn_bwd_persist_supported(B, Hp, bp.ksplit, T);
    if (fused) {   // K4 fused persistent: every step of the h-chain in one launch
      char* Rk = sc<char>(off_Rk);
      CUDA_TRY(cudaMemsetAsync(Rk, 0, (size_t)Hp * Hp * e, st));
      copy_pad(ot, p("R"), OT::F32, H, H, H, Rk, Hp, st);   // rows k, columns j (padding exactly zero)
      ScrnBpttArgs ba{};
      ba.B = B; ba.H = H; ba.Hp = Hp; ba.nsplit = bp.ksplit;
      ba.dy = lm_mode ? (const void*)lm_dy : dy; ba.ldy = ldy;
      ba.dhT = dhT; ba.Hf = Hf; ba.DZ = (__nv_bfloat16*)DZS; ba.lddz = Yw; ba.part = part;
      ba.flags = sc<unsigned>(off_flags);
      CUDA_TRY(cudaMemsetAsync(ba.flags, 0, 4096, st));
      scrn_bwd_persist_launch(DZS, Yw, Rk, T, lm_mode, ba, st);
    }
    for (int t = T - 1; t >= 0 && !fused; --t) {
      const float* dh = dhT;
      long ld_dh = H;
      int nsplit = 1;
      if (t < T - 1) {
        EpiStore eh = epi(dH, Hp, B, Hp);
        eh.split_stride = (long)B * Hp;
        run_gemm(3, bp, eh, t + 1, 0, var.g[G_BPTT], st);
        dh = dH;
        ld_dh = Hp;
        nsplit = bp.ksplit;
      }
      const void* dyt = lm_mode ? (const void*)(lm_dy + (long)t * B * Yw) : (const char*)dy + (size_t)t * B * ldy * e;
      scrn_bwd_pw(ot, B, H, Hp, dyt, ldy, lm_mode, dh, ld_dh, nsplit, (long)B * Hp, Hf + (long)(t + 1) * B * Hp,
                  DZS + (size_t)t * B * Yw * e, Yw, part, t == T - 1, st);
    }
    if (dh0) run_gemm(13, bp0, epi(dh0, H, B, H), 0, 0, var.g[G_BPTT], st);
    // s-chain: DSP = DZ·Pᵀ then the reverse scan
    GemmSpec dsp;
    dsp.A = mat(DZS, Hp, TB, Yw);
    dsp.B = mat(MP, S, Hp, Sp);
    dsp.b_mn = true;
    dsp.M = (int)TB; dsp.N = S; dsp.K = Hp;
    run_gemm(4, dsp, epi(DSP, Sp, (int)TB, S), 0, 0, var.g[G_DX], st);
    const void* dys = lm_mode ? (const void*)(lm_dy + Hp) : (const char*)dy + (size_t)H * e;
    scrn_scan_bwd(ot, B, S, Sp, T, alpha, dys, ldy, lm_mode, DSP, Sp, dsT, DZS + (size_t)Hp * e, Yw, ds0, st);
    mark(R_BPTT, 1, st);

    // a6: weight gradients and the input gradient
    mark(R_SE4, 0, st);
    const Mat2 dz = mat(DZS, Hp, TB, Yw), dsa = mat(DZS + (size_t)Hp * e, S, TB, Yw);
    GemmSpec g1;
    g1.A = mat(HSrow(0), Hp, TB, Yw); g1.a_mn = true;
    g1.B = dz; g1.b_mn = true;
    g1.M = Hp; g1.N = Hp; g1.K = (int)TB;
    mark(R_DU, 0, st);
    run_gemm(5, g1, epi(g("R"), H, H, H), 0, 0, var.g[G_DU], st);
    mark(R_DU, 1, st);
    mark(R_DW, 0, st);
    GemmSpec g2;
    g2.A = mat(X, I, TB, Ip); g2.a_mn = true;
    g2.B = dz; g2.b_mn = true;
    g2.M = I; g2.N = Hp; g2.K = (int)TB;
    run_gemm(6, g2, epi(g("A"), H, I, H), 0, 0, var.g[G_DW], st);
    GemmSpec g3;
    g3.A = mat(HSrow(1) + (size_t)Hp * e, S, TB, Yw); g3.a_mn = true;
    g3.B = dz; g3.b_mn = true;
    g3.M = S; g3.N = Hp; g3.K = (int)TB;
    run_gemm(7, g3, epi(g("P"), H, S, H), 0, 0, var.g[G_DW], st);
    GemmSpec g4;
    g4.A = mat(X, I, TB, Ip); g4.a_mn = true;
    g4.B = dsa; g4.b_mn = true;
    g4.M = I; g4.N = S; g4.K = (int)TB;
    run_gemm(8, g4, epi(g("Bm"), S, I, S), 0, 0, var.g[G_DW], st);
    mark(R_DW, 1, st);
    reduce_blocked_partials(part, nchunk, 1, H, Hp, g("b_h"), st);
    if (dx) {
      GemmSpec gx;
      gx.A = mat(DZS, Yw, TB, Yw);
      gx.B = mat(MAB, I, Yw, Ip); gx.b_mn = true;
      gx.M = (int)TB; gx.N = I; gx.K = Yw;
      mark(R_DX, 0, st);
      if (lm_mode) run_gemm(9, gx, epi(dx, Ip, (int)TB, I), 0, 0, var.g[G_DX], st);
      else run_gemm(9, gx, epi(dx, I, (int)TB, I, ot == OT::BF16), 0, 0, var.g[G_DX], st);
      mark(R_DX, 1, st);
    }
    mark(R_SE4, 1, st);
    grad_bucket(G, n_params, st);   // one bucket for the cell's parameters
    if (!lm_mode) grad_join(st);
    if (!lm_mode) mark(R_STEP, 1, st);
  }
};

std::unique_ptr<Cell> make_scrn_cell(const astra_cell_desc& d) { return std::unique_ptr<Cell>(new ScrnCell(d)); }

}  // namespace astra
