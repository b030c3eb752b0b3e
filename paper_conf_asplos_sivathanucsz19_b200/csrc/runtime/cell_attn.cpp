// LSTM with attention — the reduced GNMT model [35] (
// BASELINE configs[3]; reading R10): a 1-layer LSTM encoder over Ts source steps and a 1-layer
// attentive LSTM decoder over Tt target steps with input feeding, A = H, decoder initialised from
// the encoder's final state, y_i = [h_i | ctx_i].
//
//   encoder: the LSTM plan of cell_lstm.cpp (an internal LstmCell sharing our params/grads)
//   keys:    K = enc·W_k (K1, hoisted)                                                   (row a2)
//   decoder: WXd = Xd·W_d (K1, hoisted); for i: z = [h_{i−1} | ctx_{i−1}]·[U_d; C_d] (one
//            K-concatenated K1 GEMM, the P:190-196 ladder) → LSTM gates → h_i; q_i = h_i·W_q (K1);
//            attention step (K3): e = vᵀtanh(q + k_j), p = softmax, ctx = Σ p_j enc_j      (a3, a3′)
//   BPTT:    [dh | dctx]_rec = da_{i+1}·[U_d; C_d]ᵀ; attention backward (K3); dh += dq·W_qᵀ
//            (K1, accumulated); LSTM cell backward; then the weight gradients, the keys backward
//            (dW_k, denc += dk·W_kᵀ) and the encoder BPTT driven by denc.                   (a5, a6)
#include "../kernels/cell_math.cuh"
#include "../kernels/rec_fused.h"
#include "cell.h"

namespace astra {

std::unique_ptr<Cell> make_lstm_cell(const astra_cell_desc& d);

class AttnCell : public Cell {
 public:
  int Ts, A, Ap, NG, nchunk;
  std::unique_ptr<Cell> enc;
  size_t off_encsaved, off_encscratch;
  size_t off_Encf, off_Keys, off_Xd, off_WXd, off_UHd, off_Cd, off_HC, off_Q, off_Pr, off_MWd, off_MUC, off_MWq,
      off_MWk, off_he, off_ce;
  size_t off_DA, off_dHC, off_dC, off_DQ, off_denc, off_DKf, off_DK, off_dvb, off_part, off_dh0e, off_dc0e,
      off_colsum, off_att, off_dctxs, off_des;

  // Reading R42: the decoder's per-step BPTT GEMM [dh | dctx]_rec = da·[U_d; C_d]ᵀ (M = B, K = 4Hp)
  // gets a fixed split-K like R25 — K chunks accumulated from zero, summed in chunk order by the
  // attention backward (ctx part) and the pointwise kernel (h part; the dq·W_qᵀ GEMM split the same
  // way, chunk k accumulated into partial k) — at cfg4 (K = 4096) 4 chunks of 16 k-blocks on 4× the
  // CTAs (bf16 path; the same for every variant)
  int bptt_ksplit() const { return ot != OT::BF16 ? 1 : NG >= 4096 ? 4 : NG >= 2048 ? 2 : 1; }

  explicit AttnCell(const astra_cell_desc& dd) : Cell(dd) {
    Ts = d.src_seq;
    A = d.attn_dim;
    ASTRA_CHECK_ARG(Ts > 0 && A > 0, "attention: src_seq and attn_dim must be positive");
    Hp = (int)round_up(H, GATE_U);
    Ap = (int)round_up(A, 64);
    NG = 4 * Hp;
    Hout = 2 * H;
    astra_cell_desc de = d;
    de.cell_type = ASTRA_LSTM;
    de.seq = Ts;
    enc = make_lstm_cell(de);
    // the encoder's W, U, b coincide with our first three tensors (same shapes, same alignment)
    add_param("W_e", I, 4 * H);
    add_param("U_e", H, 4 * H);
    add_param("b_e", 1, 4 * H);
    add_param("W_k", H, A);
    add_param("W_d", I, 4 * H);
    add_param("U_d", H, 4 * H);
    add_param("C_d", H, 4 * H);
    add_param("b_d", 1, 4 * H);
    add_param("W_q", H, A);
    add_param("v", 1, A);
    const size_t e = esz();
    const size_t SB = (size_t)Ts * B, TB = (size_t)T * B;
    Carve s;
    off_encsaved = s.take(enc->saved_bytes);
    off_Encf = s.take(SB * Hp * 4);
    off_Keys = s.take(SB * Ap * 4);
    off_Xd = s.take(TB * Ip * e);
    off_WXd = s.take(TB * NG * 4);
    off_UHd = s.take(TB * NG * 4);
    off_Cd = s.take((TB + B) * Hp * 4);
    off_HC = s.take((TB + B) * 2 * Hp * e);
    off_Q = s.take(TB * Ap * 4);
    off_Pr = s.take(TB * Ts * 4);
    off_MWd = s.take((size_t)NG * Ip * e);
    off_MUC = s.take((size_t)NG * 2 * Hp * e);
    off_MWq = s.take((size_t)Ap * Hp * e);
    off_MWk = s.take((size_t)Ap * Hp * e);
    off_he = s.take((size_t)B * H * 4);
    off_ce = s.take((size_t)B * H * 4);
    saved_bytes = s.o;
    nchunk = lstm_bwd_row_chunks(B);
    Carve c;
    off_encscratch = c.take(enc->scratch_bytes);
    off_DA = c.take(TB * NG * e);
    off_dHC = c.take((size_t)bptt_ksplit() * B * 2 * Hp * 4);   // the split-K partials of [dh | dctx]_rec
    off_dC = c.take((size_t)B * Hp * 4);
    off_DQ = c.take(TB * Ap * e);
    off_denc = c.take(SB * Hp * 4);
    off_DKf = c.take(SB * Ap * 4);
    off_DK = c.take(SB * Ap * e);
    off_dvb = c.take((size_t)B * Ap * 4);
    off_part = c.take((size_t)nchunk * 4 * NG * 4);
    off_dh0e = c.take((size_t)B * H * 4);
    off_dc0e = c.take((size_t)B * H * 4);
    off_colsum = c.take(colsum_scratch_floats(B, A) * 4);
    off_att = c.take((size_t)B * Ts * 4);   // attention scores / dp_j between a step's two kernels
    off_dctxs = c.take(TB * Hp * 4);        // per-step dctx and de rows for the deferred denc / dk
    off_des = c.take(TB * Ts * 4);
    scratch_bytes = c.o;
  }

  char* HC(int i) { return saved + off_HC + (size_t)i * B * 2 * Hp * esz(); }
  void* x_operand() override { return nullptr; }
  bool lm_capable() const override { return false; }   // reading R10: no vocabulary head
  Mat2 y_operand() override { return mat(HC(1), Hp, (long)T * B, 2 * Hp); }
  int y_width() const override { return 2 * Hp; }
  std::vector<KSeg> y_segments() const override { return {}; }
  void role_shape(int role, int& M, int& N) const override {
    const int TB = T * B;
    switch (role) {
      case G_A1: M = TB; N = NG; break;
      case G_REC: M = B; N = NG; break;
      case G_BPTT: M = B; N = 2 * Hp; break;
      case G_DU: M = Hp; N = NG; break;
      case G_DW: M = I; N = NG; break;
      case G_DX: M = TB; N = I; break;
      default: M = 0; N = 0; break;
    }
  }

  void sync_encoder() {
    if (enc->P != P || enc->saved != saved + off_encsaved || enc->scratch != scratch + off_encscratch)
      enc->bind(P, G, saved + off_encsaved, scratch + off_encscratch);
    enc->main_st = main_st;
    enc->side = side;
    enc->var = var;
    // the attention cell's fuse_fwd AV (bf16): bit 0 runs the encoder chain as the small-batch
    // persistent forward (fwd_mode 3, B ≤ 128); bit 1 runs each decoder step's K-concatenated
    // recurrent GEMM with the LSTM gate epilogue fused (lstm_rec_fwd_kernel, one launch per step —
    // the attention sub-step between steps rules out a persistent decoder)
    enc->var.fwd_mode = (var.fwd_mode & 1) ? 3 : 0;
  }
  // modes 0..3 (bit 0 is a no-op where the persistent encoder is unsupported: B > 128)
  int fwd_fusions() const override { return ot == OT::BF16 ? 4 : 1; }
  // the encoder runs outside the decoder-chain region: the choice is judged on the whole step
  const char* fwd_fusion_metric() const override { return "t_step"; }

  void forward(const void* x, const float* h0, const float* c0, void* y, float* hT, float* cT) override {
    ASTRA_CHECK_STATE(bound, "step_fwd: call astra_bind first");
    ASTRA_CHECK_ARG(x, "step_fwd: x is null");
    sync_encoder();
    cudaStream_t st = main_st;
    const long TB = (long)T * B, SB = (long)Ts * B;
    const size_t e = esz();
    float* Encf = sv<float>(off_Encf);
    float* Keys = sv<float>(off_Keys);
    void* Xd = sv<char>(off_Xd);
    float* WXd = sv<float>(off_WXd);
    float* UHd = sv<float>(off_UHd);
    float* Cd = sv<float>(off_Cd);
    float* Q = sv<float>(off_Q);
    float* Pr = sv<float>(off_Pr);
    char* MWd = sv<char>(off_MWd);
    char* MUC = sv<char>(off_MUC);
    char* MWq = sv<char>(off_MWq);
    char* MWk = sv<char>(off_MWk);
    float* he = sv<float>(off_he);
    float* ce = sv<float>(off_ce);
    const long ldy = 2L * H;

    mark(R_STEP, 0, st);
    // encoder (its own plan: mirrors, a1, recurrent chain); enc in fp32 for the context sums
    enc->y_f32 = Encf;
    enc->forward(x, h0, c0, nullptr, he, ce);
    // keys K = enc·W_k and the decoder's operand mirrors
    mirror_T(ot, p("W_k"), H, A, Ap, Hp, MWk, Hp, st);
    mirror_T(ot, p("W_q"), H, A, Ap, Hp, MWq, Hp, st);
    mirror_gates_T(ot, p("W_d"), I, H, Hp, MWd, Ip, st);
    mirror_gates_T(ot, p("U_d"), H, H, Hp, MUC, 2L * Hp, st, Hp);
    mirror_gates_T(ot, p("C_d"), H, H, Hp, MUC + (size_t)Hp * e, 2L * Hp, st, Hp);
    mark(R_A1, 0, st);
    GemmSpec kg;
    kg.A = enc->y_operand();
    kg.B = mat(MWk, Hp, Ap, Hp);
    kg.M = (int)SB; kg.N = Ap; kg.K = Hp;
    run_gemm(0, kg, epi(Keys, Ap, (int)SB, Ap), 0, 0, var.g[G_A1], st);
    copy_pad(ot, (const char*)x + (size_t)SB * I * e, ot, TB, I, I, Xd, Ip, st);
    GemmSpec a1;
    a1.A = mat(Xd, I, TB, Ip);
    a1.B = mat(MWd, I, NG, Ip);
    a1.M = (int)TB; a1.N = NG; a1.K = I;
    run_gemm(1, a1, epi(WXd, NG, (int)TB, NG), 0, 0, var.g[G_A1], st);
    mark(R_A1, 1, st);

    // decoder chain
    mark(R_FWD, 0, st);
    copy_pad(ot, he, OT::F32, B, H, H, HC(0), 2L * Hp, st, Hp);
    copy_pad(ot, nullptr, OT::F32, B, 0, 0, HC(0) + (size_t)Hp * e, 2L * Hp, st, Hp);
    copy_pad(OT::F32, ce, OT::F32, B, H, H, Cd, Hp, st);
    GateParams gp;
    gp.b = p("b_d");
    GemmSpec rec;
    rec.A = mat(HC(0), 2L * Hp, B, 2L * Hp, T + 1, (long)B * 2 * Hp);
    rec.B = mat(MUC, 2L * Hp, NG, 2L * Hp);
    rec.M = B; rec.N = NG; rec.K = 2 * Hp;
    rec.b_keep = true;
    GemmSpec qg;
    qg.A = mat(HC(0), Hp, B, 2L * Hp, T + 1, (long)B * 2 * Hp);
    qg.B = mat(MWq, Hp, Ap, Hp);
    qg.M = B; qg.N = Ap; qg.K = Hp;
    // K2 fused decoder step (fuse_fwd bit 1): the same MMAs in the same K order as the K1 GEMM below
    // and cell_math.cuh's gate arithmetic on the bf16 path, so the same bits (R17)
    const bool fused_dec = ot == OT::BF16 && (var.fwd_mode & 2);
    const bool dec_persist = fused_dec && lstm_fwd_persist_supported(B, Hp);   // B ≤ 128: 16-unit tiles
    RecPersistArgs pa{};
    if (dec_persist) {
      pa.B = B; pa.H = H; pa.Hp = Hp; pa.NG = NG; pa.T = T;
      pa.WX = WXd; pa.UH = UHd; pa.C = Cd; pa.Hb = (__nv_bfloat16*)HC(0);
      pa.y = y; pa.ldy = ldy; pa.y_kind = y ? 1 : 0;
      pa.gp = gp;
      pa.flags = nullptr;   // one step per launch: no grid barrier, the counter is never touched
      pa.K = 2 * Hp;
      pa.max_resident = 0;
      pa.b_old = 1;   // MUC is mirrored at the start of forward, many launches before the decoder chain
    }
    RecFwdArgs ra{};
    const TcGemm* tg = nullptr;
    if (fused_dec && !dec_persist) {
      tg = &tc_get(2, rec, KCfg{256, 1, 1}, true);
      ra.B = B; ra.H = H; ra.Hp = Hp; ra.NG = NG; ra.T = T;
      ra.num_m = cdiv(B, TC_BM); ra.num_n = NG / 256;
      ra.idesc = tg->args.idesc;
      ra.WX = WXd; ra.UH = UHd; ra.C = Cd; ra.Hb = (__nv_bfloat16*)HC(0);
      ra.y = y; ra.ldy = ldy; ra.y_kind = y ? 1 : 0;
      ra.gp = gp;
      ra.persistent = 0;
      ra.K = 2 * Hp;
      ra.ldh = 2L * Hp;
    }
    for (int i = 0; i < T; ++i) {
      float* UHi = UHd + (long)i * B * NG;
      const bool last = i == T - 1;
      if (dec_persist) {
        pa.t0 = i; pa.t1 = i + 1;
        pa.hT = last ? hT : nullptr;
        pa.cT = last ? cT : nullptr;
        lstm_fwd_persist_launch(K_LSTM, HC(0), MUC, T, pa, st);
      } else if (fused_dec) {
        ra.t0 = i; ra.t1 = i + 1;
        ra.hT = last ? hT : nullptr;
        ra.cT = last ? cT : nullptr;
        lstm_rec_fwd_launch(K_LSTM, tg->mapA, tg->mapB, ra, st);
      } else {
        run_gemm(2, rec, epi(UHi, NG, B, NG), i, 0, var.g[G_REC], st);
        lstm_fwd_pointwise(K_LSTM, ot, B, H, Hp, WXd + (long)i * B * NG, UHi, gp, Cd + (long)i * B * Hp,
                           Cd + (long)(i + 1) * B * Hp, HC(i + 1), 2L * Hp,
                           y ? (char*)y + (size_t)i * B * ldy * e : nullptr, ldy, ot, last ? hT : nullptr,
                           last ? cT : nullptr, st);
      }
      float* Qi = Q + (long)i * B * Ap;
      run_gemm(3, qg, epi(Qi, Ap, B, Ap), i + 1, 0, var.g[G_REC], st);
      attn_fwd(ot, B, Ts, H, Hp, A, Ap, Qi, Keys, p("v"), Encf, Pr + (long)i * B * Ts, sc<float>(off_att), HC(i + 1) + (size_t)Hp * e,
               2L * Hp, y ? (char*)y + ((size_t)i * B * ldy + H) * e : nullptr, ldy, st);
    }
    mark(R_FWD, 1, st);
    fwd_done = true;
  }

  void backward(const void* dy, const float* dhT, const float* dcT, void* dx, float* dh0, float* dc0) override {
    ASTRA_CHECK_STATE(bound && fwd_done, "step_bwd: needs a preceding step_fwd");
    ASTRA_CHECK_ARG(dy, "step_bwd: dy is null");
    sync_encoder();
    cudaStream_t st = main_st;
    const long TB = (long)T * B, SB = (long)Ts * B;
    const size_t e = esz();
    float* Encf = sv<float>(off_Encf);
    float* Keys = sv<float>(off_Keys);
    void* Xd = sv<char>(off_Xd);
    float* WXd = sv<float>(off_WXd);
    float* UHd = sv<float>(off_UHd);
    float* Cd = sv<float>(off_Cd);
    float* Q = sv<float>(off_Q);
    float* Pr = sv<float>(off_Pr);
    char* MWd = sv<char>(off_MWd);
    char* MUC = sv<char>(off_MUC);
    char* MWq = sv<char>(off_MWq);
    char* MWk = sv<char>(off_MWk);
    char* DA = sc<char>(off_DA);
    float* dHC = sc<float>(off_dHC);
    float* dC = sc<float>(off_dC);
    char* DQ = sc<char>(off_DQ);
    float* denc = sc<float>(off_denc);
    float* DKf = sc<float>(off_DKf);
    char* DK = sc<char>(off_DK);
    float* dvb = sc<float>(off_dvb);
    float* part = sc<float>(off_part);
    float* dh0e = sc<float>(off_dh0e);
    float* dc0e = sc<float>(off_dc0e);
    const long ldy = 2L * H;
    const long ld2 = 2L * Hp;

    mark(R_BPTT, 0, st);
    copy_pad(OT::F32, dhT, OT::F32, B, H, H, dHC, ld2, st);   // h-part = dhT, ctx-part = 0
    copy_pad(OT::F32, dcT, OT::F32, B, H, H, dC, Hp, st);
    GateParams gp;
    gp.b = p("b_d");
    GemmSpec bp;                       // [dh | dctx]_rec = da_{i+1}·[U_d; C_d]ᵀ
    bp.A = mat(DA, NG, B, NG, T, (long)B * NG);
    bp.B = mat(MUC, ld2, NG, ld2);
    bp.b_mn = true;
    bp.M = B; bp.N = (int)ld2; bp.K = NG;
    bp.b_keep = true;
    GemmSpec bp0 = bp;                 // the decoder's initial-state gradient (once, no split)
    const int nsp = bptt_ksplit();
    bp.ksplit = nsp;
    const long sstr = (long)B * ld2;   // partial k of [dh | dctx]_rec at dHC + k·sstr
    EpiStore ebp = epi(dHC, ld2, B, (int)ld2);
    ebp.split_stride = sstr;
    GemmSpec dqw;                      // dh += dq·W_qᵀ
    dqw.A = mat(DQ, Ap, B, Ap, T, (long)B * Ap);
    dqw.B = mat(MWq, Hp, Ap, Hp);
    dqw.b_mn = true;
    dqw.M = B; dqw.N = Hp; dqw.K = Ap;
    // R42: split like bp — K chunk k of dq·W_qᵀ accumulates into partial k of dh_rec, so partial k =
    // bp_k + dqw_k and the pointwise kernel sums them in chunk order (the last step, which has no
    // bp partials yet, runs it unsplit onto dhT)
    GemmSpec dqw0 = dqw;
    dqw.ksplit = nsp;
    EpiStore edq = accum(epi(dHC, ld2, B, Hp));
    edq.split_stride = sstr;
    for (int i = T - 1; i >= 0; --i) {
      // the last step starts from dhT (one "partial": no GEMM yet), the others from the split GEMM
      const int ns_i = i < T - 1 ? nsp : 1;
      if (i < T - 1) run_gemm(4, bp, ebp, i + 1, 0, var.g[G_BPTT], st);
      attn_bwd(ot, B, Ts, H, Hp, A, Ap, (const char*)dy + ((size_t)i * B * ldy + H) * e, ldy, false, dHC + Hp, ld2,
               Pr + (long)i * B * Ts, sc<float>(off_att), Q + (long)i * B * Ap, Keys, p("v"), Encf, DQ + (size_t)i * B * Ap * e,
               sc<float>(off_dctxs) + (long)i * B * Hp, sc<float>(off_des) + (long)i * B * Ts, dvb, i == T - 1, st, ns_i,
               sstr);
      if (i < T - 1) run_gemm(5, dqw, edq, i, 0, var.g[G_BPTT], st);
      else run_gemm(14, dqw0, accum(epi(dHC, ld2, B, Hp)), i, 0, var.g[G_BPTT], st);
      lstm_bwd_pointwise(K_LSTM, ot, B, H, Hp, (const char*)dy + (size_t)i * B * ldy * e, ldy, ot, false, dHC, ld2, ns_i, sstr,
                         dC, WXd + (long)i * B * NG, UHd + (long)i * B * NG, Cd + (long)(i + 1) * B * Hp,
                         Cd + (long)i * B * Hp, gp, DA + (size_t)i * B * NG * e, DA + (size_t)i * B * NG * e, part, 1,
                         i == T - 1, st);
    }
    // encoder-side attention accumulators over the T steps (same per-element order as per-step updates)
    attn_acc(ot, T, B, Ts, Hp, A, Ap, Pr, sc<float>(off_des), sc<float>(off_dctxs), Q, Keys, p("v"), denc, DKf, st);
    // decoder initial-state gradient → encoder final-state gradient
    run_gemm(13, bp0, epi(dHC, ld2, B, (int)ld2), 0, 0, var.g[G_BPTT], st);
    copy_pad(OT::F32, dHC, OT::F32, B, H, ld2, dh0e, H, st);
    copy_pad(OT::F32, dC, OT::F32, B, H, Hp, dc0e, H, st);
    mark(R_BPTT, 1, st);

    // decoder weight gradients
    mark(R_SE4, 0, st);
    const Mat2 da = mat(DA, NG, TB, NG);
    GemmSpec g1;
    g1.A = mat(HC(0), Hp, TB, ld2); g1.a_mn = true;
    g1.B = da; g1.b_mn = true;
    g1.M = Hp; g1.N = NG; g1.K = (int)TB;
    run_gemm(6, g1, epi_perm(g("U_d"), 4L * H, H, NG, GATE_U, 0, H), 0, 0, var.g[G_DU], st);
    GemmSpec g2 = g1;
    g2.A = mat(HC(0) + (size_t)Hp * e, Hp, TB, ld2);
    run_gemm(7, g2, epi_perm(g("C_d"), 4L * H, H, NG, GATE_U, 0, H), 0, 0, var.g[G_DU], st);
    GemmSpec g3;
    g3.A = mat(Xd, I, TB, Ip); g3.a_mn = true;
    g3.B = da; g3.b_mn = true;
    g3.M = I; g3.N = NG; g3.K = (int)TB;
    run_gemm(8, g3, epi_perm(g("W_d"), 4L * H, I, NG, GATE_U, 0, H), 0, 0, var.g[G_DW], st);
    float* gq[4] = {g("b_d"), nullptr, nullptr, nullptr};
    reduce_gate_partials(part, nchunk, 1, H, Hp, gq, st);
    GemmSpec g4;
    g4.A = mat(HC(1), Hp, TB, ld2); g4.a_mn = true;
    g4.B = mat(DQ, Ap, TB, Ap); g4.b_mn = true;
    g4.M = Hp; g4.N = Ap; g4.K = (int)TB;
    run_gemm(9, g4, epi(g("W_q"), A, H, A), 0, 0, var.g[G_DW], st);
    colsum(dvb, B, A, Ap, sc<float>(off_colsum), g("v"), st);
    if (dx) {
      GemmSpec gx;
      gx.A = da;
      gx.B = mat(MWd, I, NG, Ip); gx.b_mn = true;
      gx.M = (int)TB; gx.N = I; gx.K = NG;
      run_gemm(10, gx, epi((char*)dx + (size_t)SB * I * e, I, (int)TB, I, ot == OT::BF16), 0, 0, var.g[G_DX], st);
    }
    // keys backward: dW_k = encᵀ·dK, denc += dK·W_kᵀ
    copy_pad(ot, DKf, OT::F32, SB, Ap, Ap, DK, Ap, st);
    const Mat2 encop = enc->y_operand();
    GemmSpec g5;
    g5.A = encop; g5.a_mn = true;
    g5.B = mat(DK, Ap, SB, Ap); g5.b_mn = true;
    g5.M = Hp; g5.N = Ap; g5.K = (int)SB;
    run_gemm(11, g5, epi(g("W_k"), A, H, A), 0, 0, var.g[G_DW], st);
    GemmSpec g6;
    g6.A = mat(DK, Ap, SB, Ap);
    g6.B = mat(MWk, Hp, Ap, Hp); g6.b_mn = true;
    g6.M = (int)SB; g6.N = Hp; g6.K = Ap;
    run_gemm(12, g6, accum(epi(denc, Hp, (int)SB, Hp)), 0, 0, var.g[G_DX], st);
    mark(R_SE4, 1, st);

    // encoder BPTT driven by denc, from the decoder's initial-state gradient
    enc->lm_dy = denc;
    enc->backward(nullptr, dh0e, dc0e, dx, dh0, dc0);
    enc->lm_dy = nullptr;
    grad_bucket(G, n_params, st);
    grad_join(st);
    mark(R_STEP, 1, st);
  }
};

std::unique_ptr<Cell> make_attn_cell(const astra_cell_desc& d) { return std::unique_ptr<Cell>(new AttnCell(d)); }

}  // namespace astra
