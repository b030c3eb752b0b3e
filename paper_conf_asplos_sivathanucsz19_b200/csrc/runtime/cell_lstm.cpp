// LSTM-family cells: LSTM, MI-LSTM [36] and subLSTM [8]
// on both precision paths.
//
// Step anatomy:
//   fwd : mirrors(K9) → x copy → state init → a1 hoisted GEMM WX = X·W (K1) →
//         for t: UH_t = h_{t-1}·U (K1) ; pointwise gate epilogue (K2 half)
//   bwd : for t desc: dh_rec = D_uh[t+1]·Uᵀ (K1) ; pointwise cell backward (K4 half, K5 partials)
//         → dh0 → wgrad dU = Hᵀ·D_uh, dW = Xᵀ·D_wx (K1) → dX = D_wx·Wᵀ (K1) → bias/α/β reductions (K5)
//         → gradient sum over ranks (K11) when world > 1.
#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "../kernels/cell_math.cuh"
#include "../kernels/rec_fused.h"
#include "cell.h"

namespace astra {

class LstmCell : public Cell {
 public:
  int kind, NG, nchunk;
  size_t off_X, off_WX, off_UH, off_C, off_H, off_Wm, off_Um;
  size_t off_Duh, off_Dwx, off_dH, off_dC, off_part, off_flags, off_UHr;
  int rc_steps = 1;   // recompute variant: timesteps per recomputed UH chunk (ring of 2 chunks)
  cudaEvent_t ev_rc_done[2] = {nullptr, nullptr}, ev_rc_free[2] = {nullptr, nullptr};

  explicit LstmCell(const astra_cell_desc& dd) : Cell(dd) {
    kind = d.cell_type == ASTRA_MILSTM ? K_MILSTM : d.cell_type == ASTRA_SUBLSTM ? K_SUBLSTM : K_LSTM;
    Hp = (int)round_up(H, GATE_U);
    NG = 4 * Hp;
    add_param("W", I, 4 * H);
    add_param("U", H, 4 * H);
    add_param("b", 1, 4 * H);
    if (kind == K_MILSTM) {
      add_param("alpha", 1, 4 * H);
      add_param("beta1", 1, 4 * H);
      add_param("beta2", 1, 4 * H);
    }
    const size_t e = esz();
    const size_t TB = (size_t)T * B;
    Carve s;
    off_X = s.take(TB * Ip * e);
    off_WX = s.take(TB * NG * 4);
    off_UH = s.take(TB * NG * 4);
    off_C = s.take((TB + B) * Hp * 4);
    off_H = s.take((TB + B) * Hp * e);
    off_Wm = s.take((size_t)NG * Ip * e);
    off_Um = s.take((size_t)NG * Hp * e);
    saved_bytes = s.o;
    nchunk = lstm_bwd_row_chunks(B);
    Carve c;
    off_Duh = c.take(TB * NG * e);
    off_Dwx = kind == K_MILSTM ? c.take(TB * NG * e) : off_Duh;
    off_dH = c.take((size_t)bptt_ksplit() * B * Hp * 4);
    off_dC = c.take((size_t)B * Hp * 4);
    off_part = c.take((size_t)nchunk * 4 * NG * 4);
    off_flags = c.take(4096);
    // recompute variant (Variant::recomp): a ring of two UH chunks of rc_steps timesteps each, sized
    // so the ring stays L2-resident next to U (the forward writes UH_t into slot 0 of the ring)
    rc_steps = (int)std::max<long>(1, std::min<long>(T, (32L << 20) / ((long)B * NG * 4)));
    if (const char* ev = std::getenv("ASTRA_RC_STEPS")) rc_steps = std::max(1, std::min(T, std::atoi(ev)));   // tests
    off_UHr = c.take((size_t)2 * rc_steps * B * NG * 4);
    scratch_bytes = c.o;
  }
  ~LstmCell() override {
    for (cudaEvent_t e : ev_wgs)
      if (e) cudaEventDestroy(e);
    for (cudaEvent_t e : ev_rs)
      if (e) cudaEventDestroy(e);
    for (int i = 0; i < 2; ++i) {
      if (ev_rc_done[i]) cudaEventDestroy(ev_rc_done[i]);
      if (ev_rc_free[i]) cudaEventDestroy(ev_rc_free[i]);
    }
  }
  bool supports_recompute() const override { return true; }
  bool supports_gate_blocked() const override { return ot == OT::BF16; }
  // the `alloc` gate layout (Variant::gblk, reading R38): unit block of the gate order (cell_math.cuh
  // gcol_u) and the k-block permutation the gate-contracting GEMMs read in the canonical order with
  bool blocked() const { return var.gblk != 0 && ot == OT::BF16; }
  int gate_u() const { return blocked() ? Hp : GATE_U; }
  int kperm() const { return blocked() ? Hp / TC_BK : 0; }

  // Fixed split-K of the per-step BPTT GEMM (K = 4·Hp): with B rows the GEMM has few output tiles,
  // so each SM would stream a whole K-panel of Uᵀ; four K-chunks cut the bytes per SM 4× while the
  // chunk partials are summed in a fixed order by the pointwise kernel (identical for every variant).
  int bptt_ksplit() const { return (ot == OT::BF16 && NG >= 4096) ? 4 : (ot == OT::BF16 && NG >= 2048) ? 2 : 1; }

  // K2 fusion choices (AV fuse_fwd): 0 GEMM + pointwise, 1 fused per step (CTA pairs), 2 fused
  // persistent (256-column tiles), 3 small-batch persistent with the U slice resident (B ≤ 128)
  int gate_chunkings() const override { return ot == OT::BF16 ? (side.empty() ? 3 : 5) : 1; }
  int wgrad_schedules() const override { return (ot == OT::BF16 && T >= 4) ? 3 : 1; }
  // backward pointwise forms (AV bwd_pw): 0 row-lane, 1 wide, 2 wide with TMA-tiled operands (the LM's fp32 dY)
  int bwd_pw_forms() const override { return ot == OT::BF16 ? (lm_mode ? 3 : 2) : 1; }
  int row_stream_options() const override { return (ot == OT::BF16 && B >= 256 && B % 64 == 0) ? 2 : 1; }
  cudaEvent_t ev_rs[2] = {nullptr, nullptr};   // row_streams fork / join
  // the two row halves of the chains as independent chains on (main, side[0]): value-preserving —
  // row chunks of the same GEMMs (R1), the same per-row pointwise arithmetic, 32-row partial chunks
  bool row_split_ok(bool hooks) const {
    return var.rsp == 1 && ot == OT::BF16 && B >= 256 && B % 64 == 0 && !side.empty() && !var.recomp && !hooks;
  }
  void rs_fork(cudaStream_t st) {
    for (int i = 0; i < 2; ++i)
      if (!ev_rs[i]) CUDA_TRY(cudaEventCreateWithFlags(&ev_rs[i], cudaEventDisableTiming));
    CUDA_TRY(cudaEventRecord(ev_rs[0], st));
    CUDA_TRY(cudaStreamWaitEvent(side[0], ev_rs[0], 0));
  }
  void rs_join(cudaStream_t st) {
    CUDA_TRY(cudaEventRecord(ev_rs[1], side[0]));
    CUDA_TRY(cudaStreamWaitEvent(st, ev_rs[1], 0));
  }
  cudaEvent_t ev_wgs[11] = {};          // wgrad_schedule: chunk k's D_wx rows complete (+ join)
  int fwd_fusions() const override { return (ot == OT::BF16 && lstm_fwd_persist_supported(B, Hp)) ? 4 : 3; }
  bool chain_prefetch() const override { return true; }
  bool supports_ranges() const override { return true; }
  RecFwd2Maps fm;                       // tensor maps of the fused CTA-pair forward (built at first use)
  const void* fm_key = (const void*)1;  // y pointer the maps were built for
  const void* fm_wx = nullptr;          // workspace they were built for (rebind ⇒ rebuild)
  int fm_T = 0;                         // active length the y map was built for
  BpttFusedMaps bm;                     // tensor maps of the fused BPTT kernel
  const void* bm_key[4] = {nullptr, nullptr, nullptr, nullptr};   // (WX, dy, Duh, T) they were built for

  // K4 fusion choices (AV fuse_bwd): GEMM + pointwise kernel, or the fused BPTT kernel
  // K4 fusion choices (AV fuse_bwd): 0 GEMM + pointwise kernel, 1 the fused BPTT kernel per step.
  // bwd=2 (or 3), the small-batch persistent BPTT chain (B ≤ 128, 4 K chunks, bptt_persist.cu), is
  // a frozen-variant option only: at cfg5 B = 64 it is slower than the launched chain (2.26 vs
  // 2.03 ms per 100 steps, profiles/r2_pb_sweep23.jsonl), and its t_bptt beats the launched chain
  // measured next to wgrad_schedule's side-stream dX, which made the tuner pick it for a slower step.
  bool bptt_persist_ok() const {
    return ot == OT::BF16 && lstm_bptt_persist_supported(B, Hp, bptt_ksplit()) && lstm_bptt_persist_fits(kind, B, Hp, NG);
  }
  int bwd_fusions() const override {
    return (ot == OT::BF16 && lstm_bptt_fused_supported(B, Hp, bptt_ksplit())) ? 2 : 1;
  }

  void* Hrow(int t) { return saved + off_H + (size_t)t * B * Hp * esz(); }
  void* x_operand() override { return sv<char>(off_X); }
  Mat2 y_operand() override { return mat(Hrow(1), Hp, (long)T * B, Hp); }
  int y_width() const override { return Hp; }
  std::vector<KSeg> y_segments() const override { return {{0, 0, H}}; }
  void role_shape(int role, int& M, int& N) const override {
    const int TB = T * B;
    switch (role) {
      case G_A1: M = TB; N = NG; break;
      case G_REC: M = B; N = NG; break;
      case G_BPTT: M = B; N = Hp; break;
      case G_DU: M = Hp; N = NG; break;
      case G_DW: M = I; N = NG; break;
      case G_DX: M = TB; N = I; break;
      default: M = lm_mode ? TB : 0; N = lm_V; break;
    }
  }
  void forward(const void* x, const float* h0, const float* c0, void* y, float* hT, float* cT) override;
  void backward(const void* dy, const float* dhT, const float* dcT, void* dx, float* dh0, float* dc0) override;
};

void LstmCell::forward(const void* x, const float* h0, const float* c0, void* y, float* hT, float* cT) {
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

  // time range of this call (the layer wavefront of a stacked LM runs the forward in chunks)
  const int t0 = rg_t1 < 0 ? 0 : rg_t0, t1 = rg_t1 < 0 ? T : rg_t1;
  const bool whole = t0 == 0 && t1 == T;
  if (t0 == 0) {
    if (!lm_mode) mark(R_STEP, 0, st);   // an LM marks its step itself (embedding included)
    // K9 second half: operand mirrors in the internal gate-interleaved layout
    mirror_gates_T(ot, p("W"), I, H, Hp, Wm, Ip, st, -1, gate_u());
    mirror_gates_T(ot, p("U"), H, H, Hp, Um, Hp, st, -1, gate_u());
    if (!lm_mode) copy_pad(ot, x, ot, TB, I, I, X, Ip, st);
    copy_pad(ot, h0, OT::F32, B, H, H, Hrow(0), Hp, st);
    copy_f32_pad(c0, B, H, H, Cb, Hp, H, st);
  }

  GateParams gp;
  gp.b = p("b");
  if (kind == K_MILSTM) { gp.alpha = p("alpha"); gp.beta1 = p("beta1"); gp.beta2 = p("beta2"); }

  // a1: hoisted input projection for the range's timesteps (row chunks of one GEMM: same bits).
  // gate_chunking (§8(a.9)): the fused gate GEMM cut into nc GEMMs over ranges of whole 256-column
  // gate blocks (every output element keeps its single from-zero accumulation over K: same bits,
  // R1), alternating between the main and a side stream when ns = 2
  if (t0 == 0) mark(R_A1, 0, st);
  const long rows = (long)(t1 - t0) * B;
  const int nblk = NG / (4 * GATE_U);
  const int nc = std::min(GCHUNK_N[var.gchunk], nblk);
  const bool two = GCHUNK_S[var.gchunk] == 2 && nc > 1 && !side.empty();
  if (two) {
    CUDA_TRY(cudaEventRecord(ev_fork, st));
    CUDA_TRY(cudaStreamWaitEvent(side[0], ev_fork, 0));
  }
  for (int k = 0; k < nc; ++k) {
    // gate-interleaved: ranges of whole 256-column unit blocks; gate-blocked: whole gates (nc ∈ {1, 2, 4}:
    // G/nc gates per GEMM — the paper's G separate gate GEMMs, G/2, or one fused)
    int n0 = (int)((long)nblk * k / nc) * 4 * GATE_U, n1 = (int)((long)nblk * (k + 1) / nc) * 4 * GATE_U;
    if (blocked()) { n0 = (int)((long)NG * k / nc); n1 = (int)((long)NG * (k + 1) / nc); }
    GemmSpec a1;
    a1.A = mat((const char*)X + (size_t)t0 * B * Ip * e, I, rows, Ip);
    a1.B = mat((const char*)Wm + (size_t)n0 * Ip * e, I, n1 - n0, Ip);
    a1.M = (int)rows; a1.N = n1 - n0; a1.K = I;
    const int id = (whole ? 0 : 100000 + t0 * 1024 + (t1 - t0)) + (nc > 1 ? 9000000 + nc * 64 + k : 0);
    run_gemm(id, a1, epi(WX + (size_t)t0 * B * NG + n0, NG, (int)rows, n1 - n0), 0, 0, var.g[G_A1],
             two && (k & 1) ? side[0] : st);
  }
  if (two) {
    CUDA_TRY(cudaEventRecord(ev_join, side[0]));
    CUDA_TRY(cudaStreamWaitEvent(st, ev_join, 0));
  }
  if (t0 == 0) mark(R_A1, 1, st);

  // a3: recurrent chain
  if (t0 == 0) mark(R_FWD, 0, st);
  GemmSpec rec;
  rec.A = mat(Hrow(0), Hp, B, Hp, T + 1, (long)B * Hp);
  rec.B = mat(Um, Hp, NG, Hp);
  rec.M = B; rec.N = NG; rec.K = Hp;
  rec.b_keep = true;
  // the fused / persistent forms tile a unit's four gates together: gate-interleaved context only
  const int fmode = blocked() ? 0 : var.fwd_mode;
  if (ot == OT::BF16 && fmode == 1 && !y_f32) {
    // K2 fused, CTA-pair form: GEMM + gate epilogue with TMA-staged epilogue I/O, one launch per step
    const TcGemm& tg = tc_get(1, rec, KCfg{256, 1, 1, 2}, true);
    if (fm_key != (const void*)y || fm_wx != (const void*)WX || fm_T != T) {
      fm.A = tg.mapA;
      fm.B = tg.mapB;
      make_tile_map(&fm.WX, WX, false, NG, B, Tmax, NG, (long)B * NG, 32, 32, 128);
      make_tile_map(&fm.UH, UH, false, NG, B, Tmax, NG, (long)B * NG, 32, 32, 128);
      make_tile_map(&fm.C, Cb, false, Hp, B, Tmax + 1, Hp, (long)B * Hp, 32, 32, 128);
      make_tile_map(&fm.H, Hrow(0), true, Hp, B, Tmax + 1, Hp, (long)B * Hp, 32, 32, 64);
      if (y && H % 8 == 0 && ((uintptr_t)y & 15) == 0) make_tile_map(&fm.Y, y, true, H, B, T, H, (long)B * H, 32, 32, 64);
      else fm.Y = fm.H;
      fm_key = (const void*)y;
      fm_wx = (const void*)WX;
      fm_T = T;
    }
    RecFwd2Args ra;
    ra.B = B; ra.H = H; ra.Hp = Hp; ra.NG = NG; ra.T = T;
    ra.num_mp = cdiv(B, 2 * TC_BM); ra.num_n = NG / 256;
    ra.idesc = tg.args.idesc;
    ra.y_kind = !y ? 0 : (H % 8 == 0 && ((uintptr_t)y & 15) == 0) ? 1 : 2;
    ra.y = y;
    ra.gp = gp;
    for (int t = t0; t < t1; ++t) {
      ra.t = t;
      const bool last = t == T - 1;
      ra.hT = last ? hT : nullptr;
      ra.cT = last ? cT : nullptr;
      lstm_fwd_pair_launch(kind, fm, ra, st);
      fwd_step_done(t, st);
    }
  } else if (ot == OT::BF16 && fmode == 3 && lstm_fwd_persist_supported(B, Hp)) {
    // K2 small-batch persistent: the whole range in one cooperative launch, U slices resident
    RecPersistArgs pa{};
    pa.B = B; pa.H = H; pa.Hp = Hp; pa.NG = NG; pa.T = T; pa.t0 = t0; pa.t1 = t1;
    pa.WX = WX; pa.UH = var.recomp ? nullptr : UH; pa.C = Cb; pa.Hb = (__nv_bfloat16*)Hrow(0);
    if (y_f32) { pa.y = y_f32; pa.ldy = Hp; pa.y_kind = 2; }
    else if (y) { pa.y = y; pa.ldy = H; pa.y_kind = 1; }
    else { pa.y = nullptr; pa.ldy = 0; pa.y_kind = 0; }
    pa.hT = hT; pa.cT = cT; pa.gp = gp;
    pa.flags = sc<unsigned>(off_flags);
    pa.trace = trace_buffer(TRACE_SB_FWD);   // diagnostics only (null: no stamps)
    CUDA_TRY(cudaMemsetAsync(pa.flags, 0, 4096, st));
    lstm_fwd_persist_launch(kind, Hrow(0), Um, Tmax, pa, st);
    for (int t = t0; t < t1; ++t) fwd_step_done(t, st);   // one kernel: every step is done at its end
  } else if (ot == OT::BF16 && fmode > 0 && fmode < 3) {
    // K2 fused: GEMM + gate epilogue in one kernel (per step, or persistent over all steps)
    const TcGemm& tg = tc_get(1, rec, KCfg{256, 1, 1}, true);
    RecFwdArgs ra;
    ra.B = B; ra.H = H; ra.Hp = Hp; ra.NG = NG; ra.T = T;
    ra.num_m = cdiv(B, TC_BM); ra.num_n = NG / 256;
    ra.idesc = tg.args.idesc;
    ra.WX = WX; ra.UH = UH; ra.C = Cb; ra.Hb = (__nv_bfloat16*)Hrow(0);
    if (y_f32) { ra.y = y_f32; ra.ldy = Hp; ra.y_kind = 2; }
    else if (y) { ra.y = y; ra.ldy = H; ra.y_kind = 1; }
    else { ra.y = nullptr; ra.ldy = 0; ra.y_kind = 0; }
    ra.hT = hT; ra.cT = cT; ra.gp = gp;
    ra.flags = sc<unsigned>(off_flags);
    const bool persistent = fmode == 2 && ra.num_m * ra.num_n <= num_sms() && ra.num_m <= 1024;
    if (persistent) {
      CUDA_TRY(cudaMemsetAsync(ra.flags, 0, 4096, st));
      ra.persistent = 1; ra.t0 = t0; ra.t1 = t1;
      lstm_rec_fwd_launch(kind, tg.mapA, tg.mapB, ra, st);
      for (int t = t0; t < t1; ++t) fwd_step_done(t, st);   // one kernel: every step is done at its end
    } else {
      ra.persistent = 0;
      for (int t = t0; t < t1; ++t) {
        ra.t0 = t; ra.t1 = t + 1;
        lstm_rec_fwd_launch(kind, tg.mapA, tg.mapB, ra, st);
        fwd_step_done(t, st);
      }
    }
  } else if (row_split_ok((bool)fwd_hook)) {
    // row_streams: rows [0, B/2) on the main stream, [B/2, B) on side[0], each an independent chain
    const int Bh = B / 2;
    rs_fork(st);
    for (int t = t0; t < t1; ++t) {
      const bool last = t == T - 1;
      for (int hh = 0; hh < 2; ++hh) {
        const cudaStream_t S = hh ? side[0] : st;
        const long r0 = (long)hh * Bh;
        GemmSpec rh = rec;
        rh.A = mat((const char*)Hrow(0) + (size_t)r0 * Hp * e, Hp, Bh, Hp, T + 1, (long)B * Hp);
        rh.M = Bh;
        float* UHt = UH + (long)t * B * NG + r0 * NG;
        run_gemm(1, rh, epi(UHt, NG, Bh, NG), t, 0, var.g[G_REC], S);
        const long rr = (long)t * B + r0;
        if (y_f32)
          lstm_fwd_pointwise(kind, ot, Bh, H, Hp, WX + rr * NG, UHt, gp, Cb + rr * Hp, Cb + (rr + B) * Hp,
                             (char*)Hrow(t + 1) + (size_t)r0 * Hp * e, Hp, y_f32 + (size_t)rr * Hp, Hp, OT::F32,
                             last && hT ? hT + r0 * H : nullptr, last && cT ? cT + r0 * H : nullptr, S, gate_u());
        else
          lstm_fwd_pointwise(kind, ot, Bh, H, Hp, WX + rr * NG, UHt, gp, Cb + rr * Hp, Cb + (rr + B) * Hp,
                             (char*)Hrow(t + 1) + (size_t)r0 * Hp * e, Hp, y ? (char*)y + (size_t)rr * H * e : nullptr,
                             H, ot, last && hT ? hT + r0 * H : nullptr, last && cT ? cT + r0 * H : nullptr, S, gate_u());
      }
    }
    rs_join(st);
  } else {
    for (int t = t0; t < t1; ++t) {
      // recompute variant: UH_t is consumed by this step's pointwise kernel only (one L2-resident slot)
      float* UHt = var.recomp ? sc<float>(off_UHr) : UH + (long)t * B * NG;
      L2Pf pf{};   // R31: WX_t, read by this step's pointwise kernel
      pf.p[0] = WX + (long)t * B * NG; pf.n[0] = (var.l2pf & 1) ? (unsigned long long)B * NG * 4 : 0;
      run_gemm(1, rec, epi(UHt, NG, B, NG), t, 0, var.g[G_REC], st, &pf);
      const bool last = t == T - 1;
      if (y_f32)   // internal fp32 output (e.g. the encoder of LSTM-attention), row stride Hp
        lstm_fwd_pointwise(kind, ot, B, H, Hp, WX + (long)t * B * NG, UHt, gp, Cb + (long)t * B * Hp,
                           Cb + (long)(t + 1) * B * Hp, Hrow(t + 1), Hp, y_f32 + (size_t)t * B * Hp, Hp, OT::F32,
                           last ? hT : nullptr, last ? cT : nullptr, st, gate_u());
      else
        lstm_fwd_pointwise(kind, ot, B, H, Hp, WX + (long)t * B * NG, UHt, gp, Cb + (long)t * B * Hp,
                           Cb + (long)(t + 1) * B * Hp, Hrow(t + 1), Hp, y ? (char*)y + (size_t)t * B * H * e : nullptr,
                           H, ot, last ? hT : nullptr, last ? cT : nullptr, st, gate_u());
      fwd_step_done(t, st);
    }
  }
  if (t1 == T) {
    mark(R_FWD, 1, st);
    fwd_done = true;
  }
}

void LstmCell::backward(const void* dy, const float* dhT, const float* dcT, void* dx, float* dh0, float* dc0) {
  ASTRA_CHECK_STATE(bound && fwd_done, "step_bwd: needs a preceding step_fwd");
  ASTRA_CHECK_ARG(lm_dy || dy, "step_bwd: dy is null");
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

  // time range of this call (descending chunks under the layer wavefront of a stacked LM)
  const int t0 = rg_t1 < 0 ? 0 : rg_t0, t1 = rg_t1 < 0 ? T : rg_t1;
  const bool whole = t0 == 0 && t1 == T;
  if (t1 == T) {
    copy_f32_pad(dcT, B, H, H, dC, Hp, H, st);
    // a5: BPTT chain
    mark(R_BPTT, 0, st);
  }
  GemmSpec bp;
  bp.A = mat(Duh, NG, B, NG, T, (long)B * NG);
  bp.B = mat(Um, Hp, NG, Hp);
  bp.b_mn = true;
  bp.M = B; bp.N = Hp; bp.K = NG;
  bp.b_keep = true;
  bp.kperm = kperm();   // K over the gate columns: the canonical (interleaved) k-block order in any layout
  GemmSpec bp0 = bp;   // dh0 (once, no split)
  bp.ksplit = bptt_ksplit();
  // fused BPTT step (K4 fused): dy must be TMA-mappable (the LM's fp32 dY, or bf16 with H % 8 == 0)
  const int bmode = blocked() ? 0 : var.bwd_mode;   // fused / persistent: gate-interleaved context only
  const bool fuse = bmode == 1 && lstm_bptt_fused_supported(B, Hp, bp.ksplit) && ot == OT::BF16 && T > 1 &&
                    (lm_dy || (H % 8 == 0 && ((uintptr_t)dy & 15) == 0));
  // small-batch persistent BPTT chain (bptt_persist.cu): the whole range in one launch
  const bool persist = !fuse && bmode >= 2 && whole && var.recomp == 0 && bptt_persist_ok();
  BpttFusedArgs fa{};
  if (fuse) {
    const TcGemm& tg = tc_get(2, bp, KCfg{64, 1, 1}, true);
    const void* key[4] = {WX, lm_dy ? (const void*)lm_dy : dy, Duh, (const void*)(uintptr_t)T};
    if (std::memcmp(key, bm_key, sizeof(key)) != 0) {
      bm.A = tg.mapA;
      bm.B = tg.mapB;
      make_tile_map(&bm.WX, WX, false, NG, B, Tmax, NG, (long)B * NG, 256, 16, 0);
      make_tile_map(&bm.UH, UH, false, NG, B, Tmax, NG, (long)B * NG, 256, 16, 0);
      make_tile_map(&bm.C, Cb, false, Hp, B, Tmax + 1, Hp, (long)B * Hp, 64, 16, 0);
      make_tile_map(&bm.DC, dC, false, Hp, B, 1, Hp, 0, 64, 16, 0);
      if (lm_dy) make_tile_map(&bm.DY, lm_dy, false, Hp, B, Tmax, Hp, (long)B * Hp, 64, 16, 0);
      else make_tile_map(&bm.DY, dy, true, H, B, T, H, (long)B * H, 64, 16, 0);
      std::memcpy(bm_key, key, sizeof(key));
    }
    fa.B = B; fa.H = H; fa.Hp = Hp; fa.NG = NG;
    fa.nk = cdiv(NG, TC_BK);
    fa.nsplit = bp.ksplit;
    fa.kper = cdiv(fa.nk, fa.nsplit);
    fa.idesc = tg.args.idesc;
    fa.nq = nq;
    fa.gp = gp;
    fa.D_uh = Duh; fa.D_wx = Dwx; fa.dc = dC; fa.partials = part;
  }
  // Recompute variant: UH_t = h_{t-1}·U is rebuilt here from the saved bf16
  // h operands — the forward's GEMM on the same operands in the same K order, so the same bits
  // (R1, R7).  Chunks of rc_steps timesteps into a two-slot ring, computed on a side stream one
  // chunk ahead of the BPTT chain (the fused BPTT kernel reads UH through its tensor map: there
  // the whole range is recomputed into the UH array up front).
  const bool rc = var.recomp != 0;
  const int RC = rc_steps;
  float* UHr = sc<float>(off_UHr);
  cudaStream_t rs = st;
  if (rc && !fuse && !side.empty()) rs = side[0];
  if (rc && !ev_rc_done[0])
    for (int i = 0; i < 2; ++i) {
      CUDA_TRY(cudaEventCreateWithFlags(&ev_rc_done[i], cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&ev_rc_free[i], cudaEventDisableTiming));
    }
  auto recompute = [&](int ta, int tb, float* dst, cudaStream_t s2, int id) {   // UH rows of steps [ta, tb)
    GemmSpec r = GemmSpec();
    r.A = mat(Hrow(ta), Hp, (long)(tb - ta) * B, Hp);
    r.B = mat(Um, Hp, NG, Hp);
    r.M = (tb - ta) * B; r.N = NG; r.K = Hp;
    run_gemm(id, r, epi(dst, NG, r.M, NG), 0, 0, var.g[G_REC], s2);
  };
  const int kb = t0 / RC;
  bool released[2] = {false, false};   // slot freed by the chain in this call (else free since the fork)
  auto chunk_lo = [&](int k) { return std::max(t0, k * RC); };
  auto chunk_hi = [&](int k) { return std::min(t1, (k + 1) * RC); };
  auto issue = [&](int k) {   // chunk k into ring slot k & 1, after the chain released that slot
    if (k < kb) return;
    const int sl = k & 1;
    if (rs != st && released[sl]) CUDA_TRY(cudaStreamWaitEvent(rs, ev_rc_free[sl], 0));
    const int lo = chunk_lo(k), hi = chunk_hi(k);
    // GEMM id unique per row range: the prepared tensor maps are cached per id (and carry pointers)
    recompute(lo, hi, UHr + ((size_t)sl * RC + (lo - k * RC)) * B * NG, rs, 7000000 + lo * 1024 + (hi - lo));
    if (rs != st) CUDA_TRY(cudaEventRecord(ev_rc_done[sl], rs));
  };
  auto uh_of = [&](int t) -> float* {
    if (!rc || fuse) return UH + (long)t * B * NG;
    const int k = t / RC;
    return UHr + ((size_t)(k & 1) * RC + (t - k * RC)) * B * NG;
  };
  if (rc && fuse) {
    recompute(t0, t1, UH + (long)t0 * B * NG, st, 8000000 + t0 * 1024 + (t1 - t0));
  } else if (rc) {
    if (rs != st) {   // the side stream starts after everything enqueued so far (h operands, Um mirror)
      CUDA_TRY(cudaEventRecord(ev_fork, st));
      CUDA_TRY(cudaStreamWaitEvent(rs, ev_fork, 0));
    }
    issue((t1 - 1) / RC);
    issue((t1 - 1) / RC - 1);
  }
  auto dx_rows = [&](int r0, int r1, int id, cudaStream_t s_, int max_ctas) {   // dX = D_wx·Wᵀ, timesteps [r0, r1)
    const long rows = (long)(r1 - r0) * B;   // (row chunks of one GEMM: same bits, R1)
    GemmSpec gx;
    gx.A = mat(Dwx + (size_t)r0 * B * NG * e, NG, rows, NG);
    gx.B = mat(Wm, I, NG, Ip);
    gx.b_mn = true;
    gx.M = (int)rows; gx.N = I; gx.K = NG;
    gx.kperm = kperm();
    if (lm_mode)
      run_gemm(id, gx, epi((float*)dx + (size_t)r0 * B * Ip, Ip, (int)rows, I), 0, 0, var.g[G_DX], s_, nullptr, max_ctas);
    else
      run_gemm(id, gx, epi((char*)dx + (size_t)r0 * B * I * ot_size(ot), I, (int)rows, I, ot == OT::BF16), 0, 0,
               var.g[G_DX], s_, nullptr, max_ctas);
  };
  // wgrad_schedule (§8(a.9)): the input dgrad in time chunks on a side stream, each as
  // soon as the chain has produced its D_wx rows, on the SMs the per-step BPTT GEMM leaves free
  const int wgs_n = (whole && dx && var.wgs > 0 && !side.empty() && ot == OT::BF16 && !fuse && !persist)
                        ? std::min(WGS_CHUNKS[var.wgs], T) : 1;
  cudaStream_t wst = side.empty() ? st : side.back();
  int wgs_k = 0;
  auto wgs_lo = [&](int k) { return (int)((long)T * (wgs_n - 1 - k) / wgs_n); };   // chunk k: [lo(k), lo(k-1))
  int wgs_ctas = 0;
  if (wgs_n > 1) {
    const KCfg& kb = var.g[G_BPTT];
    const int chain = cdiv(B, TC_BM * kb.cg) * cdiv(Hp, kb.bn) * bp.ksplit * kb.cg;
    wgs_ctas = std::max(8, num_sms() - chain);
    for (int i = 0; i < wgs_n + 1; ++i)
      if (!ev_wgs[i]) CUDA_TRY(cudaEventCreateWithFlags(&ev_wgs[i], cudaEventDisableTiming));
  }
  const bool rsplit = row_split_ok(bwd_hook != nullptr) && !fuse && !persist && whole && wgs_n == 1;
  if (persist) {
    BpttPersistArgs pa{};
    pa.B = B; pa.H = H; pa.Hp = Hp; pa.NG = NG; pa.T = T; pa.nq = nq; pa.gp = gp;
    if (lm_dy) { pa.dy = lm_dy; pa.ldy = Hp; }
    else { pa.dy = dy; pa.ldy = H; }
    pa.dhT = dhT; pa.WX = WX; pa.UH = UH; pa.C = Cb; pa.dc = dC;
    pa.D_uh = (__nv_bfloat16*)Duh; pa.D_wx = (__nv_bfloat16*)Dwx; pa.partials = part;
    pa.flags = sc<unsigned>(off_flags);
    pa.trace = trace_buffer(TRACE_SB_BWD);   // diagnostics only (null: no stamps)
    CUDA_TRY(cudaMemsetAsync(pa.flags, 0, 64, st));
    lstm_bptt_persist_launch(kind, lm_dy != nullptr, Duh, Um, Tmax, pa, st);
  }
  if (rsplit) {   // row_streams: the two row halves' BPTT chains on (main, side[0])
    const int Bh = B / 2;
    rs_fork(st);
    for (int t = T - 1; t >= 0; --t) {
      for (int hh = 0; hh < 2; ++hh) {
        const cudaStream_t S = hh ? side[0] : st;
        const long r0 = (long)hh * Bh;
        const long rr = (long)t * B + r0;
        const void* dyt;
        long ldy;
        bool dyf32;
        if (lm_dy) { dyt = lm_dy + rr * Hp; ldy = Hp; dyf32 = true; }
        else { dyt = (const char*)dy + (size_t)rr * H * e; ldy = H; dyf32 = false; }
        const float* dh_rec;
        long ld_dh;
        int nsplit = 1;
        if (t == T - 1) {
          dh_rec = dhT ? dhT + r0 * H : nullptr;
          ld_dh = H;
        } else {
          GemmSpec bh = bp;
          bh.A = mat(Duh + (size_t)r0 * NG * e, NG, Bh, NG, T, (long)B * NG);
          bh.M = Bh;
          EpiStore eh = epi(dH + r0 * Hp, Hp, Bh, Hp);
          eh.split_stride = (long)B * Hp;
          run_gemm(2, bh, eh, t + 1, 0, var.g[G_BPTT], S);
          dh_rec = dH + r0 * Hp;
          ld_dh = Hp;
          nsplit = bp.ksplit;
        }
        lstm_bwd_pointwise(kind, ot, Bh, H, Hp, dyt, ldy, ot, dyf32, dh_rec, ld_dh, nsplit, (long)B * Hp, dC + r0 * Hp,
                           WX + rr * NG, UH + rr * NG, Cb + (rr + B) * Hp, Cb + rr * Hp, gp,
                           Duh + (size_t)rr * NG * e, Dwx + (size_t)rr * NG * e,
                           part + (size_t)(r0 / BWD_ROW_CHUNK) * nq * NG, nq, t == T - 1, S, var.bpw, gate_u());
      }
    }
    rs_join(st);
  }
  for (int t = (rsplit || persist) ? t0 - 1 : t1 - 1; t >= t0; --t) {
    const int kc = t / RC;
    if (rc && !fuse && rs != st && t == chunk_hi(kc) - 1) CUDA_TRY(cudaStreamWaitEvent(st, ev_rc_done[kc & 1], 0));
    if (fuse && t < T - 1) {
      fa.t = t;
      lstm_bptt_fused_launch(kind, !lm_dy, bm, fa, st);
      continue;
    }
    const void* dyt;
    long ldy;
    bool dyf32;
    if (lm_dy) { dyt = lm_dy + (long)t * B * Hp; ldy = Hp; dyf32 = true; }
    else { dyt = (const char*)dy + (size_t)t * B * H * e; ldy = H; dyf32 = false; }
    const float* dh_rec;
    long ld_dh;
    int nsplit = 1;
    if (t == T - 1) {
      dh_rec = dhT;
      ld_dh = H;
    } else {
      EpiStore e = epi(dH, Hp, B, Hp);
      e.split_stride = (long)B * Hp;
      // R31: the saved tensors step t's pointwise kernel reads (WX_t, UH_t, c_{t-1..t}, dy_t)
      L2Pf pf{};
      if (var.l2pf & 2) {
        pf.p[0] = WX + (long)t * B * NG; pf.n[0] = (unsigned long long)B * NG * 4;
        pf.p[1] = uh_of(t); pf.n[1] = (unsigned long long)B * NG * 4;
        pf.p[2] = Cb + (long)t * B * Hp; pf.n[2] = (unsigned long long)2 * B * Hp * 4;
        pf.p[3] = dyt; pf.n[3] = (unsigned long long)B * ldy * (dyf32 ? 4 : esz());
      }
      run_gemm(2, bp, e, t + 1, 0, var.g[G_BPTT], st, &pf);
      dh_rec = dH;
      ld_dh = Hp;
      nsplit = bp.ksplit;
    }
    lstm_bwd_pointwise(kind, ot, B, H, Hp, dyt, ldy, ot, dyf32, dh_rec, ld_dh, nsplit, (long)B * Hp, dC, WX + (long)t * B * NG,
                       uh_of(t), Cb + (long)(t + 1) * B * Hp, Cb + (long)t * B * Hp, gp,
                       Duh + (size_t)t * B * NG * e, Dwx + (size_t)t * B * NG * e, part, nq, t == T - 1, st, var.bpw, gate_u());
    if (rc && !fuse && t == chunk_lo(kc)) {   // chunk kc consumed: its slot takes chunk kc - 2
      if (rs != st) CUDA_TRY(cudaEventRecord(ev_rc_free[kc & 1], st));
      released[kc & 1] = true;
      issue(kc - 2);
    }
    if (wgs_n > 1 && t == wgs_lo(wgs_k)) {   // D_wx of chunk wgs_k complete: its dX rows on the side stream
      const int hi = wgs_k == 0 ? T : wgs_lo(wgs_k - 1);
      CUDA_TRY(cudaEventRecord(ev_wgs[wgs_k], st));
      CUDA_TRY(cudaStreamWaitEvent(wst, ev_wgs[wgs_k], 0));
      dx_rows(t, hi, 400000 + t * 1024 + (hi - t), wst, wgs_ctas);
      ++wgs_k;
    }
  }
  if (!whole && dx) dx_rows(t0, t1, 200000 + t0 * 1024 + (t1 - t0), st, 0);   // the layer below's dy for this chunk, right away
  if (bwd_hook) bwd_hook();
  if (t0 > 0) return;
  if (dh0) run_gemm(3, bp0, epi(dh0, H, B, H), 0, 0, var.g[G_BPTT], st);
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
  run_gemm(4, gu, blocked() ? epi_perm(g("U"), 4L * H, H, NG, 0, Hp, H) : epi_perm(g("U"), 4L * H, H, NG, GATE_U, 0, H),
           0, 0, var.g[G_DU], st_u);
  if (st_u == st) mark(R_DU, 1, st);
  grad_bucket(g("U"), (size_t)H * 4 * H, st_u);

  GemmSpec gw;
  gw.A = mat(X, I, TB, Ip);
  gw.a_mn = true;
  gw.B = mat(Dwx, NG, TB, NG);
  gw.b_mn = true;
  gw.M = I; gw.N = NG; gw.K = (int)TB;
  mark(R_DW, 0, st);
  run_gemm(5, gw, blocked() ? epi_perm(g("W"), 4L * H, I, NG, 0, Hp, H) : epi_perm(g("W"), 4L * H, I, NG, GATE_U, 0, H),
           0, 0, var.g[G_DW], st);
  mark(R_DW, 1, st);
  grad_bucket(g("W"), (size_t)I * 4 * H, st);

  if (dx && whole && wgs_n == 1) {
    mark(R_DX, 0, st);
    dx_rows(0, T, 6, st, 0);
    mark(R_DX, 1, st);
  }
  float* gq[4] = {g("b"), nullptr, nullptr, nullptr};
  if (kind == K_MILSTM) { gq[1] = g("alpha"); gq[2] = g("beta1"); gq[3] = g("beta2"); }
  reduce_gate_partials(part, nchunk, nq, H, Hp, gq, st, gate_u());
  grad_bucket(g("b"), (size_t)(G + n_params - g("b")), st);   // b (and α, β1, β2): the tail of the cell block
  if (st_u != st) {
    CUDA_TRY(cudaEventRecord(ev_join, st_u));
    CUDA_TRY(cudaStreamWaitEvent(st, ev_join, 0));
  }
  if (wgs_n > 1) {   // the dX chunks (on the side stream since BPTT) are part of the step
    CUDA_TRY(cudaEventRecord(ev_wgs[wgs_n], wst));
    CUDA_TRY(cudaStreamWaitEvent(st, ev_wgs[wgs_n], 0));
  }
  mark(R_SE4, 1, st);
  if (!lm_mode) grad_join(st);
  if (!lm_mode) mark(R_STEP, 1, st);
}

std::unique_ptr<Cell> make_lstm_cell(const astra_cell_desc& d) { return std::unique_ptr<Cell>(new LstmCell(d)); }

}  // namespace astra
