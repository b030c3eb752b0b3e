// Language-model wrapper (SURVEY §8(a) rows a0, a4, a6 embedding part, a7, a8): embedding gather →
// cell forward → head GEMM + mean cross-entropy → head backward → cell BPTT → embedding backward →
// gradient sum over ranks → SGD.  Works for every cell family through the Cell hooks
// (x_operand / y_operand / y_segments).
#include <algorithm>
#include <cstdlib>

#include "cell.h"

namespace astra {

LM::LM(Cell* c, int vocab) : LM(std::vector<Cell*>{c}, vocab) {}

// A stack of layers (the paper's PTB stacked LSTM, Table 5):
// layer l+1 reads layer l's output operand as its input, the embedding feeds layer 0 and the
// head reads the top layer.  Parameters: each layer's block (names prefixed "L<l>." when there is
// more than one layer), then E, W_o, b_o.
LM::LM(std::vector<Cell*> cs, int vocab) : layers(cs), cell(cs.empty() ? nullptr : cs.back()), V(vocab) {
  ASTRA_CHECK_ARG(vocab > 1, "lm: vocab must be > 1");
  ASTRA_CHECK_ARG(!layers.empty(), "lm: at least one layer");
  for (size_t l = 0; l < layers.size(); ++l) {
    Cell* c = layers[l];
    ASTRA_CHECK_ARG(c != nullptr, "lm: null layer");
    if (!c->lm_capable()) throw Error(ASTRA_E_UNSUPPORTED, "lm: this cell type has no LM wrapper (reading R10)");
    for (size_t k = 0; k < l; ++k) ASTRA_CHECK_ARG(layers[k] != c, "lm: a cell can appear only once in a stack");
    if (l > 0) {
      const Cell* b = layers[l - 1];
      ASTRA_CHECK_ARG(c->B == b->B && c->Tmax == b->Tmax && c->ot == b->ot,
                      "lm: stacked layers need the same batch, seq and dtype");
      ASTRA_CHECK_ARG(b->y_segments().size() == 1 && c->I == b->y_segments()[0].n && c->Ip == b->y_width(),
                      "lm: layer l+1's input size must be layer l's output size (single-segment outputs only)");
    }
  }
  Cell* c0 = layers[0];
  Vp = (int)round_up(V, 8);
  Yw = cell->y_width();
  cell->lm_V = V;
  n_params = 0;
  const bool multi = layers.size() > 1;
  for (size_t l = 0; l < layers.size(); ++l) {
    layer_poff.push_back(n_params);
    for (const ParamInfo& q : layers[l]->params) {
      ParamInfo r = q;
      if (multi) r.name = "L" + std::to_string(l) + "." + q.name;
      r.offset += n_params;
      params.push_back(r);
    }
    n_params += (layers[l]->n_params + 63) / 64 * 64;
  }
  n_cell = n_params;
  auto add = [&](const char* n, int r, int cc) {
    params.push_back({n, n_params, r, cc});
    n_params = (n_params + (size_t)r * cc + 63) / 64 * 64;
  };
  add("E", V, c0->I);
  add("W_o", cell->Hout, V);
  add("b_o", 1, V);
  const long TB = (long)cell->T * cell->B;
  const size_t e = cell->esz();
  Carve w;
  int max_ip = 0;
  for (Cell* c : layers) {
    off_lsaved.push_back(w.take(c->saved_bytes));
    off_lscratch.push_back(w.take(c->scratch_bytes));
    off_lh.push_back(w.take((size_t)c->B * c->H * 4));
    off_lc.push_back(w.take((size_t)c->B * (c->c_width() > 0 ? c->c_width() : 1) * 4));
    max_ip = std::max(max_ip, c->Ip);
  }
  off_logits = w.take((size_t)TB * V * 4);
  off_dlog = w.take((size_t)TB * Vp * e);
  off_dlog32 = w.take((size_t)TB * V * 4);
  off_rowloss = w.take((size_t)TB * 4);
  off_dY = w.take((size_t)TB * Yw * 4);
  off_Wo = w.take((size_t)round_up(V, 256) * Yw * e);
  off_colsum = w.take(colsum_scratch_floats(TB, V) * 4);
  sort_bytes = embed_bwd_scratch_bytes(TB, V);
  off_sort = w.take(sort_bytes);
  off_embpart = w.take(embed_bwd_partial_floats(TB, V, c0->I) * 4);
  off_loss = w.take(256);
  off_dx = w.take((size_t)TB * c0->Ip * 4);
  // inter-layer input gradients (fp32, ping-pong: layer l's dx is layer l-1's dy)
  if (multi) {
    off_dxl[0] = w.take((size_t)TB * max_ip * 4);
    off_dxl[1] = w.take((size_t)TB * max_ip * 4);
  }
  // R28: dW_o = Yᵀ·dlogits has few output tiles (Hout x V) and a long K = T·B; a fixed split of K
  // into wo_ksplit chunks (partials summed in chunk order) lets it use the whole GPU.  The split
  // depends only on the shapes, so every variant (and the fp32 path) computes the same sums.
  {
    int maxn = 0;
    for (const KSeg& sg : cell->y_segments()) maxn = std::max(maxn, sg.n);
    wo_ksplit = wo_split(TB);   // non-decreasing in T·B: the largest bucket sizes the partials
    off_wopart = w.take((size_t)wo_ksplit * maxn * V * 4);
  }
  off_tokpad = w.take((size_t)(cell->Tmax + 1) * cell->B * 4);
  off_nv = w.take(4);
  ws_bytes = w.o;
}

int LM::wo_split(long TB) const {
  int maxn = 0;
  for (const KSeg& sg : cell->y_segments()) maxn = std::max(maxn, sg.n);
  const long tiles = (long)cdiv(maxn, 256) * cdiv(V, 256);
  const long kb = cdiv(TB, 64);
  return (int)std::max(1L, std::min(std::min(64L / std::max(1L, tiles), 16L), kb / 8));
}

int LM::bucket_for(int len) const {
  for (int b : buckets)
    if (b >= len) return b;
  return cell->Tmax;
}

// One variable-length step: map len to its bucket, right-pad the tokens into the
// workspace, run the bucket-shaped step with the loss restricted to the first len positions.
void LM::step_var(const int32_t* tokens, int len, float lr, float* loss_dev, bool do_sgd) {
  ASTRA_CHECK_STATE(bound, "lm_train_step_len: not bound");
  ASTRA_CHECK_ARG(tokens, "lm_train_step_len: tokens is null");
  Cell& c = *cell;
  ASTRA_CHECK_ARG(len >= 1 && len <= c.Tmax, "lm_train_step_len: len must be in [1, seq]");
  const int Tb = bucket_for(len);
  set_active_T(Tb);
  cudaStream_t st = c.main_st;
  int32_t* tp = (int32_t*)(ws + off_tokpad);
  CUDA_TRY(cudaMemcpyAsync(tp, tokens, (size_t)(len + 1) * c.B * 4, cudaMemcpyDeviceToDevice, st));
  if (Tb > len) CUDA_TRY(cudaMemsetAsync(tp + (size_t)(len + 1) * c.B, 0, (size_t)(Tb - len) * c.B * 4, st));
  set_state(nullptr, nullptr);   // sentence-level mini-batches: zero initial state, no carry
  set_i32((int*)(ws + off_nv), len * c.B, st);   // read on the device: one graph per bucket
  step_len = len;
  try {
    step(tp, lr, loss_dev, do_sgd);
  } catch (...) {
    step_len = 0;
    throw;
  }
  step_len = 0;
}

size_t LM::find(const std::string& n) const {
  for (auto& p : params)
    if (p.name == n) return p.offset;
  throw Error(ASTRA_E_ARG, "no parameter " + n);
}

void LM::bind(float* pp, float* gg, void* wsp) {
  ASTRA_CHECK_ARG(pp && gg && wsp, "lm_bind: null pointer");
  P = pp; G = gg; ws = (char*)wsp;
  bool ranges = true;
  for (Cell* L : layers) ranges = ranges && L->supports_ranges();
  for (size_t l = 0; l < layers.size(); ++l) {
    layers[l]->lm_mode = true;
    layers[l]->lm_role = l + 1 == layers.size() ? 2 : 1;
    layers[l]->lm_layers = (int)layers.size();
    layers[l]->lm_wavefront = ranges && layers.size() > 1;
    layers[l]->bind(pp + layer_poff[l], gg + layer_poff[l], ws + off_lsaved[l], ws + off_lscratch[l]);
  }
  set_state(nullptr, nullptr);
  bound = true;
}

// h, c: the layers' states concatenated in layer order ([B][H_l] and [B][c_width_l] each).
void LM::set_state(const float* h, const float* c) {
  cudaStream_t st = layers[0]->main_st;
  for (size_t l = 0; l < layers.size(); ++l) {
    const Cell* L = layers[l];
    const size_t nh = (size_t)L->B * L->H * 4, nc = (size_t)L->B * L->c_width() * 4;
    if (h) {
      CUDA_TRY(cudaMemcpyAsync(ws + off_lh[l], h, nh, cudaMemcpyDeviceToDevice, st));
      h += nh / 4;
    } else {
      CUDA_TRY(cudaMemsetAsync(ws + off_lh[l], 0, nh, st));
    }
    if (nc) {
      if (c) {
        CUDA_TRY(cudaMemcpyAsync(ws + off_lc[l], c, nc, cudaMemcpyDeviceToDevice, st));
        c += nc / 4;
      } else {
        CUDA_TRY(cudaMemsetAsync(ws + off_lc[l], 0, nc, st));
      }
    }
  }
}

cudaEvent_t LM::wf_event(int i) {
  if ((int)wf_ev.size() <= i) {
    const size_t n0 = wf_ev.size();
    wf_ev.resize(i + 1, nullptr);
    for (size_t j = n0; j < wf_ev.size(); ++j) CUDA_TRY(cudaEventCreateWithFlags(&wf_ev[j], cudaEventDisableTiming));
  }
  return wf_ev[i];
}

void LM::set_active_T(int t) {
  for (Cell* c : layers) c->set_active_T(t);
}

static bool graphs_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("ASTRA_GRAPH");
    return !(e && e[0] == '0');
  }();
  return on;
}

void LM::clear_graphs() {
  for (auto& g : graphs) cudaGraphExecDestroy(g.exec);
  graphs.clear();
}

LM::~LM() {
  clear_graphs();
  if (cap_st) cudaStreamDestroy(cap_st);
  for (cudaEvent_t ev : {ev_hfork, ev_hdy, ev_hdone})
    if (ev) cudaEventDestroy(ev);
  for (cudaEvent_t ev : ev_chunk)
    if (ev) cudaEventDestroy(ev);
  for (cudaEvent_t ev : wf_ev) cudaEventDestroy(ev);
  for (cudaStream_t s2 : lstreams)
    if (s2) cudaStreamDestroy(s2);
}

void LM::step(const int32_t* tokens, float lr, float* loss_dev, bool do_sgd) {
  ASTRA_CHECK_STATE(bound, "lm_train_step: not bound");
  ASTRA_CHECK_ARG(tokens, "lm_train_step: tokens is null");
  Cell& c = *cell;
  // data parallelism needs one communicator across every layer (the embedding and head buckets
  // go through layer 0 / the top layer): a layer without one would silently stay unreduced
  int wmax = 1;
  for (Cell* L : layers) wmax = std::max(wmax, L->world);
  if (wmax > 1)
    for (Cell* L : layers)
      ASTRA_CHECK_STATE(L->world == wmax && (L->nccl_comm || L->peer),
                        "lm_train_step: world > 1 but a layer has no communicator (use astra_lm_comm_init / "
                        "astra_lm_comm_peer_init on the LM, not on one cell)");
  // exploration steps (and the fp32 parity path) run eagerly; a frozen / untuned / converged bf16 step replays
  // multi-rank steps stay eager unless ASTRA_GRAPH_NCCL=1 (NCCL inside a capture is supported, but
  // a capture mismatch across ranks would hang the job; not exercisable on a 1-GPU test box).  The
  // peer-memory backend never replays: its kernels take the host's barrier sequence number as an
  // argument, which a captured graph would freeze (every replay would pass the barriers at once)
  static const bool graph_nccl = [] {
    const char* e = std::getenv("ASTRA_GRAPH_NCCL");
    return e && e[0] == '1';
  }();
  bool exploring = false;
  std::string vs;
  for (Cell* L : layers) {
    exploring |= L->tune_mode == ASTRA_TUNE_ON && (!(L->wirer && L->wirer->converged()) || L->racing);
    // a captured step records into the region-event slot current at capture time
    vs += L->var.str() + (L->profiling ? ";p" + std::to_string(L->ev_slot) + (L->regions_needed() ? "r;" : ";") : ";");
  }
  if (!use_graphs || !graphs_enabled() || exploring || c.ot != OT::BF16 ||
      (c.world > 1 && (!graph_nccl || c.peer))) {
    enqueue_step(tokens, lr, loss_dev, do_sgd);
    return;
  }
  for (auto& g : graphs)
    if (g.tokens == tokens && g.lr == lr && g.loss == loss_dev && g.sgd == do_sgd && g.variant == vs &&
        g.T == c.T && g.len == (step_len > 0)) {
      CUDA_TRY(cudaGraphLaunch(g.exec, c.main_st));
      count_launch(g.launches);
      return;
    }
  if (!cap_st) CUDA_TRY(cudaStreamCreateWithFlags(&cap_st, cudaStreamNonBlocking));
  // the captured work must follow everything already queued on the caller's stream
  cudaEvent_t e0;
  CUDA_TRY(cudaEventCreateWithFlags(&e0, cudaEventDisableTiming));
  CUDA_TRY(cudaEventRecord(e0, c.main_st));
  CUDA_TRY(cudaStreamWaitEvent(cap_st, e0, 0));
  CUDA_TRY(cudaEventDestroy(e0));
  cudaStream_t user = c.main_st;
  for (Cell* L : layers) L->main_st = cap_st;
  const uint64_t l0 = g_launches.load();
  cudaGraph_t graph = nullptr;
  CUDA_TRY(cudaStreamBeginCapture(cap_st, cudaStreamCaptureModeThreadLocal));
  try {
    enqueue_step(tokens, lr, loss_dev, do_sgd);
  } catch (...) {
    cudaStreamEndCapture(cap_st, &graph);
    if (graph) cudaGraphDestroy(graph);
    for (Cell* L : layers) L->main_st = user;
    throw;
  }
  for (Cell* L : layers) L->main_st = user;
  CUDA_TRY(cudaStreamEndCapture(cap_st, &graph));
  GraphEntry ge;
  ge.tokens = tokens; ge.lr = lr; ge.loss = loss_dev; ge.sgd = do_sgd; ge.variant = vs;
  ge.T = c.T; ge.len = step_len > 0;
  ge.launches = g_launches.load() - l0;
  CUDA_TRY(cudaGraphInstantiate(&ge.exec, graph, 0));
  CUDA_TRY(cudaGraphDestroy(graph));
  g_launches.fetch_sub(ge.launches);   // captured, not yet launched
  if (graphs.size() >= 8) {
    cudaGraphExecDestroy(graphs.front().exec);
    graphs.erase(graphs.begin());
  }
  graphs.push_back(ge);
  CUDA_TRY(cudaGraphLaunch(ge.exec, c.main_st));
  count_launch(ge.launches);
}

void LM::enqueue_step(const int32_t* tokens, float lr, float* loss_dev, bool do_sgd) {
  Cell& c = *cell;
  cudaStream_t st = c.main_st;
  const long TB = (long)c.T * c.B;
  const size_t e = c.esz();
  Cell& c0 = *layers[0];
  const int nl = (int)layers.size();
  float* logits = (float*)(ws + off_logits);
  void* dlog = ws + off_dlog;
  float* dlog32 = (float*)(ws + off_dlog32);
  float* rowloss = (float*)(ws + off_rowloss);
  float* dY = (float*)(ws + off_dY);
  char* Wom = ws + off_Wo;
  float* dX = (float*)(ws + off_dx);
  float* lossp = loss_dev ? loss_dev : (float*)(ws + off_loss);
  const int Vr = (int)round_up(V, 256);
  const std::vector<KSeg> segs = c.y_segments();

  // rows that carry a loss: a device scalar, so a captured step serves every length of its bucket
  int* nvd = (int*)(ws + off_nv);
  if (step_len == 0) set_i32(nvd, (int)TB, st);

  // B3 stream assignment of the head (AV head_ov): the head of time chunk k (logits, CE, dgrad)
  // runs on a side stream as soon as forward step t_k is done, overlapping the rest of the forward
  // chain; its weight gradient overlaps the BPTT chain.  Row chunks of the same GEMMs, same CE and
  // reductions: bitwise identical to the sequential head.
  const int nch = HEAD_CHUNKS[std::min(2, std::max(0, c.var.head_ov))];
  const bool ov = nch > 1 && !c.side.empty() && c.T >= nch;
  cudaStream_t hst = ov ? c.side.back() : st;
  if (ov) {
    if (!ev_hfork) {
      CUDA_TRY(cudaEventCreateWithFlags(&ev_hfork, cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&ev_hdy, cudaEventDisableTiming));
      CUDA_TRY(cudaEventCreateWithFlags(&ev_hdone, cudaEventDisableTiming));
      for (auto& e5 : ev_chunk) CUDA_TRY(cudaEventCreateWithFlags(&e5, cudaEventDisableTiming));
    }
    CUDA_TRY(cudaEventRecord(ev_hfork, st));
    CUDA_TRY(cudaStreamWaitEvent(hst, ev_hfork, 0));
  }
  std::vector<int> t_end(nch);   // last forward step of each time chunk
  for (int k = 0; k < nch; ++k) t_end[k] = (int)((long)(k + 1) * c.T / nch) - 1;

  for (Cell* L : layers) L->mark(R_STEP, 0, st);
  if (c.peer) {
    c.peer->begin_step();
    c.peer->dpb = c.var.dpb;   // the top layer's AV sizes every layer's buckets
  }
  // layer wavefront (AV lwf of the top layer): layer l runs on its own stream, time chunk by time
  // chunk; chunk k of layer l starts when layer l-1 finished chunk k (forward) / layer l+1 produced
  // the dX rows of chunk k (backward).  Row chunks of the same GEMMs, the chains unchanged: the
  // same bits as layers one after the other.
  bool wf_ok = nl > 1;
  for (Cell* L : layers) wf_ok = wf_ok && L->supports_ranges();
  const int nwc = wf_ok ? std::min({WF_CHUNKS[std::min(2, std::max(0, c.var.lwf))], c.T, 64}) : 1;
  std::vector<int> tb(nwc + 1);
  for (int k = 0; k <= nwc; ++k) tb[k] = (int)((long)k * c.T / nwc);
  auto lst = [&](int l) { return l == 0 || nwc == 1 ? st : lstreams[l]; };
  if (nwc > 1) {
    while ((int)lstreams.size() < nl) {
      cudaStream_t s2 = nullptr;
      if (!lstreams.empty()) CUDA_TRY(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
      lstreams.push_back(s2);
    }
    CUDA_TRY(cudaEventRecord(wf_event(0), st));
    for (int l = 1; l < nl; ++l) CUDA_TRY(cudaStreamWaitEvent(lstreams[l], wf_event(0), 0));
  }
  auto ev_f = [&](int l, int k) { return wf_event(1 + l * 64 + k); };
  auto ev_b = [&](int l, int k) { return wf_event(1 + 32 * 64 + l * 64 + k); };

  // a0: embedding gather into layer 0's operand buffer
  embed_gather(c.ot, tokens, TB, P + find("E"), c0.I, c0.x_operand(), c0.Ip, st);
  // head weight mirror (independent of the forward)
  // each segment's mirror writes its whole padded width [k0, next k0) × Vr rows (zeros past the
  // segment's rows and past V), so the mirror covers [0, Yw) without a separate memset
  if (segs.empty() || segs[0].k0 != 0) CUDA_TRY(cudaMemsetAsync(Wom, 0, (size_t)Vr * Yw * e, hst));
  for (size_t i = 0; i < segs.size(); ++i) {
    const KSeg& s = segs[i];
    const int kend = i + 1 < segs.size() ? segs[i + 1].k0 : Yw;
    mirror_T(c.ot, P + find("W_o") + (size_t)s.r0 * V, s.n, V, Vr, kend - s.k0, Wom + (size_t)s.k0 * e, Yw, hst);
  }
  // a4 per time chunk: head forward + CE + head dgrad (SE2).  The head reads the cell's output
  // operand (SCRN: [h | s], a K-concatenated "ladder" [h|s]·[U;V]).
  const Mat2 Y = c.y_operand();
  auto head_chunk = [&](int k) {
    const long r0 = k == 0 ? 0 : (long)(t_end[k - 1] + 1) * c.B, r1 = (long)(t_end[k] + 1) * c.B;
    const int rows = (int)(r1 - r0);
    if (ov) {   // recorded on the stream the top layer's forward runs on
      CUDA_TRY(cudaEventRecord(ev_chunk[k], c.main_st));
      CUDA_TRY(cudaStreamWaitEvent(hst, ev_chunk[k], 0));
    }
    if (k == 0) c.mark(R_HEAD, 0, hst);   // region: first head chunk → head weight gradient done
    GemmSpec hd;
    hd.A = mat((const char*)Y.ptr + (size_t)r0 * Y.ld * e, Y.inner, rows, Y.ld);
    hd.B = mat(Wom, Yw, V, Yw);
    hd.M = rows; hd.N = V; hd.K = Yw;
    c.run_gemm(nch > 1 ? 120 + k : 100, hd, epi(logits + r0 * V, V, rows, V, 0, P + find("b_o")), 0, 0,
               c.var.g[G_HEAD], hst);
    ce_fwd_bwd(c.ot, logits + r0 * V, V, V, tokens + c.B + r0, rows, 0.f, rowloss + r0, (char*)dlog + (size_t)r0 * Vp * e,
               Vp, dlog32 + r0 * V, hst, nvd, r0);
    GemmSpec dy;
    dy.A = mat((const char*)dlog + (size_t)r0 * Vp * e, V, rows, Vp);
    dy.B = mat(Wom, Yw, V, Yw);
    dy.b_mn = true;
    dy.M = rows; dy.N = Yw; dy.K = V;
    c.run_gemm(nch > 1 ? 130 + k : 101, dy, epi(dY + r0 * Yw, Yw, rows, Yw), 0, 0, c.var.g[G_HDY], hst);
  };
  // cell forward (SE1); final state carried for the next step (truncated BPTT) — except for a
  // variable-length step, whose padded tail would corrupt it (zero state, no carry)
  if (ov)
    c.fwd_hook = [&](int t) {
      for (int k = 0; k < nch; ++k)
        if (t == t_end[k]) head_chunk(k);
    };
  auto restore = [&] {
    c.fwd_hook = nullptr;
    for (Cell* L : layers) {
      L->main_st = st;
      L->rg_t0 = 0;
      L->rg_t1 = -1;
      L->bwd_hook = nullptr;
    }
  };
  try {
    for (int k = 0; k < nwc; ++k) {
      for (int l = 0; l < nl; ++l) {
        Cell& L = *layers[l];
        const cudaStream_t S = lst(l);
        L.main_st = S;
        if (nwc > 1) {
          L.rg_t0 = tb[k];
          L.rg_t1 = tb[k + 1];
          if (l > 0) CUDA_TRY(cudaStreamWaitEvent(S, ev_f(l - 1, k), 0));
        }
        if (l > 0) {   // layer l's input operand = layer l-1's output operand (bf16 / fp32, [T·B][H])
          const Mat2 yp = layers[l - 1]->y_operand();
          const long r0 = (long)tb[k] * c.B, rows = (long)(tb[k + 1] - tb[k]) * c.B;
          copy_pad(L.ot, (const char*)yp.ptr + (size_t)r0 * yp.ld * e, L.ot, rows, L.I, yp.ld,
                   (char*)L.x_operand() + (size_t)r0 * L.Ip * e, L.Ip, S);
        }
        float* hs = (float*)(ws + off_lh[l]);
        float* cs = L.c_width() > 0 ? (float*)(ws + off_lc[l]) : nullptr;
        if (step_len > 0) L.forward(nullptr, hs, cs, nullptr, nullptr, nullptr);
        else L.forward(nullptr, hs, cs, nullptr, hs, cs);
        if (nwc > 1) CUDA_TRY(cudaEventRecord(ev_f(l, k), S));
      }
    }
  } catch (...) {
    restore();
    throw;
  }
  if (nwc > 1) CUDA_TRY(cudaStreamWaitEvent(st, ev_f(nl - 1, nwc - 1), 0));   // top done ⇒ every layer done
  restore();
  if (!ov) head_chunk(0);
  if (ov) {   // BPTT needs every dY row; the weight gradient of the head stays on the side stream
    CUDA_TRY(cudaEventRecord(ev_hdy, hst));
    CUDA_TRY(cudaStreamWaitEvent(st, ev_hdy, 0));
  }
  sum_rows_to_scalar(rowloss, TB, 0.f, lossp, hst, nvd);
  int id = 102;
  for (const KSeg& s : segs) {
    GemmSpec dwo;
    dwo.A = mat((const char*)Y.ptr + (size_t)s.k0 * e, s.n, TB, Y.ld);
    dwo.a_mn = true;
    dwo.B = mat(dlog, V, TB, Vp);
    dwo.b_mn = true;
    dwo.M = s.n; dwo.N = V; dwo.K = (int)TB;
    const int wks = wo_split(TB);
    dwo.ksplit = wks;
    float* dWo = G + find("W_o") + (size_t)s.r0 * V;
    if (wks > 1) {
      float* part = (float*)(ws + off_wopart);
      EpiStore ep = epi(part, V, s.n, V);
      ep.split_stride = (long)s.n * V;
      c.run_gemm(id++, dwo, ep, 0, 0, c.var.g[G_HEAD], hst);
      sum_split_partials(part, wks, (long)s.n * V, dWo, hst);
    } else {
      c.run_gemm(id++, dwo, epi(dWo, V, s.n, V), 0, 0, c.var.g[G_HEAD], hst);
    }
  }
  colsum(dlog32, TB, V, V, (float*)(ws + off_colsum), G + find("b_o"), hst);
  c.mark(R_HEAD, 1, hst);
  // a7 bucket 1: the head gradients are final before BPTT — their sum overlaps the chain
  c.grad_bucket(G + find("W_o"), n_params - find("W_o"), hst);
  if (ov) CUDA_TRY(cudaEventRecord(ev_hdone, hst));

  // layers' backward (SE3 + SE4), top down: layer l's input gradient is layer l-1's dy; then the
  // embedding backward
  try {
    if (nwc > 1) {   // dY is ready on the main stream
      CUDA_TRY(cudaEventRecord(wf_event(1 + 64 * 64), st));
      CUDA_TRY(cudaStreamWaitEvent(lst(nl - 1), wf_event(1 + 64 * 64), 0));
    }
    for (int k = nwc - 1; k >= 0; --k) {
      for (int l = nl - 1; l >= 0; --l) {
        Cell& L = *layers[l];
        const cudaStream_t S = lst(l);
        L.main_st = S;
        L.lm_dy = l == nl - 1 ? dY : (float*)(ws + off_dxl[(l + 1) % 2]);
        float* dx_l = l == 0 ? dX : (float*)(ws + off_dxl[l % 2]);
        if (nwc > 1) {
          L.rg_t0 = tb[k];
          L.rg_t1 = tb[k + 1];
          if (l < nl - 1) CUDA_TRY(cudaStreamWaitEvent(S, ev_b(l + 1, k), 0));
          cudaEvent_t done = ev_b(l, k);
          L.bwd_hook = [done, S] { CUDA_TRY(cudaEventRecord(done, S)); };
        }
        L.backward(nullptr, nullptr, nullptr, dx_l, nullptr, nullptr);
      }
    }
    if (nwc > 1)
      for (int l = 1; l < nl; ++l) {   // join every layer stream (its weight gradients included)
        CUDA_TRY(cudaEventRecord(wf_event(2 + 64 * 64 + l), lst(l)));
        CUDA_TRY(cudaStreamWaitEvent(st, wf_event(2 + 64 * 64 + l), 0));
      }
  } catch (...) {
    restore();
    throw;
  }
  restore();
  embed_bwd(tokens, TB, V, dX, c0.Ip, c0.I, G + find("E"), ws + off_sort, sort_bytes, (float*)(ws + off_embpart), st);
  // a7: last bucket (embedding), join, then a8: SGD
  c0.grad_bucket(G + find("E"), (size_t)V * c0.I, st);
  if (ov) CUDA_TRY(cudaStreamWaitEvent(st, ev_hdone, 0));   // head gradients (and their bucket) done
  for (Cell* L : layers) L->grad_join(st);
  if (do_sgd) {
    if (c.peer && c.world > 1) {   // K11p: owned shards updated and all-gathered into every rank
      std::vector<std::pair<size_t, size_t>> cover;
      for (const ParamInfo& q : params) cover.push_back({q.offset, (size_t)q.rows * q.cols});
      c.peer->sgd(lr, st, cover);
    } else {
      sgd(P, G, n_params, lr, st);
    }
  }
  for (Cell* L : layers) L->mark(R_STEP, 1, st);
}

}  // namespace astra
