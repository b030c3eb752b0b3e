// L3: the C ABI (include/astra.h).  Every entry point converts C++ exceptions into status codes;
// argument and state errors are raised before any device work is enqueued.
#include <nccl.h>

#include <cstring>
#include <memory>
#include <string>

#include "common.h"
#include "runtime/cell.h"
#include "tuner/tuner.h"

namespace astra {
std::atomic<uint64_t> g_launches{0};
static thread_local std::string t_err;
void set_error(const std::string& s) { t_err = s; }
}  // namespace astra

using namespace astra;

namespace astra {   // kernels/micro.cu
void micro_stream_read(const void* buf, size_t bytes, int passes, float* sink, cudaStream_t st);
void micro_grid_barrier(unsigned* counter, int iters, cudaStream_t st);
void micro_launch_chain(int n, int pdl, int blocks, cudaStream_t st);
void micro_mma_chain(int M, int N, int iters, int ctas, int mode, long long* cycles, float* dump, cudaStream_t st);
void micro_tma_read(const void* buf, long rows, int kb, int box_rows, int ctas, int stages, int nbox, int same,
                    cudaStream_t st);
void micro_peer_reduce(float* const* bufs, uint32_t* const* sigs, int world, size_t n, int reps, uint32_t seq0,
                       const cudaStream_t* streams);
}  // namespace astra

struct astra_cell_s {
  std::unique_ptr<Cell> c;
};
struct astra_lm_s {
  std::unique_ptr<LM> m;
};

template <class F>
static astra_status guard(F&& f) {
  try {
    f();
    return ASTRA_OK;
  } catch (const Error& e) {
    set_error(e.what());
    return e.code;
  } catch (const std::exception& e) {
    set_error(e.what());
    return ASTRA_E_ARG;
  } catch (...) {
    set_error("unknown error");
    return ASTRA_E_ARG;
  }
}

#define NEED(p) do { if (!(p)) throw Error(ASTRA_E_ARG, #p " is null"); } while (0)

extern "C" {

astra_status astra_cell_create_ex(astra_cell* out, const astra_cell_desc* d) {
  return guard([&] {
    NEED(out); NEED(d);
    astra_cell_desc dd = *d;
    if (dd.depth <= 0) dd.depth = 10;
    if (dd.context <= 0) dd.context = dd.hidden;
    if (dd.scrn_alpha == 0.f) dd.scrn_alpha = 0.95f;
    if (dd.src_seq <= 0) dd.src_seq = dd.seq;
    if (dd.attn_dim <= 0) dd.attn_dim = dd.hidden;
    auto h = std::make_unique<astra_cell_s>();
    h->c = make_cell(dd);
    *out = h.release();
  });
}

astra_status astra_cell_create(astra_cell* out, int cell_type, int hidden, int input, int batch, int seq) {
  astra_cell_desc d;
  std::memset(&d, 0, sizeof(d));
  d.cell_type = cell_type; d.hidden = hidden; d.input = input; d.batch = batch; d.seq = seq;
  d.dtype = ASTRA_BF16;
  return astra_cell_create_ex(out, &d);
}

astra_status astra_cell_destroy(astra_cell c) {
  return guard([&] { delete c; });
}

astra_status astra_param_count(astra_cell c, size_t* n) {
  return guard([&] { NEED(c); NEED(n); *n = c->c->n_params; });
}

astra_status astra_param_info(astra_cell c, int idx, const char** name, size_t* offset, int* rows, int* cols) {
  return guard([&] {
    NEED(c);
    auto& ps = c->c->params;
    if (idx < 0 || idx >= (int)ps.size()) throw Error(ASTRA_E_ARG, "param index out of range");
    if (name) *name = ps[idx].name.c_str();
    if (offset) *offset = ps[idx].offset;
    if (rows) *rows = ps[idx].rows;
    if (cols) *cols = ps[idx].cols;
  });
}

astra_status astra_workspace_size(astra_cell c, size_t* saved, size_t* scratch) {
  return guard([&] {
    NEED(c);
    if (saved) *saved = c->c->saved_bytes;
    if (scratch) *scratch = c->c->scratch_bytes;
  });
}

astra_status astra_bind(astra_cell c, float* params, float* grads, void* saved, void* scratch) {
  return guard([&] { NEED(c); c->c->bind(params, grads, saved, scratch); });
}

astra_status astra_set_streams(astra_cell c, astra_stream main, const astra_stream* side, int n_side, astra_stream comm) {
  return guard([&] {
    NEED(c);
    ASTRA_CHECK_ARG(n_side >= 0 && (n_side == 0 || side), "set_streams: bad side streams");
    c->c->main_st = (cudaStream_t)main;
    c->c->side.clear();
    for (int i = 0; i < n_side; ++i) c->c->side.push_back((cudaStream_t)side[i]);
    c->c->comm_st = (cudaStream_t)comm;
  });
}

astra_status astra_step_fwd(astra_cell c, const void* x, const float* h0, const float* c0, void* y, float* hT,
                            float* cT) {
  return guard([&] {
    NEED(c);
    ASTRA_CHECK_STATE(!c->c->lm_mode, "step_fwd: cell is owned by an LM");
    c->c->forward(x, h0, c0, y, hT, cT);
  });
}

astra_status astra_step_bwd(astra_cell c, const void* dy, const float* dhT, const float* dcT, void* dx, float* dh0,
                            float* dc0) {
  return guard([&] {
    NEED(c);
    ASTRA_CHECK_STATE(!c->c->lm_mode, "step_bwd: cell is owned by an LM");
    if (c->c->peer) c->c->peer->begin_step();
    c->c->backward(dy, dhT, dcT, dx, dh0, dc0);
  });
}

astra_status astra_sgd(astra_cell c, float lr) {
  return guard([&] { NEED(c); c->c->sgd_step(lr); });
}

astra_status astra_tune_next(astra_cell c, int* state) {
  return guard([&] {
    NEED(c);
    int s = c->c->tune_next();
    if (state) *state = s;
  });
}

astra_status astra_tune_mode(astra_cell c, int mode, const char* forced) {
  return guard([&] {
    NEED(c);
    Cell& cc = *c->c;
    ASTRA_CHECK_ARG(mode == ASTRA_TUNE_OFF || mode == ASTRA_TUNE_ON || mode == ASTRA_TUNE_FROZEN, "tune_mode: bad mode");
    // every bucket restarts — except a plain freeze, which keeps each bucket's current variant
    if (!(mode == ASTRA_TUNE_FROZEN && !forced)) cc.tune_ctx.clear();
    if (mode == ASTRA_TUNE_ON) cc.profiling = true;   // exploration reads the region events
    if (mode == ASTRA_TUNE_OFF) {
      cc.var = Variant();
      cc.wirer.reset();
    } else if (mode == ASTRA_TUNE_ON) {
      cc.wirer.reset();
      cc.var = Variant();
    } else if (forced) {
      cc.var = Variant::parse(forced);
    }
    cc.tune_mode = mode;
    cc.racing = false;
    cc.race_pending.clear();
  });
}

astra_status astra_set_profiling(astra_cell c, int on) {
  return guard([&] {
    NEED(c);
    Cell& cc = *c->c;
    ASTRA_CHECK_STATE(on || cc.tune_mode != ASTRA_TUNE_ON, "set_profiling: exploration needs the region events");
    ASTRA_CHECK_ARG(on >= 0 && on <= 2, "set_profiling: on must be 0, 1 or 2");
    cc.profiling = on != 0;
    cc.full_regions = on == 2;
  });
}

astra_status astra_tune_report(astra_cell c, char* buf, size_t len, size_t* needed) {
  return guard([&] {
    NEED(c);
    std::string r = c->c->report();
    if (needed) *needed = r.size() + 1;
    if (buf && len) {
      size_t n = std::min(len - 1, r.size());
      std::memcpy(buf, r.data(), n);
      buf[n] = 0;
    }
  });
}

astra_status astra_comm_unique_id(void* out, size_t len) {
  return guard([&] {
    NEED(out);
    ASTRA_CHECK_ARG(len >= sizeof(ncclUniqueId), "comm_unique_id: buffer too small");
    ncclUniqueId id;
    ncclResult_t r = ncclGetUniqueId(&id);
    if (r != ncclSuccess) throw Error(ASTRA_E_NCCL, std::string("ncclGetUniqueId: ") + ncclGetErrorString(r));
    std::memcpy(out, &id, sizeof(id));
  });
}

// One NCCL communicator shared by `cells` (a cell, or every layer of an LM); cells[0] owns it.
static void comm_init_cells(const std::vector<Cell*>& cells, const void* uid, int rank, int world) {
  ASTRA_CHECK_ARG(world >= 1 && rank >= 0 && rank < world, "comm_init: bad rank/world");
  for (Cell* c : cells)
    ASTRA_CHECK_ARG(!c->peer || !c->peer->ready || c->peer->world == world, "comm_init: world differs from the peer backend's");
  Cell& c0 = *cells[0];
  CUDA_TRY(cudaSetDevice(c0.d.device));
  ncclUniqueId id;
  std::memcpy(&id, uid, sizeof(id));
  ncclComm_t comm;
  ncclResult_t r = ncclCommInitRank(&comm, world, id, rank);
  if (r != ncclSuccess) throw Error(ASTRA_E_NCCL, std::string("ncclCommInitRank: ") + ncclGetErrorString(r));
  for (Cell* c : cells)
    if (c->nccl_comm && c->own_nccl) ncclCommDestroy((ncclComm_t)c->nccl_comm);
  for (size_t i = 0; i < cells.size(); ++i) {
    Cell& cc = *cells[i];
    cc.nccl_comm = comm;
    cc.own_nccl = i == 0;
    cc.rank = rank;
    cc.world = world;
    cc.ensure_comm_stream();
    if (!cc.tune_dev) CUDA_TRY(cudaMalloc(&cc.tune_dev, 64 * sizeof(double)));
  }
}

astra_status astra_comm_init(astra_cell c, const void* uid, int rank, int world) {
  return guard([&] {
    NEED(c); NEED(uid);
    comm_init_cells({c->c.get()}, uid, rank, world);
  });
}

astra_status astra_lm_comm_init(astra_lm m, const void* uid, int rank, int world) {
  return guard([&] {
    NEED(m); NEED(uid);
    comm_init_cells(m->m->layers, uid, rank, world);
  });
}

// K11p (SURVEY §8(e) backend 2): the peer-memory window is the flat params / grads vector that
// SGD updates — the cell's, or the LM's when the cell belongs to one.
static void peer_export(std::vector<Cell*> cells, float* P, float* G, size_t n, void* out, size_t len) {
  Cell& c0 = *cells[0];
  if (!c0.peer) {
    auto pc = std::make_shared<PeerComm>(c0.d.device, P, G, n);
    for (Cell* c : cells) c->peer = pc;
  }
  ASTRA_CHECK_STATE(c0.peer->P == P && c0.peer->G == G, "comm_peer_handle: rebound since the peer window was made");
  c0.peer->export_handle(out, len);
}

static void peer_init(std::vector<Cell*> cells, const void* handles, int rank, int world) {
  Cell& c0 = *cells[0];
  ASTRA_CHECK_STATE(c0.peer, "comm_peer_init: call comm_peer_handle first (and exchange the handles)");
  for (Cell* c : cells)
    ASTRA_CHECK_ARG(!c->nccl_comm || c->world == world, "comm_peer_init: world differs from the NCCL communicator's");
  c0.peer->import_handles(handles, rank, world);
  for (Cell* c : cells) {
    c->rank = rank;
    c->world = world;
    c->ensure_comm_stream();
  }
}

astra_status astra_comm_peer_handle(astra_cell c, void* out, size_t len) {
  return guard([&] {
    NEED(c); NEED(out);
    Cell& cc = *c->c;
    ASTRA_CHECK_STATE(cc.bound && !cc.lm_mode, "comm_peer_handle: cell not bound, or owned by an LM (use the lm_ form)");
    peer_export({&cc}, cc.P, cc.G, cc.n_params, out, len);
  });
}

astra_status astra_comm_peer_init(astra_cell c, const void* handles, int rank, int world) {
  return guard([&] {
    NEED(c);
    ASTRA_CHECK_STATE(!c->c->lm_mode, "comm_peer_init: cell owned by an LM (use the lm_ form)");
    peer_init({c->c.get()}, handles, rank, world);
  });
}

astra_status astra_lm_comm_peer_handle(astra_lm m, void* out, size_t len) {
  return guard([&] {
    NEED(m); NEED(out);
    LM& lm = *m->m;
    ASTRA_CHECK_STATE(lm.bound, "lm_comm_peer_handle: not bound");
    peer_export(lm.layers, lm.P, lm.G, lm.n_params, out, len);
  });
}

astra_status astra_lm_comm_peer_init(astra_lm m, const void* handles, int rank, int world) {
  return guard([&] {
    NEED(m);
    peer_init(m->m->layers, handles, rank, world);
  });
}

astra_status astra_lm_create(astra_lm* out, astra_cell c, int vocab) {
  return guard([&] {
    NEED(out); NEED(c);
    auto h = std::make_unique<astra_lm_s>();
    h->m.reset(new LM(c->c.get(), vocab));
    *out = h.release();
  });
}

astra_status astra_lm_create_stacked(astra_lm* out, const astra_cell* cells, int n_layers, int vocab) {
  return guard([&] {
    NEED(out); NEED(cells);
    ASTRA_CHECK_ARG(n_layers >= 1, "lm_create_stacked: n_layers must be >= 1");
    std::vector<Cell*> v;
    for (int l = 0; l < n_layers; ++l) {
      NEED(cells[l]);
      v.push_back(cells[l]->c.get());
    }
    auto h = std::make_unique<astra_lm_s>();
    h->m.reset(new LM(v, vocab));
    *out = h.release();
  });
}

astra_status astra_lm_destroy(astra_lm m) {
  return guard([&] { delete m; });
}

astra_status astra_lm_param_count(astra_lm m, size_t* n) {
  return guard([&] { NEED(m); NEED(n); *n = m->m->n_params; });
}

astra_status astra_lm_param_info(astra_lm m, int idx, const char** name, size_t* offset, int* rows, int* cols) {
  return guard([&] {
    NEED(m);
    auto& ps = m->m->params;
    if (idx < 0 || idx >= (int)ps.size()) throw Error(ASTRA_E_ARG, "param index out of range");
    if (name) *name = ps[idx].name.c_str();
    if (offset) *offset = ps[idx].offset;
    if (rows) *rows = ps[idx].rows;
    if (cols) *cols = ps[idx].cols;
  });
}

astra_status astra_lm_workspace_size(astra_lm m, size_t* bytes) {
  return guard([&] { NEED(m); NEED(bytes); *bytes = m->m->ws_bytes; });
}

astra_status astra_lm_bind(astra_lm m, float* params, float* grads, void* ws) {
  return guard([&] { NEED(m); m->m->bind(params, grads, ws); });
}

astra_status astra_lm_set_state(astra_lm m, const float* h, const float* c) {
  return guard([&] { NEED(m); m->m->set_state(h, c); });
}

astra_status astra_lm_train_step(astra_lm m, const int32_t* tokens, float lr, float* loss_dev) {
  return guard([&] {
    NEED(m);
    m->m->set_active_T(m->m->cell->Tmax);
    m->m->step(tokens, lr, loss_dev, true);
  });
}

astra_status astra_lm_set_buckets(astra_lm m, const int* sizes, int n) {
  return guard([&] {
    NEED(m);
    ASTRA_CHECK_ARG(n >= 0 && (n == 0 || sizes), "lm_set_buckets: sizes is null");
    std::vector<int> b(sizes, sizes + n);
    for (int i = 0; i < n; ++i) {
      ASTRA_CHECK_ARG(b[i] >= 1 && b[i] <= m->m->cell->Tmax, "lm_set_buckets: bucket sizes must be in [1, seq]");
      ASTRA_CHECK_ARG(i == 0 || b[i] > b[i - 1], "lm_set_buckets: bucket sizes must be ascending");
    }
    m->m->buckets = b;
  });
}

astra_status astra_lm_train_step_len(astra_lm m, const int32_t* tokens, int len, float lr, float* loss_dev) {
  return guard([&] { NEED(m); m->m->step_var(tokens, len, lr, loss_dev, true); });
}

astra_status astra_lm_fwd_bwd_len(astra_lm m, const int32_t* tokens, int len, float* loss_dev) {
  return guard([&] { NEED(m); m->m->step_var(tokens, len, 0.f, loss_dev, false); });
}

astra_status astra_lm_set_graph(astra_lm m, int on) {
  return guard([&] {
    NEED(m);
    m->m->use_graphs = on != 0;
    if (!on) m->m->clear_graphs();
  });
}

astra_status astra_lm_fwd_bwd(astra_lm m, const int32_t* tokens, float* loss_dev) {
  return guard([&] {
    NEED(m);
    m->m->set_active_T(m->m->cell->Tmax);
    m->m->step(tokens, 0.f, loss_dev, false);
  });
}

astra_status astra_gemm_bf16_ex(int M, int N, int K, const void* A, int a_mn, long lda, const void* Bp, int b_mn,
                                long ldb, float* C, long ldc, int bn, int cm, int cn, int cta_group, int ksplit,
                                astra_stream stream) {
  return guard([&] {
    NEED(A); NEED(Bp); NEED(C);
    ASTRA_CHECK_ARG(M > 0 && N > 0 && K > 0, "gemm: sizes must be positive");
    ASTRA_CHECK_ARG(ldc >= N, "gemm: ldc < N");
    ASTRA_CHECK_ARG(ksplit >= 1 && ksplit <= 16, "gemm: ksplit must be in [1, 16]");
    ASTRA_CHECK_ARG(cta_group == 1 || cta_group == 2, "gemm: cta_group must be 1 or 2");
    Mat2 a, b;
    a.ptr = A; a.ld = lda;
    if (a_mn) { a.inner = M; a.outer = K; } else { a.inner = K; a.outer = M; }
    b.ptr = Bp; b.ld = ldb;
    if (b_mn) { b.inner = N; b.outer = K; } else { b.inner = K; b.outer = N; }
    ASTRA_CHECK_ARG(lda >= a.inner && ldb >= b.inner, "gemm: leading dimension too small");
    TcGemm g;
    tc_gemm_prepare(g, a, a_mn != 0, b, b_mn != 0, M, N, K, bn, cm, cn, false, ksplit, cta_group);
    EpiStore e = epi(C, ldc, M, N);
    e.split_stride = (long)M * ldc;
    tc_gemm_launch(g, e, 0, 0, (cudaStream_t)stream);
  });
}

astra_status astra_gemm_bf16(int M, int N, int K, const void* A, int a_mn, long lda, const void* Bp, int b_mn,
                             long ldb, float* C, long ldc, int bn, int cm, int cn, astra_stream stream) {
  return astra_gemm_bf16_ex(M, N, K, A, a_mn, lda, Bp, b_mn, ldb, C, ldc, bn, cm, cn, 1, 1, stream);
}

const char* astra_status_string(astra_status s) {
  switch (s) {
    case ASTRA_OK: return "ASTRA_OK";
    case ASTRA_E_ARG: return "ASTRA_E_ARG";
    case ASTRA_E_UNSUPPORTED: return "ASTRA_E_UNSUPPORTED";
    case ASTRA_E_STATE: return "ASTRA_E_STATE";
    case ASTRA_E_CUDA: return "ASTRA_E_CUDA";
    case ASTRA_E_NCCL: return "ASTRA_E_NCCL";
    case ASTRA_E_WORKSPACE: return "ASTRA_E_WORKSPACE";
    default: return "ASTRA_E_UNKNOWN";
  }
}

const char* astra_last_error(void) { return t_err.c_str(); }

uint64_t astra_kernel_launch_count(void) { return g_launches.load(); }

astra_status astra_micro_stream_read(const void* buf, size_t bytes, int passes, float* sink, astra_stream stream) {
  return guard([&] { micro_stream_read(buf, bytes, passes, sink, (cudaStream_t)stream); });
}

astra_status astra_micro_grid_barrier(unsigned* counter, int iters, astra_stream stream) {
  return guard([&] { micro_grid_barrier(counter, iters, (cudaStream_t)stream); });
}

astra_status astra_micro_mma_chain(int M, int N, int iters, int ctas, int mode, long long* cycles, float* dump,
                                   astra_stream stream) {
  return guard([&] { micro_mma_chain(M, N, iters, ctas, mode, cycles, dump, (cudaStream_t)stream); });
}
astra_status astra_micro_tma_read(const void* buf, long rows, int kb, int box_rows, int ctas, int stages, int nbox,
                                  int same, astra_stream stream) {
  return guard([&] { micro_tma_read(buf, rows, kb, box_rows, ctas, stages, nbox, same, (cudaStream_t)stream); });
}

astra_status astra_micro_launch_chain(int n, int pdl, int blocks, astra_stream stream) {
  return guard([&] { micro_launch_chain(n, pdl, blocks, (cudaStream_t)stream); });
}

astra_status astra_debug_set_trace(int kind, void* device_buffer) {
  return guard([&] { set_trace_buffer(kind, (unsigned long long*)device_buffer); });
}

astra_status astra_micro_peer_reduce(float* const* bufs, unsigned* const* sigs, int world, size_t n, int reps,
                                     unsigned seq0, const astra_stream* streams) {
  return guard([&] {
    micro_peer_reduce(bufs, (uint32_t* const*)sigs, world, n, reps, seq0, (const cudaStream_t*)streams);
  });
}

astra_status astra_region_times(astra_cell c, double* out, int cap, int* n) {
  return guard([&] {
    NEED(c); NEED(out);
    Cell& cc = *c->c;
    ASTRA_CHECK_STATE(cc.bound, "region_times: not bound");
    // the most recently completed step's slot (the tuner may already record into the next one)
    cudaEvent_t (*E)[2] = cc.evr[cc.last_step_slot];
    const bool* used = cc.used_r[cc.last_step_slot];
    CUDA_TRY(cudaEventSynchronize(E[R_STEP][1]));
    int k = 0;
    for (int r = 0; r < R_COUNT && k < cap; ++r, ++k) {
      float ms = 0.f;
      if (used[r] && cudaEventElapsedTime(&ms, E[r][0], E[r][1]) != cudaSuccess) {
        cudaGetLastError();
        ms = 0.f;
      }
      out[k] = used[r] ? ms : 0.0;
    }
    if (n) *n = k;
  });
}

astra_status astra_tuner_selftest(const char* tree, astra_fake_cost_fn cost, void* user, int* trials_out,
                                  int max_trials, int* n_trials, int* final_out, int* n_avs) {
  return guard([&] {
    NEED(tree); NEED(cost);
    tuner::Tree t = tuner::parse(tree);
    tuner::Wirer w(&t);
    w.start();
    tuner::Config c;
    int k = 0;
    const int na = (int)t.avs.size();
    tuner::Metrics m(t.metrics.size(), 0.0);
    while (w.propose(c)) {
      if (trials_out && k < max_trials)
        for (int i = 0; i < na; ++i) trials_out[k * na + i] = c[i];
      cost(c.data(), na, m.data(), (int)m.size(), user);
      w.feed(m);
      ++k;
    }
    if (n_trials) *n_trials = k;
    if (n_avs) *n_avs = na;
    if (final_out) {
      tuner::Config f = w.final_config();
      for (int i = 0; i < na; ++i) final_out[i] = f[i];
    }
  });
}

}  // extern "C"
