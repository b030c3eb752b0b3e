// L1 runtime: per-cell step plan, workspace carving, the executor of one training step for each
// variant, and the LM wrapper.  The tuner (L2) chooses the Variant; every variant computes the
// same bits (R1-R7).
//
// Cell families (each a subclass with its own plan):
//   LstmCell  — LSTM, MI-LSTM [36], subLSTM [8]      (cell_lstm.cpp)
//   ScrnCell  — SC-RNN / SCRN [22]                    (cell_scrn.cpp)
//   RhnCell   — recurrent highway network [39]        (cell_rhn.cpp)
//   AttnCell  — LSTM encoder + attentive decoder [35] (cell_attn.cpp)
#pragma once
#include <functional>
#include <cuda_runtime.h>

#include <map>
#include <memory>
#include <string>
#include <tuple>
#include <vector>

#include "../common.h"
#include "../kernels/gemm.h"
#include "../kernels/kernels.h"
#include "../tuner/tuner.h"
#include "peer.h"

namespace astra {

struct ParamInfo {
  std::string name;
  size_t offset;
  int rows, cols;
};

// K1 kernel choice for one GEMM role (B1, "GEMM kernel selection", as a choice among our
// own sm_100a kernels): CTA tile width and cluster multicast shape.
struct KCfg {
  int bn = 256, cm = 1, cn = 1;
  int cg = 1;   // 2: CTA pair (cta_group::2, 256-row tiles)
  bool operator==(const KCfg& o) const { return bn == o.bn && cm == o.cm && cn == o.cn && cg == o.cg; }
};
enum GemmRole { G_A1 = 0, G_REC, G_BPTT, G_DU, G_DW, G_DX, G_HEAD, G_HDY, G_ROLES };
extern const char* const ROLE_NAMES[G_ROLES];

// One binding of every adaptive variable (the enumerator's output for a cell).
constexpr int HEAD_CHUNKS[3] = {1, 2, 5};
constexpr int GCHUNK_N[5] = {1, 2, 4, 2, 4};   // gate GEMMs: 1 fused, G/2, G (G = 4 gate blocks)
constexpr int WGS_CHUNKS[3] = {1, 4, 10};      // wgrad_schedule time chunks (1: dX after BPTT)
constexpr int GCHUNK_S[5] = {1, 1, 1, 2, 2};   // streams they run on
constexpr int WF_CHUNKS[3] = {1, 5, 1 << 20};   // clipped to T: the last option is one chunk per step
struct Variant {
  KCfg g[G_ROLES];      // a1 hoisted projection, recurrent step, BPTT step, dU, dW, dX, LM head (logits, dW_o),
                        // LM head dgrad dY = dlogits·W_o (N = the cell's output width, not V: its own tile choice)
  int wg_side = 0;      // 1: dU on a side stream concurrently with dW/dX (B3)
  int fwd_mode = 0;     // K2 (LSTM family, bf16): 0 GEMM + pointwise kernel, 1 fused per step, 2 fused persistent
  int bwd_mode = 0;     // K4: same encoding
  int lwf = 0;          // stacked LM: layer wavefront in WF_CHUNKS[lwf] time chunks (1 = layers one after the other)
  int head_ov = 0;      // LM head overlapped with the forward chain in HEAD_CHUNKS[head_ov] time chunks (B3)
  int l2pf = 0;         // chain GEMMs prefetch the next pointwise kernel's saved tensors into L2 (R31): bit 0 fwd, bit 1 BPTT
  int dpb = 0;          // K11p bucket cap (§8(a.9) dp_bucket): 0 whole tensors, 1/2/3 = 128/32/8 MB pieces
  int rsp = 0;          // row_streams (B3 stream assignment): 1 = the batch's two row halves run as two
                        // independent chains on two streams (the sequences are independent), so one half's
                        // pointwise kernel overlaps the other half's recurrent GEMM (LSTM family, B ≥ 256)
  int bpw = 0;          // bwd_pw (§8(a.9) bwd_kernel / bwd_epilogue): backward pointwise form, 0 row-lane (unit per
                        // thread, 8 rows walked), 1 wide (row x 4 units per thread, whole 32-row chunk in flight),
                        // 2 wide with every operand tile landed in shared memory by TMA (fp32 dY: LM mode)
  int wgs = 0;          // wgrad_schedule (§8(a.9)): the input dgrad dX in WGS_CHUNKS[wgs] time chunks,
                        // each issued on a side stream as soon as BPTT has produced its rows (0: after BPTT)
  int gchunk = 0;       // gate_chunking (§8(a.9), "chunking the fusion group", P:220 chunk sizes): the
                        // fused gate GEMM of the hoisted projection as GCHUNK_N[gchunk] GEMMs over gate-column
                        // ranges, on GCHUNK_S[gchunk] streams (P:122 two streams vs one fused GEMM)
  int recomp = 0;       // alloc fork: 1 = the recurrent projection UH_t is not
                        // kept for BPTT but recomputed there from the saved h_{t-1} operands (same bits)
  int gblk = 0;         // alloc fork (§8(a.9) `alloc`, reading R38): internal gate layout of the LSTM
                        // family's mirrors and gate-column tensors, 0 gate-interleaved (64-unit blocks), 1 gate-
                        // blocked ([K, G·Hp]); the GEMMs contracting over gates read k-blocks in the interleaved
                        // order (TcArgs::kperm), so the same bits; the fused / persistent K2 / K4 forms need a
                        // unit's four gates in one tile, so they exist only under the interleaved context
  Variant() { g[G_BPTT].bn = 128; }
  std::string str() const;                    // "a1=256.1.1,rec=...,wg_side=0"
  static Variant parse(const std::string& s); // inverse of str(); throws ASTRA_E_ARG
};

// GEMM problem in storage terms; drives both engines (tcgen05 for bf16, SIMT for fp32).
struct GemmSpec {
  Mat2 A, B;
  bool a_mn = false, b_mn = false;
  bool b_keep = false;   // B is a weight re-read every step: keep it in L2 (evict_last)
  int ksplit = 1;        // fixed split-K (part of the canonical numerics: every variant uses it)
  int M = 0, N = 0, K = 0;
  int kperm = 0;         // K over gate-blocked gate columns, read in the canonical interleaved order (TcArgs::kperm)
};

Mat2 mat(const void* p, long inner, long outer, long ld, long z = 1, long zstride = 0);
EpiStore epi(void* C, long ldc, int Mv, int Nv, int out_bf16 = 0, const float* bias = nullptr);
EpiStore epi_perm(void* C, long ldc, int Mv, int Nv, int perm_u, int perm_blk, int perm_H);
inline EpiStore accum(EpiStore e) { e.accumulate = 1; return e; }

enum Region { R_A1 = 0, R_FWD, R_HEAD, R_BPTT, R_DU, R_DW, R_DX, R_SE4, R_STEP, R_COUNT };

// A segment of the head weight's K dimension: operand columns [k0, k0+n) ↔ W_o rows [r0, r0+n).
struct KSeg { int k0, r0, n; };

class Cell {
 public:
  explicit Cell(const astra_cell_desc& d);
  virtual ~Cell();

  astra_cell_desc d;
  OT ot;
  int H, I, B, T, Hp, Ip, Hout;
  int Tmax;   // sequence length the workspace is carved for; T = the active length (bucket) ≤ Tmax
  std::vector<ParamInfo> params;
  size_t n_params = 0;
  size_t saved_bytes = 0, scratch_bytes = 0;

  // binding
  float* P = nullptr;
  float* G = nullptr;
  char* saved = nullptr;
  char* scratch = nullptr;
  bool bound = false, fwd_done = false;

  // streams / events
  cudaStream_t main_st = nullptr;
  std::vector<cudaStream_t> side;
  cudaStream_t comm_st = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;

  // variant + tuner
  Variant var;
  int tune_mode = ASTRA_TUNE_OFF;
  std::unique_ptr<tuner::Tree> tree;
  std::unique_ptr<tuner::Wirer> wirer;
  std::vector<Variant> configs_seen;
  int tune_reps = 3, rep_i = 0;
  // measured steps left in flight when the host waits for a configuration's reps (1: the step just
  // enqueued).  2 was measured at cfg5 (profiles/r2s5_tune_lag.txt): the same decisions, the same
  // exploration-vs-frozen gap of the unfused forward chain (2.7 vs 3.1 ms), 20 % more steps — kept 1
  int tune_lag = 1;
  tuner::Metrics rep_min;
  // Region events live in a ring of per-step slots, so the tuner can harvest a
  // measured step with cudaEventQuery some steps later instead of blocking on it (include/astra.h
  // astra_tune_next "never blocks"): `ev` / `region_used` point at the slot being recorded.
  static constexpr int EV_SLOTS = 8;
  cudaEvent_t evr[EV_SLOTS][R_COUNT][2];
  bool used_r[EV_SLOTS][R_COUNT];
  int ev_slot = 0, last_step_slot = 0;
  cudaEvent_t (*ev)[2] = evr[0];
  bool* region_used = used_r[0];
  // measured exploration steps whose events are not harvested yet: (slot, bucket T, config serial)
  struct PendingRep { int slot, T; long serial; };
  std::vector<PendingRep> pending;
  long cfg_serial = 0, next_serial = 1;
  int reps_harvested = 0;
  long tune_blocks = 0;      // harvests that had to wait (ring full, or world > 1: reading R29)
  void use_slot(int s);
  tuner::Metrics read_metrics(int slot);
  void harvest(int wait);
  // Final race (reading R41): once the wirer converges, the close alternatives of the chain-form
  // AVs and of the per-step chain GEMMs' kernel choices (fuse_fwd, fuse_bwd, bwd_pw, row_streams,
  // g_rec, g_bptt: options within 10 % of the chosen one in the profile index, the 5 closest) are
  // re-measured against the converged configuration in interleaved rounds
  // (5 rounds of 1 warm-up + 1 measured step each) on t_step, and the fastest is kept.  The exploration
  // measured them minutes apart while the power-capped SM clock drifted; interleaving
  // removes the drift from the comparison.  One rank, no buckets; ASTRA_TUNE_RACE=0 disables it.
  bool racing = false;
  std::vector<tuner::Config> race_cfg;
  std::vector<double> race_best;
  std::vector<int> race_seq;
  size_t race_pos = 0;
  int race_sub = 0;
  struct RacePend { int slot, cand; };
  std::vector<RacePend> race_pending;
  int race_winner = -1;
  bool race_start();
  int race_step();
  void race_harvest(bool wait_all);
  void race_advance();
  bool profiling = true;
  // Profiling levels: the step region is always recorded; the phase regions
  // (a1, chains, head, SE4, dU / dW / dX) only while the tuner needs them — exploring or racing —
  // or when asked for (astra_set_profiling(c, 2): diagnostics such as bench.py's region table).  A
  // frozen step then carries 2 event records instead of 18, each of which would otherwise sit
  // between two chain kernels in the step graph and cost their programmatic overlap.
  bool full_regions = false;
  bool regions_needed() const {
    return full_regions || (tune_mode == ASTRA_TUNE_ON && (!wirer || !wirer->converged() || racing));
  }
  std::vector<KCfg> allowed[G_ROLES];  // statically pruned options per role (A19), default first
  // prepared GEMMs keyed by (gemm id, T, bn, cm, cn, cg, A, B, M, N, K): the tensor maps carry the
  // operand pointers and extents, so two row ranges of one role never share an entry
  using TcKey = std::tuple<int, int, int, int, int, int, const void*, const void*, int, int, int, bool, int>;
  std::map<TcKey, TcGemm> tc_cache;

  // Bucketed profiling: one independent exploration per active length T, the
  // profile index keys prefixed by the bucket; the workspace stays the one of the largest bucket.
  struct TuneCtx {
    Variant var;
    std::unique_ptr<tuner::Tree> tree;
    std::unique_ptr<tuner::Wirer> wirer;
    std::vector<Variant> configs_seen;
    int rep_i = 0;
    tuner::Metrics rep_min;
    std::vector<KCfg> allowed[G_ROLES];
    long cfg_serial = 0;
    int reps_harvested = 0;
  };
  std::map<int, TuneCtx> tune_ctx;   // parked contexts of the inactive buckets
  void set_active_T(int t);

  // NCCL
  void* nccl_comm = nullptr;
  bool own_nccl = true;   // false: a communicator shared with the other layers of an LM (layer 0 owns it)
  int rank = 0, world = 1;
  // K11p: deterministic peer-memory gradient sum + fused SGD / all-gather (SURVEY §8(e) backend
  // 2).  When set (world > 1), grad_bucket() launches the rank-ordered reduce instead of NCCL and
  // SGD is the owned-shard update written to every rank.  Shared by the layers of one LM.
  std::shared_ptr<PeerComm> peer;
  void ensure_comm_stream();

  // LM mode hooks (set by LM)
  bool lm_mode = false;
  const float* lm_dy = nullptr;  // fp32 [T*B][y_width()] internal dY for the backward (null: external dy)
  float* y_f32 = nullptr;        // optional internal fp32 output [T*B][y_width()] (LSTM family)
  int lm_V = 0;

  // time range [rg_t0, rg_t1) of the next forward / backward call (rg_t1 < 0: all of [0, T)): a
  // stacked LM's layer wavefront runs layers chunk by chunk (cells with supports_ranges() only)
  int rg_t0 = 0, rg_t1 = -1;
  virtual bool supports_ranges() const { return false; }
  int lm_role = 0;      // 0 not in an LM, 1 lower layer of a stack, 2 the layer the head reads
  int lm_layers = 1;    // layers of the LM this cell belongs to
  bool lm_wavefront = false;   // (top layer) every layer of the stack supports ranges: AV lwf exists
  std::function<void()> bwd_hook;   // called after a ranged backward call enqueued its dX rows

  // ---- per-family interface
  virtual void forward(const void* x, const float* h0, const float* c0, void* y, float* hT, float* cT) = 0;
  virtual void backward(const void* dy, const float* dhT, const float* dcT, void* dx, float* dh0, float* dc0) = 0;
  virtual void* x_operand() = 0;                 // [T*B][Ip] operand buffer (the LM gathers here)
  virtual Mat2 y_operand() = 0;                  // [T*B][y_width()] operand (A of the head GEMM)
  virtual int y_width() const = 0;               // padded K of the head
  virtual std::vector<KSeg> y_segments() const = 0;
  virtual int c_width() const { return H; }      // width of the second state (c or s); 0 = none
  virtual bool lm_capable() const { return true; }
  virtual bool chain_prefetch() const { return false; }   // supports Variant::l2pf (tuner AVs pf_fwd / pf_bwd)
  virtual bool supports_recompute() const { return false; }   // Variant::recomp (tuner root fork "recomp")
  virtual bool supports_gate_blocked() const { return false; }   // Variant::gblk (tuner root fork "alloc")
  virtual int fwd_fusions() const { return 1; }   // number of K2 fusion choices (tuner AV "fuse_fwd")
  virtual const char* fwd_fusion_metric() const { return "t_fwd"; }   // the region that judges it
  virtual int bwd_fusions() const { return 1; }   // number of K4 fusion choices (tuner AV "fuse_bwd")
  virtual int gate_chunkings() const { return 1; }   // options of the tuner AV "gate_chunking" (1: none)
  virtual int wgrad_schedules() const { return 1; }  // options of the tuner AV "wgrad_schedule" (1: none)
  virtual int bwd_pw_forms() const { return 1; }     // options of the tuner AV "bwd_pw" (1: none)
  virtual int row_stream_options() const { return 1; }   // options of the tuner AV "row_streams" (1: none)
  virtual void role_shape(int role, int& M, int& N) const = 0;

  // forward-step hook (set by the LM): called after forward step t is enqueued on the main stream,
  // so the head of a finished time chunk is enqueued on a side stream in host order too (the
  // overlap then also happens in eager, exploring steps, not only in a replayed graph)
  std::function<void(int)> fwd_hook;   // called (host side) right after step t is enqueued
  void fwd_step_done(int t, cudaStream_t) {
    if (fwd_hook) fwd_hook(t);
  }

  // ---- shared machinery
  void add_param(const char* n, int r, int c);
  size_t find_param(const std::string& n) const;
  float* p(const std::string& n) { return P + find_param(n); }
  float* g(const std::string& n) { return G + find_param(n); }
  void bind(float* params, float* grads, void* saved_p, void* scratch_p);
  void sgd_step(float lr);
  void grad_bucket(float* p, size_t n, cudaStream_t producer);   // K11: launch one DP bucket
  void grad_join(cudaStream_t main);                               // main waits for all buckets
  cudaEvent_t ev_bucket[4] = {nullptr, nullptr, nullptr, nullptr};
  int bucket_i = 0;
  bool sync_pending = false;
  cudaStream_t own_comm_st = nullptr;
  double* tune_dev = nullptr;          // 64 doubles: cross-rank max of the tuner's metric vector
  size_t esz() const { return ot_size(ot); }
  template <typename T_> T_* sv(size_t off) { return reinterpret_cast<T_*>(saved + off); }
  template <typename T_> T_* sc(size_t off) { return reinterpret_cast<T_*>(scratch + off); }
  void run_gemm(int id, const GemmSpec& s, const EpiStore& e, int az, int bz, const KCfg& k, cudaStream_t st,
                const L2Pf* pf = nullptr, int max_ctas = 0);
  // prepared tensor maps (bf16 path); plain_maps: single-k-block maps for the fused kernels
  TcGemm& tc_get(int id, const GemmSpec& s, const KCfg& k, bool plain_maps = false);
  void mark(Region r, int which, cudaStream_t st);
  void tuner_setup();
  void apply_config(const tuner::Config& c);
  int tune_next();
  std::string report();
};

std::unique_ptr<Cell> make_cell(const astra_cell_desc& d);

// Byte-offset allocator for workspace carving (256-byte aligned regions).
struct Carve {
  size_t o = 0;
  size_t take(size_t bytes) {
    size_t r = o;
    o = (o + bytes + 255) / 256 * 256;
    return r;
  }
};

class LM {
 public:
  LM(Cell* c, int vocab);
  LM(std::vector<Cell*> layers, int vocab);   // stacked layers, bottom first
  std::vector<Cell*> layers;
  Cell* cell;                                 // the top layer (the head reads its output)
  std::vector<size_t> layer_poff, off_lsaved, off_lscratch, off_lh, off_lc;
  size_t off_dxl[2] = {0, 0};
  void set_active_T(int t);
  int V, Vp, Yw;
  size_t n_cell, n_params;
  std::vector<ParamInfo> params;
  size_t off_logits, off_dlog, off_dlog32, off_rowloss, off_dY, off_Wo, off_colsum, off_sort, off_loss, off_embpart,
      off_dx, off_wopart, ws_bytes;
  size_t sort_bytes;
  int wo_ksplit = 1;   // fixed split of the head weight-gradient GEMM over K = T·B (reading R28)
  float* P = nullptr;
  float* G = nullptr;
  char* ws = nullptr;
  bool bound = false;
  size_t find(const std::string& n) const;
  void bind(float* params, float* grads, void* workspace);
  void set_state(const float* h, const float* c);
  void step(const int32_t* tokens, float lr, float* loss_dev, bool do_sgd);
  void enqueue_step(const int32_t* tokens, float lr, float* loss_dev, bool do_sgd);
  // Bucketed profiling for variable-length mini-batches: a step of length len runs
  // at the smallest bucket T_b ≥ len on right-padded tokens, its loss and gradients restricted to
  // the first len positions (padding contributes exact zeros), from a zero initial state.
  std::vector<int> buckets;   // ascending, last ≤ cell seq; empty = every step runs at seq
  int step_len = 0;           // valid length of the step being enqueued (0 = full T)
  size_t off_tokpad = 0;      // int32 [Tmax+1][B] padded token buffer
  size_t off_nv = 0;          // int32 device scalar: rows of the step that carry a loss
  cudaEvent_t ev_hfork = nullptr, ev_hdy = nullptr, ev_hdone = nullptr, ev_chunk[5] = {};
  // layer wavefront: one stream per layer above the bottom, events per (layer, chunk)
  std::vector<cudaStream_t> lstreams;
  std::vector<cudaEvent_t> wf_ev;
  cudaEvent_t wf_event(int i);
  int bucket_for(int len) const;
  void step_var(const int32_t* tokens, int len, float lr, float* loss_dev, bool do_sgd);
  int wo_split(long TB) const;   // R28 split for the active T·B
  ~LM();

  // CUDA-graph replay of a frozen step (no exploration): the whole step — every kernel, the side
  // and comm stream forks/joins, the NCCL buckets, the region events — is captured once per
  // (tokens, lr, loss, sgd, variant) and replayed with one cudaGraphLaunch, removing the host's
  // per-kernel launch cost (~10 µs per step-kernel at cfg5) from the critical path.
  struct GraphEntry {
    const int32_t* tokens;
    float lr;
    float* loss;
    bool sgd;
    std::string variant;
    int T, len;   // active length; len = 1 for a variable-length (bucketed) step
    cudaGraphExec_t exec;
    uint64_t launches;
  };
  std::vector<GraphEntry> graphs;
  bool use_graphs = true;
  cudaStream_t cap_st = nullptr;
  void clear_graphs();
};

}  // namespace astra
