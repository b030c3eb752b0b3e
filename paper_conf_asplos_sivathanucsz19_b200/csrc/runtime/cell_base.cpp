// L1 runtime, shared machinery of every cell family: parameters, binding, workspace, the GEMM
// dispatch (tcgen05 for the bf16 path, SIMT for the fp32 path), cudaEvent-pair profiling regions
// (P:286-288), the tuner glue (L2) and the DP gradient sum (K11).
#include <cstdlib>
#include <nccl.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <sstream>

#include "cell.h"

namespace astra {

const char* const ROLE_NAMES[G_ROLES] = {"a1", "rec", "bptt", "du", "dw", "dx", "head", "hdy"};

std::string Variant::str() const {
  std::ostringstream o;
  for (int r = 0; r < G_ROLES; ++r) {
    o << ROLE_NAMES[r] << "=" << g[r].bn << "." << g[r].cm << "." << g[r].cn;
    if (g[r].cg != 1) o << "." << g[r].cg;
    o << ",";
  }
  o << "wg_side=" << wg_side << ",fwd=" << fwd_mode << ",bwd=" << bwd_mode << ",pf=" << l2pf << ",hov=" << head_ov;
  if (lwf) o << ",lwf=" << lwf;
  if (recomp) o << ",rc=" << recomp;
  if (gblk) o << ",gb=" << gblk;
  if (dpb) o << ",dpb=" << dpb;
  if (gchunk) o << ",gc=" << gchunk;
  if (wgs) o << ",wgs=" << wgs;
  if (bpw) o << ",bpw=" << bpw;
  if (rsp) o << ",rsp=" << rsp;
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
    if (k == "dpb") {
      v.dpb = std::stoi(val);
      ASTRA_CHECK_ARG(v.dpb >= 0 && v.dpb <= 3, "variant: dpb must be 0..3 (whole tensors, 128, 32 or 8 MB buckets)");
      continue;
    }
    if (k == "rsp") {
      v.rsp = std::stoi(val);
      ASTRA_CHECK_ARG(v.rsp == 0 || v.rsp == 1, "variant: rsp (row_streams) must be 0 or 1");
      continue;
    }
    if (k == "bpw") {
      v.bpw = std::stoi(val);
      ASTRA_CHECK_ARG(v.bpw >= 0 && v.bpw <= 2, "variant: bpw (backward pointwise form) must be 0..2");
      continue;
    }
    if (k == "wgs") {
      v.wgs = std::stoi(val);
      ASTRA_CHECK_ARG(v.wgs >= 0 && v.wgs <= 2, "variant: wgs (wgrad_schedule) must be 0..2");
      continue;
    }
    if (k == "gc") {
      v.gchunk = std::stoi(val);
      ASTRA_CHECK_ARG(v.gchunk >= 0 && v.gchunk <= 4, "variant: gc (gate_chunking) must be 0..4");
      continue;
    }
    if (k == "gb") {
      v.gblk = std::stoi(val);
      ASTRA_CHECK_ARG(v.gblk == 0 || v.gblk == 1, "variant: gb must be 0 (gate-interleaved) or 1 (gate-blocked layout)");
      continue;
    }
    if (k == "rc") {
      v.recomp = std::stoi(val);
      ASTRA_CHECK_ARG(v.recomp == 0 || v.recomp == 1, "variant: rc must be 0 (store UH) or 1 (recompute UH in BPTT)");
      continue;
    }
    if (k == "lwf") {
      v.lwf = std::stoi(val);
      ASTRA_CHECK_ARG(v.lwf >= 0 && v.lwf <= 2, "variant: lwf must be 0..2 (layer wavefront in 1, 5 or T chunks)");
      continue;
    }
    if (k == "hov") {
      v.head_ov = std::stoi(val);
      ASTRA_CHECK_ARG(v.head_ov >= 0 && v.head_ov <= 2, "variant: hov must be 0..2 (head in 1, 2 or 5 time chunks)");
      continue;
    }
    if (k == "pf") {
      v.l2pf = std::stoi(val);
      ASTRA_CHECK_ARG(v.l2pf >= 0 && v.l2pf <= 3, "variant: pf must be 0..3 (bit 0 fwd chain, bit 1 BPTT chain)");
      continue;
    }
    if (k == "fwd" || k == "bwd") {
      const int mode = std::stoi(val);
      ASTRA_CHECK_ARG(mode >= 0 && mode <= 3, "variant: fwd/bwd mode must be 0 (unfused), 1 (fused per step), 2 "
                                               "(fused persistent) or 3 (small-batch persistent, weight-resident)");
      (k == "fwd" ? v.fwd_mode : v.bwd_mode) = mode;
      continue;
    }
    int r = -1;
    for (int i = 0; i < G_ROLES; ++i)
      if (k == ROLE_NAMES[i]) r = i;
    ASTRA_CHECK_ARG(r >= 0, "variant: unknown variable '" + k + "'");
    KCfg c;
    int n = std::sscanf(val.c_str(), "%d.%d.%d.%d", &c.bn, &c.cm, &c.cn, &c.cg);
    ASTRA_CHECK_ARG(n >= 1, "variant: bad kernel choice '" + val + "'");
    if (n < 4) c.cg = 1;
    if (n < 3) c.cn = 1;
    if (n < 2) c.cm = 1;
    ASTRA_CHECK_ARG(c.cg == 1 || (c.cg == 2 && c.cm == 1 && c.cn == 1 && c.bn >= 128),
                    "variant: CTA pair (4th field 2) needs tile width 128/256 and a 1x1 multicast cluster");
    ASTRA_CHECK_ARG((c.bn == 64 || c.bn == 128 || c.bn == 256 || (c.bn == 224 && c.cg == 2)) &&
                        (c.cm == 1 || c.cm == 2 || c.cm == 4) && (c.cn == 1 || c.cn == 2 || c.cn == 4) && c.cm * c.cn <= 8,
                    "variant: tile width must be 64/128/256 (224: CTA pairs only) and cluster cm, cn in {1,2,4} with cm*cn <= 8");
    v.g[r] = c;
  }
  return v;
}

Mat2 mat(const void* p, long inner, long outer, long ld, long z, long zstride) {
  Mat2 m;
  m.ptr = p; m.inner = inner; m.outer = outer; m.ld = ld; m.z = z; m.zstride = zstride;
  return m;
}
EpiStore epi(void* C, long ldc, int Mv, int Nv, int out_bf16, const float* bias) {
  EpiStore e;
  std::memset(&e, 0, sizeof(e));
  e.C = C; e.ldc = ldc; e.Mv = Mv; e.Nv = Nv; e.out_bf16 = out_bf16; e.bias = bias;
  return e;
}
EpiStore epi_perm(void* C, long ldc, int Mv, int Nv, int perm_u, int perm_blk, int perm_H) {
  EpiStore e = epi(C, ldc, Mv, Nv);
  e.perm_u = perm_u; e.perm_blk = perm_blk; e.perm_H = perm_H;
  return e;
}

Cell::Cell(const astra_cell_desc& dd) : d(dd) {
  ASTRA_CHECK_ARG(d.hidden > 0 && d.input > 0 && d.batch > 0 && d.seq > 0, "cell: sizes must be positive");
  ASTRA_CHECK_ARG(d.dtype == ASTRA_BF16 || d.dtype == ASTRA_FP32, "cell: dtype must be ASTRA_BF16 or ASTRA_FP32");
  ot = d.dtype == ASTRA_BF16 ? OT::BF16 : OT::F32;
  H = d.hidden; I = d.input; B = d.batch; T = d.seq; Tmax = T;
  Hp = (int)round_up(H, 64);
  Ip = (int)round_up(I, 64);
  Hout = H;
  ASTRA_CHECK_ARG((long)T * B < (1L << 31) / 64, "cell: T*B too large");
  std::memset(used_r, 0, sizeof(used_r));
  std::memset(evr, 0, sizeof(evr));
  use_slot(0);
}

void Cell::use_slot(int s) {
  ev_slot = s;
  ev = evr[s];
  region_used = used_r[s];
  for (int r = 0; r < R_COUNT; ++r) region_used[r] = false;
}

void Cell::add_param(const char* n, int r, int c) {
  params.push_back({n, n_params, r, c});
  n_params = (n_params + (size_t)r * c + 63) / 64 * 64;   // every tensor 256-byte aligned
}

Cell::~Cell() {
  for (int k = 0; k < EV_SLOTS; ++k)
    for (int r = 0; r < R_COUNT; ++r)
      for (int w = 0; w < 2; ++w)
        if (evr[k][r][w]) cudaEventDestroy(evr[k][r][w]);
  if (ev_fork) cudaEventDestroy(ev_fork);
  if (ev_join) cudaEventDestroy(ev_join);
  for (int k = 0; k < 4; ++k)
    if (ev_bucket[k]) cudaEventDestroy(ev_bucket[k]);
  if (own_comm_st) cudaStreamDestroy(own_comm_st);
  if (tune_dev) cudaFree(tune_dev);
  if (nccl_comm && own_nccl) ncclCommDestroy((ncclComm_t)nccl_comm);
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
    for (int k = 0; k < 4; ++k) CUDA_TRY(cudaEventCreateWithFlags(&ev_bucket[k], cudaEventDisableTiming));
    for (int k = 0; k < EV_SLOTS; ++k)
      for (int r = 0; r < R_COUNT; ++r)
        for (int w = 0; w < 2; ++w) CUDA_TRY(cudaEventCreate(&evr[k][r][w]));
  }
  bound = true;
  fwd_done = false;
}

void Cell::mark(Region r, int which, cudaStream_t st) {
  if (!profiling) return;
  if (r != R_STEP && !regions_needed()) return;
  if (r == R_STEP && which == 0 && !regions_needed())   // this step's phase regions are not recorded
    for (int q = 0; q < R_COUNT; ++q)
      if (q != R_STEP) region_used[q] = false;
  // External: inside a CUDA-graph capture this becomes a real event-record node (replays keep
  // timing the regions); outside a capture it is a plain record
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  CUDA_TRY(cudaStreamIsCapturing(st, &cs));
  if (cs == cudaStreamCaptureStatusActive)
    CUDA_TRY(cudaEventRecordWithFlags(ev[r][which], st, cudaEventRecordExternal));
  else
    CUDA_TRY(cudaEventRecord(ev[r][which], st));
  if (which) region_used[r] = true;
  if (which && r == R_STEP) last_step_slot = ev_slot;
}

TcGemm& Cell::tc_get(int id, const GemmSpec& s, const KCfg& k, bool plain_maps) {
  // split-K only runs without clusters; the cluster choice then falls back to 1x1 (same numerics)
  const int cm = s.ksplit > 1 ? 1 : k.cm, cn = s.ksplit > 1 ? 1 : k.cn;
  const TcKey key{id, T, k.bn, cm, cn, k.cg, s.A.ptr, s.B.ptr, s.M, s.N, s.K, plain_maps, s.kperm};
  auto it = tc_cache.find(key);
  if (it == tc_cache.end()) {
    TcGemm g;
    // A/B knob: cap the shared memory of the per-step BPTT GEMM (id 2) so the backward pointwise
    // kernel's CTAs can be resident beside it and load their first row before the grid dependency.
    // Same for the per-step recurrent GEMM (id 1) and the forward pointwise kernel.
    static const int bptt_cap = [] {
      const char* e = std::getenv("ASTRA_BPTT_SMEM_KB");
      return e ? std::atoi(e) * 1024 : 0;
    }();
    static const int rec_cap = [] {
      const char* e = std::getenv("ASTRA_REC_SMEM_KB");
      return e ? std::atoi(e) * 1024 : 0;
    }();
    tc_gemm_prepare(g, s.A, s.a_mn, s.B, s.b_mn, s.M, s.N, s.K, k.bn, cm, cn, s.b_keep, s.ksplit, k.cg,
                    id == 2 ? bptt_cap : id == 1 ? rec_cap : 0, plain_maps, s.kperm);
    it = tc_cache.emplace(key, g).first;
  }
  return it->second;
}

void Cell::run_gemm(int id, const GemmSpec& s, const EpiStore& e, int az, int bz, const KCfg& k, cudaStream_t st,
                    const L2Pf* pf, int max_ctas) {
  if (ot == OT::BF16) {
    tc_gemm_launch(tc_get(id, s, k), e, az, bz, st, max_ctas, pf);
  } else {
    const float* A = (const float*)s.A.ptr + (long)az * s.A.zstride;
    const float* Bm = (const float*)s.B.ptr + (long)bz * s.B.zstride;
    long sam, sak, sbk, sbn;
    if (!s.a_mn) { sam = s.A.ld; sak = 1; } else { sam = 1; sak = s.A.ld; }
    if (!s.b_mn) { sbk = 1; sbn = s.B.ld; } else { sbk = s.B.ld; sbn = 1; }
    if (s.ksplit <= 1) {
      simt_gemm(A, sam, sak, Bm, sbk, sbn, s.M, s.N, s.K, e, st);
    } else {
      const int kper = cdiv(cdiv(s.K, TC_BK), s.ksplit) * TC_BK;
      for (int ks = 0; ks < s.ksplit; ++ks) {
        const int k0 = ks * kper, kn = std::min(s.K - k0, kper);
        EpiStore ek = e;
        ek.C = (char*)e.C + (size_t)ks * e.split_stride * 4;
        if (kn > 0) simt_gemm(A + (long)k0 * sak, sam, sak, Bm + (long)k0 * sbk, sbk, sbn, s.M, s.N, kn, ek, st);
      }
    }
  }
}

// K11: bucketed data-parallel gradient sum.  Each bucket is launched on the comm
// stream as soon as the kernel producing it has been enqueued on `producer` (event edge), so the
// NCCL all-reduce of the head / dU / dW buckets overlaps the remaining BPTT and weight-gradient
// work; grad_join() makes `main` wait for every bucket before SGD.  Sum then ×1/world: the mean
// of the shard-mean gradients = the full-batch mean gradient (oracle/dp.py).
void Cell::grad_bucket(float* p, size_t n, cudaStream_t producer) {
  if (world <= 1 || (!nccl_comm && !peer) || n == 0) return;
  cudaStream_t cs = comm_st ? comm_st : producer;
  cudaEvent_t evb = ev_bucket[bucket_i++ % 4];
  if (cs != producer) {
    CUDA_TRY(cudaEventRecord(evb, producer));
    CUDA_TRY(cudaStreamWaitEvent(cs, evb, 0));
  }
  if (peer) {   // K11p: rank-ordered mean of our shard of the bucket, read over NVLink
    ASTRA_CHECK_STATE(p >= peer->G && p + n <= peer->G + peer->n, "grad_bucket: bucket outside the peer window");
    // AV dp_bucket: pieces of at most 128 / 32 / 8 MB (value-neutral: the sum is per element);
    // ASTRA_DPB_DIV shrinks the caps for tests of the splitting on small models
    static const size_t div = [] {
      const char* e = std::getenv("ASTRA_DPB_DIV");
      return e ? std::max<size_t>(1, std::strtoull(e, nullptr, 10)) : 1;
    }();
    const size_t capb[4] = {0, 128u << 20, 32u << 20, 8u << 20};
    // the dp_bucket AV lives on the top layer of an LM (its tree); every layer follows it
    const int dpb = peer->dpb >= 0 ? peer->dpb : var.dpb;
    const size_t cap = dpb > 0 ? std::max<size_t>(64, capb[dpb] / div / 4) : n;
    for (size_t o = 0; o < n; o += cap) peer->reduce((size_t)(p - peer->G) + o, std::min(cap, n - o), cs);
    sync_pending = true;
    return;
  }
  ncclResult_t r = ncclAllReduce(p, p, n, ncclFloat, ncclSum, (ncclComm_t)nccl_comm, cs);
  if (r != ncclSuccess) throw Error(ASTRA_E_NCCL, std::string("ncclAllReduce: ") + ncclGetErrorString(r));
  count_launch();
  scale_inplace(p, n, 1.0f / (float)world, cs);
  sync_pending = true;
}

void Cell::grad_join(cudaStream_t main) {
  if (!sync_pending) return;
  if (comm_st && comm_st != main) {
    CUDA_TRY(cudaEventRecord(ev_join, comm_st));
    CUDA_TRY(cudaStreamWaitEvent(main, ev_join, 0));
  }
  sync_pending = false;
}

void Cell::sgd_step(float lr) {
  ASTRA_CHECK_STATE(bound, "sgd: not bound");
  if (peer && world > 1) {   // owned shards updated, written into every rank's parameters
    std::vector<std::pair<size_t, size_t>> cover;
    for (const ParamInfo& q : params) cover.push_back({q.offset, (size_t)q.rows * q.cols});
    peer->sgd(lr, main_st, cover);
    return;
  }
  sgd(P, G, n_params, lr, main_st);
}

void Cell::ensure_comm_stream() {
  if (comm_st) return;   // no caller comm stream: own a high-priority one so buckets overlap compute
  int lo = 0, hi = 0;
  CUDA_TRY(cudaDeviceGetStreamPriorityRange(&lo, &hi));
  CUDA_TRY(cudaStreamCreateWithPriority(&own_comm_st, cudaStreamNonBlocking, hi));
  comm_st = own_comm_st;
}

// ------------------------------------------------------------------------ tuner glue
// The enumerator's static pruning (A19): per GEMM role, the kernel choices whose tile
// and cluster shape fit the problem; the default (Variant()) first.
static const KCfg CANDIDATES[] = {{256, 1, 1}, {128, 1, 1}, {64, 1, 1}, {256, 1, 1, 2}, {128, 1, 1, 2}, {224, 1, 1, 2},
                                  {256, 2, 1}, {256, 4, 1}, {256, 2, 2}, {256, 1, 2}, {128, 2, 1}, {128, 4, 1},
                                  {128, 2, 2}, {128, 1, 2}, {64, 2, 1}, {64, 4, 1}, {64, 2, 2}};

// Switch the active sequence length (bucket).  The exploration state of the bucket being left is
// parked and the target bucket's restored (or started fresh: the default variant under TUNE_ON,
// the current variant otherwise), so each bucket explores its own update tree.
void Cell::set_active_T(int t) {
  ASTRA_CHECK_ARG(t >= 1 && t <= Tmax, "cell: active length must be in [1, seq]");
  if (t == T) return;
  TuneCtx& cur = tune_ctx[T];
  cur.var = var;
  cur.tree = std::move(tree);
  cur.wirer = std::move(wirer);
  cur.configs_seen = std::move(configs_seen);
  cur.rep_i = rep_i;
  cur.rep_min = rep_min;
  cur.cfg_serial = cfg_serial;
  cur.reps_harvested = reps_harvested;
  for (int r = 0; r < G_ROLES; ++r) cur.allowed[r] = allowed[r];
  auto it = tune_ctx.find(t);
  if (it != tune_ctx.end()) {
    TuneCtx& nx = it->second;
    var = nx.var;
    tree = std::move(nx.tree);
    wirer = std::move(nx.wirer);
    configs_seen = std::move(nx.configs_seen);
    rep_i = nx.rep_i;
    rep_min = nx.rep_min;
    cfg_serial = nx.cfg_serial;
    reps_harvested = nx.reps_harvested;
    for (int r = 0; r < G_ROLES; ++r) allowed[r] = nx.allowed[r];
    tune_ctx.erase(it);
  } else {
    if (tune_mode == ASTRA_TUNE_ON) var = Variant();
    tree.reset();
    wirer.reset();
    configs_seen.clear();
    rep_i = 0;
    rep_min.clear();
    cfg_serial = 0;
    reps_harvested = 0;
  }
  T = t;
  fwd_done = false;
}

void Cell::tuner_setup() {
  const Variant def;
  std::string par;
  const char* metric[G_ROLES] = {"t_a1", "t_fwd", "t_bptt", "t_du", "t_dw", "t_dx", "t_head", "t_head"};
  if (ot == OT::BF16) {
    for (int r = 0; r < G_ROLES; ++r) {
      if ((r == G_HEAD || r == G_HDY) && !lm_mode) continue;
      int M, N;
      if (r == G_HDY) {
        M = T * B;
        N = y_width();
      } else {
        role_shape(r, M, N);
      }
      if (M <= 0 || N <= 0) continue;
      allowed[r].clear();
      allowed[r].push_back(def.g[r]);
      for (const KCfg& k : CANDIDATES) {
        if (k == def.g[r]) continue;
        const int num_m = cdiv(M, TC_BM), num_n = cdiv(N, k.bn);
        if (k.bn > 64 && N <= k.bn / 2) continue;                                     // tile wider than N
        if (k.cm > num_m || k.cn > num_n) continue;                                    // idle cluster ranks
        if (k.cg == 2 && num_m < 2) continue;                                          // idle pair half
        allowed[r].push_back(k);
      }
      par += std::string(" (leaf g_") + ROLE_NAMES[r] + " " + std::to_string(allowed[r].size()) + " " + metric[r] + ")";
    }
  }
  // §8(a.9) gate_chunking: how many GEMMs the fused gate projection a1 is cut into
  // and on how many streams they run — a parallel sibling of the kernel choices, metric t_a1
  if (ot == OT::BF16 && gate_chunkings() > 1)
    par += " (leaf gate_chunking " + std::to_string(gate_chunkings()) + " t_a1)";
  std::string t = par.empty() ? "" : "(par" + par + ")";
  // reading R26: the forward fusion choice (GEMM + pointwise kernel vs the fused recurrent kernel,
  // P:120-126 "fusion" AV) is tuned after the kernel choices, against the forward-chain time
  if (ot == OT::BF16 && fwd_fusions() > 1)
    t = "(pre " + t + " (leaf fuse_fwd " + std::to_string(fwd_fusions()) + " " + fwd_fusion_metric() + "))";
  if (ot == OT::BF16 && bwd_fusions() > 1)
    t = "(pre " + t + " (leaf fuse_bwd " + std::to_string(bwd_fusions()) + " t_bptt))";
  // the backward pointwise kernel's form (bwd_kernel AV), against the BPTT-chain time
  if (ot == OT::BF16 && bwd_pw_forms() > 1)
    t = "(pre " + t + " (leaf bwd_pw " + std::to_string(bwd_pw_forms()) + " t_bptt))";
  // B3 stream assignment of the chains themselves: the batch's row halves as two independent chains
  // on two streams, against the whole step (both chains and everything they overlap with)
  if (ot == OT::BF16 && !side.empty() && row_stream_options() > 1)
    t = "(pre " + t + " (leaf row_streams " + std::to_string(row_stream_options()) + " t_step))";
  // reading R31: L2 prefetch by the chain GEMMs, per chain, after the kernel and fusion choices
  if (ot == OT::BF16 && chain_prefetch())
    t = "(pre " + t + " (par (leaf pf_fwd 2 t_fwd) (leaf pf_bwd 2 t_bptt)))";
  if (!side.empty()) t = t.empty() ? "(leaf wg_side 2 t_se4)" : "(pre " + t + " (leaf wg_side 2 t_se4))";
  // §8(a.9) wgrad_schedule (P:245-247 equivalence over streams): the input dgrad's time chunks run
  // on a side stream during BPTT instead of after it; BPTT + SE4 together, so the step metric
  if (ot == OT::BF16 && !side.empty() && wgrad_schedules() > 1)
    t = "(pre " + t + " (leaf wgrad_schedule " + std::to_string(wgrad_schedules()) + " t_step))";
  // B3 stream assignment for the LM head: time-chunked on a side stream, overlapping the forward
  // chain (its chunks' logits / CE / dgrad) and the BPTT chain (its weight gradient); step metric
  if (lm_mode && lm_role == 2 && !side.empty() && T >= 2)
    t = "(pre " + t + " (leaf head_ov " + std::to_string(T >= 5 ? 3 : 2) + " t_step))";
  // stacked LM (top layer): layer wavefront, against the whole step
  if (lm_mode && lm_role == 2 && lm_layers > 1 && lm_wavefront && T >= 2)
    t = "(pre " + t + " (leaf lwf " + std::to_string(T > 5 ? 3 : 2) + " t_step))";
  // §8(a.9) dp_bucket: the gradient bucket size is a free variable only under the rank-ordered
  // peer-memory sum (K11p: the bits do not depend on it); last in the prefix order, step metric
  if (world > 1 && peer && peer->ready && (!lm_mode || lm_role == 2))
    t = t.empty() ? "(leaf dp_bucket 4 t_step)" : "(pre " + t + " (leaf dp_bucket 4 t_step))";
  if (t.empty()) t = "(leaf none 1 t_step)";
  // SURVEY §8(f) rank 4 / §8(a.9) `alloc`: store-vs-recompute of the recurrent projection is a
  // memory-allocation context: the whole tree is explored under each context, then
  // each context's best configuration is raced end to end, 3 steps each
  // The gate layout (gate-interleaved vs gate-blocked, reading R38) is the other allocation context:
  // with both, the fork leaf `alloc` has 4 contexts, option o = recompute (o & 1) × gate-blocked (o >> 1)
  if (ot == OT::BF16 && supports_recompute() && supports_gate_blocked())
    t = "(fork (leaf alloc 4 t_step) t_step " + t + " 3)";
  else if (ot == OT::BF16 && supports_recompute())
    t = "(fork (leaf recomp 2 t_step) t_step " + t + " 3)";
  tree.reset(new tuner::Tree(tuner::parse(t)));
  wirer.reset(new tuner::Wirer(tree.get()));
  wirer->index().bucket = T;
  wirer->start();
  configs_seen.clear();
  tuner::Config c;
  if (wirer->propose(c)) apply_config(c);
  rep_i = 0;
  cfg_serial = next_serial++;
  reps_harvested = 0;
}

void Cell::apply_config(const tuner::Config& c) {
  Variant v = var;
  for (size_t i = 0; i < tree->avs.size(); ++i) {
    const std::string& n = tree->avs[i];
    const int o = c[i];
    if (n == "wg_side") { v.wg_side = o; continue; }
    if (n == "fuse_fwd") { v.fwd_mode = o; continue; }
    if (n == "fuse_bwd") { v.bwd_mode = o; continue; }
    if (n == "head_ov") { v.head_ov = o; continue; }
    if (n == "lwf") { v.lwf = o; continue; }
    if (n == "recomp") { v.recomp = o; continue; }
    if (n == "alloc") { v.recomp = o & 1; v.gblk = o >> 1; continue; }
    if (n == "dp_bucket") { v.dpb = o; continue; }
    if (n == "gate_chunking") { v.gchunk = o; continue; }
    if (n == "wgrad_schedule") { v.wgs = o; continue; }
    if (n == "bwd_pw") { v.bpw = o; continue; }
    if (n == "row_streams") { v.rsp = o; continue; }
    if (n == "pf_fwd") { v.l2pf = (v.l2pf & ~1) | o; continue; }
    if (n == "pf_bwd") { v.l2pf = (v.l2pf & ~2) | (o << 1); continue; }
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

tuner::Metrics Cell::read_metrics(int slot) {
  cudaEvent_t (*E)[2] = evr[slot];
  const bool* used = used_r[slot];
  tuner::Metrics m(tree->metrics.size(), 0.0);
  for (size_t i = 0; i < tree->metrics.size(); ++i) {
    const std::string& n = tree->metrics[i];
    double v = 0;
    if (n == "t_a1") v = elapsed(E[R_A1][0], E[R_A1][1]);
    else if (n == "t_fwd") v = elapsed(E[R_FWD][0], E[R_FWD][1]);
    else if (n == "t_bptt") v = elapsed(E[R_BPTT][0], E[R_BPTT][1]);
    else if (n == "t_du") v = used[R_DU] ? elapsed(E[R_DU][0], E[R_DU][1]) : 0;
    else if (n == "t_dw") v = used[R_DW] ? elapsed(E[R_DW][0], E[R_DW][1]) : 0;
    else if (n == "t_dx") v = used[R_DX] ? elapsed(E[R_DX][0], E[R_DX][1]) : 0;
    else if (n == "t_head") v = used[R_HEAD] ? elapsed(E[R_HEAD][0], E[R_HEAD][1]) : 0;
    else if (n == "t_se4") v = elapsed(E[R_SE4][0], E[R_SE4][1]);
    else v = elapsed(E[R_STEP][0], E[R_STEP][1]);
    m[i] = v;
  }
  return m;
}

// Fold the finished measured steps, oldest first, into the min-over-reps of the configuration
// (and bucket) they measured.  A step is finished when its step-end event has completed
// (cudaEventQuery).  wait = 1: also wait for every pending step except the newest — the step just
// enqueued is never waited for, so the GPU always has it queued while the host decides; wait = 2:
// wait for all of them (a cross-rank decision, reading R29).
void Cell::harvest(int wait) {
  size_t k = 0;
  for (; k < pending.size(); ++k) {
    const PendingRep& p = pending[k];
    cudaEvent_t end = evr[p.slot][R_STEP][1];
    if (wait == 2 || (wait == 1 && k + tune_lag < pending.size())) {
      if (cudaEventQuery(end) == cudaErrorNotReady) ++tune_blocks;
      CUDA_TRY(cudaEventSynchronize(end));
    } else {
      const cudaError_t q = cudaEventQuery(end);
      if (q == cudaErrorNotReady) break;
      if (q != cudaSuccess) CUDA_TRY(q);
    }
    // the measured configuration is the active one, or a parked bucket's (still current there)
    tuner::Metrics* rm = nullptr;
    int* nh = nullptr;
    if (p.T == T && p.serial == cfg_serial) { rm = &rep_min; nh = &reps_harvested; }
    else {
      auto it = tune_ctx.find(p.T);
      if (it != tune_ctx.end() && it->second.cfg_serial == p.serial) { rm = &it->second.rep_min; nh = &it->second.reps_harvested; }
    }
    if (!rm) continue;   // a configuration that has been decided already: surplus measurement
    tuner::Metrics m = read_metrics(p.slot);
    if (*nh == 0 || rm->size() != m.size()) *rm = m;
    else
      for (size_t i = 0; i < m.size(); ++i) (*rm)[i] = std::min((*rm)[i], m[i]);
    ++*nh;
  }
  pending.erase(pending.begin(), pending.begin() + k);
}

// One call per step (after the step's work is enqueued).  Per configuration: one warm-up step
// (absorbs lazy tensor-map creation), then measured steps whose region times are min-reduced
// (reading R19: clocks float on B200 so k = 3 reps instead of the paper's pinned clocks).
// Never waits for the step just enqueued (include/astra.h): a measured step's events are harvested
// with cudaEventQuery once the GPU has finished it; the configuration keeps running (real training
// steps, so the exploration stays work-conserving) until tune_reps of its measured steps are in,
// waiting at most for the steps before the newest tune_lag (1) — the GPU is busy with those
// meanwhile, so host and GPU stay pipelined and a configuration costs at most 1 warm-up + tune_reps
// + tune_lag steps.  With world > 1 every rank must decide at the same step (reading R29), so there the
// decision step is fixed — the tune_reps-th measured step — and waits for its events.
int Cell::tune_next() {
  if (tune_mode != ASTRA_TUNE_ON) return tune_mode == ASTRA_TUNE_FROZEN ? ASTRA_TUNE_CONVERGED : ASTRA_TUNE_IDLE;
  ASTRA_CHECK_STATE(world <= 1 || nccl_comm,
                    "tune_next: exploring with world > 1 needs astra_comm_init (cross-rank decisions, reading R29)");
  if (!wirer) tuner_setup();
  if (racing) return race_step();
  if (wirer->converged()) return ASTRA_TUNE_CONVERGED;
  auto advance = [&] {   // the next step records into a slot no pending measurement uses
    int s = (ev_slot + 1) % EV_SLOTS;
    for (int tries = 0; tries < EV_SLOTS; ++tries, s = (s + 1) % EV_SLOTS) {
      bool busy = false;
      for (const PendingRep& p : pending) busy |= p.slot == s;
      if (!busy) break;
    }
    for (const PendingRep& p : pending)
      if (p.slot == s) { harvest(1); break; }   // ring full: wait for the older ones
    use_slot(s);
  };
  if (rep_i == 0) {  // warm-up step done
    rep_i = 1;
    advance();
    return ASTRA_TUNE_EXPLORING;
  }
  pending.push_back({ev_slot, T, cfg_serial});
  ++rep_i;
  // world > 1: decide at the tune_reps-th measured step on every rank (wait for all of them);
  // one rank: once tune_reps measured steps precede the newest, wait for those (the newest keeps
  // running on the GPU), else only fold in what has finished
  if (world > 1) harvest(rep_i > tune_reps ? 2 : 0);
  else harvest(rep_i > tune_reps + tune_lag ? 1 : 0);
  if (reps_harvested < tune_reps) {
    advance();
    return ASTRA_TUNE_EXPLORING;
  }
  if (world > 1 && nccl_comm) {
    // reading R29: every rank must take the same decision — max-reduce the metric vector
    const size_t n = rep_min.size();
    ASTRA_CHECK_STATE(n <= 64, "tuner: too many metrics");
    CUDA_TRY(cudaMemcpyAsync(tune_dev, rep_min.data(), n * sizeof(double), cudaMemcpyHostToDevice, main_st));
    ncclResult_t r = ncclAllReduce(tune_dev, tune_dev, n, ncclDouble, ncclMax, (ncclComm_t)nccl_comm, main_st);
    if (r != ncclSuccess) throw Error(ASTRA_E_NCCL, std::string("ncclAllReduce(max): ") + ncclGetErrorString(r));
    CUDA_TRY(cudaMemcpyAsync(rep_min.data(), tune_dev, n * sizeof(double), cudaMemcpyDeviceToHost, main_st));
    CUDA_TRY(cudaStreamSynchronize(main_st));
  }
  wirer->feed(rep_min);
  rep_i = 0;
  reps_harvested = 0;
  cfg_serial = next_serial++;
  advance();
  tuner::Config c;
  if (wirer->propose(c)) {
    apply_config(c);
    return ASTRA_TUNE_EXPLORING;
  }
  apply_config(wirer->final_config());
  configs_seen.pop_back();
  if (race_start()) return ASTRA_TUNE_EXPLORING;
  return ASTRA_TUNE_CONVERGED;
}

bool Cell::race_start() {
  race_winner = -1;
  const char* e = std::getenv("ASTRA_TUNE_RACE");
  if ((e && e[0] == '0') || world > 1 || !tune_ctx.empty() || !tree || !wirer) return false;
  const tuner::Config fin = wirer->final_config();
  int ctx = 0;   // the allocation context of the converged configuration: the fork leaf's option
  for (const char* f : {"alloc", "recomp"}) {
    const int i = tree->av_index(f);
    if (i >= 0) { ctx = fin[i]; break; }
  }
  const char* me = std::getenv("ASTRA_TUNE_RACE_MARGIN");   // tests: widen the 10 % window
  const double margin = me ? std::atof(me) : 0.10;
  const auto& d = wirer->index().d;
  race_cfg.assign(1, fin);
  // the alternatives (at most 5): the chain-form AVs' options, then the per-step chain GEMMs' kernel
  // choices, closest first within each group, each within `margin` of the chosen one in the index
  std::vector<std::pair<double, tuner::Config>> alts;
  for (const char* a : {"fuse_fwd", "fuse_bwd", "bwd_pw", "row_streams", "g_rec", "g_bptt"}) {
    const int i = tree->av_index(a);
    if (i < 0) continue;
    auto key = [&](int k) { return tuner::ProfileIndex::key(ctx, a, std::to_string(k), wirer->index().bucket); };
    const auto it = d.find(key(fin[i]));
    if (it == d.end() || !(it->second > 0)) continue;
    for (int k = 0; k < tree->av_n[i]; ++k) {
      if (k == fin[i]) continue;
      const auto jt = d.find(key(k));
      if (jt == d.end() || jt->second > it->second * (1.0 + margin)) continue;
      tuner::Config c = fin;
      c[i] = k;
      // the chain-form AVs first (their options differ most in clock sensitivity), then the kernels
      const bool form = a[0] != 'g';
      alts.push_back({jt->second / it->second + (form ? 0.0 : 10.0), c});
    }
  }
  std::stable_sort(alts.begin(), alts.end(), [](const auto& x, const auto& y) { return x.first < y.first; });
  for (size_t k = 0; k < alts.size() && race_cfg.size() < 6; ++k) race_cfg.push_back(alts[k].second);
  if (race_cfg.size() < 2) return false;
  constexpr int ROUNDS = 5;
  race_seq.clear();
  for (int r = 0; r < ROUNDS; ++r)
    for (int c = 0; c < (int)race_cfg.size(); ++c) race_seq.push_back(c);
  race_best.assign(race_cfg.size(), 1e30);
  race_pending.clear();
  race_pos = 0;
  race_sub = 0;
  racing = true;
  apply_config(race_cfg[race_seq[0]]);   // the next step: warm-up of the first candidate
  return true;
}

void Cell::race_harvest(bool wait_all) {
  size_t k = 0;
  for (; k < race_pending.size(); ++k) {
    cudaEvent_t end = evr[race_pending[k].slot][R_STEP][1];
    if (wait_all) {
      if (cudaEventQuery(end) == cudaErrorNotReady) ++tune_blocks;
      CUDA_TRY(cudaEventSynchronize(end));
    } else {
      const cudaError_t q = cudaEventQuery(end);
      if (q == cudaErrorNotReady) break;
      if (q != cudaSuccess) CUDA_TRY(q);
    }
    const int s = race_pending[k].slot;
    const double v = elapsed(evr[s][R_STEP][0], evr[s][R_STEP][1]);
    double& b = race_best[race_pending[k].cand];
    b = std::min(b, v);
  }
  race_pending.erase(race_pending.begin(), race_pending.begin() + k);
}

void Cell::race_advance() {   // the next step records into a slot no pending race measurement uses
  for (int tries = 0; tries < 2; ++tries) {
    int s = (ev_slot + 1) % EV_SLOTS;
    for (int n = 0; n < EV_SLOTS; ++n, s = (s + 1) % EV_SLOTS) {
      bool busy = false;
      for (const RacePend& p : race_pending) busy |= p.slot == s;
      if (!busy) { use_slot(s); return; }
    }
    race_harvest(true);   // ring full: wait for the older measurements
  }
  use_slot((ev_slot + 1) % EV_SLOTS);
}

int Cell::race_step() {
  if (race_sub == 0) {   // the warm-up step of race_seq[race_pos] ran: the next one is measured
    race_sub = 1;
    race_advance();
    return ASTRA_TUNE_EXPLORING;
  }
  race_pending.push_back({ev_slot, race_seq[race_pos]});
  ++race_pos;
  race_sub = 0;
  race_harvest(false);
  if (race_pos < race_seq.size()) {
    apply_config(race_cfg[race_seq[race_pos]]);
    race_advance();
    return ASTRA_TUNE_EXPLORING;
  }
  race_harvest(true);
  int best = 0;   // an alternative replaces the converged configuration only if faster by > TOL
  for (int c = 1; c < (int)race_cfg.size(); ++c)
    if (race_best[c] < race_best[best] * (1.0 - tuner::TOL)) best = c;
  race_winner = best;
  apply_config(race_cfg[best]);
  racing = false;
  race_advance();
  return ASTRA_TUNE_CONVERGED;
}

std::string Cell::report() {
  std::ostringstream o;
  o << "{\"variant\": \"" << var.str() << "\", \"mode\": " << tune_mode << ", \"bucket\": " << T;
  if (!tune_ctx.empty()) {   // the parked buckets: their current variant and exploration state
    o << ", \"other_buckets\": {";
    size_t k = 0;
    for (auto& kv : tune_ctx)
      o << (k++ ? ", " : "") << "\"" << kv.first << "\": {\"variant\": \"" << kv.second.var.str()
        << "\", \"converged\": " << (kv.second.wirer && kv.second.wirer->converged() ? "true" : "false")
        << ", \"configs_explored\": " << (kv.second.wirer ? kv.second.wirer->trials() : 0) << "}";
    o << "}";
  }
  if (wirer) {
    o << ", \"converged\": " << (wirer->converged() ? "true" : "false") << ", \"configs_explored\": "
      << wirer->trials() << ", \"measured_reps\": " << tune_reps << ", \"harvest_waits\": " << tune_blocks
      << ", \"index_entries\": "
      << wirer->index().d.size() << ", \"tree_avs\": [";
    for (size_t i = 0; i < tree->avs.size(); ++i) o << (i ? ", " : "") << "\"" << tree->avs[i] << "\"";
    o << "]";
    if (!race_cfg.empty() && race_cfg.size() == race_best.size()) {   // the final race (R41)
      o << ", \"race\": {\"winner\": " << race_winner << ", \"candidates\": [";
      for (size_t c = 0; c < race_cfg.size(); ++c) {
        Variant v = var;
        for (size_t i = 0; i < tree->avs.size() && i < race_cfg[c].size(); ++i) {
          const std::string& n = tree->avs[i];
          const int x = race_cfg[c][i];
          if (n == "fuse_fwd") v.fwd_mode = x;
          else if (n == "fuse_bwd") v.bwd_mode = x;
          else if (n == "bwd_pw") v.bpw = x;
          else if (n == "row_streams") v.rsp = x;
          else if (n == "g_rec" && x < (int)allowed[G_REC].size()) v.g[G_REC] = allowed[G_REC][x];
          else if (n == "g_bptt" && x < (int)allowed[G_BPTT].size()) v.g[G_BPTT] = allowed[G_BPTT][x];
        }
        o << (c ? ", " : "") << "{\"fwd\": " << v.fwd_mode << ", \"bwd\": " << v.bwd_mode << ", \"bpw\": " << v.bpw
          << ", \"rsp\": " << v.rsp << ", \"rec\": \"" << v.g[G_REC].bn << "." << v.g[G_REC].cm << "." << v.g[G_REC].cn
          << "." << v.g[G_REC].cg << "\", \"bptt\": \"" << v.g[G_BPTT].bn << "." << v.g[G_BPTT].cm << "." << v.g[G_BPTT].cn
          << "." << v.g[G_BPTT].cg << "\", \"t_step_min\": " << race_best[c] << "}";
      }
      o << "]}";
    }
    o << ", \"index\": {";
    size_t k = 0;
    for (auto& kv : wirer->index().d) o << (k++ ? ", " : "") << "\"" << kv.first << "\": " << kv.second;
    o << "}";
  }
  o << "}";
  return o.str();
}

std::unique_ptr<Cell> make_lstm_cell(const astra_cell_desc& d);
std::unique_ptr<Cell> make_scrn_cell(const astra_cell_desc& d);
std::unique_ptr<Cell> make_rhn_cell(const astra_cell_desc& d);
std::unique_ptr<Cell> make_attn_cell(const astra_cell_desc& d);

std::unique_ptr<Cell> make_cell(const astra_cell_desc& d) {
  switch (d.cell_type) {
    case ASTRA_LSTM:
    case ASTRA_MILSTM:
    case ASTRA_SUBLSTM: return make_lstm_cell(d);
    case ASTRA_SCRNN: return make_scrn_cell(d);
    case ASTRA_RHN: return make_rhn_cell(d);
    case ASTRA_LSTM_ATTN: return make_attn_cell(d);
    default: throw Error(ASTRA_E_ARG, "cell: unknown cell_type");
  }
}

}  // namespace astra
