// libasgd host side: the C ABI of include/asgd.h.
//  - replica ctx (the paper's GPU manager, PAPER.md P:1184-1198 / Fig. 3):
//    workspace carve-up, per-step kernel sequence, merge entry points;
//  - host-pure algorithms: Alg. 1, Alg. 2 lines 1-7,
//    routing replay / simulated clock, P@k counting;
//  - the dynamic scheduler as a lock-free ticket counter in
//    POSIX shared memory, shared by the one-process-per-GPU ranks.
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <list>
#include <map>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include <cuda.h>

#include "asgd_internal.h"

using namespace asgd;

namespace {

thread_local std::string g_err;

int fail(int code, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

int cuda_fail(cudaError_t e, const char* where) {
  return fail(ASGD_E_CUDA, "%s: %s (%s)", where, cudaGetErrorName(e), cudaGetErrorString(e));
}

#define CU(call)                                              \
  do {                                                        \
    cudaError_t _e = (call);                                  \
    if (_e != cudaSuccess) return cuda_fail(_e, #call);       \
  } while (0)

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

size_t up256(size_t x) { return (x + 255) & ~size_t(255); }

constexpr int kSqnormParts = 1024;
constexpr int kMaxInflight = 8;
constexpr size_t kMaxTrace = 1 << 16;   // traced steps kept between two asgd_trace_read calls
// Above this many bytes of fp32 logits per step the bf16 path fuses softmax-CE
// into the GEMMs (Z never written); below, Z stays L2-resident and is stored.
// Measured: AmazonCat-13K (54.6 MB) 4.99M -> 5.35M samples/s fused; Wiki10-31K
// (31.7 MB) neutral; EURLex-4K (4 MB) stays unfused.
constexpr int64_t kFusedCeBytes = 32ll << 20;
// threshold override in MB (A/B experiments only)
int64_t fused_ce_bytes() {
  static const int64_t v = [] {
    const char* e = getenv("ASGD_FUSED_CE_MB");
    return e ? (int64_t)atoll(e) << 20 : kFusedCeBytes;
  }();
  return v;
}

// K-3's dH1 half (k_bwd_dh) in the fused softmax-CE regime (default); ASGD_BWD_FUSE=0 keeps
// G1b + G2 (A/B).
bool bwd_fuse() {
  static const bool v = [] { const char* e = getenv("ASGD_BWD_FUSE"); return !(e && e[0] == '0'); }();
  return v;
}
// K-3's dW2 half (k_bwd_dw, replaces G3 there and dZ never reaches HBM): ASGD_BWD_DW=1.
// Off by default: measured at Amazon-670K 2.59 ms vs 2.16 ms per step -- k_bwd_dh without the
// dZ store drops 885 -> 644 us, but k_bwd_dw takes 1,374 us against G3's 625 (its SGD
// epilogue, 128 KB of fp32 W2 read-modify-write per tile, cannot overlap the next tile's
// MMAs: the dW2 accumulator takes 256 of TMEM's 512 columns and cannot be double-buffered).
bool bwd_dw() {
  static const bool v = [] { const char* e = getenv("ASGD_BWD_DW"); return e && e[0] == '1'; }();
  return v;
}

// G2 with the dH1 reduce + b1 update fused into its tail (ASGD_G2_FUSE=1).  Off by default:
// measured on EURLex-4K (bf16) 6.99 ms vs 6.30 ms per mega-batch -- the tail's grid barrier
// and its 30-CTA reduce cost more than the separate 256-CTA k_dh_reduce launch (b1 runs
// off the critical path on s3).  The same tail ends K-3's k_bwd_dh, where the grid is 144 CTAs.
// K-3 one-pass for the stored-Z regime (bf16, softmax, H = 256: EURLex-4K): k_bwd_dh alone
// replaces G1 + softmax-CE + G2 + the dH reduce on the critical path (ASGD_ONEPASS=1).
// Measured slower at EURLex (34 vs ~25 us for the four kernels): with one label tile per
// CTA the 63 dH1 partials (16 MB) and two grid barriers outweigh the launches it saves.
bool one_pass_on() {
  static const bool v = [] { const char* e = getenv("ASGD_ONEPASS"); return e && e[0] == '1'; }();
  return v;
}
// K-3 softmax-only for the stored-Z regime (ASGD_K3DZ=1): k_bwd_dh with one label tile per
// CTA stands for G1 + softmax-CE (statistics from its S tiles, a grid barrier, dZ stored)
bool k3dz_on() {
  static const bool v = [] { const char* e = getenv("ASGD_K3DZ"); return e && e[0] == '1'; }();
  return v;
}
bool g2_fuse() {
  static const bool v = [] { const char* e = getenv("ASGD_G2_FUSE"); return e && e[0] == '1'; }();
  return v;
}

int splitk_for(const asgd_model_desc& d) {
  // G2 (dH1 = dZ W2, M = b_max, N = H, K = L): split K so ~2 waves of CTAs run (ASGD_G2_WAVES;
  // one wave measured: Amazon-670K G2 372 -> 602 us, Delicious-200K 125 -> 192 us, AmazonCat even)
  int64_t tiles;
  // N tile: 256 (bf16) or 128 (bf16x3 fp32 path, R14: hi + lo stages)
  if (d.precision == ASGD_PREC_BF16) tiles = ((d.b_max + 127) / 128) * ((d.H + 255) / 256);
  else tiles = ((d.b_max + 127) / 128) * ((d.H + 127) / 128);
  static const int64_t waves = [] { const char* e = getenv("ASGD_G2_WAVES"); return e ? atoll(e) : 2ll; }();
  int64_t s = (waves * 148 + tiles - 1) / tiles;
  s = std::min<int64_t>(s, std::max<int64_t>(1, d.L / 256));
  if (const char* e = getenv("ASGD_SPLITK")) s = std::max<int64_t>(1, atoll(e));   // A/B override
  return (int)std::max<int64_t>(1, std::min<int64_t>(s, 64));
}

}  // namespace

namespace asgd {

WsLayout ws_layout(const asgd_model_desc& d) {
  WsLayout L{};
  const int64_t F = d.F, H = d.H, Lb = d.L, B = d.b_max;
  L.nz_cap = d.max_step_nnz;
  L.nl_cap = d.max_step_labels;
  L.u_cap = std::min<int64_t>(F, L.nz_cap);
  L.n_pieces = (L.nz_cap + kPiece - 1) / kPiece;
  L.n_tiles_f = (F + kScanTile - 1) / kScanTile;
  L.splitk = splitk_for(d);
  L.n_rowblk = (B + row_block() - 1) / row_block();
  const int64_t Lp = padded_ld(Lb);
  L.n_red = kSqnormParts;
  L.part_stride = B * H;
  // both paths run the output layer on the tensor cores: bf16 operands, or (fp32 path,
  // R14) bf16x3 hi + lo operands -- every bf16 operand buffer exists on both paths
  const bool bf = true;
  L.x3 = d.precision != ASGD_PREC_BF16;
  size_t o = 0;
  auto take = [&](size_t bytes) { size_t r = o; o = up256(o + std::max<size_t>(bytes, 1)); return r; };
  L.meta = take(64 * 4);
  L.boff = take((B + 1) * 4);
  L.loff = take((B + 1) * 4);
  L.cnt = take(F * 4);
  L.fseg = take(F * 4);
  L.fuid = take(F * 4);
  L.uniq = take((L.u_cap + 1) * 4);
  L.useg = take((L.u_cap + 1) * 4);
  L.tsum = take(L.n_tiles_f * 16);   // K-0 tile (count, touched) sums, double-buffered
  L.tpre = take(L.n_tiles_f * 8);
  L.e_n = take(L.nz_cap * 4);
  L.e_v = take(L.nz_cap * 4);
  L.e_u = take(L.nz_cap * 4);
  L.e_f = take(L.nz_cap * 4);
  L.part1 = take((size_t)2 * L.n_pieces * H * 4);
  L.rowcnt = take(B * 4);
  L.part5 = take((size_t)2 * L.n_pieces * H * 4);
  L.ucnt = take((L.u_cap + 1) * 4 * 8);   // per (segment, column slice)
  L.bits = take((size_t)F * ((B + 31) / 32) * 4);   // K-0 row bitmap per feature (zero between steps)
  L.h1 = take(B * H * 4);
  L.h1b = take(bf ? B * H * 2 : 0);
  L.z = take((size_t)B * Lp * 4);
  L.dzb = take(bf ? (size_t)B * Lp * 2 : 0);
  L.rbase = take((size_t)(B + 1) * 8);
  L.da1b = take(bf ? (size_t)B * H * 2 : 0);
  L.stats_ld = B;
  L.lse = take(B * 4);
  L.zstat = take(bf ? (size_t)((Lb + 31) / 32 + 8) * B * 8 : 0);   // G1 partials (2 or 4 per N tile)
  L.rowloss = take(B * 4);
  // K-3 one-pass regime (bf16 softmax, H = 256, logits below the fused-CE bound): room for
  // one dH1 partial per label tile of 64 (at most 64), so every SM gets a K-3 CTA
  L.dh_parts = L.splitk;
  if (d.precision == ASGD_PREC_BF16 && d.loss == ASGD_LOSS_SOFTMAX && H == 256 && B * Lb * 4 <= fused_ce_bytes())
    L.dh_parts = std::max<int64_t>(L.splitk, std::min<int64_t>((Lb + 63) / 64, 64));
  L.dhpart = take((size_t)L.dh_parts * B * H * 4);
  L.da1 = take(B * H * 4);
  L.db1part = take(std::max<int64_t>(L.n_rowblk, 160) * H * 4);   // + G2's fused column partials
  L.w2b = take(bf ? (size_t)Lb * H * 2 : 0);
  L.w2b2 = take(bf ? (size_t)Lb * H * 2 : 0);
  L.red = take((L.n_red + 8) * 8);
  L.eval_top = take(B * 8 * 4);
  L.rowsc = take(B * 4);
  L.cen = take(bf ? (size_t)2 * H * 4 : 0);
  L.cenpart = take(bf ? (size_t)2 * kCenterParts * H * 4 : 0);
  L.h1l = take(L.x3 ? B * H * 2 : 0);
  L.dzl = take(L.x3 ? (size_t)B * Lp * 2 : 0);
  L.w2l = take(L.x3 ? (size_t)Lb * H * 2 : 0);
  L.w2l2 = take(L.x3 ? (size_t)Lb * H * 2 : 0);
  L.total = o;
  return L;
}

Ptrs ws_ptrs(char* b, const WsLayout& L) {
  Ptrs p;
  p.meta = (int32_t*)(b + L.meta); p.boff = (int32_t*)(b + L.boff); p.loff = (int32_t*)(b + L.loff);
  p.cnt = (int32_t*)(b + L.cnt); p.fseg = (int32_t*)(b + L.fseg); p.fuid = (int32_t*)(b + L.fuid);
  p.uniq = (int32_t*)(b + L.uniq); p.useg = (int32_t*)(b + L.useg); p.tsum = (int32_t*)(b + L.tsum);
  p.tpre = (int32_t*)(b + L.tpre); p.e_n = (int32_t*)(b + L.e_n); p.e_v = (float*)(b + L.e_v);
  p.e_u = (int32_t*)(b + L.e_u); p.e_f = (int32_t*)(b + L.e_f);
  p.bits = (uint32_t*)(b + L.bits); p.part1 = (float*)(b + L.part1); p.rowcnt = (int32_t*)(b + L.rowcnt);
  p.part5 = (float*)(b + L.part5); p.ucnt = (int32_t*)(b + L.ucnt); p.h1 = (float*)(b + L.h1);
  p.h1b = (bf16*)(b + L.h1b); p.z = (float*)(b + L.z); p.dzb = (bf16*)(b + L.dzb);
  p.rowloss = (float*)(b + L.rowloss); p.dhpart = (float*)(b + L.dhpart); p.da1 = (float*)(b + L.da1);
  p.db1part = (float*)(b + L.db1part); p.w2b = (bf16*)(b + L.w2b); p.red = (double*)(b + L.red);
  p.eval_top = (int32_t*)(b + L.eval_top);
  p.rbase = (int64_t*)(b + L.rbase);
  p.da1b = (bf16*)(b + L.da1b);
  p.lse = (float*)(b + L.lse);
  p.rowsc = (int32_t*)(b + L.rowsc);
  p.cen = (float*)(b + L.cen);
  p.cenpart = (float*)(b + L.cenpart);
  p.h1l = L.x3 ? (bf16*)(b + L.h1l) : nullptr;
  p.dzl = L.x3 ? (bf16*)(b + L.dzl) : nullptr;
  p.w2l = L.x3 ? (bf16*)(b + L.w2l) : nullptr;
  return p;
}

}  // namespace asgd

// One captured local step (everything after K-0 (a), which is launched eagerly
// with the step's row ids, lr and loss pointer and publishes them to the rest).
struct StepGraph {
  int n = 0, cur = 0, steps = 1;      // steps: local steps captured back to back (step groups)
  asgd_csr data{};                    // the dataset its kernels were captured with
  uint32_t mask = 0;
  int seen = 0;                       // captured on the 2nd step with this key
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t exec = nullptr;
  int64_t kernels = 0;                // kernel nodes (asgd_kernel_launches per replay)
  struct Prof { cudaGraphNode_t node; int cls; bool begin; };
  std::vector<Prof> prof;             // profiling event-record nodes, capture order
  struct ArgNode { cudaGraphNode_t node; cudaKernelNodeParams p; std::vector<void*> args; };
  std::vector<ArgNode> arg_nodes;     // K-0 and K-1 of each step: parameter 0 (StepArgs) per replay
  std::vector<StepArgs> sas;          // per step: storage parameter 0 of its arg_nodes points at
  std::vector<cudaEvent_t> placeholders;
  uint64_t last_use = 0;
};

struct asgd_ctx {
  asgd_model_desc d;
  int device;
  int sms;
  cudaStream_t s;
  float* params;
  float* w;
  float* dd;
  char* ws;
  size_t ws_bytes;
  WsLayout L;
  Ptrs P;
  asgd_csr data;
  bool has_data;
  const void* eval_validated;
  float* dbg;
  int64_t u;
  int64_t launches;
  int64_t Pn;
  int64_t o_w1, o_b1, o_w2, o_b2;
  uint32_t prof_mask = 0;                        // kernel classes timed with events
  std::vector<cudaEvent_t> pev[ASGD_PROF_N];   // (start, end) pairs
  size_t pused[ASGD_PROF_N] = {};
  cudaStream_t s2 = nullptr;                     // side stream: K-0 overlaps the dense chain
  cudaStream_t s3 = nullptr;                     // side stream: G3 + b1 (bf16 path)
  cudaStream_t sc = nullptr;                     // private stream the step graphs are captured on
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr, ev_sm = nullptr, ev_dh = nullptr, ev_a = nullptr;
  bf16* w2b_buf[2] = {nullptr, nullptr};         // double-buffered bf16 W2 shadow (hi half on fp32)
  bf16* w2l_buf[2] = {nullptr, nullptr};         // fp32 path: its bf16x3 lo half (R14)
  // step trace (asgd_trace_enable / asgd_trace_read): timing events around each local step
  bool trace = false;
  cudaEvent_t trace_ref = nullptr;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> trace_ev;
  std::vector<int64_t> trace_meta;   // (stream start, rows) per traced step
  size_t trace_n = 0;
  int64_t cur_start = -1;            // stream position of the step being enqueued (run_steps)
  int w2b_cur = 0;
  std::list<StepGraph> graphs;                   // CUDA-graph cache of the step, LRU (stable addresses:
                                                 // the graphs point at their own StepArgs)
  uint64_t graph_clock = 0;
  bool capturing = false;
  std::vector<std::pair<cudaEvent_t, int>> cap_ph;   // (placeholder, cls * 2 + begin) during capture
  std::vector<std::pair<cudaGraphNode_t, int>> cap_args;   // K-0 (0) / K-1 (1) nodes, capture order
  cudaEvent_t prof_sink = nullptr;                // target of profiling nodes past kMaxProfPairs
  std::vector<std::pair<const int64_t*, cudaEvent_t>> staged;   // asgd_data_stage: per buffer, its copies
  cudaEvent_t ev_ring[8] = {};                    // asgd_run_tickets: completion of the last steps
  StepArgs sa{};                                  // current step's arguments (K-0 / K-1 parameter)
  // fused peer-memory merge (asgd_peer_open / asgd_merge_fused)
  int peer_rank = -1, peer_world = 0;
  float* peer_params[kMaxPeers] = {};
  unsigned long long* peer_sync[kMaxPeers] = {};
  std::vector<void*> peer_mapped;                 // IPC mappings to close
  unsigned long long merge_epoch = 0;
  Launch lc() { return Launch{s, &launches, sms, pdl_for(d.precision == ASGD_PREC_BF16)}; }
  Launch lc2() { return Launch{s2, &launches, sms, pdl_for(d.precision == ASGD_PREC_BF16)}; }
  Launch lc3() { return Launch{s3, &launches, sms, pdl_for(d.precision == ASGD_PREC_BF16)}; }
};

namespace {
constexpr size_t kMaxProfPairs = 8192;

// The GEMM operand copy of W2 (bf16 shadow; fp32 path: its hi and lo halves) from params.
cudaError_t refresh_shadow(asgd_ctx* c) {
  return launch_to_bf16(c->lc(), c->params + c->o_w2, c->w2b_buf[c->w2b_cur], c->d.L * c->d.H,
                        c->w2l_buf[c->w2b_cur]);
}

// Record an event on stream st at the start / end of a kernel-class section.
void prof_mark(asgd_ctx* c, int cls, bool begin, cudaStream_t st) {
  if (!(c->prof_mask & (1u << cls))) return;
  if (c->capturing) {   // an event-record node; its event is set per replay (bind_prof_events)
    cudaEvent_t ph;
    if (cudaEventCreate(&ph) != cudaSuccess) return;
    cudaEventRecordWithFlags(ph, st, cudaEventRecordExternal);
    c->cap_ph.push_back({ph, cls * 2 + (begin ? 1 : 0)});
    return;
  }
  auto& v = c->pev[cls];
  size_t& u = c->pused[cls];
  if (begin) {
    if (u >= kMaxProfPairs) return;
    if (v.size() < 2 * (u + 1)) {
      cudaEvent_t a, b;
      if (cudaEventCreate(&a) != cudaSuccess) return;
      if (cudaEventCreate(&b) != cudaSuccess) { cudaEventDestroy(a); return; }
      v.push_back(a);
      v.push_back(b);
    }
    cudaEventRecord(v[2 * u], st);
  } else {
    if (u >= kMaxProfPairs || v.size() < 2 * (u + 1)) return;
    cudaEventRecord(v[2 * u + 1], st);
    ++u;
  }
}

void destroy_graph(StepGraph& g) {
  if (g.exec) cudaGraphExecDestroy(g.exec);
  if (g.graph) cudaGraphDestroy(g.graph);
  for (cudaEvent_t e : g.placeholders) cudaEventDestroy(e);
  g = StepGraph{};
}

void clear_graphs(asgd_ctx* c) {
  for (auto& g : c->graphs) destroy_graph(g);
  c->graphs.clear();
}

bool graphs_enabled() {
  static const int on = [] {
    const char* e = getenv("ASGD_GRAPH");
    return (e && e[0] == '0') ? 0 : 1;
  }();
  return on != 0;
}

// Point the graph's profiling nodes at fresh pool events, in the order prof_mark
// would have used them for an eager step.
void bind_prof_events(asgd_ctx* c, StepGraph& g) {
  for (const auto& pn : g.prof) {
    auto& v = c->pev[pn.cls];
    size_t& u = c->pused[pn.cls];
    cudaEvent_t ev = c->prof_sink;
    if (u < kMaxProfPairs) {
      if (v.size() < 2 * (u + 1)) {
        cudaEvent_t a, b;
        if (cudaEventCreate(&a) == cudaSuccess) {
          if (cudaEventCreate(&b) == cudaSuccess) { v.push_back(a); v.push_back(b); }
          else cudaEventDestroy(a);
        }
      }
      if (v.size() >= 2 * (u + 1)) ev = v[2 * u + (pn.begin ? 0 : 1)];
      if (!pn.begin) ++u;
    }
    if (ev) cudaGraphExecEventRecordNodeSetEvent(g.exec, pn.node, ev);
  }
}
}  // namespace

#define PCU_ON(st, cls, call)                               \
  do {                                                      \
    prof_mark(c, cls, true, st);                            \
    cudaError_t _e = (call);                                \
    prof_mark(c, cls, false, st);                           \
    if (_e != cudaSuccess) return cuda_fail(_e, #call);     \
  } while (0)
#define PCU(cls, call) PCU_ON(c->s, cls, call)

extern "C" {

const char* asgd_last_error(void) { return g_err.c_str(); }

const char* asgd_version(void) { return "libasgd sm_100a (tcgen05/TMA: bf16, fp32 as bf16x3) r2 bf16-ready"; }

size_t asgd_workspace_bytes(const asgd_model_desc* d) {
  if (!d || d->F <= 0 || d->L <= 0 || d->b_max <= 0 || d->max_step_nnz <= 0) return 0;
  return ws_layout(*d).total;
}

int asgd_replica_init(asgd_ctx** out, const asgd_model_desc* desc, int device, void* stream,
                      float* params, float* w, float* d, void* ws, size_t ws_bytes) {
  if (!out || !desc || !params || !w || !d || !ws) return fail(ASGD_E_ARG, "null argument");
  if (!aligned16(params) || !aligned16(w) || !aligned16(d) || !aligned16(ws))
    return fail(ASGD_E_ARG, "device buffers must be 16-byte aligned");
  const asgd_model_desc& m = *desc;
  if (m.H != 64 && m.H != 128 && m.H != 256 && m.H != 512)
    return fail(ASGD_E_UNSUPPORTED, "H=%lld not in {64,128,256,512}", (long long)m.H);
  if (m.F <= 0 || m.L <= 0 || m.b_max <= 0 || m.b_max > 2048 || m.max_step_nnz <= 0 ||
      m.max_step_nnz >= (1ll << 31) || m.max_step_labels <= 0 || (int64_t)m.b_max * m.L >= (1ll << 40))
    return fail(ASGD_E_SHAPE, "bad model desc (F=%lld L=%lld b_max=%d nnz=%lld)", (long long)m.F,
                (long long)m.L, m.b_max, (long long)m.max_step_nnz);
  if (m.precision != ASGD_PREC_FP32 && m.precision != ASGD_PREC_BF16)
    return fail(ASGD_E_ARG, "precision %d", m.precision);
  if ((m.loss != ASGD_LOSS_SOFTMAX && m.loss != ASGD_LOSS_SIGMOID) || m.reserved != 0)
    return fail(ASGD_E_ARG, "loss %d / reserved %d", m.loss, m.reserved);
  const size_t need = ws_layout(m).total;
  if (ws_bytes < need) return fail(ASGD_E_SHAPE, "workspace %zu < %zu bytes", ws_bytes, need);
  CU(cudaSetDevice(device));
  cudaDeviceProp prop;
  CU(cudaGetDeviceProperties(&prop, device));
  if (prop.major != 10 || prop.minor != 0)
    return fail(ASGD_E_UNSUPPORTED, "device %d is sm_%d%d; libasgd is built for sm_100a only", device,
                prop.major, prop.minor);
  if (m.precision == ASGD_PREC_BF16 && m.H > 256)   // G1's resident H1 block holds K = H <= 256
    return fail(ASGD_E_UNSUPPORTED, "bf16 path: H=%lld > 256", (long long)m.H);
  if (!tc_available())   // both precisions run the output layer on tcgen05
    return fail(ASGD_E_UNSUPPORTED, "tcgen05 path unavailable (cuTensorMapEncodeTiled)");
  asgd_ctx* c = new (std::nothrow) asgd_ctx();
  if (!c) return fail(ASGD_E_ARG, "out of host memory");
  c->d = m;
  c->device = device;
  c->sms = prop.multiProcessorCount;
  c->s = static_cast<cudaStream_t>(stream);
  c->params = params;
  c->w = w;
  c->dd = d;
  c->ws = static_cast<char*>(ws);
  c->ws_bytes = ws_bytes;
  c->L = ws_layout(m);
  c->P = ws_ptrs(c->ws, c->L);
  c->has_data = false;
  c->eval_validated = nullptr;
  c->dbg = nullptr;
  c->u = 0;
  c->launches = 0;
  c->o_w1 = 0;
  c->o_b1 = m.F * m.H;
  c->o_w2 = c->o_b1 + m.H;
  c->o_b2 = c->o_w2 + m.L * m.H;
  c->Pn = c->o_b2 + m.L;
  c->w2b_buf[0] = c->P.w2b;
  c->w2b_buf[1] = reinterpret_cast<bf16*>(c->ws + c->L.w2b2);
  if (c->L.x3) {
    c->w2l_buf[0] = c->P.w2l;
    c->w2l_buf[1] = reinterpret_cast<bf16*>(c->ws + c->L.w2l2);
  }
  cudaError_t e = cudaStreamCreateWithFlags(&c->s2, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->s3, cudaStreamNonBlocking);
  for (cudaEvent_t* ev : {&c->ev_fork, &c->ev_join, &c->ev_sm, &c->ev_dh, &c->ev_a})
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(ev, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaMemsetAsync(c->ws, 0, c->L.total, c->s);
  if (e == cudaSuccess) e = refresh_shadow(c);
  if (e == cudaSuccess) e = cudaStreamSynchronize(c->s);
  if (e != cudaSuccess) { asgd_replica_destroy(c); return cuda_fail(e, "replica_init"); }
  *out = c;
  return ASGD_OK;
}

int asgd_replica_destroy(asgd_ctx* c) {
  if (c) {
    clear_graphs(c);
    for (void* pm : c->peer_mapped) cudaIpcCloseMemHandle(pm);
    if (c->prof_sink) cudaEventDestroy(c->prof_sink);
    if (c->trace_ref) cudaEventDestroy(c->trace_ref);
    for (auto& pr : c->trace_ev) { cudaEventDestroy(pr.first); cudaEventDestroy(pr.second); }
    for (cudaEvent_t ev : c->ev_ring)
      if (ev) cudaEventDestroy(ev);
    for (auto& v : c->pev)
      for (cudaEvent_t e : v) cudaEventDestroy(e);
    for (cudaEvent_t ev : {c->ev_fork, c->ev_join, c->ev_sm, c->ev_dh, c->ev_a})
      if (ev) cudaEventDestroy(ev);
    for (auto& se : c->staged) cudaEventDestroy(se.second);
    if (c->s2) cudaStreamDestroy(c->s2);
    if (c->s3) cudaStreamDestroy(c->s3);
    if (c->sc) cudaStreamDestroy(c->sc);
  }
  delete c;
  return ASGD_OK;
}

int asgd_set_stream(asgd_ctx* c, void* stream) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  c->s = static_cast<cudaStream_t>(stream);
  return ASGD_OK;
}

int asgd_params_changed(asgd_ctx* c) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  CU(refresh_shadow(c));
  return ASGD_OK;
}

static int validate(asgd_ctx* c, const asgd_csr* x) {
  int32_t* err = c->P.meta + 16;
  CU(cudaMemsetAsync(err, 0, 4, c->s));
  CU(launch_validate_csr(c->lc(), x, c->d.F, c->d.L, err));
  int32_t h = 0;
  CU(cudaMemcpyAsync(&h, err, 4, cudaMemcpyDeviceToHost, c->s));
  CU(cudaStreamSynchronize(c->s));
  if (h) return fail(ASGD_E_SHAPE, "CSR invariant violated (bits 0x%x)", h);
  return ASGD_OK;
}

int asgd_data_register(asgd_ctx* c, const asgd_csr* x) {
  if (!c || !x || !x->row_ptr || !x->col || !x->val || !x->lab_ptr || !x->lab)
    return fail(ASGD_E_ARG, "null argument");
  if (x->n_rows <= 0 || x->nnz < 0 || x->n_lab <= 0) return fail(ASGD_E_SHAPE, "empty split");
  int rc = validate(c, x);
  if (rc) return rc;
  if (!c->has_data || memcmp(&c->data, x, sizeof(*x)) != 0) clear_graphs(c);   // graphs hold the pointers
  c->data = *x;
  c->has_data = true;
  return ASGD_OK;
}

int asgd_data_upload(asgd_ctx* c, const asgd_csr* h, const asgd_csr* dv) {
  const int rc = asgd_data_stage(c, h, dv, nullptr);
  if (rc != ASGD_OK) return rc;
  asgd_csr d = *dv;
  d.nnz = h->nnz;
  d.n_lab = h->n_lab;
  return asgd_data_use(c, &d);
}

int asgd_data_stage(asgd_ctx* c, const asgd_csr* h, const asgd_csr* dv, void* stream) {
  if (!c || !h || !dv) return fail(ASGD_E_ARG, "null argument");
  if (h->n_rows != dv->n_rows || h->nnz > dv->nnz || h->n_lab > dv->n_lab)
    return fail(ASGD_E_SHAPE, "destination too small");
  cudaStream_t st = stream ? static_cast<cudaStream_t>(stream) : c->s;
  CU(cudaMemcpyAsync((void*)dv->row_ptr, h->row_ptr, (h->n_rows + 1) * 8, cudaMemcpyHostToDevice, st));
  CU(cudaMemcpyAsync((void*)dv->col, h->col, h->nnz * 4, cudaMemcpyHostToDevice, st));
  CU(cudaMemcpyAsync((void*)dv->val, h->val, h->nnz * 4, cudaMemcpyHostToDevice, st));
  CU(cudaMemcpyAsync((void*)dv->lab_ptr, h->lab_ptr, (h->n_rows + 1) * 8, cudaMemcpyHostToDevice, st));
  CU(cudaMemcpyAsync((void*)dv->lab, h->lab, h->n_lab * 4, cudaMemcpyHostToDevice, st));
  if (st != c->s) {   // asgd_data_use of this buffer makes the ctx stream wait for these copies
    cudaEvent_t ev = nullptr;
    for (auto& se : c->staged)
      if (se.first == dv->row_ptr) ev = se.second;
    if (!ev) {
      CU(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
      c->staged.push_back({dv->row_ptr, ev});
    }
    CU(cudaEventRecord(ev, st));
  }
  return ASGD_OK;
}

int asgd_data_use(asgd_ctx* c, const asgd_csr* dv) {
  if (!c || !dv || !dv->row_ptr || !dv->col || !dv->val || !dv->lab_ptr || !dv->lab)
    return fail(ASGD_E_ARG, "null argument");
  if (dv->n_rows <= 0 || dv->nnz < 0 || dv->n_lab <= 0) return fail(ASGD_E_SHAPE, "empty split");
  for (auto& se : c->staged)
    if (se.first == dv->row_ptr) CU(cudaStreamWaitEvent(c->s, se.second, 0));
  // the step graphs are keyed by the dataset (pointers and row count): alternating staging
  // buffers keep both sets of graphs
  c->data = *dv;
  c->has_data = true;
  return ASGD_OK;
}

}  // extern "C"

namespace {
// During capture: the kernel node just captured on `st` (the stream's single capture
// dependency) is a K-0 (kind 0) or K-1 (kind 1) node whose StepArgs parameter is rebound per replay.
int record_cap_node(asgd_ctx* c, cudaStream_t st, int kind) {
  cudaStreamCaptureStatus cs;
  const cudaGraphNode_t* deps = nullptr;
  size_t nd = 0;
  CU(cudaStreamGetCaptureInfo(st, &cs, nullptr, nullptr, &deps, &nd));
  if (cs != cudaStreamCaptureStatusActive || nd != 1) return fail(ASGD_E_STATE, "capture: %zu nodes after K-%d", nd, kind);
  c->cap_args.push_back({deps[0], kind});
  return ASGD_OK;
}

// Everything of a local step after K-0 (a): reads the step's rows / lr / loss
// pointer from the workspace (P.rowsc, meta), so it can be captured once per
// (n, shadow buffer, profile mask) and replayed.
// (b-f): touched-feature set on side stream s2, joined before K-5.
int enqueue_step(asgd_ctx* c, int n) {
  Launch lc = c->lc();
  const Ptrs& P = c->P;
  const asgd_csr& x = c->data;
  const asgd_model_desc& m = c->d;
  const bool bf = m.precision == ASGD_PREC_BF16;
  const int H = (int)m.H;
  const int64_t Lb = m.L;
  const int64_t Lp = padded_ld(Lb);
  float* W1 = c->params + c->o_w1;
  float* b1 = c->params + c->o_b1;
  float* W2 = c->params + c->o_w2;
  float* b2 = c->params + c->o_b2;
  float* g = c->dbg;
  // K-0 after K-1 (ASGD_K0_LATE=1, or with K-0's phase A folded into K-1)
  static const bool k0_late = [] { const char* e = getenv("ASGD_K0_LATE"); return (e && e[0] == '1') || k0_fold(); }();
  auto fork_k0 = [&]() -> int {
    CU(cudaEventRecord(c->ev_fork, c->s));
    CU(cudaStreamWaitEvent(c->s2, c->ev_fork, 0));
    PCU_ON(c->s2, ASGD_K_TOUCHED, launch_touched(c->lc2(), c->sa, x, m.F, P, c->L, m.b_max));
    if (c->capturing) { const int rc = record_cap_node(c, c->s2, 0); if (rc != ASGD_OK) return rc; }
    CU(cudaEventRecord(c->ev_join, c->s2));
    return ASGD_OK;
  };
  if (!k0_late) { const int rc = fork_k0(); if (rc != ASGD_OK) return rc; }
  // K-1
  PCU(ASGD_K_SPMM, launch_spmm_fwd(lc, c->sa, x, W1, b1, H, P, c->L, true, k0_fold(), (int)m.b_max));   // H1 fp32 + bf16 (+ lo)
  if (c->capturing) { const int rc = record_cap_node(c, c->s, 1); if (rc != ASGD_OK) return rc; }
  // With the fold, K-0 forks after the loss stage (G1 + softmax, or K-3's softmax-only
  // kernel), beside G2 / the dH reduce instead of beside G1, on the bf16 path when the
  // feature space has at most 8 scan tiles (F <= 8192: K-0's scan is short and it ends
  // inside the G2 / dH window).  Measured: EURLex bf16 4.54 -> 4.64 M samples/s; EURLex fp32
  // 3.99 -> 3.68 M, AmazonCat 181.9 -> 204.9 and Wiki10 179.2 -> 193.6 us per step (K-0 then
  // ends after the dH reduce and holds up K-5).  ASGD_K0_AFTER=0 / 1 forces it.
  static const int k0_after_env = [] { const char* e = getenv("ASGD_K0_AFTER"); return e ? (e[0] == '1' ? 1 : 0) : -1; }();
  const bool k0_after = k0_fold() && (k0_after_env >= 0 ? k0_after_env == 1
                                                         : (bf && m.F <= 8 * (int64_t)kScanTile));
  if (k0_late && !k0_after) { const int rc = fork_k0(); if (rc != ASGD_OK) return rc; }
  {
    // A DAG over three streams (both precisions; the fp32 path's GEMMs take bf16x3
    // hi + lo operands, R14, and always store Z):
    //   s : G1 -> softmax -> G2 -> dH reduce -> [K-0 joined] K-5
    //   s3: [after softmax] G3 (W2, b2 and the next step's bf16 W2 shadow) -> [after dH] b1
    // G1/G2 read the bf16 shadow w2b[cur]; G3 writes w2b[cur ^ 1], so G2 and G3 never race.
    const bool x3 = c->L.x3;
    Ptrs Pr = P, Pw = P;
    Pr.w2b = c->w2b_buf[c->w2b_cur];
    Pw.w2b = c->w2b_buf[c->w2b_cur ^ 1];
    Pr.w2l = c->w2l_buf[c->w2b_cur];
    Pw.w2l = c->w2l_buf[c->w2b_cur ^ 1];
    // G3 (s3) runs beside G2 (s): both need ~200 KB of smem per CTA, so G3's
    // persistent grid leaves G2's CTAs their own SMs when G2 is small
    Launch lc3 = c->lc3();
    const int g2c = gemm_tc_g2_ctas(n, H, c->L, c->sms);
    if (2 * g2c <= c->sms) lc3.sms = c->sms - g2c;
    float2* zstat = reinterpret_cast<float2*>(c->ws + c->L.zstat);
    int ntiles = 0;
    // K-3 (dH1 half): the fused softmax-CE regime on the bf16 path with H = 256
    const bool k3 = bf && m.loss == ASGD_LOSS_SOFTMAX && (int64_t)m.b_max * Lb * 4 > fused_ce_bytes() && H == 256 &&
                    bwd_fuse();
    const bool k3dw = k3 && bwd_dw() && n <= 1024;
    // K-3 one-pass: no G1 / softmax launch before it (the statistics come from its S tiles)
    const bool k3one = bf && m.loss == ASGD_LOSS_SOFTMAX && H == 256 && !k3 && bwd_fuse() && one_pass_on() &&
                       bwd_dh_one_pass_fits(n, Lb, c->L, c->sms);
    const bool k3dz = !k3one && bf && m.loss == ASGD_LOSS_SOFTMAX && H == 256 && !k3 && k3dz_on() &&
                      (int64_t)m.b_max * Lb * 4 <= fused_ce_bytes();
    if (k3one) {
      // nothing before K-3: G3 follows it (needs its dZ)
    } else if (k3dz) {
      // G1 + softmax-CE as one kernel: S tiles -> statistics -> grid barrier -> lse, row loss -> dZ
      const DhFuse fz{nullptr, nullptr, nullptr, bf};
      PCU(ASGD_K_G1, launch_bwd_dh(lc, n, Lb, H, Pr, c->L, b2, P.rowsc, x.lab_ptr, x.lab, fz, true, true, zstat, true));
    } else if (x3) {
      // fp32 path: G1 stores Z (+ per-tile softmax partials), then the loss kernel writes dZ
      // as bf16x3 hi + lo (sigmoid: centred, R11 / R14)
      PCU(ASGD_K_G1, launch_gemm_tc(lc, 1, n, Lb, H, Pr, c->L, W2, b2, nullptr, nullptr, zstat, &ntiles));
      if (m.loss == ASGD_LOSS_SIGMOID)
        PCU(ASGD_K_SOFTMAX, ([&]() -> cudaError_t {
              cudaError_t e = launch_sigmoid_ce(lc, n, Lb, Lp, P.rowsc, x.lab_ptr, x.lab, P, true);
              return e != cudaSuccess ? e
                                      : launch_sig_center(lc, nullptr, W2, Lb, H, P.h1, n, P.cenpart,
                                                          reinterpret_cast<unsigned int*>(P.meta + M_CEN), P.cen);
            })());
      else
        PCU(ASGD_K_SOFTMAX, launch_softmax_ce(lc, n, Lb, Lp, P.rowsc, x.lab_ptr, x.lab, P, true, zstat, ntiles,
                                              c->L.stats_ld));
    } else if (m.loss == ASGD_LOSS_SIGMOID) {
      // sigmoid-BCE needs no row normaliser: G1's epilogue writes dZ (bf16) and per-tile
      // row-loss partials directly, Z never stored, at every L (R11)
      PCU(ASGD_K_G1, launch_gemm_tc(lc, 6, n, Lb, H, Pr, c->L, W2, b2, nullptr, nullptr, zstat, &ntiles, P.rowsc,
                                    x.lab_ptr, x.lab));
      PCU(ASGD_K_SOFTMAX, ([&]() -> cudaError_t {
            cudaError_t e = launch_tile_loss(lc, n, ntiles, c->L.stats_ld, zstat, P);
            return e != cudaSuccess ? e
                                    : launch_sig_center(lc, Pr.w2b, nullptr, Lb, H, P.h1, n, P.cenpart,
                                                        reinterpret_cast<unsigned int*>(P.meta + M_CEN), P.cen);
          })());
    } else if ((int64_t)m.b_max * Lb * 4 <= fused_ce_bytes()) {
      // logits fit in L2: G1 stores Z (+ per-tile softmax partials), one pass of softmax-CE
      PCU(ASGD_K_G1, launch_gemm_tc(lc, 1, n, Lb, H, Pr, c->L, W2, b2, nullptr, nullptr, zstat, &ntiles));
      PCU(ASGD_K_SOFTMAX, launch_softmax_ce(lc, n, Lb, Lp, P.rowsc, x.lab_ptr, x.lab, P, true, zstat, ntiles,
                                            c->L.stats_ld));
    } else {
      // fused softmax-CE: G1 keeps only per-tile (max, sum exp); k_lse -> lse, row loss;
      // G1b recomputes Z tile by tile and writes dZ = (softmax - T)/B (bf16) -- Z never hits HBM
      PCU(ASGD_K_G1, launch_gemm_tc(lc, 5, n, Lb, H, Pr, c->L, W2, b2, nullptr, nullptr, zstat, &ntiles));
      if (k3)   // lse only; dZ is formed inside k_bwd_dh (K-3)
        PCU(ASGD_K_SOFTMAX, launch_lse(lc, n, H, ntiles, c->L.stats_ld, zstat, P.rowsc, x.lab_ptr, x.lab, P.h1b,
                                       Pr.w2b, b2, P));
      else
        PCU(ASGD_K_SOFTMAX, ([&]() -> cudaError_t {
              cudaError_t e = launch_lse(lc, n, H, ntiles, c->L.stats_ld, zstat, P.rowsc, x.lab_ptr, x.lab, P.h1b,
                                         Pr.w2b, b2, P);
              return e != cudaSuccess ? e
                                      : launch_gemm_tc(lc, 4, n, Lb, H, Pr, c->L, W2, b2, nullptr, nullptr,
                                                       nullptr, nullptr, P.rowsc, x.lab_ptr, x.lab);
            })());
    }
    if (k0_after) { const int rc = fork_k0(); if (rc != ASGD_OK) return rc; }
    const bool centred = m.loss == ASGD_LOSS_SIGMOID;   // G1 stored dZ - 1/(2B) (R11)
    auto g3 = [&](const Launch& l) {
      if (k3dw)   // K-3's dW2 half: Z^T recomputed, dZ^T on chip, W2 / b2 SGD
        return launch_bwd_dw(l, n, Lb, H, Pr, Pw, W2, b2, P.rowsc, x.lab_ptr, x.lab, g ? g + c->o_w2 : nullptr,
                             g ? g + c->o_b2 : nullptr);
      return launch_gemm_tc(l, 3, n, Lb, H, Pw, c->L, W2, b2, g ? g + c->o_w2 : nullptr, g ? g + c->o_b2 : nullptr,
                            nullptr, nullptr, nullptr, nullptr, nullptr, centred ? P.cen + H : nullptr);
    };
    // G3 beside G2 only when G2 leaves at least half the SMs idle; when both fill the GPU
    // (Amazon-670K: 148 persistent CTAs each, one per SM) concurrent launches interleave
    // their CTAs and the later kernel's static tile split waits on the earlier one's SMs
    // (measured 1024 us for the pair against 326 + 572 us back to back), so G3 runs last
    const bool g3_side = 2 * g2c <= c->sms && !k3one;
    if (g3_side) {
      CU(cudaEventRecord(c->ev_sm, c->s));
      CU(cudaStreamWaitEvent(c->s3, c->ev_sm, 0));
      PCU_ON(c->s3, ASGD_K_G3, g3(lc3));
    }
    if (k3one) {
      // K-3 one-pass: S tiles -> softmax partials -> grid barrier -> lse, row loss -> dZ (on
      // chip into dH1, TMA-stored for G3) -> dH1 reduce + b1 in the tail; G3 beside K-5
      const DhFuse fz{b1, g ? g + c->o_b1 : nullptr, nullptr, bf};
      PCU(ASGD_K_G2, launch_bwd_dh(lc, n, Lb, H, Pr, c->L, b2, P.rowsc, x.lab_ptr, x.lab, fz, true, true, zstat));
      CU(cudaEventRecord(c->ev_sm, c->s));
      CU(cudaStreamWaitEvent(c->s3, c->ev_sm, 0));
      PCU_ON(c->s3, ASGD_K_G3, g3(c->lc3()));
    } else if (k3) {
      // K-3: Z recomputed, dZ on chip into dH1 (+ TMA-stored for G3), dH1 reduce + b1 in the tail
      const DhFuse fz{b1, g ? g + c->o_b1 : nullptr, nullptr, bf};
      PCU(ASGD_K_G2, launch_bwd_dh(lc, n, Lb, H, Pr, c->L, b2, P.rowsc, x.lab_ptr, x.lab, fz, !k3dw));
    } else if (g2_fuse()) {
      // G2 + the dH1 reduce + ReLU' + b1 update + mean loss in one launch (grid barrier)
      const DhFuse fz{b1, g ? g + c->o_b1 : nullptr, centred ? P.cen : nullptr, bf};
      PCU(ASGD_K_G2, launch_gemm_tc(lc, 2, n, Lb, H, Pr, c->L, W2, b2, nullptr, nullptr, nullptr, nullptr,
                                    nullptr, nullptr, nullptr, nullptr, &fz));
    } else {
      PCU(ASGD_K_G2, launch_gemm_tc(lc, 2, n, Lb, H, Pr, c->L, W2, b2, nullptr, nullptr));
      PCU(ASGD_K_DH, launch_dh_reduce(lc, n, H, (int)c->L.splitk, P, c->L, bf, centred ? P.cen : nullptr));
      CU(cudaEventRecord(c->ev_dh, c->s));
      CU(cudaStreamWaitEvent(c->s3, c->ev_dh, 0));
      PCU_ON(c->s3, ASGD_K_DH, launch_b1_update(lc3, n, H, b1, P, c->L, g ? g + c->o_b1 : nullptr));
    }
    // join s3 back into s only when work went there (an event recorded on a stream outside
    // the capture cannot be waited on inside it)
    const bool s3_used = g3_side || k3one || !(k3 || g2_fuse());
    if (s3_used) CU(cudaEventRecord(c->ev_a, c->s3));
    // K-5 (needs K-0's segments)
    CU(cudaStreamWaitEvent(c->s, c->ev_join, 0));
    PCU(ASGD_K_SCATTER, launch_scatter_sgd(lc, W1, H, P, c->L, g ? g + c->o_w1 : nullptr, bf ? P.da1b : nullptr, m.b_max));
    if (!g3_side && !k3one) PCU(ASGD_K_G3, g3(lc));
    if (s3_used) CU(cudaStreamWaitEvent(c->s, c->ev_a, 0));
  }
  return ASGD_OK;
}


constexpr size_t kMaxGraphs = 16;

// the dataset fields a captured step bakes into its kernel parameters
bool same_data(const asgd_csr& a, const asgd_csr& b) {
  return a.row_ptr == b.row_ptr && a.col == b.col && a.val == b.val && a.lab_ptr == b.lab_ptr && a.lab == b.lab &&
         a.n_rows == b.n_rows;
}

// Replay (capturing on the 2nd use of a key) `steps` local steps as one CUDA graph
// (steps > 1: a step group, run_steps at N = 1); sas[i] = step i's StepArgs.  c->w2b_cur
// is left as it was (the caller flips it per step).
int step_graph(asgd_ctx* c, int n, int steps, const StepArgs* sas) {
  StepGraph* hit = nullptr;
  for (auto& gr : c->graphs)
    if (gr.n == n && gr.steps == steps && gr.cur == c->w2b_cur && gr.mask == c->prof_mask && same_data(gr.data, c->data)) {
      hit = &gr;
      break;
    }
  if (!hit) {
    if (c->graphs.size() >= kMaxGraphs) {
      auto lru = std::min_element(c->graphs.begin(), c->graphs.end(),
                                  [](const StepGraph& a, const StepGraph& b) { return a.last_use < b.last_use; });
      destroy_graph(*lru);
      c->graphs.erase(lru);
    }
    c->graphs.emplace_back();
    hit = &c->graphs.back();
    hit->n = n; hit->steps = steps; hit->cur = c->w2b_cur; hit->mask = c->prof_mask; hit->data = c->data;
  }
  StepGraph& G = *hit;
  G.last_use = ++c->graph_clock;
  const int cur0 = c->w2b_cur;
  auto enqueue_all = [&]() -> int {
    for (int i = 0; i < steps; ++i) {
      c->sa = sas[i];
      const int rc = enqueue_step(c, n);
      c->w2b_cur ^= 1;
      if (rc != ASGD_OK) { c->w2b_cur = cur0; return rc; }
    }
    c->w2b_cur = cur0;
    return ASGD_OK;
  };
  if (!G.exec && G.seen++ == 0) return enqueue_all();   // first use: eager (warms attributes)
  if (!G.exec) {
    // capture on the private stream sc (the ctx stream may be the legacy default
    // stream, which cannot capture); the graph itself is launched on c->s
    if (!c->sc) CU(cudaStreamCreateWithFlags(&c->sc, cudaStreamNonBlocking));
    const int64_t l0 = c->launches;
    c->cap_ph.clear();
    c->cap_args.clear();
    cudaStream_t user = c->s;
    c->s = c->sc;
    cudaError_t eb = cudaStreamBeginCapture(c->s, cudaStreamCaptureModeThreadLocal);
    if (eb != cudaSuccess) { c->s = user; return cuda_fail(eb, "cudaStreamBeginCapture"); }
    c->capturing = true;
    const int rc = enqueue_all();
    c->capturing = false;
    cudaGraph_t graph = nullptr;
    const cudaError_t ec = cudaStreamEndCapture(c->s, &graph);
    c->s = user;
    for (auto& ph : c->cap_ph) G.placeholders.push_back(ph.first);
    G.kernels = c->launches - l0;
    c->launches = l0;
    if (rc != ASGD_OK || ec != cudaSuccess) {
      if (graph) cudaGraphDestroy(graph);
      c->cap_args.clear();
      return rc != ASGD_OK ? rc : cuda_fail(ec, "cudaStreamEndCapture");
    }
    G.graph = graph;
    CU(cudaGraphInstantiate(&G.exec, graph, 0));
    {  // each step's K-0 / K-1 nodes (recorded at capture): their StepArgs parameter is
       // rebound per replay to G.sas[step]
      G.sas.assign(steps, StepArgs{});
      int seen[2] = {0, 0};
      for (auto& ca : c->cap_args) {
        // the recorded node may be a profiling event-record node behind the kernel: walk back
        cudaGraphNodeType t;
        for (int hop = 0;; ++hop) {
          CU(cudaGraphNodeGetType(ca.first, &t));
          if (t == cudaGraphNodeTypeKernel) break;
          size_t nd = 0;
          CU(cudaGraphNodeGetDependencies(ca.first, nullptr, &nd));
          if (nd != 1 || hop > 4) return fail(ASGD_E_STATE, "step graph: K-%d node not found", ca.second);
          CU(cudaGraphNodeGetDependencies(ca.first, &ca.first, &nd));
        }
        cudaKernelNodeParams kp;
        CU(cudaGraphKernelNodeGetParams(ca.first, &kp));
        const int na = ca.second == 1 ? spmm_fwd_nargs() : touched_nargs();
        const int step = seen[ca.second]++;
        if (step >= steps) return fail(ASGD_E_STATE, "step graph: extra K-%d node", ca.second);
        StepGraph::ArgNode an{ca.first, kp, std::vector<void*>(kp.kernelParams, kp.kernelParams + na)};
        an.args[0] = &G.sas[step];
        G.arg_nodes.push_back(std::move(an));
      }
      c->cap_args.clear();
      if (seen[0] != steps || seen[1] != steps)
        return fail(ASGD_E_STATE, "step graph: %d K-0 / %d K-1 nodes for %d steps", seen[0], seen[1], steps);
    }
    if (!c->cap_ph.empty()) {
      size_t nn = 0;
      CU(cudaGraphGetNodes(graph, nullptr, &nn));
      std::vector<cudaGraphNode_t> nodes(nn);
      CU(cudaGraphGetNodes(graph, nodes.data(), &nn));
      std::vector<cudaGraphNode_t> by_ph(c->cap_ph.size(), nullptr);
      for (cudaGraphNode_t nd : nodes) {
        cudaGraphNodeType t;
        if (cudaGraphNodeGetType(nd, &t) != cudaSuccess || t != cudaGraphNodeTypeEventRecord) continue;
        cudaEvent_t ev;
        if (cudaGraphEventRecordNodeGetEvent(nd, &ev) != cudaSuccess) continue;
        for (size_t i = 0; i < c->cap_ph.size(); ++i)
          if (c->cap_ph[i].first == ev) by_ph[i] = nd;
      }
      for (size_t i = 0; i < c->cap_ph.size(); ++i)
        if (by_ph[i]) G.prof.push_back({by_ph[i], c->cap_ph[i].second / 2, (c->cap_ph[i].second & 1) != 0});
      if (!c->prof_sink) CU(cudaEventCreate(&c->prof_sink));
    }
    c->cap_ph.clear();
  }
  if (!G.prof.empty()) bind_prof_events(c, G);
  for (int i = 0; i < steps; ++i) G.sas[i] = sas[i];
  for (auto& an : G.arg_nodes) {
    cudaKernelNodeParams kp = an.p;
    kp.kernelParams = an.args.data();
    kp.extra = nullptr;
    CU(cudaGraphExecKernelNodeSetParams(G.exec, an.node, &kp));
  }
  CU(cudaGraphLaunch(G.exec, c->s));
  c->launches += G.kernels;
  return ASGD_OK;
}
}  // namespace

extern "C" {

int asgd_local_step(asgd_ctx* c, const int32_t* rows, int32_t n, float lr, float* loss_dev) {
  if (!c || !rows) return fail(ASGD_E_ARG, "null argument");
  if (!c->has_data) return fail(ASGD_E_STATE, "no data registered");
  const asgd_model_desc& m = c->d;
  if (n < 1 || n > m.b_max) return fail(ASGD_E_SHAPE, "n_rows=%d not in [1, %d]", n, m.b_max);
  Launch lc = c->lc();
  const Ptrs& P = c->P;
  const asgd_csr& x = c->data;
  float* g = c->dbg;
  if (g) CU(cudaMemsetAsync(g, 0, c->Pn * sizeof(float), c->s));
  // the step's only per-call arguments; K-0 and K-1 build the batch view from them
  c->sa = StepArgs{rows, loss_dev, lr, n};
  const bool tr = c->trace && c->trace_n < kMaxTrace;
  if (tr) {
    if (c->trace_ev.size() <= c->trace_n) {
      cudaEvent_t a, b;
      CU(cudaEventCreate(&a));
      CU(cudaEventCreate(&b));
      c->trace_ev.push_back({a, b});
    }
    CU(cudaEventRecord(c->trace_ev[c->trace_n].first, c->s));
  }
  const int rc = (graphs_enabled() && !g) ? step_graph(c, n, 1, &c->sa) : enqueue_step(c, n);
  if (rc != ASGD_OK) return rc;
  if (tr) {
    CU(cudaEventRecord(c->trace_ev[c->trace_n].second, c->s));
    c->trace_meta.push_back(c->cur_start);
    c->trace_meta.push_back(n);
    ++c->trace_n;
  }
  c->w2b_cur ^= 1;   // G3 wrote the other shadow buffer
  ++c->u;
  return ASGD_OK;
}

int asgd_trace_enable(asgd_ctx* c, int32_t on) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  if (on) {
    if (!c->trace_ref) CU(cudaEventCreate(&c->trace_ref));
    CU(cudaEventRecord(c->trace_ref, c->s));
    c->trace_n = 0;
    c->trace_meta.clear();
  }
  c->trace = on != 0;
  return ASGD_OK;
}

int asgd_trace_read(asgd_ctx* c, int64_t* out, int64_t cap, int64_t* n_out) {
  if (!c || !out || !n_out) return fail(ASGD_E_ARG, "null argument");
  if (!c->trace_ref) return fail(ASGD_E_STATE, "asgd_trace_enable first");
  if ((int64_t)c->trace_n > cap) return fail(ASGD_E_SHAPE, "cap %lld < %zu traced steps", (long long)cap, c->trace_n);
  if (c->trace_n) CU(cudaEventSynchronize(c->trace_ev[c->trace_n - 1].second));
  for (size_t i = 0; i < c->trace_n; ++i) {
    float t0 = 0.f, t1 = 0.f;
    CU(cudaEventElapsedTime(&t0, c->trace_ref, c->trace_ev[i].first));
    CU(cudaEventElapsedTime(&t1, c->trace_ref, c->trace_ev[i].second));
    out[4 * i] = c->trace_meta[2 * i];
    out[4 * i + 1] = c->trace_meta[2 * i + 1];
    out[4 * i + 2] = (int64_t)((double)t0 * 1e6);
    out[4 * i + 3] = (int64_t)((double)t1 * 1e6);
  }
  *n_out = (int64_t)c->trace_n;
  c->trace_n = 0;
  c->trace_meta.clear();
  return ASGD_OK;
}

int asgd_timeline_set(void* buf) {
  unsigned long long* p = static_cast<unsigned long long*>(buf);
  for (auto fn : {tl_set_sparse, tl_set_dense, tl_set_tc, tl_set_merge}) {
    const cudaError_t e = fn(p);
    if (e == cudaErrorNotSupported) return fail(ASGD_E_UNSUPPORTED, "libasgd built without -DASGD_TIMELINE");
    if (e != cudaSuccess) return cuda_fail(e, "asgd_timeline_set");
  }
  return ASGD_OK;
}

int asgd_updates(const asgd_ctx* c, int64_t* u) {
  if (!c || !u) return fail(ASGD_E_ARG, "null argument");
  *u = c->u;
  return ASGD_OK;
}

int asgd_set_debug_grads(asgd_ctx* c, float* g) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  if (g && !aligned16(g)) return fail(ASGD_E_ARG, "grad buffer must be 16-byte aligned");
  c->dbg = g;
  return ASGD_OK;
}

int asgd_last_touched(asgd_ctx* c, int32_t* out, int64_t cap, int64_t* n_out) {
  if (!c || !out || !n_out) return fail(ASGD_E_ARG, "null argument");
  int32_t U = 0;
  CU(cudaMemcpyAsync(&U, c->P.meta + M_U, 4, cudaMemcpyDeviceToHost, c->s));
  CU(cudaStreamSynchronize(c->s));
  *n_out = U;
  if (U > cap) return fail(ASGD_E_SHAPE, "cap %lld < %d touched", (long long)cap, U);
  CU(cudaMemcpyAsync(out, c->P.uniq, (size_t)U * 4, cudaMemcpyDeviceToDevice, c->s));
  CU(cudaStreamSynchronize(c->s));
  return ASGD_OK;
}

int asgd_replica_sqnorm(asgd_ctx* c, double* out_dev) {
  if (!c || !out_dev) return fail(ASGD_E_ARG, "null argument");
  PCU(ASGD_K_MERGE, launch_sqnorm(c->lc(), c->params, c->Pn, c->P.red, (int)c->L.n_red, out_dev));
  return ASGD_OK;
}

int asgd_merge_prescale(asgd_ctx* c, double alpha) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  PCU(ASGD_K_MERGE, launch_scale(c->lc(), c->params, c->Pn, alpha));
  return ASGD_OK;
}

int asgd_merge_finish(asgd_ctx* c, float gamma) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  PCU(ASGD_K_MERGE, launch_finish(c->lc(), c->params, c->w, c->dd, c->Pn, gamma));
  CU(refresh_shadow(c));
  c->u = 0;
  return ASGD_OK;
}

namespace {
struct PeerHandle {                 // ASGD_PEER_HANDLE_BYTES, opaque to the caller
  cudaIpcMemHandle_t params;        // allocation holding the replica
  int64_t params_off;               // replica offset inside it
  cudaIpcMemHandle_t ws;            // allocation holding the workspace (arrival counter)
  int64_t ws_off;
  int32_t device, pad;
};
static_assert(sizeof(PeerHandle) <= ASGD_PEER_HANDLE_BYTES, "peer handle size");

using PFN_getRange = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);

int alloc_base(const void* p, char** base) {
  static PFN_getRange fn = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return (PFN_getRange) nullptr;
    return reinterpret_cast<PFN_getRange>(f);
  }();
  if (!fn) return fail(ASGD_E_CUDA, "cuMemGetAddressRange unavailable");
  CUdeviceptr b = 0;
  size_t sz = 0;
  if (fn(&b, &sz, (CUdeviceptr)p) != CUDA_SUCCESS) return fail(ASGD_E_ARG, "not a device allocation");
  *base = reinterpret_cast<char*>(b);
  return ASGD_OK;
}
}  // namespace

int asgd_peer_export(asgd_ctx* c, void* out) {
  if (!c || !out) return fail(ASGD_E_ARG, "null argument");
  PeerHandle h{};
  char* bp = nullptr;
  char* bw = nullptr;
  int rc = alloc_base(c->params, &bp);
  if (rc) return rc;
  rc = alloc_base(c->ws, &bw);
  if (rc) return rc;
  CU(cudaIpcGetMemHandle(&h.params, bp));
  CU(cudaIpcGetMemHandle(&h.ws, bw));
  h.params_off = reinterpret_cast<char*>(c->params) - bp;
  h.ws_off = c->ws - bw;
  h.device = c->device;
  memset(out, 0, ASGD_PEER_HANDLE_BYTES);
  memcpy(out, &h, sizeof(h));
  return ASGD_OK;
}

int asgd_peer_open(asgd_ctx* c, int32_t rank, int32_t world, const void* handles) {
  if (!c || !handles) return fail(ASGD_E_ARG, "null argument");
  if (world < 1 || world > kMaxPeers || rank < 0 || rank >= world)
    return fail(ASGD_E_ARG, "rank %d / world %d (world <= %d)", rank, world, kMaxPeers);
  CU(cudaSetDevice(c->device));
  for (void* pm : c->peer_mapped) cudaIpcCloseMemHandle(pm);
  c->peer_mapped.clear();
  std::vector<std::pair<cudaIpcMemHandle_t, char*>> opened;   // one mapping per distinct allocation
  auto open = [&](const cudaIpcMemHandle_t& hd, char** base) -> int {
    for (auto& o : opened)
      if (memcmp(&o.first, &hd, sizeof(hd)) == 0) { *base = o.second; return ASGD_OK; }
    void* p = nullptr;
    CU(cudaIpcOpenMemHandle(&p, hd, cudaIpcMemLazyEnablePeerAccess));
    c->peer_mapped.push_back(p);
    opened.push_back({hd, static_cast<char*>(p)});
    *base = static_cast<char*>(p);
    return ASGD_OK;
  };
  for (int j = 0; j < world; ++j) {
    if (j == rank) {
      c->peer_params[j] = c->params;
      c->peer_sync[j] = reinterpret_cast<unsigned long long*>(c->P.meta + M_MSYNC);
      continue;
    }
    PeerHandle h;
    memcpy(&h, static_cast<const char*>(handles) + (size_t)j * ASGD_PEER_HANDLE_BYTES, sizeof(h));
    char* bp = nullptr;
    char* bw = nullptr;
    int rc = open(h.params, &bp);
    if (rc) return rc;
    rc = open(h.ws, &bw);
    if (rc) return rc;
    c->peer_params[j] = reinterpret_cast<float*>(bp + h.params_off);
    c->peer_sync[j] = reinterpret_cast<unsigned long long*>(bw + h.ws_off + (size_t)c->L.meta + M_MSYNC * 4);
  }
  c->peer_rank = rank;
  c->peer_world = world;
  CU(cudaStreamSynchronize(c->s));
  c->merge_epoch = 0;
  CU(cudaMemsetAsync(c->P.meta + M_MSYNC, 0, 12, c->s));   // arrival counter + CTA counter
  CU(cudaStreamSynchronize(c->s));
  return ASGD_OK;
}

int asgd_peer_close(asgd_ctx* c) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  CU(cudaSetDevice(c->device));
  CU(cudaStreamSynchronize(c->s));
  for (void* pm : c->peer_mapped) cudaIpcCloseMemHandle(pm);
  c->peer_mapped.clear();
  for (int j = 0; j < kMaxPeers; ++j) { c->peer_params[j] = nullptr; c->peer_sync[j] = nullptr; }
  c->peer_rank = -1;
  c->peer_world = 0;
  return ASGD_OK;
}

int asgd_merge_fused(asgd_ctx* c, const double* alpha, float gamma) {
  if (!c || !alpha) return fail(ASGD_E_ARG, "null argument");
  if (c->peer_world < 1) return fail(ASGD_E_STATE, "asgd_peer_open first");
  const int N = c->peer_world, r = c->peer_rank;
  PeerSet ps{};
  ps.n = N;
  for (int j = 0; j < N; ++j) { ps.p[j] = c->peer_params[j]; ps.sync[j] = c->peer_sync[j]; ps.alpha[j] = alpha[j]; }
  const int64_t P4 = c->Pn / 4, per = (P4 + N - 1) / N;
  const int64_t lo = std::min(P4, (int64_t)r * per) * 4;
  const int64_t hi = (r == N - 1) ? c->Pn : std::min(P4, (int64_t)(r + 1) * per) * 4;
  const unsigned long long goal = (++c->merge_epoch) * (unsigned long long)N;
  PCU(ASGD_K_MERGE, launch_merge_fused(c->lc(), ps, c->w, c->dd, lo, hi, gamma,
                                       reinterpret_cast<unsigned int*>(c->P.meta + M_MDONE),
                                       reinterpret_cast<unsigned long long*>(c->P.meta + M_MSYNC), goal));
  CU(refresh_shadow(c));
  c->u = 0;
  return ASGD_OK;
}

int asgd_replicas_weighted_sum(asgd_ctx* c, const float* const* reps, const double* alpha, int32_t n,
                               float* out) {
  if (!c || !reps || !alpha || !out || n < 1) return fail(ASGD_E_ARG, "bad argument");
  CU(launch_wsum(c->lc(), reps, alpha, n, c->Pn, out));
  return ASGD_OK;
}

int asgd_eval_topk(asgd_ctx* c, const asgd_csr* t, const int32_t* rows, int32_t n, int32_t k,
                   int32_t* topk) {
  if (!c || !t || !rows || !topk) return fail(ASGD_E_ARG, "null argument");
  if (k < 1 || k > 8) return fail(ASGD_E_ARG, "k=%d not in [1, 8]", k);
  if (c->eval_validated != (const void*)t->row_ptr) {
    int rc = validate(c, t);
    if (rc) return rc;
    c->eval_validated = t->row_ptr;
  }
  const asgd_model_desc& m = c->d;
  Launch lc = c->lc();
  const Ptrs& P = c->P;
  const int H = (int)m.H;
  const bool bf = m.precision == ASGD_PREC_BF16;
  float* W1 = c->params + c->o_w1;
  float* b1 = c->params + c->o_b1;
  float* W2 = c->params + c->o_w2;
  float* b2 = c->params + c->o_b2;
  for (int32_t r0 = 0; r0 < n; r0 += m.b_max) {
    const int nb = std::min<int32_t>(m.b_max, n - r0);
    CU(launch_spmm_fwd(lc, StepArgs{rows + r0, nullptr, 0.f, nb}, *t, W1, b1, H, P, c->L, true));
    Ptrs Pr = P;   // Z = H1 W2^T + b2 on the tensor cores (bf16, or bf16x3 on the fp32 path)
    Pr.w2b = c->w2b_buf[c->w2b_cur];
    Pr.w2l = c->w2l_buf[c->w2b_cur];
    CU(launch_gemm_tc(lc, 1, nb, m.L, H, Pr, c->L, W2, b2, nullptr, nullptr));
    CU(launch_topk(lc, nb, m.L, padded_ld(m.L), k, P.z, topk + (int64_t)r0 * k));
  }
  return ASGD_OK;
}

int asgd_sync(asgd_ctx* c) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  CU(cudaStreamSynchronize(c->s));
  CU(cudaGetLastError());
  int32_t err = 0;
  CU(cudaMemcpy(&err, c->P.meta + M_ERR, 4, cudaMemcpyDeviceToHost));
  if (err) {
    CU(cudaMemset(c->P.meta + M_ERR, 0, 4));
    return fail(ASGD_E_SHAPE, "device-side error 0x%x (1: step nnz > max_step_nnz, 2: labels > "
                "max_step_labels, 4: row id out of range)", err);
  }
  return ASGD_OK;
}

int asgd_kernel_launches(const asgd_ctx* c, int64_t* out) {
  if (!c || !out) return fail(ASGD_E_ARG, "null argument");
  *out = c->launches;
  return ASGD_OK;
}

int asgd_profile(asgd_ctx* c, int32_t class_mask) {
  if (!c) return fail(ASGD_E_ARG, "null ctx");
  c->prof_mask = (uint32_t)class_mask & ((1u << ASGD_PROF_N) - 1);
  for (int k = 0; k < ASGD_PROF_N; ++k) c->pused[k] = 0;
  return ASGD_OK;
}

int asgd_profile_read(asgd_ctx* c, double* ms, int64_t* cnt) {
  if (!c || !ms || !cnt) return fail(ASGD_E_ARG, "null argument");
  CU(cudaStreamSynchronize(c->s));
  CU(cudaStreamSynchronize(c->s2));
  CU(cudaStreamSynchronize(c->s3));
  for (int k = 0; k < ASGD_PROF_N; ++k) {
    double t = 0.0;
    for (size_t i = 0; i < c->pused[k]; ++i) {
      float e = 0.f;
      CU(cudaEventElapsedTime(&e, c->pev[k][2 * i], c->pev[k][2 * i + 1]));
      t += e;
    }
    ms[k] = t;
    cnt[k] = (int64_t)c->pused[k];
  }
  return ASGD_OK;
}

int asgd_copy_to_host(asgd_ctx* c, void* dst, const void* src, size_t bytes) {
  if (!c || !dst || !src) return fail(ASGD_E_ARG, "null argument");
  CU(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, c->s));
  return ASGD_OK;
}

// =================================================================== host-pure

int asgd_merge_weights(int32_t n, const int64_t* u, const int64_t* b, const double* nu,
                       double pert_thr, double delta, int32_t flags, double* alpha,
                       int32_t* r_out, int32_t* s_out, int32_t* perturbed_out) {
  if (n < 1 || !u || !b || !nu || !alpha) return fail(ASGD_E_ARG, "bad argument");
  if (flags & ~(ASGD_MERGE_RENORM | ASGD_MERGE_NORM_UB)) return fail(ASGD_E_ARG, "unknown merge flag");
  bool equal = true;                                   // Alg. 2 line 2
  for (int i = 1; i < n; ++i) equal = equal && (u[i] == u[0]);
  if (equal) {
    int64_t sb = 0;
    for (int i = 0; i < n; ++i) sb += b[i];
    const double d = (double)sb;
    for (int i = 0; i < n; ++i) alpha[i] = (double)b[i] / d;
  } else if (!(flags & ASGD_MERGE_NORM_UB)) {          // line 3
    int64_t su = 0;
    for (int i = 0; i < n; ++i) su += u[i];
    const double d = (double)su;
    for (int i = 0; i < n; ++i) alpha[i] = (double)u[i] / d;
  } else {                                             // R12: u_i b_i
    int64_t sub = 0;
    for (int i = 0; i < n; ++i) sub += u[i] * b[i];
    const double d = (double)sub;
    for (int i = 0; i < n; ++i) alpha[i] = (double)(u[i] * b[i]) / d;
  }
  bool gate = true;                                    // line 4 (Q16: strict <)
  for (int i = 0; i < n; ++i) gate = gate && (nu[i] < pert_thr);
  int r = 0, s = 0, pert = 0;
  if (gate) {                                          // line 5 (Q17: key (u, b), lowest index)
    for (int i = 1; i < n; ++i) {
      if (u[i] > u[r] || (u[i] == u[r] && b[i] > b[r])) r = i;
      if (u[i] < u[s] || (u[i] == u[s] && b[i] < b[s])) s = i;
    }
    if (u[r] != u[s] || b[r] != b[s]) {                // line 6
      alpha[r] = (1.0 + delta) * alpha[r];
      alpha[s] = (1.0 - delta) * alpha[s];
      pert = 1;
    }
  }
  if (flags & ASGD_MERGE_RENORM) {                     // Q34 option
    double tot = 0.0;
    for (int i = 0; i < n; ++i) tot += alpha[i];
    for (int i = 0; i < n; ++i) alpha[i] = alpha[i] / tot;
  }
  if (r_out) *r_out = r;
  if (s_out) *s_out = s;
  if (perturbed_out) *perturbed_out = pert;
  return ASGD_OK;
}

int asgd_scale_frequency(int32_t n, const int64_t* b_before, const int64_t* b_after, int32_t* last_sign,
                         int32_t interval, int32_t max_interval, int32_t* interval_out) {
  if (n < 1 || !b_before || !b_after || !last_sign || !interval_out || interval < 1 || max_interval < 1)
    return fail(ASGD_E_ARG, "bad argument");
  bool stable = true, osc = false;
  for (int i = 0; i < n; ++i) {   // R17: d_i = sign of rank i's move
    const int d = (b_after[i] > b_before[i]) - (b_after[i] < b_before[i]);
    if (d != 0) stable = false;
    if (d != 0 && last_sign[i] != 0 && d == -last_sign[i]) osc = true;
    if (d != 0) last_sign[i] = d;
  }
  *interval_out = (stable || osc) ? std::min(2 * interval, max_interval) : 1;
  return ASGD_OK;
}

int asgd_norm_per_param(int32_t n, const double* sqnorm, int64_t P, double* nu) {
  if (n < 1 || !sqnorm || !nu || P < 1) return fail(ASGD_E_ARG, "bad argument");
  for (int i = 0; i < n; ++i) {
    if (!(sqnorm[i] >= 0.0)) return fail(ASGD_E_ARG, "sqnorm[%d] = %g is negative or NaN", i, sqnorm[i]);
    nu[i] = std::sqrt(sqnorm[i]) / (double)P;        // Q16: ||w_i||_2 / |w|
  }
  return ASGD_OK;
}

int asgd_elastic_weights(int32_t n, double* alpha) {
  if (n < 1 || !alpha) return fail(ASGD_E_ARG, "bad argument");
  for (int i = 0; i < n; ++i) alpha[i] = 1.0 / (double)n;   // R10: alpha_i = 1/N
  return ASGD_OK;
}

int asgd_scale_batches(int32_t n, const int64_t* u, int64_t* b, double* lr_out, int64_t b_min,
                       int64_t b_max, int64_t beta, double lr_max) {
  if (n < 1 || !u || !b || b_min < 1 || b_max < b_min) return fail(ASGD_E_ARG, "bad argument");
  int64_t su = 0;                                      // Alg. 1 line 1
  for (int i = 0; i < n; ++i) su += u[i];
  for (int i = 0; i < n; ++i) {                        // line 2
    const int64_t num = beta * ((int64_t)n * u[i] - su);
    const int64_t delta = num >= 0 ? num / n : -((-num) / n);   // Q12: truncate toward 0
    if ((int64_t)n * u[i] > su && b[i] + delta <= b_max) b[i] += delta;        // lines 3-5
    else if ((int64_t)n * u[i] < su && b[i] + delta >= b_min) b[i] += delta;   // lines 6-8
  }
  if (lr_out)
    for (int i = 0; i < n; ++i) lr_out[i] = lr_max * (double)b[i] / (double)b_max;  // Q14
  return ASGD_OK;
}

int asgd_route_replay(int32_t n_ranks, int32_t nt, const int32_t* order, const int64_t* b, int64_t M,
                      int64_t* out, int64_t cap, int64_t* n_out) {
  if (n_ranks < 1 || nt < 0 || (nt && !order) || !b || !out || !n_out) return fail(ASGD_E_ARG, "bad argument");
  int64_t c = 0, k = 0;
  for (int32_t t = 0; t < nt && c < M; ++t) {
    const int32_t r = order[t];
    if (r < 0 || r >= n_ranks) return fail(ASGD_E_ARG, "order[%d] = %d not in [0, %d)", t, r, n_ranks);
    const int64_t len = std::min<int64_t>(b[r], M - c);
    if (k >= cap) return fail(ASGD_E_SHAPE, "route cap %lld too small", (long long)cap);
    out[3 * k] = r; out[3 * k + 1] = c; out[3 * k + 2] = len;
    ++k;
    c += len;
  }
  *n_out = k;
  return ASGD_OK;
}

int asgd_route_static(int32_t n, int64_t b, int64_t M, int64_t* out, int64_t cap, int64_t* n_out) {
  if (n < 1 || b < 1 || M < 0 || !out || !n_out) return fail(ASGD_E_ARG, "bad argument");
  int64_t k = 0;
  for (int64_t c = 0; c < M; c += b, ++k) {   // R10: batch k -> rank k mod n
    if (k >= cap) return fail(ASGD_E_SHAPE, "route cap %lld too small", (long long)cap);
    out[3 * k] = k % n; out[3 * k + 1] = c; out[3 * k + 2] = std::min<int64_t>(b, M - c);
  }
  *n_out = k;
  return ASGD_OK;
}

int asgd_route_simulate(int32_t n, const int64_t* b, int64_t M, const double* cf, double per_row,
                        const int64_t* row_nnz, int64_t* out, int64_t cap, int64_t* n_out) {
  if (n < 1 || !b || !cf || !row_nnz || !out || !n_out) return fail(ASGD_E_ARG, "bad argument");
  std::vector<double> fr(n, 0.0);
  int64_t c = 0, k = 0;
  while (c < M) {
    int r = 0;
    for (int i = 1; i < n; ++i) if (fr[i] < fr[r]) r = i;   // ties: lowest id
    const int64_t len = std::min<int64_t>(b[r], M - c);
    if (len < 1) return fail(ASGD_E_ARG, "batch size < 1");
    int64_t nnz = 0;
    for (int64_t j = c; j < c + len; ++j) nnz += row_nnz[j];
    if (k >= cap) return fail(ASGD_E_SHAPE, "route cap %lld too small", (long long)cap);
    out[3 * k] = r; out[3 * k + 1] = c; out[3 * k + 2] = len;
    ++k;
    fr[r] += cf[r] * ((double)nnz + per_row * (double)len);
    c += len;
  }
  *n_out = k;
  return ASGD_OK;
}

int asgd_precision_at_k(const int32_t* top, const int64_t* lab_ptr, const int32_t* lab, int32_t n,
                        int32_t k, int64_t* hits_out) {
  if (!top || !lab_ptr || !lab || !hits_out || k < 1) return fail(ASGD_E_ARG, "bad argument");
  int64_t hits = 0;
  for (int32_t r = 0; r < n; ++r) {
    const int32_t* y = lab + lab_ptr[r];
    const int64_t ny = lab_ptr[r + 1] - lab_ptr[r];
    for (int32_t j = 0; j < k; ++j) {
      const int32_t p = top[(int64_t)r * k + j];
      if (std::binary_search(y, y + ny, p)) ++hits;   // labels sorted within a row
    }
  }
  *hits_out = hits;
  return ASGD_OK;
}

// ------------------------------------------------------------------- scheduler
struct ShmSched {
  std::atomic<uint64_t> packed;   // ticket << 40 | cursor
  int64_t M;
  int64_t mb;
  int64_t n_ranks;
  int64_t cap;
  int64_t log[1][4];
};

struct asgd_sched {
  ShmSched* h;
  size_t bytes;
  std::string name;
};

static constexpr uint64_t kCurMask = (1ull << 40) - 1;

int asgd_sched_open(const char* name, int32_t n_ranks, int64_t M, int32_t create, asgd_sched** out) {
  if (!name || !out || n_ranks < 1 || M < 1 || M >= (1ll << 38)) return fail(ASGD_E_ARG, "bad argument");
  const int64_t cap = M + 16;
  const size_t bytes = sizeof(ShmSched) + (size_t)cap * 4 * sizeof(int64_t);
  int fd = shm_open(name, create ? (O_CREAT | O_RDWR) : O_RDWR, 0600);
  if (fd < 0) return fail(ASGD_E_ARG, "shm_open(%s) failed", name);
  if (create && ftruncate(fd, (off_t)bytes) != 0) { close(fd); return fail(ASGD_E_ARG, "ftruncate failed"); }
  void* p = mmap(nullptr, bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (p == MAP_FAILED) return fail(ASGD_E_ARG, "mmap failed");
  ShmSched* h = static_cast<ShmSched*>(p);
  if (create) {
    new (&h->packed) std::atomic<uint64_t>(0);
    h->M = M; h->mb = 0; h->n_ranks = n_ranks; h->cap = cap;
  }
  asgd_sched* s = new (std::nothrow) asgd_sched{h, bytes, name};
  if (!s) { munmap(p, bytes); return fail(ASGD_E_ARG, "out of host memory"); }
  *out = s;
  return ASGD_OK;
}

int asgd_sched_next(asgd_sched* s, int32_t rank, int64_t b, int64_t* start, int64_t* len) {
  if (!s || !start || !len || b < 1) return -ASGD_E_ARG;
  ShmSched* h = s->h;
  const uint64_t v = h->packed.fetch_add((1ull << 40) | (uint64_t)b, std::memory_order_acq_rel);
  const int64_t ticket = (int64_t)(v >> 40), c = (int64_t)(v & kCurMask);
  if (c >= h->M) return 0;
  const int64_t l = std::min<int64_t>(b, h->M - c);
  if (ticket < h->cap) {   // entry [0] = mega-batch generation << 40 | ticket, stored last (release)
    const int64_t gen = __atomic_load_n(&h->mb, __ATOMIC_ACQUIRE);
    h->log[ticket][1] = rank; h->log[ticket][2] = c; h->log[ticket][3] = l;
    __atomic_store_n(&h->log[ticket][0], (gen << 40) | ticket, __ATOMIC_RELEASE);
  }
  *start = c;
  *len = l;
  return 1;
}

}  // extern "C"

namespace {
// The rank's step loop shared by the dynamic and the static schedule: next(&start, &len)
// returns 1 for a batch, 0 when the rank's share is done, < 0 on error.
// Step groups: with a schedule that gives this rank its tickets regardless of timing (one
// rank, or Elastic's static split), up to step_group() consecutive tickets of equal length
// are enqueued as one graph replay of that many steps -- the ~3.5 us between two step
// graphs becomes an in-graph kernel boundary.  ASGD_STEP_GROUP (default kDefGroup, 1 = off).
// Measured (EURLex bench line): 1 / 4 / 8 / 16 steps per replay -> 4.25 / 4.55 / 4.54 / 4.52 M
// samples/s; results bitwise equal to one graph per step (tests/test_gpu_step_groups.py).
constexpr int kMaxGroup = 16, kDefGroup = 4;
int step_group() {
  static const int v = [] {
    const char* e = getenv("ASGD_STEP_GROUP");
    return std::max(1, std::min(kMaxGroup, e ? atoi(e) : kDefGroup));
  }();
  return v;
}

template <typename Next>
int run_steps(asgd_ctx* c, Next next, const int32_t* stream_rows, float lr, float* losses, int64_t losses_cap,
              int32_t inflight, int64_t* n_steps, bool may_group = false) {
  if (inflight < 1 || inflight > kMaxInflight) return fail(ASGD_E_ARG, "inflight=%d not in [1, %d]", inflight, kMaxInflight);
  for (auto& ev : c->ev_ring)
    if (!ev) CU(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  // only in the stored-Z regime (no K-3): with K-3's grid-barrier kernels in the group graph
  // AmazonCat-13K measured 4.66 vs 5.46 M samples/s at 4 steps per replay
  const bool stored_z = (int64_t)c->d.b_max * c->d.L * 4 <= fused_ce_bytes();
  const int grp = (may_group && stored_z && graphs_enabled() && !c->dbg && !c->trace && c->prof_mask == 0)
                      ? step_group() : 1;
  int64_t k = 0, launches = 0;
  int64_t pend_st = -1, pend_len = 0;   // a ticket taken but not yet enqueued (length change)
  for (;;) {
    if (launches >= inflight) CU(cudaEventSynchronize(c->ev_ring[(launches - inflight) % kMaxInflight]));
    if (grp == 1) {
      int64_t start = 0, len = 0;
      const int r = next(&start, &len);
      if (r < 0) return fail(-r, "scheduler failed");
      if (r == 0) break;
      c->cur_start = start;
      const int rc = asgd_local_step(c, stream_rows + start, (int32_t)len, lr,
                                     (losses && k < losses_cap) ? losses + k : nullptr);
      c->cur_start = -1;
      if (rc != ASGD_OK) return rc;
      ++k;
    } else {
      int64_t st[kMaxGroup];
      int64_t len = 0;
      int g = 0;
      if (pend_st >= 0) { st[g++] = pend_st; len = pend_len; pend_st = -1; }
      while (g < grp) {
        int64_t a = 0, l = 0;
        const int r = next(&a, &l);
        if (r < 0) return fail(-r, "scheduler failed");
        if (r == 0) break;
        if (g > 0 && l != len) { pend_st = a; pend_len = l; break; }
        st[g++] = a;
        len = l;
      }
      if (g == 0) break;
      const asgd_model_desc& m = c->d;
      if (len < 1 || len > m.b_max) return fail(ASGD_E_SHAPE, "n_rows=%lld not in [1, %d]", (long long)len, m.b_max);
      if (!c->has_data) return fail(ASGD_E_STATE, "no data registered");
      StepArgs sas[kMaxGroup];
      for (int i = 0; i < g; ++i)
        sas[i] = StepArgs{stream_rows + st[i], (losses && k + i < losses_cap) ? losses + k + i : nullptr, lr, (int)len};
      const int rc = step_graph(c, (int)len, g, sas);
      if (rc != ASGD_OK) return rc;
      c->w2b_cur ^= (g & 1);
      c->u += g;
      k += g;
    }
    CU(cudaEventRecord(c->ev_ring[launches % kMaxInflight], c->s));
    ++launches;
  }
  *n_steps = k;
  return ASGD_OK;
}
}  // namespace

extern "C" {

int asgd_run_tickets(asgd_ctx* c, asgd_sched* s, int32_t rank, int64_t b_i, const int32_t* stream_rows,
                     float lr, float* losses, int64_t losses_cap, int32_t inflight, int64_t* n_steps) {
  if (!c || !s || !stream_rows || !n_steps || b_i < 1) return fail(ASGD_E_ARG, "bad argument");
  // one rank takes every ticket in order whatever the timing: its tickets may be grouped
  return run_steps(c, [&](int64_t* st, int64_t* ln) { return asgd_sched_next(s, rank, b_i, st, ln); }, stream_rows,
                   lr, losses, losses_cap, inflight, n_steps, s->h->n_ranks == 1);
}

int asgd_run_static(asgd_ctx* c, int32_t rank, int32_t world, int64_t b, const int32_t* stream_rows, int64_t M,
                    float lr, float* losses, int64_t losses_cap, int32_t inflight, int64_t* n_steps) {
  if (!c || !stream_rows || !n_steps || b < 1 || M < 0 || world < 1 || rank < 0 || rank >= world)
    return fail(ASGD_E_ARG, "bad argument");
  int64_t cur = (int64_t)rank * b;
  return run_steps(c, [&](int64_t* st, int64_t* ln) {
                     if (cur >= M) return 0;
                     *st = cur;
                     *ln = std::min<int64_t>(b, M - cur);
                     cur += (int64_t)world * b;
                     return 1;
                   },
                   stream_rows, lr, losses, losses_cap, inflight, n_steps, true);   // static split: groupable
}

int asgd_sched_log(asgd_sched* s, int64_t* out, int64_t cap, int64_t* n_out) {
  if (!s || !out || !n_out) return fail(ASGD_E_ARG, "null argument");
  ShmSched* h = s->h;
  const int64_t T = (int64_t)(h->packed.load(std::memory_order_acquire) >> 40);
  const int64_t gen = __atomic_load_n(&h->mb, __ATOMIC_ACQUIRE);
  int64_t c = 0, k = 0;
  while (k < T && k < h->cap && c < h->M) {
    // an entry of an earlier mega-batch (same ticket slot) carries an older generation
    const int64_t tag = __atomic_load_n(&h->log[k][0], __ATOMIC_ACQUIRE);
    if (tag != ((gen << 40) | k) || h->log[k][2] != c)
      return fail(ASGD_E_STATE, "log entry %lld of mega-batch %lld not yet written", (long long)k, (long long)gen);
    if (k >= cap) return fail(ASGD_E_SHAPE, "cap too small");
    out[4 * k] = k;
    for (int j = 1; j < 4; ++j) out[4 * k + j] = h->log[k][j];
    c += h->log[k][3];
    ++k;
  }
  *n_out = k;
  return ASGD_OK;
}

int asgd_sched_reset(asgd_sched* s, int64_t mb) {
  if (!s) return fail(ASGD_E_ARG, "null argument");
  s->h->packed.store(0, std::memory_order_release);
  reinterpret_cast<std::atomic<int64_t>*>(&s->h->mb)->store(mb, std::memory_order_release);
  return ASGD_OK;
}

int asgd_sched_wait(asgd_sched* s, int64_t mb, int64_t timeout_ms) {
  if (!s) return fail(ASGD_E_ARG, "null argument");
  auto* p = reinterpret_cast<std::atomic<int64_t>*>(&s->h->mb);
  for (int64_t spins = 0;; ++spins) {
    if (p->load(std::memory_order_acquire) >= mb) return ASGD_OK;
    if (spins / 20 > timeout_ms) return fail(ASGD_E_STATE, "timeout waiting for mega-batch %lld", (long long)mb);
    usleep(50);
  }
}

int asgd_sched_close(asgd_sched* s, int32_t unlink_shm) {
  if (!s) return fail(ASGD_E_ARG, "null argument");
  munmap(s->h, s->bytes);
  if (unlink_shm) shm_unlink(s->name.c_str());
  delete s;
  return ASGD_OK;
}

}  // extern "C"

namespace asgd {
cudaError_t smem_attr_raw(const void* kernel, size_t bytes) {
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, size_t> done;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  std::lock_guard<std::mutex> g(mu);
  size_t& have = done[{kernel, dev}];
  if (have >= bytes) return cudaSuccess;
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
  if (e == cudaSuccess) have = bytes;
  return e;
}

// Programmatic dependent launch: each kernel's prologue overlaps its predecessor's tail.
// Measured (samples/s, PDL off -> on): bf16 EURLex 4.01 -> 4.22 M, AmazonCat 5.35 -> 5.46 M,
// Wiki10 1.356 -> 1.383 M, Amazon-670K / Delicious-200K even.  (Round 1's fp32 path, SIMT
// GEMMs, measured 1.52 -> 1.34 M with it; the fp32 path now runs the same tcgen05 DAG.)
// ASGD_PDL: unset = on; 0 = off; 1 = every kernel; 2 = GEMMs only.
int pdl_mode() {
  static const int m = [] {
    const char* v = getenv("ASGD_PDL");
    return v ? atoi(v) : -1;
  }();
  return m;
}
bool pdl_for(bool) { return pdl_mode() < 0 ? true : pdl_mode() == 1; }
}  // namespace asgd
