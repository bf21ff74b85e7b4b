// Internal declarations shared by the libasgd translation units (not ABI).
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include "../../include/asgd.h"

namespace asgd {

// Entries per work piece of the nnz-balanced sparse kernels (K-1, K-5).
constexpr int kPiece = 32;
// Max labels per row the softmax kernel stages in shared memory.
constexpr int kMaxRowLabels = 1024;
// Features per tile of the touched-feature scan.
constexpr int kScanTile = 1024;
// meta[] slots (int32, device)
// M_LR: the step's learning rate (float bits), M_LOSS: 64-bit device pointer the
// step's mean loss goes to (slots 10-11), both written by K-0 (a) so that the
// rest of the step (and its CUDA graph) takes no per-step scalar arguments;
// M_BAR: 64-bit grid-barrier counter (slots 32-33).
// M_K0PAR: parity of K-0's double-buffered tile sums.
// M_MSYNC: fused merge arrival counter (64-bit, slots 40-41), M_MDONE: its CTA counter.
enum { M_NNZ = 0, M_NLAB = 1, M_U = 2, M_ERR = 3, M_NROWS = 4, M_TILE = 5, M_LR = 6, M_K0PAR = 7, M_COUNT = 8,
       M_LOSS = 10, M_BAR = 32, M_MSYNC = 40, M_MDONE = 42, M_CEN = 44, M_G2BAR = 46 /* 46-48 */,
       M_KBAR = 50 /* 50-51: K-3's packed grid barrier */ };
// error bits in meta[M_ERR]
enum { ERR_NNZ_CAP = 1, ERR_LAB_CAP = 2, ERR_ROW_ID = 4 };

typedef __nv_bfloat16 bf16;

// Device workspace carve-up (byte offsets from ws base; all 256-B aligned).
struct WsLayout {
  size_t meta, boff, loff, cnt, fseg, fuid, uniq, useg, tsum, tpre;
  size_t e_n, e_v, e_u, e_f, part1, rowcnt, part5, ucnt, bits;
  size_t h1, h1b, z, dzb, rowloss, dhpart, da1, db1part, w2b, w2b2, red, eval_top, rbase, da1b, zstat, lse;
  size_t rowsc, cen, cenpart;
  size_t h1l, dzl, w2l, w2l2;   // bf16x3 lo halves (fp32 path, R14)
  bool x3;                      // fp32 path: GEMM operands split hi + lo (R14)
  size_t total;
  int64_t nz_cap, nl_cap, u_cap, n_tiles_f, n_pieces, splitk, n_rowblk, n_red, part_stride, stats_ld;
  int64_t dh_parts;             // dH1 partial slices (>= splitk; K-3 one-pass: up to one per label tile)
};

WsLayout ws_layout(const asgd_model_desc& d);

struct Ptrs {  // typed views of the workspace
  int32_t* meta; int32_t* boff; int32_t* loff; int32_t* cnt; int32_t* fseg; int32_t* fuid;
  int32_t* uniq; int32_t* useg; int32_t* tsum; int32_t* tpre;
  int32_t* e_n; float* e_v; int32_t* e_u; int32_t* e_f; uint32_t* bits; float* part1; int32_t* rowcnt; float* part5;
  int32_t* ucnt; float* h1; bf16* h1b; float* z; bf16* dzb; float* rowloss; float* dhpart;
  float* da1; float* db1part; bf16* w2b; double* red; int32_t* eval_top;
  int64_t* rbase;   // row_ptr[rows[r]] of the current batch (written by K-0 (a))
  bf16* da1b;       // bf16 copy of dA1 (bf16 path; staged by K-5)
  float* lse;       // per-row log-sum-exp of Z (bf16 path)
  int32_t* rowsc;   // copy of the step's dataset row ids (written by K-0 (a))
  float* cen;       // centred sigmoid offsets [2 H] (bf16 path, R11)
  float* cenpart;   // their per-CTA partials [kCenterParts H]
  // fp32 path (R14): the bf16x3 lo halves of H1, dZ and the W2 shadow (h1b / dzb / w2b are
  // the hi halves); null on the bf16 path
  bf16* h1l; bf16* dzl; bf16* w2l;
};
__device__ __forceinline__ float step_lr(const int32_t* meta) { return __int_as_float(meta[M_LR]); }
__device__ __forceinline__ float* step_loss(const int32_t* meta) {
  return *reinterpret_cast<float* const*>(meta + M_LOSS);
}
int row_block();   // rows per db1 partial (kernels_dense.cu)
Ptrs ws_ptrs(char* base, const WsLayout& L);

struct Launch {       // launch bookkeeping of one ctx
  cudaStream_t s;
  int64_t* counter;
  int sms;
  bool pdl;           // programmatic dependent launch (see pdl_mode)
};

// Programmatic dependent launch: every kernel of the step lets its successor be
// scheduled as soon as all of its own CTAs run (pdl_trigger at entry) and waits
// for its predecessor's completion + memory flush (pdl_wait) before touching
// the predecessor's outputs, so prologues (smem carve-up, mbarrier init, TMEM
// alloc, tensormap prefetch) overlap the previous kernel's tail.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

// Kernel timeline (asgd_timeline_set, tools/timeline.py), compiled in only with
// -DASGD_TIMELINE: per kernel class, [0] the earliest CTA arrival, [1] the earliest
// return from griddepcontrol.wait (the predecessor's outputs are visible: on the
// step's chain, the predecessor's end), [2] the latest CTA end (its last thread), in
// %globaltimer ns.  Each translation unit holds its own copy of the buffer pointer.
// TL_MARK(k): phase marks inside a kernel (slots [3 k], [3 k + 1] = the earliest and [3 k + 2]
// the latest time a CTA's calling thread passed mark k; TL_PH0.. are the K-3 phases).
enum { TL_TOUCHED = 0, TL_SPMM, TL_G1, TL_SOFTMAX, TL_G2, TL_DH, TL_B1, TL_G3, TL_SCATTER, TL_G1B, TL_MERGE,
       TL_OTHER, TL_PH0, TL_PH1, TL_PH2, TL_PH3, TL_PH4, TL_PH5, TL_PH6, TL_PH7, TL_N };
#ifdef ASGD_TIMELINE
static __device__ unsigned long long* g_tl;
__device__ __forceinline__ unsigned long long tl_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
struct Tl {
  int id;
  unsigned long long t0;
  __device__ explicit Tl(int i) : id(i), t0(tl_now()) {}
  __device__ void ready() {
    if (threadIdx.x == 0 && g_tl) {
      atomicMin(&g_tl[3 * id], t0);
      atomicMin(&g_tl[3 * id + 1], tl_now());
    }
  }
  __device__ ~Tl() {
    if (threadIdx.x == blockDim.x - 1 && g_tl) atomicMax(&g_tl[3 * id + 2], tl_now());
  }
};
#define ASGD_TL_SETTER(fn) \
  cudaError_t fn(unsigned long long* p) { return cudaMemcpyToSymbol(g_tl, &p, sizeof(p)); }
#define TL_MARK(k)                                  \
  do {                                              \
    if (g_tl) {                                     \
      const unsigned long long t_ = tl_now();       \
      atomicMin(&g_tl[3 * (k)], t_);                \
      atomicMin(&g_tl[3 * (k) + 1], t_);            \
      atomicMax(&g_tl[3 * (k) + 2], t_);            \
    }                                               \
  } while (0)
#else
#define TL_MARK(k) do { } while (0)
struct Tl {
  __device__ explicit Tl(int) {}
  __device__ void ready() {}
};
#define ASGD_TL_SETTER(fn) \
  cudaError_t fn(unsigned long long*) { return cudaErrorNotSupported; }
#endif
cudaError_t tl_set_sparse(unsigned long long*);
cudaError_t tl_set_dense(unsigned long long*);
cudaError_t tl_set_tc(unsigned long long*);
cudaError_t tl_set_merge(unsigned long long*);

// ASGD_PDL: unset = on for the bf16 path, off for fp32; 0 off; 1 every kernel; 2 the
// tcgen05 GEMMs only
int pdl_mode();
bool pdl_for(bool bf16);   // launch_k: this ctx's kernels use PDL

// fp32 path on the tensor cores ("bf16x3", R14): x = hi + lo with hi = bf16(x)
// and lo = bf16(x - hi) (x - hi is exact in fp32); a product x y is taken as
// hi_x hi_y + hi_x lo_y + lo_x hi_y in three bf16 MMAs with fp32 accumulation.
__device__ __forceinline__ float bf16_lo_of(float x) {
  return x - __bfloat162float(__float2bfloat16_rn(x));
}

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) is a per-device setting: it is
// applied once per (kernel, current device) and raised when a larger size is needed.
cudaError_t smem_attr_raw(const void* kernel, size_t bytes);   // thread-safe
template <typename... KArgs>
cudaError_t ensure_smem(void (*kernel)(KArgs...), size_t bytes) {
  return smem_attr_raw(reinterpret_cast<const void*>(kernel), bytes);
}

template <typename... KArgs, typename... Args>
cudaError_t launch_k(const Launch& lc, void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem,
                     Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = lc.s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = lc.pdl ? 1 : 0;
  ++*lc.counter;
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

template <typename... KArgs, typename... Args>
cudaError_t launch_k_pdl(const Launch& lc, bool pdl, void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem,
                     Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = lc.s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  ++*lc.counter;
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

// ---------------------------------------------------------------- K-0
// The step's per-call arguments: the only kernel arguments that change from
// step to step (the first parameter of K-0 and K-1; CUDA-graph replays update
// just these two nodes).
struct StepArgs {
  const int32_t* rows;   // dataset row ids of the batch (device)
  float* loss;           // nullable device scalar for the mean loss
  float lr;
  int n;
};
// Global batch view published by CTA 0 of K-1 for the rest of the step.
struct ViewOut {
  int32_t* boff; int32_t* loff; int64_t* rbase; int32_t* rowsc; int32_t* meta;
};
// K-0 (b-e): touched-feature set; builds its own batch view.
cudaError_t launch_touched(const Launch&, const StepArgs&, const asgd_csr&, int64_t F, const Ptrs&,
                           const WsLayout&, int b_max);
// ---------------------------------------------------------------- K-1
// Builds the batch view (K-0 (a)) and publishes it, meta and the row ids for the step.
// fold: K-0's phase A inside K-1 (k0_fold(); the step's K-0 then starts at phase C)
cudaError_t launch_spmm_fwd(const Launch&, const StepArgs&, const asgd_csr&, const float* W1, const float* b1,
                            int H, const Ptrs&, const WsLayout&, bool want_bf16, bool fold = false, int b_max = 0);
bool k0_fold();
const void* spmm_fwd_func(int H);
const void* touched_func(int b_max);
int spmm_fwd_nargs();   // parameter counts (all K-1 instantiations share the signature)
int touched_nargs();
// ---------------------------------------------------------------- K-5
// dA1b: bf16 copy of dA1 (bf16 path) or null (fp32 path stages fp32 dA1).
// The learning rate of every SGD update is the step's meta[M_LR].
cudaError_t launch_scatter_sgd(const Launch&, float* W1, int H, const Ptrs&,
                               const WsLayout&, float* grad_w1, const bf16* dA1b, int b_max);
// ---------------------------------------------------------------- dense (CUDA cores)
// Leading dimension of the B x L logit buffers (16-byte rows for TMA).
int64_t padded_ld(int64_t L);
// stats (nullable): G1's per (N tile, row) (max, sum exp) partials -> one pass over Z.
cudaError_t launch_softmax_ce(const Launch&, int n, int64_t L, int64_t ldz, const int32_t* rows,
                              const int64_t* lab_ptr, const int32_t* lab, const Ptrs&,
                              bool bf16_out, const float2* stats = nullptr, int ntiles = 0,
                              int64_t stats_ld = 0);
// Sigmoid-BCE (R11) over the stored Z (fp32 path): row loss, dZ = (sigmoid(Z) - Y)/B.
cudaError_t launch_sigmoid_ce(const Launch&, int n, int64_t L, int64_t ldz, const int32_t* rows,
                              const int64_t* lab_ptr, const int32_t* lab, const Ptrs&, bool bf16_out);
// Row loss of the fused sigmoid path from G1's per-(tile half, row) BCE partials.
cudaError_t launch_tile_loss(const Launch&, int n, int ntiles, int64_t stats_ld, const float2* stats, const Ptrs&);
cudaError_t launch_dh_reduce(const Launch&, int n, int H, int splitk, const Ptrs&, const WsLayout&,
                             bool want_bf16, const float* dh_off = nullptr);
// Centred sigmoid dZ (R11): cen[0:H] = (1/(2B)) sum_j W2_j (bf16 shadow, the dH1 offset),
// cen[H:2H] = (1/(2B)) sum_n H1_n (the dW2 offset).  part: fp32[2 parts H]; counter: zeroed.
// w2f (nullable): sum the fp32 W2 instead (bf16x3 fp32 path, R14).
cudaError_t launch_sig_center(const Launch&, const bf16* w2b, const float* w2f, int64_t L, int H, const float* h1,
                              int n, float* part, unsigned int* counter, float* cen);
constexpr int kCenterParts = 148;
cudaError_t launch_b1_update(const Launch&, int n, int H, float* b1, const Ptrs&,
                             const WsLayout&, float* grad_b1);
// dst_lo (nullable): also the bf16x3 lo half bf16(x - bf16(x)) (R14)
cudaError_t launch_to_bf16(const Launch&, const float* src, bf16* dst, int64_t count, bf16* dst_lo = nullptr);
// ---------------------------------------------------------------- tcgen05 (bf16)
bool tc_available();
// which: 1 = G1 (Z = H1 W2^T + b2), 2 = G2 (dH1 split-K partials), 3 = G3 (W2 -= lr dZ^T H1 and
// b2 -= lr 1^T dZ, both fused in the epilogue)
// stats (G1 only, nullable): per (N tile, row) softmax partials; *stats_ntiles = N tiles.
// G2 with the dH1 reduce, ReLU' and the b1 update fused into its tail (which = 2).
struct DhFuse {
  float* b1; float* grad_b1; const float* dh_off; bool want_bf16;
};
cudaError_t launch_gemm_tc(const Launch&, int which, int n_rows, int64_t L, int H,
                           const Ptrs&, const WsLayout&, float* W2, float* b2, float* grad_w2,
                           float* grad_b2, float2* stats = nullptr, int* stats_ntiles = nullptr,
                           const int32_t* dz_rows = nullptr, const int64_t* dz_lab_ptr = nullptr,
                           const int32_t* dz_lab = nullptr, const float* hoff = nullptr,
                           const DhFuse* fuse = nullptr);
// K-3 (dH1 half): G1b + G2 + the dH1 reduce in one persistent kernel for the fused
// softmax-CE regime (bf16, H = 256): Z tiles recomputed from the resident H1 block, dZ
// formed on chip and fed straight into dH1 += dZ W2; write_dz also TMA-stores dZ for G3.
// one_pass: no G1 / k_lse before it -- a first sweep of S tiles gives the softmax
// statistics (partials in stats), a grid barrier, then lse, the row losses and the dZ /
// dH1 sweep (S recomputed).
cudaError_t launch_bwd_dh(const Launch&, int n, int64_t L, int H, const Ptrs&, const WsLayout&, float* b2,
                          const int32_t* rows, const int64_t* lab_ptr, const int32_t* lab, const DhFuse& fz,
                          bool write_dz, bool one_pass = false, float2* stats = nullptr, bool dz_only = false);
// dz_only: one label tile per CTA (LR = label tiles), no MMA 2 / reduce: the kernel replaces
// G1 + softmax-CE (dZ to P.dzb, row losses), G2 and the dH reduce run after it.
// the one-pass mode's partials fit the workspace (LR x MT CTAs of K-3 for n rows)
bool bwd_dh_one_pass_fits(int n, int64_t L, const WsLayout&, int sms);
// K-3 (dW2 half): G1b + G3 in one persistent kernel: per W2 row tile, Z^T recomputed per row
// chunk, dZ^T on chip into dW2, then W2 / b2 SGD and the next bf16 shadow (Pw.w2b).
cudaError_t launch_bwd_dw(const Launch&, int n, int64_t L, int H, const Ptrs& Pr, const Ptrs& Pw, float* W2,
                          float* b2, const int32_t* rows, const int64_t* lab_ptr, const int32_t* lab,
                          float* grad_w2, float* grad_b2);
// CTAs G2 runs with (the concurrent G3 leaves those SMs to it).
int gemm_tc_g2_ctas(int n, int H, const WsLayout&, int sms);
// which = 4 (G1b): dZ = (softmax - T)/B from a recomputed Z tile; needs P.lse from k_lse.
// which = 5: G1 without storing Z (only the softmax partials), for the fused path.
// which = 6: G1 with the sigmoid-BCE epilogue (R11): dZ = (sigmoid(Z) - Y)/B stored bf16,
//            per-(tile half, row) loss partials in stats; Z never stored.
cudaError_t launch_lse(const Launch&, int n, int H, int ntiles, int64_t stats_ld, const float2* stats,
                       const int32_t* rows, const int64_t* lab_ptr, const int32_t* lab, const bf16* h1b,
                       const bf16* w2b, const float* b2, const Ptrs&);
// ---------------------------------------------------------------- merge / eval
cudaError_t launch_sqnorm(const Launch&, const float* x, int64_t P, double* partials, int nparts,
                          double* out);
cudaError_t launch_scale(const Launch&, float* x, int64_t P, double alpha);
cudaError_t launch_finish(const Launch&, float* params, float* w, float* d, int64_t P, float gamma);
cudaError_t launch_wsum(const Launch&, const float* const* reps, const double* alpha, int n,
                        int64_t P, float* out);
// Fused peer-memory merge (NEXT-1): replica pointers, arrival counters and
// weights of the N ranks (N <= 8), by value.
constexpr int kMaxPeers = 8;
struct PeerSet {
  float* p[kMaxPeers];
  unsigned long long* sync[kMaxPeers];
  double alpha[kMaxPeers];
  int n;
};
cudaError_t launch_merge_fused(const Launch&, const PeerSet&, float* w, float* d, int64_t lo, int64_t hi,
                               float gamma, unsigned int* cta_done, const unsigned long long* arrived,
                               unsigned long long goal);
cudaError_t launch_topk(const Launch&, int n, int64_t L, int64_t ldz, int k, const float* z,
                        int32_t* out);
cudaError_t launch_validate_csr(const Launch&, const asgd_csr* c, int64_t F, int64_t L, int32_t* err);

}  // namespace asgd
