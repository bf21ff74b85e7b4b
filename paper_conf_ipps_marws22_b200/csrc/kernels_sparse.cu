// Sparse kernels of the local step (sm_100a):
//   K-0  batch CSR view + touched-feature set (rows a2 of DESIGN.md),
//   K-1  CSR SpMM forward A1 = X W1 + b1, H1 = ReLU(A1)   (row a3),
//   K-5  scatter-SGD  W1[f,:] -= lr sum_n X_nf dA1[n,:]     (row a8).
// The first layer is X (B x F, CSR) times W1 (F x H)
// (§V-A) with the sparse algebra the paper ran through cuSPARSE
// (P:1503-1506); its cost tracks the batch's nnz, so both K-1 and
// K-5 split the batch's nnz into fixed pieces of kPiece entries (one warp
// each) instead of one warp per row / per feature: a skewed row (Wiki10-shaped
// rows reach 10^4 nnz) spans many warps.  Segments spanning pieces are
// combined by the last-arriving warp in piece order, so every sum has a
// fixed order: results are bitwise deterministic.
#include <algorithm>
#include <cstdlib>

#include "asgd_internal.h"

namespace asgd {

namespace {

constexpr unsigned kFull = 0xffffffffu;

// Message-passing fence of the last-arriver combines (partial stores -> counter atomic,
// counter observed -> partial loads): acquire-release at GPU scope is all the pattern needs
// (ASGD_FENCE_SC=1 compiles the sequentially consistent __threadfence instead; ncu showed
// the SC fences as K-5's top stall, 21 % membar).
__device__ __forceinline__ void fence_mp() {
#ifdef ASGD_FENCE_SC
  __threadfence();
#else
  asm volatile("fence.acq_rel.gpu;" ::: "memory");
#endif
}

__device__ __forceinline__ int entry_row(const int32_t* sboff, int n, int e) {
  // largest r in [0, n) with sboff[r] <= e (rows may be empty)
  int lo = 0, hi = n;          // invariant: answer in [lo, hi)
  while (hi - lo > 1) {
    int mid = (lo + hi) >> 1;
    if (sboff[mid] <= e) lo = mid; else hi = mid;
  }
  // skip empty rows that share the offset
  while (lo + 1 < n && sboff[lo + 1] <= e) ++lo;
  return lo;
}

// lane <-> column map of a row of H = 32 * VPL floats
template <int VPL>
struct RowIO {
  __device__ __forceinline__ static int col(int lane, int i) {
    if constexpr (VPL == 2) return 2 * lane + i;
    else return (i >> 2) * 128 + 4 * lane + (i & 3);
  }
  __device__ __forceinline__ static void load_ldg(const float* row, int lane, float (&v)[VPL]) {
    if constexpr (VPL == 2) {
      float2 t = __ldg(reinterpret_cast<const float2*>(row) + lane);
      v[0] = t.x; v[1] = t.y;
    } else {
#pragma unroll
      for (int j = 0; j < VPL / 4; ++j) {
        float4 t = __ldg(reinterpret_cast<const float4*>(row + j * 128) + lane);
        v[4 * j] = t.x; v[4 * j + 1] = t.y; v[4 * j + 2] = t.z; v[4 * j + 3] = t.w;
      }
    }
  }
  __device__ __forceinline__ static void load_cg(const float* row, int lane, float (&v)[VPL]) {
    if constexpr (VPL == 2) {
      float2 t = __ldcg(reinterpret_cast<const float2*>(row) + lane);
      v[0] = t.x; v[1] = t.y;
    } else {
#pragma unroll
      for (int j = 0; j < VPL / 4; ++j) {
        float4 t = __ldcg(reinterpret_cast<const float4*>(row + j * 128) + lane);
        v[4 * j] = t.x; v[4 * j + 1] = t.y; v[4 * j + 2] = t.z; v[4 * j + 3] = t.w;
      }
    }
  }
  __device__ __forceinline__ static void load(const float* row, int lane, float (&v)[VPL]) {
    if constexpr (VPL == 2) {
      float2 t = reinterpret_cast<const float2*>(row)[lane];
      v[0] = t.x; v[1] = t.y;
    } else {
#pragma unroll
      for (int j = 0; j < VPL / 4; ++j) {
        float4 t = reinterpret_cast<const float4*>(row + j * 128)[lane];
        v[4 * j] = t.x; v[4 * j + 1] = t.y; v[4 * j + 2] = t.z; v[4 * j + 3] = t.w;
      }
    }
  }
  __device__ __forceinline__ static void store(float* row, int lane, const float (&v)[VPL]) {
    if constexpr (VPL == 2) {
      reinterpret_cast<float2*>(row)[lane] = make_float2(v[0], v[1]);
    } else {
#pragma unroll
      for (int j = 0; j < VPL / 4; ++j)
        reinterpret_cast<float4*>(row + j * 128)[lane] =
            make_float4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]);
    }
  }
  __device__ __forceinline__ static void store_cg(float* row, int lane, const float (&v)[VPL]) {
    if constexpr (VPL == 2) {
      __stcg(reinterpret_cast<float2*>(row) + lane, make_float2(v[0], v[1]));
    } else {
#pragma unroll
      for (int j = 0; j < VPL / 4; ++j)
        __stcg(reinterpret_cast<float4*>(row + j * 128) + lane,
               make_float4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]));
    }
  }
  // the lo half of the bf16x3 split (R14): bf16(v - bf16(v))
  __device__ __forceinline__ static void store_bf16_lo(bf16* row, int lane, const float (&v)[VPL]) {
    float r[VPL];
#pragma unroll
    for (int i = 0; i < VPL; ++i) r[i] = bf16_lo_of(v[i]);
    store_bf16(row, lane, r);
  }
  __device__ __forceinline__ static void store_bf16(bf16* row, int lane, const float (&v)[VPL]) {
    if constexpr (VPL == 2) {
      reinterpret_cast<__nv_bfloat162*>(row)[lane] = __floats2bfloat162_rn(v[0], v[1]);
    } else {
#pragma unroll
      for (int j = 0; j < VPL / 4; ++j) {
        __nv_bfloat162 a = __floats2bfloat162_rn(v[4 * j], v[4 * j + 1]);
        __nv_bfloat162 b = __floats2bfloat162_rn(v[4 * j + 2], v[4 * j + 3]);
        uint2 pk;
        pk.x = *reinterpret_cast<uint32_t*>(&a);
        pk.y = *reinterpret_cast<uint32_t*>(&b);
        reinterpret_cast<uint2*>(row + j * 128)[lane] = pk;
      }
    }
  }
};

// Batch view in shared memory: sboff[n + 1] entry offsets, then srbase[n] (8-byte
// aligned) = row_ptr[rows[r]], both written by K-0 (a).
__host__ __device__ __forceinline__ size_t view_smem(int n) {
  return (((size_t)(n + 1) * 4 + 7) & ~size_t(7)) + (size_t)n * 8;
}
__device__ __forceinline__ const int64_t* view_rbase(const int32_t* sboff, int n) {
  return reinterpret_cast<const int64_t*>(reinterpret_cast<const char*>(sboff) + (((size_t)(n + 1) * 4 + 7) & ~size_t(7)));
}

// map a flat batch entry e to its dataset index; returns row in *r
__device__ __forceinline__ int64_t entry_index(const int32_t* sboff, int n, int e, int* r) {
  int rr = entry_row(sboff, n, e);
  *r = rr;
  return view_rbase(sboff, n)[rr] + (e - sboff[rr]);
}

// -------------------------------------------------------------------------
// K-0 (a): the batch view, built in shared memory by every CTA of K-0 and K-1
// (no separate launch on the step's critical path): sboff[r] = flat offset of
// row r's entries (clamped to nz_cap), srb[r] = row_ptr[rows[r]].  With
// `publish` (CTA 0 of K-1) it also writes the global view for the later
// kernels: row ids (rowsc), label offsets, meta (nnz, labels, rows, lr, loss
// pointer) and the error bits.  Returns the batch nnz (clamped).
// -------------------------------------------------------------------------
constexpr int kViewPer = 8;   // rows per thread: n <= kViewPer * blockDim (b_max <= 2048, >= 256 threads)

// build_view's label counts, then (defer) the label offsets; (defer) nnz, labels, error bits
__shared__ int32_t s_llen[kViewPer * 256];
__shared__ long long s_vtot[3];

__device__ int build_view(const StepArgs& sa, const int64_t* __restrict__ row_ptr,
                          const int64_t* __restrict__ lab_ptr, int64_t n_data_rows, int64_t nz_cap,
                          int64_t nl_cap, int32_t* sboff, bool publish, const ViewOut& out, bool defer = false) {
  __shared__ long long wf[32], wl[32];
  __shared__ int s_bad;
  const int n = sa.n;
  int64_t* srb = const_cast<int64_t*>(view_rbase(sboff, n));
  const int t = threadIdx.x, lane = t & 31, wid = t >> 5, nw = blockDim.x >> 5;
  // loads spread over every thread (row r on thread r % blockDim: one rows[] -> row_ptr[]
  // round trip for the whole block); row lengths parked in sboff / s_llen for the scan
  if (t == 0) s_bad = 0;
  __syncthreads();
  for (int r = t; r < n; r += blockDim.x) {
    const int64_t id = sa.rows[r];
    int32_t ln = 0, ll = 0;
    if (id < 0 || id >= n_data_rows) {
      s_bad = 1;
      srb[r] = 0;
    } else {
      const int64_t a = row_ptr[id];
      ln = (int32_t)(row_ptr[id + 1] - a);
      srb[r] = a;
      if (publish) {
        ll = (int32_t)(lab_ptr[id + 1] - lab_ptr[id]);
        if (!defer) {
          out.rowsc[r] = (int32_t)id;
          out.rbase[r] = a;
        }
      }
    }
    sboff[r] = ln;
    if (publish) s_llen[r] = ll;
  }
  __syncthreads();
  const int bad = s_bad;
  const int r0 = t * kViewPer;
  int64_t len[kViewPer], llen[kViewPer];
  long long sf = 0, sl = 0;
#pragma unroll
  for (int i = 0; i < kViewPer; ++i) {
    const int r = r0 + i;
    len[i] = r < n ? sboff[r] : 0;
    llen[i] = (publish && r < n) ? s_llen[r] : 0;
    sf += len[i];
    sl += llen[i];
  }
  long long xf = sf, xl = sl;   // inclusive warp scan
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const long long yf = __shfl_up_sync(kFull, xf, o), yl = __shfl_up_sync(kFull, xl, o);
    if (lane >= o) { xf += yf; xl += yl; }
  }
  if (lane == 31) { wf[wid] = xf; wl[wid] = xl; }
  __syncthreads();
  if (wid == 0) {
    long long a = lane < nw ? wf[lane] : 0, c = lane < nw ? wl[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const long long ya = __shfl_up_sync(kFull, a, o), yc = __shfl_up_sync(kFull, c, o);
      if (lane >= o) { a += ya; c += yc; }
    }
    wf[lane] = a; wl[lane] = c;
  }
  __syncthreads();
  long long pf = xf - sf + (wid ? wf[wid - 1] : 0), pl = xl - sl + (wid ? wl[wid - 1] : 0);
#pragma unroll
  for (int i = 0; i < kViewPer; ++i) {
    const int r = r0 + i;
    if (r < n) {
      sboff[r] = (int32_t)min(pf, (long long)nz_cap);
      if (publish) {
        if (defer) {
          s_llen[r] = (int32_t)min(pl, (long long)nl_cap);   // this thread's own rows: read above
        } else {
          out.boff[r] = (int32_t)min(pf, (long long)nz_cap);
          out.loff[r] = (int32_t)min(pl, (long long)nl_cap);
        }
      }
      pf += len[i];
      pl += llen[i];
    }
  }
  long long tf = wf[nw - 1], tl = wl[nw - 1];
  if (t == 0) sboff[n] = (int32_t)min(tf, (long long)nz_cap);
  if (publish && defer) {
    if (t == 0) {
      int err = bad ? ERR_ROW_ID : 0;
      if (tf > nz_cap) err |= ERR_NNZ_CAP;
      if (tl > nl_cap) err |= ERR_LAB_CAP;
      s_vtot[0] = min(tf, (long long)nz_cap);
      s_vtot[1] = min(tl, (long long)nl_cap);
      s_vtot[2] = err;
    }
  } else if (publish) {
    if (bad && t == 0) atomicOr(&out.meta[M_ERR], ERR_ROW_ID);
    if (t == 0) {
      int err = 0;
      if (tf > nz_cap) { err |= ERR_NNZ_CAP; tf = nz_cap; }
      if (tl > nl_cap) { err |= ERR_LAB_CAP; tl = nl_cap; }
      out.boff[n] = (int32_t)tf;
      out.loff[n] = (int32_t)tl;
      out.meta[M_NNZ] = (int32_t)tf;
      out.meta[M_NLAB] = (int32_t)tl;
      out.meta[M_NROWS] = n;
      out.meta[M_LR] = __float_as_int(sa.lr);
      *reinterpret_cast<float**>(out.meta + M_LOSS) = sa.loss;
      if (err) atomicOr(&out.meta[M_ERR], err);
    }
  }
  __syncthreads();
  return (int)min(tf, (long long)nz_cap);
}

// The deferred publication of build_view(..., defer = true) (K-1's CTA 0, after its
// griddepcontrol.wait: the previous step's kernels may still read the published view
// while K-1 builds its own in shared memory).
__device__ void publish_view(const StepArgs& sa, int64_t n_data_rows, const int32_t* sboff, const ViewOut& out) {
  const int n = sa.n;
  const int64_t* srb = view_rbase(sboff, n);
  for (int r = threadIdx.x; r < n; r += blockDim.x) {
    const int64_t id = sa.rows[r];
    if (id >= 0 && id < n_data_rows) {
      out.rowsc[r] = (int32_t)id;
      out.rbase[r] = srb[r];
    }
    out.boff[r] = sboff[r];
    out.loff[r] = s_llen[r];
  }
  if (threadIdx.x == 0) {
    const int tf = (int)s_vtot[0], tl = (int)s_vtot[1], err = (int)s_vtot[2];
    out.boff[n] = tf;
    out.loff[n] = tl;
    out.meta[M_NNZ] = tf;
    out.meta[M_NLAB] = tl;
    out.meta[M_NROWS] = n;
    out.meta[M_LR] = __float_as_int(sa.lr);
    *reinterpret_cast<float**>(out.meta + M_LOSS) = sa.loss;
    if (err) atomicOr(&out.meta[M_ERR], err);
  }
}

// -------------------------------------------------------------------------
// K-0 (b-e) fused: one persistent kernel of co-operating CTAs (one per SM at
// most) with two software grid barriers (the only other work on the GPU is the
// dense chain on other streams, which never waits for this kernel, so every CTA
// eventually runs).  Phases:
//   A  per batch entry (row r, feature f): cnt[f] += 1 and the row bitmap
//      bits[f][r / 32] |= 1 << r % 32; per-tile (count, touched) histograms in
//      shared memory, flushed to tsum[par] once per CTA
//   C  tile prefix + in-tile scan: segment starts fseg, ranks fuid, sorted
//      unique ids uniq, segment offsets useg; tsum[par ^ 1] zeroed for the next step
//   E  deterministic placement: the entry of row r in feature f's segment goes
//      to fseg[f] + #{rows r' < r of the batch containing f} (popcounts of
//      bits[f]), so every segment is sorted by row without a sort
// cnt[f] and bits[f][*] go back to zero in K-5, which finishes each segment.
// -------------------------------------------------------------------------
// 64 CTAs: enough entries in flight, while leaving the register file of most
// SMs to K-1, which runs beside K-0 (measured: 148 CTAs slow K-1 by ~3 us).
constexpr int kTouchCtas = 64;
constexpr int kK0OneCta = 0;   // folded K-0: feature tiles up to which CTA 0 alone scans (measured slower
                               // at EURLex's 5 tiles: 63.5 vs 58.5 us per step; kept at 0)

__device__ __forceinline__ void grid_barrier(unsigned long long* ctr) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned long long arrive = atomicAdd(ctr, 1ull) + 1ull;
    const unsigned long long goal = (arrive + gridDim.x - 1) / gridDim.x * gridDim.x;
    volatile unsigned long long* vc = ctr;
    while (*vc < goal) __nanosleep(32);
    __threadfence();
  }
  __syncthreads();
}

// FOLD (k0_fold()): phase A ran inside K-1 (counts, row bitmaps and tile sums as K-1 reads
// the entries); this kernel starts at phase C from the batch view K-1 published (gboff,
// grbase) and runs after K-1 on the side stream.
template <int NT, bool FOLD>   // threads per CTA: 128, 256 or 512 (the batch view needs 8 NT >= n)
__global__ void __launch_bounds__(NT) k_touched(StepArgs sa, const int64_t* __restrict__ row_ptr,
                                                 int64_t n_data_rows, int64_t nz_cap,
                                                 const int32_t* __restrict__ col,
                                                 const float* __restrict__ val, int32_t* meta,
                                                 int32_t* cnt, int32_t* tsum, int64_t F, int ntiles,
                                                 int32_t* fseg, int32_t* fuid, int32_t* uniq,
                                                 int32_t* useg, uint32_t* bits, int W, int32_t* e_n,
                                                 float* e_v, int32_t* e_u, int32_t* e_f,
                                                 const int32_t* __restrict__ gboff,
                                                 const int64_t* __restrict__ grbase) {
  Tl tl_(TL_TOUCHED);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  extern __shared__ int32_t sboff[];
  __shared__ int s_red[2][16];
  __shared__ int s_pre[2];
  unsigned long long* bar = reinterpret_cast<unsigned long long*>(meta + M_BAR);
  const int par = meta[M_K0PAR] & 1;
  int32_t* ts = tsum + (size_t)par * 2 * ntiles;          // this step's tile (count, touched) sums
  int32_t* ts_next = tsum + (size_t)(par ^ 1) * 2 * ntiles;
  const int n = sa.n;
  int32_t* hist = sboff + ((view_smem(n) + 3) / 4);       // [ntiles][2] after the batch view
  const int gt = blockIdx.x * blockDim.x + threadIdx.x, gs = gridDim.x * blockDim.x;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  int nnz;
  if constexpr (FOLD) {
    // the view K-1 published: entry offsets and row bases
    int64_t* srb = const_cast<int64_t*>(view_rbase(sboff, n));
    for (int r = threadIdx.x; r <= n; r += blockDim.x) {
      sboff[r] = gboff[r];
      if (r < n) srb[r] = grbase[r];
    }
    __syncthreads();
    nnz = sboff[n];
    if (threadIdx.x == 0) TL_MARK(TL_PH0);   // K-0 (fold): view copied
    // ---- C0: this step's tile sums (count, touched features) from the counts K-1 left.
    // Few tiles (F <= kK0OneCta tiles, EURLex-4K: 5): CTA 0 runs C0 and C alone, the other
    // CTAs go straight to the barrier before E (one grid barrier instead of two)
    const bool one = ntiles <= kK0OneCta;
    for (int t = one ? (blockIdx.x == 0 ? 0 : ntiles) : blockIdx.x; t < ntiles; t += one ? 1 : gridDim.x) {
      int a = 0, b = 0;
      for (int64_t f = (int64_t)t * kScanTile + threadIdx.x; f < min((int64_t)(t + 1) * kScanTile, F); f += blockDim.x) {
        const int c = cnt[f];
        a += c;
        b += c > 0;
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) { a += __shfl_xor_sync(kFull, a, o); b += __shfl_xor_sync(kFull, b, o); }
      if (lane == 0) { s_red[0][wid] = a; s_red[1][wid] = b; }
      __syncthreads();
      if (threadIdx.x == 0) {
        int x = 0, y = 0;
        for (int w = 0; w < nw; ++w) { x += s_red[0][w]; y += s_red[1][w]; }
        ts[2 * t] = x;
        ts[2 * t + 1] = y;
      }
      __syncthreads();
    }
    if (!one) grid_barrier(bar);
    if (threadIdx.x == 0) TL_MARK(TL_PH1);   // K-0 (fold): C0 done, barrier 1 passed
  } else {
    for (int i = threadIdx.x; i < 2 * ntiles; i += blockDim.x) hist[i] = 0;
    nnz = build_view(sa, row_ptr, nullptr, n_data_rows, nz_cap, 0, sboff, false, ViewOut{});
    // ---- A
    for (int e = gt; e < nnz; e += gs) {
      int r;
      const int f = col[entry_index(sboff, n, e, &r)];
      const int old = atomicAdd(&cnt[f], 1);
      atomicOr(&bits[(int64_t)f * W + (r >> 5)], 1u << (r & 31));
      const int t = f / kScanTile;
      atomicAdd(&hist[2 * t], 1);
      if (old == 0) atomicAdd(&hist[2 * t + 1], 1);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 2 * ntiles; i += blockDim.x)
      if (hist[i]) atomicAdd(&ts[i], hist[i]);
    grid_barrier(bar);
  }
  // ---- C: prefix of the earlier tiles + in-tile scan
  constexpr int PER = kScanTile / NT;
  const bool one_cta = FOLD && ntiles <= kK0OneCta;   // CTA 0 scans every tile (after its own C0)
  for (int t = one_cta ? (blockIdx.x == 0 ? 0 : ntiles) : blockIdx.x; t < ntiles; t += one_cta ? 1 : gridDim.x) {
    int a = 0, b = 0;
    for (int j = threadIdx.x; j < t; j += blockDim.x) { a += ts[2 * j]; b += ts[2 * j + 1]; }
#pragma unroll
    for (int o = 16; o; o >>= 1) { a += __shfl_xor_sync(kFull, a, o); b += __shfl_xor_sync(kFull, b, o); }
    if (lane == 0) { s_red[0][wid] = a; s_red[1][wid] = b; }
    __syncthreads();
    if (threadIdx.x == 0) {
      int x = 0, y = 0;
      for (int w = 0; w < nw; ++w) { x += s_red[0][w]; y += s_red[1][w]; }
      s_pre[0] = x; s_pre[1] = y;
      if (t == ntiles - 1) {
        meta[M_U] = y + ts[2 * t + 1];
        useg[y + ts[2 * t + 1]] = x + ts[2 * t];
      }
      ts_next[2 * t] = 0;
      ts_next[2 * t + 1] = 0;
    }
    __syncthreads();
    const int64_t f0 = (int64_t)t * kScanTile + threadIdx.x * PER;
    int c[PER];
    int ta = 0, tb = 0;
#pragma unroll
    for (int i = 0; i < PER; ++i) {
      c[i] = (f0 + i < F) ? cnt[f0 + i] : 0;
      ta += c[i]; tb += (c[i] > 0);
    }
    // block exclusive scan of (ta, tb)
    int xa = ta, xb = tb;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int ya = __shfl_up_sync(kFull, xa, o), yb = __shfl_up_sync(kFull, xb, o);
      if (lane >= o) { xa += ya; xb += yb; }
    }
    __syncthreads();
    if (lane == 31) { s_red[0][wid] = xa; s_red[1][wid] = xb; }
    __syncthreads();
    int oa = 0, ob = 0;
    for (int w = 0; w < wid; ++w) { oa += s_red[0][w]; ob += s_red[1][w]; }
    int pa = s_pre[0] + oa + xa - ta, pb = s_pre[1] + ob + xb - tb;
#pragma unroll
    for (int i = 0; i < PER; ++i) {
      if (c[i] > 0) {
        fseg[f0 + i] = pa;
        fuid[f0 + i] = pb;
        uniq[pb] = (int32_t)(f0 + i);
        useg[pb] = pa;
        ++pb;
      }
      pa += c[i];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) TL_MARK(TL_PH2);   // K-0: C done
  grid_barrier(bar);
  if (threadIdx.x == 0) TL_MARK(TL_PH3);   // K-0: C done, barrier 2 passed
  // ---- E: placement, kE entries per thread at a time (their dependent loads overlap)
  constexpr int kE = 4;
  for (int e0 = gt; e0 < nnz; e0 += kE * gs) {
    int r[kE], f[kE], seg[kE], uid[kE], rank[kE];
    int64_t k[kE];
    float v[kE];
#pragma unroll
    for (int i = 0; i < kE; ++i) {
      const int e = e0 + i * gs;
      k[i] = e < nnz ? entry_index(sboff, n, e, &r[i]) : -1;
      f[i] = k[i] >= 0 ? col[k[i]] : 0;
      v[i] = k[i] >= 0 ? val[k[i]] : 0.f;
    }
#pragma unroll
    for (int i = 0; i < kE; ++i) {
      rank[i] = 0;
      seg[i] = 0;
      uid[i] = 0;
      if (k[i] >= 0) {
        const uint32_t* bw = bits + (int64_t)f[i] * W;
        const int wr = r[i] >> 5;
        rank[i] = __popc(bw[wr] & ((1u << (r[i] & 31)) - 1u));
        // the bitmap words below row r's word: loaded 8 at a time (independent loads in
        // flight together, one round for b_max <= 256) instead of one after another
        for (int w0 = 0; w0 < wr; w0 += 8) {
          uint32_t wv[8];
#pragma unroll
          for (int w = 0; w < 8; ++w) wv[w] = w0 + w < wr ? bw[w0 + w] : 0u;
#pragma unroll
          for (int w = 0; w < 8; ++w) rank[i] += __popc(wv[w]);
        }
        seg[i] = fseg[f[i]];
        uid[i] = fuid[f[i]];
      }
    }
#pragma unroll
    for (int i = 0; i < kE; ++i) {
      if (k[i] < 0) continue;
      const int pos = seg[i] + rank[i];
      e_n[pos] = r[i];
      e_v[pos] = v[i];
      e_u[pos] = uid[i];
      e_f[pos] = f[i];
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) meta[M_K0PAR] = par ^ 1;   // every CTA read par before barrier 1
}

// -------------------------------------------------------------------------
// K-1: A1 = X W1 + b1, H1 = ReLU(A1)
// -------------------------------------------------------------------------
#ifndef ASGD_K1_GROUP
// warps per K-1 CTA = the largest group.  Round 1 (fixed 16-piece groups, 117 of 148 CTAs busy
// at EURLex): 8 / 16 -> 3.64 / 4.02 M samples/s.  Round 2, groups sized to the batch (gs):
// 8 / 16 -> 4.14 / 4.05 M (8-warp CTAs, two per SM, 235 groups of 8 pieces)
#define ASGD_K1_GROUP 8
#endif
template <int VPL>   // pieces per group = warps per K-1 CTA (H = 512: 8, the partials fill 32 KB)
constexpr int k1_group() { return VPL >= 16 ? 8 : ASGD_K1_GROUP; }
// TMA-staged K-1 (k1_tma()): every W1 row of a warp's piece is requested at once as one
// bulk async copy per entry into the warp's 32-row shared-memory slot array, completed on
// the warp's mbarrier; the FMAs then read shared memory.  fp32 rows of H floats: 5 warps
// x 32 KB at H = 256 (one CTA per SM; with the static view and partials ~207 KB), 8 warps below.
template <int VPL>
constexpr int k1_group_tma() { return VPL >= 8 ? 5 : 8; }
template <int VPL, bool TMA>
constexpr int k1_warps() { return TMA ? k1_group_tma<VPL>() : k1_group<VPL>(); }
template <int VPL, bool TMA>
constexpr int k1_min_ctas() { return TMA ? (VPL >= 8 ? 1 : 2) : 16 / k1_group<VPL>(); }
// dynamic shared memory of K-1: the batch view of up to b_max = 2048 rows, then (TMA) the
// row slots, 128-B aligned
constexpr size_t k1_view_bytes() { return (view_smem(2048) + 127) & ~size_t(127); }
template <int VPL, bool TMA>
constexpr size_t k1_smem() { return k1_view_bytes() + (TMA ? (size_t)k1_warps<VPL, TMA>() * kPiece * VPL * 128 : 0); }

template <int VPL, bool TMA>
// (256, 2): two CTAs per SM, all kU gathers of a group in flight (<= 128 regs)
__global__ void __launch_bounds__(32 * k1_warps<VPL, TMA>(), (k1_min_ctas<VPL, TMA>())) k_spmm_fwd(StepArgs sa, const int64_t* __restrict__ row_ptr,
                                                  const int64_t* __restrict__ lab_ptr, int64_t n_data_rows,
                                                  int64_t nz_cap, int64_t nl_cap, ViewOut vo,
                                                  const int32_t* __restrict__ col,
                                                  const float* __restrict__ val,
                                                  const float* __restrict__ W1,
                                                  const float* __restrict__ b1, float* H1,
                                                  bf16* H1b, bf16* H1l, float* part, int32_t* rowcnt,
                                                  int32_t* kcnt, uint32_t* kbits, int W, int32_t* tsum,
                                                  int ntiles) {
  Tl tl_(TL_SPMM);
  pdl_trigger();
  using IO = RowIO<VPL>;
  constexpr int H = 32 * VPL;
  constexpr int kU = VPL >= 16 ? 4 : 8;   // W1 rows in flight per warp
  extern __shared__ int32_t sboff[];
  const int n = sa.n;
  // The batch view reads only the step's rows and the dataset, which no kernel writes: it is
  // built before griddepcontrol.wait, so under programmatic dependent launch (a step group's
  // graph) it overlaps the previous step's tail; CTA 0 publishes it after the wait.
  const int nnz = build_view(sa, row_ptr, lab_ptr, n_data_rows, nz_cap, nl_cap, sboff, blockIdx.x == 0, vo, true);
  pdl_wait();
  tl_.ready();
  if (blockIdx.x == 0) publish_view(sa, n_data_rows, sboff, vo);
  const int64_t* srb = view_rbase(sboff, n);
  const int lane = threadIdx.x & 31;
  const int npieces = (nnz + kPiece - 1) / kPiece;
  const int nwarps = gridDim.x * (blockDim.x >> 5);
  // K-0 phase A folded in (ntiles > 0, k0_fold()): per entry cnt[f] += 1 and the row bitmap
  // bit, as reductions; K-0 derives the tile sums from the counts

  // Pieces are taken in groups of 8 consecutive pieces, one per warp of the CTA, so a
  // row that crosses pieces is first combined inside the CTA through shared memory;
  // only rows that cross a group boundary go through global partials, one per group.
  constexpr int kGroup = k1_warps<VPL, TMA>();   // pieces per group = warps per CTA
  __shared__ __align__(16) float spart[kGroup][2][H];   // per warp: [0] its first segment, [1] its last
  const int warp = threadIdx.x >> 5;
  // TMA: this warp's kPiece row slots and its mbarrier (one phase per piece)
  float* slots = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(sboff) + k1_view_bytes()) +
                 (size_t)warp * kPiece * H;
  __shared__ __align__(8) uint64_t sbar[kGroup];
  const uint32_t bar = static_cast<uint32_t>(__cvta_generic_to_shared(&sbar[warp]));
  uint32_t phase = 0;
  if constexpr (TMA) {
    if (lane == 0) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar) : "memory");
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
  }
  // pieces per group: up to one per warp, fewer when the batch has fewer than kGroup
  // pieces per CTA, so every CTA of the grid gets a group (EURLex: 1,875 pieces -> 13 per
  // group on 145 CTAs instead of 16 on 117); the idle warps only join the barriers
  const int gs = max(1, min(kGroup, (npieces + (int)gridDim.x - 1) / (int)gridDim.x));
  const int ngroups = (npieces + gs - 1) / gs;
  auto finish = [&](int r, float (&acc)[VPL]) {
    float bias[VPL];   // b1 re-read (L1) instead of held in registers across the gathers
    IO::load_ldg(b1, lane, bias);
#pragma unroll
    for (int i = 0; i < VPL; ++i) acc[i] = fmaxf(acc[i] + bias[i], 0.f);
    IO::store(H1 + (int64_t)r * H, lane, acc);
    if (H1b) IO::store_bf16(H1b + (int64_t)r * H, lane, acc);
    if (H1l) IO::store_bf16_lo(H1l + (int64_t)r * H, lane, acc);
  };
  // group g's partial of row r (global): slot 2 g + 1 if r starts in g, else 2 g; the
  // last group to arrive sums the row's group partials in group order and finishes
  auto publish = [&](int g, int r, float (&acc)[VPL]) {
    const int GE = gs * kPiece;                  // entries per group
    const int rs = sboff[r], re = sboff[r + 1];
    const int g0 = rs / GE, g1 = (re - 1) / GE;
    IO::store_cg(part + (int64_t)(g == g0 ? 2 * g + 1 : 2 * g) * H, lane, acc);
    fence_mp();
    int old = 0;
    if (lane == 0) old = atomicAdd(&rowcnt[r], 1);
    old = __shfl_sync(kFull, old, 0);
    if (old != g1 - g0) return;
    fence_mp();
#pragma unroll
    for (int i = 0; i < VPL; ++i) acc[i] = 0.f;
    for (int q = g0; q <= g1; q += 4) {   // 4 partials in flight, summed in group order
      float t[4][VPL];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        if (q + u <= g1) IO::load_cg(part + (int64_t)(q + u == g0 ? 2 * g0 + 1 : 2 * (q + u)) * H, lane, t[u]);
        else {
#pragma unroll
          for (int i = 0; i < VPL; ++i) t[u][i] = 0.f;
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        if (q + u <= g1) {
#pragma unroll
          for (int i = 0; i < VPL; ++i) acc[i] += t[u][i];
        }
      }
    }
    if (lane == 0) rowcnt[r] = 0;
    finish(r, acc);
  };

  for (int g = blockIdx.x; g < ngroups; g += gridDim.x) {
    const int p = g * gs + warp;
    const int G0 = g * gs * kPiece, G1 = min(G0 + gs * kPiece, nnz);
    const int e0 = warp < gs ? p * kPiece : nnz;   // idle warps (warp >= gs): an empty piece
    const int e1 = min(e0 + kPiece, nnz), cnt = max(0, e1 - e0);
    // Row segment of row r ends inside this piece: finish it (ReLU(acc + b1)) when the
    // piece holds the whole row, else park it in shared memory for the group combine
    auto flush = [&](int r, float (&acc)[VPL]) {
      const int rs = sboff[r], re = sboff[r + 1];
      const bool before = rs < e0, after = re > e1;
      if (!before && !after) { finish(r, acc); return; }
      IO::store(&spart[warp][before ? 0 : 1][0], lane, acc);
    };
    int rfirst = -1, rlast = -1;   // rows of this piece's first / last entry
    if (cnt > 0) {
      // lane j holds entry e0 + j: its row, column and value (one round trip)
      int myr = 0, mycol = 0;
      float myval = 0.f;
      if (lane < cnt) {
        myr = entry_row(sboff, n, e0 + lane);
        const int64_t k = srb[myr] + (e0 + lane - sboff[myr]);
        mycol = __ldg(col + k);
        myval = __ldg(val + k);
      }
      if (ntiles && lane < cnt) {   // folded phase A: fire-and-forget reductions
        atomicAdd(&kcnt[mycol], 1);
        atomicOr(&kbits[(int64_t)mycol * W + (myr >> 5)], 1u << (myr & 31));
      }
      int rcur = __shfl_sync(kFull, myr, 0);
      rfirst = rcur;
      rlast = __shfl_sync(kFull, myr, cnt - 1);
      float acc[VPL];
#pragma unroll
      for (int i = 0; i < VPL; ++i) acc[i] = 0.f;
      if constexpr (TMA) {
        // every row of the piece in flight at once: one bulk copy per entry into slot j
        if (lane == 0)
          asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar),
                       "r"((uint32_t)(cnt * H * 4))
                       : "memory");
        __syncwarp();
        if (lane < cnt)
          asm volatile(
              "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                  static_cast<uint32_t>(__cvta_generic_to_shared(slots + (size_t)lane * H))),
              "l"(W1 + (int64_t)mycol * H), "r"((uint32_t)(H * 4)), "r"(bar)
              : "memory");
        uint32_t ok = 0;
        while (!ok)
          asm volatile(
              "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
              : "=r"(ok)
              : "r"(bar), "r"(phase)
              : "memory");
        phase ^= 1u;
        for (int j = 0; j < cnt; ++j) {
          float w[VPL];
          IO::load(slots + (size_t)j * H, lane, w);
          const int rq = __shfl_sync(kFull, myr, j);
          const float v = __shfl_sync(kFull, myval, j);
          if (rq != rcur) {
            flush(rcur, acc);
#pragma unroll
            for (int i = 0; i < VPL; ++i) acc[i] = 0.f;
            rcur = rq;
          }
#pragma unroll
          for (int i = 0; i < VPL; ++i) acc[i] = fmaf(v, w[i], acc[i]);
        }
        __syncwarp();   // every lane has read the slots before the next piece's copies land
      } else {
      // groups of kU W1 rows in flight, row changes handled between FMAs
        for (int j0 = 0; j0 < cnt; j0 += kU) {
          float w[kU][VPL];
  #pragma unroll
          for (int q = 0; q < kU; ++q) {
            const int c = __shfl_sync(kFull, mycol, j0 + q);
            if (j0 + q < cnt) IO::load_ldg(W1 + (int64_t)c * H, lane, w[q]);
            else {
  #pragma unroll
              for (int i = 0; i < VPL; ++i) w[q][i] = 0.f;
            }
          }
  #pragma unroll
          for (int q = 0; q < kU; ++q) {
            const int j = j0 + q;
            const int rq = __shfl_sync(kFull, myr, j);
            const float v = __shfl_sync(kFull, myval, j);
            if (j < cnt) {
              if (rq != rcur) {
                flush(rcur, acc);
  #pragma unroll
                for (int i = 0; i < VPL; ++i) acc[i] = 0.f;
                rcur = rq;
              }
  #pragma unroll
              for (int i = 0; i < VPL; ++i) acc[i] = fmaf(v, w[q][i], acc[i]);
            }
          }
        }
      }
      flush(rcur, acc);
    }
    __syncthreads();
    // group combine: warp w takes the rows whose first segment inside the group is in
    // its piece and that continue past it (or reach back before the group, warp 0),
    // sums the parked segments of the following warps in warp order, then finishes
    // the row or publishes the group's partial
    if (cnt > 0) {
      for (int k = 0; k < 2; ++k) {
        if (k == 1 && rlast == rfirst) break;
        const int r = k == 0 ? rfirst : rlast;
        const int rs = sboff[r], re = sboff[r + 1];
        const bool before = rs < e0, after = re > e1;
        if (!before && !after) continue;        // finished in flush
        if (max(rs, G0) < e0) continue;          // an earlier warp of the group holds its first segment
        float acc[VPL];
        IO::load(&spart[warp][before ? 0 : 1][0], lane, acc);
        for (int w2 = warp + 1; w2 < gs && (g * gs + w2) * kPiece < min(re, G1); ++w2) {
          float t[VPL];
          IO::load(&spart[w2][0][0], lane, t);   // row r is w2's first segment
#pragma unroll
          for (int i = 0; i < VPL; ++i) acc[i] += t[i];
        }
        if (rs >= G0 && re <= G1) finish(r, acc);
        else publish(g, r, acc);
      }
    }
    if (g + (int)gridDim.x < ngroups) __syncthreads();   // spart is reused by this CTA's next group
  }
  // rows without entries: H1 = ReLU(b1)
  const int gw = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  for (int r = gw; r < n; r += nwarps) {
    if (sboff[r + 1] == sboff[r]) {
      float acc[VPL];
#pragma unroll
      for (int i = 0; i < VPL; ++i) acc[i] = 0.f;
      finish(r, acc);
    }
  }
}

// K-0's per-feature count and row bitmap back to zero (the warp that finishes
// feature f's segment; K-0 of the next step starts from zeros).
__device__ __forceinline__ void reset_feature(int32_t* cnt, uint32_t* bits, int W, int f, int lane) {
  if (lane == 0) cnt[f] = 0;
  for (int w = lane; w < W; w += 32) bits[(int64_t)f * W + w] = 0u;
}

// -------------------------------------------------------------------------
// K-5: W1[f,:] -= lr * sum_{entries of f, ascending row} v * dA1[row,:]
// -------------------------------------------------------------------------
template <int VPL>
__global__ void __launch_bounds__(256) k_scatter_sgd(const int32_t* __restrict__ e_n,
                                                     const float* __restrict__ e_v,
                                                     const int32_t* __restrict__ e_u,
                                                     const int32_t* __restrict__ useg,
                                                     const int32_t* __restrict__ uniq,
                                                     const int32_t* __restrict__ meta,
                                                     const float* __restrict__ dA1, float* W1,
                                                     float* part, int32_t* ucnt,
                                                     float* grad_w1, int32_t* cnt, uint32_t* bits, int W) {
  Tl tl_(TL_SCATTER);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const float lr = step_lr(meta);
  using IO = RowIO<VPL>;
  constexpr int H = 32 * VPL;
  constexpr int kU = VPL >= 16 ? 4 : 8;   // dA1 rows in flight per warp
  const int lane = threadIdx.x & 31;
  const int nnz = meta[M_NNZ];
  const int npieces = (nnz + kPiece - 1) / kPiece;
  const int nwarps = gridDim.x * (blockDim.x >> 5);
  for (int p = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); p < npieces; p += nwarps) {
    const int e0 = p * kPiece, e1 = min(e0 + kPiece, nnz);
    int myn = 0;
    float myv = 0.f;
    if (e0 + lane < e1) { myn = e_n[e0 + lane]; myv = e_v[e0 + lane]; }
    int u = e_u[e0];
    int e = e0;
    while (e < e1) {
      const int ss = useg[u], se_ = useg[u + 1];
      const int se = min(se_, e1);
      float acc[VPL];
#pragma unroll
      for (int i = 0; i < VPL; ++i) acc[i] = 0.f;
      int j = e - e0;
      const int jend = se - e0;
      for (; j + kU <= jend; j += kU) {
        float g[kU][VPL];
#pragma unroll
        for (int q = 0; q < kU; ++q) {
          int r = __shfl_sync(kFull, myn, j + q);
          IO::load_ldg(dA1 + (int64_t)r * H, lane, g[q]);
        }
#pragma unroll
        for (int q = 0; q < kU; ++q) {
          float v = __shfl_sync(kFull, myv, j + q);
#pragma unroll
          for (int i = 0; i < VPL; ++i) acc[i] = fmaf(v, g[q][i], acc[i]);
        }
      }
      for (; j < jend; ++j) {
        int r = __shfl_sync(kFull, myn, j);
        float v = __shfl_sync(kFull, myv, j);
        float g[VPL];
        IO::load_ldg(dA1 + (int64_t)r * H, lane, g);
#pragma unroll
        for (int i = 0; i < VPL; ++i) acc[i] = fmaf(v, g[i], acc[i]);
      }
      const bool before = ss < e0, after = se_ > e1;
      bool finish = !before && !after;
      if (!finish) {
        const int slot = before ? 2 * p : 2 * p + 1;
        IO::store_cg(part + (int64_t)slot * H, lane, acc);
        fence_mp();
        int old = 0;
        if (lane == 0) old = atomicAdd(&ucnt[u], 1);
        old = __shfl_sync(kFull, old, 0);
        const int q0 = ss / kPiece, q1 = (se_ - 1) / kPiece;
        if (old == q1 - q0) {
          fence_mp();
#pragma unroll
          for (int i = 0; i < VPL; ++i) acc[i] = 0.f;
          for (int q = q0; q <= q1; ++q) {
            float t[VPL];
            IO::load_cg(part + (int64_t)(q == q0 ? 2 * q + 1 : 2 * q) * H, lane, t);
#pragma unroll
            for (int i = 0; i < VPL; ++i) acc[i] += t[i];
          }
          if (lane == 0) ucnt[u] = 0;
          finish = true;
        }
      }
      if (finish) {
        const int64_t f = uniq[u];
        float w[VPL];
        IO::load(W1 + f * H, lane, w);
#pragma unroll
        for (int i = 0; i < VPL; ++i) w[i] = w[i] - lr * acc[i];
        IO::store(W1 + f * H, lane, w);
        if (grad_w1) IO::store(grad_w1 + f * H, lane, acc);
        reset_feature(cnt, bits, W, (int)f, lane);
      }
      e = se;
      ++u;
    }
  }
}

// K-5 with the batch's dA1 column slice staged in shared memory (one CTA per SM,
// grid.y = column slice).  Gathers become shared-memory reads; per piece only the
// entry list, the segment bounds and the touched W1 row go to L2/HBM.  Same
// pieces, combine order and results as k_scatter_sgd (bitwise, for T = float).
template <typename T, int CPL>
struct SliceIO {
  // lane's CPL contiguous columns of a staged row -> fp32
  __device__ __forceinline__ static void load(const T* row, int lane, float (&v)[CPL]) {
    if constexpr (sizeof(T) == 2) {
      if constexpr (CPL == 8) {
        uint4 q = reinterpret_cast<const uint4*>(row)[lane];
        const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&q);
#pragma unroll
        for (int i = 0; i < 4; ++i) { float2 f = __bfloat1622float2(h[i]); v[2 * i] = f.x; v[2 * i + 1] = f.y; }
      } else if constexpr (CPL == 4) {
        uint2 q = reinterpret_cast<const uint2*>(row)[lane];
        const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&q);
#pragma unroll
        for (int i = 0; i < 2; ++i) { float2 f = __bfloat1622float2(h[i]); v[2 * i] = f.x; v[2 * i + 1] = f.y; }
      } else {
        float2 f = __bfloat1622float2(reinterpret_cast<const __nv_bfloat162*>(row)[lane]);
        v[0] = f.x; v[1] = f.y;
      }
    } else {
      if constexpr (CPL >= 4) {
#pragma unroll
        for (int i = 0; i < CPL / 4; ++i) {
          float4 f = reinterpret_cast<const float4*>(row)[lane * (CPL / 4) + i];
          v[4 * i] = f.x; v[4 * i + 1] = f.y; v[4 * i + 2] = f.z; v[4 * i + 3] = f.w;
        }
      } else {
        float2 f = reinterpret_cast<const float2*>(row)[lane];
        v[0] = f.x; v[1] = f.y;
      }
    }
  }
};

template <int CPL>
__device__ __forceinline__ void ld_cols(const float* p, float (&v)[CPL], bool cg) {
#pragma unroll
  for (int i = 0; i < CPL; i += (CPL >= 4 ? 4 : 2)) {
    if constexpr (CPL >= 4) {
      float4 f = cg ? __ldcg(reinterpret_cast<const float4*>(p + i)) : *reinterpret_cast<const float4*>(p + i);
      v[i] = f.x; v[i + 1] = f.y; v[i + 2] = f.z; v[i + 3] = f.w;
    } else {
      float2 f = cg ? __ldcg(reinterpret_cast<const float2*>(p + i)) : *reinterpret_cast<const float2*>(p + i);
      v[i] = f.x; v[i + 1] = f.y;
    }
  }
}
template <int CPL>
__device__ __forceinline__ void st_cols(float* p, const float (&v)[CPL], bool cg) {
#pragma unroll
  for (int i = 0; i < CPL; i += (CPL >= 4 ? 4 : 2)) {
    if constexpr (CPL >= 4) {
      const float4 f = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
      if (cg) __stcg(reinterpret_cast<float4*>(p + i), f); else *reinterpret_cast<float4*>(p + i) = f;
    } else {
      const float2 f = make_float2(v[i], v[i + 1]);
      if (cg) __stcg(reinterpret_cast<float2*>(p + i), f); else *reinterpret_cast<float2*>(p + i) = f;
    }
  }
}

// Threads per K-5 CTA: the bf16 64-column slices (AmazonCat, Amazon-670K: ~10 short
// segments per piece, each waiting on one W1 row slice from HBM) fit 64 registers, so
// they run 32 warps per SM instead of 16 for twice the row loads in flight.
template <typename T, int CPL>
constexpr int scatter_threads() { return (sizeof(T) == 2 && CPL == 2) ? 1024 : 512; }

template <typename T, int CPL>
__global__ void __launch_bounds__(scatter_threads<T, CPL>(), 1) k_scatter_sgd_s(const int32_t* __restrict__ e_n,
                                                          const float* __restrict__ e_v,
                                                          const int32_t* __restrict__ e_u,
                                                          const int32_t* __restrict__ e_f,
                                                          const int32_t* __restrict__ useg,
                                                          const int32_t* __restrict__ meta,
                                                          const T* __restrict__ dA1, int H, float* W1,
                                                          float* part, int32_t* ucnt,
                                                          float* grad_w1, int32_t* fcnt, uint32_t* bits,
                                                          int W) {
  Tl tl_(TL_SCATTER);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const float lr = step_lr(meta);
  constexpr int CS = 32 * CPL;               // columns of this CTA's slice
  constexpr int kU = 8;
#ifndef ASGD_SEG_AHEAD
#define ASGD_SEG_AHEAD 1
#endif
  constexpr int kSegAhead = ASGD_SEG_AHEAD;   // segments whose W1 rows are in flight together
  extern __shared__ __align__(16) uint8_t sm_raw[];
  T* sd = reinterpret_cast<T*>(sm_raw);      // [n][CS]
  const int nsl = gridDim.y, slice = blockIdx.y, c0 = slice * CS;
  const int n = meta[M_NROWS];
  // stage dA1[:, c0 : c0 + CS] with bulk async copies (one for the whole block when the
  // slice is the full row, else one per row, issued by every thread); the warps load their
  // piece entries while the copy is in flight and wait on the mbarrier only before the
  // first shared-memory gather
  __shared__ __align__(8) uint64_t sbar;
  const uint32_t bar = static_cast<uint32_t>(__cvta_generic_to_shared(&sbar));
  const uint32_t row_bytes = CS * (uint32_t)sizeof(T);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"((uint32_t)n * row_bytes)
                 : "memory");
  }
  __syncthreads();
  {
    const uint32_t dst0 = static_cast<uint32_t>(__cvta_generic_to_shared(sd));
    if (nsl == 1) {   // the slice is the whole row: one copy
      if (threadIdx.x == 0 && n > 0)
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst0),
                     "l"(dA1), "r"((uint32_t)n * row_bytes), "r"(bar)
                     : "memory");
    } else {          // one copy per row, issued by every thread of the block
      for (int r = threadIdx.x; r < n; r += blockDim.x)
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         dst0 + (uint32_t)r * row_bytes),
                     "l"(dA1 + (int64_t)r * H + c0), "r"(row_bytes), "r"(bar)
                     : "memory");
    }
  }
  bool staged = false;
  auto wait_staged = [&]() {
    if (staged) return;
    uint32_t ok = 0;
    while (!ok)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(ok) : "r"(bar) : "memory");
    staged = true;
  };
  const int lane = threadIdx.x & 31;
  const int nnz = meta[M_NNZ];
  const int npieces = (nnz + kPiece - 1) / kPiece;
  const int nwarps = gridDim.x * (blockDim.x >> 5);
  using IO = SliceIO<T, CPL>;
  for (int p = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); p < npieces; p += nwarps) {
    const int e0 = p * kPiece, e1 = min(e0 + kPiece, nnz), cnt = e1 - e0;
    // one round trip for the whole piece: entries + the neighbours' features
    int myn = 0, myf = -1, myu = 0;
    float myv = 0.f;
    if (lane < cnt) { myn = e_n[e0 + lane]; myv = e_v[e0 + lane]; myf = e_f[e0 + lane]; myu = e_u[e0 + lane]; }
    int nb = -1;
    if (lane == 0 && e0 > 0) nb = e_f[e0 - 1];
    if (lane == 1 && e1 < nnz) nb = e_f[e1];
    const int fprev = __shfl_sync(kFull, nb, 0), fnext = __shfl_sync(kFull, nb, 1);
    const int fup = __shfl_up_sync(kFull, myf, 1);
    uint32_t smask = __ballot_sync(kFull, lane < cnt && (lane == 0 || myf != fup));
    while (smask) {
      // kSegAhead segments at a time: their W1 row slices are all requested before the
      // first one is summed (1 = one segment at a time; A/B switch ASGD_SEG_AHEAD)
      int sj0[kSegAhead], sj1[kSegAhead];
      float wp[kSegAhead][CPL];
#pragma unroll
      for (int d = 0; d < kSegAhead; ++d) {
        sj0[d] = -1;
        sj1[d] = 0;
        if (smask) {   // warp-uniform
          const int a = __ffs(smask) - 1;
          smask &= smask - 1;
          const int b = smask ? __ffs(smask) - 1 : cnt;
          sj0[d] = a;
          sj1[d] = b;
          const int fa = __shfl_sync(kFull, myf, a);
          if (!((a == 0 && fprev == fa) || (b == cnt && fnext == fa)))   // in flight during the gathers
            ld_cols<CPL>(W1 + (int64_t)fa * H + c0 + lane * CPL, wp[d], false);
        }
      }
#pragma unroll
      for (int d = 0; d < kSegAhead; ++d) {
      if (sj0[d] < 0) break;   // warp-uniform
      const int j0 = sj0[d], j1 = sj1[d];
      const int f = __shfl_sync(kFull, myf, j0), u = __shfl_sync(kFull, myu, j0);
      const bool before = (j0 == 0 && fprev == f), after = (j1 == cnt && fnext == f);
      float* wrow = W1 + (int64_t)f * H + c0 + lane * CPL;
      float w[CPL];
#pragma unroll
      for (int i = 0; i < CPL; ++i) w[i] = wp[d][i];   // boundary segments reload it below
      float acc[CPL];
#pragma unroll
      for (int i = 0; i < CPL; ++i) acc[i] = 0.f;
      wait_staged();   // after the first W1 row slice was requested: its load overlaps the staging
      int j = j0;
      for (; j + kU <= j1; j += kU) {
        float g[kU][CPL];
#pragma unroll
        for (int q = 0; q < kU; ++q) IO::load(sd + (int64_t)__shfl_sync(kFull, myn, j + q) * CS, lane, g[q]);
#pragma unroll
        for (int q = 0; q < kU; ++q) {
          const float v = __shfl_sync(kFull, myv, j + q);
#pragma unroll
          for (int i = 0; i < CPL; ++i) acc[i] = fmaf(v, g[q][i], acc[i]);
        }
      }
      for (; j < j1; ++j) {
        float g[CPL];
        IO::load(sd + (int64_t)__shfl_sync(kFull, myn, j) * CS, lane, g);
        const float v = __shfl_sync(kFull, myv, j);
#pragma unroll
        for (int i = 0; i < CPL; ++i) acc[i] = fmaf(v, g[i], acc[i]);
      }
      bool finish = !before && !after;
      if (!finish) {
        const int slot = before ? 2 * p : 2 * p + 1;
        st_cols<CPL>(part + (int64_t)slot * H + c0 + lane * CPL, acc, true);
        fence_mp();
        int old = 0;
        if (lane == 0) old = atomicAdd(&ucnt[(int64_t)u * nsl + slice], 1);
        old = __shfl_sync(kFull, old, 0);
        const int q0 = useg[u] / kPiece, q1 = (useg[u + 1] - 1) / kPiece;
        if (old == q1 - q0) {
          fence_mp();
          ld_cols<CPL>(wrow, w, false);
#pragma unroll
          for (int i = 0; i < CPL; ++i) acc[i] = 0.f;
          for (int q = q0; q <= q1; q += 4) {   // 4 partials in flight, summed in piece order
            float t[4][CPL];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              if (q + u <= q1)
                ld_cols<CPL>(part + (int64_t)(q + u == q0 ? 2 * q0 + 1 : 2 * (q + u)) * H + c0 + lane * CPL, t[u], true);
              else {
#pragma unroll
                for (int i = 0; i < CPL; ++i) t[u][i] = 0.f;
              }
            }
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              if (q + u <= q1) {
#pragma unroll
                for (int i = 0; i < CPL; ++i) acc[i] += t[u][i];
              }
            }
          }
          if (lane == 0) ucnt[(int64_t)u * nsl + slice] = 0;
          finish = true;
        }
      }
      if (finish) {
#pragma unroll
        for (int i = 0; i < CPL; ++i) w[i] = w[i] - lr * acc[i];
        st_cols<CPL>(wrow, w, false);
        if (grad_w1) st_cols<CPL>(grad_w1 + (int64_t)f * H + c0 + lane * CPL, acc, false);
        if (slice == 0) reset_feature(fcnt, bits, W, f, lane);
      }
      }
    }
  }
  wait_staged();   // no CTA exits with its bulk copy still writing shared memory
}

// K-5, segment-per-warp variant: warp w owns whole feature segments u = w, w + W, ...
// (K-0's entries of feature uniq[u], sorted by row), so no segment is split across warps:
// no partials, no atomics, no fences.  The W1 row slice is requested when the segment
// starts and its latency hides under the segment's gathers from the staged dA1 slice;
// the sum runs in the segment's (row) order, so it is deterministic.  A segment has at
// most B entries (one per batch row), which bounds the per-warp imbalance.
template <typename T, int CPL>
__global__ void __launch_bounds__(scatter_threads<T, CPL>(), 1)
    k_scatter_seg(const int32_t* __restrict__ e_n, const float* __restrict__ e_v,
                  const int32_t* __restrict__ useg, const int32_t* __restrict__ uniq,
                  const int32_t* __restrict__ meta, const T* __restrict__ dA1, int H, float* W1,
                  float* grad_w1, int32_t* fcnt, uint32_t* bits, int W) {
  Tl tl_(TL_SCATTER);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const float lr = step_lr(meta);
  constexpr int CS = 32 * CPL;
  extern __shared__ __align__(16) uint8_t sm_raw[];
  T* sd = reinterpret_cast<T*>(sm_raw);      // [n][CS]
  const int nsl = gridDim.y, slice = blockIdx.y, c0 = slice * CS;
  const int n = meta[M_NROWS];
  __shared__ __align__(8) uint64_t sbar;
  const uint32_t bar = static_cast<uint32_t>(__cvta_generic_to_shared(&sbar));
  const uint32_t row_bytes = CS * (uint32_t)sizeof(T);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"((uint32_t)n * row_bytes)
                 : "memory");
  }
  __syncthreads();
  {
    const uint32_t dst0 = static_cast<uint32_t>(__cvta_generic_to_shared(sd));
    if (nsl == 1) {
      if (threadIdx.x == 0 && n > 0)
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst0),
                     "l"(dA1), "r"((uint32_t)n * row_bytes), "r"(bar)
                     : "memory");
    } else {
      for (int r = threadIdx.x; r < n; r += blockDim.x)
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         dst0 + (uint32_t)r * row_bytes),
                     "l"(dA1 + (int64_t)r * H + c0), "r"(row_bytes), "r"(bar)
                     : "memory");
    }
  }
  const int lane = threadIdx.x & 31;
  const int U = meta[M_U];
  const int nwarps = gridDim.x * (blockDim.x >> 5);
  using IO = SliceIO<T, CPL>;
  bool staged = false;
  for (int u = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); u < U; u += nwarps) {
    const int j0 = useg[u], j1 = useg[u + 1];
    const int f = uniq[u];
    float* wrow = W1 + (int64_t)f * H + c0 + lane * CPL;
    float w[CPL];
    ld_cols<CPL>(wrow, w, false);                 // in flight during the gathers
    if (!staged) {
      uint32_t ok = 0;
      while (!ok)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok) : "r"(bar) : "memory");
      staged = true;
    }
    float acc[CPL];
#pragma unroll
    for (int i = 0; i < CPL; ++i) acc[i] = 0.f;
    for (int jb = j0; jb < j1; jb += 32) {
      const int cnt = min(32, j1 - jb);
      int myn = 0;
      float myv = 0.f;
      if (lane < cnt) { myn = e_n[jb + lane]; myv = e_v[jb + lane]; }
      int j = 0;
      for (; j + 8 <= cnt; j += 8) {
        float g[8][CPL];
#pragma unroll
        for (int q = 0; q < 8; ++q) IO::load(sd + (int64_t)__shfl_sync(kFull, myn, j + q) * CS, lane, g[q]);
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const float v = __shfl_sync(kFull, myv, j + q);
#pragma unroll
          for (int i = 0; i < CPL; ++i) acc[i] = fmaf(v, g[q][i], acc[i]);
        }
      }
      for (; j < cnt; ++j) {
        float g[CPL];
        IO::load(sd + (int64_t)__shfl_sync(kFull, myn, j) * CS, lane, g);
        const float v = __shfl_sync(kFull, myv, j);
#pragma unroll
        for (int i = 0; i < CPL; ++i) acc[i] = fmaf(v, g[i], acc[i]);
      }
    }
#pragma unroll
    for (int i = 0; i < CPL; ++i) w[i] = w[i] - lr * acc[i];
    st_cols<CPL>(wrow, w, false);
    if (grad_w1) st_cols<CPL>(grad_w1 + (int64_t)f * H + c0 + lane * CPL, acc, false);
    if (slice == 0) reset_feature(fcnt, bits, W, f, lane);
  }
  if (!staged) {   // no CTA exits with its bulk copy still writing shared memory
    uint32_t ok = 0;
    while (!ok)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(ok) : "r"(bar) : "memory");
  }
}

// K-5 for 64-column bf16 slices (b_max = 1024 shapes): a quarter-warp (8 lanes x 8 columns)
// per feature segment, so each warp keeps four segments' W1 row slices and entry loads in
// flight instead of one (the segment-per-warp form waits on two dependent round trips --
// entries, then the W1 row -- per short segment: AmazonCat averages 3 entries).  Sums run
// in the segment's row order: deterministic.
__global__ void __launch_bounds__(1024, 1)
    k_scatter_q(const int32_t* __restrict__ e_n, const float* __restrict__ e_v,
                const int32_t* __restrict__ useg, const int32_t* __restrict__ uniq,
                const int32_t* __restrict__ meta, const bf16* __restrict__ dA1, int H, float* W1,
                float* grad_w1, int32_t* fcnt, uint32_t* bits, int W) {
  Tl tl_(TL_SCATTER);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const float lr = step_lr(meta);
  constexpr int CS = 64;
  extern __shared__ __align__(16) uint8_t sm_raw[];
  bf16* sd = reinterpret_cast<bf16*>(sm_raw);   // [n][CS]
  const int slice = blockIdx.y, c0 = slice * CS;
  const int n = meta[M_NROWS];
  __shared__ __align__(8) uint64_t sbar;
  const uint32_t bar = static_cast<uint32_t>(__cvta_generic_to_shared(&sbar));
  const uint32_t row_bytes = CS * 2;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"((uint32_t)n * row_bytes)
                 : "memory");
  }
  __syncthreads();
  {
    const uint32_t dst0 = static_cast<uint32_t>(__cvta_generic_to_shared(sd));
    for (int r = threadIdx.x; r < n; r += blockDim.x)
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       dst0 + (uint32_t)r * row_bytes),
                   "l"(dA1 + (int64_t)r * H + c0), "r"(row_bytes), "r"(bar)
                   : "memory");
  }
  const int lane = threadIdx.x & 31, grp = lane >> 3, gl = lane & 7;
  const unsigned gmask = 0xFFu << (grp * 8);
  const int U = meta[M_U];
  const int nwarps = gridDim.x * (blockDim.x >> 5);
  const int wid = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int ngroups = 4 * nwarps;
  bool staged = false;
  for (int u = 4 * wid + grp; u - grp < U; u += ngroups) {   // warp-uniform trip count
    const bool active = u < U;
    int j0 = 0, j1 = 0, f = 0;
    float w[8];
    if (active) {
      j0 = useg[u]; j1 = useg[u + 1]; f = uniq[u];
      const float4* wp = reinterpret_cast<const float4*>(W1 + (int64_t)f * H + c0 + gl * 8);
      const float4 a = wp[0], b = wp[1];   // in flight during the gathers
      w[0] = a.x; w[1] = a.y; w[2] = a.z; w[3] = a.w; w[4] = b.x; w[5] = b.y; w[6] = b.z; w[7] = b.w;
    }
    if (!staged) {
      uint32_t ok = 0;
      while (!ok)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(ok) : "r"(bar) : "memory");
      staged = true;
    }
    if (!active) continue;
    float acc[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] = 0.f;
    for (int jb = j0; jb < j1; jb += 8) {
      const int cnt = min(8, j1 - jb);
      int myn = 0;
      float myv = 0.f;
      if (gl < cnt) { myn = e_n[jb + gl]; myv = e_v[jb + gl]; }
      for (int q = 0; q < cnt; ++q) {
        const int rr = __shfl_sync(gmask, myn, grp * 8 + q);
        const float v = __shfl_sync(gmask, myv, grp * 8 + q);
        const uint4 pk = reinterpret_cast<const uint4*>(sd + (int64_t)rr * CS)[gl];
        const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&pk);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float2 g = __bfloat1622float2(h[i]);
          acc[2 * i] = fmaf(v, g.x, acc[2 * i]);
          acc[2 * i + 1] = fmaf(v, g.y, acc[2 * i + 1]);
        }
      }
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) w[i] = w[i] - lr * acc[i];
    float4* wp = reinterpret_cast<float4*>(W1 + (int64_t)f * H + c0 + gl * 8);
    wp[0] = make_float4(w[0], w[1], w[2], w[3]);
    wp[1] = make_float4(w[4], w[5], w[6], w[7]);
    if (grad_w1) {
      float4* gp = reinterpret_cast<float4*>(grad_w1 + (int64_t)f * H + c0 + gl * 8);
      gp[0] = make_float4(acc[0], acc[1], acc[2], acc[3]);
      gp[1] = make_float4(acc[4], acc[5], acc[6], acc[7]);
    }
    if (slice == 0) {   // K-0's per-feature count and row bitmap back to zero
      if (gl == 0) fcnt[f] = 0;
      for (int ww = gl; ww < W; ww += 8) bits[(int64_t)f * W + ww] = 0u;
    }
  }
  if (!staged) {
    uint32_t ok = 0;
    while (!ok)
      asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                   : "=r"(ok) : "r"(bar) : "memory");
  }
}

// One resident wave of 256-thread CTAs (occupancy from the compiled kernel), no
// more CTAs than there are 8-piece groups for the largest step.
template <typename K>
int wave_grid(const Launch& lc, K kernel, size_t smem, int64_t pieces, int& occ, int warps = 8) {
  if (!occ && (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, 32 * warps, smem) != cudaSuccess || occ < 1))
    occ = 1;
  const int64_t need = (pieces + warps - 1) / warps;
  return (int)std::max<int64_t>(1, std::min<int64_t>(need, (int64_t)lc.sms * occ));
}

// K-1 grid cap (ASGD_K1_CTAS, A/B): the CTAs that stay resident beside K-0's
int k1_cap() {
  static const int v = [] { const char* e = getenv("ASGD_K1_CTAS"); return e ? atoi(e) : 0; }();
  return v;
}

template <int VPL, bool TMA>
cudaError_t spmm_fwd_t(const Launch& lc, const StepArgs& sa, const asgd_csr& x, const float* W1, const float* b1,
                       const Ptrs& P, const WsLayout& L, bool want_bf16, bool fold, int b_max) {
  const int ntiles = fold ? (int)L.n_tiles_f : 0;
  const size_t smem = TMA ? k1_smem<VPL, TMA>() : view_smem(sa.n);
  // the batch view (dynamic) + the group partials (static) exceed 48 KB at b_max = 2048
  cudaError_t e = ensure_smem(k_spmm_fwd<VPL, TMA>, TMA ? k1_smem<VPL, TMA>() : view_smem(2048));
  if (e != cudaSuccess) return e;
  static int occ = 0;
  int grid = wave_grid(lc, k_spmm_fwd<VPL, TMA>, TMA ? k1_smem<VPL, TMA>() : view_smem(2048), L.n_pieces, occ,
                       k1_warps<VPL, TMA>());
  if (k1_cap() > 0) grid = std::min(grid, k1_cap());
  const ViewOut vo{P.boff, P.loff, P.rbase, P.rowsc, P.meta};
  launch_k(lc, k_spmm_fwd<VPL, TMA>, dim3(grid), dim3(32 * k1_warps<VPL, TMA>()), smem, sa, x.row_ptr, x.lab_ptr,
           x.n_rows, L.nz_cap, L.nl_cap, vo, x.col, x.val, W1, b1, P.h1, want_bf16 ? P.h1b : nullptr,
           want_bf16 ? P.h1l : nullptr, P.part1, P.rowcnt, P.cnt, P.bits, (b_max + 31) / 32, P.tsum, ntiles);
  return cudaGetLastError();
}

template <int VPL>
cudaError_t scatter_t(const Launch& lc, float* W1, const Ptrs& P, const WsLayout& L,
                      float* grad_w1, int b_max) {
  const int W = (b_max + 31) / 32;
  static int occ = 0;
  const int grid = wave_grid(lc, k_scatter_sgd<VPL>, 0, L.n_pieces, occ);
  launch_k(lc, k_scatter_sgd<VPL>, dim3(grid), dim3(256), 0, P.e_n, P.e_v, P.e_u, P.useg, P.uniq, P.meta, P.da1,
                                             W1, P.part5, P.ucnt, grad_w1, P.cnt, P.bits, W);
  return cudaGetLastError();
}

}  // namespace

// K-0 threads per CTA (ASGD_K0_THREADS = 128 / 256 / 512): fewer threads leave more of
// each SM's register file to the kernels beside it (K-1 or the dense chain); at least
// b_max / 8 (the batch view: 8 rows per thread)
int touched_threads(int b_max) {
  static const int v = [] { const char* e = getenv("ASGD_K0_THREADS"); return e ? atoi(e) : 512; }();
  int t = v == 128 || v == 256 ? v : 512;
  while (8 * t < b_max && t < 512) t *= 2;
  return t;
}

template <int NT, bool FOLD>
cudaError_t touched_t(const Launch& lc, const StepArgs& sa, const asgd_csr& x, int64_t F, const Ptrs& P,
                      const WsLayout& L, int W, int ctas, size_t smem_all) {
  if (smem_all > 48 * 1024) {
    cudaError_t e = ensure_smem(k_touched<NT, FOLD>, smem_all);
    if (e != cudaSuccess) return e;
  }
  // K-0's two software grid barriers need every CTA resident at once: at most one CTA per
  // SM, and the kernel alone must fit ctas CTAs (asserted here instead of a cooperative
  // launch, which graphs with programmatic dependent launch do not capture; the kernels
  // beside it on other streams never wait for K-0, so its CTAs always get their SMs)
  int occ = 0;
  {
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_touched<NT, FOLD>, NT, smem_all);
    if (e != cudaSuccess) return e;
  }
  if ((int64_t)occ * lc.sms < ctas) return cudaErrorCooperativeLaunchTooLarge;
  return launch_k(lc, k_touched<NT, FOLD>, dim3(ctas), dim3(NT), smem_all, sa, x.row_ptr, x.n_rows, L.nz_cap, x.col,
                  x.val, P.meta, P.cnt, P.tsum, F, (int)L.n_tiles_f, P.fseg, P.fuid, P.uniq, P.useg, P.bits, W, P.e_n,
                  P.e_v, P.e_u, P.e_f, P.boff, P.rbase);
}

cudaError_t launch_touched(const Launch& lc, const StepArgs& sa, const asgd_csr& x, int64_t F, const Ptrs& P,
                           const WsLayout& L, int b_max) {
  const int n = sa.n;
  const size_t smem = view_smem(n);
  const int nt = (int)L.n_tiles_f;
  const int W = (b_max + 31) / 32;
  const size_t smem_all = ((smem + 3) / 4) * 4 + (size_t)nt * 8;
  static const int max_ctas = [] { const char* e = getenv("ASGD_K0_CTAS"); return e ? atoi(e) : 0; }();
  int64_t cap = max_ctas > 0 ? max_ctas : kTouchCtas;
  const int ctas = (int)std::max<int64_t>(1, std::min<int64_t>({(int64_t)lc.sms, cap, (L.nz_cap + 1023) / 1024}));
  const bool fd = k0_fold();
  switch (touched_threads(b_max)) {
    case 128: return fd ? touched_t<128, true>(lc, sa, x, F, P, L, W, ctas, smem_all)
                        : touched_t<128, false>(lc, sa, x, F, P, L, W, ctas, smem_all);
    case 256: return fd ? touched_t<256, true>(lc, sa, x, F, P, L, W, ctas, smem_all)
                        : touched_t<256, false>(lc, sa, x, F, P, L, W, ctas, smem_all);
    default: return fd ? touched_t<512, true>(lc, sa, x, F, P, L, W, ctas, smem_all)
                       : touched_t<512, false>(lc, sa, x, F, P, L, W, ctas, smem_all);
  }
}

// K-1 with TMA-staged W1 rows (H <= 256, ASGD_K1_TMA=1; measured slower at EURLex: 31 vs 21 us live)
bool k1_tma() {
  static const bool v = [] { const char* e = getenv("ASGD_K1_TMA"); return e && e[0] == '1'; }();
  return v;
}

// K-0's phase A inside K-1 (default; ASGD_K0_FOLD=0 keeps the separate K-0 beside K-1): K-1
// counts the batch's features as it reads the entries, and K-0 (phases C, E) runs after it
// on the side stream.  Measured at EURLex (live kernel timeline): K-1 beside the full K-0
// 21.4 us, alone 10.8, with the folded counts 15.1; step 66.8 -> 61.3 us back to back.
bool k0_fold() {
  static const bool v = [] { const char* e = getenv("ASGD_K0_FOLD"); return !(e && e[0] == '0'); }();
  return v;
}

cudaError_t launch_spmm_fwd(const Launch& lc, const StepArgs& sa, const asgd_csr& x, const float* W1,
                            const float* b1, int H, const Ptrs& P, const WsLayout& L, bool want_bf16, bool fold,
                            int b_max) {
  const bool t = k1_tma();
  switch (H) {
    case 64: return t ? spmm_fwd_t<2, true>(lc, sa, x, W1, b1, P, L, want_bf16, fold, b_max)
                      : spmm_fwd_t<2, false>(lc, sa, x, W1, b1, P, L, want_bf16, fold, b_max);
    case 128: return t ? spmm_fwd_t<4, true>(lc, sa, x, W1, b1, P, L, want_bf16, fold, b_max)
                       : spmm_fwd_t<4, false>(lc, sa, x, W1, b1, P, L, want_bf16, fold, b_max);
    case 256: return t ? spmm_fwd_t<8, true>(lc, sa, x, W1, b1, P, L, want_bf16, fold, b_max)
                       : spmm_fwd_t<8, false>(lc, sa, x, W1, b1, P, L, want_bf16, fold, b_max);
    case 512: return spmm_fwd_t<16, false>(lc, sa, x, W1, b1, P, L, want_bf16, fold, b_max);
    default: return cudaErrorInvalidValue;
  }
}

const void* spmm_fwd_func(int H) {
  const bool t = k1_tma();
  switch (H) {
    case 64: return t ? reinterpret_cast<const void*>(k_spmm_fwd<2, true>) : reinterpret_cast<const void*>(k_spmm_fwd<2, false>);
    case 128: return t ? reinterpret_cast<const void*>(k_spmm_fwd<4, true>) : reinterpret_cast<const void*>(k_spmm_fwd<4, false>);
    case 256: return t ? reinterpret_cast<const void*>(k_spmm_fwd<8, true>) : reinterpret_cast<const void*>(k_spmm_fwd<8, false>);
    default: return reinterpret_cast<const void*>(k_spmm_fwd<16, false>);
  }
}

const void* touched_func(int b_max) {
  const bool fd = k0_fold();
  switch (touched_threads(b_max)) {
    case 128: return fd ? reinterpret_cast<const void*>(k_touched<128, true>) : reinterpret_cast<const void*>(k_touched<128, false>);
    case 256: return fd ? reinterpret_cast<const void*>(k_touched<256, true>) : reinterpret_cast<const void*>(k_touched<256, false>);
    default: return fd ? reinterpret_cast<const void*>(k_touched<512, true>) : reinterpret_cast<const void*>(k_touched<512, false>);
  }
}

template <typename... A>
constexpr int nargs_of(void (*)(A...)) { return (int)sizeof...(A); }
int spmm_fwd_nargs() { return nargs_of(k_spmm_fwd<8, false>); }
int touched_nargs() { return nargs_of(k_touched<512, false>); }

// K-5 layout: ASGD_K5_SEG=1 -> one warp per feature segment (k_scatter_seg), else nnz pieces
bool k5_seg() {
  static const bool v = [] { const char* e = getenv("ASGD_K5_SEG"); return e && e[0] == '1'; }();
  return v;
}
// 64-column bf16 slices: ASGD_K5_Q=1 -> a quarter-warp per feature segment (k_scatter_q)
bool k5_quarter() {
  static const bool v = [] { const char* e = getenv("ASGD_K5_Q"); return e && e[0] == '1'; }();
  return v;
}

template <typename T, int CPL>
cudaError_t scatter_s_t(const Launch& lc, const T* dA1, int H, int b_max, float* W1,
                        const Ptrs& P, float* grad_w1) {
  constexpr int CS = 32 * CPL;
  const int nsl = H / CS;
  const size_t smem = (size_t)b_max * CS * sizeof(T);
  const int gx = std::max(1, lc.sms / nsl);
  if constexpr (sizeof(T) == 2 && CS == 64) {
    if (k5_quarter()) {   // 64-column bf16 slices: a quarter-warp per feature segment
      cudaError_t e = ensure_smem(k_scatter_q, 200 * 1024);
      if (e != cudaSuccess) return e;
      return launch_k(lc, k_scatter_q, dim3(gx, nsl), dim3(1024), smem, P.e_n, P.e_v, P.useg, P.uniq, P.meta,
                      reinterpret_cast<const bf16*>(dA1), H, W1, grad_w1, P.cnt, P.bits, (b_max + 31) / 32);
    }
  }
  if (k5_seg()) {
    cudaError_t e = ensure_smem(k_scatter_seg<T, CPL>, 200 * 1024);
    if (e != cudaSuccess) return e;
    return launch_k(lc, k_scatter_seg<T, CPL>, dim3(gx, nsl), dim3(scatter_threads<T, CPL>()), smem, P.e_n, P.e_v,
                    P.useg, P.uniq, P.meta, dA1, H, W1, grad_w1, P.cnt, P.bits, (b_max + 31) / 32);
  }
  cudaError_t e = ensure_smem(k_scatter_sgd_s<T, CPL>, 200 * 1024);
  if (e != cudaSuccess) return e;
  return launch_k(lc, k_scatter_sgd_s<T, CPL>, dim3(gx, nsl), dim3(scatter_threads<T, CPL>()), smem, P.e_n, P.e_v, P.e_u,
                  P.e_f, P.useg, P.meta, dA1, H, W1, P.part5, P.ucnt, grad_w1, P.cnt, P.bits,
                  (b_max + 31) / 32);
}

// Widest column slice whose staged dA1 fits 160 KB of shared memory (0 = none).
int scatter_slice(int H, int b_max, size_t elem) {
  for (int cs = std::min(H, 256); cs >= 64; cs /= 2)
    if (H % cs == 0 && (size_t)b_max * cs * elem <= 160 * 1024) return cs;
  return 0;
}

cudaError_t launch_scatter_sgd(const Launch& lc, float* W1, int H, const Ptrs& P,
                               const WsLayout& L, float* grad_w1, const bf16* dA1b, int b_max) {
  const size_t elem = dA1b ? 2 : 4;
  const int cs = scatter_slice(H, b_max, elem);
  if (cs) {
    if (dA1b) {
      if (cs == 256) return scatter_s_t<bf16, 8>(lc, dA1b, H, b_max, W1, P, grad_w1);
      if (cs == 128) return scatter_s_t<bf16, 4>(lc, dA1b, H, b_max, W1, P, grad_w1);
      return scatter_s_t<bf16, 2>(lc, dA1b, H, b_max, W1, P, grad_w1);
    }
    if (cs == 256) return scatter_s_t<float, 8>(lc, P.da1, H, b_max, W1, P, grad_w1);
    if (cs == 128) return scatter_s_t<float, 4>(lc, P.da1, H, b_max, W1, P, grad_w1);
    return scatter_s_t<float, 2>(lc, P.da1, H, b_max, W1, P, grad_w1);
  }
  switch (H) {
    case 64: return scatter_t<2>(lc, W1, P, L, grad_w1, b_max);
    case 128: return scatter_t<4>(lc, W1, P, L, grad_w1, b_max);
    case 256: return scatter_t<8>(lc, W1, P, L, grad_w1, b_max);
    case 512: return scatter_t<16>(lc, W1, P, L, grad_w1, b_max);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace asgd


namespace asgd {
ASGD_TL_SETTER(tl_set_sparse)
}  // namespace asgd
