// Merge, evaluation and validation kernels (sm_100a).
//   K-6  ||w_i||^2 (fp64, fixed order) and the prescale w_i <- alpha_i w_i
//        (Alg. 2 lines 4 and 8; reading Q16)
//   K-7  momentum epilogue w' = S + gamma (w - w_p); w_p <- w; w <- w'
//        (Alg. 2 lines 8-9) -- on every GPU instead of
//        the paper's CPU scheduler (reading Q20)
//   wsum single-device stand-in of the all-reduce for simulated replicas
//   top-k evaluation (reading Q23)
// All HBM-bound: float4 streams, grids sized in multiples of the SM count.
#include <algorithm>

#include "asgd_internal.h"

namespace asgd {
namespace {

constexpr unsigned kFull = 0xffffffffu;

__global__ void __launch_bounds__(256) k_sqnorm_part(const float* __restrict__ x, int64_t P,
                                                     double* partials) {
  Tl tl_(TL_MERGE);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  double s = 0.0;
  const int64_t P4 = P / 4;
  const float4* x4 = reinterpret_cast<const float4*>(x);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < P4;
       i += (int64_t)gridDim.x * blockDim.x) {
    float4 v = __ldcs(x4 + i);
    s += (double)v.x * v.x + (double)v.y * v.y + (double)v.z * v.z + (double)v.w * v.w;
  }
  if (blockIdx.x == 0)
    for (int64_t i = P4 * 4 + threadIdx.x; i < P; i += blockDim.x) s += (double)x[i] * x[i];
  __shared__ double sh[8];
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int w = 0; w < 8; ++w) t += sh[w];
    partials[blockIdx.x] = t;
  }
}

__global__ void k_sqnorm_final(const double* __restrict__ partials, int n, double* out) {
  Tl tl_(TL_MERGE);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  __shared__ double sh[32];
  double s = 0.0;
  // fixed assignment: thread t sums partials t, t+blockDim, ... in order
  for (int i = threadIdx.x; i < n; i += blockDim.x) s += partials[i];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(kFull, s, o);
  if (lane == 0) sh[wid] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += sh[w];
    *out = t;
  }
}

__global__ void __launch_bounds__(256) k_scale(float* x, int64_t P, double alpha) {
  Tl tl_(TL_MERGE);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const int64_t P4 = P / 4;
  float4* x4 = reinterpret_cast<float4*>(x);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < P4;
       i += (int64_t)gridDim.x * blockDim.x) {
    float4 v = x4[i];
    v.x = (float)(alpha * v.x); v.y = (float)(alpha * v.y);
    v.z = (float)(alpha * v.z); v.w = (float)(alpha * v.w);
    x4[i] = v;
  }
  if (blockIdx.x == 0)
    for (int64_t i = P4 * 4 + threadIdx.x; i < P; i += blockDim.x) x[i] = (float)(alpha * x[i]);
}

__device__ __forceinline__ void finish1(float& p, float& w, float& d, float gamma) {
  const float wn = fmaf(gamma, d, p);   // w' = S + gamma (w - w_p)
  d = wn - w;                            // next (w - w_p)
  w = wn;
  p = wn;                                // replica <- w'
}

__global__ void __launch_bounds__(256) k_finish(float* params, float* w, float* d, int64_t P,
                                                float gamma) {
  Tl tl_(TL_MERGE);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const int64_t P4 = P / 4;
  float4* p4 = reinterpret_cast<float4*>(params);
  float4* w4 = reinterpret_cast<float4*>(w);
  float4* d4 = reinterpret_cast<float4*>(d);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < P4;
       i += (int64_t)gridDim.x * blockDim.x) {
    float4 p = p4[i], ww = w4[i], dd = d4[i];
    finish1(p.x, ww.x, dd.x, gamma); finish1(p.y, ww.y, dd.y, gamma);
    finish1(p.z, ww.z, dd.z, gamma); finish1(p.w, ww.w, dd.w, gamma);
    p4[i] = p; w4[i] = ww; d4[i] = dd;
  }
  if (blockIdx.x == 0)
    for (int64_t i = P4 * 4 + threadIdx.x; i < P; i += blockDim.x) finish1(params[i], w[i], d[i], gamma);
}

__global__ void __launch_bounds__(256) k_wsum(const float* const* __restrict__ reps,
                                              const double* __restrict__ alpha, int n, int64_t P,
                                              float* out) {
  Tl tl_(TL_MERGE);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < P;
       i += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int r = 0; r < n; ++r) s += alpha[r] * (double)reps[r][i];
    out[i] = (float)s;
  }
}

// ------------------------------------------------ fused peer-memory merge (NEXT-1)
// Alg. 2 lines 8-9 over NVLink peer memory in one kernel (SURVEY §8(f) NEXT-1,
// the B200 analogue of the paper's multi-stream ring all-reduce):
// rank r owns the parameter shard [lo, hi).  For each element it reads every
// replica j's value over P2P (fixed order j = 0..N-1, fp64), forms
// S = sum_j alpha_j w_j, applies the momentum epilogue on its own shard of
// (w, d), and stores w' into every replica (P2P stores).  Every element is
// computed by exactly one rank and broadcast, so the replicas end bitwise
// identical; no prescale pass, no NCCL staging.  The last CTA signals every
// peer's arrival counter (system-scope atomics); k_merge_wait blocks the stream
// until all N ranks have delivered their shards.
__device__ __forceinline__ void merge1(const PeerSet& ps, int64_t i, float& w, float& d, float gamma) {
  double s = 0.0;
  for (int j = 0; j < ps.n; ++j) s += ps.alpha[j] * (double)ps.p[j][i];
  const float wn = fmaf(gamma, d, (float)s);
  d = wn - w;
  w = wn;
  for (int j = 0; j < ps.n; ++j) ps.p[j][i] = wn;
}

__global__ void __launch_bounds__(256) k_merge_fused(PeerSet ps, float* w, float* d, int64_t lo, int64_t hi,
                                                     float gamma, unsigned int* cta_done) {
  Tl tl_(TL_MERGE);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const int64_t lo4 = lo / 4, hi4 = hi / 4;   // lo is a multiple of 4; the tail (hi % 4) is scalar
  for (int64_t i4 = lo4 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i4 < hi4;
       i4 += (int64_t)gridDim.x * blockDim.x) {
    double s[4] = {0.0, 0.0, 0.0, 0.0};
    for (int j = 0; j < ps.n; ++j) {
      const float4 v = reinterpret_cast<const float4*>(ps.p[j])[i4];
      const double a = ps.alpha[j];
      s[0] += a * (double)v.x; s[1] += a * (double)v.y; s[2] += a * (double)v.z; s[3] += a * (double)v.w;
    }
    float4 ww = reinterpret_cast<float4*>(w)[i4], dd = reinterpret_cast<float4*>(d)[i4];
    float4 o;
    o.x = fmaf(gamma, dd.x, (float)s[0]); o.y = fmaf(gamma, dd.y, (float)s[1]);
    o.z = fmaf(gamma, dd.z, (float)s[2]); o.w = fmaf(gamma, dd.w, (float)s[3]);
    dd.x = o.x - ww.x; dd.y = o.y - ww.y; dd.z = o.z - ww.z; dd.w = o.w - ww.w;
    reinterpret_cast<float4*>(w)[i4] = o;
    reinterpret_cast<float4*>(d)[i4] = dd;
    for (int j = 0; j < ps.n; ++j) reinterpret_cast<float4*>(ps.p[j])[i4] = o;
  }
  if (blockIdx.x == 0)
    for (int64_t i = hi4 * 4 + threadIdx.x; i < hi; i += blockDim.x) merge1(ps, i, w[i], d[i], gamma);
  // completion: the last CTA tells every rank that this shard has arrived
  __threadfence_system();
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned int old = atomicAdd(cta_done, 1u);
    if (old == gridDim.x - 1) {
      *cta_done = 0u;
      __threadfence_system();
      for (int j = 0; j < ps.n; ++j) atomicAdd_system(ps.sync[j], 1ull);
    }
  }
}

__global__ void k_merge_wait(const unsigned long long* arrived, unsigned long long goal) {
  pdl_wait();   // launched with programmatic dependent launch: start polling after k_merge_fused completed
  unsigned long long v;
  do {
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(arrived) : "memory");
    if (v < goal) __nanosleep(256);
  } while (v < goal);
  __threadfence_system();
}

// ------------------------------------------------------------------- top-k
struct Cand { float v; int id; };
__device__ __forceinline__ bool better(const Cand& a, const Cand& b) {
  return a.v > b.v || (a.v == b.v && a.id < b.id);
}

template <int K>
__global__ void __launch_bounds__(256) k_topk(int64_t L, int64_t ldz, int k, const float* __restrict__ z,
                                              int32_t* out) {
  Tl tl_(TL_OTHER);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const int n = blockIdx.x;
  const float* row = z + (int64_t)n * ldz;
  Cand top[K];
#pragma unroll
  for (int i = 0; i < K; ++i) top[i] = Cand{-INFINITY, 0x7fffffff};
  for (int64_t j = threadIdx.x; j < L; j += blockDim.x) {
    Cand c{row[j], (int)j};
    if (better(c, top[K - 1])) {
      top[K - 1] = c;
#pragma unroll
      for (int i = K - 1; i > 0; --i)
        if (better(top[i], top[i - 1])) { Cand t = top[i]; top[i] = top[i - 1]; top[i - 1] = t; }
    }
  }
  __shared__ Cand sh[8];
  int head = 0;
  for (int r = 0; r < k; ++r) {
    Cand c = head < K ? top[head] : Cand{-INFINITY, 0x7fffffff};
    // warp argmax
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      Cand oth{__shfl_xor_sync(kFull, c.v, o), __shfl_xor_sync(kFull, c.id, o)};
      if (better(oth, c)) c = oth;
    }
    if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = c;
    __syncthreads();
    Cand best = sh[0];
    for (int w = 1; w < (int)(blockDim.x >> 5); ++w) if (better(sh[w], best)) best = sh[w];
    if (head < K && top[head].id == best.id && top[head].v == best.v) ++head;
    if (threadIdx.x == 0) out[(int64_t)n * k + r] = best.id;
    __syncthreads();
  }
}

// -------------------------------------------------------------- validation
__global__ void k_validate(asgd_csr c, int64_t F, int64_t L, int32_t* err) {
  Tl tl_(TL_OTHER);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < c.n_rows;
       r += (int64_t)gridDim.x * blockDim.x) {
    int e = 0;
    const int64_t a = c.row_ptr[r], b = c.row_ptr[r + 1];
    if (r == 0 && a != 0) e |= 1;
    if (r == c.n_rows - 1 && b != c.nnz) e |= 1;
    if (b < a) e |= 1;
    else
      for (int64_t k = a; k < b; ++k) {
        const int32_t f = c.col[k];
        if (f < 0 || f >= F) { e |= 2; break; }
        if (k > a && f <= c.col[k - 1]) { e |= 4; break; }
      }
    const int64_t la = c.lab_ptr[r], lb = c.lab_ptr[r + 1];
    if (r == 0 && la != 0) e |= 8;
    if (r == c.n_rows - 1 && lb != c.n_lab) e |= 8;
    if (lb <= la || lb - la > kMaxRowLabels) e |= 16;
    else
      for (int64_t k = la; k < lb; ++k) {
        const int32_t y = c.lab[k];
        if (y < 0 || y >= L) { e |= 32; break; }
        if (k > la && y <= c.lab[k - 1]) { e |= 64; break; }
      }
    if (e) atomicOr(err, e);
  }
}

inline int grid_for(const Launch& lc, int64_t work) {
  const int64_t g = std::min<int64_t>((work + 255) / 256, (int64_t)lc.sms * 8);
  return (int)std::max<int64_t>(g, 1);
}

}  // namespace

cudaError_t launch_sqnorm(const Launch& lc, const float* x, int64_t P, double* partials,
                          int nparts, double* out) {
  launch_k(lc, k_sqnorm_part, dim3(nparts), dim3(256), 0, x, P, partials);
  launch_k(lc, k_sqnorm_final, dim3(1), dim3(1024), 0, partials, nparts, out);
  return cudaGetLastError();
}

cudaError_t launch_scale(const Launch& lc, float* x, int64_t P, double alpha) {
  launch_k(lc, k_scale, dim3(grid_for(lc, P / 4)), dim3(256), 0, x, P, alpha);
  return cudaGetLastError();
}

cudaError_t launch_finish(const Launch& lc, float* params, float* w, float* d, int64_t P,
                          float gamma) {
  launch_k(lc, k_finish, dim3(grid_for(lc, P / 4)), dim3(256), 0, params, w, d, P, gamma);
  return cudaGetLastError();
}

cudaError_t launch_wsum(const Launch& lc, const float* const* reps, const double* alpha, int n,
                        int64_t P, float* out) {
  launch_k(lc, k_wsum, dim3(grid_for(lc, P)), dim3(256), 0, reps, alpha, n, P, out);
  return cudaGetLastError();
}

cudaError_t launch_merge_fused(const Launch& lc, const PeerSet& ps, float* w, float* d, int64_t lo, int64_t hi,
                               float gamma, unsigned int* cta_done, const unsigned long long* arrived,
                               unsigned long long goal) {
  launch_k(lc, k_merge_fused, dim3(grid_for(lc, std::max<int64_t>((hi - lo) / 4, 1))), dim3(256), 0, ps, w, d, lo, hi,
           gamma, cta_done);
  launch_k(lc, k_merge_wait, dim3(1), dim3(32), 0, arrived, goal);
  return cudaGetLastError();
}

cudaError_t launch_topk(const Launch& lc, int n, int64_t L, int64_t ldz, int k, const float* z,
                        int32_t* out) {
  if (k <= 0 || k > 8) return cudaErrorInvalidValue;
  launch_k(lc, k_topk<8>, dim3(n), dim3(256), 0, L, ldz, k, z, out);
  return cudaGetLastError();
}

cudaError_t launch_validate_csr(const Launch& lc, const asgd_csr* c, int64_t F, int64_t L,
                                int32_t* err) {
  launch_k(lc, k_validate, dim3(grid_for(lc, c->n_rows)), dim3(256), 0, *c, F, L, err);
  return cudaGetLastError();
}

}  // namespace asgd


namespace asgd {
ASGD_TL_SETTER(tl_set_merge)
}  // namespace asgd
