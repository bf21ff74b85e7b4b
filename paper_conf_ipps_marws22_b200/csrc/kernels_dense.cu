// Dense element-wise / reduction kernels of the local step (sm_100a) around the
// tcgen05 GEMMs G1-G3 of kernels_tc.cu:
//   softmax-CE: lse, loss, dZ = (softmax(Z) - T)/B   (row a5; sigmoid-BCE, R11)
//   dA1 = dH1 * [A1 > 0] from G2's split-K partials, b1 update (rows a6, a7)
//   merge-side helpers: the bf16 W2 shadow (and its bf16x3 lo half, R14)
// Model: PAPER.md P:1525-1531 (§V-A); SGD: P:437-455 (§II); fused element-wise
// work follows the paper's kernel fusion (§IV).  Both precisions run
// the contractions on the tensor cores; the fp32 path as bf16x3 (R14).
#include <algorithm>

#include "asgd_internal.h"

namespace asgd {
namespace {

constexpr unsigned kFull = 0xffffffffu;

// ------------------------------------------------------------ softmax + CE
// One CTA per batch row n: lse = log sum_j exp(Z_nj); loss_n = lse - mean_{y in Y_n} Z_ny;
// dZ_nj = (exp(Z_nj - lse) - T_nj) / B with T_nj = 1/|Y_n| on Y_n (Q3, Q4).
__global__ void __launch_bounds__(512) k_softmax_ce(int B, int64_t L, int64_t ldz,
                                                    const int32_t* __restrict__ rows,
                                                    const int64_t* __restrict__ lab_ptr,
                                                    const int32_t* __restrict__ lab, float* Z,
                                                    bf16* dZb, bf16* dZl, float* rowloss,
                                                    const float2* __restrict__ stats, int ntiles,
                                                    int64_t stats_ld) {
  Tl tl_(TL_SOFTMAX);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  __shared__ int s_lab[kMaxRowLabels];
  __shared__ float s_lz[kMaxRowLabels];
  __shared__ float s_m[16], s_s[16];
  __shared__ float s_lse, s_lsum;
  const int n = blockIdx.x;
  const int64_t id = rows[n];   // in flight with the partials below
  // pass 1: online max / sum-exp, kSU loads in flight per thread -- or, when G1
  // left per-tile partials, combine those instead of re-reading the row.  The
  // partials need only n, so they are combined before the label chain
  // (rows -> lab_ptr -> lab -> Z) starts instead of after it.
  constexpr int kSU = 8;
  float m = -INFINITY, s = 0.f;
  if (stats) {
    for (int t = threadIdx.x; t < ntiles; t += blockDim.x) {
      const float2 p = stats[(int64_t)t * stats_ld + n];
      if (p.x == -INFINITY) continue;
      if (p.x > m) { s = (m == -INFINITY ? 0.f : s * __expf(m - p.x)) + p.y; m = p.x; }
      else s += p.y * __expf(p.x - m);
    }
  }
  float* z = Z + (int64_t)n * ldz;
  // with G1's partials and a row that fits one pass (EURLex: 3,993 <= 8 x 512), the row's Z
  // is loaded now, in flight with the partials; the dZ pass below uses these registers
  // (measured: EURLex bf16 4.53 -> 4.55 M samples/s, fp32 3.96 -> 4.00 M)
  const bool one = stats && dZb && L <= (int64_t)kSU * blockDim.x;   // (in-place dZ needs Z's labels first)
  float zv[kSU];
  if (one) {
#pragma unroll
    for (int k = 0; k < kSU; ++k) {
      const int64_t j = threadIdx.x + (int64_t)k * blockDim.x;
      zv[k] = j < L ? z[j] : 0.f;
    }
  }
  const int64_t l0 = lab_ptr[id];
  const int64_t nl64 = lab_ptr[id + 1] - l0;
  const int nl = (int)(nl64 < kMaxRowLabels ? nl64 : kMaxRowLabels);
  // the row's label logits (rows -> lab_ptr -> lab -> Z, a dependent chain): gathered here
  // unless `one`, where they are gathered after the lse, beside the dZ stores
  auto gather_labels = [&]() {
    for (int i = threadIdx.x; i < nl; i += blockDim.x) {
      int y = lab[l0 + i];
      s_lab[i] = y;
      s_lz[i] = z[y];
    }
  };
  if (!one) gather_labels();
  for (int64_t j0 = stats ? L : threadIdx.x; j0 < L; j0 += (int64_t)kSU * blockDim.x) {
    float v[kSU];
#pragma unroll
    for (int k = 0; k < kSU; ++k) {
      const int64_t j = j0 + (int64_t)k * blockDim.x;
      v[k] = j < L ? z[j] : -INFINITY;
    }
    float bm = v[0];
#pragma unroll
    for (int k = 1; k < kSU; ++k) bm = fmaxf(bm, v[k]);
    if (bm > m) { s = (m == -INFINITY) ? 0.f : s * __expf(m - bm); m = bm; }
#pragma unroll
    for (int k = 0; k < kSU; ++k) s += __expf(v[k] - m);   // exp(-inf) = 0 for the tail
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const float om = __shfl_xor_sync(kFull, m, o), os = __shfl_xor_sync(kFull, s, o);
    const float nm = fmaxf(m, om);
    s = (m == -INFINITY ? 0.f : s * __expf(m - nm)) + (om == -INFINITY ? 0.f : os * __expf(om - nm));
    m = nm;
  }
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) { s_m[wid] = m; s_s[wid] = s; }
  __syncthreads();
  if (threadIdx.x == 0) {
    float M = -INFINITY, S = 0.f;
    const int nw = blockDim.x >> 5;
    for (int w = 0; w < nw; ++w) M = fmaxf(M, s_m[w]);
    for (int w = 0; w < nw; ++w) S += (s_m[w] == -INFINITY) ? 0.f : s_s[w] * __expf(s_m[w] - M);
    const float lse = M + logf(S);
    s_lse = lse;
    if (!one) {
      float ls = 0.f;
      for (int i = 0; i < nl; ++i) ls += s_lz[i];
      s_lsum = ls;
      rowloss[n] = lse - ls / (float)nl;
    }
  }
  __syncthreads();
  const float lse = s_lse, invB = 1.f / (float)B;
  if (one) gather_labels();   // in flight with the dZ stores below; the barrier before the
                              // label fix-up orders them
  if (dZb) {   // bf16 dZ, with dZl its bf16x3 lo half (fp32 path, R14)
    bf16* d = dZb + (int64_t)n * ldz;
    bf16* dl = dZl ? dZl + (int64_t)n * ldz : nullptr;
    for (int64_t j0 = threadIdx.x; j0 < L; j0 += (int64_t)kSU * blockDim.x) {
      float v[kSU];
#pragma unroll
      for (int k = 0; k < kSU; ++k) {
        const int64_t j = j0 + (int64_t)k * blockDim.x;
        v[k] = one ? zv[k] : (j < L ? z[j] : 0.f);
      }
#pragma unroll
      for (int k = 0; k < kSU; ++k) {
        const int64_t j = j0 + (int64_t)k * blockDim.x;
        if (j < L) {
          const float g = __expf(v[k] - lse) * invB;
          d[j] = __float2bfloat16_rn(g);
          if (dl) dl[j] = __float2bfloat16_rn(bf16_lo_of(g));
        }
      }
    }
    __syncthreads();
    if (one && threadIdx.x == 0) {   // the row loss, same order as above
      float ls = 0.f;
      for (int i = 0; i < nl; ++i) ls += s_lz[i];
      rowloss[n] = lse - ls / (float)nl;
    }
    for (int i = threadIdx.x; i < nl; i += blockDim.x) {
      const float g = (__expf(s_lz[i] - lse) - 1.f / (float)nl) * invB;
      d[s_lab[i]] = __float2bfloat16_rn(g);
      if (dl) dl[s_lab[i]] = __float2bfloat16_rn(bf16_lo_of(g));
    }
  } else {
    for (int64_t j0 = threadIdx.x; j0 < L; j0 += (int64_t)kSU * blockDim.x) {
      float v[kSU];
#pragma unroll
      for (int k = 0; k < kSU; ++k) {
        const int64_t j = j0 + (int64_t)k * blockDim.x;
        v[k] = j < L ? z[j] : 0.f;
      }
#pragma unroll
      for (int k = 0; k < kSU; ++k) {
        const int64_t j = j0 + (int64_t)k * blockDim.x;
        if (j < L) z[j] = __expf(v[k] - lse) * invB;
      }
    }
    __syncthreads();
    for (int i = threadIdx.x; i < nl; i += blockDim.x)
      z[s_lab[i]] = (__expf(s_lz[i] - lse) - 1.f / (float)nl) * invB;
  }
}

// ------------------------------------------------------- sigmoid + BCE (R11)
// One CTA per batch row n (fp32 path, Z stored): per-label binary cross-entropy
// with 0/1 targets, loss_n = sum_j softplus(Z_nj) - sum_{y in Y_n} Z_ny;
// dZ_nj = (sigmoid(Z_nj) - Y_nj) / B, written in place (or as bf16).
__device__ __forceinline__ float softplus_f(float z) { return fmaxf(z, 0.f) + log1pf(expf(-fabsf(z))); }
__device__ __forceinline__ float sigmoid_f(float z) {
  const float e = expf(-fabsf(z));
  return z >= 0.f ? 1.f / (1.f + e) : e / (1.f + e);
}
// sigmoid(z) - 1/2 without cancellation: (1 - e) / (2 (1 + e)), e = exp(-|z|), sign of z
__device__ __forceinline__ float sigmoid_c(float z) {
  const float e = expf(-fabsf(z));
  const float c = 0.5f * (1.f - e) / (1.f + e);
  return z >= 0.f ? c : -c;
}

__global__ void __launch_bounds__(512) k_sigmoid_ce(int B, int64_t L, int64_t ldz,
                                                    const int32_t* __restrict__ rows,
                                                    const int64_t* __restrict__ lab_ptr,
                                                    const int32_t* __restrict__ lab, float* Z,
                                                    bf16* dZb, bf16* dZl, float* rowloss) {
  Tl tl_(TL_SOFTMAX);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  __shared__ int s_lab[kMaxRowLabels];
  __shared__ float s_lz[kMaxRowLabels];
  __shared__ float s_sp[16];
  // dZl (bf16x3 fp32 path, R14): dZ is stored CENTRED as hi + lo of (sigmoid(Z) - 1/2 - Y) / B,
  // as on the bf16 path (R11): the z-dependent part of sigmoid near 1/2 would otherwise sit
  // below the split's 2^-17 relative precision; the offsets come back through k_sig_center
  const bool centred = dZl != nullptr;
  const int n = blockIdx.x;
  const int64_t id = rows[n];
  const int64_t l0 = lab_ptr[id];
  const int64_t nl64 = lab_ptr[id + 1] - l0;
  const int nl = (int)(nl64 < kMaxRowLabels ? nl64 : kMaxRowLabels);
  float* z = Z + (int64_t)n * ldz;
  for (int i = threadIdx.x; i < nl; i += blockDim.x) {
    const int y = lab[l0 + i];
    s_lab[i] = y;
    s_lz[i] = z[y];
  }
  __syncthreads();   // label logits are read before dZ overwrites Z
  const float invB = 1.f / (float)B;
  constexpr int kSU = 8;
  float sp = 0.f;
  bf16* d = dZb ? dZb + (int64_t)n * ldz : nullptr;
  for (int64_t j0 = threadIdx.x; j0 < L; j0 += (int64_t)kSU * blockDim.x) {
    float v[kSU];
#pragma unroll
    for (int k = 0; k < kSU; ++k) {
      const int64_t j = j0 + (int64_t)k * blockDim.x;
      v[k] = j < L ? z[j] : 0.f;
    }
#pragma unroll
    for (int k = 0; k < kSU; ++k) {
      const int64_t j = j0 + (int64_t)k * blockDim.x;
      if (j < L) {
        sp += softplus_f(v[k]);
        if (centred) {
          const float g = sigmoid_c(v[k]) * invB;
          d[j] = __float2bfloat16_rn(g);
          dZl[(int64_t)n * ldz + j] = __float2bfloat16_rn(bf16_lo_of(g));
        } else {
          const float g = sigmoid_f(v[k]) * invB;
          if (d) d[j] = __float2bfloat16_rn(g); else z[j] = g;
        }
      }
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) sp += __shfl_xor_sync(kFull, sp, o);
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) s_sp[wid] = sp;
  __syncthreads();
  if (threadIdx.x == 0) {
    float S = 0.f, ls = 0.f;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) S += s_sp[w];
    for (int i = 0; i < nl; ++i) ls += s_lz[i];
    rowloss[n] = S - ls;
  }
  __syncthreads();   // the label columns' non-label values are written before they are replaced
  for (int i = threadIdx.x; i < nl; i += blockDim.x) {
    if (centred) {
      const float g = (sigmoid_c(s_lz[i]) - 1.f) * invB;
      d[s_lab[i]] = __float2bfloat16_rn(g);
      dZl[(int64_t)n * ldz + s_lab[i]] = __float2bfloat16_rn(bf16_lo_of(g));
    } else {
      const float g = (sigmoid_f(s_lz[i]) - 1.f) * invB;
      if (d) d[s_lab[i]] = __float2bfloat16_rn(g); else z[s_lab[i]] = g;
    }
  }
}

// Row loss of the fused sigmoid path: rowloss[n] = sum over G1's column tiles t
// of the per-(tile half, row) BCE partials stats[t][n].x, in tile order.
__global__ void __launch_bounds__(256) k_tile_loss(int ntiles, int64_t stats_ld, const float2* __restrict__ stats,
                                                   float* rowloss) {
  Tl tl_(TL_SOFTMAX);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  __shared__ float s_w[8];
  const int n = blockIdx.x;
  float a = 0.f;
  for (int t = threadIdx.x; t < ntiles; t += blockDim.x) a += stats[(int64_t)t * stats_ld + n].x;
#pragma unroll
  for (int o = 16; o; o >>= 1) a += __shfl_xor_sync(kFull, a, o);
  if ((threadIdx.x & 31) == 0) s_w[threadIdx.x >> 5] = a;
  __syncthreads();
  if (threadIdx.x == 0) {
    float S = 0.f;
    for (int w = 0; w < 8; ++w) S += s_w[w];
    rowloss[n] = S;
  }
}

// ------------------------------------------ centred sigmoid dZ offsets (R11)
// G1 stores dZc = dZ - 1/(2B) (bf16 keeps the z-dependent part near sigmoid = 1/2);
// the constant comes back exactly through
//   dH1 = dZc W2 + (1/(2B)) 1 (1^T W2)     -> cen[0:H]  = (1/(2B)) sum_j W2_j
//   dW2 = dZc^T H1 + (1/(2B)) 1 (1^T H1)   -> cen[H:2H] = (1/(2B)) sum_n H1_n
// (db2's + 1/2 is G3's).  W2 is the bf16 shadow G2 multiplies with.  Phase 1: each
// CTA sums a contiguous label range (8 columns per thread, 16-B loads, 4 in
// flight); phase 2: the last CTA adds the partials in CTA order (deterministic).
__global__ void __launch_bounds__(256) k_sig_center(const bf16* __restrict__ w2b, const float* __restrict__ w2f,
                                                    int64_t L, int H, const float* __restrict__ h1, int n,
                                                    float* part, unsigned int* counter, float* cen) {
  Tl tl_(TL_OTHER);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  __shared__ float s_acc[8][512];
  __shared__ bool s_last;
  const int tpr = H / 8;                   // threads per W2 row (H <= 512 -> <= 64)
  const int rows_per_it = 256 / tpr;
  const int c8 = (threadIdx.x % tpr) * 8, r0 = threadIdx.x / tpr;
  const int64_t j0 = (int64_t)blockIdx.x * L / gridDim.x, j1 = (int64_t)(blockIdx.x + 1) * L / gridDim.x;
  float a[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
  int64_t j = j0 + r0;
  if (w2f) {   // bf16x3 fp32 path (R14): the offset from the fp32 W2
    for (; j < j1; j += rows_per_it) {
      const float4 u0 = __ldcs(reinterpret_cast<const float4*>(w2f + j * H + c8));
      const float4 u1 = __ldcs(reinterpret_cast<const float4*>(w2f + j * H + c8 + 4));
      a[0] += u0.x; a[1] += u0.y; a[2] += u0.z; a[3] += u0.w;
      a[4] += u1.x; a[5] += u1.y; a[6] += u1.z; a[7] += u1.w;
    }
  }
  for (; j + 3 * rows_per_it < j1; j += 4 * rows_per_it) {
    uint4 u[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) u[q] = __ldcs(reinterpret_cast<const uint4*>(w2b + (j + q * rows_per_it) * H + c8));
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const __nv_bfloat162* b = reinterpret_cast<const __nv_bfloat162*>(&u[q]);
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const float2 f = __bfloat1622float2(b[i]);
        a[2 * i] += f.x; a[2 * i + 1] += f.y;
      }
    }
  }
  for (; j < j1; j += rows_per_it) {
    const uint4 u = __ldcs(reinterpret_cast<const uint4*>(w2b + j * H + c8));
    const __nv_bfloat162* b = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const float2 f = __bfloat1622float2(b[i]);
      a[2 * i] += f.x; a[2 * i + 1] += f.y;
    }
  }
  // combine the rows_per_it row groups of this CTA in fixed order
  const int grp = r0 & 7, sub = r0 >> 3;   // <= 8 groups per pass
  for (int pass = 0; pass * 8 < rows_per_it; ++pass) {
    if (sub == pass)
      for (int i = 0; i < 8; ++i) s_acc[grp][c8 + i] = (pass == 0 ? 0.f : s_acc[grp][c8 + i]) + a[i];
    __syncthreads();
  }
  // this CTA's slice of the batch rows of H1 (fp32), rows in order
  const int n0 = (int)((int64_t)blockIdx.x * n / gridDim.x), n1 = (int)((int64_t)(blockIdx.x + 1) * n / gridDim.x);
  float* part2 = part + (int64_t)gridDim.x * H;
  for (int c = threadIdx.x; c < H; c += blockDim.x) {
    float t = 0.f;
    for (int g = 0; g < min(8, rows_per_it); ++g) t += s_acc[g][c];
    part[(int64_t)blockIdx.x * H + c] = t;
    float hs = 0.f;
    for (int r = n0; r < n1; ++r) hs += h1[(int64_t)r * H + c];
    part2[(int64_t)blockIdx.x * H + c] = hs;
  }
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) s_last = atomicAdd(counter, 1u) == gridDim.x - 1;
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  const float o = 0.5f / (float)n;
  for (int c = threadIdx.x; c < 2 * H; c += blockDim.x) {   // both sums, partials in CTA order
    const float* pp = (c < H ? part : part2) + (c % H);
    float t[4] = {0.f, 0.f, 0.f, 0.f};
    int b = 0;
    for (; b + 4 <= (int)gridDim.x; b += 4) {
#pragma unroll
      for (int q = 0; q < 4; ++q) t[q] += __ldcg(pp + (int64_t)(b + q) * H);
    }
    for (; b < (int)gridDim.x; ++b) t[0] += __ldcg(pp + (int64_t)b * H);
    cen[c] = o * ((t[0] + t[1]) + (t[2] + t[3]));
  }
  if (threadIdx.x == 0) *counter = 0u;
}

// ------------------------------------------------------------ fused CE: lse
// lse_n from G1's per-tile (max, sum exp) partials; the label logits
// Z_ny = H1_n . W2_y + b2_y (bf16 operands, fp32 sum, as on the tensor cores);
// row loss = lse_n - mean_y Z_ny (Q3, Q4).  One CTA per row.
__global__ void __launch_bounds__(256) k_lse(int H, int ntiles, int64_t stats_ld, const float2* __restrict__ stats,
                                             const int32_t* __restrict__ rows, const int64_t* __restrict__ lab_ptr,
                                             const int32_t* __restrict__ lab, const bf16* __restrict__ h1b,
                                             const bf16* __restrict__ w2b, const float* __restrict__ b2,
                                             float* lse, float* rowloss) {
  Tl tl_(TL_SOFTMAX);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  __shared__ float s_m[8], s_s[8], s_z[8];
  const int n = blockIdx.x, lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  float m = -INFINITY, s = 0.f;
  for (int t = threadIdx.x; t < ntiles; t += blockDim.x) {
    const float2 p = stats[(int64_t)t * stats_ld + n];
    if (p.x == -INFINITY) continue;
    if (p.x > m) { s = (m == -INFINITY ? 0.f : s * __expf(m - p.x)) + p.y; m = p.x; }
    else s += p.y * __expf(p.x - m);
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const float om = __shfl_xor_sync(kFull, m, o), os = __shfl_xor_sync(kFull, s, o);
    const float nm = fmaxf(m, om);
    s = (m == -INFINITY ? 0.f : s * __expf(m - nm)) + (om == -INFINITY ? 0.f : os * __expf(om - nm));
    m = nm;
  }
  // label logits: warp w takes labels w, w + 8, ...
  const int64_t id = rows[n];
  const int64_t l0 = lab_ptr[id], l1 = lab_ptr[id + 1];
  float zs = 0.f;
  for (int64_t i = l0 + wid; i < l1; i += 8) {
    const int y = lab[i];
    float d = 0.f;
    for (int k = lane * 2; k < H; k += 64) {
      const float2 a = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(h1b + (int64_t)n * H + k));
      const float2 b = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(w2b + (int64_t)y * H + k));
      d = fmaf(a.x, b.x, fmaf(a.y, b.y, d));
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) d += __shfl_xor_sync(kFull, d, o);
    zs += d + b2[y];
  }
  if (lane == 0) { s_m[wid] = m; s_s[wid] = s; s_z[wid] = zs; }
  __syncthreads();
  if (threadIdx.x == 0) {
    float M = -INFINITY, S = 0.f, Zs = 0.f;
    for (int w = 0; w < 8; ++w) M = fmaxf(M, s_m[w]);
    for (int w = 0; w < 8; ++w) {
      S += (s_m[w] == -INFINITY) ? 0.f : s_s[w] * __expf(s_m[w] - M);
      Zs += s_z[w];
    }
    const float l = M + logf(S);
    lse[n] = l;
    rowloss[n] = l - Zs / (float)(l1 - l0);
  }
}

// ------------------------------------------------------ dH1 reduce + ReLU'
// dA1[r][c] = [H1[r][c] > 0] * sum_z part[z][r][c]: one thread per element, its
// split-K loads all in flight; fixed summation order (deterministic).
__global__ void k_dh_reduce(int n, int H, int splitk, int64_t part_stride,
                            const float* __restrict__ part, const float* __restrict__ H1, float* dA1,
                            bf16* dA1b, const float* __restrict__ dh_off) {
  Tl tl_(TL_DH);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const int r = blockIdx.x, c = threadIdx.x;
  const int64_t o = (int64_t)r * H + c;
  float a[8];
#pragma unroll
  for (int q = 0; q < 8; ++q) a[q] = 0.f;
  for (int z = 0; z < splitk; z += 8) {
#pragma unroll
    for (int q = 0; q < 8; ++q)
      if (z + q < splitk) a[q] += __ldcs(part + (int64_t)(z + q) * part_stride + o);
  }
  float s = ((a[0] + a[1]) + (a[2] + a[3])) + ((a[4] + a[5]) + (a[6] + a[7]));
  if (dh_off) s += dh_off[c];   // centred sigmoid dZ: + (1/(2B)) sum_j W2_j
  const float v = H1[o] > 0.f ? s : 0.f;
  dA1[o] = v;
  if (dA1b) dA1b[o] = __float2bfloat16_rn(v);
}

// db1[c] = sum_r dA1[r][c] (one warp per column, lanes over rows, fixed shuffle
// tree); b1 -= lr db1.  The extra last warp computes the mean loss.
__global__ void __launch_bounds__(256) k_b1_update(int n, int H, const float* __restrict__ dA1, float* b1,
                                                   const int32_t* __restrict__ meta, float* grad_b1,
                                                   const float* __restrict__ rowloss) {
  Tl tl_(TL_B1);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  const float lr = step_lr(meta);
  float* loss_dev = step_loss(meta);
  const int lane = threadIdx.x & 31;
  const int c = blockIdx.x * 8 + (threadIdx.x >> 5);
  if (c < H) {
    float t[4] = {0.f, 0.f, 0.f, 0.f};
    int r = lane;
    for (; r + 96 < n; r += 128) {
#pragma unroll
      for (int q = 0; q < 4; ++q) t[q] += dA1[(int64_t)(r + 32 * q) * H + c];
    }
    for (; r < n; r += 32) t[0] += dA1[(int64_t)r * H + c];
    float v = (t[0] + t[1]) + (t[2] + t[3]);
#pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    if (lane == 0) {
      b1[c] -= lr * v;
      if (grad_b1) grad_b1[c] = v;
    }
  } else if (c == H && loss_dev) {
    float t = 0.f;
    for (int r = lane; r < n; r += 32) t += rowloss[r];
#pragma unroll
    for (int o = 16; o; o >>= 1) t += __shfl_xor_sync(kFull, t, o);
    if (lane == 0) *loss_dev = t / (float)n;
  }
}

__global__ void k_to_bf16(const float* __restrict__ src, bf16* dst, bf16* dst_lo, int64_t count) {
  Tl tl_(TL_OTHER);
  pdl_trigger();
  pdl_wait();
  tl_.ready();
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
       i += (int64_t)gridDim.x * blockDim.x) {
    const float x = src[i];
    dst[i] = __float2bfloat16_rn(x);
    if (dst_lo) dst_lo[i] = __float2bfloat16_rn(bf16_lo_of(x));
  }
}

}  // namespace

cudaError_t launch_softmax_ce(const Launch& lc, int n, int64_t L, int64_t ldz, const int32_t* rows,
                              const int64_t* lab_ptr, const int32_t* lab, const Ptrs& P,
                              bool bf16_out, const float2* stats, int ntiles, int64_t stats_ld) {
  launch_k(lc, k_softmax_ce, dim3(n), dim3(512), 0, n, L, ldz, rows, lab_ptr, lab, P.z, bf16_out ? P.dzb : nullptr,
           bf16_out ? P.dzl : nullptr, P.rowloss, stats, ntiles, stats_ld);
  return cudaGetLastError();
}

cudaError_t launch_sigmoid_ce(const Launch& lc, int n, int64_t L, int64_t ldz, const int32_t* rows,
                              const int64_t* lab_ptr, const int32_t* lab, const Ptrs& P, bool bf16_out) {
  launch_k(lc, k_sigmoid_ce, dim3(n), dim3(512), 0, n, L, ldz, rows, lab_ptr, lab, P.z, bf16_out ? P.dzb : nullptr,
           bf16_out ? P.dzl : nullptr, P.rowloss);
  return cudaGetLastError();
}

cudaError_t launch_tile_loss(const Launch& lc, int n, int ntiles, int64_t stats_ld, const float2* stats, const Ptrs& P) {
  return launch_k(lc, k_tile_loss, dim3(n), dim3(256), 0, ntiles, stats_ld, stats, P.rowloss);
}

cudaError_t launch_sig_center(const Launch& lc, const bf16* w2b, const float* w2f, int64_t L, int H, const float* h1,
                              int n, float* part, unsigned int* counter, float* cen) {
  return launch_k(lc, k_sig_center, dim3(kCenterParts), dim3(256), 0, w2b, w2f, L, H, h1, n, part, counter, cen);
}

cudaError_t launch_lse(const Launch& lc, int n, int H, int ntiles, int64_t stats_ld, const float2* stats,
                       const int32_t* rows, const int64_t* lab_ptr, const int32_t* lab, const bf16* h1b,
                       const bf16* w2b, const float* b2, const Ptrs& P) {
  return launch_k(lc, k_lse, dim3(n), dim3(256), 0, H, ntiles, stats_ld, stats, rows, lab_ptr, lab, h1b, w2b, b2,
                  P.lse, P.rowloss);
}

cudaError_t launch_dh_reduce(const Launch& lc, int n, int H, int splitk, const Ptrs& P,
                             const WsLayout& L, bool want_bf16, const float* dh_off) {
  // split-K partial z of dH1 lives at dhpart + z * (b_max * H)
  launch_k(lc, k_dh_reduce, dim3(n), dim3(H), 0, n, H, splitk, L.part_stride, P.dhpart, P.h1, P.da1,
                  want_bf16 ? P.da1b : nullptr, dh_off);
  return cudaGetLastError();
}

cudaError_t launch_b1_update(const Launch& lc, int n, int H, float* b1, const Ptrs& P,
                             const WsLayout& L, float* grad_b1) {
  launch_k(lc, k_b1_update, dim3(H / 8 + 1), dim3(256), 0, n, H, P.da1, b1, P.meta, grad_b1, P.rowloss);
  return cudaGetLastError();
}

cudaError_t launch_to_bf16(const Launch& lc, const float* src, bf16* dst, int64_t count, bf16* dst_lo) {
  const int64_t blocks = std::min<int64_t>((count + 255) / 256, (int64_t)lc.sms * 16);
  launch_k(lc, k_to_bf16, dim3((int)std::max<int64_t>(blocks, 1)), dim3(256), 0, src, dst, dst_lo, count);
  return cudaGetLastError();
}

int row_block() { return 1; }

}  // namespace asgd


namespace asgd {
ASGD_TL_SETTER(tl_set_dense)
}  // namespace asgd
