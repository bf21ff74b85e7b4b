// Microbenchmark: EURLex-shaped W1 row gathers (B = 256 rows x ~237 nnz, F = 5000, H = 256).
// Times variants of the K-1 inner loop in isolation (warm L2, CUDA events).
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1);} } while (0)

__global__ void k_empty() {}

// each warp: PIECE entries; lanes own 8 columns (2 x float4); UNROLL rows in flight
template <int PIECE, int UNROLL>
__global__ void __launch_bounds__(256, 1) k_gather(const int* __restrict__ col, const float* __restrict__ val, int nnz,
                                                   const float* __restrict__ W1, float* out) {
  const int lane = threadIdx.x & 31;
  const int nw = gridDim.x * (blockDim.x >> 5);
  const int np = (nnz + PIECE - 1) / PIECE;
  for (int p = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); p < np; p += nw) {
    const int e0 = p * PIECE, cnt = min(PIECE, nnz - e0);
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (int jb = 0; jb < cnt; jb += 32) {
      int mc = 0; float mv = 0.f;
      if (jb + lane < cnt) { mc = col[e0 + jb + lane]; mv = val[e0 + jb + lane]; }
      const int c2 = min(32, cnt - jb);
      for (int j0 = 0; j0 < c2; j0 += UNROLL) {
        float4 w[UNROLL][2];
#pragma unroll
        for (int q = 0; q < UNROLL; ++q) {
          const int c = __shfl_sync(~0u, mc, j0 + q);
          if (j0 + q < c2) {
            w[q][0] = __ldg(reinterpret_cast<const float4*>(W1 + (size_t)c * 256) + lane);
            w[q][1] = __ldg(reinterpret_cast<const float4*>(W1 + (size_t)c * 256 + 128) + lane);
          } else { w[q][0] = w[q][1] = make_float4(0, 0, 0, 0); }
        }
#pragma unroll
        for (int q = 0; q < UNROLL; ++q) {
          const float v = __shfl_sync(~0u, mv, j0 + q);
          acc[0] += v * w[q][0].x; acc[1] += v * w[q][0].y; acc[2] += v * w[q][0].z; acc[3] += v * w[q][0].w;
          acc[4] += v * w[q][1].x; acc[5] += v * w[q][1].y; acc[6] += v * w[q][1].z; acc[7] += v * w[q][1].w;
        }
      }
    }
    float4* o = reinterpret_cast<float4*>(out + (size_t)p * 256);
    o[lane] = make_float4(acc[0], acc[1], acc[2], acc[3]);
    o[lane + 32] = make_float4(acc[4], acc[5], acc[6], acc[7]);
  }
}

// CTA-per-row-chunk variant: 4 groups of 64 threads; thread owns 4 columns (float4); group g takes entries g, g+4, ...
template <int UNROLL>
__global__ void __launch_bounds__(256) k_gather_cta(const int* __restrict__ rowoff, const int* __restrict__ col,
                                                    const float* __restrict__ val, const float* __restrict__ W1, float* out) {
  __shared__ float4 red[4][64];
  const int r = blockIdx.x, g = threadIdx.x >> 6, t = threadIdx.x & 63;
  const int s = rowoff[r], e = rowoff[r + 1];
  float4 acc = make_float4(0, 0, 0, 0);
  for (int j0 = s + g; j0 < e; j0 += 4 * UNROLL) {
    float4 w[UNROLL]; float v[UNROLL];
#pragma unroll
    for (int q = 0; q < UNROLL; ++q) {
      const int j = j0 + 4 * q;
      if (j < e) { const int c = __ldg(col + j); v[q] = __ldg(val + j); w[q] = __ldg(reinterpret_cast<const float4*>(W1 + (size_t)c * 256) + t); }
      else { v[q] = 0; w[q] = make_float4(0, 0, 0, 0); }
    }
#pragma unroll
    for (int q = 0; q < UNROLL; ++q) { acc.x += v[q] * w[q].x; acc.y += v[q] * w[q].y; acc.z += v[q] * w[q].z; acc.w += v[q] * w[q].w; }
  }
  red[g][t] = acc;
  __syncthreads();
  if (g == 0) {
    float4 a = red[0][t], b = red[1][t], c = red[2][t], d = red[3][t];
    reinterpret_cast<float4*>(out + (size_t)r * 256)[t] =
        make_float4(a.x + b.x + c.x + d.x, a.y + b.y + c.y + d.y, a.z + b.z + c.z + d.z, a.w + b.w + c.w + d.w);
  }
}

int main() {
  const int B = 256, F = 5000, H = 256;
  std::vector<int> off(B + 1), cols; std::vector<float> vals;
  srand(1);
  // Zipf(1)-ish features, ~237 distinct per row
  std::vector<double> cdf(F); double z = 0; for (int f = 0; f < F; ++f) { z += 1.0 / (f + 1); cdf[f] = z; }
  for (int r = 0; r < B; ++r) {
    off[r] = cols.size();
    int s = 120 + rand() % 240;
    std::vector<int> row;
    while ((int)row.size() < s) {
      double u = (rand() / (double)RAND_MAX) * z;
      int f = std::lower_bound(cdf.begin(), cdf.end(), u) - cdf.begin();
      f = (int)(((long long)f * 2654435761ll) % F);
      if (std::find(row.begin(), row.end(), f) == row.end()) row.push_back(f);
    }
    std::sort(row.begin(), row.end());
    for (int f : row) { cols.push_back(f); vals.push_back(0.1f); }
  }
  off[B] = cols.size();
  const int nnz = cols.size();
  printf("nnz %d\n", nnz);
  int *dcol, *doff; float *dval, *dW, *dout;
  CK(cudaMalloc(&dcol, nnz * 4)); CK(cudaMalloc(&dval, nnz * 4)); CK(cudaMalloc(&doff, (B + 1) * 4));
  CK(cudaMalloc(&dW, (size_t)F * H * 4)); CK(cudaMalloc(&dout, (size_t)(nnz + 64) * H * 4));
  CK(cudaMemcpy(dcol, cols.data(), nnz * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dval, vals.data(), nnz * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(doff, off.data(), (B + 1) * 4, cudaMemcpyHostToDevice));
  CK(cudaMemset(dW, 0, (size_t)F * H * 4));
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  auto timeit = [&](const char* name, auto fn) {
    for (int i = 0; i < 20; ++i) fn();
    CK(cudaDeviceSynchronize());
    const int R = 200;
    cudaEventRecord(a);
    for (int i = 0; i < R; ++i) fn();
    cudaEventRecord(b);
    CK(cudaEventSynchronize(b));
    float ms; cudaEventElapsedTime(&ms, a, b);
    printf("%-40s %8.2f us/launch (back-to-back)\n", name, ms * 1e3 / R);
  };
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  timeit("empty<<<1,32>>>", [&] { k_empty<<<1, 32>>>(); });
  timeit("empty<<<444,256>>>", [&] { k_empty<<<444, 256>>>(); });
  auto G = [&](int piece, int ctas) { return std::min(ctas, ((nnz + piece - 1) / piece + 7) / 8); };
  timeit("gather piece32 u8  grid=np/8", [&] { k_gather<32, 8><<<G(32, 10000), 256>>>(dcol, dval, nnz, dW, dout); });
  timeit("gather piece32 u16 grid=np/8", [&] { k_gather<32, 16><<<G(32, 10000), 256>>>(dcol, dval, nnz, dW, dout); });
  timeit("gather piece32 u8  grid=148", [&] { k_gather<32, 8><<<sms, 256>>>(dcol, dval, nnz, dW, dout); });
  timeit("gather piece16 u8  grid=np/8", [&] { k_gather<16, 8><<<G(16, 10000), 256>>>(dcol, dval, nnz, dW, dout); });
  timeit("gather piece16 u16 grid=np/8", [&] { k_gather<16, 16><<<G(16, 10000), 256>>>(dcol, dval, nnz, dW, dout); });
  timeit("gather piece64 u8  grid=np/8", [&] { k_gather<64, 8><<<G(64, 10000), 256>>>(dcol, dval, nnz, dW, dout); });
  timeit("gather piece8  u8  grid=np/8", [&] { k_gather<8, 8><<<G(8, 10000), 256>>>(dcol, dval, nnz, dW, dout); });
  timeit("cta-per-row u4", [&] { k_gather_cta<4><<<B, 256>>>(doff, dcol, dval, dW, dout); });
  timeit("cta-per-row u8", [&] { k_gather_cta<8><<<B, 256>>>(doff, dcol, dval, dW, dout); });
  timeit("cta-per-row u16", [&] { k_gather_cta<16><<<B, 256>>>(doff, dcol, dval, dW, dout); });
  // single launches with sync between (latency incl. launch)
  auto single = [&](const char* name, auto fn) {
    for (int i = 0; i < 5; ++i) fn();
    CK(cudaDeviceSynchronize());
    float tot = 0;
    for (int i = 0; i < 50; ++i) {
      cudaEventRecord(a); fn(); cudaEventRecord(b); CK(cudaEventSynchronize(b));
      float ms; cudaEventElapsedTime(&ms, a, b); tot += ms;
    }
    printf("%-40s %8.2f us (isolated, event-bracketed)\n", name, tot * 1e3 / 50);
  };
  single("empty<<<1,32>>>", [&] { k_empty<<<1, 32>>>(); });
  single("gather piece32 u8", [&] { k_gather<32, 8><<<G(32, 10000), 256>>>(dcol, dval, nnz, dW, dout); });
  single("gather piece16 u8", [&] { k_gather<16, 8><<<G(16, 10000), 256>>>(dcol, dval, nnz, dW, dout); });
  single("cta-per-row u8", [&] { k_gather_cta<8><<<B, 256>>>(doff, dcol, dval, dW, dout); });
  return 0;
}
