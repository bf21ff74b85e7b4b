// tcgen05 tensor-core GEMMs of the bf16 path (sm_100a): the three dense
// contractions of the output layer (§V-A: the 3-layer
// MLP's hidden->output layer; rows a4 and a6 of DESIGN.md):
//   G1  Z[B x L]   = H1[B x H] . W2[L x H]^T + b2        (A, B K-major)
//   G2  dH1[B x H] = dZ[B x L] . W2[L x H]   (split-K)    (A K-major, B MN-major)
//   G3  W2 -= lr dZ[B x L]^T . H1[B x H]    (fused SGD)  (A, B MN-major)
// bf16 operands staged by TMA (128B swizzle) in a 4-stage mbarrier ring,
// one elected thread issues tcgen05.mma (M = 128, N = BN, K = 16) into a TMEM
// accumulator, four epilogue warps drain TMEM with tcgen05.ld and apply the
// fused epilogue (bias, split-K partial store, or the W2 SGD update + bf16
// shadow refresh).  fp32 accumulation throughout.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>

#include "asgd_internal.h"

namespace asgd {
namespace {

constexpr int BM = 128, BK = 64;

// Z: fp32 Z store (+ softmax partials); PART: split-K partial store; SGD: W2 update;
// DZ: softmax dZ (bf16); SIG: sigmoid dZ (bf16) + BCE partials; STATS: softmax partials only
enum { TC_EPI_Z = 0, TC_EPI_PART = 1, TC_EPI_SGD = 2, TC_EPI_DZ = 3, TC_EPI_SIG = 4, TC_EPI_STATS = 5 };

struct TcArgs {
  int M, N, K;
  // epilogue
  float* out; int64_t ldo;            // Z (ldo = Lp) / partials (ldo = H) / W2 (ldo = H)
  int64_t part_stride;                // split-K partial z offset
  const float* bias;                  // G1
  const int32_t* meta; bf16* shadow; float* grad;// G3 (lr = meta[M_LR])
  bf16* shadow_lo;                    // G3, bf16x3 (R14): the lo half of the new W2 shadow
  float* b2; float* grad_b2;          // G3: db2 = dZ^T 1 via an extra N = 16 MMA on N-tile 0
  float2* stats; int64_t stats_ld;    // G1: per (N-tile half, row) softmax partials (max, sum exp)
  int splits;                         // split-K factor (tiles = M tiles x N tiles x splits)
  int n_fast;                         // tile order: N tiles vary fastest (else M tiles)
  int chunked;                        // CTA c runs the contiguous tiles [c T / G, (c + 1) T / G) in
                                      // M-major order (N fastest): its rows change at most once or
                                      // twice, and the G CTAs sweep the N tiles in lockstep per M
                                      // tile, so every W2 tile is read from HBM about once
  int write_z;                        // G1: store Z (eval) or only the softmax partials (step)
  // G3, centred sigmoid dZ (R11): dW2 += hoff (per H column: (1/(2B)) sum_n H1_n), db2 += db2_off
  const float* hoff; float db2_off;
  // G1b (TC_EPI_DZ): dZ = (exp(Z - lse) - T) / B recomputed from the MMA, stored bf16;
  // G1 sigmoid (TC_EPI_SIG): dZ = (sigmoid(Z) - Y) / B, BCE row partials in stats
  const float* lse; const int32_t* rows; const int64_t* lab_ptr; const int32_t* lab; float invB;
  // G2 fused with the dH1 reduce (DH_FUSE): after a grid barrier, CTA k sums the split-K
  // partials of its (row block, column block), applies ReLU' (dA1 = dH1 [H1 > 0]), writes
  // dA1 (fp32, + bf16) and its column sums; the last CTA applies b1 -= lr db1 and the mean loss
  int dh_fuse;
  const float* h1; float* da1; bf16* da1b; const float* dh_off;
  float* b1; float* grad_b1; float* colpart; const float* rowloss; int32_t* bar;
  // K-3 one-pass (k_bwd_dh): the softmax statistics come from a first sweep of S tiles
  // (recomputed in the second): per (label range, row) partials (max2, sum
  // 2^(t - max2)) in stats[lr][row], then the label-logit sums as floats [lr][row];
  // after a grid barrier lse -> g.lse, row loss -> rowloss_w
  int one_pass; float* rowloss_w;
  // K-3 softmax-only (dz_only, implies one_pass): no MMA 2 / dH1 partials / reduce tail --
  // the kernel stands for G1 + softmax-CE (dZ TMA-stored, row losses), G2 follows it
  int dz_only; unsigned long long* gbar;   // packed grid barrier (generation << 32 | count)
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  uint32_t ok = 0;
  while (!ok) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(a), "r"(parity), "r"(1000000u)   // suspend up to 1 ms instead of spinning on issue slots
        : "memory");
  }
}

__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0,
                                            int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
      : "memory");
}

__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}

// SM100 shared-memory matrix descriptor, 128B swizzle.
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
  d |= (uint64_t)1 << 46;  // descriptor version (sm_100)
  d |= (uint64_t)2 << 61;  // SWIZZLE_128B
  return d;
}

// Instruction descriptor: kind::f16, bf16 x bf16 -> f32, M = 128.
__host__ __device__ constexpr uint32_t make_idesc(int N, bool a_mn, bool b_mn) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((a_mn ? 1u : 0u) << 15) | ((b_mn ? 1u : 0u) << 16) |
         ((uint32_t)(N >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

__device__ __forceinline__ void mma_bf16(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t idesc,
                                         uint32_t accum) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(accum)
      : "memory");
}

__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float (&v)[32]) {
  uint32_t r[32];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
      "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]),
        "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]),
        "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}

// Asynchronous variant: the 32 registers are written when tcgen05.wait::ld retires;
// tmem_wait_regs() waits and then ties the registers to that point (empty asm with
// "+r"), so no use can be scheduled before the wait.
__device__ __forceinline__ void tmem_ld32_async(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, "
      "%16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]),
        "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]),
        "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_regs(uint32_t (&r)[32]) {
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
  asm volatile(""
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]), "+r"(r[6]),
                 "+r"(r[7]), "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]), "+r"(r[12]), "+r"(r[13]),
                 "+r"(r[14]), "+r"(r[15]), "+r"(r[16]), "+r"(r[17]), "+r"(r[18]), "+r"(r[19]), "+r"(r[20]),
                 "+r"(r[21]), "+r"(r[22]), "+r"(r[23]), "+r"(r[24]), "+r"(r[25]), "+r"(r[26]), "+r"(r[27]),
                 "+r"(r[28]), "+r"(r[29]), "+r"(r[30]), "+r"(r[31]));
}

__device__ __forceinline__ float ex2_approx(float x) {   // 2^x on the MUFU (ex2.approx, -inf -> 0)
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// 2^x for x <= 0 on the FMA/ALU pipes (no MUFU): round-to-nearest split x = k + f,
// f in [-1/2, 1/2] via the 1.5 * 2^23 magic add, degree-3 polynomial for 2^f (relative
// error 7.7e-5, below bf16's 2^-9 and far below the 2e-2 gradient tolerance), k added to
// the exponent field.  x is clamped at -125 (result ~2e-38, i.e. 0 in every sum it
// enters; -inf padding columns included).  The softmax epilogues are MUFU-bound at 16
// ex2/clk/SM -- exactly the tcgen05 rate of a 128 x 256 x 256 tile -- so a quarter of
// the exponentials go here instead (the FA4 split).
__device__ __forceinline__ float ex2_poly(float x) {
  x = fmaxf(x, -125.f);
  const float t = x + 12582912.f;
  const float f = x - (t - 12582912.f);
  float p = fmaf(fmaf(fmaf(0.05508868396282196f, f, 0.24260404706001282f), f, 0.6932762265205383f), f,
                 0.9999289512634277f);
  return __int_as_float(__float_as_int(p) + (__float_as_int(t) << 23));
}
#ifndef ASGD_POLY_EXP
#define ASGD_POLY_EXP 0   // measured: G1 389 -> 430 us with the split (not MUFU-throughput bound)
#endif
// every 4th exponential of the softmax epilogues on the FMA pipes (ASGD_POLY_EXP=0: all MUFU)
__device__ __forceinline__ float ex2_mix(float x) {
#if ASGD_POLY_EXP
  return ex2_poly(x);
#else
  return ex2_approx(x);
#endif
}

__device__ __forceinline__ float rcp_approx(float x) {
  float y;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// log1p(x) for x in [0, 1] on the FMA pipe: degree-8 Chebyshev fit, |error| < 2e-7
// (keeps the sigmoid epilogue at 2 MUFU ops per element: ex2 and rcp).
__device__ __forceinline__ float log1p_01(float x) {
  float p = -0.0060747526586055756f;
  p = fmaf(p, x, 0.03441791236400604f);
  p = fmaf(p, x, -0.09231230616569519f);
  p = fmaf(p, x, 0.16478188335895538f);
  p = fmaf(p, x, -0.2391897290945053f);
  p = fmaf(p, x, 0.3313336670398712f);
  p = fmaf(p, x, -0.4998010993003845f);
  p = fmaf(p, x, 0.9999914765357971f);
  return fmaf(p, x, 9.099033349002639e-08f);
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

constexpr uint32_t pow2ceil(uint32_t x) {
  uint32_t p = 32;
  while (p < x) p <<= 1;
  return p;
}

// G2's fused tail (TC_EPI_PART with g.dh_fuse, rows a6/a7 of DESIGN.md): replaces the
// k_dh_reduce and k_b1_update launches.  Every CTA of the persistent grid is resident
// (one per SM, grid <= SMs; the kernels beside it on other streams never wait for G2),
// so a software grid barrier is safe.  CTA k then owns rows [r0, r1) x columns [c0, c1)
// of dH1 (GC column blocks of >= 32 columns, GR = grid / GC row blocks):
//   dA1 = [H1 > 0] * (sum_z part[z] (+ the centred-sigmoid offset))  -> dA1 (fp32, bf16)
//   colpart[row block][c] = sum_{r in block} dA1[r][c]   (fixed order)
// and the last CTA to finish sums colpart over the row blocks in order: b1 -= lr db1,
// grad_b1 = db1, and the mean loss from the per-row losses (deterministic).
// Software grid barrier over every CTA of the launch (all resident: one per SM), one
// thread per CTA; bar[0] = arrivals, bar[1] = generation (reusable).
__device__ __forceinline__ void grid_sync_thread(int32_t* bar, int G) {
  volatile int32_t* cnt = bar;
  volatile int32_t* gen = bar + 1;
  const int32_t g0 = *gen;
  __threadfence();
  if (atomicAdd(bar, 1) == G - 1) {
    *cnt = 0;
    __threadfence();
    atomicAdd(bar + 1, 1);
  } else {
    while (*gen == g0) __nanosleep(64);
  }
  __threadfence();
}

// The same with one 64-bit word, generation << 32 | count: the last arriver resets the count
// and bumps the generation in one atomic (one round trip fewer than the two-word version).
__device__ __forceinline__ void grid_sync_packed(unsigned long long* bar, int G) {
  __threadfence();
  const unsigned long long old = atomicAdd(bar, 1ull);
  const unsigned int g0 = (unsigned int)(old >> 32);
  if ((unsigned int)(old & 0xffffffffull) == (unsigned int)(G - 1)) {
    atomicAdd(bar, (1ull << 32) - (unsigned long long)G);
  } else {
    volatile unsigned long long* vb = bar;
    while ((unsigned int)(*vb >> 32) == g0) __nanosleep(32);
  }
  __threadfence();
}

__device__ void dh_reduce_phase(const TcArgs& g, float* sred) {
  const int G = gridDim.x, k = blockIdx.x, H = g.N, n = g.M, S = g.splits;
  __shared__ int s_last;
  // (1) every CTA's partial stores are complete (each epilogue lane waited on its bulk
  // groups before the kernel's final barrier): make them visible, then the grid barrier
  asm volatile("fence.proxy.async.global;" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) grid_sync_thread(g.bar, G);
  __syncthreads();
  if (threadIdx.x == 0) TL_MARK(TL_PH7);
  // (2) this CTA's block
  int GC = H / 32;
  if (GC > G) GC = G;
  const int GR = G / GC;
  if (k >= GR * GC) {   // no block (G not a multiple of GC): still arrive at the last-CTA count
    __syncthreads();
  } else {
    const int cb = k % GC, rb = k / GC;
    const int c0 = cb * H / GC, c1 = (cb + 1) * H / GC, nc = c1 - c0;
    const int r0 = rb * n / GR, r1 = (rb + 1) * n / GR;
    const float lr = step_lr(g.meta);
    (void)lr;
    // float4 groups of 4 columns (column blocks are multiples of 32), all of a group's
    // split-K partial loads in flight (16 per round), summed in split order
    const int nc4 = nc / 4;
    for (int e = threadIdx.x; e < (r1 - r0) * nc4; e += blockDim.x) {
      const int rl = e / nc4, cl = 4 * (e % nc4);
      const int r = r0 + rl, c = c0 + cl;
      const int64_t o = (int64_t)r * H + c;
      float4 sum = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int z = 0; z < S; z += 16) {
        float4 t[16];
#pragma unroll
        for (int q = 0; q < 16; ++q)
          t[q] = (z + q < S) ? __ldcg(reinterpret_cast<const float4*>(g.out + (int64_t)(z + q) * g.part_stride + o))
                             : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
        for (int q = 0; q < 16; ++q) {
          sum.x += t[q].x; sum.y += t[q].y; sum.z += t[q].z; sum.w += t[q].w;
        }
      }
      if (g.dh_off) {   // centred sigmoid dZ: + (1/(2B)) sum_j W2_j
        sum.x += g.dh_off[c]; sum.y += g.dh_off[c + 1]; sum.z += g.dh_off[c + 2]; sum.w += g.dh_off[c + 3];
      }
      const float4 hv = *reinterpret_cast<const float4*>(g.h1 + o);
      const float4 v = make_float4(hv.x > 0.f ? sum.x : 0.f, hv.y > 0.f ? sum.y : 0.f,
                                   hv.z > 0.f ? sum.z : 0.f, hv.w > 0.f ? sum.w : 0.f);
      *reinterpret_cast<float4*>(g.da1 + o) = v;
      if (g.da1b) {
        __nv_bfloat162 p0 = __floats2bfloat162_rn(v.x, v.y), p1 = __floats2bfloat162_rn(v.z, v.w);
        uint2 pk;
        pk.x = *reinterpret_cast<uint32_t*>(&p0); pk.y = *reinterpret_cast<uint32_t*>(&p1);
        *reinterpret_cast<uint2*>(g.da1b + o) = pk;
      }
      *reinterpret_cast<float4*>(sred + rl * nc + cl) = v;
    }
    __syncthreads();
    // column sums of the block, rows in order (one thread per column, 4 partial chains)
    for (int c = threadIdx.x; c < nc; c += blockDim.x) {
      float t[4] = {0.f, 0.f, 0.f, 0.f};
      const int nr = r1 - r0;
      int r = 0;
      for (; r + 4 <= nr; r += 4) {
#pragma unroll
        for (int q = 0; q < 4; ++q) t[q] += sred[(r + q) * nc + c];
      }
      for (; r < nr; ++r) t[0] += sred[r * nc + c];
      g.colpart[(int64_t)rb * H + c0 + c] = (t[0] + t[1]) + (t[2] + t[3]);
    }
  }
  // (3) the last CTA: db1 = sum over row blocks in order; b1 -= lr db1; mean loss
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) s_last = atomicAdd(g.bar + 2, 1) == G - 1;
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  const float lr = step_lr(g.meta);
  for (int c = threadIdx.x; c < H; c += blockDim.x) {
    float t = 0.f;
    for (int rb = 0; rb < GR; ++rb) t += __ldcg(g.colpart + (int64_t)rb * H + c);
    g.b1[c] -= lr * t;
    if (g.grad_b1) g.grad_b1[c] = t;
  }
  float* loss_dev = step_loss(g.meta);
  if (threadIdx.x < 32 && loss_dev) {
    float t = 0.f;
    for (int r = threadIdx.x; r < n; r += 32) t += __ldcg(g.rowloss + r);
#pragma unroll
    for (int o = 16; o; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
    if (threadIdx.x == 0) *loss_dev = t / (float)n;
  }
  if (threadIdx.x == 0) g.bar[2] = 0;
}

// Persistent tcgen05 GEMM.  CTA = 4 + E warps: warp 0 TMA producer, warp 1 MMA
// issuer, warp 2 TMEM allocator, warps 4..3+E epilogue (warp w drains TMEM lanes
// 32 (w % 4) .. + 31, column group (w - 4) / 4 of E / 4).  E = 16 for the
// MUFU-heavy softmax / sigmoid epilogues on wide tiles (4 warps per scheduler
// hide the exp latency), else 8.  Tiles (M fastest, or N fastest
// when g.n_fast) are strided over the grid; the smem ring (full/empty mbarriers)
// and the TMEM accumulators (tfull/tempty, double-buffered when 2 fit in 512
// columns) carry across tiles, so a tile's epilogue overlaps the next tile's
// loads and MMAs.
template <int BN, int EPI>
constexpr int epi_warps() {
  return (BN >= 128 && (EPI == TC_EPI_DZ || EPI == TC_EPI_SIG || EPI == TC_EPI_STATS)) ? 16 : 8;
}
template <int EPI, bool X3 = false>
constexpr int stages_of() {   // G3 streams dZ^T from HBM: the deepest ring (its epilogue needs no smem)
  // bf16x3 (R14): every stage holds hi and lo tiles of both operands, 2 stages fit
  return X3 ? 2 : (EPI == TC_EPI_SGD ? 5 : (EPI == TC_EPI_STATS ? 4 : (EPI == TC_EPI_Z ? 2 : 3)));
}
template <int EPI>
constexpr uint32_t box_bytes() {   // one 32 x 32 store box: fp32 (Z, PART) or bf16 (DZ, SIG)
  return (EPI == TC_EPI_DZ || EPI == TC_EPI_SIG) ? 2048u : 4096u;
}
template <int EPI>
constexpr bool has_bias() {
  return EPI == TC_EPI_Z || EPI == TC_EPI_DZ || EPI == TC_EPI_SIG || EPI == TC_EPI_STATS;
}
template <int BN, int EPI>
constexpr uint32_t bias_bytes() {   // per epilogue warp: its tile columns' b2 (smem broadcast copy)
  return has_bias<EPI>() ? (uint32_t)epi_warps<BN, EPI>() * (uint32_t)(BN / (epi_warps<BN, EPI>() / 4)) * 4u : 0u;
}
// G1 variants with the A operand (the H1 row block, K = H <= 256) resident in smem: a CTA
// keeps its M block for many consecutive tiles (chunked order), so only W2 tiles stream.
template <int EPI, bool A_MN>
constexpr bool a_resident() {
  return !A_MN && (EPI == TC_EPI_STATS || EPI == TC_EPI_DZ || EPI == TC_EPI_SIG);
}
constexpr int kAresK = 256;   // largest K (= H) of the resident A block
template <int EPI, bool A_MN>
constexpr int store_bufs() { return a_resident<EPI, A_MN>() ? 1 : 2; }   // TMA-store boxes per warp
template <int BN, int EPI, bool A_MN>
constexpr uint32_t staging_bytes() {   // per epilogue warp: store boxes / G3 transpose tile
  return EPI == TC_EPI_STATS ? 0u
                             : (EPI == TC_EPI_SGD ? 8u * 4096u   // per warp: one 32 x 32 fp32 transpose tile
                                                  : (uint32_t)epi_warps<BN, EPI>() * store_bufs<EPI, A_MN>() *
                                                        box_bytes<EPI>());
}

// X3 (fp32 path, R14): both operands come as bf16 hi + lo halves (tmA2 / tmB2 map the lo
// halves, loaded into the same stage right after the hi tiles) and every K step issues
// three MMAs, hi.hi + hi.lo + lo.hi, into the same fp32 accumulator.
template <int BN, bool A_MN, bool B_MN, int EPI, bool X3>
__global__ void __launch_bounds__(128 + 32 * epi_warps<BN, EPI>(), 1)
    k_gemm_tc(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
              const __grid_constant__ CUtensorMap tmC, const __grid_constant__ CUtensorMap tmD,
              const __grid_constant__ CUtensorMap tmA2, const __grid_constant__ CUtensorMap tmB2, TcArgs g) {
  constexpr int STAGES = stages_of<EPI, X3>();
  constexpr bool ARES = a_resident<EPI, A_MN>();
  static_assert(!(X3 && ARES), "bf16x3 GEMMs stream A");
  constexpr uint32_t XF = X3 ? 2u : 1u;
  constexpr uint32_t A_BYTES = BM * BK * 2, B_BYTES = BN * BK * 2;   // one half (hi or lo)
  constexpr uint32_t A_SLOT = A_BYTES * XF, B_SLOT = B_BYTES * XF;
  constexpr uint32_t STAGE = (ARES ? 0u : A_SLOT) + B_SLOT;
  constexpr uint32_t ARES_BYTES = ARES ? (uint32_t)(kAresK / BK) * A_BYTES : 0u;
  constexpr int NSTG = store_bufs<EPI, A_MN>();
  constexpr bool ONES = (EPI == TC_EPI_SGD);           // db2 column block after the accumulator
  constexpr int ACC_COLS = BN + (ONES ? 32 : 0);
  constexpr int NACC = (2 * ACC_COLS <= 512) ? 2 : 1;
  constexpr uint32_t TMEM_COLS = pow2ceil(NACC * ACC_COLS);
  constexpr uint32_t ONES_BYTES = ONES ? 16 * 128 : 0; // K-major 16 x 64 bf16 tile, row 0 = 1
  constexpr int EPI_WARPS = epi_warps<BN, EPI>();
  constexpr int NQ = EPI_WARPS / 4;      // column groups
  constexpr int CW = BN / NQ;            // columns per epilogue warp
  static_assert(CW % 32 == 0, "epilogue chunks are 32 columns");
  constexpr uint32_t BOX = box_bytes<EPI>();
  extern __shared__ uint8_t smem_raw[];
  // 1024-aligned base, derived from smem_raw by an offset so the compiler keeps the shared
  // address space (LDS/STS instead of generic LD/ST in the epilogues)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sA = smem;                                          // ring A stages, or the resident A block
  uint8_t* sB = smem + (ARES ? ARES_BYTES : STAGES * A_SLOT);
  uint8_t* sOnes = smem + ARES_BYTES + STAGES * STAGE;
  uint8_t* sStg = sOnes + ONES_BYTES;   // TMA-store staging (1024-aligned)
  float* sBias = reinterpret_cast<float*>(sStg + staging_bytes<BN, EPI, A_MN>());
  uint64_t* full = reinterpret_cast<uint64_t*>(sStg + staging_bytes<BN, EPI, A_MN>() + bias_bytes<BN, EPI>());
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;
  uint64_t* tempty = tfull + 2;
  uint64_t* afull = tempty + 2;   // resident A block loaded
  uint32_t* tbase = reinterpret_cast<uint32_t*>(afull + 1);

  Tl tl_((EPI == TC_EPI_PART ? TL_G2 : EPI == TC_EPI_SGD ? TL_G3 : EPI == TC_EPI_DZ ? TL_G1B : TL_G1));
  pdl_trigger();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int MT = (g.M + BM - 1) / BM, NT = (g.N + BN - 1) / BN, Z = g.splits;
  const int T = MT * NT * Z;
  const int nkb = (g.K + BK - 1) / BK;
  const int per = (nkb + Z - 1) / Z;
  // this CTA's tiles: t = t_first, t_first + t_step, ... < t_end
  const int t_first = g.chunked ? (int)((int64_t)blockIdx.x * T / gridDim.x) : (int)blockIdx.x;
  const int t_end = g.chunked ? (int)((int64_t)(blockIdx.x + 1) * T / gridDim.x) : T;
  const int t_step = g.chunked ? 1 : (int)gridDim.x;
  auto decode = [&](int t, int& mt, int& nt, int& z, int& kb0, int& nk) {
    if (g.n_fast || g.chunked) { nt = t % NT; mt = (t / NT) % MT; } else { mt = t % MT; nt = (t / MT) % NT; }
    z = t / (MT * NT);
    kb0 = z * per;
    nk = max(0, min(nkb, kb0 + per) - kb0);
  };

  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmA)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmB)) : "memory");
    if constexpr (X3) {
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmA2)) : "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmB2)) : "memory");
    }
    for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(&tfull[a], 1); mbar_init(&tempty[a], EPI_WARPS); }
    mbar_init(afull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tbase)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if constexpr (ONES) {
    if (warp == 3) {   // row 0 = 64 x bf16(1.0) (unswizzled: row 0 of the atom), rows 1..15 = 0
      uint32_t* p = reinterpret_cast<uint32_t*>(sOnes);
      for (int i = lane; i < (int)(ONES_BYTES / 4); i += 32) p[i] = (i < 32) ? 0x3F803F80u : 0u;
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tbase;
  pdl_wait();   // operands / outputs of the previous kernel are visible from here on
  tl_.ready();

  if (warp == 0) {
    if (lane == 0) {
      // ------------------------------------------------ TMA producer
      int it = 0, amt = -1;
      for (int t = t_first; t < t_end; t += t_step) {
        int mt, nt, z, kb0, nk;
        decode(t, mt, nt, z, kb0, nk);
        const int m0 = mt * BM, n0 = nt * BN;
        if constexpr (ARES) {
          if (mt != amt) {   // new M block: reload the resident A once every MMA reading it retired
            if (it > 0) mbar_wait(&empty[(it - 1) % STAGES], ((it - 1) / STAGES) & 1);
            mbar_expect_tx(afull, (uint32_t)nk * A_BYTES);
            for (int i = 0; i < nk; ++i) tma_load_2d(sA + i * A_BYTES, &tmA, afull, (kb0 + i) * BK, m0);
            amt = mt;
          }
        }
        for (int i = 0; i < nk; ++i, ++it) {
          const int s = it % STAGES;
          const uint32_t ph = (it / STAGES) & 1;
          mbar_wait(&empty[s], ph ^ 1);
          mbar_expect_tx(&full[s], STAGE);
          const int kc = (kb0 + i) * BK;
          uint8_t* a = sA + s * A_SLOT;
          uint8_t* b = sB + s * B_SLOT;
#pragma unroll
          for (int h = 0; h < (int)XF; ++h) {   // h = 1: the lo halves (bf16x3)
            const CUtensorMap* ma = h ? &tmA2 : &tmA;
            const CUtensorMap* mb = h ? &tmB2 : &tmB;
            uint8_t* ah = a + h * A_BYTES;
            uint8_t* bh = b + h * B_BYTES;
            if constexpr (ARES) {
            } else if constexpr (!A_MN) {
              tma_load_2d(ah, ma, &full[s], kc, m0);
            } else {
              tma_load_2d(ah, ma, &full[s], m0, kc);
              tma_load_2d(ah + 8192, ma, &full[s], m0 + 64, kc);
            }
            if constexpr (!B_MN) {
              tma_load_2d(bh, mb, &full[s], kc, n0);
            } else {
#pragma unroll
              for (int j = 0; j < BN / 64; ++j) tma_load_2d(bh + j * 8192, mb, &full[s], n0 + 64 * j, kc);
            }
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ------------------------------------------------ MMA issuer
      constexpr uint32_t idesc = make_idesc(BN, A_MN, B_MN);
      constexpr uint32_t idesc1 = make_idesc(16, A_MN, false);
      const uint32_t ones_base = smem_u32(sOnes);
      int it = 0, tl = 0, amt = -1, aloads = 0;
      for (int t = t_first; t < t_end; t += t_step, ++tl) {
        int mt, nt, z, kb0, nk;
        decode(t, mt, nt, z, kb0, nk);
        const int acc = tl % NACC;
        const uint32_t aph = (tl / NACC) & 1;
        mbar_wait(&tempty[acc], aph ^ 1);     // epilogue drained this accumulator
        if constexpr (ARES) {
          if (mt != amt) { mbar_wait(afull, (uint32_t)aloads & 1u); ++aloads; amt = mt; }
        }
        tc_fence_after();
        const uint32_t d = tmem + (uint32_t)(acc * ACC_COLS);
        const bool ones = ONES && nt == 0;
        for (int i = 0; i < nk; ++i, ++it) {
          const int s = it % STAGES;
          const uint32_t ph = (it / STAGES) & 1;
          mbar_wait(&full[s], ph);
          tc_fence_after();
          const uint32_t a_base = smem_u32(sA + (ARES ? i * A_BYTES : s * A_SLOT)), b_base = smem_u32(sB + s * B_SLOT);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            // K-major: advance 16 elements (32 B) inside the 128B swizzle atom.
            // MN-major: advance 16 K-rows (2 atoms of 8 rows x 128 B = 2048 B).
            const uint64_t ad = A_MN ? desc_sw128(a_base + k * 2048, 8192, 1024) : desc_sw128(a_base + k * 32, 16, 1024);
            const uint64_t bd = B_MN ? desc_sw128(b_base + k * 2048, 8192, 1024) : desc_sw128(b_base + k * 32, 16, 1024);
            const uint32_t first = (i > 0 || k > 0) ? 1u : 0u;
            mma_bf16(d, ad, bd, idesc, first);
            if constexpr (X3) {   // + hi.lo + lo.hi (the lo tiles sit one half further in the stage)
              const uint64_t bdl = B_MN ? desc_sw128(b_base + B_BYTES + k * 2048, 8192, 1024)
                                        : desc_sw128(b_base + B_BYTES + k * 32, 16, 1024);
              const uint64_t adl = A_MN ? desc_sw128(a_base + A_BYTES + k * 2048, 8192, 1024)
                                        : desc_sw128(a_base + A_BYTES + k * 32, 16, 1024);
              mma_bf16(d, ad, bdl, idesc, 1u);
              mma_bf16(d, adl, bd, idesc, 1u);
              if (ONES && ones) {
                mma_bf16(d + BN, ad, desc_sw128(ones_base + k * 32, 16, 1024), idesc1, first);
                mma_bf16(d + BN, adl, desc_sw128(ones_base + k * 32, 16, 1024), idesc1, 1u);
              }
            } else {
              if (ONES && ones)   // TMEM column BN += dZ^T tile . e_0  (db2)
                mma_bf16(d + BN, ad, desc_sw128(ones_base + k * 32, 16, 1024), idesc1, first);
            }
          }
          mma_commit(&empty[s]);   // frees the smem stage once these MMAs retire
        }
        mma_commit(&tfull[acc]);   // accumulator ready (immediately if nk == 0)
      }
    }
  } else if (warp >= 4) {
    // ------------------------------------------------ epilogue (EPI_WARPS warps)
    const int wq = (warp - 4) & 3, wh = (warp - 4) >> 2;
    const float lr = EPI == TC_EPI_SGD ? step_lr(g.meta) : 0.f;
    int tl = 0, sbuf = 0;
    static_assert(EPI != TC_EPI_SGD || CW <= 64, "G3: at most 2 W2 row segments per warp per tile");
    // G1b / sigmoid: row m's lse, 1 / (|Y_m| B) and label cursor, kept while the tile's M
    // block does not change (chunked order: N increases, so the cursor only moves forward)
    int row_mt = -1;
    float lse_m = 0.f, tinv = 0.f, crow = 0.f;   // crow (DZ): -lse log2(e) - log2(B)
    int64_t lab_cur = 0, lab_end = 0;
    int nxt = 0x7fffffff;                        // next label column of row m (labels sorted)
    float* bias_w = sBias + (has_bias<EPI>() ? (warp - 4) * CW : 0);
    // b2 of the tile after the current one (prefetched one tile ahead)
    float bpre[has_bias<EPI>() ? CW / 32 : 1];
    auto load_bias = [&](int tt) {
      if constexpr (has_bias<EPI>()) {
        int mt_, nt_, z_, kb_, nk_;
        decode(tt, mt_, nt_, z_, kb_, nk_);
#pragma unroll
        for (int c = 0; c < CW / 32; ++c) {
          const int col = nt_ * BN + wh * CW + 32 * c + lane;
          bpre[c] = col < g.N ? __ldg(g.bias + col) : 0.f;
        }
      }
    };
    if (t_first < t_end) load_bias(t_first);
    for (int t = t_first; t < t_end; t += t_step, ++tl) {
      int mt, nt, z, kb0, nk;
      decode(t, mt, nt, z, kb0, nk);
      const int m0 = mt * BM, n0 = nt * BN;
      const int acc = tl % NACC;
      const uint32_t aph = (tl / NACC) & 1;
      const int m = m0 + wq * 32 + lane;
      // before waiting for the accumulator: this warp's b2 columns into smem (read back
      // below as broadcast float4), then the next tile's b2 loads are issued into
      // registers -- their latency hides under this tile's epilogue instead of stalling
      // the warp at the top of every tile -- and the row state of a new M block
      if constexpr (has_bias<EPI>()) {
        __syncwarp();
#pragma unroll
        for (int c = 0; c < CW / 32; ++c)   // DZ: log2 domain
          bias_w[32 * c + lane] = EPI == TC_EPI_DZ ? bpre[c] * 1.4426950408889634f : bpre[c];
        __syncwarp();
        if (t + t_step < t_end) load_bias(t + t_step);
      }
      if constexpr (EPI == TC_EPI_DZ || EPI == TC_EPI_SIG) {
        if (mt != row_mt) {
          row_mt = mt;
          lab_cur = lab_end = 0;
          if (m < g.M) {
            if constexpr (EPI == TC_EPI_DZ) {
              lse_m = g.lse[m];
              crow = -lse_m * 1.4426950408889634f - __log2f(1.f / g.invB);
            }
            const int64_t id = g.rows[m];
            lab_cur = g.lab_ptr[id];
            lab_end = g.lab_ptr[id + 1];
            tinv = g.invB / (float)(lab_end - lab_cur);
          }
          nxt = lab_cur < lab_end ? g.lab[lab_cur] : 0x7fffffff;
        }
        // skip labels left of this warp's first column (cursor is monotone within an M block
        // in the chunked order; a restart at a lower column would need the full walk)
        const int cfirst = n0 + wh * CW;
        while (nxt < cfirst) {
          ++lab_cur;
          nxt = lab_cur < lab_end ? g.lab[lab_cur] : 0x7fffffff;
        }
      }
      if constexpr (EPI == TC_EPI_SGD) {
        // G3: W2 -= lr (dZ^T H1 [+ centred-sigmoid offset]), b2 -= lr db2, bf16 shadow refresh.
        // Per 32 x 32 chunk: the accumulator (lane = W2 row) goes through a swizzled smem
        // tile so that W2 is read and written coalesced (8 lanes x 16 B per row, 4 rows
        // per instruction); the W2 chunks are loaded into registers before the
        // accumulator wait, so their HBM latency hides under this tile's MMAs.
        constexpr int NCH = CW / 32;
        const int cb = n0 + wh * CW;
        const int m0w = m0 + wq * 32;
        const int lr8 = lane >> 3, lc4 = (lane & 7) * 4;   // coalesced layout: row 4 i + lr8, cols lc4..+3
        uint8_t* tt = sStg + (warp - 4) * 4096;
        float4 wr[NCH][8];
#pragma unroll
        for (int ch = 0; ch < NCH; ++ch)
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const int r = m0w + 4 * i + lr8;
            wr[ch][i] = r < g.M ? *reinterpret_cast<const float4*>(g.out + (int64_t)r * g.ldo + cb + 32 * ch + lc4)
                                : make_float4(0.f, 0.f, 0.f, 0.f);
          }
        mbar_wait(&tfull[acc], aph);
        tc_fence_after();
        const uint32_t d = tmem + (uint32_t)(acc * ACC_COLS) + ((uint32_t)(wq * 32) << 16);
#pragma unroll
        for (int ch = 0; ch < NCH; ++ch) {
          float v[32];
          if (nk > 0) {
            tmem_ld32(d + (uint32_t)(wh * CW + 32 * ch), v);
          } else {
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
          }
          __syncwarp();   // the previous chunk's reads of tt are done
#pragma unroll
          for (int q = 0; q < 8; ++q)
            *reinterpret_cast<float4*>(tt + lane * 128 + ((q ^ (lane & 7)) * 16)) =
                make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
          __syncwarp();
          float4 ho = make_float4(0.f, 0.f, 0.f, 0.f);
          if (g.hoff) ho = __ldg(reinterpret_cast<const float4*>(g.hoff + cb + 32 * ch + lc4));   // centred sigmoid
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const int rl = 4 * i + lr8, r = m0w + rl;
            float4 a = *reinterpret_cast<const float4*>(tt + rl * 128 + (((lane & 7) ^ (rl & 7)) * 16));
            a.x += ho.x; a.y += ho.y; a.z += ho.z; a.w += ho.w;
            if (r < g.M) {
              float4 x = wr[ch][i];
              x.x -= lr * a.x; x.y -= lr * a.y; x.z -= lr * a.z; x.w -= lr * a.w;
              const int64_t o = (int64_t)r * g.ldo + cb + 32 * ch + lc4;
              __stcs(reinterpret_cast<float4*>(g.out + o), x);
              __nv_bfloat162 p0 = __floats2bfloat162_rn(x.x, x.y), p1 = __floats2bfloat162_rn(x.z, x.w);
              uint2 pk;
              pk.x = *reinterpret_cast<uint32_t*>(&p0); pk.y = *reinterpret_cast<uint32_t*>(&p1);
              __stcs(reinterpret_cast<uint2*>(g.shadow + o), pk);
              if constexpr (X3) {   // lo half of the new shadow (R14)
                __nv_bfloat162 q0 = __floats2bfloat162_rn(x.x - __low2float(p0), x.y - __high2float(p0));
                __nv_bfloat162 q1 = __floats2bfloat162_rn(x.z - __low2float(p1), x.w - __high2float(p1));
                uint2 pl;
                pl.x = *reinterpret_cast<uint32_t*>(&q0); pl.y = *reinterpret_cast<uint32_t*>(&q1);
                __stcs(reinterpret_cast<uint2*>(g.shadow_lo + o), pl);
              }
              if (g.grad) *reinterpret_cast<float4*>(g.grad + o) = a;
            }
          }
        }
      } else {
      mbar_wait(&tfull[acc], aph);
      tc_fence_after();
      const uint32_t d = tmem + (uint32_t)(acc * ACC_COLS) + ((uint32_t)(wq * 32) << 16);
      float st_m = -INFINITY, st_s = 0.f;   // G1 softmax partials of row m over this column group
      // chunks of 32 columns; the next chunk's TMEM load is in flight while this one is processed
      constexpr int NCHK = CW / 32;
      const bool have = EPI != TC_EPI_PART || nk > 0;   // only split-K slices can be empty
      uint32_t rr[2][32];
      if (have) tmem_ld32_async(d + (uint32_t)(wh * CW), rr[0]);
#pragma unroll
      for (int k = 0; k < NCHK; ++k) {
        const int c = wh * CW + 32 * k;
        float v[32];
        if (have) {
          tmem_wait_regs(rr[k & 1]);
          if (k + 1 < NCHK) tmem_ld32_async(d + (uint32_t)(c + 32), rr[(k + 1) & 1]);
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(rr[k & 1][i]);
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = 0.f;
        }
        const int n = n0 + c;
        if (n >= g.N) continue;   // warp-uniform
        if constexpr (EPI == TC_EPI_Z || EPI == TC_EPI_SIG || EPI == TC_EPI_STATS) {
          // + b2 (the same 32 values for every lane: broadcast smem reads); columns >= N -> -inf
          const float4* b4 = reinterpret_cast<const float4*>(bias_w + (c - wh * CW));
#pragma unroll
          for (int q = 0; q < 8; ++q) {
            const float4 t = b4[q];
            v[4 * q] += t.x; v[4 * q + 1] += t.y; v[4 * q + 2] += t.z; v[4 * q + 3] += t.w;
          }
          if (n + 32 > g.N) {
#pragma unroll
            for (int j = 0; j < 32; ++j)
              if (n + j >= g.N) v[j] = -INFINITY;
          }
        }
        if constexpr (EPI == TC_EPI_DZ || EPI == TC_EPI_SIG) {
          constexpr float kL2E = 1.4426950408889634f;
          if constexpr (EPI == TC_EPI_DZ) {
            // softmax - uniform target over the row's labels (Q3), / B (Q4):
            // exp(acc + b2 - lse) / B = 2^(acc log2(e) + b2 log2(e) - lse log2(e) - log2(B)),
            // b2 log2(e) staged per column; labels are sorted, nxt walks forward with the columns
            const float4* b4 = reinterpret_cast<const float4*>(bias_w + (c - wh * CW));
#pragma unroll
            for (int q = 0; q < 8; ++q) {
              const float4 t = b4[q];
              v[4 * q] = ex2_approx(fmaf(v[4 * q], kL2E, t.x + crow));
              v[4 * q + 1] = ex2_approx(fmaf(v[4 * q + 1], kL2E, t.y + crow));
              v[4 * q + 2] = ex2_approx(fmaf(v[4 * q + 2], kL2E, t.z + crow));
              v[4 * q + 3] = ex2_mix(fmaf(v[4 * q + 3], kL2E, t.w + crow));
            }
            if (n + 32 > g.N) {   // columns >= N (stores are clipped; keep them finite)
#pragma unroll
              for (int j = 0; j < 32; ++j)
                if (n + j >= g.N) v[j] = 0.f;
            }
            while (nxt < n + 32) {   // rare: a label of row m in this chunk
              const int jy = nxt - n;
#pragma unroll
              for (int j = 0; j < 32; ++j)
                if (j == jy) v[j] -= tinv;
              ++lab_cur;
              nxt = lab_cur < lab_end ? g.lab[lab_cur] : 0x7fffffff;
            }
          } else {
            // sigmoid BCE (R11): row partial += softplus(z) - y z; dZ is stored CENTRED,
            // dZc = (sigmoid(z) - 1/2 - y) / B: near initialisation sigmoid(z) = 1/2 + z/4 with
            // |z| ~ 1e-3, and bf16(sigmoid / B) would round the z-dependent part away.  The
            // constant 1/(2B) is added back exactly by k_sig_center (dH1, dW2) and G3 (db2).
            // e = exp(-|z|) in (0, 1]; sigmoid(|z|) - 1/2 = (1 - e) / (2 (1 + e));
            // softplus(z) = max(z, 0) + log1p(e).  Padding columns carry z = -inf: e = 0,
            // softplus = 0 (their dZ is clipped by the store).
            uint32_t ym = 0;   // label columns of this 32-column chunk (labels sorted)
            while (nxt < n + 32) {
              ym |= 1u << (nxt - n);
              ++lab_cur;
              nxt = lab_cur < lab_end ? g.lab[lab_cur] : 0x7fffffff;
            }
            float a0 = 0.f, a1 = 0.f;
#pragma unroll
            for (int j = 0; j < 32; ++j) {
              const float z = v[j];
              const float e = ex2_approx(-fabsf(z) * kL2E);
              const float r = rcp_approx(1.f + e);
              const float ch = 0.5f * (1.f - e) * r;              // sigmoid(|z|) - 1/2
              const float cz = z >= 0.f ? ch : -ch;               // sigmoid(z) - 1/2
              const float sp = fmaxf(z, 0.f) + log1p_01(e);
              const bool y = (ym >> j) & 1u;
              if (j & 1) a1 += y ? sp - z : sp; else a0 += y ? sp - z : sp;
              v[j] = (y ? cz - 1.f : cz) * g.invB;
            }
            st_s += a0 + a1;
          }
          // stage a 32 x 32 bf16 box (64B swizzle) and TMA-store it into dZ
          uint8_t* buf = sStg + ((warp - 4) * NSTG + (NSTG > 1 ? sbuf : 0)) * BOX;
          if (lane == 0) {
            if constexpr (NSTG > 1) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
            else asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
          }
          __syncwarp();
          {
            uint8_t* rowp = buf + lane * 64;
            const int sw = (lane >> 1) & 3;   // 64B swizzle of this row's four 16-byte chunks
#pragma unroll
            for (int h = 0; h < 4; ++h) {
              __nv_bfloat162 p0 = __floats2bfloat162_rn(v[8 * h], v[8 * h + 1]);
              __nv_bfloat162 p1 = __floats2bfloat162_rn(v[8 * h + 2], v[8 * h + 3]);
              __nv_bfloat162 p2 = __floats2bfloat162_rn(v[8 * h + 4], v[8 * h + 5]);
              __nv_bfloat162 p3 = __floats2bfloat162_rn(v[8 * h + 6], v[8 * h + 7]);
              uint4 pk;
              pk.x = *reinterpret_cast<uint32_t*>(&p0); pk.y = *reinterpret_cast<uint32_t*>(&p1);
              pk.z = *reinterpret_cast<uint32_t*>(&p2); pk.w = *reinterpret_cast<uint32_t*>(&p3);
              *reinterpret_cast<uint4*>(rowp + ((h ^ sw) * 16)) = pk;
            }
          }
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          __syncwarp();
          if (lane == 0) {
            asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                             reinterpret_cast<uint64_t>(&tmC)), "r"(smem_u32(buf)), "r"(n), "r"(m0 + wq * 32)
                         : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          }
          sbuf ^= 1;
          continue;
        }
        if constexpr (EPI == TC_EPI_Z || EPI == TC_EPI_STATS) {
          if (g.stats) {   // online (max, sum exp) of row m over the columns seen so far
            float mx[16];   // max as a depth-5 tree (a 31-long FMNMX chain is 124 cycles of latency)
#pragma unroll
            for (int j = 0; j < 16; ++j) mx[j] = fmaxf(v[j], v[j + 16]);
#pragma unroll
            for (int w = 8; w; w >>= 1)
#pragma unroll
              for (int j = 0; j < w; ++j) mx[j] = fmaxf(mx[j], mx[j + w]);
            const float cm = mx[0];
            constexpr float kL2E = 1.4426950408889634f;
            if (cm > st_m) { st_s = (st_m == -INFINITY) ? 0.f : st_s * ex2_approx((st_m - cm) * kL2E); st_m = cm; }
            const float ms = st_m * kL2E;
            float a0 = 0.f, a1 = 0.f, a2 = 0.f, a3 = 0.f;   // 4 independent MUFU -> FADD chains
#pragma unroll
            for (int j = 0; j < 32; j += 4) {
              a0 += ex2_approx(fmaf(v[j], kL2E, -ms));
              a1 += ex2_approx(fmaf(v[j + 1], kL2E, -ms));
              a2 += ex2_approx(fmaf(v[j + 2], kL2E, -ms));
              a3 += ex2_mix(fmaf(v[j + 3], kL2E, -ms));
            }
            st_s += (a0 + a1) + (a2 + a3);
          }
        }
        if constexpr (EPI == TC_EPI_STATS) continue;   // step: only the softmax partials are needed
        if constexpr (EPI == TC_EPI_Z || EPI == TC_EPI_PART) {
          // stage the warp's 32 x 32 fp32 box (128B swizzle: conflict-free) and TMA-store it;
          // rows >= M / columns >= N are clipped by the tensor map
          uint8_t* buf = sStg + ((warp - 4) * 2 + sbuf) * BOX;
          if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
          __syncwarp();
#pragma unroll
          for (int q = 0; q < 8; ++q)
            *reinterpret_cast<float4*>(buf + lane * 128 + ((q ^ (lane & 7)) * 16)) =
                make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          __syncwarp();
          if (lane == 0) {
            if constexpr (EPI == TC_EPI_Z)
              asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                               reinterpret_cast<uint64_t>(&tmC)),
                           "r"(smem_u32(buf)), "r"(n), "r"(m0 + wq * 32)
                           : "memory");
            else
              asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                               reinterpret_cast<uint64_t>(&tmC)),
                           "r"(smem_u32(buf)), "r"(n), "r"(m0 + wq * 32), "r"(z)
                           : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          }
          sbuf ^= 1;
        }
      }
      if constexpr (EPI == TC_EPI_Z || EPI == TC_EPI_STATS) {
        if (g.stats && m < g.M) g.stats[(int64_t)(nt * NQ + wh) * g.stats_ld + m] = make_float2(st_m, st_s);
      }
      if constexpr (EPI == TC_EPI_SIG) {
        if (m < g.M) g.stats[(int64_t)(nt * NQ + wh) * g.stats_ld + m] = make_float2(st_s, 0.f);
      }
      }   // EPI != SGD
      if constexpr (ONES) {
        if (nt == 0 && wh == 0) {   // db2[m] = sum_n dZ[n, m]; b2 -= lr db2
          float v[32];
          if (nk > 0) {
            tmem_ld32(tmem + (uint32_t)(acc * ACC_COLS + BN) + ((uint32_t)(wq * 32) << 16), v);
          } else {
            v[0] = 0.f;
          }
          if (m < g.M) {
            const float db = v[0] + g.db2_off;
            g.b2[m] -= lr * db;
            if (g.grad_b2) g.grad_b2[m] = db;
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&tempty[acc]);   // accumulator may be overwritten
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");   // stores complete
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
  }
  if constexpr (EPI == TC_EPI_PART) {
    if (g.dh_fuse) dh_reduce_phase(g, reinterpret_cast<float*>(smem));
  }
}

// ------------------------------------------------------------------ K-3 (dH1 half)
// Fused output-layer backward for the fused softmax-CE regime (PAPER.md
// P:1286-1309 fuses the element-wise work into the GEMMs): G1b + G2 + the dH1 reduce in
// one persistent kernel, so the logits of a label tile never leave the SM on their way
// into dH1.  CTA (label range lr, row block mb) keeps H1[mb] (128 x 256 bf16) resident and
// sweeps its label tiles j (64 labels each, in increasing order):
//   MMA 1   S     = H1_mb . W2_j^T                 (TMEM, 128 x 64, double-buffered)
//   epi     dZ    = exp(S + b2 - lse) / B - T      (bf16, written K-major into smem)
//   MMA 2   dH1  += dZ . W2_j                      (TMEM, 128 x 256; the SAME W2_j tile,
//                                                  read MN-major)
//   [dZ tile TMA-stored to global for G3 when g.write_z]
// then its dH1 partial (over its label range) goes to dhpart[lr] and, after a grid
// barrier, dh_reduce_phase sums the LR partials, applies ReLU' and updates b1.
constexpr int kBwdBN = 64, kBwdEpi = 8, kBwdStages = 3;
constexpr uint32_t kBwdH1Bytes = 4u * 16384u, kBwdW2Bytes = 4u * 8192u, kBwdDzBytes = 16384u;

// EG epilogue groups of kBwdEpi warps: group g drains the label tiles i = g, g + EG, ... (its
// own S buffer and dZ buffer when EG = 2), so two tiles' epilogues run at once.
template <int EG>
__global__ void __launch_bounds__(128 + 32 * kBwdEpi * EG, 1)
    k_bwd_dh(const __grid_constant__ CUtensorMap tmH1, const __grid_constant__ CUtensorMap tmW2,
             const __grid_constant__ CUtensorMap tmDZ, TcArgs g, int LR) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sH1 = smem;
  uint8_t* sW2 = sH1 + kBwdH1Bytes;
  uint8_t* sDZ = sW2 + kBwdStages * kBwdW2Bytes;
  float* sBias = reinterpret_cast<float*>(sDZ + 2 * kBwdDzBytes);          // [EG kBwdEpi][32], then [128][3]
  uint64_t* w2full = reinterpret_cast<uint64_t*>(sBias + EG * kBwdEpi * 32 + 128 * 3);
  uint64_t* w2empty = w2full + kBwdStages;
  uint64_t* sfull = w2empty + kBwdStages;
  uint64_t* sempty = sfull + 2;
  uint64_t* dzfull = sempty + 2;
  uint64_t* dzempty = dzfull + 2;
  uint64_t* hfull = dzempty + 2;
  uint64_t* dhfull = hfull + 1;
  uint32_t* tbase = reinterpret_cast<uint32_t*>(dhfull + 1);

  Tl tl_(g.dz_only ? TL_G1 : TL_G2);
  pdl_trigger();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int MT = (g.M + BM - 1) / BM, T = (g.N + kBwdBN - 1) / kBwdBN;
  const int mb = blockIdx.x % MT, lr = blockIdx.x / MT;
  const int t0 = (int)((int64_t)lr * T / LR), t1 = (int)((int64_t)(lr + 1) * T / LR), nt = t1 - t0;
  const int m0 = mb * BM;
  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmH1)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmW2)) : "memory");
    for (int s = 0; s < kBwdStages; ++s) { mbar_init(&w2full[s], 1); mbar_init(&w2empty[s], 1); }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&sfull[a], 1); mbar_init(&sempty[a], kBwdEpi);
      mbar_init(&dzfull[a], kBwdEpi); mbar_init(&dzempty[a], 1);
    }
    mbar_init(hfull, 1);
    mbar_init(dhfull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tbase)), "r"(512)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tbase;
  pdl_wait();
  tl_.ready();

  if (warp == 0) {
    if (lane == 0 && nt > 0) {   // ------------------------------------ TMA producer
      mbar_expect_tx(hfull, kBwdH1Bytes);
      for (int kb = 0; kb < 4; ++kb) tma_load_2d(sH1 + kb * 16384, &tmH1, hfull, kb * 64, m0);
      // one-pass: the range's W2 tiles twice (statistics sweep, then the dZ / dH1 sweep),
      // once when the S tiles stay in TMEM (keep: nt <= 2)
      const bool keep = g.one_pass && nt <= 2;
      const int nu = (g.one_pass && !keep) ? 2 * nt : nt;
      for (int u = 0; u < nu; ++u) {
        const int st = u % kBwdStages, i = u % nt;
        mbar_wait(&w2empty[st], ((u / kBwdStages) & 1) ^ 1);
        mbar_expect_tx(&w2full[st], kBwdW2Bytes);
        for (int kb = 0; kb < 4; ++kb)
          tma_load_2d(sW2 + st * kBwdW2Bytes + kb * 8192, &tmW2, &w2full[st], kb * 64, (t0 + i) * kBwdBN);
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && nt > 0) {   // ------------------------------------ MMA issuer
      constexpr uint32_t idesc1 = make_idesc(kBwdBN, false, false);   // S = H1 W2_j^T
      constexpr uint32_t idesc2 = make_idesc(256, false, true);       // dH1 += dZ W2_j
      mbar_wait(hfull, 0);
      // one-pass statistics sweep: S tiles only (use u = i of the S buffers / W2 stages);
      // keep (nt <= 2): they stay in their TMEM buffers and W2 stages for the second sweep
      const bool keep = g.one_pass && nt <= 2;
      const int base = (g.one_pass && !keep) ? nt : 0;
      for (int u = 0; u < (g.one_pass ? nt : 0); ++u) {
        const int st = u % kBwdStages, acc = u & 1;
        mbar_wait(&w2full[st], (u / kBwdStages) & 1);
        mbar_wait(&sempty[acc], ((u >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t d = tmem + (uint32_t)(acc * kBwdBN);
        const uint32_t wb = smem_u32(sW2 + st * kBwdW2Bytes);
#pragma unroll
        for (int kb = 0; kb < 4; ++kb)
#pragma unroll
          for (int k = 0; k < 4; ++k)
            mma_bf16(d, desc_sw128(smem_u32(sH1 + kb * 16384) + k * 32, 16, 1024),
                     desc_sw128(wb + kb * 8192 + k * 32, 16, 1024), idesc1, (kb | k) ? 1u : 0u);
        mma_commit(&sfull[acc]);
        if (!keep) mma_commit(&w2empty[st]);
      }
      for (int i = 0; i <= nt; ++i) {
        if (i < nt && !keep) {
          const int u = base + i, st = u % kBwdStages, acc = u & 1;
          mbar_wait(&w2full[st], (u / kBwdStages) & 1);
          mbar_wait(&sempty[acc], ((u >> 1) & 1) ^ 1);
          tc_fence_after();
          const uint32_t d = tmem + (uint32_t)(acc * kBwdBN);
          const uint32_t wb = smem_u32(sW2 + st * kBwdW2Bytes);
#pragma unroll
          for (int kb = 0; kb < 4; ++kb)
#pragma unroll
            for (int k = 0; k < 4; ++k)
              mma_bf16(d, desc_sw128(smem_u32(sH1 + kb * 16384) + k * 32, 16, 1024),
                       desc_sw128(wb + kb * 8192 + k * 32, 16, 1024), idesc1, (kb | k) ? 1u : 0u);
          mma_commit(&sfull[acc]);
        }
        if (i > 0) {
          const int j = i - 1, st = (base + j) % kBwdStages, buf = j & 1;
          mbar_wait(&dzfull[buf], (j >> 1) & 1);
          tc_fence_after();
          const uint32_t wb = smem_u32(sW2 + st * kBwdW2Bytes);
          const uint32_t zb = smem_u32(sDZ + buf * kBwdDzBytes);
          if (!g.dz_only) {
#pragma unroll
            for (int k = 0; k < kBwdBN / 16; ++k)
              mma_bf16(tmem + 256, desc_sw128(zb + k * 32, 16, 1024), desc_sw128(wb + k * 2048, 8192, 1024), idesc2,
                       (j > 0 || k > 0) ? 1u : 0u);
          }
          mma_commit(&dzempty[buf]);
          mma_commit(&w2empty[st]);
        }
      }
      mma_commit(dhfull);
    }
  } else if (warp >= 4) {   // -------------------------------------------- epilogue
    const int grp = (warp - 4) / kBwdEpi, ew = (warp - 4) % kBwdEpi;   // group, warp in group
    const int q = ew & 3, wh = ew >> 2;
    const bool lead = ew == 0 && lane == 0;   // the group's TMA-store thread
    const int m = m0 + q * 32 + lane;
    constexpr float kL2E = 1.4426950408889634f;
    float crow = 0.f, tinv = 0.f;
    int64_t lab_cur = 0, lab_end = 0;
    if (m < g.M) {
      if (!g.one_pass) crow = -g.lse[m] * kL2E - __log2f(1.f / g.invB);
      const int64_t id = g.rows[m];
      lab_cur = g.lab_ptr[id];
      lab_end = g.lab_ptr[id + 1];
      tinv = g.invB / (float)(lab_end - lab_cur);
    }
    int nxt = lab_cur < lab_end ? g.lab[lab_cur] : 0x7fffffff;
    if (warp == 4 && lane == 0) TL_MARK(TL_PH0);
    if (g.one_pass) {
      // (A) this CTA's softmax partials of row m over its label range, from a first sweep
      // of S tiles (the MMA warp's statistics sweep), in base 2: t = (S + b2) log2 e
      float mx = -INFINITY, se = 0.f, zs = 0.f;
      int64_t lc = lab_cur;
      int ny = nxt;
      for (int i = 0; i < nt; ++i) {
        const int c = (t0 + i) * kBwdBN + wh * 32, acc = i & 1;
        mbar_wait(&sfull[acc], (i >> 1) & 1);
        tc_fence_after();
        float v[32];
        tmem_ld32(tmem + (uint32_t)(acc * kBwdBN + wh * 32) + ((uint32_t)(q * 32) << 16), v);
        if (nt > 2) {   // recomputed in the second sweep: release the buffer
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&sempty[acc]);
        }
        float tm = -INFINITY;
#pragma unroll
        for (int jj = 0; jj < 32; ++jj) {
          const bool ok = c + jj < g.N;
          v[jj] = ok ? v[jj] + __ldg(g.bias + c + jj) : -INFINITY;   // Z (natural units)
          tm = fmaxf(tm, v[jj]);
        }
        while (ny < c) {
          ++lc;
          ny = lc < lab_end ? g.lab[lc] : 0x7fffffff;
        }
        while (ny < c + 32) {   // the row's labels among these columns: sum of Z_y
          const int jy = ny - c;
#pragma unroll
          for (int jj = 0; jj < 32; ++jj)
            if (jj == jy) zs += v[jj];
          ++lc;
          ny = lc < lab_end ? g.lab[lc] : 0x7fffffff;
        }
        const float tm2 = tm * kL2E;
        float ts = 0.f;
#pragma unroll
        for (int jj = 0; jj < 32; ++jj) ts += ex2_approx(fmaf(v[jj], kL2E, -tm2));
        if (tm2 > mx) { se = (mx == -INFINITY ? 0.f : se * ex2_approx(mx - tm2)) + ts; mx = tm2; }
        else if (tm2 != -INFINITY) se += ts * ex2_approx(tm2 - mx);
      }
      if (warp == 4 && lane == 0) TL_MARK(TL_PH1);
      // the two column halves (wh) of a row: wh = 1 hands its partial to wh = 0 via smem
      float* xch = sBias + EG * kBwdEpi * 32;   // [128][3] after the bias rows (EG = 1 here)
      const int rl = q * 32 + lane;
      if (wh == 1) { xch[3 * rl] = mx; xch[3 * rl + 1] = se; xch[3 * rl + 2] = zs; }
      asm volatile("bar.sync 1, %0;" ::"r"(32 * kBwdEpi) : "memory");
      if (wh == 0 && m < g.M) {
        const float om = xch[3 * rl], os = xch[3 * rl + 1];
        const float nm = fmaxf(mx, om);
        se = (mx == -INFINITY ? 0.f : se * ex2_approx(mx - nm)) + (om == -INFINITY ? 0.f : os * ex2_approx(om - nm));
        mx = nm;
        zs += xch[3 * rl + 2];
        // [range][row] layout: the reads in (C) are coalesced over a warp's 32 rows
        g.stats[(int64_t)lr * g.stats_ld + m] = make_float2(mx, se);
        reinterpret_cast<float*>(g.stats + (int64_t)g.stats_ld * LR)[(int64_t)lr * g.stats_ld + m] = zs;
      }
      // (B) grid barrier over the CTAs (all resident); the producer / MMA warps go on
      asm volatile("bar.sync 1, %0;" ::"r"(32 * kBwdEpi) : "memory");
      if (warp == 4 && lane == 0) grid_sync_packed(g.gbar, (int)gridDim.x);
      if (warp == 4 && lane == 0) TL_MARK(TL_PH2);
      asm volatile("bar.sync 1, %0;" ::"r"(32 * kBwdEpi) : "memory");
      // (C) lse of row m from the LR partials: the row's two warps (wh) each combine half of
      // the ranges, 16 loads in flight, then exchange through smem; range 0 writes the row loss
      float M2 = -INFINITY, S2 = 0.f, Zs = 0.f;
      const int hh = (LR + 1) / 2, ra = wh ? hh : 0, rb = wh ? LR : hh;
      if (m < g.M) {
        const float2* pp = g.stats + m;
        for (int r0 = ra; r0 < rb; r0 += 16) {
          float2 pm[16];
#pragma unroll
          for (int u = 0; u < 16; ++u)
            pm[u] = r0 + u < rb ? __ldcg(pp + (int64_t)(r0 + u) * g.stats_ld) : make_float2(-INFINITY, 0.f);
#pragma unroll
          for (int u = 0; u < 16; ++u) {
            if (pm[u].x == -INFINITY) continue;
            if (pm[u].x > M2) { S2 = (M2 == -INFINITY ? 0.f : S2 * ex2_approx(M2 - pm[u].x)) + pm[u].y; M2 = pm[u].x; }
            else S2 += pm[u].y * ex2_approx(pm[u].x - M2);
          }
        }
        if (warp == 4 && lane == 0) TL_MARK(TL_PH5);
        if (lr == 0) {   // the row's label-logit sum (range order), for the row loss
          const float* zp = reinterpret_cast<const float*>(g.stats + (int64_t)g.stats_ld * LR) + m;
          for (int r0 = ra; r0 < rb; r0 += 16) {
            float z[16];
#pragma unroll
            for (int u = 0; u < 16; ++u) z[u] = r0 + u < rb ? __ldcg(zp + (int64_t)(r0 + u) * g.stats_ld) : 0.f;
#pragma unroll
            for (int u = 0; u < 16; ++u) Zs += z[u];
          }
        }
      }
      if (warp == 4 && lane == 0) TL_MARK(TL_PH6);
      if (wh == 1) { xch[3 * rl] = M2; xch[3 * rl + 1] = S2; xch[3 * rl + 2] = Zs; }
      asm volatile("bar.sync 1, %0;" ::"r"(32 * kBwdEpi) : "memory");
      if (wh == 0) {
        const float om = xch[3 * rl], os = xch[3 * rl + 1];
        const float nm = fmaxf(M2, om);
        S2 = (M2 == -INFINITY ? 0.f : S2 * ex2_approx(M2 - nm)) + (om == -INFINITY ? 0.f : os * ex2_approx(om - nm));
        M2 = nm;
        Zs += xch[3 * rl + 2];
      }
      asm volatile("bar.sync 1, %0;" ::"r"(32 * kBwdEpi) : "memory");
      if (wh == 0) { xch[3 * rl] = M2; xch[3 * rl + 1] = S2; }
      asm volatile("bar.sync 1, %0;" ::"r"(32 * kBwdEpi) : "memory");
      if (wh == 1) { M2 = xch[3 * rl]; S2 = xch[3 * rl + 1]; }
      if (m < g.M) {
        const float lse2 = M2 + __log2f(S2);   // lse log2 e
        crow = -lse2 - __log2f(1.f / g.invB);
        if (lr == 0 && wh == 0) {
          const float lse = lse2 * 0.6931471805599453f;
          g.rowloss_w[m] = lse - Zs / (float)(lab_end - lab_cur);
          const_cast<float*>(g.lse)[m] = lse;
        }
      }
    }
    float* bias_w = sBias + (warp - 4) * 32;
    const uint32_t gbar = 1 + grp;   // the group's named barrier
    if (warp == 4 && lane == 0 && g.one_pass) TL_MARK(TL_PH3);
    // b2 of the next tile's columns, loaded one tile ahead (its latency hides under this
    // tile's epilogue instead of heading it: the top stall site in ncu before)
    auto b2_of = [&](int i) {
      const int cc = (t0 + i) * kBwdBN + wh * 32 + lane;
      return (i < nt && cc < g.N) ? __ldg(g.bias + cc) * kL2E : 0.f;
    };
    float bnext = b2_of(grp);
    const int base = (g.one_pass && nt > 2) ? nt : 0;   // S-buffer uses of the statistics sweep
    for (int i = grp; i < nt; i += EG) {
      const int acc = (base + i) & 1, buf = i & 1;
      const int c = (t0 + i) * kBwdBN + wh * 32;        // this warp's first label column
      __syncwarp();
      bias_w[lane] = bnext;
      __syncwarp();
      bnext = b2_of(i + EG);
      while (nxt < c) {
        ++lab_cur;
        nxt = lab_cur < lab_end ? g.lab[lab_cur] : 0x7fffffff;
      }
      mbar_wait(&sfull[acc], ((base + i) >> 1) & 1);
      tc_fence_after();
      float v[32];
      tmem_ld32(tmem + (uint32_t)(acc * kBwdBN + wh * 32) + ((uint32_t)(q * 32) << 16), v);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&sempty[acc]);
      const float4* b4 = reinterpret_cast<const float4*>(bias_w);
#pragma unroll
      for (int qq = 0; qq < 8; ++qq) {
        const float4 t = b4[qq];
        v[4 * qq] = ex2_approx(fmaf(v[4 * qq], kL2E, t.x + crow));
        v[4 * qq + 1] = ex2_approx(fmaf(v[4 * qq + 1], kL2E, t.y + crow));
        v[4 * qq + 2] = ex2_approx(fmaf(v[4 * qq + 2], kL2E, t.z + crow));
        v[4 * qq + 3] = ex2_approx(fmaf(v[4 * qq + 3], kL2E, t.w + crow));
      }
      if (c + 32 > g.N || m >= g.M) {   // padding columns / rows: dZ = 0
#pragma unroll
        for (int jj = 0; jj < 32; ++jj)
          if (c + jj >= g.N || m >= g.M) v[jj] = 0.f;
      }
      while (nxt < c + 32) {            // the row's labels in this chunk: - 1/(|Y| B)
        const int jy = nxt - c;
#pragma unroll
        for (int jj = 0; jj < 32; ++jj)
          if (jj == jy) v[jj] -= tinv;
        ++lab_cur;
        nxt = lab_cur < lab_end ? g.lab[lab_cur] : 0x7fffffff;
      }
      // the dZ buffer: MMA 2 of tile i - 2 done, and (write_z) its TMA store done reading
      mbar_wait(&dzempty[buf], ((i >> 1) & 1) ^ 1);
      if (g.write_z) {
        if (lead) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
        asm volatile("bar.sync %0, %1;" ::"r"(gbar), "r"(32 * kBwdEpi) : "memory");
      }
      uint8_t* rowp = sDZ + buf * kBwdDzBytes + (q * 32 + lane) * 128;
      const int sw = (q * 32 + lane) & 7;
#pragma unroll
      for (int h = 0; h < 4; ++h) {     // 16-byte chunk wh * 4 + h of the row, 128B-swizzled
        __nv_bfloat162 p0 = __floats2bfloat162_rn(v[8 * h], v[8 * h + 1]);
        __nv_bfloat162 p1 = __floats2bfloat162_rn(v[8 * h + 2], v[8 * h + 3]);
        __nv_bfloat162 p2 = __floats2bfloat162_rn(v[8 * h + 4], v[8 * h + 5]);
        __nv_bfloat162 p3 = __floats2bfloat162_rn(v[8 * h + 6], v[8 * h + 7]);
        uint4 pk;
        pk.x = *reinterpret_cast<uint32_t*>(&p0); pk.y = *reinterpret_cast<uint32_t*>(&p1);
        pk.z = *reinterpret_cast<uint32_t*>(&p2); pk.w = *reinterpret_cast<uint32_t*>(&p3);
        *reinterpret_cast<uint4*>(rowp + (((wh * 4 + h) ^ sw) * 16)) = pk;
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      if (g.write_z) {
        asm volatile("bar.sync %0, %1;" ::"r"(gbar), "r"(32 * kBwdEpi) : "memory");
        if (lead) {
          asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                           reinterpret_cast<uint64_t>(&tmDZ)), "r"(smem_u32(sDZ + buf * kBwdDzBytes)),
                       "r"((t0 + i) * kBwdBN), "r"(m0)
                       : "memory");
          asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&dzfull[buf]);
    }
    if (warp == 4 && lane == 0) TL_MARK(TL_PH4);
    // this CTA's dH1 partial (rows m, columns wh * 128 .. + 127) -> dhpart[lr]
    float* dst = g.out + (int64_t)lr * g.part_stride + (int64_t)m * g.ldo + wh * 128;
    if (nt > 0 && !g.dz_only) {
      mbar_wait(dhfull, 0);
      if (warp == 4 && lane == 0) TL_MARK(TL_PH5);
      tc_fence_after();
    }
#pragma unroll 1
    for (int ch = grp * (4 / EG); ch < (g.dz_only ? 0 : (grp + 1) * (4 / EG)); ++ch) {
      float v[32];
      if (nt > 0) {
        tmem_ld32(tmem + 256 + (uint32_t)(wh * 128 + ch * 32) + ((uint32_t)(q * 32) << 16), v);
      } else {
#pragma unroll
        for (int jj = 0; jj < 32; ++jj) v[jj] = 0.f;
      }
      if (m < g.M) {
#pragma unroll
        for (int qq = 0; qq < 8; ++qq)
          *reinterpret_cast<float4*>(dst + ch * 32 + 4 * qq) =
              make_float4(v[4 * qq], v[4 * qq + 1], v[4 * qq + 2], v[4 * qq + 3]);
      }
    }
    if (lead) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
  }
  __threadfence();
  if (g.dz_only) return;   // G2 and the dH1 reduce follow as kernels of their own
  TcArgs gt = g;    // the tail reduces H columns: N = H there
  gt.N = g.K;
  if (threadIdx.x == 0) TL_MARK(TL_PH6);
  dh_reduce_phase(gt, reinterpret_cast<float*>(smem));
}

// ------------------------------------------------------------------ K-3 (dW2 half)
// G1b + G3 in one persistent kernel for the fused softmax-CE regime: the dZ^T tiles a W2
// row tile needs are recomputed on chip instead of read back from HBM (K-3's second half,
// SURVEY §7; with it the logits never reach HBM).  CTA c owns a contiguous range of label
// tiles (128 labels = the MMA M) and, per tile j, sweeps the batch in row chunks of 64:
//   MMA 1   S^T   = W2_j . H1_m^T          (TMEM 128 x 64, double-buffered)
//   epi     dZ^T  = exp(S^T + b2 - lse) / B - T   (bf16, K-major smem tile; db2 in registers)
//   MMA 2   dW2_j += dZ^T . H1_m          (TMEM 128 x 256; the SAME H1 chunk, MN-major)
// then the SGD epilogue W2_j -= lr dW2_j (fp32, coalesced through a smem transpose), the next
// bf16 shadow, b2_j -= lr db2_j.  A helper warp turns the rows' sorted label lists into a
// per-(label, row) bitmap of the chunk (cursors in smem, advanced as the tiles increase).
constexpr int kDwBM = 128, kDwRB = 64;
constexpr uint32_t kDwW2Bytes = 4u * 16384u, kDwH1Bytes = 4u * 8192u, kDwDzBytes = 16384u;
constexpr int kDwMaxRows = 1024;

__global__ void __launch_bounds__(128 + 32 * kBwdEpi, 1)
    k_bwd_dw(const __grid_constant__ CUtensorMap tmW2, const __grid_constant__ CUtensorMap tmH1, TcArgs g) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sW2 = smem;                                   // 4 boxes [128 labels x 64 H]
  uint8_t* sH1 = sW2 + kDwW2Bytes;                       // 2 stages x 4 boxes [64 rows x 64 H]
  uint8_t* sDZ = sH1 + 2 * kDwH1Bytes;                   // 2 x [128 labels x 64 rows]
  uint8_t* sStg = sDZ + 2 * kDwDzBytes;                  // SGD transpose: 8 warps x 4 KB
  float* sCrow = reinterpret_cast<float*>(sStg + kBwdEpi * 4096);   // [2][64]
  float* sTinv = sCrow + 2 * kDwRB;                                  // [2][64]
  uint32_t* sBits = reinterpret_cast<uint32_t*>(sTinv + 2 * kDwRB);  // [2][128][2]
  float* sDb = reinterpret_cast<float*>(sBits + 2 * kDwBM * 2);      // [2][128]
  int32_t* sCur = reinterpret_cast<int32_t*>(sDb + 2 * kDwBM);       // [rows] label cursor
  int32_t* sNxt = sCur + kDwMaxRows;                                 // [rows] next label
  uint64_t* w2full = reinterpret_cast<uint64_t*>(sNxt + kDwMaxRows);
  uint64_t* w2empty = w2full + 1;
  uint64_t* h1full = w2empty + 1;    // [2]
  uint64_t* h1empty = h1full + 2;    // [2]
  uint64_t* sfull = h1empty + 2;     // [2]
  uint64_t* sempty = sfull + 2;      // [2]
  uint64_t* dzfull = sempty + 2;     // [2]
  uint64_t* dzempty = dzfull + 2;    // [2]
  uint64_t* auxfull = dzempty + 2;   // [2]
  uint64_t* auxempty = auxfull + 2;  // [2]
  uint64_t* tfull = auxempty + 2;
  uint64_t* tempty = tfull + 1;
  uint32_t* tbase = reinterpret_cast<uint32_t*>(tempty + 1);

  Tl tl_(TL_G3);
  pdl_trigger();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n = g.K;                                     // batch rows
  const int T = (g.M + kDwBM - 1) / kDwBM, NM = (n + kDwRB - 1) / kDwRB;
  const int j0 = (int)((int64_t)blockIdx.x * T / gridDim.x), j1 = (int)((int64_t)(blockIdx.x + 1) * T / gridDim.x);
  const int nt = j1 - j0;
  if (warp == 0 && lane == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmW2)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmH1)) : "memory");
    mbar_init(w2full, 1); mbar_init(w2empty, 1);
    for (int a = 0; a < 2; ++a) {
      mbar_init(&h1full[a], 1); mbar_init(&h1empty[a], 1);
      mbar_init(&sfull[a], 1); mbar_init(&sempty[a], kBwdEpi);
      mbar_init(&dzfull[a], kBwdEpi); mbar_init(&dzempty[a], 1);
      mbar_init(&auxfull[a], 1); mbar_init(&auxempty[a], kBwdEpi);
    }
    mbar_init(tfull, 1); mbar_init(tempty, kBwdEpi);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tbase)), "r"(512)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tbase;
  pdl_wait();
  tl_.ready();
  // label cursors: the first label of each row >= this CTA's first label (binary search,
  // all threads, rows strided), kept in smem and advanced as the tiles increase
  if (nt > 0) {
    const int l0 = j0 * kDwBM;
    for (int r = threadIdx.x; r < n; r += blockDim.x) {
      const int64_t id = g.rows[r];
      int64_t lo = g.lab_ptr[id], hi = g.lab_ptr[id + 1];
      const int64_t end = hi;
      while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (g.lab[mid] < l0) lo = mid + 1; else hi = mid;
      }
      sCur[r] = (int32_t)(lo - g.lab_ptr[id]);
      sNxt[r] = lo < end ? g.lab[lo] : 0x7fffffff;
    }
  }
  __syncthreads();

  if (warp == 0) {
    if (lane == 0 && nt > 0) {   // ------------------------------------ TMA producer
      int k = 0;
      for (int t = 0; t < nt; ++t) {
        mbar_wait(w2empty, (t & 1) ^ 1);
        mbar_expect_tx(w2full, kDwW2Bytes);
        for (int kb = 0; kb < 4; ++kb) tma_load_2d(sW2 + kb * 16384, &tmW2, w2full, kb * 64, (j0 + t) * kDwBM);
        for (int m = 0; m < NM; ++m, ++k) {
          const int st = k & 1;
          mbar_wait(&h1empty[st], ((k >> 1) & 1) ^ 1);
          mbar_expect_tx(&h1full[st], kDwH1Bytes);
          for (int kb = 0; kb < 4; ++kb)
            tma_load_2d(sH1 + st * kDwH1Bytes + kb * 8192, &tmH1, &h1full[st], kb * 64, m * kDwRB);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && nt > 0) {   // ------------------------------------ MMA issuer
      constexpr uint32_t idesc1 = make_idesc(kDwRB, false, false);   // S^T = W2_j H1_m^T
      constexpr uint32_t idesc2 = make_idesc(256, false, true);      // dW2 += dZ^T H1_m
      const int K = nt * NM;
      for (int k = 0; k <= K; ++k) {
        if (k < K) {
          const int t = k / NM, m = k % NM, st = k & 1, acc = k & 1;
          if (m == 0) mbar_wait(w2full, t & 1);
          mbar_wait(&h1full[st], (k >> 1) & 1);
          mbar_wait(&sempty[acc], ((k >> 1) & 1) ^ 1);
          tc_fence_after();
          const uint32_t d = tmem + (uint32_t)(acc * kDwRB);
          const uint32_t hb = smem_u32(sH1 + st * kDwH1Bytes);
#pragma unroll
          for (int kb = 0; kb < 4; ++kb)
#pragma unroll
            for (int kk = 0; kk < 4; ++kk)
              mma_bf16(d, desc_sw128(smem_u32(sW2 + kb * 16384) + kk * 32, 16, 1024),
                       desc_sw128(hb + kb * 8192 + kk * 32, 16, 1024), idesc1, (kb | kk) ? 1u : 0u);
          mma_commit(&sfull[acc]);
          if (m == NM - 1) mma_commit(w2empty);   // W2_j read by every MMA 1 of the tile
        }
        if (k > 0) {
          const int kp = k - 1, t = kp / NM, m = kp % NM, st = kp & 1, buf = kp & 1;
          if (m == 0) mbar_wait(tempty, (t & 1) ^ 1);   // the SGD epilogue drained dW2
          mbar_wait(&dzfull[buf], (kp >> 1) & 1);
          tc_fence_after();
          const uint32_t zb = smem_u32(sDZ + buf * kDwDzBytes), hb = smem_u32(sH1 + st * kDwH1Bytes);
#pragma unroll
          for (int kk = 0; kk < kDwRB / 16; ++kk)
            mma_bf16(tmem + 128, desc_sw128(zb + kk * 32, 16, 1024), desc_sw128(hb + kk * 2048, 8192, 1024), idesc2,
                     (m > 0 || kk > 0) ? 1u : 0u);
          mma_commit(&dzempty[buf]);
          mma_commit(&h1empty[st]);
          if (m == NM - 1) mma_commit(tfull);
        }
      }
    }
  } else if (warp == 3) {
    if (nt > 0) {               // ------------------------------------ label bitmap helper
      int k = 0;
      for (int t = 0; t < nt; ++t) {
        const int l0 = (j0 + t) * kDwBM;
        // the tile's fp32 W2 rows (128 x 1 KB) into L2 while the chunks run, so the SGD
        // epilogue's read-modify-write finds them there instead of paying HBM latency
        for (int i = lane; i < kDwBM * 8; i += 32) {
          const int r = l0 + (i >> 3);
          if (r < g.M)
            asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(g.out + (int64_t)r * g.ldo + (i & 7) * 32)
                         : "memory");
        }
        for (int m = 0; m < NM; ++m, ++k) {
          const int a = k & 1;
          mbar_wait(&auxempty[a], ((k >> 1) & 1) ^ 1);
          uint32_t* bits = sBits + a * kDwBM * 2;
          for (int i = lane; i < kDwBM * 2; i += 32) bits[i] = 0u;
          __syncwarp();
          for (int rr = lane; rr < kDwRB; rr += 32) {
            const int r = m * kDwRB + rr;
            float cr = 0.f, ti = 0.f;
            if (r < n) {
              const int64_t id = g.rows[r];
              const int64_t lb = g.lab_ptr[id], le = g.lab_ptr[id + 1];
              cr = -g.lse[r] * 1.4426950408889634f - __log2f(1.f / g.invB);
              ti = g.invB / (float)(le - lb);
              int cur = sCur[r], nx = sNxt[r];
              while (nx < l0 + kDwBM) {   // this tile's labels of row r (sorted)
                atomicOr(&bits[(nx - l0) * 2 + (rr >> 5)], 1u << (rr & 31));
                ++cur;
                nx = lb + cur < le ? g.lab[lb + cur] : 0x7fffffff;
              }
              sCur[r] = cur;
              sNxt[r] = nx;
            }
            sCrow[a * kDwRB + rr] = cr;
            sTinv[a * kDwRB + rr] = ti;
          }
          __syncwarp();
          if (lane == 0) mbar_arrive(&auxfull[a]);
        }
      }
    }
  } else if (warp >= 4) {       // -------------------------------------------- epilogue
    const int q = (warp - 4) & 3, wh = (warp - 4) >> 2;
    const int ll = q * 32 + lane;                  // this thread's label within the tile
    constexpr float kL2E = 1.4426950408889634f;
    const float lr = step_lr(g.meta);
    int k = 0;
    for (int t = 0; t < nt; ++t) {
      const int l = (j0 + t) * kDwBM + ll;
      const float b2l = l < g.M ? __ldg(g.bias + l) * kL2E : 0.f;
      float db = 0.f;
      for (int m = 0; m < NM; ++m, ++k) {
        const int acc = k & 1, buf = k & 1, a = k & 1;
        mbar_wait(&auxfull[a], (k >> 1) & 1);
        mbar_wait(&sfull[acc], (k >> 1) & 1);
        tc_fence_after();
        float v[32];
        tmem_ld32(tmem + (uint32_t)(acc * kDwRB + wh * 32) + ((uint32_t)(q * 32) << 16), v);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&sempty[acc]);
        const uint32_t bw = sBits[a * kDwBM * 2 + ll * 2 + wh];
        const float* cr = sCrow + a * kDwRB + wh * 32;
        const float* ti = sTinv + a * kDwRB + wh * 32;
        const int rbase = m * kDwRB + wh * 32;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
          float z = ex2_approx(fmaf(v[i], kL2E, b2l + cr[i]));
          if ((bw >> i) & 1u) z -= ti[i];
          if (l >= g.M || rbase + i >= n) z = 0.f;
          v[i] = z;
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&auxempty[a]);
        mbar_wait(&dzempty[buf], ((k >> 1) & 1) ^ 1);
        uint8_t* rowp = sDZ + buf * kDwDzBytes + ll * 128;
        const int sw = ll & 7;
#pragma unroll
        for (int h = 0; h < 4; ++h) {
          __nv_bfloat162 p0 = __floats2bfloat162_rn(v[8 * h], v[8 * h + 1]);
          __nv_bfloat162 p1 = __floats2bfloat162_rn(v[8 * h + 2], v[8 * h + 3]);
          __nv_bfloat162 p2 = __floats2bfloat162_rn(v[8 * h + 4], v[8 * h + 5]);
          __nv_bfloat162 p3 = __floats2bfloat162_rn(v[8 * h + 6], v[8 * h + 7]);
          db += ((__low2float(p0) + __high2float(p0)) + (__low2float(p1) + __high2float(p1))) +
                ((__low2float(p2) + __high2float(p2)) + (__low2float(p3) + __high2float(p3)));
          uint4 pk;
          pk.x = *reinterpret_cast<uint32_t*>(&p0); pk.y = *reinterpret_cast<uint32_t*>(&p1);
          pk.z = *reinterpret_cast<uint32_t*>(&p2); pk.w = *reinterpret_cast<uint32_t*>(&p3);
          *reinterpret_cast<uint4*>(rowp + (((wh * 4 + h) ^ sw) * 16)) = pk;
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncwarp();
        if (lane == 0) mbar_arrive(&dzfull[buf]);
      }
      // ---- SGD: W2_j -= lr dW2_j (rows = labels, this warp's 32 labels x 128 columns),
      //      coalesced through a swizzled 32 x 32 smem transpose; next bf16 shadow; b2
      const int m0w = (j0 + t) * kDwBM + q * 32;
      const int lr8 = lane >> 3, lc4 = (lane & 7) * 4;
      uint8_t* tt = sStg + (warp - 4) * 4096;
      mbar_wait(tfull, t & 1);
      tc_fence_after();
#pragma unroll 1
      for (int ch = 0; ch < 4; ++ch) {
        const int cb = wh * 128 + ch * 32;
        float4 wr[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int r = m0w + 4 * i + lr8;
          wr[i] = r < g.M ? *reinterpret_cast<const float4*>(g.out + (int64_t)r * g.ldo + cb + lc4)
                          : make_float4(0.f, 0.f, 0.f, 0.f);
        }
        float vv[32];
        tmem_ld32(tmem + 128 + (uint32_t)cb + ((uint32_t)(q * 32) << 16), vv);
        __syncwarp();
#pragma unroll
        for (int qq = 0; qq < 8; ++qq)
          *reinterpret_cast<float4*>(tt + lane * 128 + ((qq ^ (lane & 7)) * 16)) =
              make_float4(vv[4 * qq], vv[4 * qq + 1], vv[4 * qq + 2], vv[4 * qq + 3]);
        __syncwarp();
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int rl = 4 * i + lr8, r = m0w + rl;
          const float4 gv = *reinterpret_cast<const float4*>(tt + rl * 128 + (((lane & 7) ^ (rl & 7)) * 16));
          if (r < g.M) {
            float4 x = wr[i];
            x.x -= lr * gv.x; x.y -= lr * gv.y; x.z -= lr * gv.z; x.w -= lr * gv.w;
            const int64_t o = (int64_t)r * g.ldo + cb + lc4;
            __stcs(reinterpret_cast<float4*>(g.out + o), x);
            __nv_bfloat162 p0 = __floats2bfloat162_rn(x.x, x.y), p1 = __floats2bfloat162_rn(x.z, x.w);
            uint2 pk;
            pk.x = *reinterpret_cast<uint32_t*>(&p0); pk.y = *reinterpret_cast<uint32_t*>(&p1);
            __stcs(reinterpret_cast<uint2*>(g.shadow + o), pk);
            if (g.grad) *reinterpret_cast<float4*>(g.grad + o) = gv;
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(tempty);
      // db2: the two column halves' row sums, added in half order
      sDb[wh * kDwBM + ll] = db;
      asm volatile("bar.sync 2, %0;" ::"r"(32 * kBwdEpi) : "memory");
      if (wh == 0 && l < g.M) {
        const float dbt = sDb[ll] + sDb[kDwBM + ll];
        g.b2[l] -= lr * dbt;
        if (g.grad_b2) g.grad_b2[l] = dbt;
      }
      asm volatile("bar.sync 2, %0;" ::"r"(32 * kBwdEpi) : "memory");
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
  }
}

// ------------------------------------------------------------------ host side
PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;
std::once_flag g_once;

void init_encode() {
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) == cudaSuccess &&
      q == cudaDriverEntryPointSuccess)
    g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
}

// fp32 store maps (128B swizzle, 32 x 32 boxes): Z [rows][ldz] and the split-K partials
// [splits][b_max][H] (3D, so rows >= b_max of a slice never spill into the next slice).
cudaError_t make_store_map(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer,
                           uint64_t row_bytes, uint64_t depth, uint64_t slice_bytes, int rank) {
  cuuint64_t dims[3] = {inner, outer, depth};
  cuuint64_t strides[2] = {row_bytes, slice_bytes};
  cuuint32_t box[3] = {32, 32, 1};
  cuuint32_t es[3] = {1, 1, 1};
  if (rank == 3 && slice_bytes == 0) slice_bytes = row_bytes * outer;
  strides[1] = slice_bytes;
  CUresult r = g_encode(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, rank, const_cast<void*>(base), dims,
                        strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

// bf16 [outer][inner] store map, 32 x 32 boxes (64 B rows, 64B swizzle)
cudaError_t make_bf16_store_map(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer,
                                uint64_t row_bytes = 0) {
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {row_bytes ? row_bytes : inner * 2};
  cuuint32_t box[2] = {32, 32};
  cuuint32_t es[2] = {1, 1};
  CUresult r = g_encode(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

cudaError_t make_map(CUtensorMap* m, const void* base, uint64_t inner, uint64_t outer, uint64_t row_bytes,
                     uint32_t box_inner, uint32_t box_outer) {
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {row_bytes};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = g_encode(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

template <int BN, bool A_MN, bool B_MN, int EPI, bool X3 = false>
cudaError_t run(const Launch& lc, const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& c,
               const CUtensorMap& d, TcArgs g, int splits, const CUtensorMap* a2 = nullptr,
               const CUtensorMap* b2 = nullptr) {
  constexpr bool ARES = a_resident<EPI, A_MN>();
  constexpr size_t XF = X3 ? 2 : 1;
  const size_t smem = (ARES ? (size_t)(kAresK / BK) * BM * BK * 2 : 0) +
                      (size_t)stages_of<EPI, X3>() * XF * ((ARES ? 0 : BM * BK * 2) + BN * BK * 2) +
                      (EPI == TC_EPI_SGD ? 2048 : 0) + staging_bytes<BN, EPI, A_MN>() + bias_bytes<BN, EPI>() + 1024 + 512;
  if (ARES && g.K > kAresK) return cudaErrorNotSupported;   // resident A block holds K <= 256
  if (X3 && (!a2 || !b2)) return cudaErrorInvalidValue;
  {
    cudaError_t e = ensure_smem(k_gemm_tc<BN, A_MN, B_MN, EPI, X3>, smem);
    if (e != cudaSuccess) return e;
  }
  g.splits = splits;
  const int64_t tiles = (int64_t)((g.M + BM - 1) / BM) * ((g.N + BN - 1) / BN) * splits;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, lc.sms));
  return launch_k_pdl(lc, lc.pdl || pdl_mode() == 2, k_gemm_tc<BN, A_MN, B_MN, EPI, X3>, dim3(grid),
                      dim3(128 + 32 * epi_warps<BN, EPI>()), smem, a, b, c, d, X3 ? *a2 : a, X3 ? *b2 : b, g);
}

// Widest N tile that still gives >= one CTA per SM (and does not overhang N by 2x).
int pick_bn(int64_t tiles_m, int64_t N, int sms) {
  int bn = 256;
  while (bn > 64 && (N <= bn / 2 || tiles_m * ((N + bn - 1) / bn) < sms)) bn /= 2;
  return bn;
}

}  // namespace

int gemm_tc_g2_ctas(int n, int H, const WsLayout& W, int sms) {
  const int bn = W.x3 ? std::min(H, 128) : (H >= 256 ? 256 : H);
  const int64_t tiles = (int64_t)((n + BM - 1) / BM) * ((H + bn - 1) / bn) * W.splitk;
  return (int)std::min<int64_t>(tiles, sms);
}

bool tc_available() {
  std::call_once(g_once, init_encode);
  return g_encode != nullptr;
}

int64_t padded_ld(int64_t L) { return (L + 7) / 8 * 8; }

cudaError_t launch_gemm_tc(const Launch& lc, int which, int n, int64_t L, int H, const Ptrs& P,
                           const WsLayout& W, float* W2, float* b2, float* grad_w2, float* grad_b2,
                           float2* stats, int* stats_ntiles, const int32_t* dz_rows,
                           const int64_t* dz_lab_ptr, const int32_t* dz_lab, const float* hoff,
                           const DhFuse* fuse) {
  if (!tc_available()) return cudaErrorNotSupported;
  const int64_t Lp = padded_ld(L);
  CUtensorMap ta, tb, tc, ta2, tb2;
  TcArgs g{};
  cudaError_t e;
  const bool x3 = P.w2l != nullptr;   // fp32 path: bf16x3 operands (R14)
  if (x3 && which != 1 && which != 2 && which != 3) return cudaErrorNotSupported;   // Z is stored on that path
  if (which == 1 || which == 5) {  // Z = H1 W2^T + b2 (5: only the per-tile softmax partials)
    g.M = n; g.N = (int)L; g.K = H;
    g.out = P.z; g.ldo = Lp; g.bias = b2;
    const int bn = std::min(pick_bn((n + BM - 1) / BM, L, lc.sms), x3 ? 128 : 256);
    g.stats = stats; g.stats_ld = W.stats_ld;
    g.write_z = which == 1;
    g.chunked = 1;
    // per tile, one partial per epilogue column group
    const int nq = which == 1 ? 2 : (bn >= 128 ? 4 : 2);
    if (stats_ntiles) *stats_ntiles = (int)(nq * ((L + bn - 1) / bn));
    if ((e = make_map(&ta, P.h1b, H, n, (uint64_t)H * 2, 64, BM)) != cudaSuccess) return e;
    if ((e = make_map(&tb, P.w2b, H, L, (uint64_t)H * 2, 64, bn)) != cudaSuccess) return e;
    if ((e = make_store_map(&tc, P.z, L, n, (uint64_t)Lp * 4, 1, 0, 2)) != cudaSuccess) return e;
    if (x3) {
      if ((e = make_map(&ta2, P.h1l, H, n, (uint64_t)H * 2, 64, BM)) != cudaSuccess) return e;
      if ((e = make_map(&tb2, P.w2l, H, L, (uint64_t)H * 2, 64, bn)) != cudaSuccess) return e;
      if (bn == 128) return run<128, false, false, TC_EPI_Z, true>(lc, ta, tb, tc, tc, g, 1, &ta2, &tb2);
      return run<64, false, false, TC_EPI_Z, true>(lc, ta, tb, tc, tc, g, 1, &ta2, &tb2);
    }
    if (which == 5) {
      if (bn == 256) return run<256, false, false, TC_EPI_STATS>(lc, ta, tb, tc, tc, g, 1);
      if (bn == 128) return run<128, false, false, TC_EPI_STATS>(lc, ta, tb, tc, tc, g, 1);
      return run<64, false, false, TC_EPI_STATS>(lc, ta, tb, tc, tc, g, 1);
    }
    if (bn == 256) return run<256, false, false, TC_EPI_Z>(lc, ta, tb, tc, tc, g, 1);
    if (bn == 128) return run<128, false, false, TC_EPI_Z>(lc, ta, tb, tc, tc, g, 1);
    return run<64, false, false, TC_EPI_Z>(lc, ta, tb, tc, tc, g, 1);
  }
  if (which == 4 || which == 6) {
    // 4 (G1b): dZ (bf16) = (softmax(H1 W2^T + b2) - T) / B, recomputed tile by tile;
    // 6 (G1 sigmoid): dZ (bf16) = (sigmoid(H1 W2^T + b2) - Y) / B + BCE row partials
    g.M = n; g.N = (int)L; g.K = H;
    g.bias = b2; g.lse = P.lse; g.rows = dz_rows; g.lab_ptr = dz_lab_ptr; g.lab = dz_lab; g.invB = 1.f / (float)n;
    g.chunked = 1;
    const int bn = pick_bn((n + BM - 1) / BM, L, lc.sms);
    if ((e = make_map(&ta, P.h1b, H, n, (uint64_t)H * 2, 64, BM)) != cudaSuccess) return e;
    if ((e = make_map(&tb, P.w2b, H, L, (uint64_t)H * 2, 64, bn)) != cudaSuccess) return e;
    if ((e = make_bf16_store_map(&tc, P.dzb, L, n, (uint64_t)Lp * 2)) != cudaSuccess) return e;
    if (which == 6) {
      g.stats = stats; g.stats_ld = W.stats_ld;
      if (stats_ntiles) *stats_ntiles = (int)((bn >= 128 ? 4 : 2) * ((L + bn - 1) / bn));
      if (bn == 256) return run<256, false, false, TC_EPI_SIG>(lc, ta, tb, tc, tc, g, 1);
      if (bn == 128) return run<128, false, false, TC_EPI_SIG>(lc, ta, tb, tc, tc, g, 1);
      return run<64, false, false, TC_EPI_SIG>(lc, ta, tb, tc, tc, g, 1);
    }
    if (bn == 256) return run<256, false, false, TC_EPI_DZ>(lc, ta, tb, tc, tc, g, 1);
    if (bn == 128) return run<128, false, false, TC_EPI_DZ>(lc, ta, tb, tc, tc, g, 1);
    return run<64, false, false, TC_EPI_DZ>(lc, ta, tb, tc, tc, g, 1);
  }
  if (which == 2) {  // dH1 partials = dZ W2 (fuse: + the dH1 reduce, ReLU', b1 update)
    g.M = n; g.N = H; g.K = (int)L;
    g.out = P.dhpart; g.ldo = H; g.part_stride = W.part_stride;
    if (fuse) {
      g.dh_fuse = 1; g.meta = P.meta;
      g.h1 = P.h1; g.da1 = P.da1; g.da1b = fuse->want_bf16 ? P.da1b : nullptr; g.dh_off = fuse->dh_off;
      g.b1 = fuse->b1; g.grad_b1 = fuse->grad_b1; g.colpart = P.db1part; g.rowloss = P.rowloss;
      g.bar = P.meta + M_G2BAR;
    }
    const int nkb = (int)((L + BK - 1) / BK);
    const int splits = std::max(1, std::min<int>((int)W.splitk, nkb));
    if ((e = make_map(&ta, P.dzb, L, n, (uint64_t)Lp * 2, 64, BM)) != cudaSuccess) return e;
    if ((e = make_map(&tb, P.w2b, H, L, (uint64_t)H * 2, 64, 64)) != cudaSuccess) return e;
    // partial slices beyond `splits` stay untouched; dh_reduce sums W.splitk slices
    if (splits != W.splitk) return cudaErrorInvalidValue;
    const int64_t bmax = W.part_stride / H;
    if ((e = make_store_map(&tc, P.dhpart, H, bmax, (uint64_t)H * 4, splits,
                            (uint64_t)W.part_stride * 4, 3)) != cudaSuccess) return e;
    if (x3) {
      if ((e = make_map(&ta2, P.dzl, L, n, (uint64_t)Lp * 2, 64, BM)) != cudaSuccess) return e;
      if ((e = make_map(&tb2, P.w2l, H, L, (uint64_t)H * 2, 64, 64)) != cudaSuccess) return e;
      if (H >= 128) return run<128, false, true, TC_EPI_PART, true>(lc, ta, tb, tc, tc, g, splits, &ta2, &tb2);
      return run<64, false, true, TC_EPI_PART, true>(lc, ta, tb, tc, tc, g, splits, &ta2, &tb2);
    }
    if (H >= 256) return run<256, false, true, TC_EPI_PART>(lc, ta, tb, tc, tc, g, splits);
    if (H == 128) return run<128, false, true, TC_EPI_PART>(lc, ta, tb, tc, tc, g, splits);
    return run<64, false, true, TC_EPI_PART>(lc, ta, tb, tc, tc, g, splits);
  }
  // which == 3: W2 -= lr dZ^T H1
  g.M = (int)L; g.N = H; g.K = n;
  g.out = W2; g.ldo = H; g.meta = P.meta; g.shadow = P.w2b; g.grad = grad_w2;
  g.b2 = b2; g.grad_b2 = grad_b2;
  g.hoff = hoff; g.db2_off = hoff ? 0.5f : 0.f;   // centred sigmoid dZ: sum_n 1/(2B) = 1/2
  if ((e = make_map(&ta, P.dzb, L, n, (uint64_t)Lp * 2, 64, 64)) != cudaSuccess) return e;
  if ((e = make_map(&tb, P.h1b, H, n, (uint64_t)H * 2, 64, 64)) != cudaSuccess) return e;
  // N tiles of one M tile run back to back (n_fast), so the dZ^T tile is read
  // once from HBM; BN <= 128 keeps two accumulators (+ db2 column) in TMEM.
  const int64_t tiles_m = (L + BM - 1) / BM;
  int bn = std::min(H, 128);
  while (bn > 64 && tiles_m * (H / bn) < lc.sms) bn /= 2;
  g.n_fast = 1;
  CUtensorMap td;   // W2 fp32 boxes (load + store) and the bf16 shadow boxes (store)
  if ((e = make_store_map(&tc, W2, H, L, (uint64_t)H * 4, 1, 0, 2)) != cudaSuccess) return e;
  if ((e = make_bf16_store_map(&td, P.w2b, H, L)) != cudaSuccess) return e;
  if (x3) {
    g.shadow_lo = P.w2l;
    if ((e = make_map(&ta2, P.dzl, L, n, (uint64_t)Lp * 2, 64, 64)) != cudaSuccess) return e;
    if ((e = make_map(&tb2, P.h1l, H, n, (uint64_t)H * 2, 64, 64)) != cudaSuccess) return e;
    if (bn == 128) return run<128, true, true, TC_EPI_SGD, true>(lc, ta, tb, tc, td, g, 1, &ta2, &tb2);
    return run<64, true, true, TC_EPI_SGD, true>(lc, ta, tb, tc, td, g, 1, &ta2, &tb2);
  }
  if (bn == 128) return run<128, true, true, TC_EPI_SGD>(lc, ta, tb, tc, td, g, 1);
  return run<64, true, true, TC_EPI_SGD>(lc, ta, tb, tc, td, g, 1);
}

bool bwd_dh_one_pass_fits(int n, int64_t L, const WsLayout& W, int sms) {
  const int MT = (n + BM - 1) / BM;
  const int64_t T = (L + kBwdBN - 1) / kBwdBN;
  const int64_t LR = std::max<int64_t>(1, std::min<int64_t>({(int64_t)(sms / MT), T, (int64_t)W.dh_parts}));
  return 2 * LR <= (L + 31) / 32 + 8;   // the partials fit the G1 stats area
}

cudaError_t launch_bwd_dh(const Launch& lc, int n, int64_t L, int H, const Ptrs& P, const WsLayout& W, float* b2,
                          const int32_t* rows, const int64_t* lab_ptr, const int32_t* lab, const DhFuse& fz,
                          bool write_dz, bool one_pass, float2* stats, bool dz_only) {
  if (!tc_available()) return cudaErrorNotSupported;
  if (H != 256 || P.w2l) return cudaErrorNotSupported;   // bf16 path, H = 256 (one N = 256 MMA)
  const int64_t Lp = padded_ld(L);
  const int MT = (n + BM - 1) / BM;
  const int64_t T = (L + kBwdBN - 1) / kBwdBN;
  // label ranges: one per SM pair of row blocks, at most the dH1 partial slices the
  // workspace holds (the one-pass regime has room for one range per tile)
  if (dz_only) one_pass = write_dz = true;
  const int LR = (int)std::max<int64_t>(
      1, std::min<int64_t>({(int64_t)(lc.sms / MT), T,
                            (int64_t)(dz_only ? T : one_pass ? W.dh_parts : W.splitk)}));
  CUtensorMap th, tw, tz;
  cudaError_t e;
  if ((e = make_map(&th, P.h1b, H, n, (uint64_t)H * 2, 64, BM)) != cudaSuccess) return e;
  if ((e = make_map(&tw, P.w2b, H, L, (uint64_t)H * 2, 64, kBwdBN)) != cudaSuccess) return e;
  if ((e = make_map(&tz, P.dzb, L, n, (uint64_t)Lp * 2, kBwdBN, BM)) != cudaSuccess) return e;
  TcArgs g{};
  g.M = n; g.N = (int)L; g.K = H;
  g.out = P.dhpart; g.ldo = H; g.part_stride = W.part_stride; g.splits = LR;
  g.bias = b2; g.lse = P.lse; g.rows = rows; g.lab_ptr = lab_ptr; g.lab = lab; g.invB = 1.f / (float)n;
  g.write_z = write_dz ? 1 : 0;
  g.dh_fuse = 1; g.meta = P.meta;
  g.h1 = P.h1; g.da1 = P.da1; g.da1b = fz.want_bf16 ? P.da1b : nullptr; g.dh_off = fz.dh_off;
  g.b1 = fz.b1; g.grad_b1 = fz.grad_b1; g.colpart = P.db1part; g.rowloss = P.rowloss;
  g.bar = P.meta + M_G2BAR;
  if (one_pass) {
    // (max, sum) partials [LR][B] float2 + label-logit sums [LR][B] float: the G1 stats area
    if (2 * LR > (L + 31) / 32 + 8) return cudaErrorNotSupported;
    g.one_pass = 1;
    g.stats = stats; g.stats_ld = W.stats_ld;
    g.rowloss_w = P.rowloss;
    g.gbar = reinterpret_cast<unsigned long long*>(P.meta + M_KBAR);
    g.dz_only = dz_only ? 1 : 0;
  }
  // two epilogue groups (two label tiles drained at once) unless a one-pass mode needs the
  // single-group statistics exchange; ASGD_K3_EG=1 keeps one group.  Measured: Amazon-670K
  // 0.467 -> 0.490 M samples/s, AmazonCat-13K even (5.48 / 5.46 M)
  static const int eg_env = [] { const char* v = getenv("ASGD_K3_EG"); return v ? atoi(v) : 2; }();
  const int eg = (one_pass || eg_env == 1) ? 1 : 2;
  const size_t smem = kBwdH1Bytes + kBwdStages * kBwdW2Bytes + 2 * kBwdDzBytes + eg * kBwdEpi * 32 * 4 +
                      128 * 3 * 4 + 1024 + 256;
  if (eg == 2) {
    if ((e = ensure_smem(k_bwd_dh<2>, smem)) != cudaSuccess) return e;
    return launch_k_pdl(lc, lc.pdl || pdl_mode() == 2, k_bwd_dh<2>, dim3(MT * LR), dim3(128 + 32 * kBwdEpi * 2),
                        smem, th, tw, tz, g, LR);
  }
  if ((e = ensure_smem(k_bwd_dh<1>, smem)) != cudaSuccess) return e;
  return launch_k_pdl(lc, lc.pdl || pdl_mode() == 2, k_bwd_dh<1>, dim3(MT * LR), dim3(128 + 32 * kBwdEpi), smem, th,
                      tw, tz, g, LR);
}

cudaError_t launch_bwd_dw(const Launch& lc, int n, int64_t L, int H, const Ptrs& Pr, const Ptrs& Pw, float* W2,
                          float* b2, const int32_t* rows, const int64_t* lab_ptr, const int32_t* lab,
                          float* grad_w2, float* grad_b2) {
  if (!tc_available()) return cudaErrorNotSupported;
  if (H != 256 || Pr.w2l || n > kDwMaxRows) return cudaErrorNotSupported;
  CUtensorMap tw, th;
  cudaError_t e;
  if ((e = make_map(&tw, Pr.w2b, H, L, (uint64_t)H * 2, 64, kDwBM)) != cudaSuccess) return e;
  if ((e = make_map(&th, Pr.h1b, H, n, (uint64_t)H * 2, 64, kDwRB)) != cudaSuccess) return e;
  TcArgs g{};
  g.M = (int)L; g.N = H; g.K = n;
  g.out = W2; g.ldo = H; g.meta = Pr.meta; g.shadow = Pw.w2b; g.grad = grad_w2;
  g.b2 = b2; g.grad_b2 = grad_b2; g.bias = b2;
  g.lse = Pr.lse; g.rows = rows; g.lab_ptr = lab_ptr; g.lab = lab; g.invB = 1.f / (float)n;
  const size_t smem = kDwW2Bytes + 2 * kDwH1Bytes + 2 * kDwDzBytes + kBwdEpi * 4096 + 2 * kDwRB * 8 +
                      2 * kDwBM * 2 * 4 + 2 * kDwBM * 4 + 2 * kDwMaxRows * 4 + 256 + 1024;
  if ((e = ensure_smem(k_bwd_dw, smem)) != cudaSuccess) return e;
  const int64_t T = (L + kDwBM - 1) / kDwBM;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(T, lc.sms));
  return launch_k_pdl(lc, lc.pdl || pdl_mode() == 2, k_bwd_dw, dim3(grid), dim3(128 + 32 * kBwdEpi), smem, tw, th, g);
}

}  // namespace asgd


namespace asgd {
ASGD_TL_SETTER(tl_set_tc)
}  // namespace asgd
