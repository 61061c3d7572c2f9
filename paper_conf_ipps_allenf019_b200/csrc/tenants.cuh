// tenants.cuh -- tenant kernel bodies K(B,T).
//
// Each body is written once as cta_block(): what the T threads of original
// block (x,y,z) do.  It is called both by the original kernel on the hardware
// block scheduler (standalone<Tn>) and by the slate worker (slate_worker<Tn>)
// with the block index the worker decoded, so the outputs of the two are
// bit-identical: the per-element arithmetic is the same instruction sequence
// (explicit __fmaf_rn etc. so the compiler cannot contract differently).
// Blocks own disjoint output slices; a body may use __syncthreads (all T
// threads of the worker CTA reach it).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "../../include/slate.h"

namespace slate {

__device__ __forceinline__ float4 ld_stream(const float4* p) { return __ldcs(p); }
__device__ __forceinline__ void st_stream(float4* p, float4 v) { __stcs(p, v); }

// ============================================================== triad  a = b + s*c
// 1024 elements per block; thread t handles the float4 at x*256 + t.
struct Triad {
  using Args = slate_args_triad;
  static constexpr int kThreads = 256;
  static constexpr int kSmem = 0;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char*) {
    const uint64_t v = uint64_t(x) * 256 + threadIdx.x;
    const uint64_t i0 = v * 4;
    if (i0 + 4 <= a.n) {
      const float4 b = ld_stream(reinterpret_cast<const float4*>(a.b) + v);
      const float4 c = ld_stream(reinterpret_cast<const float4*>(a.c) + v);
      st_stream(reinterpret_cast<float4*>(a.a) + v,
                make_float4(__fmaf_rn(a.s, c.x, b.x), __fmaf_rn(a.s, c.y, b.y), __fmaf_rn(a.s, c.z, b.z),
                            __fmaf_rn(a.s, c.w, b.w)));
    } else {
      const float* b = reinterpret_cast<const float*>(a.b);
      const float* c = reinterpret_cast<const float*>(a.c);
      float* o = reinterpret_cast<float*>(a.a);
      for (uint64_t i = i0; i < a.n && i < i0 + 4; ++i) o[i] = __fmaf_rn(a.s, c[i], b[i]);
    }
  }
};

// ============================================================== copy  a = b
// 4096 elements (16 KiB) per block; thread t copies float4s x*1024 + t + 128 j.
struct Copy {
  using Args = slate_args_copy;
  static constexpr int kThreads = 128;
  static constexpr int kSmem = 0;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char*) {
    const float4* B = reinterpret_cast<const float4*>(a.b);
    float4* A = reinterpret_cast<float4*>(a.a);
    const uint64_t base = uint64_t(x) * 1024 + threadIdx.x;
    if ((uint64_t(x) + 1) * 4096 <= a.n) {
      float4 v[8];
#pragma unroll
      for (int j = 0; j < 8; ++j) v[j] = ld_stream(B + base + 128 * j);
#pragma unroll
      for (int j = 0; j < 8; ++j) st_stream(A + base + 128 * j, v[j]);
    } else {
      const float* b = reinterpret_cast<const float*>(a.b);
      float* o = reinterpret_cast<float*>(a.a);
      for (int j = 0; j < 8; ++j) {
        const uint64_t i0 = (base + 128 * j) * 4;
        for (uint64_t i = i0; i < i0 + 4 && i < a.n; ++i) o[i] = b[i];
      }
    }
  }
};

// ============================================================== naive SGEMM  C = A B
// The CUDA-sample-style naive kernel: one thread per C element, no tiling.
struct SgemmNaive {
  using Args = slate_args_sgemm;
  static constexpr int kThreads = 256;        // 16 x 16
  static constexpr int kSmem = 0;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t y, uint32_t, char*) {
    const uint32_t tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
    const uint32_t r = y * 16 + ty, c = x * 16 + tx;
    if (r >= a.m || c >= a.n) return;
    const float* A = reinterpret_cast<const float*>(a.A) + uint64_t(r) * a.k;
    const float* B = reinterpret_cast<const float*>(a.B) + c;
    float acc = 0.f;
    for (uint32_t k = 0; k < a.k; ++k) acc = __fmaf_rn(__ldg(A + k), __ldg(B + uint64_t(k) * a.n), acc);
    reinterpret_cast<float*>(a.C)[uint64_t(r) * a.n + c] = acc;
  }
};

// ============================================================== CSR SpMV  y = A x
// 32 rows per block; warp w handles rows 4w..4w+3 with 8 lanes per row: lane l
// sums j = rp[row]+l, +8, ... in order (fmaf chain), then a butterfly
// (xor 4, 2, 1) inside the 8-lane group.
struct SpmvCsr {
  using Args = slate_args_spmv;
  static constexpr int kThreads = 256;
  static constexpr int kSmem = 0;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char*) {
    const int* rp = reinterpret_cast<const int*>(a.rowptr);
    const int* col = reinterpret_cast<const int*>(a.col);
    const float* val = reinterpret_cast<const float*>(a.val);
    const float* xv = reinterpret_cast<const float*>(a.x);
    const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint32_t l = lane & 7;
    const uint32_t row = x * 32 + w * 4 + (lane >> 3);
    int lo = 0, hi = 0;
    if (row < a.n_rows) {
      lo = __ldg(rp + row) + int(l);
      hi = __ldg(rp + row + 1);
    }
    float acc = 0.f;
    int j = lo;
    // two independent gathers in flight per lane per round (rows of ~16 nnz: one round)
    for (; j + 8 < hi; j += 16) {
      const int c0 = __ldcs(col + j), c1 = __ldcs(col + j + 8);
      const float v0 = __ldcs(val + j), v1 = __ldcs(val + j + 8);
      const float x0 = __ldg(xv + c0), x1 = __ldg(xv + c1);
      acc = __fmaf_rn(v0, x0, acc);
      acc = __fmaf_rn(v1, x1, acc);
    }
    if (j < hi) acc = __fmaf_rn(__ldcs(val + j), __ldg(xv + __ldcs(col + j)), acc);
    acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, 4));
    acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, 2));
    acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, 1));
    if (l == 0 && row < a.n_rows) __stcs(reinterpret_cast<float*>(a.y) + row, acc);
  }
};

// ============================================================== Black-Scholes
// European call/put; each option priced under n_scen volatilities (reading
// Q16), output the mean.  Thread t of block x prices options 4(x*256+t)..+3.
struct BlackScholes {
  using Args = slate_args_bs;
  static constexpr int kThreads = 256;
  static constexpr int kSmem = 0;

  __device__ __forceinline__ static void price(float S, float X, float T, float r, const float* sig, uint32_t P,
                                               float& call, float& put) {
    const float sqt = sqrtf(T);
    const float lsx = logf(__fdiv_rn(S, X));
    const float xd = __fmul_rn(X, expf(__fmul_rn(-r, T)));
    float cs = 0.f, ps = 0.f;
    for (uint32_t p = 0; p < P; ++p) {
      const float sg = __ldg(sig + p);
      const float sst = __fmul_rn(sg, sqt);
      const float d1 = __fdiv_rn(__fmaf_rn(__fmaf_rn(0.5f * sg, sg, r), T, lsx), sst);
      const float d2 = __fsub_rn(d1, sst);
      const float n1 = normcdff(d1), n2 = normcdff(d2);
      const float m1 = normcdff(-d1), m2 = normcdff(-d2);
      cs = __fadd_rn(cs, __fsub_rn(__fmul_rn(S, n1), __fmul_rn(xd, n2)));
      ps = __fadd_rn(ps, __fsub_rn(__fmul_rn(xd, m2), __fmul_rn(S, m1)));
    }
    call = __fdiv_rn(cs, float(P));
    put = __fdiv_rn(ps, float(P));
  }
  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char*) {
    const uint64_t v = uint64_t(x) * 256 + threadIdx.x;
    const uint64_t i0 = v * 4;
    const float* sig = reinterpret_cast<const float*>(a.sigmas);
    if (i0 + 4 <= a.n) {
      const float4 S = __ldcs(reinterpret_cast<const float4*>(a.S) + v);
      const float4 X = __ldcs(reinterpret_cast<const float4*>(a.X) + v);
      const float4 T = __ldcs(reinterpret_cast<const float4*>(a.T) + v);
      float4 c, p;
      price(S.x, X.x, T.x, a.r, sig, a.n_scen, c.x, p.x);
      price(S.y, X.y, T.y, a.r, sig, a.n_scen, c.y, p.y);
      price(S.z, X.z, T.z, a.r, sig, a.n_scen, c.z, p.z);
      price(S.w, X.w, T.w, a.r, sig, a.n_scen, c.w, p.w);
      __stcs(reinterpret_cast<float4*>(a.call) + v, c);
      __stcs(reinterpret_cast<float4*>(a.put) + v, p);
    } else {
      for (uint64_t i = i0; i < a.n && i < i0 + 4; ++i) {
        float c, p;
        price(reinterpret_cast<const float*>(a.S)[i], reinterpret_cast<const float*>(a.X)[i],
              reinterpret_cast<const float*>(a.T)[i], a.r, sig, a.n_scen, c, p);
        reinterpret_cast<float*>(a.call)[i] = c;
        reinterpret_cast<float*>(a.put)[i] = p;
      }
    }
  }
};

// ============================================================== 2-D 5-point stencil
// One Jacobi sweep of an h x w field; 32 x 8 points per block.  Each thread
// owns one point; the up/down neighbours come from the rows above/below
// (L1/L2 reuse across the block's warps), left/right via warp shuffles with
// the two block-edge columns loaded directly.
struct Stencil2D {
  using Args = slate_args_stencil;
  static constexpr int kThreads = 256;        // 32 x 8
  static constexpr int kSmem = 0;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t bx, uint32_t by, uint32_t, char*) {
    const float* in = reinterpret_cast<const float*>(a.in);
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const int i = int(by) * 8 + ty, j = int(bx) * 32 + tx;
    const int h = int(a.h), w = int(a.w);
    const bool inside = i < h && j < w;
    const float c = inside ? __ldg(in + uint64_t(i) * w + j) : 0.f;
    float left = __shfl_up_sync(0xffffffffu, c, 1);
    float right = __shfl_down_sync(0xffffffffu, c, 1);
    if (!inside) return;
    if (i == 0 || j == 0 || i == h - 1 || j == w - 1) {
      reinterpret_cast<float*>(a.out)[uint64_t(i) * w + j] = c;
      return;
    }
    if (tx == 0) left = __ldg(in + uint64_t(i) * w + j - 1);
    if (tx == 31) right = __ldg(in + uint64_t(i) * w + j + 1);
    const float up = __ldg(in + uint64_t(i - 1) * w + j), down = __ldg(in + uint64_t(i + 1) * w + j);
    const float v = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(up, down), __fadd_rn(left, right)));
    reinterpret_cast<float*>(a.out)[uint64_t(i) * w + j] = v;
  }
};

}  // namespace slate
