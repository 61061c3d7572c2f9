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
#include "slate_device.cuh"   // TenantBase

namespace slate {

__device__ __forceinline__ float4 ld_stream(const float4* p) { return __ldcs(p); }
__device__ __forceinline__ void st_stream(float4* p, float4 v) { __stcs(p, v); }

#ifndef SLATE_SPEC_SHORT
#define SLATE_SPEC_SHORT 0   // experiment switch: speculative task fetch for the short-block Tab II tenants
#endif


// ------------------------------------------------------------------ bulk async copies (TMA engine)
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// streaming data is marked evict-first in L2 so a co-running tenant's working
// set (e.g. the GEMM's operand panels) is not flushed by it
__device__ __forceinline__ uint64_t l2_evict_first() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void bulk_g2s(void* dst_smem, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst_smem)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(l2_evict_first())  // racecheck: mbarrier-ordered
      : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src_smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(dst),
               "r"(smem_u32(src_smem)), "r"(bytes), "l"(l2_evict_first())
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// ============================================================== triad  a = b + s*c
// 1024 elements per block; thread t handles the float4 at x*256 + t.
struct Triad : TenantBase {
  using Args = slate_args_triad;
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 8;       // 32 registers, no spill: 64 warps/SM for HBM latency
  static constexpr int kSmem = 0, kSmemStandalone = 0;

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
// 4096 elements (16 KiB) per block, moved global -> shared -> global by the
// bulk-copy (TMA) engine: one thread issues, no registers hold data.  The
// worker streams a task's blocks -- contiguous in memory -- through kStages
// shared-memory stages of kUnit blocks each: one bulk load and one bulk store
// per unit, loads of later units in flight while earlier ones are stored.
// Units never cross a task boundary (the next task's blocks are elsewhere in
// memory).  Measured (round 2, tools/copy_probe.py): with 1-block units in 4
// stages (64 KiB, 3 CTAs per SM) an SM moves ~100 GB/s of copy traffic (read +
// write), HBM saturates at ~70 of 148 SMs; 64-KiB units in 3 stages (1 CTA
// per SM) reach only ~64 GB/s per SM, 32-KiB units x 2 stages (3 CTAs) the
// same ~100: the SM's own memory interface, not the per-copy cost, is the
// limit, and a copy tenant cannot saturate HBM on fewer SMs.
struct Copy : TenantBase {
  using Args = slate_args_copy;
  static constexpr int kThreads = 128;
#ifndef SLATE_COPY_STAGES
#define SLATE_COPY_STAGES 4
#endif
#ifndef SLATE_COPY_UNIT
#define SLATE_COPY_UNIT 1
#endif
  static constexpr int kStages = SLATE_COPY_STAGES;
  static constexpr int kUnit = SLATE_COPY_UNIT;           // blocks per stage
  static constexpr int kBlockBytes = 16384;
  static constexpr int kHdr = 128;                        // barriers + parity word
  static constexpr int kSmem = kHdr + kStages * kUnit * kBlockBytes;
  static constexpr int kSmemStandalone = kHdr + kBlockBytes;
  static constexpr bool kHasInit = true, kLookahead = true, kHasFini = true;

  __device__ __forceinline__ static uint64_t* bars(char* smem) { return reinterpret_cast<uint64_t*>(smem); }
  __device__ __forceinline__ static uint32_t* parity(char* smem) { return reinterpret_cast<uint32_t*>(smem + 64); }
  __device__ __forceinline__ static uint32_t* state(char* smem) { return reinterpret_cast<uint32_t*>(smem + 72); }
  __device__ __forceinline__ static char* stage(char* smem, int s) { return smem + kHdr + s * kUnit * kBlockBytes; }

  __device__ __forceinline__ static void cta_init(char* smem) {
    if (threadIdx.x == 0) {
      for (int i = 0; i < kStages; ++i) mbar_init(bars(smem) + i, 1);
      *parity(smem) = 0;
      state(smem)[0] = 0;
      state(smem)[1] = 0;
      fence_mbar_init();
    }
  }
  __device__ __forceinline__ static void cta_fini(char*) {
    if (threadIdx.x == 0) bulk_wait0();          // stores complete before the CTA exits
  }
  // bytes of blocks [x0, x1) moved by the bulk engine (a multiple of 16); the rest by threads
  __device__ __forceinline__ static uint32_t bulk_bytes(const Args& a, uint32_t x0, uint32_t x1) {
    const uint64_t e0 = uint64_t(x0) * 4096;
    const uint64_t e1 = min(uint64_t(x1) * 4096, a.n);
    return e1 > e0 ? uint32_t(((e1 - e0) * 4) & ~uint64_t(15)) : 0u;
  }
  __device__ __forceinline__ static void tail(const Args& a, uint32_t x0, uint32_t x1) {
    const uint64_t e0 = uint64_t(x0) * 4096 + bulk_bytes(a, x0, x1) / 4;
    const uint64_t e1 = min(uint64_t(x1) * 4096, a.n);
    for (uint64_t i = e0; i < e1; ++i) reinterpret_cast<float*>(a.a)[i] = reinterpret_cast<const float*>(a.b)[i];
  }
  __device__ __forceinline__ static void issue_load(const Args& a, char* smem, uint32_t x0, uint32_t x1, int s) {
    const uint32_t nb = bulk_bytes(a, x0, x1);
    mbar_expect_tx(bars(smem) + s, nb);
    bulk_g2s(stage(smem, s), reinterpret_cast<const char*>(a.b) + uint64_t(x0) * kBlockBytes, nb, bars(smem) + s);
  }
  __device__ __forceinline__ static void wait_load(char* smem, int s) {
    uint32_t& par = *parity(smem);
    mbar_wait(bars(smem) + s, (par >> s) & 1u);
    par ^= 1u << s;
  }
  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char* smem) {
    if (threadIdx.x != 0) return;
    bulk_wait_read0();                           // the buffer is free
    if (bulk_bytes(a, x, x + 1)) {
      issue_load(a, smem, x, x + 1, 0);
      wait_load(smem, 0);
      bulk_s2g(reinterpret_cast<char*>(a.a) + uint64_t(x) * kBlockBytes, stage(smem, 0), bulk_bytes(a, x, x + 1));
      bulk_commit();
    }
    tail(a, x, x + 1);
  }
  // The units of this task (blocks [g, g+n)) and of the next one ([g2, g2+n2))
  // form one stream through the stage ring: while the last stores of this task
  // drain, the first loads of the next task are already in flight.  state: [0]
  // units of this task already loaded by the previous call, [1] stage of this
  // task's first unit.
  __device__ __forceinline__ static void cta_task2(const Args& a, uint32_t g, uint32_t n, uint32_t g2, uint32_t n2,
                                                   char* smem) {
    if (threadIdx.x != 0) return;
    uint32_t* st = state(smem);
    const uint32_t pre = st[0], seq = st[1];
    const uint32_t ua = (n + kUnit - 1) / kUnit, ub = (n2 + kUnit - 1) / kUnit;
    const uint32_t total = ua + ub;
    auto first = [&](uint32_t k) { return k < ua ? g + k * kUnit : g2 + (k - ua) * kUnit; };
    auto last = [&](uint32_t k) { return k < ua ? min(g + (k + 1) * kUnit, g + n) : min(g2 + (k - ua + 1) * kUnit, g2 + n2); };
    auto stg = [&](uint32_t k) { return int((seq + k) % kStages); };
    uint32_t issued = pre;
    if (issued < kStages) bulk_wait_read0();   // stages about to be refilled have been read out
    for (; issued < min(total, uint32_t(kStages)); ++issued)
      if (bulk_bytes(a, first(issued), last(issued))) issue_load(a, smem, first(issued), last(issued), stg(issued));
    for (uint32_t i = 0; i < ua; ++i) {
      const uint32_t x0 = first(i), x1 = last(i);
      const uint32_t nb = bulk_bytes(a, x0, x1);
      if (nb) {
        wait_load(smem, stg(i));
        bulk_s2g(reinterpret_cast<char*>(a.a) + uint64_t(x0) * kBlockBytes, stage(smem, stg(i)), nb);
        bulk_commit();
      }
      tail(a, x0, x1);
      if (issued < total && issued == i + kStages) {
        bulk_wait_read0();                       // the stage of unit i has been read by its store
        if (bulk_bytes(a, first(issued), last(issued))) issue_load(a, smem, first(issued), last(issued), stg(issued));
        ++issued;
      }
    }
    st[0] = issued > ua ? issued - ua : 0;
    st[1] = (seq + ua) % kStages;
  }
};

// ============================================================== naive SGEMM  C = A B
// The CUDA-sample-style naive kernel: one thread per C element, no tiling.
struct SgemmNaive : TenantBase {
  using Args = slate_args_sgemm;
  static constexpr int kThreads = 256;        // 16 x 16
  static constexpr int kMinBlocks = 8;       // 32 registers, no spill (the worker logic alone pushed it to 64)
  static constexpr int kSmem = 0, kSmemStandalone = 0;

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
// The row reduction order, shared by the original kernel below and the worker
// (spmv_ws.cu), so their y are bit-identical: a row's nonzeros are taken in
// aligned 16-byte segments -- entries 4s .. 4s+3 of the col / val arrays, those
// outside the row's [rp[row], rp[row+1]) skipped -- and lane q of the row's
// 4-lane group sums segments s0+q, s0+q+4, ... (s0 = rp[row] / 4) in ascending
// order, each segment's entries ascending, as one fmaf chain from 0; the group
// then adds with a xor 2, 1 butterfly.  One 128-bit load of columns and one of
// values per lane and segment (coalesced: a warp reads 8 rows x 16 nonzeros as
// 512 contiguous bytes of each array).  The oracle is order-free (fp64; exact
// on integer inputs), so the order is this build's choice.
namespace spmvseg {
struct Seg {
  int4 c;
  float4 v;
};
// entries base .. base+3 (base a multiple of 4) that exist in the arrays (< nnz)
__device__ __forceinline__ Seg load(const int* __restrict__ col, const float* __restrict__ val, int base, int nnz,
                                    bool any) {
  Seg s;
  s.c = make_int4(0, 0, 0, 0);
  s.v = make_float4(0.f, 0.f, 0.f, 0.f);
  if (!any) return s;
  if (base + 4 <= nnz) {
    s.c = __ldcs(reinterpret_cast<const int4*>(col + base));
    s.v = __ldcs(reinterpret_cast<const float4*>(val + base));
  } else {   // the array's last, partial segment
    if (base + 0 < nnz) { s.c.x = __ldcs(col + base + 0); s.v.x = __ldcs(val + base + 0); }
    if (base + 1 < nnz) { s.c.y = __ldcs(col + base + 1); s.v.y = __ldcs(val + base + 1); }
    if (base + 2 < nnz) { s.c.z = __ldcs(col + base + 2); s.v.z = __ldcs(val + base + 2); }
  }
  return s;
}
// acc <- the segment's entries of the row [lo, hi), ascending.  Branch-free:
// an entry outside the row contributes fmaf(0, x[csafe], acc) with csafe a
// column whose x is finite (the original kernel and the worker compute the
// same expression, so their bits agree; a -0 sum may become +0, which the
// oracle's comparison does not distinguish)
template <class XF>
__device__ __forceinline__ float fma_seg(float acc, const Seg& s, int base, int lo, int hi, int csafe, XF xval) {
  const bool e0 = base + 0 >= lo && base + 0 < hi, e1 = base + 1 >= lo && base + 1 < hi;
  const bool e2 = base + 2 >= lo && base + 2 < hi, e3 = base + 3 >= lo && base + 3 < hi;
  const float x0 = xval(e0 ? s.c.x : csafe), x1 = xval(e1 ? s.c.y : csafe);
  const float x2 = xval(e2 ? s.c.z : csafe), x3 = xval(e3 ? s.c.w : csafe);
  acc = __fmaf_rn(e0 ? s.v.x : 0.f, x0, acc);
  acc = __fmaf_rn(e1 ? s.v.y : 0.f, x1, acc);
  acc = __fmaf_rn(e2 ? s.v.z : 0.f, x2, acc);
  acc = __fmaf_rn(e3 ? s.v.w : 0.f, x3, acc);
  return acc;
}
// lane q's chain over segments s0+q+4m for m >= m0 (the row's remaining segments)
template <class XF>
__device__ __forceinline__ float row_tail(float acc, const int* col, const float* val, int nnz, int lo, int hi, int q,
                                          int m0, int csafe, XF xval) {
  for (int base = ((lo >> 2) + q + 4 * m0) * 4; base < hi; base += 16)
    acc = fma_seg(acc, load(col, val, base, nnz, true), base, lo, hi, csafe, xval);
  return acc;
}
__device__ __forceinline__ float reduce4(float v) {
  v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, 2));
  v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, 1));
  return v;
}
}  // namespace spmvseg

// The original kernel K(B,T): 32 rows per block, 4 lanes per row (T = 128), x
// from global memory.  Its slate worker is the warp-specialised one in
// spmv_ws.cu (same per-row arithmetic).
struct SpmvSeg : TenantBase {
  using Args = slate_args_spmv;
  static constexpr int kThreads = 128;
  static constexpr int kMinBlocks = 16;
  static constexpr int kSmem = 0, kSmemStandalone = 0;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char*) {
    const int* __restrict__ rp = reinterpret_cast<const int*>(a.rowptr);
    const int* __restrict__ col = reinterpret_cast<const int*>(a.col);
    const float* __restrict__ val = reinterpret_cast<const float*>(a.val);
    const float* __restrict__ xv = reinterpret_cast<const float*>(a.x);
    const uint32_t row = x * 32 + (threadIdx.x >> 2);
    const int q = int(threadIdx.x & 3);
    const int nnz = __ldg(rp + a.n_rows);
    int lo = 0, hi = 0;
    if (row < a.n_rows) {
      lo = __ldg(rp + row);
      hi = __ldg(rp + row + 1);
    }
    const float acc = spmvseg::row_tail(0.f, col, val, nnz, lo, hi, q, 0, 0, [&](int c) { return __ldg(xv + c); });
    const float v = spmvseg::reduce4(acc);
    if (q == 0 && row < a.n_rows) __stcs(reinterpret_cast<float*>(a.y) + row, v);
  }
};

// ============================================================== Black-Scholes
// European call/put as in the CUDA SDK BlackScholes sample: the normal CDF by
// the Abramowitz-Stegun polynomial (|error| < 7.5e-8), put by 1 - CND; each
// option priced under n_scen volatilities (reading Q16) and the mean written.
// Thread t of block x prices options 4(x*256+t)..+3.
// B200 has one MUFU (SFU) op per 2 FP32 lanes' worth of issue less than B300, so
// the body is arranged around MUFU count (5 -> 2.25 per option-scenario),
// with exact identities: 1/(sigma sqrt T) = (1/sigma)(1/sqrt T) with 1/sigma
// shared by a thread's 4 options; both A&S K = 1/(1 + 0.2316419|d|) from one
// reciprocal (K1 = u2/(u1 u2), K2 = u1/(u1 u2)); and the density at d2 from the
// one at d1: exp(-d2^2/2) = exp(-d1^2/2) S / (X e^{-rT}) (d1 sigma sqrt T =
// ln(S/X) + (r + sigma^2/2) T); the put by put-call parity, put = call + X e^{-rT}
// - S for every scenario, hence for their mean.
#ifndef SLATE_BS_MINB
#define SLATE_BS_MINB 4
#endif
struct BlackScholes : TenantBase {
  using Args = slate_args_bs;
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = SLATE_BS_MINB;
  static constexpr bool kLateCtrl = !SLATE_SPEC_SHORT;    // a block is ~30 us at P = 32: honour a resize after it
  static constexpr bool kSpeculative = SLATE_SPEC_SHORT;
  static constexpr int kSmem = 0, kSmemStandalone = 0;

  // one MUFU op each, no denormal range handling: every argument here is a
  // normal float (u1 u2 >= 1, sigma > 0), and an exponent below -126 only
  // flushes a density of < 1e-38 to 0 (__fdividef / __expf spend 4-5 more
  // instructions per call on those guards; the body is issue-bound)
  __device__ __forceinline__ static float rcp(float x) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
  }
  __device__ __forceinline__ static float exp_(float x) {
    float r;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(__fmul_rn(x, 1.44269504088896341f)));
    return r;
  }
  __device__ __forceinline__ static float poly(float K) {
    const float A1 = 0.31938153f, A2 = -0.356563782f, A3 = 1.781477937f, A4 = -1.821255978f, A5 = 1.330274429f;
    return __fmul_rn(K, __fmaf_rn(K, __fmaf_rn(K, __fmaf_rn(K, __fmaf_rn(K, A5, A4), A3), A2), A1));
  }
  // options o = 0..k-1 of this thread (k = 4, or 1..3 on the ragged tail)
  // ---- packed FP32x2 (sm_100: FFMA2 / FMUL2 / FADD2): two options per instruction
  // The body is issue-bound (~39 instructions per option-scenario against ~30
  // FP32-pipe cycles); a packed op does two options' work in one issue slot
  // (tools/probe/ffma2_rate.cu: the FP32 pipe rate is the same, so this pays
  // only where issue, not the pipe, is the limit).  Per element the same
  // round-to-nearest ops as price<k>; ptxas may contract a packed mul + add
  // into FFMA2, so results can differ from price<k> by an ulp (Q39).
  typedef unsigned long long f2;
  __device__ __forceinline__ static f2 pk(float a, float b) {
    f2 r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
  }
  __device__ __forceinline__ static void up(f2 v, float& a, float& b) { asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v)); }
  __device__ __forceinline__ static f2 fma2(f2 a, f2 b, f2 c) {
    f2 d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
    return d;
  }
  __device__ __forceinline__ static f2 mul2(f2 a, f2 b) {
    f2 d;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
  }
  __device__ __forceinline__ static f2 add2(f2 a, f2 b) {
    f2 d;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
  }
  __device__ __forceinline__ static f2 sub2(f2 a, f2 b) {
    f2 d;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
  }
  __device__ __forceinline__ static f2 abs2(f2 a) { return a & 0x7fffffff7fffffffull; }
  // the A&S polynomial, negated, with 1/sqrt(2 pi) folded into its coefficients
  __device__ __forceinline__ static f2 poly2rn(f2 K) {
    const float R = -0.39894228040143267794f;
    const f2 A1 = pk(0.31938153f * R, 0.31938153f * R), A2 = pk(-0.356563782f * R, -0.356563782f * R),
             A3 = pk(1.781477937f * R, 1.781477937f * R), A4 = pk(-1.821255978f * R, -1.821255978f * R),
             A5 = pk(1.330274429f * R, 1.330274429f * R);
    return mul2(K, fma2(K, fma2(K, fma2(K, fma2(K, A5, A4), A3), A2), A1));
  }
  // 4 options as two packed pairs (0,1) and (2,3); the per-option setup and the
  // final mean are price<4>'s scalar code
  __device__ __forceinline__ static void price4_x2(const float (&S)[4], const float (&X)[4], const float (&T)[4], float r,
                                                   const float* sig, uint32_t P, float (&call)[4], float (&put)[4]) {
    float sqt[4], rsqt[4], lsx[4], xd[4], sxd[4];
#pragma unroll
    for (int o = 0; o < 4; ++o) {
      sqt[o] = sqrtf(T[o]);
      rsqt[o] = __fdiv_rn(1.0f, sqt[o]);
      lsx[o] = logf(__fdiv_rn(S[o], X[o]));
      xd[o] = __fmul_rn(X[o], expf(__fmul_rn(-r, T[o])));
      sxd[o] = __fdiv_rn(S[o], xd[o]);
    }
    // per option: sqrt(T), ln(S/X)/sqrt(T), S, -X e^{-rT}, S/(X e^{-rT}); then per
    // scenario d1 = (hs2 sqrt(T) + ln(S/X)/sqrt(T)) / sigma  (= (ln(S/X) + hs2 T) /
    // (sigma sqrt(T))) and d2 = d1 - sigma sqrt(T): 3 FP32 ops instead of 5
    f2 SQT[2], LQ[2], SS[2], NXD[2], SXD[2], CS[2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      SQT[h] = pk(sqt[2 * h], sqt[2 * h + 1]);
      LQ[h] = pk(__fmul_rn(lsx[2 * h], rsqt[2 * h]), __fmul_rn(lsx[2 * h + 1], rsqt[2 * h + 1]));
      SS[h] = pk(S[2 * h], S[2 * h + 1]);
      NXD[h] = pk(-xd[2 * h], -xd[2 * h + 1]);
      SXD[h] = pk(sxd[2 * h], sxd[2 * h + 1]);
      CS[h] = pk(0.f, 0.f);
    }
    // d1, d2 are carried scaled by C = sqrt(log2(e)/2): exp(-d1^2/2) = 2^-(C d1)^2
    // (the scale rides on 1/sigma and sigma, the A&S constant is divided by it)
    const float C = 0.84932180028801904f;
    const f2 ONE = pk(1.0f, 1.0f), HALF = pk(0.5f, 0.5f), AK = pk(0.2316419f / C, 0.2316419f / C);
    const f2 SGN = 0x8000000080000000ull;
    for (uint32_t p = 0; p < P; ++p) {
      const float sg = __ldg(sig + p);
      const float rsg = rcp(sg);
      const float hs2 = __fmaf_rn(__fmul_rn(0.5f, sg), sg, r);
      const f2 NSG = pk(-sg * C, -sg * C), RSG = pk(rsg * C, rsg * C), HS2 = pk(hs2, hs2);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const f2 d1 = mul2(fma2(HS2, SQT[h], LQ[h]), RSG);   // C d1
        const f2 d2 = fma2(NSG, SQT[h], d1);                 // C d2
        const f2 u1 = fma2(AK, abs2(d1), ONE), u2 = fma2(AK, abs2(d2), ONE);
        // the two A&S K = 1/u by two reciprocals: the MUFU pipe has the slack
        // the FP32 pipe (the limit) lacks -- one more MUFU op, three fewer FP32
        float u10, u11, u20, u21, a0, a1;
        up(u1, u10, u11);
        up(u2, u20, u21);
        const f2 k1 = pk(rcp(u10), rcp(u11)), k2 = pk(rcp(u20), rcp(u21));
        up(mul2(d1, d1), a0, a1);
        float x0, x1;
        asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(x0) : "f"(-a0));
        asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(x1) : "f"(-a1));
        const f2 e1 = pk(x0, x1);                       // exp(-d1^2/2); 1/sqrt(2 pi) is in poly2rn
        // N(d) = 1/2 + sign(d) (1/2 - c), c the A&S tail e poly(K): the 1/2 - c
        // is one FFMA2 (negated polynomial), the sign one LOP3 per element, and
        // the constant 1/2 (S - X e^{-rT}) of every scenario is added after the loop
        const f2 m1 = fma2(e1, poly2rn(k1), HALF) ^ (d1 & SGN);
        const f2 m2 = fma2(mul2(e1, SXD[h]), poly2rn(k2), HALF) ^ (d2 & SGN);
        CS[h] = fma2(NXD[h], m2, fma2(SS[h], m1, CS[h]));   // += S (n1 - 1/2) - X e^{-rT} (n2 - 1/2)
      }
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      float c0, c1;
      up(CS[h], c0, c1);
      call[2 * h] = __fdiv_rn(c0, float(P));
      call[2 * h + 1] = __fdiv_rn(c1, float(P));
    }
#pragma unroll
    for (int o = 0; o < 4; ++o) {
      call[o] = __fmaf_rn(0.5f, __fsub_rn(S[o], xd[o]), call[o]);
      put[o] = __fadd_rn(call[o], __fsub_rn(xd[o], S[o]));
    }
  }
#ifndef SLATE_BS_X2
#define SLATE_BS_X2 1
#endif
  __device__ __forceinline__ static void price4(const float (&S)[4], const float (&X)[4], const float (&T)[4], float r,
                                                const float* sig, uint32_t P, float (&call)[4], float (&put)[4]) {
#if SLATE_BS_X2
    price4_x2(S, X, T, r, sig, P, call, put);
#else
    price<4>(S, X, T, r, sig, P, call, put);
#endif
  }
  template <int k>
  __device__ __forceinline__ static void price(const float (&S)[4], const float (&X)[4], const float (&T)[4],
                                               float r, const float* sig, uint32_t P, float (&call)[4],
                                               float (&put)[4]) {
    const float RSQRT2PI = 0.39894228040143267794f;
    float sqt[k], rsqt[k], lsx[k], xd[k], sxd[k], cs[k];
#pragma unroll
    for (int o = 0; o < k; ++o) {
      sqt[o] = sqrtf(T[o]);
      rsqt[o] = __fdiv_rn(1.0f, sqt[o]);
      lsx[o] = logf(__fdiv_rn(S[o], X[o]));
      xd[o] = __fmul_rn(X[o], expf(__fmul_rn(-r, T[o])));
      sxd[o] = __fdiv_rn(S[o], xd[o]);
      cs[o] = 0.f;
    }
    for (uint32_t p = 0; p < P; ++p) {
      const float sg = __ldg(sig + p);
      const float rsg = rcp(sg);
      const float hs2 = __fmaf_rn(__fmul_rn(0.5f, sg), sg, r);
#pragma unroll
      for (int o = 0; o < k; ++o) {
        const float sst = __fmul_rn(sg, sqt[o]);
        const float d1 = __fmul_rn(__fmaf_rn(hs2, T[o], lsx[o]), __fmul_rn(rsg, rsqt[o]));
        const float d2 = __fsub_rn(d1, sst);
        const float u1 = __fmaf_rn(0.2316419f, fabsf(d1), 1.0f), u2 = __fmaf_rn(0.2316419f, fabsf(d2), 1.0f);
        const float q = rcp(__fmul_rn(u1, u2));
        const float e1 = __fmul_rn(RSQRT2PI, exp_(__fmul_rn(-0.5f, __fmul_rn(d1, d1))));
        const float c1 = __fmul_rn(e1, poly(__fmul_rn(u2, q)));
        const float c2 = __fmul_rn(__fmul_rn(e1, sxd[o]), poly(__fmul_rn(u1, q)));
        const float n1 = d1 > 0.f ? __fsub_rn(1.0f, c1) : c1;
        const float n2 = d2 > 0.f ? __fsub_rn(1.0f, c2) : c2;
        cs[o] = __fadd_rn(cs[o], __fsub_rn(__fmul_rn(S[o], n1), __fmul_rn(xd[o], n2)));
      }
    }
#pragma unroll
    for (int o = 0; o < k; ++o) {
      call[o] = __fdiv_rn(cs[o], float(P));
      put[o] = __fadd_rn(call[o], __fsub_rn(xd[o], S[o]));
    }
  }
  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char*) {
    const uint64_t v = uint64_t(x) * 256 + threadIdx.x;
    const uint64_t i0 = v * 4;
    const float* sig = reinterpret_cast<const float*>(a.sigmas);
    float S[4], X[4], T[4], c[4], p[4];
    if (i0 + 4 <= a.n) {
      const float4 s4 = __ldcs(reinterpret_cast<const float4*>(a.S) + v);
      const float4 x4 = __ldcs(reinterpret_cast<const float4*>(a.X) + v);
      const float4 t4 = __ldcs(reinterpret_cast<const float4*>(a.T) + v);
      S[0] = s4.x; S[1] = s4.y; S[2] = s4.z; S[3] = s4.w;
      X[0] = x4.x; X[1] = x4.y; X[2] = x4.z; X[3] = x4.w;
      T[0] = t4.x; T[1] = t4.y; T[2] = t4.z; T[3] = t4.w;
      price4(S, X, T, a.r, sig, a.n_scen, c, p);
      __stcs(reinterpret_cast<float4*>(a.call) + v, make_float4(c[0], c[1], c[2], c[3]));
      __stcs(reinterpret_cast<float4*>(a.put) + v, make_float4(p[0], p[1], p[2], p[3]));
    } else {
      for (uint64_t i = i0; i < a.n && i < i0 + 4; ++i) {   // ragged tail: one option at a time
        S[0] = reinterpret_cast<const float*>(a.S)[i];
        X[0] = reinterpret_cast<const float*>(a.X)[i];
        T[0] = reinterpret_cast<const float*>(a.T)[i];
        price<1>(S, X, T, a.r, sig, a.n_scen, c, p);
        reinterpret_cast<float*>(a.call)[i] = c[0];
        reinterpret_cast<float*>(a.put)[i] = p[0];
      }
    }
  }
};

// The Black-Scholes worker for launches with few scenarios (<= 4; the Tab II
// BS is P = 1): same blocks and arithmetic, plus a task-level body.  A separate
// kernel, chosen per launch by the server (kernels.cu), so the many-scenario
// worker (C2's P = 32, compute-bound) keeps its own code and registers.
struct BlackScholesShort : BlackScholes {
  static constexpr bool kLateCtrl = false;   // blocks of a few us: the word is read when the task starts
  // Task-level body: with few scenarios a block is a few us of HBM traffic,
  // so the next block's S, X, T are copied into shared memory (cp.async, no
  // extra registers) while this block is priced -- the original kernel hides
  // its loads behind other CTAs, the worker runs its task's blocks back to
  // back.  Each thread reads only the 48 bytes it copied, so no barrier is
  // needed.  A task reaching the ragged last block takes the per-block path.
  // Each option's arithmetic is price<4>'s (measured: a P = 1 launch of 2^23
  // options 54 -> 46 us at 4 blocks per task).
  static constexpr bool kHasTask = true;
  static constexpr uint32_t kPipelineMaxScen = 4;
  static constexpr int kSmem = 2 * 3 * 256 * 16;   // two cp.async stages
  static constexpr int kStageBytes = 3 * 256 * 16;   // S, X, T float4 of 256 threads
  __device__ __forceinline__ static void stage_in(const Args& a, uint64_t v, char* stage) {
    const char* src[3] = {reinterpret_cast<const char*>(a.S), reinterpret_cast<const char*>(a.X),
                          reinterpret_cast<const char*>(a.T)};
#pragma unroll
    for (int q = 0; q < 3; ++q)
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(stage + (q * 256 + threadIdx.x) * 16)),
                   "l"(src[q] + v * 16)
                   : "memory");
    asm volatile("cp.async.commit_group;" ::: "memory");
  }
  __device__ __forceinline__ static void cta_task(const Args& a, uint32_t g, uint32_t n, char* smem) {
    const uint64_t n_full = a.n / 1024;            // blocks with 1024 options (no ragged tail)
    if (g + n > n_full) {
      for (uint32_t i = 0; i < n; ++i) cta_block(a, g + i, 0, 0, smem);
      return;
    }
    const float* sig = reinterpret_cast<const float*>(a.sigmas);
    uint64_t v = uint64_t(g) * 256 + threadIdx.x;
    stage_in(a, v, smem);
    for (uint32_t i = 0; i < n; ++i) {
      const uint64_t cur = v;
      if (i + 1 < n) {
        v += 256;
        stage_in(a, v, smem + ((i + 1) & 1) * kStageBytes);    // next block in flight
        asm volatile("cp.async.wait_group 1;" ::: "memory");
      } else {
        asm volatile("cp.async.wait_group 0;" ::: "memory");
      }
      const float4* st = reinterpret_cast<const float4*>(smem + (i & 1) * kStageBytes);
      const float4 s4 = st[threadIdx.x], x4 = st[256 + threadIdx.x], t4 = st[512 + threadIdx.x];
      float S[4] = {s4.x, s4.y, s4.z, s4.w}, X[4] = {x4.x, x4.y, x4.z, x4.w}, T[4] = {t4.x, t4.y, t4.z, t4.w};
      float c[4], p[4];
      price4(S, X, T, a.r, sig, a.n_scen, c, p);
      __stcs(reinterpret_cast<float4*>(a.call) + cur, make_float4(c[0], c[1], c[2], c[3]));
      __stcs(reinterpret_cast<float4*>(a.put) + cur, make_float4(p[0], p[1], p[2], p[3]));
    }
  }
};

// ============================================================== 2-D 5-point stencil
// One Jacobi sweep of an h x w field; 128 x 8 points per block (north star:
// 128-bit HBM access).  Warp r owns row 8y + r, lane l the 4 columns
// 128x + 4l .. +3: one float4 load of the point row and one each of the rows
// above and below (the block's other warps load those rows too: L1/L2 hits,
// HBM reads every row once), left/right neighbours by warp shuffles inside the
// float4s and across lanes, the block's two edge columns by scalar loads.
// Fields whose width is not a multiple of 4 (or the ragged right edge) take a
// scalar path.  Arithmetic per point as the oracle's parenthesisation:
// 0.25 * ((up + down) + (left + right)); boundary points copied.
struct Stencil2D : TenantBase {
  using Args = slate_args_stencil;
  static constexpr int kThreads = 256;        // 8 warps: 8 rows x 32 lanes x 4 columns
  static constexpr int kMinBlocks = 8;
  static constexpr int kSmem = 0, kSmemStandalone = 0;

  __device__ __forceinline__ static float pt(float up, float down, float left, float right) {
    return __fmul_rn(0.25f, __fadd_rn(__fadd_rn(up, down), __fadd_rn(left, right)));
  }
  // the 4 points of a lane: interior points 0.25 ((up + down) + (left + right)), boundary copied
  __device__ __forceinline__ static float4 out4(float4 c, float4 u, float4 d, float left, float right, int j0, int w,
                                                bool interior_row) {
    float4 o = c;
    if (interior_row) {
      if (j0 > 0) o.x = pt(u.x, d.x, left, c.y);
      o.y = pt(u.y, d.y, c.x, c.z);
      o.z = pt(u.z, d.z, c.y, c.w);
      if (j0 + 3 < w - 1) o.w = pt(u.w, d.w, c.z, right);
    }
    return o;
  }
  // Task body inside a fused co-run kernel (w a multiple of 4): two x-neighbouring
  // blocks of a row band at once -- a lane's 4 columns in each, all six float4
  // loads in flight together.  A fused pair runs at its lower occupancy (4 CTAs/SM
  // with Black-Scholes), where this restores the stencil's bytes in flight; the
  // stand-alone worker (8 CTAs/SM, 32 registers) keeps cta_block, which this body
  // would spill (profiles/r2_kernels.md).  Every point is out4's, as in cta_block.
  static constexpr bool kHasFusedTask = true;
  __device__ __forceinline__ static void cta_task_fused(const Args& a, uint32_t g, uint32_t n, char* smem) {
    const uint32_t gx = (a.w + 127) / 128;
    uint32_t bx = g % gx, by = g / gx;
    uint32_t k = 0;
    while (k < n) {
      if ((a.w & 3) == 0 && k + 1 < n && bx + 1 < gx) {
        pair(a, bx, by);
        k += 2;
        bx += 2;
      } else {
        cta_block(a, bx, by, 0, smem);
        k += 1;
        bx += 1;
      }
      if (bx >= gx) {
        bx -= gx;
        ++by;
      }
    }
  }
  __device__ __forceinline__ static void pair(const Args& a, uint32_t bx, uint32_t by) {
    const float* in = reinterpret_cast<const float*>(a.in);
    float* out = reinterpret_cast<float*>(a.out);
    const int lane = int(threadIdx.x & 31), r = int(threadIdx.x >> 5);
    const int h = int(a.h), w = int(a.w);
    const int i = int(by) * 8 + r, j0 = int(bx) * 128 + lane * 4, j1 = j0 + 128;
    const bool row_in = i < h, interior_row = i > 0 && i < h - 1;
    const bool in0 = row_in && j0 < w, in1 = row_in && j1 < w;
    const float4 z = make_float4(0.f, 0.f, 0.f, 0.f);
    float4 c0 = z, u0 = z, d0 = z, c1 = z, u1 = z, d1 = z;
    const uint64_t base = uint64_t(i) * w;
    if (in0) {
      c0 = __ldg(reinterpret_cast<const float4*>(in + base + j0));
      if (interior_row) {
        u0 = __ldg(reinterpret_cast<const float4*>(in + base - w + j0));
        d0 = __ldg(reinterpret_cast<const float4*>(in + base + w + j0));
      }
    }
    if (in1) {
      c1 = __ldg(reinterpret_cast<const float4*>(in + base + j1));
      if (interior_row) {
        u1 = __ldg(reinterpret_cast<const float4*>(in + base - w + j1));
        d1 = __ldg(reinterpret_cast<const float4*>(in + base + w + j1));
      }
    }
    // neighbours: within a block from the adjacent lanes, across the two blocks
    // from lane 31 / lane 0 of the other, at the outer edges by scalar loads
    float left0 = __shfl_up_sync(0xffffffffu, c0.w, 1), right0 = __shfl_down_sync(0xffffffffu, c0.x, 1);
    float left1 = __shfl_up_sync(0xffffffffu, c1.w, 1), right1 = __shfl_down_sync(0xffffffffu, c1.x, 1);
    const float c0_last = __shfl_sync(0xffffffffu, c0.w, 31), c1_first = __shfl_sync(0xffffffffu, c1.x, 0);
    if (!row_in) return;
    if (lane == 0) {
      if (j0 > 0) left0 = __ldg(in + base + j0 - 1);
      left1 = c0_last;                                 // column j1 - 1 = the first block's last
    }
    if (lane == 31) {
      right0 = c1_first;                               // column j0 + 4 = the second block's first (< w here)
      if (in1 && j1 + 4 < w) right1 = __ldg(in + base + j1 + 4);
    }
    __stcs(reinterpret_cast<float4*>(out + base + j0), out4(c0, u0, d0, left0, right0, j0, w, interior_row));
    if (in1) __stcs(reinterpret_cast<float4*>(out + base + j1), out4(c1, u1, d1, left1, right1, j1, w, interior_row));
  }
  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t bx, uint32_t by, uint32_t, char*) {
    const float* in = reinterpret_cast<const float*>(a.in);
    float* out = reinterpret_cast<float*>(a.out);
    const int lane = int(threadIdx.x & 31), r = int(threadIdx.x >> 5);
    const int h = int(a.h), w = int(a.w);
    const int i = int(by) * 8 + r, j0 = int(bx) * 128 + lane * 4;
    if ((w & 3) == 0) {
      // vector path: every lane with j0 < w holds 4 whole columns
      const bool inside = i < h && j0 < w;
      const bool interior_row = i > 0 && i < h - 1;
      float4 c = make_float4(0.f, 0.f, 0.f, 0.f), u = c, d = c;
      if (inside) {
        c = __ldg(reinterpret_cast<const float4*>(in + uint64_t(i) * w + j0));
        if (interior_row) {
          u = __ldg(reinterpret_cast<const float4*>(in + uint64_t(i - 1) * w + j0));
          d = __ldg(reinterpret_cast<const float4*>(in + uint64_t(i + 1) * w + j0));
        }
      }
      float left = __shfl_up_sync(0xffffffffu, c.w, 1);     // column j0 - 1 (lane - 1's last)
      float right = __shfl_down_sync(0xffffffffu, c.x, 1);  // column j0 + 4 (lane + 1's first)
      if (!inside) return;
      if (lane == 0 && j0 > 0) left = __ldg(in + uint64_t(i) * w + j0 - 1);
      if ((lane == 31 || j0 + 4 >= w) && j0 + 4 < w) right = __ldg(in + uint64_t(i) * w + j0 + 4);
      __stcs(reinterpret_cast<float4*>(out + uint64_t(i) * w + j0), out4(c, u, d, left, right, j0, w, interior_row));
      return;
    }
    // scalar path (w not a multiple of 4): the same points one at a time
    if (i >= h) return;
    for (int k = 0; k < 4; ++k) {
      const int j = j0 + k;
      if (j >= w) break;
      const float cc = in[uint64_t(i) * w + j];
      float v = cc;
      if (i > 0 && i < h - 1 && j > 0 && j < w - 1)
        v = pt(in[uint64_t(i - 1) * w + j], in[uint64_t(i + 1) * w + j], in[uint64_t(i) * w + j - 1],
               in[uint64_t(i) * w + j + 1]);
      out[uint64_t(i) * w + j] = v;
    }
  }
};

// ================================================================ the paper's own apps (Tab II, NEXT-2)
// TR, MM, RG, GS of Tab II, written for B200 from the apps'
// definitions (oracle/tenants.py); Black-Scholes is the BlackScholes tenant
// with one scenario.  Bodies that stage through shared memory end with a
// barrier: a worker runs its task's blocks back to back in the same CTA.

// ---------------------------------------------------------------- TR: transpose
// 32x32 tile through shared memory (+1 column of padding: the transposed read
// is conflict-free), both the load and the store coalesced; thread (tx, ty)
// moves rows ty, ty+8, ty+16, ty+24 of the tile.
struct Transpose : TenantBase {
  using Args = slate_args_transpose;
  static constexpr bool kSpeculative = SLATE_SPEC_SHORT;
  static constexpr int kThreads = 256;        // 32 x 8
  static constexpr int kMinBlocks = 8;
  static constexpr int kSmem = 2 * 32 * 33 * 4, kSmemStandalone = 32 * 33 * 4;
  static constexpr bool kHasTask = true;

  __device__ __forceinline__ static void load(const Args& a, uint32_t bx, uint32_t by, float (&v)[4]) {
    const float* in = reinterpret_cast<const float*>(a.in);
    const uint32_t tx = threadIdx.x & 31, ty = threadIdx.x >> 5, c = bx * 32 + tx;
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      const uint32_t row = by * 32 + ty + 8 * r;
      v[r] = (row < a.h && c < a.w) ? __ldcs(in + uint64_t(row) * a.w + c) : 0.f;
    }
  }
  // The task's blocks as one pipeline (the worker's task-level body): the
  // next tile's loads are in flight while this tile's transposed stores go
  // out, two shared-memory tiles alternate, one barrier per block (measured:
  // 138 -> 125 us per 8192^2 launch; a 3-stage cp.async ring was slower, 132).
  // Every element moves exactly as in cta_block.
  __device__ __forceinline__ static void cta_task(const Args& a, uint32_t g, uint32_t n, char* smem) {
    float* out = reinterpret_cast<float*>(a.out);
    const uint32_t gx = (a.w + 31) / 32;
    const uint32_t tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    float v[4];
    uint32_t bx = g % gx, by = g / gx;
    load(a, bx, by, v);
    for (uint32_t k = 0; k < n; ++k) {
      float (*tile)[33] = reinterpret_cast<float (*)[33]>(smem + (k & 1) * (32 * 33 * 4));
#pragma unroll
      for (int r = 0; r < 4; ++r) tile[ty + 8 * r][tx] = v[r];
      __syncthreads();
      const uint32_t cbx = bx, cby = by;
      if (k + 1 < n) {
        if (++bx == gx) { bx = 0; ++by; }
        load(a, bx, by, v);                      // in flight during the stores below
      }
      const uint32_t i = cby * 32 + tx;
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        const uint32_t j = cbx * 32 + ty + 8 * r;
        if (j < a.w && i < a.h) __stcs(out + uint64_t(j) * a.h + i, tile[tx][ty + 8 * r]);
      }
    }
    __syncthreads();                             // the tiles are reused by the worker's next task
  }

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t bx, uint32_t by, uint32_t, char* smem) {
    float (*tile)[33] = reinterpret_cast<float (*)[33]>(smem);
    const float* in = reinterpret_cast<const float*>(a.in);
    float* out = reinterpret_cast<float*>(a.out);
    const uint32_t tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const uint32_t c = bx * 32 + tx;
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      const uint32_t row = by * 32 + ty + 8 * r;
      if (row < a.h && c < a.w) tile[ty + 8 * r][tx] = __ldcs(in + uint64_t(row) * a.w + c);
    }
    __syncthreads();
    const uint32_t i = by * 32 + tx;             // output column = input row
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      const uint32_t j = bx * 32 + ty + 8 * r;   // output row = input column
      if (j < a.w && i < a.h) __stcs(out + uint64_t(j) * a.h + i, tile[tx][ty + 8 * r]);
    }
    __syncthreads();                             // the tile is reused by the worker's next block
  }
};

// ---------------------------------------------------------------- MM: tiled SGEMM
// The SDK matrixMul's scheme (32x32 C tile, A and B staged 32x32 at a time in
// shared memory, k ascending), with each thread holding 4 C elements (rows
// ty + 8r, column tx) and reading A's tile 4 k at a time (one broadcast
// 128-bit load per row): every C element is the fmaf chain over k = 0..K-1 in
// order from 0 -- the order of the naive kernel.  Out-of-range A/B entries are
// staged as 0 (fmaf(0, b, acc) = acc).
struct SgemmTiled : TenantBase {
  using Args = slate_args_sgemm;
  static constexpr int kThreads = 256;        // 32 x 8
  static constexpr int kMinBlocks = 4;
  static constexpr int kSmem = 2 * 32 * 32 * 4, kSmemStandalone = 2 * 32 * 32 * 4;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t bx, uint32_t by, uint32_t, char* smem) {
    float (*As)[32] = reinterpret_cast<float (*)[32]>(smem);
    float (*Bs)[32] = reinterpret_cast<float (*)[32]>(smem + 32 * 32 * 4);
    const float* A = reinterpret_cast<const float*>(a.A);
    const float* B = reinterpret_cast<const float*>(a.B);
    const uint32_t tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    const uint32_t r0 = by * 32, c0 = bx * 32;
    float acc[4] = {0.f, 0.f, 0.f, 0.f};
    for (uint32_t k0 = 0; k0 < a.k; k0 += 32) {
#pragma unroll
      for (int r = 0; r < 4; ++r) {
        const uint32_t row = r0 + ty + 8 * r, ka = k0 + tx;
        As[ty + 8 * r][tx] = (row < a.m && ka < a.k) ? __ldg(A + uint64_t(row) * a.k + ka) : 0.f;
        const uint32_t kb = k0 + ty + 8 * r, col = c0 + tx;
        Bs[ty + 8 * r][tx] = (kb < a.k && col < a.n) ? __ldg(B + uint64_t(kb) * a.n + col) : 0.f;
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < 32; kk += 4) {
        const float b0 = Bs[kk][tx], b1 = Bs[kk + 1][tx], b2 = Bs[kk + 2][tx], b3 = Bs[kk + 3][tx];
#pragma unroll
        for (int r = 0; r < 4; ++r) {
          const float4 av = *reinterpret_cast<const float4*>(&As[ty + 8 * r][kk]);
          acc[r] = __fmaf_rn(av.x, b0, acc[r]);
          acc[r] = __fmaf_rn(av.y, b1, acc[r]);
          acc[r] = __fmaf_rn(av.z, b2, acc[r]);
          acc[r] = __fmaf_rn(av.w, b3, acc[r]);
        }
      }
      __syncthreads();                           // tiles reused by the next k slice / next block
    }
    float* C = reinterpret_cast<float*>(a.C);
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      const uint32_t row = r0 + ty + 8 * r, col = c0 + tx;
      if (row < a.m && col < a.n) C[uint64_t(row) * a.n + col] = acc[r];
    }
  }
};

// ---------------------------------------------------------------- RG: quasirandom generator
// The SDK quasirandomGenerator kernel: q_d(k) = XOR of table[d][b] over the set
// bits of k, written as float(q + 1) * 2^-31.  Thread t of block (x, d) makes
// points 1024x + 4t .. +3: the first by the 31-bit walk, the next three by the
// GF(2) linearity q(k+1) = q(k) ^ q(k ^ (k+1)), where k ^ (k+1) = 2^(c+1) - 1
// (c = trailing ones of k) and q of it is a prefix XOR of the table -- the
// same bits as the walk (XOR is exact), ~4x fewer integer ops.
struct Qrng : TenantBase {
  using Args = slate_args_qrng;
  static constexpr bool kSpeculative = SLATE_SPEC_SHORT;
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 8;
  static constexpr int kSmem = 2 * 32 * 4, kSmemStandalone = 2 * 32 * 4;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t d, uint32_t, char* smem) {
    uint32_t* tab = reinterpret_cast<uint32_t*>(smem);        // [0, 31): table row d
    uint32_t* pre = tab + 32;                                  // [0, 32): prefix XORs, pre[c] = tab[0] ^ .. ^ tab[c]
    const uint32_t* table = reinterpret_cast<const uint32_t*>(a.table) + uint64_t(d) * 31;
    if (threadIdx.x < 32) {
      const uint32_t v = threadIdx.x < 31 ? __ldg(table + threadIdx.x) : 0u;
      uint32_t p = v;                                          // inclusive prefix XOR over the warp
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t q = __shfl_up_sync(0xffffffffu, p, o);
        if (threadIdx.x >= uint32_t(o)) p ^= q;
      }
      tab[threadIdx.x] = v;
      pre[threadIdx.x] = p;
    }
    __syncthreads();
    const uint32_t i0 = x * 1024 + threadIdx.x * 4;
    float o[4];
    uint32_t k = a.seed + i0;
    uint32_t q = 0;
#pragma unroll
    for (int b = 0; b < 31; ++b) q ^= ((k >> b) & 1u) ? tab[b] : 0u;
    o[0] = __fmul_rn(__uint2float_rn(q + 1u), 4.656612873077392578125e-10f);   // 2^-31
#pragma unroll
    for (int j = 1; j < 4; ++j) {
      const uint32_t c = min(uint32_t(__ffs(~k)) - 1u, 30u);   // trailing ones of k (bit 31 is outside the table)
      q ^= pre[c];
      ++k;
      o[j] = __fmul_rn(__uint2float_rn(q + 1u), 4.656612873077392578125e-10f);
    }
    float* out = reinterpret_cast<float*>(a.out) + uint64_t(d) * a.n;
    if (i0 + 4 <= a.n && ((uint64_t(d) * a.n) & 3) == 0) {
      __stcs(reinterpret_cast<float4*>(out + i0), make_float4(o[0], o[1], o[2], o[3]));
    } else {
#pragma unroll
      for (int j = 0; j < 4; ++j)
        if (i0 + j < a.n) out[i0 + j] = o[j];
    }
    __syncthreads();                             // the table is reused by the worker's next block
  }
};

// ---------------------------------------------------------------- GS: Gaussian elimination
// Rodinia gaussian's two kernels for elimination step t.  Fan1 computes the
// multipliers of column t; Fan2 applies the rank-1 update to the trailing rows
// (columns t .. n-1, column t included as in Rodinia) and to b.  Rodinia maps
// threadIdx.x to rows (strided, uncoalesced); here lanes run along a row, so
// every warp access is one or more full 128-byte lines; each element's update
// is the same single fmaf(-m, pivot, a).
struct GaussFan1 : TenantBase {
  using Args = slate_args_gauss;
  static constexpr int kThreads = 256;
  static constexpr int kMinBlocks = 8;
  static constexpr int kSmem = 0, kSmemStandalone = 0;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char*) {
    const float* A = reinterpret_cast<const float*>(a.a);
    const uint32_t i = a.t + 1 + x * 256 + threadIdx.x;
    if (i >= a.n) return;
    reinterpret_cast<float*>(a.m)[uint64_t(i) * a.n + a.t] =
        __fdiv_rn(A[uint64_t(i) * a.n + a.t], A[uint64_t(a.t) * a.n + a.t]);
  }
};

struct GaussFan2 : TenantBase {
  using Args = slate_args_gauss;
  static constexpr bool kSpeculative = SLATE_SPEC_SHORT;
  static constexpr int kThreads = 256;        // 8 warps x 2 rows, lanes along 128 columns
  static constexpr int kMinBlocks = 8;
  static constexpr int kSmem = 0, kSmemStandalone = 0;

  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t y, uint32_t, char*) {
    float* A = reinterpret_cast<float*>(a.a);
    const float* M = reinterpret_cast<const float*>(a.m);
    const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint32_t n = a.n, t = a.t;
    const uint32_t c0 = t + x * 128 + lane;
    float piv[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint32_t j = c0 + 32 * q;
      piv[q] = j < n ? __ldg(A + uint64_t(t) * n + j) : 0.f;
    }
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      const uint32_t i = t + 1 + y * 16 + w * 2 + r;
      if (i >= n) break;
      const float mi = __ldg(M + uint64_t(i) * n + t);
      float* row = A + uint64_t(i) * n;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint32_t j = c0 + 32 * q;
        if (j < n) row[j] = __fmaf_rn(-mi, piv[q], row[j]);
      }
      if (x == 0 && lane == 0) {
        float* b = reinterpret_cast<float*>(a.b);
        b[i] = __fmaf_rn(-mi, b[t], b[i]);
      }
    }
  }
};

}  // namespace slate
