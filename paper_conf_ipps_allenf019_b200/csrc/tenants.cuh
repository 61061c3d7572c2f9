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

// Optional per-tenant hooks default to off.
struct TenantBase {
  static constexpr bool kHasInit = false;   // cta_init(smem): once per CTA before the first block
  static constexpr bool kLookahead = false; // cta_task2(args, g, n, g2, n2, smem): run task [g, g+n) of a
                                            // 1-D grid knowing the CTA's next task [g2, g2+n2) (n2 = 0: none)
  static constexpr bool kHasFini = false;   // cta_fini(smem): once per CTA before it exits
};

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
__device__ __forceinline__ void bulk_g2s(void* dst_smem, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst_smem)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void bulk_s2g(void* dst, const void* src_smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src_smem)),
               "r"(bytes)
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
// worker pipelines the blocks of a task through kStages shared-memory buffers
// (loads of later blocks in flight while earlier ones are stored), which is
// what lets a few SMs saturate HBM (the E1 knee).
struct Copy : TenantBase {
  using Args = slate_args_copy;
  static constexpr int kThreads = 128;
  static constexpr int kStages = 4;
  static constexpr int kBlockBytes = 16384;
  static constexpr int kHdr = 128;                       // barriers + parity word
  static constexpr int kSmem = kHdr + kStages * kBlockBytes;
  static constexpr int kSmemStandalone = kHdr + kBlockBytes;
  static constexpr bool kHasInit = true, kLookahead = true, kHasFini = true;

  __device__ __forceinline__ static uint64_t* bars(char* smem) { return reinterpret_cast<uint64_t*>(smem); }
  __device__ __forceinline__ static uint32_t* parity(char* smem) { return reinterpret_cast<uint32_t*>(smem + 64); }
  __device__ __forceinline__ static uint32_t* state(char* smem);
  __device__ __forceinline__ static char* stage(char* smem, int s) { return smem + kHdr + s * kBlockBytes; }

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
  // bytes of block x moved by the bulk engine (multiple of 16); the rest by threads
  __device__ __forceinline__ static uint32_t bulk_bytes(const Args& a, uint32_t x) {
    const uint64_t e0 = uint64_t(x) * 4096;
    const uint64_t e1 = min(e0 + 4096, a.n);
    return uint32_t(((e1 - e0) * 4) & ~uint64_t(15));
  }
  __device__ __forceinline__ static void tail(const Args& a, uint32_t x) {
    const uint64_t e0 = uint64_t(x) * 4096 + bulk_bytes(a, x) / 4;
    const uint64_t e1 = min(uint64_t(x) * 4096 + 4096, a.n);
    for (uint64_t i = e0; i < e1; ++i) reinterpret_cast<float*>(a.a)[i] = reinterpret_cast<const float*>(a.b)[i];
  }
  __device__ __forceinline__ static void issue_load(const Args& a, char* smem, uint32_t x, int s) {
    const uint32_t nb = bulk_bytes(a, x);
    mbar_expect_tx(bars(smem) + s, nb);
    bulk_g2s(stage(smem, s), reinterpret_cast<const char*>(a.b) + uint64_t(x) * kBlockBytes, nb, bars(smem) + s);
  }
  __device__ __forceinline__ static void wait_load(char* smem, int s) {
    uint32_t& par = *parity(smem);
    mbar_wait(bars(smem) + s, (par >> s) & 1u);
    par ^= 1u << s;
  }
  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char* smem) {
    if (threadIdx.x != 0) return;
    bulk_wait_read0();                           // the buffer is free
    if (bulk_bytes(a, x)) {
      issue_load(a, smem, x, 0);
      wait_load(smem, 0);
      bulk_s2g(reinterpret_cast<char*>(a.a) + uint64_t(x) * kBlockBytes, stage(smem, 0), bulk_bytes(a, x));
      bulk_commit();
    }
    tail(a, x);
  }
  // The blocks of this task and of the next one form one stream through the
  // stage ring: while the last stores of this task drain, the first loads of
  // the next task are already in flight.  state: [0] blocks of this task
  // already loaded by the previous call, [1] stage of this task's first block.
  __device__ __forceinline__ static void cta_task2(const Args& a, uint32_t g, uint32_t n, uint32_t g2, uint32_t n2,
                                                   char* smem) {
    if (threadIdx.x != 0) return;
    uint32_t* st = state(smem);
    const uint32_t pre = st[0], seq = st[1];
    const uint32_t total = n + n2;
    auto blk = [&](uint32_t k) { return k < n ? g + k : g2 + (k - n); };
    auto stg = [&](uint32_t k) { return int((seq + k) % kStages); };
    uint32_t issued = pre;
    if (issued < kStages) bulk_wait_read0();   // stages about to be refilled have been read out
    for (; issued < min(total, uint32_t(kStages)); ++issued)
      if (bulk_bytes(a, blk(issued))) issue_load(a, smem, blk(issued), stg(issued));
    for (uint32_t i = 0; i < n; ++i) {
      const uint32_t x = g + i;
      const uint32_t nb = bulk_bytes(a, x);
      if (nb) {
        wait_load(smem, stg(i));
        bulk_s2g(reinterpret_cast<char*>(a.a) + uint64_t(x) * kBlockBytes, stage(smem, stg(i)), nb);
        bulk_commit();
      }
      tail(a, x);
      if (issued < total && issued == i + kStages) {
        bulk_wait_read0();                       // stage of block i has been read by its store
        if (bulk_bytes(a, blk(issued))) issue_load(a, smem, blk(issued), stg(issued));
        ++issued;
      }
    }
    st[0] = issued > n ? issued - n : 0;
    st[1] = (seq + n) % kStages;
  }
};

__device__ __forceinline__ uint32_t* Copy::state(char* smem) { return reinterpret_cast<uint32_t*>(smem + 72); }

// ============================================================== naive SGEMM  C = A B
// The CUDA-sample-style naive kernel: one thread per C element, no tiling.
struct SgemmNaive : TenantBase {
  using Args = slate_args_sgemm;
  static constexpr int kThreads = 256;        // 16 x 16
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
// 32 rows per block; in the original kernel warp w handles rows 4w..4w+3 with
// 8 lanes per row: lane l sums j = rp[row]+l, +8, +16, ... in ascending order
// (an fmaf chain from 0), then a butterfly (xor 4, 2, 1) inside the 8-lane group.
//
// The worker's task body streams instead: the rows of consecutive blocks are
// consecutive, so a block's col/val entries are one contiguous range that the
// bulk-copy engine moves into shared memory.  Each warp owns whole blocks
// (w, w+8, ... of the task) with two stages: it issues the next block's copy
// before consuming the current one, and the copy of its first block of the NEXT
// task is issued during this one (lookahead), so HBM latency leaves the
// critical path.  Per row, lanes, order and reduction are exactly cta_block's.
struct SpmvCsr : TenantBase {
  using Args = slate_args_spmv;
  static constexpr int kThreads = 256;
  static constexpr int kWarps = 8;
  static constexpr int kMaxTask = 16;                    // blocks per task on the streamed path
  static constexpr int kRp = 32 * kMaxTask + 4;          // row pointers per task buffer (16-B multiple)
  static constexpr int kCap = 32 * 16 + 8;               // entries per stage (16 nnz/row + alignment slack)
  static constexpr int kStageBytes = 2 * kCap * 4;       // col then val
  static constexpr int kHdr = 256;
  static constexpr int kSmem = kHdr + 2 * kRp * 4 + 2 * kWarps * kStageBytes;
  static constexpr int kSmemStandalone = kHdr;   // cta_init runs in both kernels (harmless here)
  static constexpr bool kHasInit = true, kLookahead = true;
  static_assert((kHdr + 2 * kRp * 4) % 16 == 0 && kStageBytes % 16 == 0 && (kCap * 4) % 16 == 0,
                "bulk-copy destinations must be 16-byte aligned");

  // ---- shared-memory layout
  __device__ __forceinline__ static uint64_t* bar(char* sm, int w, int st) {
    return reinterpret_cast<uint64_t*>(sm) + 2 * w + st;
  }
  __device__ __forceinline__ static uint32_t* wstate(char* sm, int w) {   // bit0,1 parity; bit2 prefetched; bit3 stage
    return reinterpret_cast<uint32_t*>(sm + 128) + w;
  }
  __device__ __forceinline__ static uint32_t* cstate(char* sm) {          // [0] rp slot, [1] rp of current valid
    return reinterpret_cast<uint32_t*>(sm + 192);
  }
  __device__ __forceinline__ static int* rpbuf(char* sm, int slot) { return reinterpret_cast<int*>(sm + kHdr) + slot * kRp; }
  __device__ __forceinline__ static int* scol(char* sm, int w, int st) {
    return reinterpret_cast<int*>(sm + kHdr + 2 * kRp * 4 + (2 * w + st) * kStageBytes);
  }
  __device__ __forceinline__ static float* sval(char* sm, int w, int st) {
    return reinterpret_cast<float*>(scol(sm, w, st) + kCap);
  }

  __device__ __forceinline__ static void cta_init(char* sm) {
    if (threadIdx.x == 0) {
      for (int i = 0; i < 2 * kWarps; ++i) mbar_init(reinterpret_cast<uint64_t*>(sm) + i, 1);
      for (int w = 0; w < kWarps; ++w) *wstate(sm, w) = 0;
      cstate(sm)[0] = 0;
      cstate(sm)[1] = 0;
      fence_mbar_init();
    }
  }

  // the bulk-copied range of a block: entries [a0, a1) land at smem index j - base
  struct Range {
    int base, a0, a1;
    bool bulk;
  };
  __device__ __forceinline__ static Range range(int n0, int n1) {
    Range r;
    r.base = n0 & ~3;
    r.a0 = (n0 + 3) & ~3;
    r.a1 = n1 & ~3;
    r.bulk = r.a1 > r.a0 && (n1 - r.base) <= kCap;
    return r;
  }
  __device__ __forceinline__ static void issue(const Args& a, char* sm, int w, int st, const Range& r) {
    if (!r.bulk) return;
    const uint32_t bytes = uint32_t(r.a1 - r.a0) * 4;
    mbar_expect_tx(bar(sm, w, st), 2 * bytes);
    bulk_g2s(scol(sm, w, st) + (r.a0 - r.base), reinterpret_cast<const int*>(a.col) + r.a0, bytes, bar(sm, w, st));
    bulk_g2s(sval(sm, w, st) + (r.a0 - r.base), reinterpret_cast<const float*>(a.val) + r.a0, bytes, bar(sm, w, st));
  }

  // whole block x by one warp; rp = row pointers of the block's task, block at index bi
  __device__ __forceinline__ static void consume(const Args& a, const int* rp, uint32_t x, uint32_t bi, const int* sc,
                                                 const float* sv, const Range& r, uint32_t lane) {
    const int* __restrict__ col = reinterpret_cast<const int*>(a.col);
    const float* __restrict__ val = reinterpret_cast<const float*>(a.val);
    const float* __restrict__ xv = reinterpret_cast<const float*>(a.x);
    const int l = int(lane & 7), q = int(lane >> 3);
    int lo[8], hi[8], c0[8], c1[8];
    float v0[8], v1[8], acc[8];
    auto get = [&](int j, int& c, float& v) {
      if (r.bulk && j >= r.a0 && j < r.a1) {
        c = sc[j - r.base];
        v = sv[j - r.base];
      } else {
        c = __ldcs(col + j);
        v = __ldcs(val + j);
      }
    };
#pragma unroll
    for (int t = 0; t < 8; ++t) {
      const uint32_t row = x * 32 + 4 * t + q;
      const int k = int(bi) * 32 + 4 * t + q;
      lo[t] = 0; hi[t] = 0; acc[t] = 0.f; c0[t] = 0; c1[t] = 0; v0[t] = 0.f; v1[t] = 0.f;
      if (row < a.n_rows) { lo[t] = rp[k] + l; hi[t] = rp[k + 1]; }
      if (lo[t] < hi[t]) get(lo[t], c0[t], v0[t]);
      if (lo[t] + 8 < hi[t]) get(lo[t] + 8, c1[t], v1[t]);
    }
#pragma unroll
    for (int t = 0; t < 8; ++t) {
      if (lo[t] < hi[t]) acc[t] = __fmaf_rn(v0[t], __ldg(xv + c0[t]), acc[t]);
      if (lo[t] + 8 < hi[t]) acc[t] = __fmaf_rn(v1[t], __ldg(xv + c1[t]), acc[t]);
    }
#pragma unroll
    for (int t = 0; t < 8; ++t) {
      for (int j = lo[t] + 16; j < hi[t]; j += 8) {
        int c;
        float v;
        get(j, c, v);
        acc[t] = __fmaf_rn(v, __ldg(xv + c), acc[t]);
      }
      float v = acc[t];
      v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, 4));
      v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, 2));
      v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, 1));
      const uint32_t row = x * 32 + 4 * t + q;
      if (l == 0 && row < a.n_rows) __stcs(reinterpret_cast<float*>(a.y) + row, v);
    }
  }

  // the original kernel: block x, warp w rows 4w..4w+3, operands straight from global
  __device__ __forceinline__ static void cta_block(const Args& a, uint32_t x, uint32_t, uint32_t, char*) {
    const int* rp = reinterpret_cast<const int*>(a.rowptr);
    const int* __restrict__ col = reinterpret_cast<const int*>(a.col);
    const float* __restrict__ val = reinterpret_cast<const float*>(a.val);
    const float* __restrict__ xv = reinterpret_cast<const float*>(a.x);
    const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const int l = int(lane & 7);
    const uint32_t row = x * 32 + w * 4 + (lane >> 3);
    int lo = 0, hi = 0;
    if (row < a.n_rows) { lo = __ldg(rp + row) + l; hi = __ldg(rp + row + 1); }
    float acc = 0.f;
    if (lo < hi) acc = __fmaf_rn(__ldcs(val + lo), __ldg(xv + __ldcs(col + lo)), acc);
    if (lo + 8 < hi) acc = __fmaf_rn(__ldcs(val + lo + 8), __ldg(xv + __ldcs(col + lo + 8)), acc);
    for (int j = lo + 16; j < hi; j += 8) acc = __fmaf_rn(__ldcs(val + j), __ldg(xv + __ldcs(col + j)), acc);
    acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, 4));
    acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, 2));
    acc = __fadd_rn(acc, __shfl_xor_sync(0xffffffffu, acc, 1));
    if (l == 0 && row < a.n_rows) __stcs(reinterpret_cast<float*>(a.y) + row, acc);
  }

  __device__ __forceinline__ static void load_rp(const Args& a, int* dst, uint32_t g, uint32_t n) {
    const uint32_t r0 = g * 32;
    const uint32_t cnt = min(32u * n, a.n_rows - r0) + 1;
    for (uint32_t t = threadIdx.x; t < cnt; t += kThreads) dst[t] = __ldg(reinterpret_cast<const int*>(a.rowptr) + r0 + t);
  }

  __device__ __forceinline__ static void cta_task2(const Args& a, uint32_t g, uint32_t n, uint32_t g2, uint32_t n2,
                                                   char* sm) {
    if (n > uint32_t(kMaxTask)) {               // long tasks: the original per-block body
      for (uint32_t i = 0; i < n; ++i) cta_block(a, g + i, 0, 0, sm);
      __syncthreads();
      cstate(sm)[1] = 0;
      for (int w = 0; w < kWarps; ++w) *wstate(sm, w) &= ~4u;
      return;
    }
    const uint32_t slot = cstate(sm)[0];
    int* rp_cur = rpbuf(sm, int(slot));
    int* rp_nxt = rpbuf(sm, int(slot ^ 1));
    const bool have_cur = cstate(sm)[1] != 0;
    const bool stream_nxt = n2 > 0 && n2 <= uint32_t(kMaxTask);
    if (!have_cur) load_rp(a, rp_cur, g, n);
    if (stream_nxt) load_rp(a, rp_nxt, g2, n2);
    __syncthreads();
    const uint32_t lane = threadIdx.x & 31;
    const int w = int(threadIdx.x >> 5);
    uint32_t ws = *wstate(sm, w);               // same value in every lane
    int st = int((ws >> 3) & 1u);
    bool pref = (ws >> 2) & 1u;
    const uint32_t total_rows = a.n_rows;
    auto rng_of = [&](const int* rp, uint32_t gg, uint32_t bi) {
      const uint32_t k0 = bi * 32, k1 = min(bi * 32 + 32, total_rows - gg * 32);
      return range(rp[k0], rp[k1]);
    };
    // st: the stage holding (or about to hold) the warp's next block; pref: that
    // block -- index w of this task -- was issued during the previous task
    const bool w_next_task = stream_nxt && uint32_t(w) < n2;
    bool issued_cur = pref;
    for (uint32_t i = uint32_t(w); i < n; i += kWarps) {
      const Range cur = rng_of(rp_cur, g, i);
      if (!issued_cur && lane == 0) issue(a, sm, w, st, cur);
      const bool more = i + kWarps < n;
      if (lane == 0) {                           // the follower goes to the other stage now
        if (more) issue(a, sm, w, st ^ 1, rng_of(rp_cur, g, i + kWarps));
        else if (w_next_task) issue(a, sm, w, st ^ 1, rng_of(rp_nxt, g2, uint32_t(w)));
      }
      if (cur.bulk) {
        mbar_wait(bar(sm, w, st), (ws >> st) & 1u);
        ws ^= 1u << st;
      }
      consume(a, rp_cur, g + i, i, scol(sm, w, st), sval(sm, w, st), cur, lane);
      __syncwarp();
      st ^= 1;
      issued_cur = more;
    }
    if (uint32_t(w) >= n && w_next_task && lane == 0)   // no block here this time: prefetch anyway
      issue(a, sm, w, st, rng_of(rp_nxt, g2, uint32_t(w)));
    pref = w_next_task;
    if (lane == 0) *wstate(sm, w) = (ws & 3u) | (pref ? 4u : 0u) | (uint32_t(st) << 3);
    __syncthreads();                             // everyone is done with rp_cur
    if (threadIdx.x == 0) {
      cstate(sm)[0] = slot ^ 1;
      cstate(sm)[1] = stream_nxt ? 1u : 0u;
    }
  }
};

// ============================================================== Black-Scholes
// European call/put as in the CUDA SDK BlackScholes sample: the normal CDF by
// the Abramowitz-Stegun polynomial (|error| < 7.5e-8), put by 1 - CND; each
// option priced under n_scen volatilities (reading Q16) and the mean written.
// Thread t of block x prices options 4(x*256+t)..+3.
struct BlackScholes : TenantBase {
  using Args = slate_args_bs;
  static constexpr int kThreads = 256;
  static constexpr int kSmem = 0, kSmemStandalone = 0;

  __device__ __forceinline__ static float cnd(float d) {
    const float A1 = 0.31938153f, A2 = -0.356563782f, A3 = 1.781477937f, A4 = -1.821255978f, A5 = 1.330274429f;
    const float RSQRT2PI = 0.39894228040143267794f;
    const float K = __fdividef(1.0f, __fmaf_rn(0.2316419f, fabsf(d), 1.0f));
    const float poly = __fmul_rn(K, __fmaf_rn(K, __fmaf_rn(K, __fmaf_rn(K, __fmaf_rn(K, A5, A4), A3), A2), A1));
    const float c = __fmul_rn(__fmul_rn(RSQRT2PI, __expf(__fmul_rn(-0.5f, __fmul_rn(d, d)))), poly);
    return d > 0.f ? __fsub_rn(1.0f, c) : c;
  }
  __device__ __forceinline__ static void price(float S, float X, float T, float r, const float* sig, uint32_t P,
                                               float& call, float& put) {
    const float sqt = sqrtf(T);
    const float lsx = logf(__fdiv_rn(S, X));
    const float xd = __fmul_rn(X, expf(__fmul_rn(-r, T)));
    float cs = 0.f, ps = 0.f;
    for (uint32_t p = 0; p < P; ++p) {
      const float sg = __ldg(sig + p);
      const float sst = __fmul_rn(sg, sqt);
      const float d1 = __fdividef(__fmaf_rn(__fmaf_rn(__fmul_rn(0.5f, sg), sg, r), T, lsx), sst);
      const float d2 = __fsub_rn(d1, sst);
      const float n1 = cnd(d1), n2 = cnd(d2);
      cs = __fadd_rn(cs, __fsub_rn(__fmul_rn(S, n1), __fmul_rn(xd, n2)));
      ps = __fadd_rn(ps, __fsub_rn(__fmul_rn(xd, __fsub_rn(1.0f, n2)), __fmul_rn(S, __fsub_rn(1.0f, n1))));
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
struct Stencil2D : TenantBase {
  using Args = slate_args_stencil;
  static constexpr int kThreads = 256;        // 32 x 8
  static constexpr int kSmem = 0, kSmemStandalone = 0;

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
