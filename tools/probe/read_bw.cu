// Development probe (not product code): READ-ONLY HBM bandwidth per SM, on the
// first k SMs (by %smid < k), as a function of CTAs per SM and bytes in flight,
// for (a) LDG.128 streaming loads and (b) cp.async.bulk HBM -> shared copies.
// Question it answers (round 2, SpMV worker): is ~43 GB/s of reads per SM the
// SM's ceiling, or the worker's (one CTA, two 64-KB slots)?  Work is handed out
// by an atomic counter over 64-KB pieces so the live CTAs share it.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }

constexpr uint32_t kPiece = 65536;

template <int UNR>
__global__ void ldg_read(const float4* __restrict__ src, uint32_t n_pieces, uint32_t* ctr, int k, float* sink) {
  __shared__ uint32_t s_p;
  if ((int)smid() >= k) return;
  float acc = 0.f;
  const uint32_t per = kPiece / 16;  // float4 per piece
  for (;;) {
    if (threadIdx.x == 0) s_p = atomicAdd(ctr, 1u);
    __syncthreads();
    const uint32_t p = s_p;
    __syncthreads();
    if (p >= n_pieces) break;
    const float4* b = src + size_t(p) * per;
    for (uint32_t i = threadIdx.x; i < per; i += blockDim.x * UNR) {
      float4 v[UNR];
#pragma unroll
      for (int u = 0; u < UNR; ++u) {
        const uint32_t j = i + u * blockDim.x;
        if (j < per) asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v[u].x), "=f"(v[u].y), "=f"(v[u].z), "=f"(v[u].w) : "l"(b + j));
        else v[u] = make_float4(0, 0, 0, 0);
      }
#pragma unroll
      for (int u = 0; u < UNR; ++u) acc += v[u].x + v[u].y + v[u].z + v[u].w;
    }
  }
  if (acc == 1234.5f) sink[0] = acc;
}

// one thread keeps `stages` bulk copies of `bytes` in flight (pieces are split
// into kPiece/bytes copies)
__global__ void bulk_read(const char* src, uint32_t n_pieces, uint32_t* ctr, int k, uint32_t bytes, int stages) {
  extern __shared__ __align__(128) char sm[];
  __shared__ uint64_t bar[16];
  if ((int)smid() >= k) return;
  if (threadIdx.x != 0) return;
  for (int i = 0; i < stages; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[i])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const uint32_t cpp = kPiece / bytes;
  uint32_t par = 0, pend = 0, sub = 0, p = atomicAdd(ctr, 1u);
  auto wait = [&](int s) {
    const uint32_t ph = (par >> s) & 1u;
    asm volatile("{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(su32(&bar[s])), "r"(ph) : "memory");
    par ^= 1u << s; pend &= ~(1u << s);
  };
  for (uint32_t i = 0; p < n_pieces; ++i) {
    const int s = int(i % stages);
    if (pend & (1u << s)) wait(s);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(sm + size_t(s) * bytes)),
                 "l"(src + size_t(p) * kPiece + size_t(sub) * bytes), "r"(bytes), "r"(su32(&bar[s])) : "memory");
    pend |= 1u << s;
    if (++sub == cpp) { sub = 0; p = atomicAdd(ctr, 1u); }
  }
  for (int s = 0; s < stages; ++s) if (pend & (1u << s)) wait(s);
}

// one CTA, `issuers` warps each keeping its own ring of `stages` copies
// (is the single-CTA ceiling per CTA or per issuing thread?)
__global__ void bulk_multi(const char* src, uint32_t n_pieces, uint32_t* ctr, int k, uint32_t bytes, int stages) {
  extern __shared__ __align__(128) char sm[];
  __shared__ uint64_t bar[4][16];
  if ((int)smid() >= k) return;
  const int w = threadIdx.x >> 5;
  if ((threadIdx.x & 31) != 0) return;
  uint64_t* b = bar[w];
  char* ring = sm + size_t(w) * stages * bytes;
  for (int i = 0; i < stages; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&b[i])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const uint32_t cpp = kPiece / bytes;
  uint32_t par = 0, pend = 0, sub = 0, p = atomicAdd(ctr, 1u);
  auto wait = [&](int s) {
    const uint32_t ph = (par >> s) & 1u;
    asm volatile("{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(su32(&b[s])), "r"(ph) : "memory");
    par ^= 1u << s; pend &= ~(1u << s);
  };
  for (uint32_t i = 0; p < n_pieces; ++i) {
    const int s = int(i % stages);
    if (pend & (1u << s)) wait(s);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&b[s])), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(ring + size_t(s) * bytes)),
                 "l"(src + size_t(p) * kPiece + size_t(sub) * bytes), "r"(bytes), "r"(su32(&b[s])) : "memory");
    pend |= 1u << s;
    if (++sub == cpp) { sub = 0; p = atomicAdd(ctr, 1u); }
  }
  for (int s = 0; s < stages; ++s) if (pend & (1u << s)) wait(s);
}

// cp.async 16 B per thread (LDGSTS), a ring of `stages` 16-KB slots filled by
// all threads of the CTA, committed per slot
template <int G>
__global__ void ldgsts_read(const char* src, uint32_t n_pieces, uint32_t* ctr, int k, int stages) {
  extern __shared__ __align__(128) char sm[];
  __shared__ uint32_t s_p;
  if ((int)smid() >= k) return;
  const uint32_t slot = 16384;
  for (;;) {
    if (threadIdx.x == 0) s_p = atomicAdd(ctr, 1u);
    __syncthreads();
    const uint32_t p = s_p;
    __syncthreads();
    if (p >= n_pieces) break;
    const char* b = src + size_t(p) * kPiece;
    for (uint32_t c = 0; c < kPiece / slot; ++c) {
      char* d = sm + size_t(c % stages) * slot;
      for (uint32_t o = threadIdx.x * 16; o < slot; o += blockDim.x * 16)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(d + o)), "l"(b + c * slot + o) : "memory");
      asm volatile("cp.async.commit_group;" ::: "memory");
      asm volatile("cp.async.wait_group %0;" ::"n"(G - 1) : "memory");
    }
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
}

int main() {
  const size_t total = size_t(2) << 30;  // 2 GiB > L2
  char* src; CK(cudaMalloc(&src, total)); CK(cudaMemset(src, 1, total));
  char* flush; CK(cudaMalloc(&flush, 256u << 20));
  uint32_t* ctr; CK(cudaMalloc(&ctr, 4));
  float* sink; CK(cudaMalloc(&sink, 4));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  const uint32_t n_pieces = uint32_t(total / kPiece);
  int nsm = 0; cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  CK(cudaFuncSetAttribute(bulk_read, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  auto timeit = [&](auto launch, int sms, const char* what) {
    float best = 1e9f;
    for (int r = 0; r < 3; ++r) {
      CK(cudaMemset(flush, r, 256u << 20));
      CK(cudaMemset(ctr, 0, 4));
      cudaEventRecord(e0); launch(); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
    }
    const double gbs = total / (best * 1e-3) / 1e9;
    printf("sms %3d  %-40s %8.1f GB/s  %6.1f GB/s per SM\n", sms, what, gbs, gbs / sms);
  };
  char name[128];
  CK(cudaFuncSetAttribute(bulk_multi, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  CK(cudaFuncSetAttribute(ldgsts_read<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  CK(cudaFuncSetAttribute(ldgsts_read<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  CK(cudaFuncSetAttribute(ldgsts_read<12>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  // (1) LDG.128 and one-issuer bulk copies vs CTAs per SM (profiles/r2_read_bw_probe.txt)
  for (int sms : {148, 74, 37, 18}) {
    for (int cps : {1, 2, 4, 8}) for (int thr : {256, 512}) {
      if (cps * thr > 2048) continue;
      snprintf(name, sizeof name, "ldg U4  %d CTA/SM x %d thr", cps, thr);
      timeit([&] { ldg_read<4><<<nsm * cps, thr>>>((const float4*)src, n_pieces, ctr, sms, sink); }, sms, name);
      snprintf(name, sizeof name, "ldg U8  %d CTA/SM x %d thr", cps, thr);
      timeit([&] { ldg_read<8><<<nsm * cps, thr>>>((const float4*)src, n_pieces, ctr, sms, sink); }, sms, name);
    }
    for (int cps : {1, 2, 3, 4}) for (uint32_t bytes : {16384u, 32768u}) for (int st : {2, 3, 4, 6}) {
      const size_t smem = size_t(bytes) * st;
      if (smem * cps > 220 * 1024) continue;
      snprintf(name, sizeof name, "bulk %d CTA/SM  %2u KB x %d", cps, bytes / 1024, st);
      timeit([&] { bulk_read<<<nsm * cps, 32, smem>>>(src, n_pieces, ctr, sms, bytes, st); }, sms, name);
    }
  }
  // (2) one CTA, several issuing warps; LDGSTS (profiles/r2_read_bw_probe_issuers.txt)
  for (int sms : {74, 37}) {
    for (int iss : {1, 2, 3, 4}) for (uint32_t bytes : {16384u, 32768u}) for (int st : {2, 3, 4}) {
      const size_t smem = size_t(bytes) * st * iss;
      if (smem > 200 * 1024) continue;
      snprintf(name, sizeof name, "bulk 1 CTA, %d issuer warps, %2u KB x %d", iss, bytes / 1024, st);
      timeit([&] { bulk_multi<<<nsm, 32 * iss, smem>>>(src, n_pieces, ctr, sms, bytes, st); }, sms, name);
    }
    for (int thr : {256, 512, 1024}) for (int st : {4, 8, 12}) {
      snprintf(name, sizeof name, "ldgsts 1 CTA x %d thr, 16 KB x %d", thr, st);
      auto l = [&] {
        if (st == 4) ldgsts_read<4><<<nsm, thr, size_t(16384) * st>>>(src, n_pieces, ctr, sms, st);
        else if (st == 8) ldgsts_read<8><<<nsm, thr, size_t(16384) * st>>>(src, n_pieces, ctr, sms, st);
        else ldgsts_read<12><<<nsm, thr, size_t(16384) * st>>>(src, n_pieces, ctr, sms, st);
      };
      timeit(l, sms, name);
    }
  }
  return 0;
}
