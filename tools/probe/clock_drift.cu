// clock_drift.cu -- how does %globaltimer drift against the host's steady clock?
// Repeats a mapped-memory ping-pong (min over 32 rounds of device stamp - host
// raise time) every 150 ms for ~3 s and prints the offset relative to the first.
#include <chrono>
#include <cstdio>
#include <thread>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__global__ void probe(volatile unsigned* flag, volatile unsigned long long* stamp, int rounds) {
  for (int i = 0; i < rounds; ++i) {
    flag[2 * i + 1] = 1;
    __threadfence_system();
    while (flag[2 * i] == 0) {
    }
    stamp[i] = gt();
    __threadfence_system();
  }
}
static double now_us() {
  return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
int main() {
  const int R = 32;
  volatile unsigned* flag;
  volatile unsigned long long* stamp;
  cudaHostAlloc((void**)&flag, 2 * R * 4, cudaHostAllocMapped);
  cudaHostAlloc((void**)&stamp, R * 8, cudaHostAllocMapped);
  double first = 0, tfirst = 0;
  for (int it = 0; it < 20; ++it) {
    for (int i = 0; i < 2 * R; ++i) flag[i] = 0;
    for (int i = 0; i < R; ++i) stamp[i] = 0;
    probe<<<1, 1>>>((unsigned*)flag, (unsigned long long*)stamp, R);
    double best = 1e300, worst = -1e300;
    double tt = 0;
    for (int i = 0; i < R; ++i) {
      while (flag[2 * i + 1] == 0) {
      }
      const double th = now_us();
      tt = th;
      flag[2 * i] = 1;
      while (stamp[i] == 0) {
      }
      const double d = double(stamp[i] % 1000000000000ull) * 1e-3 - th;
      best = d < best ? d : best;
      worst = d > worst ? d : worst;
    }
    cudaDeviceSynchronize();
    if (it == 0) { first = best; tfirst = tt; }
    printf("t=%8.1f ms  offset-first=%8.3f us  spread=%6.3f us\n", (tt - tfirst) * 1e-3, best - first, worst - best);
    std::this_thread::sleep_for(std::chrono::milliseconds(150));
  }
  return 0;
}
