// Probe: relation between %globaltimer (GPU) and CLOCK_MONOTONIC (host).  A 1-thread kernel
// writes %globaltimer to mapped pinned memory; the host reads CLOCK_MONOTONIC before the launch
// (h0) and when it sees the value (h1).  Prints (h0 - g, h1 - g) statistics per 100 rounds, and
// the globaltimer resolution (distinct increments seen by one thread).
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/clock_probe scripts/clock_probe.cu
#include <cuda_runtime.h>
#include <time.h>
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <vector>
static uint64_t now() { timespec t; clock_gettime(CLOCK_MONOTONIC, &t); return t.tv_sec * 1000000000ull + t.tv_nsec; }
__global__ void stamp(unsigned long long* d) {
  unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  asm volatile("st.global.relaxed.sys.u64 [%0], %1;" :: "l"(d), "l"(t) : "memory");
}
__global__ void res(unsigned long long* out) {
  unsigned long long prev = 0, mind = ~0ull; int n = 0;
  for (int i = 0; i < 100000 && n < 50; ++i) {
    unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (prev && t != prev) { mind = min(mind, t - prev); ++n; }
    prev = t;
  }
  out[0] = mind;
}
int main() {
  unsigned long long *h, *d, *r;
  cudaHostAlloc(&h, 64, cudaHostAllocMapped); cudaHostGetDevicePointer((void**)&d, h, 0);
  cudaMalloc(&r, 8); res<<<1,1>>>(r); unsigned long long rr; cudaMemcpy(&rr, r, 8, cudaMemcpyDeviceToHost);
  printf("globaltimer min increment: %llu ns\n", rr);
  cudaStream_t s; cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
  for (int blk = 0; blk < 20; ++blk) {
    std::vector<long long> a, b;
    for (int i = 0; i < 100; ++i) {
      volatile unsigned long long* v = h; *v = 0;
      uint64_t h0 = now(); stamp<<<1,1,0,s>>>(d);
      unsigned long long g; while ((g = *v) == 0) {}
      uint64_t h1 = now();
      a.push_back((long long)h0 - (long long)g); b.push_back((long long)h1 - (long long)g);
    }
    std::sort(a.begin(), a.end()); std::sort(b.begin(), b.end());
    printf("block %2d: h0-g min %lld med %lld | h1-g min %lld med %lld max %lld\n", blk, a[0], a[50], b[0], b[50], b[99]);
    struct timespec ts{0, 100000000}; nanosleep(&ts, nullptr);
  }
  return 0;
}
