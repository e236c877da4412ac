// Micro-benchmark of the update kernel's critical-section skeleton on B200:
// per op a 16-lane team does [CAS lock] -> read the 128-B chunk -> write 12 entries ->
// [fence + release store], on a random chunk of M.  Variants switch parts off to see
// which one sets the throughput, at 1..6 blocks of 256 threads per SM.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubl tools/ubench_lock.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(uint64_t *p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_release(uint64_t *p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

// mode bits: 1 = CAS lock, 2 = fence on release (else relaxed store), 4 = data writes,
// 8 = read
template <int MODE>
__global__ void __launch_bounds__(256) kern(uint64_t *pool, uint32_t mask, int ops, unsigned long long *sink) {
  const int t = threadIdx.x & 15;  // 16-lane teams, one per warp (lanes 16..31 idle)
  if ((threadIdx.x & 31) >= 16) return;
  const unsigned m = 0xFFFFu;
  const uint64_t w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  uint64_t acc = 0;
  for (int i = 0; i < ops; ++i) {
    const uint32_t c = (uint32_t)mix(w * 1000003ull + i) & mask;
    uint64_t *ch = pool + (size_t)c * 16;
    if (MODE & 1) {
      bool ok = false;
      for (;;) {
        if (t == 15) ok = atomicCAS((unsigned *)(ch + 15), 0u, 1u) == 0u;
        ok = __shfl_sync(m, ok, 15);
        if (ok) break;
        __nanosleep(32);
      }
      __syncwarp(m);
    }
    uint64_t kv = 0;
    if (MODE & 8) kv = ld_relaxed(ch + t);
    acc += __shfl_sync(m, kv, 3);
    if ((MODE & 4) && t < 12) st_relaxed(ch + t, kv + 1);
    __syncwarp(m);
    if (t == 15) {
      const uint64_t lw = (MODE & 1) ? ((kv >> 32) + 1) << 32 : kv;
      if (MODE & 2) st_release(ch + 15, lw);
      else st_relaxed(ch + 15, lw);
    }
    __syncwarp(m);
  }
  if (acc == 0x12345) sink[0] = acc;
}

template <int MODE>
void run(const char *name, uint64_t *pool, uint32_t mask, unsigned long long *sink, int sms) {
  printf("%-28s", name);
  for (int bps = 1; bps <= 6; ++bps) {
    const int blocks = sms * bps, ops = 200;
    kern<MODE><<<blocks, 256>>>(pool, mask, ops, sink);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    cudaEventRecord(a);
    kern<MODE><<<blocks, 256>>>(pool, mask, ops, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double n = (double)blocks * 8 * ops;
    printf("  %d:%6.2f G/s %5.2fus", bps, n / ms / 1e6, ms * 1e3 / ops);
  }
  printf("\n");
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long *sink;
  cudaMalloc(&sink, 8);
  for (uint32_t chunks : {1u << 16, 1u << 20, 1u << 22}) {
    uint64_t *pool;
    cudaMalloc(&pool, (size_t)chunks * 128);
    cudaMemset(pool, 0, (size_t)chunks * 128);
    printf("M = %u chunks (%.0f MB); columns: blocks/SM: ops/s, us per op per team\n", chunks, chunks * 128.0 / 1e6);
    run<8>("read", pool, chunks - 1, sink, sms);
    run<8 | 4>("read+write", pool, chunks - 1, sink, sms);
    run<8 | 4 | 2>("read+write+fence", pool, chunks - 1, sink, sms);
    run<1 | 8 | 4>("cas+read+write", pool, chunks - 1, sink, sms);
    run<1 | 8 | 4 | 2>("cas+read+write+fence", pool, chunks - 1, sink, sms);
    run<1>("cas only (+relaxed unlock)", pool, chunks - 1, sink, sms);
    run<1 | 2>("cas + release", pool, chunks - 1, sink, sms);
    cudaFree(pool);
  }
  const cudaError_t e = cudaDeviceSynchronize();
  printf("%s\n", cudaGetErrorString(e));
  return 0;
}
