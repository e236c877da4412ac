// gfsl_ubench.cuh -- B6: the roofline denominators of SURVEY 8(d), measured on the box.
//
// R_rand(C_b): random, aligned C_b-byte block gathers (C_b = chunk bytes, 256 or 128)
// over a buffer much larger than L2, issued exactly like the search kernel reads a chunk
// (a team of TEAM lanes, 32-B vector loads per lane, 32/TEAM teams per warp), with many
// independent gathers in flight per warp.  This is the "achievable random-access HBM
// throughput" the north star's >= 40% target refers to.
// t_chase: the latency of one dependent C_b-byte gather (pointer chase).
#pragma once
#include <cstdint>

namespace gfsl_dev {

__device__ __forceinline__ uint64_t ub_hash(uint64_t x) {
  x ^= x >> 33;
  x *= 0xff51afd7ed558ccdull;
  x ^= x >> 33;
  x *= 0xc4ceb9fe1a85ec53ull;
  x ^= x >> 33;
  return x;
}

// Each team gathers `iters` random blocks, UNROLL independent gathers in flight (the host
// sweeps UNROLL and keeps the best: the ceiling must not be limited by the benchmark's own
// memory-level parallelism).  nblocks is a power of two (the address is a masked hash).
template <int BLOCK_BYTES, int TEAM, int UNROLL>
__global__ void __launch_bounds__(256) ubench_gather(const uint4 *__restrict__ buf, uint64_t nblocks,
                                                      uint32_t iters, uint32_t seed, uint32_t *sink) {
  constexpr int LANE_BYTES = BLOCK_BYTES / TEAM;      // 64 (256/4) or 64 (128/2)
  constexpr int V = LANE_BYTES / 32;                   // 32-B loads per lane
  const int lane = threadIdx.x & 31;
  const int t = lane % TEAM;
  const uint64_t team = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) / TEAM;
  uint32_t acc = 0;
  for (uint32_t i = 0; i < iters; i += UNROLL) {
    uint32_t r[UNROLL][8 * V];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) {
      const uint64_t b = ub_hash((team << 24) ^ ((uint64_t)(i + u) << 1) ^ seed) & (nblocks - 1);
      const uint4 *p = buf + (b * BLOCK_BYTES + (uint64_t)t * LANE_BYTES) / 16;
#pragma unroll
      for (int v = 0; v < V; ++v)
        asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=r"(r[u][8 * v + 0]), "=r"(r[u][8 * v + 1]), "=r"(r[u][8 * v + 2]),
                       "=r"(r[u][8 * v + 3]), "=r"(r[u][8 * v + 4]), "=r"(r[u][8 * v + 5]),
                       "=r"(r[u][8 * v + 6]), "=r"(r[u][8 * v + 7])
                     : "l"(p + 2 * v));
    }
#pragma unroll
    for (int u = 0; u < UNROLL; ++u)
#pragma unroll
      for (int j = 0; j < 8 * V; ++j) acc ^= r[u][j];
  }
  if (acc == 0x9E3779B9u) sink[0] = acc;  // keeps the loads alive
}

// One warp per chase: block i holds the index of the next block in its first word.
template <int BLOCK_BYTES>
__global__ void ubench_chase(const uint32_t *__restrict__ buf, uint32_t start, uint32_t steps,
                             uint32_t *sink) {
  uint32_t c = start;
  for (uint32_t i = 0; i < steps; ++i) c = __ldcg(buf + (uint64_t)c * (BLOCK_BYTES / 4));
  if (threadIdx.x == 0) sink[blockIdx.x] = c;
}

__global__ void ubench_fill_chase(uint32_t *buf, uint64_t nblocks, uint32_t block_words, uint32_t seed) {
  // a random single cycle is not needed: a hash successor visits many distinct blocks
  for (uint64_t b = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; b < nblocks;
       b += (uint64_t)gridDim.x * blockDim.x)
    buf[b * block_words] = (uint32_t)(ub_hash(b ^ seed) & (nblocks - 1));
}

}  // namespace gfsl_dev
