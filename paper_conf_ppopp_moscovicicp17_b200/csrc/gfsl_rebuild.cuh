// gfsl_rebuild.cuh -- upkeep: rebuild of the upper levels between batches (R24).
//
// "A possible reclamation scheme would be to compact the structure between
// kernel launches"; "a between-batch rebuild of levels >= 1 from level 0".
// Keys rise only through splits while deletes strip every level, so under
// churn the upper levels thin out and traversals take ever more lateral steps.  Between
// batches the structure is quiescent, so the upper levels are re-derived from level 0:
//   level 1 = [-inf -> head[0]] ++ [(min key of C) -> C for every live non-first level-0
//             chunk C holding a key, in key order], packed F entries per chunk;
//   level l+1 = [-inf -> first chunk of level l] ++ [(first key of chunk j) -> chunk j
//             of level l, j >= 1], packed F per chunk, until a level fits one chunk.
// So entry i of level l (i >= 1) carries the key of entry i*F^(l-1) of level 1, and every
// level-0 chunk is the direct target of a level-1 entry.  Level 0 is not touched.
// The chunks of levels >= 1 are rewritten in place in the upper pool: level l's first
// chunk is the head chunk l-1 of P:235, the others are allocated in level order after
// the heads; upper chunks no longer used are returned to the allocated state.
//
// Ordering level-0 chunks by key without a host round trip: every chunk marks its min key
// in a key_range-bit bitmap; a two-level popcount scan ranks the marks; each chunk writes
// itself at its rank.
#pragma once
#include "gfsl_device.cuh"

namespace gfsl_dev {

#ifndef GFSL_DIR_PER_KEY
#define GFSL_DIR_PER_KEY 4u  // directory buckets per level-1 key (R27b)
#endif

struct RebuildBufs {
  uint32_t *bitmap;       // [words]      key marks (all zero between rebuilds)
  uint32_t *word_prefix;  // [words]      exclusive popcount prefix within a 1024-word block
  uint32_t *block_sum;    // [blocks]     popcount of each block, then its exclusive prefix
  uint32_t *order_key;    // [cap_bottom] min keys in key order
  uint32_t *order_chunk;  // [cap_bottom] their chunks
  uint32_t *n1;           // [8]          marked chunks; old upper bump; dirty; active;
                          //              relocated (R38)
  void *levels;           // RbLevels computed once per rebuild (scan_top kernel)
  uint32_t words, blocks;
  uint32_t fill;          // F: entries per rebuilt upper chunk
};

constexpr int RB_BLOCK_WORDS = 1024;

// level geometry from n1 (identical in every thread)
struct RbLevels {
  uint32_t m[MAX_N];     // chunks of level l (l >= 1)
  uint32_t base[MAX_N];  // index of chunk 1 of level l (chunk 0 is the head chunk l-1)
  uint64_t pw[MAX_N];    // F^(l-1)
  int top;               // highest rebuilt level (its m == 1)
};

template <int N>
__device__ __forceinline__ void rb_levels(uint32_t n1, uint32_t F, RbLevels &L) {
  uint32_t len = n1 + 1;  // |A_1| including -inf
  uint32_t base = N - 1;
  uint64_t pw = 1;
  L.top = N - 1;
  for (int l = 1; l < N; ++l) {
    L.m[l] = (len + F - 1) / F;
    L.base[l] = base;
    L.pw[l] = pw;
    base += L.m[l] - 1;
    if (L.m[l] == 1) {
      L.top = l;
      for (int q = l + 1; q < N; ++q) {
        L.m[q] = 1;
        L.base[q] = base;
        L.pw[q] = pw * F;
      }
      break;
    }
    len = L.m[l];
    pw *= F;
  }
}

template <int N>
__device__ __forceinline__ uint32_t rb_chunk(const RbLevels &L, int l, uint32_t j) {
  return j == 0 ? (uint32_t)(l - 1) : L.base[l] + j - 1;
}


__device__ __forceinline__ bool rb_candidate(const DevState &d, uint32_t c, int N, uint32_t &minkey) {
  const uint64_t *ch = d.pool + (size_t)c * N;
  if (lo32(ch[N - 1]) == LOCK_ZOMBIE) return false;
  const uint32_t k0 = lo32(ch[0]);
  if (k0 == KEY_NEG_INF || k0 == KEY_EMPTY) return false;  // first chunk / empty last chunk
  minkey = k0;
  return true;
}

// A rebuild is skipped when no batch mutated the structure since the last one: n1[2] is
// the dirty flag (set by the update kernel), n1[3] says whether this rebuild runs.
__device__ __forceinline__ bool rb_active(const RebuildBufs &b) { return *(volatile uint32_t *)(b.n1 + 3) != 0; }

// (0) decide (one thread)
__global__ void rebuild_begin_kernel(RebuildBufs b) {
  pdl_wait();
  b.n1[3] = b.n1[2];
  b.n1[2] = 0;
  b.n1[4] = 0;  // R38: set by reloc_out_kernel when level 0 is relocated
}

// (1) mark min keys of the live non-first level-0 chunks
template <int N>
__global__ void __launch_bounds__(256) rebuild_mark_kernel(const __grid_constant__ DevState d, RebuildBufs b) {
  pdl_wait();
  if (!rb_active(b)) return;
  const uint32_t used = min(d.bump[0], d.cap_bottom);
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < used; i += gridDim.x * blockDim.x) {
    uint32_t k;
    if (rb_candidate(d, d.cap_upper + i, N, k)) atomicOr(b.bitmap + (k >> 5), 1u << (k & 31));
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) b.n1[1] = d.bump[1];
}

// (2) per-block popcount scan of the bitmap: one block of 1024 threads per 1024 words
__global__ void __launch_bounds__(1024) rebuild_scan_kernel(RebuildBufs b) {
  pdl_wait();
  if (!rb_active(b)) return;
  __shared__ uint32_t warp_tot[32];
  const uint32_t w = blockIdx.x * RB_BLOCK_WORDS + threadIdx.x;
  const uint32_t v = w < b.words ? __popc(b.bitmap[w]) : 0u;
  uint32_t incl = v;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) warp_tot[warp] = incl;
  __syncthreads();
  if (warp == 0) {
    uint32_t t = warp_tot[lane], ti = t;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, ti, o);
      if (lane >= o) ti += y;
    }
    warp_tot[lane] = ti - t;  // exclusive
    if (lane == 31) b.block_sum[blockIdx.x] = ti;
  }
  __syncthreads();
  if (w < b.words) b.word_prefix[w] = warp_tot[warp] + incl - v;
}

// (3) exclusive scan of the block sums (one block); n1 = the total; the level geometry
template <int N>
__global__ void __launch_bounds__(1024) rebuild_scan_top_kernel(RebuildBufs b) {
  pdl_wait();
  if (!rb_active(b)) return;
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  __shared__ uint32_t warp_tot[32];
  for (uint32_t base = 0; base < b.blocks; base += 1024) {
    const uint32_t i = base + threadIdx.x;
    const uint32_t v = i < b.blocks ? b.block_sum[i] : 0u;
    uint32_t incl = v;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
      if (lane >= o) incl += y;
    }
    if (lane == 31) warp_tot[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      uint32_t t = warp_tot[lane], ti = t;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, ti, o);
        if (lane >= o) ti += y;
      }
      warp_tot[lane] = ti - t;
    }
    __syncthreads();
    if (i < b.blocks) b.block_sum[i] = carry + warp_tot[warp] + incl - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry += warp_tot[warp] + incl;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    b.n1[0] = carry;  // marked chunks = total popcount
    rb_levels<N>(carry, b.fill, *(RbLevels *)b.levels);
  }
}

// rank of key k among the marked min keys: how many are <= k
__device__ __forceinline__ uint32_t rb_rank_le(const RebuildBufs &b, uint32_t k) {
  const uint32_t w = k >> 5, bit = k & 31;
  const uint32_t mask = bit == 31 ? 0xFFFFFFFFu : ((2u << bit) - 1u);
  return b.block_sum[w / RB_BLOCK_WORDS] + b.word_prefix[w] + __popc(b.bitmap[w] & mask);
}

// (4) each marked chunk writes itself at its rank
template <int N>
__global__ void __launch_bounds__(256) rebuild_rank_kernel(const __grid_constant__ DevState d, RebuildBufs b) {
  pdl_wait();
  if (!rb_active(b)) return;
  const uint32_t used = min(d.bump[0], d.cap_bottom);
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < used; i += gridDim.x * blockDim.x) {
    const uint32_t c = d.cap_upper + i;
    uint32_t k;
    if (!rb_candidate(d, c, N, k)) continue;
    const uint32_t w = k >> 5;
    const uint32_t r = b.block_sum[w / RB_BLOCK_WORDS] + b.word_prefix[w] +
                       __popc(b.bitmap[w] & ((1u << (k & 31)) - 1u));
    b.order_key[r] = k;
    b.order_chunk[r] = c;
  }
}

// ---- R38: level 0 relocated into rank order (concurrent-mode rebuilds) -------------------
// After the rank kernel, level 0 is copied chunk by chunk in key order into the bottom
// pool's unused tail (the scratch: chunks [used, used + m), m = n1 + 1 live chunks), then
// back to [0, m): chunk j holds the j-th chunk in key order (j = 0: the first chunk, -inf),
// NEXT = j + 1, the last (+inf, NULL).  Zombies, the free list and the unused chunks are
// gone (reset to the allocated state of P:237).  The rank of a key among the level-1 keys
// then IS its level-0 chunk, so a traversal can enter level 0 from the directory's rank
// refined by one 32-B read of the sorted min keys (R38 in the search kernel).
template <int N>
__global__ void __launch_bounds__(256) reloc_out_kernel(const __grid_constant__ DevState d, RebuildBufs b) {
  pdl_wait();
  if (!rb_active(b)) return;
  const uint32_t n1 = b.n1[0];
  const uint32_t used = min(d.bump[0], d.cap_bottom);
  const uint32_t m = n1 + 1;
  if ((uint64_t)used + m > d.cap_bottom) return;  // no room for the scratch: no relocation
  const uint32_t S = d.cap_upper + used;
  const int lane = threadIdx.x & 31;
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  const uint32_t head0 = d.head[0];
  for (uint32_t j = warp; j < m; j += nwarps) {
    const uint32_t src = j ? b.order_chunk[j - 1] : head0;
    if (lane < N) {
      uint64_t e = d.pool[(size_t)src * N + lane];
      if (lane == N - 2) e = (j + 1 < m) ? mk64(lo32(e), d.cap_upper + j + 1) : mk64(KEY_POS_INF, NULL_CHUNK);
      if (lane == N - 1) e = mk64(LOCK_FREE, 0u);
      d.pool[(size_t)(S + j) * N + lane] = e;
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) b.n1[4] = 1u;
}

template <int N>
__global__ void __launch_bounds__(256) reloc_in_kernel(const __grid_constant__ DevState d, RebuildBufs b) {
  pdl_wait();
  if (!rb_active(b) || !b.n1[4]) return;
  const uint32_t n1 = b.n1[0], m = n1 + 1;
  const uint32_t used = min(d.bump[0], d.cap_bottom);
  const uint32_t S = d.cap_upper + used;
  const uint64_t total = (uint64_t)m * N;
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < total; e += (uint64_t)gridDim.x * blockDim.x)
    d.pool[(size_t)d.cap_upper * N + e] = d.pool[(size_t)S * N + e];
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n1; j += gridDim.x * blockDim.x)
    b.order_chunk[j] = d.cap_upper + j + 1;  // the pack kernel's level-1 down pointers
}

template <int N>
__global__ void __launch_bounds__(256) reloc_reset_kernel(const __grid_constant__ DevState d, RebuildBufs b) {
  pdl_wait();
  if (!rb_active(b) || !b.n1[4]) return;
  const uint32_t n1 = b.n1[0], m = n1 + 1;
  const uint32_t used = min(d.bump[0], d.cap_bottom);
  const uint64_t first = (uint64_t)(d.cap_upper + m) * N, last = (uint64_t)(d.cap_upper + used + m) * N;
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = first + tid; e < last; e += stride)
    d.pool[e] = ((e % N) == (uint64_t)(N - 1)) ? (uint64_t)LOCK_HELD : EMPTY_ENTRY;
  for (uint64_t w = tid; w < 2ull * d.zwords; w += stride) d.zbits[w] = 0u;  // no zombie left
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    const bool any = n1 > 0 || lo32(d.pool[(size_t)d.cap_upper * N + 1]) != KEY_EMPTY;
    d.head[0] = d.cap_upper;
    d.counter[0] = any ? (int32_t)m : 0;
    d.bump[0] = m;
    d.fl[0] = d.fl[1] = 0;  // the free list (R25) is empty: nothing left to reclaim
  }
}

// (5) write every chunk of levels >= 1; one warp per chunk, lane e writes entry e.  And
// the level-1 directory (R27).
template <int N>
__global__ void __launch_bounds__(256) rebuild_pack_kernel(const __grid_constant__ DevState d, RebuildBufs b) {
  pdl_wait();
  if (!rb_active(b)) return;
  const uint32_t n1 = b.n1[0];
  const uint32_t F = b.fill;
  __shared__ RbLevels L;
  if (threadIdx.x == 0) L = *(const RbLevels *)b.levels;
  __syncthreads();
  {
    // R27: bucket q = keys [q << shift, (q+1) << shift); r(q) = rank(q << shift), the
    // number of marked min keys (= level-1 entries >= 1) <= q << shift, so level-1 entry
    // r(q) is the largest level-1 key <= q << shift, in chunk r / F of the packed level 1,
    // and level l's largest key <= q << shift is in its chunk r / F^l.  R27b: about four
    // buckets per level-1 key (at most dir_cap), one byte each: r(q) = base[q / 32] +
    // min(255, r(q) - base[q / 32]), base[g] = r(32 g).
    uint32_t target = 1024;
    while (target < GFSL_DIR_PER_KEY * n1 && target < d.dir_cap) target <<= 1;
    target = min(target, d.dir_cap);
    int shift = 0;
    while (((uint64_t)d.key_max >> shift) + 1 > target) ++shift;
    const uint32_t buckets = (uint32_t)((uint64_t)d.key_max >> shift) + 1;
    const bool sector = buckets <= GFSL_DIR_SECTOR_MAX;  // R27c
    for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < buckets; q += gridDim.x * blockDim.x) {
      const uint32_t r = rb_rank_le(b, q << shift);
#ifdef GFSL_DIR_U32
      ((uint32_t *)d.dir)[q] = r;
#else
      if (sector) {
        const uint32_t g = q / DIR_SEC_BUCKETS, j = q - g * DIR_SEC_BUCKETS;
        const uint32_t base = j ? rb_rank_le(b, (g * DIR_SEC_BUCKETS) << shift) : r;
        d.dir[(size_t)g * 32 + 4 + j] = (uint8_t)min(255u, r - base);
        if (j == 0) *(uint32_t *)(d.dir + (size_t)g * 32) = base;
      } else {
        const uint32_t base = (q & 31u) ? rb_rank_le(b, (q & ~31u) << shift) : r;
        d.dir[q] = (uint8_t)min(255u, r - base);
        if ((q & 31u) == 0) d.dir_base[q >> 5] = base;
      }
#endif
    }
    if (blockIdx.x == 0 && threadIdx.x < 32) {
      const int l = threadIdx.x;
      d.dir_hdr[32 + l] = (l >= 1 && l < N) ? L.base[l] : 0u;
      if (l == 0) {
        d.dir_hdr[0] = (uint32_t)shift;
        d.dir_hdr[1] = 1u;
        d.dir_hdr[2] = buckets;
        d.dir_hdr[3] = b.fill;
        // R37: entering level 0 from a bucket's rank costs ~(level-1 keys per bucket) / 2
        // lateral steps there; worth it only while the directory holds >= 1 bucket per key
        d.dir_hdr[4] = buckets >= n1 ? 1u : 0u;
        d.dir_hdr[5] = b.n1[4];  // R38: level 0 in rank order (chunk cap_upper + rank)
        d.dir_hdr[6] = n1;       // R38: min keys in order_key
        d.dir_hdr[7] = d.cap_upper;
        d.dir_hdr[8] = sector ? 1u : 0u;  // R27c: directory layout
      }
    }
  }
  uint32_t total = 0;
  for (int l = 1; l < N; ++l) total += L.m[l];
  const uint32_t head0 = d.head[0];
  const int lane = threadIdx.x & 31;
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t g = warp; g < total; g += nwarps) {
    int l = 1;
    uint32_t j = g;
    while (j >= L.m[l]) {
      j -= L.m[l];
      ++l;
    }
    // entries i in [j*F, (j+1)*F) of A_l, |A_l| = (l == 1 ? n1 + 1 : m[l-1]), or just the
    // -inf entry for levels above the top
    const uint32_t len = l > L.top ? 1u : (l == 1 ? n1 + 1 : L.m[l - 1]);
    uint64_t *ch = d.pool + (size_t)rb_chunk<N>(L, l, j) * N;
    const uint32_t i = j * F + lane;
    uint64_t ent = EMPTY_ENTRY;
    uint32_t key = 0;
    const bool has = lane < N - 2 && lane < (int)F && i < len;
    if (has) {
      uint32_t val;
      if (i == 0) {
        key = KEY_NEG_INF;
        val = (l == 1) ? head0 : (uint32_t)(l - 2);
      } else {
        key = b.order_key[(uint64_t)i * L.pw[l] - 1];
        val = (l == 1) ? b.order_chunk[i - 1] : rb_chunk<N>(L, l - 1, i);
      }
      ent = mk64(key, val);
    }
    const uint32_t hb = __ballot_sync(0xFFFFFFFFu, has);
    const int lastlane = 31 - __clz(hb);
    const uint32_t lastkey = __shfl_sync(0xFFFFFFFFu, key, lastlane);
    const bool last = (j + 1 == L.m[l]);
    if (lane < N - 2) ch[lane] = ent;
    else if (lane == N - 2) ch[N - 2] = last ? mk64(KEY_POS_INF, NULL_CHUNK) : mk64(lastkey, rb_chunk<N>(L, l, j + 1));
    else if (lane == N - 1) ch[N - 1] = mk64(LOCK_FREE, 0u);
  }
  if (blockIdx.x == 0 && threadIdx.x < N && threadIdx.x >= 1) {
    const int l = threadIdx.x;
    d.head[l] = l - 1;
    d.counter[l] = (l <= L.top && (l == 1 ? n1 > 0 : L.m[l - 1] > 1)) ? (int32_t)L.m[l] : 0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) d.bump[1] = L.base[N - 1] + (L.top == N - 1 ? L.m[N - 1] - 1 : 0);
}

// ---- R25: reclaim the zombie level-0 chunks into the free list -------------------------
// Right after a rebuild nothing points at a zombie any more: upkeep (R23) unlinked them
// from level 0 and the rebuilt upper levels only point at live chunks.  So every zombie is
// reset to the allocated state of P:237 and appended, in ascending chunk order, after the
// still-unused part of the previous free list (reclamation between launches).
constexpr int RC_TILE = 1024;  // chunks per tile: 256 threads x 4

// (6+7) clear the bitmap marks, return the upper chunks past the new bump to the
// allocated state, and count the zombies per tile
template <int N>
__global__ void __launch_bounds__(256) reclaim_count_kernel(const __grid_constant__ DevState d, RebuildBufs b,
                                                            uint32_t *tile_cnt) {
  pdl_wait();
  if (!rb_active(b)) return;
  {
    const uint32_t n1 = b.n1[0];
    const uint32_t old_used = b.n1[1];
    const uint32_t new_used = d.bump[1];
    const uint32_t stride = gridDim.x * blockDim.x;
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    for (uint32_t i = tid; i < n1; i += stride) b.bitmap[b.order_key[i] >> 5] = 0u;
    if (old_used > new_used) {
      const uint64_t first = (uint64_t)new_used * N, lastx = (uint64_t)old_used * N;
      for (uint64_t e = first + tid; e < lastx; e += stride)
        d.pool[e] = ((e % N) == (uint64_t)(N - 1)) ? (uint64_t)LOCK_HELD : EMPTY_ENTRY;
    }
  }
  const uint32_t used = min(d.bump[0], d.cap_bottom);
  const uint32_t tiles = (used + RC_TILE - 1) / RC_TILE;
  __shared__ uint32_t wsum[8];
  for (uint32_t tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    uint32_t cnt = 0;
    for (int q = 0; q < 4; ++q) {
      const uint32_t i = tile * RC_TILE + threadIdx.x * 4 + q;
      if (i < used && lo32(d.pool[(size_t)(d.cap_upper + i) * N + N - 1]) == LOCK_ZOMBIE) ++cnt;
    }
    for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(0xFFFFFFFFu, cnt, o);
    if ((threadIdx.x & 31) == 0) wsum[threadIdx.x >> 5] = cnt;
    __syncthreads();
    if (threadIdx.x == 0) {
      uint32_t t = 0;
      for (int w = 0; w < 8; ++w) t += wsum[w];
      tile_cnt[tile] = t;
    }
    __syncthreads();
  }
}

// (8) exclusive scan of the tile counts; the new list = old remainder + zombies
__global__ void __launch_bounds__(1024) reclaim_scan_kernel(const __grid_constant__ DevState d, RebuildBufs b,
                                                            uint32_t *tile_cnt) {
  pdl_wait();
  if (!rb_active(b)) return;
  const uint32_t used = min(d.bump[0], d.cap_bottom);
  const uint32_t tiles = (used + RC_TILE - 1) / RC_TILE;
  __shared__ uint32_t carry, warp_tot[32];
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (uint32_t base = 0; base < tiles; base += 1024) {
    const uint32_t i = base + threadIdx.x;
    const uint32_t v = i < tiles ? tile_cnt[i] : 0u;
    uint32_t incl = v;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
      if (lane >= o) incl += y;
    }
    if (lane == 31) warp_tot[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      uint32_t t = warp_tot[lane], ti = t;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, ti, o);
        if (lane >= o) ti += y;
      }
      warp_tot[lane] = ti - t;
    }
    __syncthreads();
    if (i < tiles) tile_cnt[i] = carry + warp_tot[warp] + incl - v;
    __syncthreads();
    if (threadIdx.x == 1023) carry += warp_tot[warp] + incl;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    const uint32_t count = d.fl[0], taken = d.fl[1], sel = d.fl[2];
    const uint32_t rem = taken < count ? count - taken : 0u;
    d.fl[3] = rem;
    d.fl[4] = sel;
    d.fl[5] = taken;
    d.fl[0] = rem + carry;
    d.fl[1] = 0;
    d.fl[2] = sel ^ 1u;
  }
}

// (9) write the new list (old remainder first, then the zombies in chunk order) and reset
// the zombies to the allocated state
template <int N>
__global__ void __launch_bounds__(256) reclaim_write_kernel(const __grid_constant__ DevState d, RebuildBufs b,
                                                            const uint32_t *tile_off) {
  pdl_wait();
  if (!rb_active(b)) return;
  const uint32_t rem = d.fl[3], oldsel = d.fl[4], taken = d.fl[5];
  const uint32_t *oldl = d.freelist + (size_t)oldsel * d.cap_bottom;
  uint32_t *newl = d.freelist + (size_t)(oldsel ^ 1u) * d.cap_bottom;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < rem; i += gridDim.x * blockDim.x)
    newl[i] = oldl[taken + i];
  const uint32_t used = min(d.bump[0], d.cap_bottom);
  const uint32_t tiles = (used + RC_TILE - 1) / RC_TILE;
  __shared__ uint32_t wsum[8];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (uint32_t tile = blockIdx.x; tile < tiles; tile += gridDim.x) {
    bool z[4];
    uint32_t cnt = 0;
    for (int q = 0; q < 4; ++q) {
      const uint32_t i = tile * RC_TILE + threadIdx.x * 4 + q;
      z[q] = i < used && lo32(d.pool[(size_t)(d.cap_upper + i) * N + N - 1]) == LOCK_ZOMBIE;
      cnt += z[q];
    }
    uint32_t incl = cnt;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
      if (lane >= o) incl += y;
    }
    if (lane == 31) wsum[warp] = incl;
    __syncthreads();
    uint32_t pos = rem + tile_off[tile] + incl - cnt;
    for (int w = 0; w < warp; ++w) pos += wsum[w];
    for (int q = 0; q < 4; ++q) {
      if (!z[q]) continue;
      const uint32_t c = d.cap_upper + tile * RC_TILE + threadIdx.x * 4 + q;
      newl[pos++] = c;
      for (uint32_t par = 0; par < 2; ++par)  // R30: the chunk is no zombie any more
        atomicAnd(d.zbits + (size_t)par * d.zwords + (c >> 5), ~(1u << (c & 31)));
      uint64_t *ch = d.pool + (size_t)c * N;
      for (int e = 0; e < N - 1; ++e) ch[e] = EMPTY_ENTRY;
      ch[N - 1] = (uint64_t)LOCK_HELD;
    }
    __syncthreads();
  }
}

}  // namespace gfsl_dev
