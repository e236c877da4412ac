// gfsl_bulk.cuh -- the bulk path: a batch far larger than the structure, by sort and merge.
//
// A batch of n ops on a map of at most U live keys with n >> U (a bulk load into an empty
// or small map; VERDICT r1 "cold-start contention cliff") would make
// the paper's protocol serialise: thousands of teams CAS the few lock words of a small
// structure and split one chunk at a time.  P:263 names the remedy -- "compact the
// structure between kernel launches" -- and a batch that dwarfs the structure is best
// applied as such a compaction: the live level-0 entries and the batch's ops are sorted
// together by key, every op's result is read off its key's group, and level 0 is written
// anew, chunk-parallel, in key order; then the upper levels are rebuilt (R24, R27).
//
// Semantics (S1, R1): per key group (the key's live entry, if any, and its ops
// in input order -- the radix sort is stable and ops precede existing entries):
//   Contains -> present before the batch;
//   Insert   -> true iff absent before the batch and it is the group's first Insert
//               (outside the contract the later ones are false: a linearization);
//   Delete   -> true iff present before the batch and it is the group's first Delete.
// The key survives iff (present and no Delete) or (absent and some Insert); its value is
// the old one or the winning Insert's.  Under the contract this is exactly S1.
//
// Layout written (R34): level 0 = chunks cap_upper + 0 .. m-1 in key order, chunk 0 starts
// with -inf, FILL entries per chunk (FILL = round(0.7 DSIZE): the fill the paper reports
// for random inserts, ~10 of 14 and ~20 of 30), NEXT = (largest key, j + 1),
// the last chunk (+inf, NULL); every other bottom chunk goes back to the allocated state of
// P:237, the free list and zombie marks are cleared.
#pragma once
#include "gfsl_device.cuh"

namespace gfsl_dev {

constexpr uint32_t BK_CONTAINS = 0u, BK_INSERT = 1u, BK_DELETE = 2u, BK_EXIST = 3u;
constexpr uint32_t BK_NONE = 0xFFFFFFFFu;

__device__ __forceinline__ uint64_t bk_payload(uint32_t value, uint32_t idx, uint32_t kind) {
  return (uint64_t)value | ((uint64_t)(idx & 0x1FFFFFFFu) << 32) | ((uint64_t)kind << 62);
}
__device__ __forceinline__ uint32_t bk_kind(uint64_t p) { return (uint32_t)(p >> 62); }
__device__ __forceinline__ uint32_t bk_idx(uint64_t p) { return (uint32_t)(p >> 32) & 0x1FFFFFFFu; }

#ifndef GFSL_BULK_FILL10
#define GFSL_BULK_FILL10 7  // tenths of DSIZE
#endif
template <int N>
constexpr uint32_t bk_fill() {
  return (uint32_t)(((N - 2) * GFSL_BULK_FILL10 + 5) / 10);  // round(0.7 DSIZE): 10 at N = 16, 21 at N = 32
}

// (1) ops at [0, n), the live level-0 entries at [n, n + used_b * DSIZE); invalid ops are
// answered now and sort last (all-ones key)
template <int N>
__global__ void __launch_bounds__(256) bulk_collect_kernel(const __grid_constant__ DevState d, const uint8_t *ops,
                                                            const uint32_t *keys, const uint32_t *vals,
                                                            uint8_t *res, uint32_t n, uint64_t key_range,
                                                            uint32_t used_b, uint32_t *sk, uint64_t *pl) {
  constexpr int DS = N - 2, LK = N - 1;
  const uint64_t total = (uint64_t)n + (uint64_t)used_b * DS;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
    if (i < n) {
      const uint32_t op = ops[i], key = keys[i];
      const bool valid = op <= 2 && (uint64_t)key < key_range;
      if (!valid) res[i] = 0xFF;
      sk[i] = valid ? key + 1u : 0xFFFFFFFFu;
      pl[i] = bk_payload((vals && op == 1) ? vals[i] : 0u, (uint32_t)i, valid ? op : 0u);
    } else {
      const uint64_t e = i - n;
      const uint32_t c = d.cap_upper + (uint32_t)(e / DS);
      const uint64_t *ch = d.pool + (size_t)c * N;
      const uint64_t kv = ch[e % DS];
      const uint32_t k = lo32(kv);
      const bool live = lo32(ch[LK]) == LOCK_FREE && k != KEY_EMPTY && k != KEY_NEG_INF;
      sk[i] = live ? k : 0xFFFFFFFFu;
      pl[i] = bk_payload(hi32(kv), 0u, BK_EXIST);
    }
  }
}

// (2) group starts: hd[i] = i at the first element of a key group, else 0 (max-scanned)
__global__ void bulk_head_kernel(const uint32_t *sk, uint64_t m, uint32_t *hd, uint32_t *fi, uint32_t *fd,
                                 uint8_t *has_e) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    hd[i] = (i == 0 || sk[i] != sk[i - 1]) ? (uint32_t)i : 0u;
    fi[i] = BK_NONE;
    fd[i] = BK_NONE;
    has_e[i] = 0;
  }
}

// (3) per group: is the key live, its first Insert, its first Delete
__global__ void bulk_group_kernel(const uint32_t *sk, const uint64_t *pl, const uint32_t *gs, uint64_t m,
                                  uint32_t *fi, uint32_t *fd, uint8_t *has_e) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    if (sk[i] == 0xFFFFFFFFu) continue;
    const uint32_t g = gs[i], kind = bk_kind(pl[i]);
    if (kind == BK_EXIST) has_e[g] = 1;
    else if (kind == BK_INSERT) atomicMin(fi + g, (uint32_t)i);
    else if (kind == BK_DELETE) atomicMin(fd + g, (uint32_t)i);
  }
}

// (4) results and survivors
__global__ void bulk_result_kernel(const uint32_t *sk, const uint64_t *pl, const uint32_t *gs, uint64_t m,
                                   const uint32_t *fi, const uint32_t *fd, const uint8_t *has_e, uint8_t *res,
                                   uint8_t *keep, unsigned long long *n_mut) {
  unsigned long long muts = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
    uint8_t kp = 0;
    if (sk[i] != 0xFFFFFFFFu) {
      const uint64_t p = pl[i];
      const uint32_t g = gs[i], kind = bk_kind(p);
      const bool e = has_e[g] != 0;
      if (kind == BK_EXIST) {
        kp = fd[g] == BK_NONE;
      } else if (kind == BK_CONTAINS) {
        res[bk_idx(p)] = e;
      } else if (kind == BK_INSERT) {
        const bool win = !e && fi[g] == (uint32_t)i;
        res[bk_idx(p)] = win;
        kp = win;
        muts += win;
      } else {
        const bool win = e && fd[g] == (uint32_t)i;
        res[bk_idx(p)] = win;
        muts += win;
      }
    }
    keep[i] = kp;
  }
  for (int o = 16; o; o >>= 1) muts += __shfl_xor_sync(0xFFFFFFFFu, muts, o);
  if ((threadIdx.x & 31) == 0 && muts) atomicAdd(n_mut, muts);
}

// (5) level 0 anew: chunk j of m holds global slots [j*FILL, (j+1)*FILL), slot 0 = -inf,
// slot g >= 1 = survivor g-1; one warp per chunk; then the old bottom chunks past m go back
// to the allocated state, and the level's metadata is set
template <int N>
__global__ void __launch_bounds__(256) bulk_write_kernel(const __grid_constant__ DevState d, const uint32_t *ck,
                                                          const uint64_t *cp, const unsigned long long *n_sel,
                                                          uint32_t old_used, unsigned long long *n_mut) {
  constexpr int DS = N - 2, NX = N - 2, LK = N - 1;
  constexpr uint32_t FILL = bk_fill<N>();
  const uint64_t S = *n_sel;
  const uint32_t m = (uint32_t)((S + 1 + FILL - 1) / FILL);
  const int lane = threadIdx.x & 31;
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  if (m > d.cap_bottom) {
    if (warp == 0 && lane == 0) set_error(d, ERR_POOL);
    return;
  }
  for (uint32_t j = warp; j < m; j += nwarps) {
    uint64_t *ch = d.pool + (size_t)(d.cap_upper + j) * N;
    const uint64_t g = (uint64_t)j * FILL + lane;
    uint64_t ent = EMPTY_ENTRY;
    uint32_t key = 0;
    const bool has = lane < (int)FILL && lane < DS && g <= S;
    if (has) {
      if (g == 0) {
        ent = mk64(KEY_NEG_INF, 0u);
        key = KEY_NEG_INF;
      } else {
        key = ck[g - 1];
        ent = mk64(key, (uint32_t)cp[g - 1]);
      }
    }
    const uint32_t hb = __ballot_sync(0xFFFFFFFFu, has);
    const uint32_t lastkey = __shfl_sync(0xFFFFFFFFu, key, 31 - __clz(hb));
    const bool last = j + 1 == m;
    if (lane < DS) ch[lane] = ent;
    else if (lane == NX) ch[NX] = last ? mk64(KEY_POS_INF, NULL_CHUNK) : mk64(lastkey, d.cap_upper + j + 1);
    else if (lane == LK) ch[LK] = mk64(LOCK_FREE, 0u);
  }
  // the rest of the used bottom pool: back to the allocated state
  const uint64_t first = (uint64_t)(d.cap_upper + m) * N, lastx = (uint64_t)(d.cap_upper + max(old_used, m)) * N;
  const uint64_t tid = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x, stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t e = first + tid; e < lastx; e += stride)
    d.pool[e] = ((e % N) == (uint64_t)(N - 1)) ? (uint64_t)LOCK_HELD : EMPTY_ENTRY;
  // zombie marks (R30) of every chunk: cleared
  for (uint64_t w = tid; w < 2ull * d.zwords; w += stride) d.zbits[w] = 0u;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    d.head[0] = d.cap_upper;
    d.counter[0] = S ? (int32_t)m : 0;
    d.bump[0] = m;
    d.fl[0] = d.fl[1] = 0;  // the free list (R25) is empty: nothing was reclaimed
    *d.dirty = 1u;          // the upper levels are rebuilt next (R24)
    stat_add(d, ST_MUTATIONS, *n_mut);
  }
}

}  // namespace gfsl_dev
