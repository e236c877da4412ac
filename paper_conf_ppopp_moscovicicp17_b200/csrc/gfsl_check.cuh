// gfsl_check.cuh -- B4: the structural check and the bottom-level export, on the device.
//
// gfsl_validate (gfsl.cu) copies the used part of the pool to the host and walks every
// level; at C5 (500M keys, ~50M chunks) that walk takes minutes.  Here every check is
// chunk-parallel, on the quiescent structure between batches (invariants of P:203 and
// §4.3, numbered as in DESIGN.md):
//   V1  a live chunk is strictly sorted, EMPTY entries grouped at the end
//   V2  a non-last live chunk holds keys and its max is its largest key; the last has
//       max = +inf
//   V3  max(c) < first key of the next live chunk (zombies skipped)
//   V4  a level-1 key is in the level-0 chunk its pointer reaches (stale separators of
//       lazy batches, R33, are counted instead when the upper levels are stale)
//   V5  every level-1 down pointer reaches laterally the level-0 chunk enclosing its key
//        within a bounded walk
//   V6  no max field grew since the last snapshot -- cross-batch, without a rebuild
//   V7  no live chunk is locked; no chunk in the allocated state is linked
//   V8  a zombie is never the last chunk of a level
//   V9  the first live chunk of each level holds -inf and is the one the head array
//       leads to (through zombies)
//   V11 a zombie's bytes never change -- cross-batch, without a rebuild
//   V12 every NEXT / down pointer names an allocated chunk
//   V14 counter[0] = the live level-0 chunks when level 0 holds a key (R9)
// plus the chain shape that the host walk gets for free: in each pool every live chunk
// has exactly one live predecessor (NEXT, zombies skipped) except one first chunk per
// level, and one last chunk per level.  With V3 (strictly increasing keys along NEXT) this
// makes every level one chain from its head.
// The export collects every live level-0 entry and sorts it by key (CUB radix sort); an
// adjacent duplicate is a violation (V3).
#pragma once
#include "gfsl_device.cuh"

namespace gfsl_dev {

constexpr uint32_t CHK_HOPS = 4096;  // bound on a lateral walk through zombies / chunks

struct CheckBufs {
  uint32_t *indeg;               // [used_u + used_b] live predecessors (NEXT, zombies skipped)
  unsigned long long *cnt;       // counters below
  uint32_t *viol;                // violation mask
  const uint32_t *snap_max;      // [snap_used] max field at the last snapshot (or NULL)
  const unsigned long long *snap_zh;  // [snap_used] zombie hash at the snapshot (0: not a zombie)
  uint32_t snap_used_u, snap_used_b;  // the bump counters at the snapshot
  uint32_t used_u, used_b;
  uint32_t stale_ok;             // R33: level-1 stale separators allowed
};
enum CheckCnt {
  CC_LIVE_B = 0, CC_LIVE_U, CC_ZOMBIE_B, CC_ZOMBIE_U, CC_KEYS_B, CC_LAST_B, CC_LAST_U,
  CC_FIRST_B, CC_FIRST_U, CC_UNDERFULL, CC_STALE, CC_SRC_B, CC_SRC_U, CC_MULTI, CC_NCNT
};

__device__ __forceinline__ uint32_t chk_slot(const CheckBufs &b, const DevState &d, uint32_t c) {
  return c < d.cap_upper ? c : b.used_u + (c - d.cap_upper);
}
__device__ __forceinline__ bool chk_allocated(const CheckBufs &b, const DevState &d, uint32_t c) {
  return c < d.cap_upper ? c < b.used_u : (c - d.cap_upper) < b.used_b && c < d.cap_upper + d.cap_bottom;
}
__device__ __forceinline__ void chk_fail(const CheckBufs &b, int v) { atomicOr(b.viol, 1u << (v - 1)); }

__device__ __forceinline__ unsigned long long chk_hash(const uint64_t *ch, int n) {
  unsigned long long h = 0x9E3779B97F4A7C15ull;
  for (int i = 0; i < n; ++i) {
    h ^= ch[i] + 0x9E3779B97F4A7C15ull + (h << 6) + (h >> 2);
    h *= 0xff51afd7ed558ccdull;
  }
  return h | 1ull;  // never 0 (0 = not a zombie)
}

// (1) one thread per used chunk
template <int N>
__global__ void __launch_bounds__(256) check_chunks_kernel(const __grid_constant__ DevState d, CheckBufs b) {
  constexpr int DS = N - 2, NX = N - 2, LK = N - 1;
  const uint32_t total = b.used_u + b.used_b;
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < total; s += gridDim.x * blockDim.x) {
    const bool upper = s < b.used_u;
    const uint32_t c = upper ? s : d.cap_upper + (s - b.used_u);
    const uint64_t *ch = d.pool + (size_t)c * N;
    const uint32_t state = lo32(ch[LK]);
    const uint32_t mx = lo32(ch[NX]);
    const uint32_t next = hi32(ch[NX]);
    // cross-batch snapshot (V6, V11): chunks that existed at the snapshot
    const bool in_snap = b.snap_max && (upper ? s < b.snap_used_u : (s - b.used_u) < b.snap_used_b);
    if (in_snap) {
      const uint32_t ss = upper ? s : b.snap_used_u + (s - b.used_u);
      if (state != LOCK_HELD && mx > b.snap_max[ss]) chk_fail(b, 6);
      if (b.snap_zh[ss] && (state != LOCK_ZOMBIE || chk_hash(ch, LK) != b.snap_zh[ss])) chk_fail(b, 11);
    }
    if (state == LOCK_HELD) continue;  // allocated state: not linked (checked via indeg)
    if (state == LOCK_ZOMBIE) {
      atomicAdd(b.cnt + (upper ? CC_ZOMBIE_U : CC_ZOMBIE_B), 1ull);
      if (next == NULL_CHUNK) chk_fail(b, 8);
      continue;
    }
    if (state != LOCK_FREE) {
      chk_fail(b, 7);
      continue;
    }
    atomicAdd(b.cnt + (upper ? CC_LIVE_U : CC_LIVE_B), 1ull);
    // V1: sorted, EMPTY grouped at the end
    uint32_t cnt = 0, last = 0;
    bool empty_seen = false;
    for (int i = 0; i < DS; ++i) {
      const uint64_t e = ch[i];
      const uint32_t k = lo32(e);
      if (k == KEY_EMPTY) {
        empty_seen = true;
        if (e != EMPTY_ENTRY) chk_fail(b, 1);
        continue;
      }
      if (empty_seen || (cnt > 0 && k <= last) || (k == KEY_NEG_INF && i != 0)) chk_fail(b, 1);
      if (!upper && k != KEY_NEG_INF && k > d.key_max) chk_fail(b, 1);
      last = k;
      ++cnt;
    }
    const uint32_t k0 = lo32(ch[0]);
    if (k0 == KEY_NEG_INF) atomicAdd(b.cnt + (upper ? CC_FIRST_U : CC_FIRST_B), 1ull);
    if (!upper) atomicAdd(b.cnt + CC_KEYS_B, (unsigned long long)(cnt - (k0 == KEY_NEG_INF ? 1u : 0u)));
    // V2
    if (next == NULL_CHUNK) {
      if (mx != KEY_POS_INF) chk_fail(b, 2);
      atomicAdd(b.cnt + (upper ? CC_LAST_U : CC_LAST_B), 1ull);
    } else {
      if (cnt == 0 || mx != last) chk_fail(b, 2);
      if (cnt < (uint32_t)max(1, DS / 3)) atomicAdd(b.cnt + CC_UNDERFULL, 1ull);
      // successor: the first live chunk along NEXT (V3, V8, V12, chain shape)
      uint32_t n = next, hops = 0;
      bool ok = true;
      while (true) {
        if (!chk_allocated(b, d, n) || (n < d.cap_upper) != upper || ++hops > CHK_HOPS) {
          chk_fail(b, 12);
          ok = false;
          break;
        }
        const uint64_t *nc = d.pool + (size_t)n * N;
        const uint32_t ns = lo32(nc[LK]);
        if (ns == LOCK_ZOMBIE) {
          n = hi32(nc[NX]);
          continue;
        }
        if (ns != LOCK_FREE) {
          chk_fail(b, 7);  // a live chunk links an allocated (unused) chunk
          ok = false;
        }
        const uint32_t nk0 = lo32(nc[0]);
        if (nk0 != KEY_EMPTY && !(mx < nk0)) chk_fail(b, 3);
        if (nk0 == KEY_NEG_INF) chk_fail(b, 9);
        break;
      }
      if (ok) atomicAdd(b.indeg + chk_slot(b, d, n), 1u);
    }
    // V12 / V4 / V5 for the down pointers of an upper chunk
    if (upper) {
      for (int i = 0; i < (int)cnt; ++i) {
        const uint32_t k = lo32(ch[i]);
        const uint32_t ptr = hi32(ch[i]);
        if (!chk_allocated(b, d, ptr)) {
          chk_fail(b, 12);
          continue;
        }
        if (ptr < d.cap_upper || k == KEY_NEG_INF) continue;  // levels >= 2: pointers checked by V12 only
        // level 1 -> level 0: walk laterally to the chunk enclosing k
        uint32_t e = ptr, hops = 0;
        bool found = false;
        while (true) {
          if (!chk_allocated(b, d, e) || ++hops > CHK_HOPS) break;
          const uint64_t *ec = d.pool + (size_t)e * N;
          if (lo32(ec[LK]) == LOCK_ZOMBIE || lo32(ec[NX]) < k) {
            e = hi32(ec[NX]);
            continue;
          }
          found = true;
          bool has = false;
          for (int j = 0; j < DS; ++j) has |= lo32(ec[j]) == k;
          if (!has) {
            if (b.stale_ok) atomicAdd(b.cnt + CC_STALE, 1ull);
            else chk_fail(b, 4);
          }
          break;
        }
        if (!found) chk_fail(b, 5);
      }
    }
  }
}

// (2) chain shape: sources (no live predecessor) and merges (two predecessors)
template <int N>
__global__ void __launch_bounds__(256) check_indeg_kernel(const __grid_constant__ DevState d, CheckBufs b) {
  constexpr int LK = N - 1;
  const uint32_t total = b.used_u + b.used_b;
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < total; s += gridDim.x * blockDim.x) {
    const bool upper = s < b.used_u;
    const uint32_t c = upper ? s : d.cap_upper + (s - b.used_u);
    const uint32_t state = lo32(d.pool[(size_t)c * N + LK]);
    const uint32_t in = b.indeg[s];
    if (state == LOCK_FREE) {
      if (in == 0) atomicAdd(b.cnt + (upper ? CC_SRC_U : CC_SRC_B), 1ull);
      if (in > 1) atomicAdd(b.cnt + CC_MULTI, 1ull);
    }
  }
}

// (3) snapshot for the next cross-batch check (V6, V11)
template <int N>
__global__ void __launch_bounds__(256) check_snapshot_kernel(const __grid_constant__ DevState d, uint32_t used_u,
                                                              uint32_t used_b, uint32_t *snap_max,
                                                              unsigned long long *snap_zh) {
  constexpr int NX = N - 2, LK = N - 1;
  const uint32_t total = used_u + used_b;
  for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < total; s += gridDim.x * blockDim.x) {
    const uint32_t c = s < used_u ? s : d.cap_upper + (s - used_u);
    const uint64_t *ch = d.pool + (size_t)c * N;
    snap_max[s] = lo32(ch[NX]);
    snap_zh[s] = lo32(ch[LK]) == LOCK_ZOMBIE ? chk_hash(ch, LK) : 0ull;
  }
}

// (4) export: every live level-0 entry (key, value) appended; sorted afterwards
template <int N>
__global__ void __launch_bounds__(256) export_collect_kernel(const __grid_constant__ DevState d, uint32_t used_b,
                                                              uint32_t *keys, uint32_t *vals,
                                                              unsigned long long *count) {
  constexpr int DS = N - 2, LK = N - 1;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < used_b; i += gridDim.x * blockDim.x) {
    const uint64_t *ch = d.pool + (size_t)(d.cap_upper + i) * N;
    if (lo32(ch[LK]) != LOCK_FREE) continue;
    uint32_t cnt = 0;
    for (int j = 0; j < DS; ++j) {
      const uint32_t k = lo32(ch[j]);
      cnt += (k != KEY_EMPTY && k != KEY_NEG_INF);
    }
    if (!cnt) continue;
    unsigned long long pos = atomicAdd(count, (unsigned long long)cnt);
    for (int j = 0; j < DS; ++j) {
      const uint64_t e = ch[j];
      const uint32_t k = lo32(e);
      if (k == KEY_EMPTY || k == KEY_NEG_INF) continue;
      keys[pos] = k;
      vals[pos] = hi32(e);
      ++pos;
    }
  }
}

template <int N>
__global__ void __launch_bounds__(256) export_count_kernel(const __grid_constant__ DevState d, uint32_t used_b,
                                                            unsigned long long *count) {
  constexpr int DS = N - 2, LK = N - 1;
  unsigned long long local = 0;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < used_b; i += gridDim.x * blockDim.x) {
    const uint64_t *ch = d.pool + (size_t)(d.cap_upper + i) * N;
    if (lo32(ch[LK]) != LOCK_FREE) continue;
    for (int j = 0; j < DS; ++j) {
      const uint32_t k = lo32(ch[j]);
      local += (k != KEY_EMPTY && k != KEY_NEG_INF);
    }
  }
  if (local) atomicAdd(count, local);
}

// (5) sorted export -> user keys; an adjacent duplicate is a violation (a key in two chunks)
__global__ void export_finish_kernel(const uint32_t *sk, const uint32_t *sv, uint64_t n, uint32_t *keys_out,
                                     uint32_t *vals_out, uint32_t *viol) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t k = sk[i];
    if (i > 0 && sk[i - 1] == k) atomicOr(viol, 1u << 2);  // V3
    if (keys_out) keys_out[i] = k - 1u;                      // user key (R3)
    if (vals_out) vals_out[i] = sv[i];
  }
}

}  // namespace gfsl_dev
