// gfsl_device.cuh -- chunk layout, sentinels and memory primitives of the GFSL device path.
//
// Chunk layout (Fig 3.1; §4.1): a chunk is N 8-byte entries.
//   entries 0..N-3  DATA  {lo32 key, hi32 value}      (value = down pointer above level 0)
//   entry   N-2     NEXT  {lo32 max field, hi32 next chunk index}
//   entry   N-1     LOCK  {lo32 lock state, hi32 version}
// Chunks live in one pre-allocated pool and are named by 32-bit indices.
// Sentinels (reading R3): internal key = user key + 1, so that
//   -inf = 0, +inf = EMPTY = 0xFFFFFFFF, null pointer = 0xFFFFFFFF.
// Lock states (reading R4): 0 unlocked, 1 locked, 2 zombie; the upper 32 bits are
// a version bumped by every unlock, which lets a reader prove that a lock-free read of a
// chunk was not torn by a writer (used where a NEGATIVE answer must be exact).
#pragma once
#include <cstdint>

namespace gfsl_dev {

constexpr uint32_t KEY_NEG_INF = 0u;
constexpr uint32_t KEY_POS_INF = 0xFFFFFFFFu;
constexpr uint32_t KEY_EMPTY = 0xFFFFFFFFu;
constexpr uint32_t NULL_CHUNK = 0xFFFFFFFFu;
constexpr uint64_t EMPTY_ENTRY = 0xFFFFFFFFFFFFFFFFull;

constexpr uint32_t LOCK_FREE = 0u;
constexpr uint32_t LOCK_HELD = 1u;
constexpr uint32_t LOCK_ZOMBIE = 2u;

constexpr int MAX_N = 32;

// error word bits (sticky)
constexpr uint32_t ERR_POOL = 1u;     // chunk pool exhausted
constexpr uint32_t ERR_HANG = 2u;     // a watchdog fired (corrupt structure / livelock)

// statistics slots
enum StatSlot {
  ST_RESTARTS = 0, ST_SPLITS, ST_MERGES, ST_ZOMBIE_UNLINKS, ST_LOCK_RETRIES,
  ST_CREADS,      // chunk reads of Contains traversals (counting build only)
  ST_CREADS_L0,   // ... of which on the bottom level
  ST_COPS,        // Contains ops counted
  ST_MUTATIONS,   // ops the update kernel applied (all batches)
  ST_GROUPED,     // R40: records applied through a chunk group of >= 2
  ST_NSTATS
};

struct BatchCtl;

// R27c: directory layout, chosen by each rebuild (dir_hdr[8]).  Sector layout: groups of
// DIR_SEC_BUCKETS = 28 buckets in one 32-B sector -- a 32-bit base (the group's first
// rank) then one byte per bucket -- so the two reads of a lookup hit one sector (one L2
// request); split layout (R27b): a byte array and a base array (32 buckets per base, two
// requests).  The sector layout is taken up to GFSL_DIR_SECTOR_MAX buckets (default: any
// size; measured C2 +1.5%, C3 +5%, C4-16 +14%, C5 -4% / +4% on two boxes);
// GFSL_DIR_SECTOR_MAX=0 restores R27b.
#ifndef GFSL_DIR_SECTOR_MAX
#define GFSL_DIR_SECTOR_MAX 0xFFFFFFFFu
#endif
constexpr uint32_t DIR_SEC_BUCKETS = 28;

// Device view of one handle.
struct DevState {
  uint64_t *pool;        // (cap_upper + cap_bottom) * N entries
  uint32_t *head;        // head[MAX_N]
  int32_t *counter;      // counter[MAX_N] "utilized chunks" per level
  uint32_t *bump;        // bump[0] bottom pool used, bump[1] upper pool used
  uint32_t *error;       // sticky error word (mapped host memory)
  unsigned long long *stats;
  uint32_t cap_bottom;   // bottom-pool chunks, indices [cap_upper, cap_upper + cap_bottom)
  uint32_t cap_upper;    // upper-pool chunks, indices [0, cap_upper)
  uint32_t key_max;      // largest valid internal key (= key_range)
  BatchCtl *ctl;         // the handle's per-batch control block
  uint32_t *dirty;       // set when a batch mutated the structure (-> upper-level rebuild)
  uint32_t *freelist;    // 2 x cap_bottom: reclaimed level-0 chunks (double-buffered)
  uint32_t *fl;          // [0] free chunks in the current list, [1] taken, [2] buffer,
                         // [3..5] reclaim scratch
  unsigned long long *debug_times;  // GFSL_DEBUG_TIMING builds: per-team (start, end, ops)
  // Directory (R27): the rank r(b) = how many level-1 keys of the last rebuild are
  // <= (b << shift), stored compactly so that it stays L2-resident under the random-gather
  // traffic of a 1B-key structure (R27b): r(b) = dir_base[b >> 5] + dir[b], one byte per
  // bucket (a delta saturated at 255: a smaller rank is still a valid start, one more
  // lateral step) and one 32-bit base per 32 buckets.  The rebuilt level l holds every
  // F^(l-1)-th level-1 key F per chunk, so the chunk of level l that holds the largest key
  // <= b << shift is chunk r / F^l of that level: chunk l-1 (the head) if 0, else
  // dir_hdr[32 + l] + r / F^l - 1.  dir_hdr = {shift, valid, buckets, F, l0_ok (R37),
  // korder (R38: level 0 in rank order), n1, cap_upper, ...,
  // [32 + l] = base of level l}; valid = 0 until the first rebuild (and after gfsl_load).
  uint8_t *dir;
  uint32_t *dir_base;
  uint32_t *dir_hdr;
  uint32_t dir_cap;      // buckets allocated (a power of two, multiple of 32)
  // Zombie marks (R30): the update kernel sets bit c of zbits[zparity] when it makes chunk c
  // a zombie; the upkeep sweep after the batch only has to follow NEXT pointers whose target
  // bit is set, instead of reading every successor's lock word.  Two bitmaps of zwords words
  // alternate by batch parity; a bit is cleared when upkeep passes the zombie two batches
  // later, or when reclamation (R25) resets the chunk.
  uint32_t *zbits;
  uint32_t zwords;
  uint32_t zparity;
  // R33: concurrent batches with the upper-level rebuild on leave the levels >= 1 to the
  // next rebuild: no raise after a split (isKeyRaised false), no updateDownPtrs, and a
  // Delete removes k from level 0 only (its upper copies stay as stale separators)
  uint32_t lazy_upper;
  uint32_t upkeep_force;  // R33: the deferred upkeep before a rebuild runs even if this
                          // batch merged nothing (earlier lazy batches did)
  uint32_t p_chunk_q32;  // isKeyRaised probability as a 32-bit fraction; 0 = 1 (R16)
  uint32_t l0_evict_first;  // R36: the search kernel loads level-0 chunks evict_first
  // R37: the rebuild's rank order of the level-0 chunks (RebuildBufs::order_chunk): entry
  // r-1 is the level-0 chunk whose min key is the r-th level-1 key, i.e. level-1 entry r's
  // down pointer, stored densely; with the directory's rank it lets a traversal enter
  // level 0 directly.  l0_entry = 1: the search kernel does so (concurrent modes).
  const uint32_t *dir_oc;
  const uint32_t *dir_ok;  // R38: the sorted min keys of the last rebuild (order_key)
  uint32_t l0_entry;
  uint32_t upd_prefetch;  // the update kernel prefetches each record's chunk into L2 (host:
                          // while level 0 fits the L2; beyond it the extra request costs
                          // more than it saves -- C5 update 2.21 vs 2.55 ms, round 2)
  unsigned long long *mut_host;  // mapped pinned host copy of the cumulative mutation count
                                 // (written by the update kernel; the rebuild policy, R29)
  uint32_t *bump_host;  // mapped pinned host copy of bump[0..1], written by the search kernel
                        // at its start (the counters after the previous batch; host heuristics)
};

// isKeyRaised's draw (R28): a counter-based hash of (raised key, level of the split), the
// murmur3 finalizer; the key is raised iff p_chunk = 1 or draw < p_chunk * 2^32.
__device__ __forceinline__ bool raise_key(const DevState &d, uint32_t rkey, int level) {
  if (d.p_chunk_q32 == 0) return true;
  uint32_t x = rkey ^ ((uint32_t)level * 0x9E3779B9u) ^ 0x2545F491u;
  x ^= x >> 16;
  x *= 0x85EBCA6Bu;
  x ^= x >> 13;
  x *= 0xC2B2AE35u;
  x ^= x >> 16;
  return x < d.p_chunk_q32;
}

// Per-batch control block (device memory, zeroed before every batch).
struct BatchCtl {
  uint32_t unused1;
  uint32_t n_vw;         // combining mode: value writes (combine kernel)
  uint32_t unused2;
  uint32_t unused0;
  uint32_t snap_height;  // height seen by the search kernel
  uint32_t n_merges;     // merges of this batch (update kernel) -> upkeep sweep
  uint32_t pad[2];
  // Mutation records are numbered per region: region r (= the writing block's index mod
  // MUT_REGIONS) owns record slots [r * region_cap, (r+1) * region_cap) and counts them
  // in mcnt[r] (records the update kernel applies) or ccnt[r] (combining mode: the search
  // kernel's candidates).  32 counters instead of one keep the appends of all blocks from
  // serialising on one L2 atomic, and each sits in its own 128-B line (CNT_STRIDE words):
  // in one line all 32 shared one L2 slice -- C5's 12.5M appends per batch on one slice,
  // whose position alternated with the control block (search 9.8 vs 14 ms, round 2).
  static constexpr int MUT_REGIONS = 32;
  static constexpr int CNT_STRIDE = 32;
  uint32_t mcnt[MUT_REGIONS * CNT_STRIDE];
  uint32_t ccnt[MUT_REGIONS * CNT_STRIDE];
  // dynamic work queues of the update kernel (one per update block, at most UQ_MAX):
  // queue j of Q hands out the mutation slots j, j + Q, j + 2Q, ... in order; one counter
  // per 32-byte sector
  static constexpr int UQ_MAX = 2048;
#ifndef GFSL_UQ_STRIDE
#define GFSL_UQ_STRIDE 8  // words between queue counters (8: one per 32-B sector; 32: per 128-B line)
#endif
  static constexpr int UQ_STRIDE = GFSL_UQ_STRIDE;
  uint32_t uq[UQ_MAX * UQ_STRIDE];
};

__device__ __forceinline__ uint32_t lo32(uint64_t x) { return (uint32_t)x; }
__device__ __forceinline__ uint32_t hi32(uint64_t x) { return (uint32_t)(x >> 32); }
__device__ __forceinline__ uint64_t mk64(uint32_t lo, uint32_t hi) {
  return (uint64_t)lo | ((uint64_t)hi << 32);
}

// ---- loads -------------------------------------------------------------------------
// Update phase: chunks are written concurrently, so every read goes to L2 (relaxed, gpu
// scope; never a stale L1 line).
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_acquire(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed32(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int32_t ld_relaxed_s32(const int32_t *p) {
  int32_t v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(uint64_t *p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t cas_acquire(uint64_t *p, uint64_t cmp, uint64_t val) {
  uint64_t old;
  asm volatile("atom.acquire.gpu.global.cas.b64 %0, [%1], %2, %3;"
               : "=l"(old)
               : "l"(p), "l"(cmp), "l"(val)
               : "memory");
  return old;
}
// 32-bit CAS with acquire on the lock-state half (lo32) of a LOCK entry.
__device__ __forceinline__ uint32_t cas32_acquire(uint64_t *p, uint32_t cmp, uint32_t val) {
  uint32_t old;
  asm volatile("atom.acquire.gpu.global.cas.b32 %0, [%1], %2, %3;"
               : "=r"(old)
               : "l"(p), "r"(cmp), "r"(val)
               : "memory");
  return old;
}
__device__ __forceinline__ void st_relaxed(uint64_t *p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// Contains phase: the structure is read-only for the whole kernel (S1), so the
// non-coherent read-only path (L1-allocating) is legal and lets hot upper-level chunks
// hit in L1.  One vector load per lane; EPL entries per lane.
template <int EPL>
struct ChunkSlice {
  uint32_t k[EPL];
  uint32_t v[EPL];
};

template <int EPL>
__device__ __forceinline__ void ld_slice_nc(const uint64_t *p, ChunkSlice<EPL> &s, uint64_t pol);

// The chunk loads of the search phase carry an L2 eviction-priority policy (createpolicy):
// level-0 chunks evict_first (a 1B-key level 0 is streamed, ~5 reads per line per batch),
// the upper levels and the directory evict_last, so that the L2 keeps as much of level 1
// as fits (R36).
__device__ __forceinline__ uint64_t l2_policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_policy_evict_last() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_policy_evict_normal() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
  return p;
}

template <>
__device__ __forceinline__ void ld_slice_nc<1>(const uint64_t *p, ChunkSlice<1> &s, uint64_t pol) {
  asm volatile("ld.global.nc.L2::cache_hint.v2.u32 {%0,%1}, [%2], %3;" : "=r"(s.k[0]), "=r"(s.v[0]) : "l"(p), "l"(pol));
}
template <>
__device__ __forceinline__ void ld_slice_nc<2>(const uint64_t *p, ChunkSlice<2> &s, uint64_t pol) {
  asm volatile("ld.global.nc.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(s.k[0]), "=r"(s.v[0]), "=r"(s.k[1]), "=r"(s.v[1])
               : "l"(p), "l"(pol));
}
template <>
__device__ __forceinline__ void ld_slice_nc<4>(const uint64_t *p, ChunkSlice<4> &s, uint64_t pol) {
  asm volatile("ld.global.nc.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
               : "=r"(s.k[0]), "=r"(s.v[0]), "=r"(s.k[1]), "=r"(s.v[1]), "=r"(s.k[2]),
                 "=r"(s.v[2]), "=r"(s.k[3]), "=r"(s.v[3])
               : "l"(p), "l"(pol));
}
template <>
__device__ __forceinline__ void ld_slice_nc<8>(const uint64_t *p, ChunkSlice<8> &s, uint64_t pol) {
  asm volatile("ld.global.nc.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
               : "=r"(s.k[0]), "=r"(s.v[0]), "=r"(s.k[1]), "=r"(s.v[1]), "=r"(s.k[2]),
                 "=r"(s.v[2]), "=r"(s.k[3]), "=r"(s.v[3])
               : "l"(p), "l"(pol));
  asm volatile("ld.global.nc.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
               : "=r"(s.k[4]), "=r"(s.v[4]), "=r"(s.k[5]), "=r"(s.v[5]), "=r"(s.k[6]),
                 "=r"(s.v[6]), "=r"(s.k[7]), "=r"(s.v[7])
               : "l"(p + 4), "l"(pol));
}

template <>
__device__ __forceinline__ void ld_slice_nc<16>(const uint64_t *p, ChunkSlice<16> &s, uint64_t pol) {
#pragma unroll
  for (int q = 0; q < 4; ++q)
    asm volatile("ld.global.nc.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                 : "=r"(s.k[4 * q]), "=r"(s.v[4 * q]), "=r"(s.k[4 * q + 1]), "=r"(s.v[4 * q + 1]),
                   "=r"(s.k[4 * q + 2]), "=r"(s.v[4 * q + 2]), "=r"(s.k[4 * q + 3]), "=r"(s.v[4 * q + 3])
                 : "l"(p + 4 * q), "l"(pol));
}

// Programmatic dependent launch: a kernel launched with programmatic stream serialization
// may start while its predecessor drains; it waits here before touching the predecessor's
// outputs, and lets its own dependents launch early.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

__device__ __forceinline__ void set_error(const DevState &d, uint32_t bit) {
  atomicOr(d.error, bit);
}
__device__ __forceinline__ void stat_add(const DevState &d, int slot, unsigned long long v = 1) {
  atomicAdd(d.stats + slot, v);
}

}  // namespace gfsl_dev
