// gfsl_search.cuh -- B1: the read-only search phase of a batch (Alg 4.1-4.4, 4.6).
//
// Under the S1 snapshot semantics (R1) every op of a batch is answered against
// the structure as it was before the batch.  So ALL traversals of a batch -- the
// Contains of Alg 4.1 and the searchSlow of every Insert/Delete (Alg 4.5 l.2, Alg 4.11
// l.3) -- run first, in this kernel, on a quiescent structure: no locks, no fences, no
// restarts, and chunk reads through the read-only L1 path.
//
// Traversal (searchDown, Alg 4.2, then searchLateral, Alg 4.4): each step is one
// coalesced chunk read followed by the team vote of getTidForNextStep (Alg 4.3):
//   DATA entry i votes  key_i <= k,   NEXT votes  max < k,   LOCK votes  zombie;
// the highest voting entry decides: LOCK -> lateral past a zombie (Alg 4.2
// l.9-11), NEXT -> lateral step keeping the previous chunk for a backtrack (l.15-18),
// DATA i -> down step through value_i (l.19-23), none -> backtrack through the previous
// chunk's highest key <= k (l.24-28, 33-38), or restart (l.25; impossible here).  On the
// bottom level the DATA vote is key_i == k (Alg 4.4).
//
// For an Insert/Delete the kernel also records what searchSlow returns (Alg 4.6): the
// path (chunk of the down step at every level, the enclosing bottom chunk at level 0)
// and the highest level at which k was seen.  Its result is exact already (under the
// <=1-mutation-per-key contract the snapshot decides "present?"), and only the ops that
// will mutate (Insert of an absent key, Delete of a present key) go on to the update
// kernel (B2), which starts from the recorded path ("the enclosing chunk must
// either be in the path or reachable from it").
//
// The kernel also does the batch intake: it reads the caller's op/key/value arrays
// directly (op i is team slot i), so no separate classify pass or op lists exist.
//
// B200 design: a team is TEAM lanes (TEAM | 32, TEAM <= N); each lane
// holds EPL = N/TEAM consecutive entries loaded with one vector load (8/16/32 B), so a
// warp runs 32/TEAM independent traversals in lockstep (P:205 allows teams smaller than
// a warp; the paper's one-team-per-warp is TEAM == N).  A team's vote is "highest lane
// holding a voting entry" (one __ballot_sync) plus that lane's own highest voting entry,
// and the down pointer comes with one __shfl_sync.  prevKv is reduced to the two
// values a backtrack needs: the previous chunk and its highest key <= k's down pointer.
#pragma once
#include "gfsl_device.cuh"

namespace gfsl_dev {

constexpr int PLAN_LEVELS = 16;  // path levels recorded per update op (height < 16)

// Op word: {op index | flags}.  A batch holds at most OPI_MASK + 1 = 2^29 ops.
constexpr uint32_t DELETE_FLAG = 0x80000000u;   // Delete
constexpr uint32_t UPDATE_FLAG = 0x40000000u;   // Insert or Delete
constexpr uint32_t INVALID_FLAG = 0x20000000u;  // bad op code or key: result 0xFF, no effect
constexpr uint32_t OPI_MASK = 0x1FFFFFFFu;
// Chunk indices are < 2^30, so a shuffled pointer carries two flag bits.
constexpr uint32_t PTR_MASK = 0x3FFFFFFFu;
constexpr uint32_t F_ZOMBIE = 0x80000000u;   // on the NEXT pointer: the chunk is a zombie
constexpr uint32_t F_LATERAL = 0x40000000u;  // on the NEXT pointer: max < k
constexpr uint32_t F_EQUAL = 0x80000000u;    // on the down pointer: the winning key == k

// The batch's input arrays (caller-owned device memory, input order).
struct BatchIn {
  const uint8_t *ops;
  const uint32_t *keys;
  const uint32_t *vals;  // may be NULL (= 0)
  uint8_t *res;
  uint32_t n;                // ops (or, with n_dev, the upper bound n_max)
  uint64_t key_range;
  const uint32_t *n_dev;     // NULL, or device word holding the op count (gfsl_batch_dn):
                             // the batch has min(*n_dev, n) ops, read at kernel time
  // Key-ordered intake (R39), or NULL: slot j is the j-th op in key order -- op sw[j] &
  // OPI_MASK, its op code (capped at 3 = invalid) in bits 29-30 of sw[j], its key skey[j]
  const uint32_t *skey;
  const uint32_t *sw;
};

// The mutations a batch's search phase hands to the update phase, compact: mutation m
// (in completion order) has its record and its path.
struct SearchOut {
  uint4 *mut_rec;       // [n]: {op index | DELETE_FLAG, internal key, path[0], top (Delete) | value (Insert)}
  uint32_t *plan_path;  // [n * PLAN_LEVELS]: mutation m's path, lane l = chunk at level l
  uint32_t *mut_of;     // [n] or NULL: op i -> its mutation index, 0xFFFFFFFF if none (serial
                        // and combining modes)
  uint32_t *mut_count;  // the MUT_REGIONS counters that number the records (ctl->mcnt, or
                        // ctl->ccnt when a combining pass selects the net mutations, R26)
  uint32_t region_cap;  // record slots per region (BatchCtl::mcnt)
  uint32_t *comb_key;   // [n] or NULL (combining mode, R26): op i's sort key = internal key
                        // for a valid Insert/Delete, else all ones
  uint32_t *comb_w;     // [n]: op i | CW_* flags (the sort's payload)
  uint32_t full_path;   // 1 = every Insert/Delete traverses from the top (serial mode)
  uint32_t spread;      // 1 = the update kernel takes the records in a spread order (R31:
                        // combining mode, whose net records come out of a key sort)
  // Chunk-grouped mutations (R40), or NULL: the records of a batch that target the same
  // level-0 chunk (path[0]) form one list -- ghead[c - cap_upper] = the last record pushed
  // for chunk c, gnext[m] = the record pushed before m (EMPTY_GROUP ends the list).  The
  // update kernel applies a list of >= 2 records in one lock session of its chunk; the
  // first record pushed (gnext == EMPTY_GROUP) is the list's leader.  ghead is all
  // EMPTY_GROUP between batches (the update kernel resets the entries it takes).
  uint32_t *ghead;
  uint32_t *gnext;
  // R41: 1 = a mutation whose traversal entered level 0 through the directory (R37) does
  // not write its path: levels >= 1 are the closed form of its key's directory rank, which
  // the update kernel recomputes in the rare cases that need them (record flag
  // PATH_DERIVED; lazy batches, update paths that support it)
  uint32_t derive_path;
};
constexpr uint32_t EMPTY_GROUP = 0xFFFFFFFFu;
constexpr uint32_t PATH_DERIVED = 0x40000000u;  // on a record's op word (R41)

// R41: the directory rank of an internal key (R27b / R27c layouts): the rank the search
// kernel entered level 0 with.  The directory is read-only from the search kernel to the
// next rebuild.
__device__ __forceinline__ uint32_t dir_rank_of(const DevState &d, uint32_t key) {
  const uint32_t q = key >> d.dir_hdr[0];
#ifdef GFSL_DIR_U32
  return ((const uint32_t *)d.dir)[q];
#else
  if (d.dir_hdr[8]) {
    const uint32_t g = q / DIR_SEC_BUCKETS;
    const uint8_t *sec = d.dir + (size_t)g * 32;
    return *(const uint32_t *)sec + sec[4 + (q - g * DIR_SEC_BUCKETS)];
  }
  return d.dir_base[q >> 5] + d.dir[q];
#endif
}
// R41: lane l's path entry of such a record (lanes above the snapshot height: head[l]),
// the chunk the search kernel would have recorded: path[0] = the record's bottom chunk,
// path[l] = the chunk of rebuilt level l that holds rank r / F^l (R27, R37).
template <int N>
__device__ __forceinline__ uint32_t derived_path_lane(const DevState &d, uint32_t k, uint32_t c0, int lane,
                                                      bool path_lane, uint32_t head_l) {
  if (!path_lane) return head_l;
  if (lane == 0) return c0;
  constexpr uint32_t F = N - 4;  // keys per rebuilt upper chunk (RebuildBufs::fill)
  uint32_t q = dir_rank_of(d, k);
  for (int l = 0; l < lane; ++l) q /= F;
  return q ? d.dir_hdr[32 + lane] + q - 1u : (uint32_t)(lane == 1 ? 0 : lane - 1);
}

// Mutation records occupy REC_STRIDE x 16 B: 1 = packed 16-B records (default); 2 = one
// full 32-B sector per record, written with one 32-B store, so that no record is a
// partial-sector write (measured: within 0.6% of 1 at C2-C5, profiles/r02/ab_record_stride.txt).
#ifndef GFSL_REC_STRIDE
#define GFSL_REC_STRIDE 1
#endif
constexpr uint32_t REC_STRIDE = GFSL_REC_STRIDE;
__device__ __forceinline__ uint4 *rec_at(uint4 *base, uint32_t m) { return base + (size_t)m * REC_STRIDE; }
__device__ __forceinline__ const uint4 *rec_at(const uint4 *base, uint32_t m) { return base + (size_t)m * REC_STRIDE; }
__device__ __forceinline__ void rec_store(uint4 *base, uint32_t m, uint4 r) {
  if (REC_STRIDE == 2) {
    asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%5,%5,%5};" ::"l"(base + (size_t)m * 2), "r"(r.x), "r"(r.y),
                 "r"(r.z), "r"(r.w), "r"(0u)
                 : "memory");
  } else {
    base[m] = r;
  }
}

// A record slot in the writing block's region (BatchCtl::mcnt).
// Warp-aggregated: the converged lanes that append take consecutive slots with one atomic.
__device__ __forceinline__ uint32_t mut_slot(const SearchOut &so) {
  const uint32_t rg = blockIdx.x % BatchCtl::MUT_REGIONS;
  const uint32_t am = __activemask();
  const int lane = threadIdx.x & 31;
  const int leader = __ffs(am) - 1;
  uint32_t base = 0;
  if (lane == leader) base = atomicAdd(so.mut_count + rg * BatchCtl::CNT_STRIDE, (uint32_t)__popc(am));
  base = __shfl_sync(am, base, leader);
  return rg * so.region_cap + base + (uint32_t)__popc(am & ((1u << lane) - 1u));
}

// Combining-mode payload flags (R26); the op index is < 2^29.
constexpr uint32_t CW_P0 = 0x80000000u;      // k was present in the snapshot
constexpr uint32_t CW_DEL = 0x40000000u;     // Delete (else Insert)
constexpr uint32_t CW_NOTMUT = 0x20000000u;  // Contains or invalid: not part of any chain

// Keys of the sorted-min-key window a coarse directory (C5) reads: 8 (two 16-B reads; 12 and 16
// measured slower at C5: every read is a request, and the kernel is request-bound)
// L2 priority of the coarse directory's min-key window reads: 0 evict_last (as the
// directory), 1 evict_normal, 2 evict_first
#ifndef GFSL_OK_POLICY
#define GFSL_OK_POLICY 0
#endif
#ifndef GFSL_OK_WIN
#define GFSL_OK_WIN 8
#endif

#ifndef GFSL_SEARCH_MIN_BLOCKS
// 4 blocks per SM (<= 64 registers, no spill): with level 0 entered directly (R37/R38) a
// traversal is ~1-2 dependent gathers, latency-bound (ncu at C5: 0.45 eligible warps per
// scheduler at 3 blocks), so more resident warps win -- one gpurun call, 3 -> 4 blocks:
// C5 7664 -> 8088, C4-16 15575 -> 21173, C3 8109 -> 8808, C2 4962 -> 5449 Mops/s (5 and 6
// blocks, 48 / 40 registers, lose at C4 / C5)
#define GFSL_SEARCH_MIN_BLOCKS 4
#endif

// The search phase of a batch: the body of search_kernel, and the first half of the
// small-batch kernel (gfsl_update.cuh).
template <int N, int TEAM, bool COUNT = false, bool IDLE_SKIP = false>
__device__ __forceinline__ void search_body(const DevState &d, const BatchIn &in, BatchCtl *__restrict__ ctl,
                                            const SearchOut &so) {
  constexpr int EPL = N / TEAM;
  static_assert(EPL * TEAM == N, "TEAM must divide N");
  constexpr int TPW = 32 / TEAM;                    // teams per warp
  constexpr uint32_t TEAM_BITS = (TEAM == 32) ? 0xFFFFFFFFu : ((1u << TEAM) - 1u);
  constexpr int NEXT_E = N - 2, LOCK_E = N - 1;
  constexpr int NEXT_LANE = NEXT_E / EPL, NEXT_J = NEXT_E % EPL;
  constexpr int LOCK_LANE = LOCK_E / EPL, LOCK_J = LOCK_E % EPL;
  constexpr uint32_t FULL = 0xFFFFFFFFu;

  __shared__ uint32_t s_start, s_height, s_dir_shift, s_head0, s_l0_ok, s_korder, s_n1, s_dsec;
  __shared__ uint32_t s_dir_base[PLAN_LEVELS];  // base of each rebuilt level (R27)
  // the path of the team's current op (written by its lane 0 only), copied out compactly
  // at the end if the op mutates (about 1 op in 10)
  __shared__ __align__(16) uint32_t s_path[(256 / 32) * TPW][PLAN_LEVELS];
  const int lane = threadIdx.x & 31;
  pdl_wait();
  pdl_trigger();
  if (threadIdx.x < 32) {
    // getHeight / firstChunkAtLevel: lane l reads level l's counter.
    const int32_t c = (lane < N) ? d.counter[lane] : 0;
    const uint32_t b = __ballot_sync(FULL, lane >= 1 && lane < N && c > 0);
    const uint32_t h = b ? 31u - __clz(b) : 0u;
    if (lane == 0) {
      s_height = h;
      s_start = d.head[h];
      s_head0 = d.head[0];
      s_l0_ok = d.dir_hdr[4];
      s_korder = d.dir_hdr[5];
      s_n1 = d.dir_hdr[6];
      s_dsec = d.dir_hdr[8];
      // R27: Contains enter at level 1 through the directory when there are levels above
      s_dir_shift = (h >= 2 && d.dir_hdr[1]) ? d.dir_hdr[0] : 32u;
      if (blockIdx.x == 0) {
        ctl->snap_height = h;
        if (d.bump_host) {  // (zero-copy: no D2H copy node per batch)
          d.bump_host[0] = d.bump[0];
          d.bump_host[1] = d.bump[1];
        }
      }
    }
    if (lane < PLAN_LEVELS) s_dir_base[lane] = d.dir_hdr[32 + lane];
  }
  __syncthreads();
  const uint32_t start = s_start;
  const int height = (int)s_height;
  const uint32_t dir_shift = s_dir_shift;
  const bool use_dir = dir_shift < 32u;
  // where a traversal starts: searchDown from the top (Alg 4.2 l.2-4), or -- when the
  // directory is valid -- at level 1, in the chunk of rank r / F that the directory names
  // for k's bucket (R27).  An Insert/Delete entered there records its path at levels 1
  // and 0 as it goes (searchSlow, Alg 4.6) and takes the levels above from the same rank
  // (chunk r / F^l of level l: a valid start for findAndLockEnclosing); a Delete
  // that finds k at level 1 starts over from the top, since its exact top level is needed.
  // Serial mode (full_path) traverses every Insert/Delete from the top.
  constexpr uint32_t F = N - 4;  // keys per rebuilt upper chunk (RebuildBufs::fill)
  const bool dir_upd = use_dir && !so.full_path;
  auto dir_op = [&](uint32_t opw) {
    return use_dir && !(opw & INVALID_FLAG) && (dir_upd || !(opw & UPDATE_FLAG));
  };
  auto l1_chunk = [&](uint32_t r) { const uint32_t q = r / F; return q ? s_dir_base[1] + q - 1u : 0u; };
  // R37: enter at level 0, in the chunk of level-1 entry r's down pointer (the rebuild's
  // rank order); the levels above are skipped (their path entries come from r, as R27's)
  const bool korder = s_korder != 0;   // R38: level 0 in rank order
  const bool dsec = s_dsec != 0;       // R27c: sector layout of the directory
  const uint32_t n1 = s_n1;
  const bool l0_entry = d.l0_entry != 0 && (s_l0_ok != 0 || korder);
  const bool fine_dir = s_l0_ok != 0;  // >= 1 directory bucket per level-1 key
  const uint32_t head0 = s_head0;
  // an Insert/Delete may skip the upper levels only in a lazy batch (R33: no raise, no
  // upper-level delete); otherwise it enters at level 1 (R27) to see its exact top
  auto l0_op = [&](uint32_t opw) { return l0_entry && (d.lazy_upper || !(opw & UPDATE_FLAG)); };
  const uint32_t n = in.n_dev ? min(*(volatile const uint32_t *)in.n_dev, in.n) : in.n;
  uint8_t *__restrict__ res = in.res;

  const int team_in_warp = lane / TEAM;
  const int t = lane - team_in_warp * TEAM;          // tId
  const bool lane_live = team_in_warp < TPW;         // lanes past TPW*TEAM idle
  const int team_base = lane_live ? team_in_warp * TEAM : lane;
  const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t total_teams = (gridDim.x * blockDim.x >> 5) * TPW;
  const int next_src = lane_live ? team_base + NEXT_LANE : lane;
  uint32_t *const my_path = s_path[((threadIdx.x >> 5) * TPW + (lane_live ? team_in_warp : 0)) % ((256 / 32) * TPW)];

  // Batch intake, fused: op slot i is input op i, read straight from the caller's arrays
  // (range/op-code check; an invalid op is traversed as a Contains of key 0 and answered
  // 0xFF).  Internal key = key + 1 (R3).  One op prefetched.
  // The prefetched op stays raw (loaded, not yet looked at) until it becomes current, so
  // its loads overlap the current traversal.
  // An Insert's value is loaded when the op becomes current (it is needed only at its end).
  // R39: with a key-ordered intake, slot j carries its input index
  struct RawOp {
    uint32_t op, key, idx;
  };
  auto load_raw = [&](uint32_t i) -> RawOp {
    RawOp r{3u, 0u, i};
    if (lane_live && i < n) {
      if (in.sw) {
        const uint32_t w = __ldg(in.sw + i);
        r.op = (w >> 29) & 3u;
        r.idx = w & OPI_MASK;
        r.key = __ldg(in.skey + i);
      } else {
        r.op = __ldg(in.ops + i);
        r.key = __ldg(in.keys + i);
      }
    }
    return r;
  };
  auto load_val = [&](uint32_t i, const RawOp &r) -> uint32_t {
    return (t == 0 && in.vals && r.op == 1 && lane_live && i < n) ? __ldg(in.vals + r.idx) : 0u;
  };
  auto decode = [&](uint32_t i, const RawOp &r) -> uint2 {
    (void)i;
    const bool valid = r.op <= 2 && (uint64_t)r.key < in.key_range;
    const uint32_t fl = !valid ? INVALID_FLAG : (r.op == 2 ? (DELETE_FLAG | UPDATE_FLAG) : (r.op == 1 ? UPDATE_FLAG : 0u));
    return make_uint2(r.idx | fl, valid ? r.key + 1u : 1u);
  };
  uint32_t slot = warp_global * TPW + team_in_warp;  // this team's current op slot
  RawOp raw = load_raw(slot);
  uint2 cur_op = decode(slot, raw);
  uint32_t cur_val = load_val(slot, raw);
  RawOp nxt = load_raw(slot + total_teams);
  bool active = lane_live && slot < n;
  uint32_t k = cur_op.y;
  bool via_dir = dir_op(cur_op.x);
  // R36: L2 eviction priorities -- level-0 chunks evict_first (when the host chose it for
  // this structure's size), the upper levels and the directory evict_last
#ifndef GFSL_SEARCH_HINTS
#define GFSL_SEARCH_HINTS 2
#endif
  const uint64_t pol_l0 = (GFSL_SEARCH_HINTS >= 1 && d.l0_evict_first) ? l2_policy_evict_first() : l2_policy_evict_normal();
  const uint64_t pol_up = GFSL_SEARCH_HINTS >= 2 ? l2_policy_evict_last() : l2_policy_evict_normal();
  // the coarse directory's min-key window (C5: a 200-MB array, larger than the L2)
#if GFSL_OK_POLICY == 1
  const uint64_t pol_ok = l2_policy_evict_normal();
#elif GFSL_OK_POLICY == 2
  const uint64_t pol_ok = l2_policy_evict_first();
#else
  const uint64_t pol_ok = pol_up;
#endif
  // the op's directory rank (R27b): base of its 32-bucket group + its byte
  auto dir_rank = [&](uint2 e, uint32_t) -> uint32_t { return e.x + e.y; };
  auto ld_dir = [&](uint32_t key) -> uint2 {
    const uint32_t q = key >> dir_shift;
#ifdef GFSL_DIR_U32
    return make_uint2(__ldg((const uint32_t *)d.dir + q), 0u);
#else
    uint32_t base, byte;
    if (dsec) {  // R27c: base and byte in one 32-B sector
      const uint32_t g = q / DIR_SEC_BUCKETS;
      const uint8_t *sec = d.dir + (size_t)g * 32;
      asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(base) : "l"(sec), "l"(pol_up));
      asm volatile("ld.global.nc.L2::cache_hint.u8 %0, [%1], %2;" : "=r"(byte) : "l"(sec + 4 + (q - g * DIR_SEC_BUCKETS)), "l"(pol_up));
      return make_uint2(base, byte);
    }
    asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(base) : "l"(d.dir_base + (q >> 5)), "l"(pol_up));
    asm volatile("ld.global.nc.L2::cache_hint.u8 %0, [%1], %2;" : "=r"(byte) : "l"(d.dir + q), "l"(pol_up));
    return make_uint2(base, byte);
#endif
  };
  auto l0_chunk = [&](uint32_t r, uint32_t key) -> uint32_t {
    if (korder) {
      // R38: rank(key) = r + the sorted min keys >= index r that are <= key (those before
      // r are <= key already).  A fine directory (>= 1 bucket per key) needs a short look-
      // ahead: one aligned 32-B read of r's group of 8; a coarse one (C5: ~3 keys per
      // bucket) three aligned 16-B reads from r rounded down to 4, >= 9 keys past r.
      if (fine_dir) {
        const uint32_t g = r & ~7u;
        uint32_t o[8];
        asm volatile("ld.global.nc.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                     : "=r"(o[0]), "=r"(o[1]), "=r"(o[2]), "=r"(o[3]), "=r"(o[4]), "=r"(o[5]), "=r"(o[6]), "=r"(o[7])
                     : "l"(d.dir_ok + g), "l"(pol_up));
        uint32_t rho = g;
#pragma unroll
        for (int i = 0; i < 8; ++i) rho += (g + i < n1 && o[i] <= key) ? 1u : 0u;
        return d.cap_upper + rho;  // the chunk of rank rho (rho = g + 8: laterally onward)
      }
      constexpr int OKQ = GFSL_OK_WIN / 4;  // 16-B reads of the window
      const uint32_t s0 = r & ~3u;
      uint32_t o[4 * OKQ];
#pragma unroll
      for (int q = 0; q < OKQ; ++q)
        asm volatile("ld.global.nc.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                     : "=r"(o[4 * q]), "=r"(o[4 * q + 1]), "=r"(o[4 * q + 2]), "=r"(o[4 * q + 3])
                     : "l"(d.dir_ok + s0 + 4 * q), "l"(pol_ok));
      uint32_t rho = s0;
#pragma unroll
      for (int i = 0; i < 4 * OKQ; ++i) rho += (s0 + i < n1 && o[i] <= key) ? 1u : 0u;
      return d.cap_upper + rho;  // the chunk of rank rho (rho = s0 + GFSL_OK_WIN: laterally onward)
    }
    if (!r) return head0;
    uint32_t c;
    asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(c) : "l"(d.dir_oc + r - 1), "l"(pol_up));
    return c;
  };
  uint32_t cur_r = via_dir ? dir_rank(ld_dir(k), k) : 0u;
  bool via_l0 = via_dir && l0_op(cur_op.x);
  uint32_t cur = via_dir ? (via_l0 ? l0_chunk(cur_r, k) : l1_chunk(cur_r)) : start;
  int level = via_dir ? (via_l0 ? 0 : 1) : height;
  // the next op's directory word is loaded one loop iteration after its raw op (so that
  // its key has arrived), and is ready when the op becomes current
  uint2 nxt_dir = make_uint2(0u, 0u);
  bool pf_dir = use_dir;
  uint32_t bt = NULL_CHUNK, bt_c = NULL_CHUNK;       // prevKv, reduced
  int seen_top = 0;                                  // highest level where k was seen
  unsigned long long restarts = 0;
  unsigned long long reads = 0, reads_l0 = 0, nops = 0;  // COUNT build only

  while (__any_sync(FULL, active)) {
    ChunkSlice<EPL> s;
    if (IDLE_SKIP && !active) {  // a team whose ops are done issues no request
#pragma unroll
      for (int j = 0; j < EPL; ++j) s.k[j] = s.v[j] = KEY_EMPTY;
    } else {
      ld_slice_nc<EPL>(d.pool + (size_t)cur * N + t * EPL, s, level == 0 ? pol_l0 : pol_up);
    }
    if (pf_dir) {
      if ((nxt.op == 0 || (dir_upd && nxt.op <= 2)) && (uint64_t)nxt.key < in.key_range) {
        nxt_dir = ld_dir(nxt.key + 1u);
      }
      pf_dir = false;
    }
    if (COUNT && active) {
      ++reads;
      reads_l0 += (level == 0);
    }
    // NEXT / LOCK entries: the lateral and zombie flags ride on the next pointer; their
    // keys are replaced by EMPTY so that they never take part in the DATA vote.
    uint32_t nx = s.v[NEXT_J] & PTR_MASK;  // NULL (last chunk) is never followed
    if (t == NEXT_LANE) {
      if (s.k[NEXT_J] < k) nx |= F_LATERAL;  // NEXT votes max < k (Alg 4.3 l.4)
      s.k[NEXT_J] = KEY_EMPTY;
    }
    if (t == LOCK_LANE) {
      if (s.k[LOCK_J] == LOCK_ZOMBIE) nx |= F_ZOMBIE;
      s.k[LOCK_J] = KEY_EMPTY;
    }
    if (LOCK_LANE != NEXT_LANE) nx |= __shfl_down_sync(FULL, nx & F_ZOMBIE, 1);
    // DATA vote as one unsigned range test klo <= key <= k: klo = 0 above the bottom
    // level (key <= k, Alg 4.3 l.3), klo = k on it (key == k, Alg 4.4 l.4).  EMPTY
    // (+inf) never votes.  Keys ascend within a lane: the last voter is the highest.
    const uint32_t klo = level == 0 ? k : 0u;
    const uint32_t span = k - klo;
    bool any = false;
    uint32_t dv = 0, dk = 0;
#pragma unroll
    for (int j = 0; j < EPL; ++j) {
      const bool v = (s.k[j] - klo) <= span;
      any |= v;
      dv = v ? s.v[j] : dv;
      dk = v ? s.k[j] : dk;
    }
    dv |= (dk == k) ? F_EQUAL : 0u;

    const uint32_t bd = __ballot_sync(FULL, active && any);
    const uint32_t tb = (bd >> (team_base & 31)) & TEAM_BITS;
    const int src = tb ? team_base + 31 - __clz(tb) : lane;
    const uint32_t dptr = __shfl_sync(FULL, dv, src);
    const uint32_t np = __shfl_sync(FULL, nx, next_src);

    if (active) {
      const bool lat = (np & (F_ZOMBIE | F_LATERAL)) != 0;  // zombie (l.9-11) / lateral (l.15-18)
      const bool done = !lat && level == 0;                 // bottom enclosing chunk (Alg 4.4)
      const bool down = !lat && level > 0;                  // down step (l.19-23) / backtrack
      const bool upd = (cur_op.x & UPDATE_FLAG) != 0;
      // restart (l.25): only from a directory entry made stale by the batches since the
      // last rebuild (R27: level-1 keys <= k deleted from that chunk), never from the top;
      // and on purpose when a Delete entered at level 1 finds k there (its exact top)
      const bool redo = via_dir && down && level == 1 && tb && (dptr & F_EQUAL) && (cur_op.x & DELETE_FLAG) &&
                        !d.lazy_upper;  // R33: a lazy Delete removes k from level 0 only
      const bool restart = (down && !tb && bt == NULL_CHUNK) || redo;
      const uint32_t here = cur;
      if (down && upd && t == 0 && level < PLAN_LEVELS)     // searchSlow's path (Alg 4.6 l.28-37)
        my_path[level] = tb ? cur : bt_c;
      if (down && tb && (dptr & F_EQUAL) && seen_top == 0) seen_top = level;
      const bool set_bt = lat && !(np & F_ZOMBIE) && level > 0;  // prevKv = currKv (l.16)
      const uint32_t next_cur = lat ? (np & PTR_MASK) : (tb ? (dptr & PTR_MASK) : bt);
      bt = set_bt ? (tb ? (dptr & PTR_MASK) : NULL_CHUNK) : (down ? NULL_CHUNK : bt);
      bt_c = set_bt ? cur : (down ? NULL_CHUNK : bt_c);
      cur = restart ? start : next_cur;
      level = restart ? height : level - (down ? 1 : 0);
      if (restart) {
        restarts += redo ? 0 : 1;
        seen_top = 0;
        via_dir = false;
        via_l0 = false;
        bt = bt_c = NULL_CHUNK;
      }
      if (done) {
        const bool te = tb != 0;
        const uint32_t opi = cur_op.x & OPI_MASK;
        if (t == 0) {
          uint32_t m = 0xFFFFFFFFu;
          if (!upd) {
            res[opi] = (cur_op.x & INVALID_FLAG) ? 0xFF : (te ? 1 : 0);
          } else {
            // Alg 4.5 l.3-4 / Alg 4.11 l.4-5 on the snapshot: exact under the contract
            const bool mut = (cur_op.x & DELETE_FLAG) ? te : !te;
            res[opi] = mut ? 1 : 0;
            if (mut) {
              m = mut_slot(so);
              // R41: entered at level 0 through the directory -> the path is derivable
              const bool derive = so.derive_path && via_l0;
              // {op index | DELETE_FLAG | PATH_DERIVED, key, path[0], top (Delete) | value (Insert)}
              const uint32_t w = opi | (cur_op.x & DELETE_FLAG) | (derive ? PATH_DERIVED : 0u);
              // R33: in lazy mode a Delete's top is 0 (level-1 copies of k stay until the
              // next rebuild, as stale separators)
              rec_store(so.mut_rec, m, make_uint4(w, k, here, (cur_op.x & DELETE_FLAG) ? (d.lazy_upper ? 0u : (uint32_t)seen_top) : cur_val));
              if (so.ghead) so.gnext[m] = atomicExch(so.ghead + (here - d.cap_upper), m);  // R40
              if (!derive) {
              my_path[0] = here;  // path[0] = the enclosing bottom chunk
              if (via_dir) {      // levels >= 2 (and 1, R37) from the directory rank (R27)
                uint32_t q = cur_r / F;
                if (via_l0) my_path[1] = q ? s_dir_base[1] + q - 1u : 0u;
#pragma unroll
                for (int l = 2; l < PLAN_LEVELS; ++l) {
                  q /= F;
                  my_path[l] = q ? s_dir_base[l] + q - 1u : (uint32_t)(l - 1);
                }
              }
              const uint4 *src = reinterpret_cast<const uint4 *>(my_path);
              uint4 *dst = reinterpret_cast<uint4 *>(so.plan_path + (size_t)m * PLAN_LEVELS);
#pragma unroll
              for (int q = 0; q < PLAN_LEVELS / 4; ++q) dst[q] = src[q];
              }
            }
          }
          if (so.mut_of) so.mut_of[opi] = m;
          if (so.comb_key) {  // R26: the op's place in its key's chain
            const bool chain = upd && !(cur_op.x & INVALID_FLAG);
            so.comb_key[opi] = chain ? k : 0xFFFFFFFFu;
            so.comb_w[opi] = opi | (chain ? ((te ? CW_P0 : 0u) | ((cur_op.x & DELETE_FLAG) ? CW_DEL : 0u)) : CW_NOTMUT);
          }
        }
        if (COUNT) ++nops;
        // next op of this team (prefetched one ahead)
        slot += total_teams;
        active = slot < n;
        cur_op = decode(slot, nxt);
        cur_val = load_val(slot, nxt);
        k = cur_op.y;
        nxt = load_raw(slot + total_teams);
        via_dir = dir_op(cur_op.x);
        cur_r = dir_rank(nxt_dir, k);
        via_l0 = via_dir && l0_op(cur_op.x);
        cur = via_dir ? (via_l0 ? l0_chunk(cur_r, k) : l1_chunk(cur_r)) : start;
        level = via_dir ? (via_l0 ? 0 : 1) : height;
        pf_dir = use_dir;
        bt = bt_c = NULL_CHUNK;
        seen_top = 0;
      }
    }
  }
  if (restarts && t == 0) stat_add(d, ST_RESTARTS, restarts);
  if (COUNT && t == 0 && lane_live) {
    stat_add(d, ST_CREADS, reads);
    stat_add(d, ST_CREADS_L0, reads_l0);
    stat_add(d, ST_COPS, nops);
  }
}

// IDLE_SKIP: a team whose ops are done issues no chunk load while its warp finishes (the
// host takes it when level 0 exceeds the L2: C5 with R41 9.8 vs 13.4-14.6 ms per batch;
// where level 0 is L2-resident the re-reads are cheap and the skip's branch is not: C3 -4%)
template <int N, int TEAM, bool COUNT = false, bool IDLE_SKIP = false>
__global__ void __launch_bounds__(256, GFSL_SEARCH_MIN_BLOCKS)
search_kernel(const __grid_constant__ DevState d, const BatchIn in, BatchCtl *__restrict__ ctl, SearchOut so) {
  search_body<N, TEAM, COUNT, IDLE_SKIP>(d, in, ctl, so);
}

// The update kernel's view of the region-numbered records: slot s in [0, total) ->
// record index.  Built once per block from the MUT_REGIONS counters (shared memory).
struct MutMap {
  const uint32_t *excl;  // [MUT_REGIONS + 1] exclusive prefix of the counts (shared)
  uint32_t cap;
  uint32_t spread;       // R31: take slot s as (s * 2654435761) mod total (a bijection: the
                         // multiplier is a prime > 2^29 >= total), so that the records the
                         // update teams hold at one time -- which the combining sort wrote
                         // in key order -- are far apart in key space
  __device__ __forceinline__ uint32_t total() const { return excl[BatchCtl::MUT_REGIONS]; }
  __device__ __forceinline__ uint32_t rec(uint32_t s) const {
    if (spread) s = (uint32_t)(((uint64_t)s * 2654435761ull) % total());
    int r = 0;  // the last region whose prefix is <= s (empty regions are skipped)
#pragma unroll
    for (int step = BatchCtl::MUT_REGIONS / 2; step >= 1; step >>= 1)
      if (excl[r + step] <= s) r += step;
    return (uint32_t)r * cap + (s - excl[r]);
  }
  // The same for a caller whose slots only grow (a work queue's items, no spread): the
  // region cursor moves forward, O(1) amortised instead of a 5-step binary search.
  __device__ __forceinline__ uint32_t rec_fwd(uint32_t s, uint32_t &rg) const {
    if (spread) return rec(s);
    while (rg + 1 < (uint32_t)BatchCtl::MUT_REGIONS && excl[rg + 1] <= s) ++rg;
    return rg * cap + (s - excl[rg]);
  }
};

// Fills s_excl (MUT_REGIONS + 1 entries) from the counters; call from every thread of
// the block before any thread returns, then __syncthreads().
__device__ __forceinline__ void mutmap_build(const uint32_t *cnt, uint32_t *s_excl) {
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    const uint32_t v = cnt[lane * BatchCtl::CNT_STRIDE];
    uint32_t incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
      if (lane >= o) incl += y;
    }
    s_excl[lane] = incl - v;
    if (lane == 31) s_excl[32] = incl;
  }
}

}  // namespace gfsl_dev
