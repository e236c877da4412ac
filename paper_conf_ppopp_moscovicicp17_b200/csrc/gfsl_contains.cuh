// gfsl_contains.cuh -- B1: the Contains phase of a batch (Alg 4.1-4.4).
//
// Under the S1 snapshot semantics (R1) every Contains of a batch runs before
// any Insert/Delete of the batch, so this kernel sees a quiescent structure: it takes no
// locks, needs no fences, and reads chunks through the read-only L1 path.  The traversal
// is the paper's: searchDown (Alg 4.2) over the upper levels, then searchLateral
// (Alg 4.4) on the bottom level; each step is one coalesced chunk read followed by a
// team vote (getTidForNextStep, Alg 4.3):
//   DATA entry i votes  key_i <= k,   NEXT votes  max < k,   LOCK votes  zombie;
// the highest voting entry decides:  LOCK -> lateral past a zombie (Alg 4.2
// l.9-11), NEXT -> lateral step keeping the previous chunk for a backtrack (l.15-18),
// DATA i -> down step through value_i (l.19-23), none -> backtrack through the previous
// chunk's highest key <= k (l.24-28, 33-38), or restart if there is none (l.25).
// On the bottom level the DATA vote is key_i == k (Alg 4.4).
//
// B200 design: a team is TEAM lanes (TEAM | 32, TEAM <= N); each lane
// holds EPL = N/TEAM consecutive entries, loaded with one vector load (8/16/32 B), so a
// warp runs 32/TEAM independent traversals in lockstep (P:205 allows teams smaller than
// a warp; the paper's one team per warp is the TEAM == N case).  The vote of a team is
// "highest lane holding a voting entry" (one __ballot_sync) plus that lane's own highest
// voting entry (registers), and the down pointer comes with one __shfl_sync.  prevKv
// is reduced to the one value a backtrack needs: the down pointer of the
// previous chunk's highest key <= k, which is known when the lateral step is taken.
#pragma once
#include "gfsl_device.cuh"

namespace gfsl_dev {

template <int N, int TEAM, bool COUNT = false>
__global__ void __launch_bounds__(256)
contains_kernel(DevState d, const uint32_t *__restrict__ keys, uint8_t *__restrict__ res,
                const uint32_t *__restrict__ list, const BatchCtl *__restrict__ ctl) {
  constexpr int DSIZE = N - 2;
  constexpr int EPL = N / TEAM;
  static_assert(EPL * TEAM == N, "TEAM must divide N");
  constexpr int TPW = 32 / TEAM;                    // teams per warp
  constexpr uint32_t TEAM_BITS = (TEAM == 32) ? 0xFFFFFFFFu : ((1u << TEAM) - 1u);
  constexpr int NEXT_E = N - 2, LOCK_E = N - 1;
  constexpr int NEXT_LANE = NEXT_E / EPL, NEXT_J = NEXT_E % EPL;
  constexpr int LOCK_LANE = LOCK_E / EPL, LOCK_J = LOCK_E % EPL;
  constexpr uint32_t FULL = 0xFFFFFFFFu;

  __shared__ uint32_t s_start, s_height;
  const int lane = threadIdx.x & 31;
  if (threadIdx.x < 32) {
    // getHeight / firstChunkAtLevel: lane l reads level l's counter.
    int32_t c = (lane < N) ? d.counter[lane] : 0;
    uint32_t b = __ballot_sync(FULL, lane >= 1 && lane < N && c > 0);
    uint32_t h = b ? 31u - __clz(b) : 0u;
    if (lane == 0) {
      s_height = h;
      s_start = d.head[h];
    }
  }
  __syncthreads();
  const uint32_t start = s_start;
  const int height = (int)s_height;
  const uint32_t n = ctl->n_contains;

  const int team_in_warp = lane / TEAM;
  const int t = lane - team_in_warp * TEAM;          // tId
  const bool lane_live = team_in_warp < TPW;         // lanes past TPW*TEAM idle
  const int team_base = team_in_warp * TEAM;
  const uint32_t warp_global = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t total_teams = (gridDim.x * blockDim.x >> 5) * TPW;

  uint32_t slot = warp_global * TPW + team_in_warp;  // this team's current op slot
  bool active = lane_live && slot < n;
  uint32_t opi = 0, k = 0;
  if (active) {
    opi = list[slot];
    k = keys[opi] + 1u;                               // internal key (R3)
  }
  uint32_t cur = start;
  int level = height;
  uint32_t bt = NULL_CHUNK;                          // backtrack pointer (reduced prevKv)
  unsigned long long restarts = 0;
  unsigned long long reads = 0, reads_l0 = 0, nops = 0;  // COUNT build only

  while (__any_sync(FULL, active)) {
    ChunkSlice<EPL> s;
    if (active) {
      ld_slice_nc<EPL>(d.pool + (size_t)cur * N + t * EPL, s);
      if (COUNT) {
        ++reads;
        reads_l0 += (level == 0);
      }
    } else {
#pragma unroll
      for (int j = 0; j < EPL; ++j) { s.k[j] = KEY_EMPTY; s.v[j] = NULL_CHUNK; }
    }
    // per-lane part of the vote
    int bj = -1;
    bool eq = false;
    uint32_t dv = NULL_CHUNK;
#pragma unroll
    for (int j = 0; j < EPL; ++j) {
      const int e = t * EPL + j;
      if (e < DSIZE) {
        if (s.k[j] <= k) { bj = j; dv = s.v[j]; }
        eq |= (s.k[j] == k);
      }
    }
    const bool lat = (t == NEXT_LANE) && (s.k[NEXT_J] < k);           // max < k
    const bool zom = (t == LOCK_LANE) && (s.k[LOCK_J] == LOCK_ZOMBIE);
    const uint32_t nxt = s.v[NEXT_J];

    const uint32_t bd = __ballot_sync(FULL, active && bj >= 0);
    const uint32_t bl = __ballot_sync(FULL, active && lat);
    const uint32_t bz = __ballot_sync(FULL, active && zom);
    const uint32_t be = __ballot_sync(FULL, active && eq);
    const uint32_t tb = (bd >> team_base) & TEAM_BITS;
    const int src = tb ? team_base + 31 - __clz(tb) : lane;
    const uint32_t dptr = __shfl_sync(FULL, dv, src);
    const uint32_t np = __shfl_sync(FULL, nxt, lane_live ? team_base + NEXT_LANE : lane);

    if (active) {
      const bool tz = (bz >> team_base) & TEAM_BITS;
      const bool tl = (bl >> team_base) & TEAM_BITS;
      bool done = false;
      if (tz) {                        // zombie: lateral, prevKv unchanged (Alg 4.2 l.9-11)
        cur = np;
      } else if (tl) {                 // lateral step (l.15-18)
        if (level > 0) bt = tb ? dptr : NULL_CHUNK;
        cur = np;
      } else if (level == 0) {         // bottom enclosing chunk reached (Alg 4.4 l.12)
        const bool te = (be >> team_base) & TEAM_BITS;
        if (t == 0) res[opi] = te ? 1 : 0;
        done = true;
        if (COUNT) ++nops;
      } else if (tb) {                 // down step (l.19-23)
        --level;
        bt = NULL_CHUNK;
        cur = dptr;
      } else if (bt != NULL_CHUNK) {   // backtrack (l.26-27)
        --level;
        cur = bt;
        bt = NULL_CHUNK;
      } else {                         // restart (l.25); impossible on a quiescent structure
        ++restarts;
        cur = start;
        level = height;
      }
      if (done) {
        slot += total_teams;
        active = slot < n;
        if (active) {
          opi = list[slot];
          k = keys[opi] + 1u;
          cur = start;
          level = height;
          bt = NULL_CHUNK;
        }
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

}  // namespace gfsl_dev
