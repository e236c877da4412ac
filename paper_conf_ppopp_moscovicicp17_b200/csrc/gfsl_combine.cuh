// gfsl_combine.cuh -- combining mode (R26): exact results for
// batches with ANY number of Insert/Delete ops per key.
//
// Semantics (R26): the Contains of a batch see the map before the batch (S1, R1); the
// Insert/Delete ops are then linearized in input order.  Per key this is the automaton of
// the paper's two update operations: Insert(k, v) is false iff k is present (Alg 4.5
// l.2-4; a present key's value is not overwritten), Delete(k) is false iff k is absent
// (Alg 4.11 l.3-5).  So the state before op j of a key's chain is decided by the op just
// before it in the chain alone: present after an Insert, absent after a Delete, and the
// snapshot answer (p0, from the search kernel) before the first op.
//
// Pipeline: the search kernel writes, for every op, a sort key (internal key, or all ones
// for Contains/invalid ops) and a payload {op index | p0 | Delete}; a stable radix sort by
// key (CUB; stable, so each chain stays in input order) groups the chains; combine_kernel
// then gives every Insert/Delete its result from its predecessor and, at the end of each
// chain, emits at most ONE net mutation for the update kernel:
//   p0 absent,  ends present -> Insert(k, v of the chain's last successful Insert)
//   p0 present, ends absent  -> Delete(k)
//   p0 present, ends present, with a successful Insert (after a Delete) -> value write
//   otherwise nothing.
// The net mutation reuses the search kernel's record and recorded path (searchSlow, Alg
// 4.6) of the chain's last op, which is exactly the op whose snapshot answer mutates.
// So the update kernel again sees at most one mutation per key -- the contract it relies
// on (R1, R12) -- whatever the batch.  Value writes (a key deleted and re-inserted in one
// batch) are applied after the update kernel by value_write_kernel, on a quiescent
// structure.
#pragma once
#include "gfsl_device.cuh"
#include "gfsl_search.cuh"

namespace gfsl_dev {

// One thread per sorted element.  sk/sw: the sorted keys and payloads (n elements).
// cand: the search kernel's records (and mut_of: op -> record); net: where the net
// mutations go (numbered per region in ctl->mcnt).  vw: value writes {internal key, value} (ctl->n_vw).
__global__ void __launch_bounds__(256)
combine_kernel(const BatchIn in, BatchCtl *__restrict__ ctl, const uint32_t *__restrict__ sk,
               const uint32_t *__restrict__ sw, SearchOut cand, SearchOut net, uint2 *__restrict__ vw) {
  pdl_wait();
  pdl_trigger();
  const uint32_t n = in.n;
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    const uint32_t w = sw[j];
    if (w & CW_NOTMUT) continue;  // Contains / invalid (sorted to the end)
    const uint32_t k = sk[j];
    const uint32_t i = w & OPI_MASK;
    const bool del = (w & CW_DEL) != 0, p0 = (w & CW_P0) != 0;
    const bool first = j == 0 || sk[j - 1] != k;
    const bool before = first ? p0 : !(sw[j - 1] & CW_DEL);  // present before op i
    in.res[i] = (del ? before : !before) ? 1 : 0;
    const bool last = j + 1 == n || sk[j + 1] != k;
    if (!last) {
      cand.mut_of[i] = 0xFFFFFFFFu;
      continue;
    }
    // chain end: the net effect of the whole chain
    const bool fin = !del;  // present after the chain
    uint32_t q = 0xFFFFFFFFu;
    // first op of the trailing run of Inserts (its Insert is the last successful one when
    // the key is absent before it: after a Delete, or at the chain start with p0 absent)
    uint32_t r = j;
    if (fin)
      while (r > 0 && sk[r - 1] == k && !(sw[r - 1] & CW_DEL)) --r;
    const bool run_after_delete = fin && r > 0 && sk[r - 1] == k;
    const uint32_t v_new = fin && in.vals ? in.vals[sw[r] & OPI_MASK] : 0u;
    if (p0 != fin) {  // net Insert (absent -> present) or net Delete (present -> absent)
      const uint32_t m = cand.mut_of[i];  // the last op's snapshot answer mutates: recorded
      q = mut_slot(net);
      uint4 rec = *rec_at(cand.mut_rec, m);
      if (fin) rec.w = v_new;
      rec_store(net.mut_rec, q, rec);
      const uint4 *src = reinterpret_cast<const uint4 *>(cand.plan_path + (size_t)m * PLAN_LEVELS);
      uint4 *dst = reinterpret_cast<uint4 *>(net.plan_path + (size_t)q * PLAN_LEVELS);
#pragma unroll
      for (int c = 0; c < PLAN_LEVELS / 4; ++c) dst[c] = src[c];
    } else if (p0 && fin && run_after_delete) {  // deleted and re-inserted: new value
      vw[atomicAdd(&ctl->n_vw, 1u)] = make_uint2(k, v_new);
    }
    cand.mut_of[i] = q;  // serial mode: op i -> its net mutation
  }
}

// Value writes of combining mode: after the update kernel, on a quiescent structure (the
// next batch waits for this kernel), one warp per write walks down to k's bottom chunk
// (the step rule of Alg 4.2-4.4: zombie / max < k -> lateral, highest key <= k -> down,
// none -> back through the previous chunk) and overwrites the value half of k's entry.
template <int N>
__global__ void __launch_bounds__(256)
value_write_kernel(const __grid_constant__ DevState d, const BatchCtl *__restrict__ ctl, const uint2 *__restrict__ vw) {
  pdl_wait();
  const uint32_t nvw = ctl->n_vw;
  const int t = threadIdx.x & 31;
  constexpr uint32_t FULL = 0xFFFFFFFFu;
  constexpr int DSIZE = N - 2;
  const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t warps = (gridDim.x * blockDim.x) >> 5;
  if (warp >= nvw) return;
  const int32_t cnt = t < N ? d.counter[t] : 0;
  const uint32_t hb = __ballot_sync(FULL, t >= 1 && t < N && cnt > 0);
  const int height = hb ? 31 - __clz(hb) : 0;
  for (uint32_t q = warp; q < nvw; q += warps) {
    const uint32_t k = vw[q].x, v = vw[q].y;
    int level = height;
    uint32_t cur = d.head[level], bt = NULL_CHUNK;
    for (uint32_t steps = 0;; ++steps) {
      if (steps > (1u << 24)) {
        if (t == 0) set_error(d, ERR_HANG);
        __trap();
      }
      const uint64_t e = t < N ? ld_relaxed(d.pool + (size_t)cur * N + t) : EMPTY_ENTRY;
      const uint32_t key = lo32(e);
      const uint32_t zombie = __shfl_sync(FULL, key, N - 1) == LOCK_ZOMBIE;
      const uint32_t maxk = __shfl_sync(FULL, key, N - 2);
      const uint32_t nxt = __shfl_sync(FULL, hi32(e), N - 2);
      const uint32_t vote = __ballot_sync(FULL, t < DSIZE && key <= k);
      const int top = vote ? 31 - __clz(vote) : -1;
      const uint32_t dptr = __shfl_sync(FULL, hi32(e), top < 0 ? 0 : top);
      if (zombie) {  // Alg 4.2 l.9-11
        cur = nxt;
        continue;
      }
      if (maxk < k) {  // lateral (l.15-18), keeping the way down for a backtrack
        if (level > 0) bt = top >= 0 ? dptr : bt;
        cur = nxt;
        continue;
      }
      if (level == 0) {
        const uint32_t eq = __ballot_sync(FULL, t < DSIZE && key == k);
        if (eq) {
          if (t == __ffs(eq) - 1) st_relaxed(d.pool + (size_t)cur * N + t, mk64(k, v));
        } else if (t == 0) {
          set_error(d, ERR_HANG);  // a present key must be in its enclosing chunk
        }
        break;
      }
      cur = top >= 0 ? dptr : bt;  // down step (l.19-23) or backtrack (l.24-28)
      bt = NULL_CHUNK;
      --level;
    }
  }
}

}  // namespace gfsl_dev
