// gfsl.cu -- libgfsl: the C ABI of include/gfsl.h over the sm_100a kernels.
//
// A batch is enqueued as (DESIGN.md §Batch pipeline):
//   memset(ctl) -> search_kernel (intake + B1, a2/a3) -> update_kernel (B2, a4/a5)
//   -> upkeep (-> upper-level rebuild, R24 / R29)
// with no host synchronization.  The library owns the chunk pool, the head
// array and per-level counters, the bump counters and the sticky error word; the
// caller owns the op / key / value / result arrays.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstddef>
#include <cstdlib>
#include <array>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/gfsl.h"
#include "gfsl_search.cuh"
#include "gfsl_device.cuh"
#include "gfsl_update.cuh"
#include "gfsl_ubench.cuh"
#include "gfsl_rebuild.cuh"
#include "gfsl_combine.cuh"
#include "gfsl_check.cuh"
#include "gfsl_bulk.cuh"

#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_select.cuh>

using namespace gfsl_dev;

#ifndef GFSL_DIR_CAP_LOG2
#define GFSL_DIR_CAP_LOG2 24  // level-1 directory buckets at most 2^24 (16 MiB of bytes + 2 MiB of bases)
#endif

// ------------------------------------------------------------------------------------
// errors
static thread_local std::string g_last_error = "no error";
static void set_last_error(const std::string &s) { g_last_error = s; }
extern "C" const char *gfsl_last_error(void) { return g_last_error.c_str(); }
void gfsl_internal_set_error(const std::string &s) { set_last_error(s); }  // gfsl_xroute.cu

#define CK(call)                                                                      \
  do {                                                                                \
    cudaError_t e_ = (call);                                                          \
    if (e_ != cudaSuccess) {                                                          \
      set_last_error(std::string(#call) + ": " + cudaGetErrorString(e_));             \
      return GFSL_ECUDA;                                                              \
    }                                                                                 \
  } while (0)

// Batches of up to this many ops take the small-batch kernel (GFSL_SMALL_BATCH in the
// environment at gfsl_create overrides; 0 = never).
// Measured: no gain at C1 (the time is the lock-session chain, not the kernel
// boundary), +3% at C2-5050 with a 128K threshold -- off by default.
#ifndef GFSL_NO_DERIVE_PATH
#define GFSL_DERIVE_PATH 1  // R41 (ablation: -DGFSL_NO_DERIVE_PATH)
#else
#define GFSL_DERIVE_PATH 0
#endif

#ifndef GFSL_REBUILD_MUT_RULE
#define GFSL_REBUILD_MUT_RULE 1  // R29's mutation rule (0: the ops rule alone, round 1)
#endif

#ifndef GFSL_SMALL_BATCH_DEFAULT
#define GFSL_SMALL_BATCH_DEFAULT 0
#endif

struct gfsl {
  int device = 0;
  int sms = 148;
  uint32_t N = 32;
  uint32_t team = 8;
  gfsl_config cfg{};
  uint64_t key_range = 0;
  DevState d{};
  BatchCtl *ctl = nullptr;        // the current batch's control block (one of ctl_buf)
  BatchCtl *ctl_buf[2] = {nullptr, nullptr};  // alternating by batch; the update kernel of a
  bool ctl_clean[2] = {true, true};           // batch zeroes the other one
  int ctl_cur = 0;
  uint32_t small_max = 0;  // batches of <= this many ops take the small-batch kernel (0: never)
  uint32_t small_grid = 0; // its cooperative grid (blocks that are co-resident)
  uint32_t *plan_path = nullptr, *mut_of = nullptr;
  uint4 *mut_rec = nullptr;
  uint32_t *gnext = nullptr;  // R40: [list_cap] group links of the records
  uint32_t *ghead = nullptr;  // R40: [cap_bottom] per level-0 chunk, EMPTY_GROUP between batches
  bool group_now = false;     // R40: this batch's records are grouped by chunk
  bool derive_now = false;    // R41: this batch's directory-entered records write no path
  bool idle_skip = false;     // this batch's search kernel: finished teams issue no loads
  bool derive_ok = true;      // R41 allowed (GFSL_DERIVE_PATH=0 in the environment at create: no)
  bool zc_values = false;     // host path: read Insert values zero-copy (GFSL_ZC_VALUES=1)
  uint64_t zc_batches = 0;
  uint64_t list_cap = 0;
  uint32_t *h_error = nullptr;  // mapped host memory, device alias in d.error
  cudaEvent_t last = nullptr;
  bool sticky_cuda = false;
  int contains_grid = 0, update_grid = 0;
  // staging for gfsl_batch_host(_async): two slots, so that the host->device copy of
  // batch b+1 (on the copy stream) overlaps the kernels of batch b
  uint8_t *st_op[2] = {nullptr, nullptr}, *st_res[2] = {nullptr, nullptr};
  uint32_t *st_key[2] = {nullptr, nullptr}, *st_val[2] = {nullptr, nullptr};
  uint64_t st_cap = 0;
  int st_slot = 0;
  cudaStream_t copy_stream = nullptr, exec_stream = nullptr, d2h_stream = nullptr;
  cudaEvent_t ev_in[2] = {nullptr, nullptr}, ev_used[2] = {nullptr, nullptr};
  cudaEvent_t ev_out[2] = {nullptr, nullptr};
  uint64_t batches = 0, ops = 0;
  uint64_t capacity = 0;           // max live keys (gfsl_create)
  uint64_t ops_since_rebuild = 0;  // default rebuild policy (R29)
  uint64_t ops_at_rebuild = 0;     // h->ops after the batch of the last rebuild
  unsigned long long *h_mut = nullptr;  // mapped: cumulative mutations (update kernel)
  uint64_t muts_at_rebuild = 0;    // *h_mut as known at the last rebuild
  bool upper_stale = false;        // R33: a lazy batch ran since the last rebuild
  bool upkeep_pending = false;     // R33: lazy batches skipped the upkeep sweep
  uint64_t launches = 0, lib_launches = 0;  // our kernels / CUB's (combining sort) enqueued by batches
  std::vector<std::array<cudaEvent_t, 5>> phase_ev;  // profile_phases
  // L2 persistence for the upper pool (the search kernel's access-policy window)
  size_t persist_max = 0, window_max = 0;
  uint32_t *h_bump = nullptr;  // pinned copy of the bump counters, refreshed every batch
  RebuildBufs rb{};            // upper-level rebuild (R24)
  uint32_t *rc_tiles = nullptr;  // zombie reclamation scratch (R25)
  // combining mode (R26): sort double buffers, net mutations, value writes, CUB scratch
  uint32_t *ck[2] = {nullptr, nullptr}, *cw[2] = {nullptr, nullptr};
  uint4 *net_rec = nullptr;
  uint32_t *net_path = nullptr;
  uint2 *vw = nullptr;
  void *cub_tmp = nullptr;
  size_t cub_bytes = 0;
  uint64_t comb_cap = 0;
  // key-ordered intake (R39)
  uint32_t *ko_key = nullptr, *ko_w[2] = {nullptr, nullptr};
  void *ko_tmp = nullptr;
  size_t ko_bytes = 0;
  uint64_t ko_cap = 0;
  int key_order = -1;     // GFSL_KEY_ORDER in the environment at create: 0 never, 1 always, -1 auto
  bool spread_now = false;
  bool ko_now = false;    // this batch takes the key-ordered intake (decided once per batch)
  int sort_bits = 32;
  uint32_t region_cap = 1;  // record slots per region for the current batch
  uint64_t n_policy = 0;    // ops of the current batch as counted by the rebuild policy (R29)
  uint64_t rebuilds = 0;    // upper-level rebuilds enqueued (R24): cross-batch checks reset
  uint64_t live_ub = 0;     // upper bound on the live keys (ops ever submitted), for the bulk path
  uint32_t l0_entry = 1;    // R37 (GFSL_NO_L0_ENTRY in the environment at create: 0)
  uint64_t bulk_batches = 0;
  // gfsl_check snapshot (V6 / V11)
  uint32_t *snap_max = nullptr;
  unsigned long long *snap_zh = nullptr;
  uint32_t snap_used_u = 0, snap_used_b = 0;
  uint64_t snap_rebuilds = ~0ull;
};

// ------------------------------------------------------------------------------------
// kernels: pool init

// Every pool chunk starts in the "allocated" state of P:237: all entries +inf, max +inf,
// locked.  Allocation is then only a bump of the counter.
__global__ void init_pool_kernel(uint64_t *pool, uint64_t total_entries, uint32_t N) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total_entries;
       i += (uint64_t)gridDim.x * blockDim.x) {
    pool[i] = (i % N == N - 1) ? (uint64_t)LOCK_HELD : EMPTY_ENTRY;
  }
}

// The initial structure: one unlocked chunk per level holding -inf, pointing to
// the level below; the head array points at them; counters are 0.
__global__ void init_heads_kernel(DevState d, uint32_t N) {
  const uint32_t l = threadIdx.x;
  if (l >= N) return;
  const uint32_t c = (l == 0) ? d.cap_upper : (l - 1);  // level 0 in the bottom pool
  const uint32_t below = (l == 0) ? 0u : ((l == 1) ? d.cap_upper : (l - 2));
  uint64_t *ch = d.pool + (size_t)c * N;
  ch[0] = mk64(KEY_NEG_INF, l == 0 ? 0u : below);
  ch[N - 2] = mk64(KEY_POS_INF, NULL_CHUNK);
  ch[N - 1] = mk64(LOCK_FREE, 0u);
  d.head[l] = c;
  d.counter[l] = 0;
  if (l == 0) {
    d.bump[0] = 1;
    d.bump[1] = N - 1;
  }
}

// ------------------------------------------------------------------------------------
// template dispatch

// Programmatic dependent launch between the kernels of a batch (search -> update ->
// upkeep): each is launched while its predecessor drains and waits in-kernel
// (griddepcontrol.wait) before reading its outputs.
static void set_pdl(gfsl *h, cudaLaunchAttribute &a) {
  a.id = cudaLaunchAttributeProgrammaticStreamSerialization;
  a.val.programmaticStreamSerializationAllowed = h->cfg.no_pdl ? 0 : 1;
}

// What the search kernel writes: the records of the ops whose snapshot answer mutates
// (numbered by ctl->n_mut, or by ctl->n_cand when the combine kernel picks the net ones).
static SearchOut search_out(gfsl *h) {
  const uint32_t full = h->cfg.serial_updates ? 1u : 0u;  // serial mode: traversals from the top
  if (h->cfg.combine)
    return SearchOut{h->mut_rec, h->plan_path, h->mut_of, h->ctl->ccnt, h->region_cap, h->ck[0], h->cw[0], full,
                     0u};
  return SearchOut{h->mut_rec, h->plan_path, h->cfg.serial_updates ? h->mut_of : nullptr,
                   h->ctl->mcnt, h->region_cap, nullptr, nullptr, full, h->spread_now ? 1u : 0u,
                   h->group_now ? h->ghead : nullptr, h->group_now ? h->gnext : nullptr, h->derive_now ? 1u : 0u};
}
// What the update kernel reads: the same records, or the net mutations of combining mode.
static SearchOut update_in(gfsl *h) {
  if (h->cfg.combine)
    return SearchOut{h->net_rec, h->net_path, h->mut_of, h->ctl->mcnt, h->region_cap, nullptr, nullptr, 0u,
                     1u};  // net records come out of the combining sort in key order (R31)
  return search_out(h);
}

// Record slots per region (BatchCtl::mcnt) for a batch of n ops: a region collects the
// records of the blocks b with b % MUT_REGIONS == r, of the search kernel (each block
// answers at most teams_per_block * ceil(n / teams) ops) and of the combine kernel.
static uint32_t region_cap_for(const gfsl *h, uint64_t n) {
  const uint64_t R = BatchCtl::MUT_REGIONS;
  const uint64_t tpb = (256 / 32) * (32 / h->team);
  const uint64_t teams = (uint64_t)h->contains_grid * tpb;
  const uint64_t s_cap = (((uint64_t)h->contains_grid + R - 1) / R) * tpb * ((n + teams - 1) / teams);
  const uint64_t cg = std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, (uint64_t)h->sms * 8));
  const uint64_t c_cap = ((cg + R - 1) / R) * 256 * ((n + 256 * cg - 1) / (256 * cg));
  return (uint32_t)std::max<uint64_t>(1, std::max(s_cap, c_cap));
}

// The upper levels live in one contiguous range (the upper pool, chunks [0, cap_upper)),
// so the search kernel is launched with an L2 access-policy window that marks the used
// part of it persisting (north_star: "upper levels pinned in L2").  The used size lags by
// one batch (read back asynchronously); it only steers a cache hint.
static void fill_window(gfsl *h, cudaLaunchAttribute &a) {
  a.id = cudaLaunchAttributeAccessPolicyWindow;
  // l2_window = 2: the level-1 directory only (R27; 8 B x its buckets); else the upper pool
  const bool dir = h->cfg.l2_window == 2;
  const size_t used = dir ? (size_t)h->d.dir_cap * 32 / 28
                          : (size_t)std::min(h->h_bump[1] + 64u, h->d.cap_upper) * h->N * 8;
  const size_t bytes = std::min(used, h->window_max);
  a.val.accessPolicyWindow.base_ptr = dir ? (void *)h->d.dir : (void *)h->d.pool;
  a.val.accessPolicyWindow.num_bytes = bytes;
  a.val.accessPolicyWindow.hitRatio = bytes ? std::min(1.0f, (float)h->persist_max / (float)bytes) : 0.f;
  a.val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
  a.val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
}

template <int N, int TEAM>
static void launch_contains(gfsl *h, const BatchIn &in, cudaStream_t s) {
  cudaLaunchConfig_t lc{};
  lc.gridDim = dim3(h->contains_grid);
  lc.blockDim = dim3(256);
  lc.stream = s;
  cudaLaunchAttribute attr[2];
  lc.attrs = attr;
  if (h->persist_max && h->window_max) fill_window(h, attr[lc.numAttrs++]);
  set_pdl(h, attr[lc.numAttrs++]);
  if (h->cfg.count_reads)
    cudaLaunchKernelEx(&lc, search_kernel<N, TEAM, true>, h->d, in, h->ctl, search_out(h));
  else if (h->idle_skip)  // level 0 beyond the L2: finished teams issue no loads
    cudaLaunchKernelEx(&lc, search_kernel<N, TEAM, false, true>, h->d, in, h->ctl, search_out(h));
  else
    cudaLaunchKernelEx(&lc, search_kernel<N, TEAM, false>, h->d, in, h->ctl, search_out(h));
  h->launches += 1;
}

#define GFSL_CONTAINS_CONFIGS(X) \
  X(32, 2) X(32, 4) X(32, 8) X(32, 16) X(32, 32) X(16, 1) X(16, 2) X(16, 4) X(16, 8) X(16, 16) \
  X(12, 12) X(6, 6)

static bool dispatch_contains(gfsl *h, const BatchIn &in, cudaStream_t s) {
  switch (h->N * 100 + h->team) {
#define X(n, t) case n * 100 + t: launch_contains<n, t>(h, in, s); return true;
    GFSL_CONTAINS_CONFIGS(X)
#undef X
  }
  return false;
}

// R24 (+ R25 reclamation, R27 directory): the upper-level rebuild sequence.  Its first
// kernel makes it a no-op unless a batch mutated the structure since the last one.
template <int N>
static void launch_rebuild(gfsl *h, cudaStream_t s) {
  h->upper_stale = false;  // R33: levels >= 1 re-derived from level 0
  h->rebuilds++;
  cudaLaunchConfig_t lc{};
  cudaLaunchAttribute attr[1];
  set_pdl(h, attr[0]);
  lc.attrs = attr;
  lc.numAttrs = 1;
  lc.stream = s;
  if (h->upkeep_pending) {  // R33: the zombie unlinking the lazy batches deferred
    DevState d = h->d;
    d.upkeep_force = 1;
    lc.gridDim = dim3(h->sms * 4);
    lc.blockDim = dim3(256);
    cudaLaunchKernelEx(&lc, upkeep_kernel<N>, d);
    h->launches += 1;
    h->upkeep_pending = false;
  }
  const RebuildBufs &b = h->rb;
  h->launches += 9;
  // R38: concurrent-mode rebuilds also relocate level 0 into rank order (serial mode keeps
  // the paper's layout: its pools are compared byte for byte with Oracle-B)
  const bool relocate = !h->cfg.serial_updates && h->l0_entry;
  lc.gridDim = dim3(1);
  lc.blockDim = dim3(32);
  cudaLaunchKernelEx(&lc, rebuild_begin_kernel, b);
  lc.blockDim = dim3(256);
  lc.gridDim = dim3(h->sms * 4);
  cudaLaunchKernelEx(&lc, rebuild_mark_kernel<N>, h->d, b);
  lc.gridDim = dim3(b.blocks);
  lc.blockDim = dim3(1024);
  cudaLaunchKernelEx(&lc, rebuild_scan_kernel, b);
  lc.gridDim = dim3(1);
  cudaLaunchKernelEx(&lc, rebuild_scan_top_kernel<N>, b);
  lc.blockDim = dim3(256);
  lc.gridDim = dim3(h->sms * 4);
  cudaLaunchKernelEx(&lc, rebuild_rank_kernel<N>, h->d, b);
  if (relocate) {
    lc.gridDim = dim3(h->sms * 8);
    cudaLaunchKernelEx(&lc, reloc_out_kernel<N>, h->d, b);
    cudaLaunchKernelEx(&lc, reloc_in_kernel<N>, h->d, b);
    cudaLaunchKernelEx(&lc, reloc_reset_kernel<N>, h->d, b);
    h->launches += 3;
  }
  lc.gridDim = dim3(h->sms * 8);
  cudaLaunchKernelEx(&lc, rebuild_pack_kernel<N>, h->d, b);
  // R25: reclaim the (now unreachable) zombie level-0 chunks (+ the bitmap clear)
  lc.gridDim = dim3(h->sms * 4);
  cudaLaunchKernelEx(&lc, reclaim_count_kernel<N>, h->d, b, h->rc_tiles);
  lc.gridDim = dim3(1);
  lc.blockDim = dim3(1024);
  cudaLaunchKernelEx(&lc, reclaim_scan_kernel, h->d, b, h->rc_tiles);
  lc.gridDim = dim3(h->sms * 4);
  lc.blockDim = dim3(256);
  cudaLaunchKernelEx(&lc, reclaim_write_kernel<N>, h->d, b, (const uint32_t *)h->rc_tiles);
}

// The small-batch kernel (search, grid barrier, update in one cooperative launch) for the
// default team shapes; false if this (N, team) has none.
template <int N, int TEAM>
static void launch_small_t(gfsl *h, const BatchIn &in, cudaStream_t s) {
  cudaLaunchConfig_t lc{};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  lc.attrs = attr;
  lc.numAttrs = 1;
  lc.stream = s;
  lc.blockDim = dim3(256);
  lc.gridDim = dim3(h->small_grid);
  cudaLaunchKernelEx(&lc, small_batch_kernel<N, TEAM>, h->d, in, h->ctl, search_out(h), h->ctl_buf[h->ctl_cur ^ 1]);
  h->launches += 1;
}
static bool launch_small(gfsl *h, const BatchIn &in, cudaStream_t s) {
  if (h->N == 16 && h->team == 2) launch_small_t<16, 2>(h, in, s);
  else if (h->N == 32 && h->team == 4) launch_small_t<32, 4>(h, in, s);
  else return false;
  return true;
}
template <int N, int TEAM>
static int occ_small() {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, small_batch_kernel<N, TEAM>, 256, 0);
  return b;
}

template <int N>
static void launch_update(gfsl *h, const BatchIn &in, cudaStream_t s, cudaEvent_t after_update, bool fused = false) {
  cudaLaunchConfig_t lc{};
  cudaLaunchAttribute attr[1];
  set_pdl(h, attr[0]);
  lc.attrs = attr;
  lc.numAttrs = 1;
  lc.stream = s;
  lc.blockDim = dim3(h->cfg.serial_updates ? 32 : 256);
  // a small batch needs no more warps than it has ops (2 per warp at N = 16, else 1;
  // 8 warps per block), and never fewer blocks than SMs
  const uint64_t per_block = N == 16 ? 16 : 8;
  const uint64_t need = std::max<uint64_t>((uint64_t)h->sms, (in.n + per_block - 1) / per_block);
  lc.gridDim = dim3(h->cfg.serial_updates ? 1 : (unsigned)std::min<uint64_t>((uint64_t)h->update_grid, need));
  const int serial = h->cfg.serial_updates ? 1 : 0;
  BatchCtl *next = h->ctl_buf[h->ctl_cur ^ 1];
  if (!fused) {  // (the small-batch kernel ran the update phase already)
    // eight mutations per warp for large batches, four below GFSL_UPD_SEG_SMALL_MAX ops
    // (R40: the grouped path is its own instantiation, so the default one carries none of it)
    const bool small = N == 16 && in.n < GFSL_UPD_SEG_SMALL_MAX;
    if (h->group_now)
      cudaLaunchKernelEx(&lc, small ? update_kernel<N, GFSL_UPD_SEG_SMALL, true> : update_kernel<N, GFSL_UPD_SEG, true>,
                         h->d, in, h->ctl, update_in(h), serial, next);
    else
      cudaLaunchKernelEx(&lc, small ? update_kernel<N, GFSL_UPD_SEG_SMALL, false> : update_kernel<N, GFSL_UPD_SEG, false>,
                         h->d, in, h->ctl, update_in(h), serial, next);
    h->launches += 1;  // update
  }
  h->ctl_clean[h->ctl_cur ^ 1] = true;
  lc.blockDim = dim3(256);
  if (h->cfg.combine) {  // R26: keys deleted and re-inserted in this batch get their new value
    lc.gridDim = dim3(h->sms * 2);
    cudaLaunchKernelEx(&lc, value_write_kernel<N>, h->d, (const BatchCtl *)h->ctl, (const uint2 *)h->vw);
    h->launches += 1;
  }
  if (after_update) cudaEventRecord(after_update, s);
  // upkeep (R23): after every batch, or -- lazy batches (R33) -- deferred to just before
  // the next rebuild (zombie chains at level 0 are passed laterally meanwhile); the
  // zombie marks (R30) then accumulate in one bitmap, cleared by the reclamation
#ifdef GFSL_NO_DEFER_UPKEEP  // ablation
  if (true) {
#else
  if (!h->d.lazy_upper) {
#endif
    DevState d = h->d;
    d.upkeep_force = h->upkeep_pending ? 1u : 0u;
    lc.gridDim = dim3(h->sms * 4);
    cudaLaunchKernelEx(&lc, upkeep_kernel<N>, d);
    h->launches += 1;
    h->upkeep_pending = false;
  } else {
    h->upkeep_pending = true;
  }
  // R24 / R29: rebuild the upper levels from level 0 -- by default after the batch at
  // which the ops since the last rebuild reach GFSL_REBUILD_DEFAULT_WEAR x L, where L =
  // min(capacity, ops ever submitted up to the last rebuild) bounds the live keys from
  // above (so a structure growing from empty is rebuilt at geometrically spaced sizes);
  // else after every `rebuild_every`-th batch
  bool rebuild;
  if (h->cfg.rebuild_every == 0) {
    h->ops_since_rebuild += h->n_policy;
    const uint64_t L = std::min(h->capacity, h->ops_at_rebuild);
    rebuild = 2 * h->ops_since_rebuild >= (uint64_t)(2 * GFSL_REBUILD_DEFAULT_WEAR) * L;
    // and the structure must have worn: successful mutations since the last rebuild >= L/2
    // (the device's count, read from mapped memory, a batch or two behind).  Both rules
    // cross together at the paper's [10,10,80] mix; a Contains-heavy mix rebuilds far less
    // often (M1-1-98: every ~80 batches instead of 8); a map growing from empty keeps the ops
    // rule (every op mutates).  Not in serial mode: its rule must stay deterministic (host
    // counts only), since its pools are compared byte for byte with Oracle-B's
    if (GFSL_REBUILD_MUT_RULE && rebuild && !h->cfg.serial_updates) {
      const uint64_t muts = *(volatile unsigned long long *)h->h_mut - h->muts_at_rebuild;
      rebuild = 2 * muts >= L;
    }
  } else {
    rebuild = h->cfg.rebuild_every != GFSL_REBUILD_NEVER && (h->batches + 1) % h->cfg.rebuild_every == 0;
  }
  if (rebuild) {
    h->ops_since_rebuild = 0;
    h->ops_at_rebuild = h->ops + h->n_policy;
    h->muts_at_rebuild = *(volatile unsigned long long *)h->h_mut;
    launch_rebuild<N>(h, s);
  }
}

template <int N, int TEAM>
static int occ_contains() {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, search_kernel<N, TEAM, false>, 256, 0);
  return b;
}
template <int N>
static int occ_update() {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, update_kernel<N>, 256, 0);
  return b;
}

static bool valid_team(uint32_t N, uint32_t team) {
  switch (N * 100 + team) {
#define X(n, t) case n * 100 + t: return true;
    GFSL_CONTAINS_CONFIGS(X)
#undef X
  }
  return false;
}

static int contains_occupancy(uint32_t N, uint32_t team) {
  switch (N * 100 + team) {
#define X(n, t) case n * 100 + t: return occ_contains<n, t>();
    GFSL_CONTAINS_CONFIGS(X)
#undef X
  }
  return 1;
}
static int update_occupancy(uint32_t N) {
  switch (N) {
    case 32: return occ_update<32>();
    case 16: return occ_update<16>();
    case 12: return occ_update<12>();
    case 6: return occ_update<6>();
  }
  return 1;
}

// ------------------------------------------------------------------------------------
// create / destroy

// Opt-in (cfg.l2_window): reserve the device's persisting-L2 carve-out for the upper
// pool.  Measured on B200: no gain for the search kernel, which is bound
// by the L1 data pipe, and a slower update kernel (the carve-out shrinks its L2), so the
// default is off.
static void setup_l2_window(gfsl *h) {
  h->persist_max = h->window_max = 0;
  if (!h->cfg.l2_window) return;
  int pmax = 0, wmax = 0;
  cudaDeviceGetAttribute(&pmax, cudaDevAttrMaxPersistingL2CacheSize, h->device);
  cudaDeviceGetAttribute(&wmax, cudaDevAttrMaxAccessPolicyWindowSize, h->device);
  if (pmax > 0 && wmax > 0) {
    size_t cur = 0;
    cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
    if (cur < (size_t)pmax) cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)pmax);
    cudaDeviceGetLimit(&cur, cudaLimitPersistingL2CacheSize);
    h->persist_max = cur;
    h->window_max = (size_t)wmax;
  }
  cudaGetLastError();
}

static void apply_launch_shape(gfsl *h) {
  {
    int bs = 0;
    if (h->N == 16 && h->team == 2) bs = occ_small<16, 2>();
    else if (h->N == 32 && h->team == 4) bs = occ_small<32, 4>();
    h->small_grid = (uint32_t)(h->sms * std::min(bs, 4));
  }
  int bc = contains_occupancy(h->N, h->team);
  if (h->cfg.contains_blocks_per_sm) bc = std::min<int>(bc, h->cfg.contains_blocks_per_sm);
  int bu = update_occupancy(h->N);
  if (h->cfg.update_blocks_per_sm) bu = std::min<int>(bu, h->cfg.update_blocks_per_sm);
  h->contains_grid = h->sms * std::max(1, bc);
  h->update_grid = h->sms * std::max(1, bu);
}

static void free_all(gfsl *h) {
  if (!h) return;
  cudaFree(h->d.pool);
  cudaFree(h->d.head);
  cudaFree(h->d.counter);
  cudaFree(h->d.bump);
  cudaFree(h->d.stats);
  cudaFree(h->ctl_buf[0]);
  cudaFree(h->plan_path);
  cudaFree(h->mut_of);
  cudaFree(h->mut_rec);
  cudaFree(h->gnext);
  cudaFree(h->ghead);
  for (int b = 0; b < 2; ++b) {
    cudaFree(h->st_op[b]);
    cudaFree(h->st_res[b]);
    cudaFree(h->st_key[b]);
    cudaFree(h->st_val[b]);
    if (h->ev_in[b]) cudaEventDestroy(h->ev_in[b]);
    if (h->ev_used[b]) cudaEventDestroy(h->ev_used[b]);
    if (h->ev_out[b]) cudaEventDestroy(h->ev_out[b]);
  }
  if (h->copy_stream) cudaStreamDestroy(h->copy_stream);
  if (h->exec_stream) cudaStreamDestroy(h->exec_stream);
  if (h->d2h_stream) cudaStreamDestroy(h->d2h_stream);
  cudaFree(h->rb.bitmap);
  cudaFree(h->rb.word_prefix);
  cudaFree(h->rb.block_sum);
  cudaFree(h->rb.order_key);
  cudaFree(h->rb.order_chunk);
  cudaFree(h->rb.n1);
  cudaFree(h->rb.levels);
  cudaFree(h->rc_tiles);
  for (int b = 0; b < 2; ++b) {
    cudaFree(h->ck[b]);
    cudaFree(h->cw[b]);
  }
  cudaFree(h->net_rec);
  cudaFree(h->net_path);
  cudaFree(h->vw);
  cudaFree(h->cub_tmp);
  cudaFree(h->ko_key);
  cudaFree(h->ko_w[0]);
  cudaFree(h->ko_w[1]);
  cudaFree(h->ko_tmp);
  cudaFree(h->d.freelist);
  cudaFree(h->d.zbits);
  cudaFree(h->d.fl);
  cudaFree(h->d.dir);
  cudaFree(h->d.dir_base);
  cudaFree(h->d.dir_hdr);
  cudaFree(h->snap_max);
  cudaFree(h->snap_zh);
  if (h->h_error) cudaFreeHost(h->h_error);
  if (h->h_bump) cudaFreeHost(h->h_bump);
  if (h->h_mut) cudaFreeHost(h->h_mut);
  if (h->last) cudaEventDestroy(h->last);
  for (auto &ev : h->phase_ev)
    for (auto &e : ev) cudaEventDestroy(e);
  delete h;
}

static gfsl_status ensure_lists(gfsl *h, uint64_t n);

extern "C" gfsl_t gfsl_create_ex(uint64_t key_range, uint64_t capacity, const gfsl_config *cfg_in) {
  gfsl_config cfg{};
  if (cfg_in) cfg = *cfg_in;
  if (cfg.chunk_entries == 0) cfg.chunk_entries = 16;  // B200 default
  const uint32_t N = cfg.chunk_entries;
  if (N != 32 && N != 16 && N != 12 && N != 6) {
    set_last_error("chunk_entries must be 6, 12, 16 or 32");
    return nullptr;
  }
  if (key_range == 0 || key_range > 0xFFFFFFFEull) {
    set_last_error("key_range must be in [1, 2^32-2]");
    return nullptr;
  }
  if (capacity == 0) capacity = key_range;
  if (cfg.contains_team == 0) cfg.contains_team = (N == 32) ? 4 : (N == 16) ? 2 : N;
  if (!valid_team(N, cfg.contains_team)) {
    set_last_error("unsupported contains_team for this chunk size");
    return nullptr;
  }
  gfsl *h = new gfsl();
  h->N = N;
  h->team = cfg.contains_team;
  h->cfg = cfg;
  h->key_range = key_range;
  h->capacity = capacity;
  {
    const char *e = getenv("GFSL_NO_L0_ENTRY");
    h->l0_entry = (e && *e && *e != '0') ? 0u : 1u;
    const char *ko = getenv("GFSL_KEY_ORDER");
    h->key_order = ko && *ko ? atoi(ko) : -1;
    const char *zc = getenv("GFSL_ZC_VALUES");
    h->zc_values = zc && *zc == '1';
    const char *dp = getenv("GFSL_DERIVE_PATH");
    h->derive_ok = !(dp && *dp == '0');
    const char *sb = getenv("GFSL_SMALL_BATCH");  // ops; 0 = never (default GFSL_SMALL_BATCH_DEFAULT)
    h->small_max = sb && *sb ? (uint32_t)atoi(sb) : (uint32_t)GFSL_SMALL_BATCH_DEFAULT;
  }
  auto fail = [&](const char *what, cudaError_t e) -> gfsl_t {
    set_last_error(std::string(what) + ": " + cudaGetErrorString(e));
    free_all(h);
    return nullptr;
  };
  cudaError_t e;
  if ((e = cudaGetDevice(&h->device)) != cudaSuccess) return fail("cudaGetDevice", e);
  cudaDeviceGetAttribute(&h->sms, cudaDevAttrMultiProcessorCount, h->device);

  // Pool sizing (R18): bottom = 2x the hard bound on live level-0 chunks
  // ((capacity+1)/floor(DSIZE/3) + 1, from V13) plus slack; upper = bottom/8.
  const uint64_t DS = N - 2;
  const uint64_t m = std::max<uint64_t>(1, DS / 3);
  uint64_t cap_b = 2 * ((capacity + 1) / m + 1) + 64;
  uint64_t cap_u = cap_b / 8 + 2 * N + 64;
  if (cap_b + cap_u >= (1ull << 30)) {  // 30-bit indices: two flag bits ride on shuffles
    free_all(h);
    set_last_error("capacity too large for 30-bit chunk indices");
    return nullptr;
  }
  h->d.cap_bottom = (uint32_t)cap_b;
  h->d.cap_upper = (uint32_t)cap_u;
  h->d.key_max = (uint32_t)key_range;
  h->d.p_chunk_q32 = cfg.p_chunk_q32;
  const uint64_t total_entries = (cap_b + cap_u) * N;
  if ((e = cudaMalloc(&h->d.pool, total_entries * 8)) != cudaSuccess) return fail("cudaMalloc(pool)", e);
  if ((e = cudaMalloc(&h->d.head, 32 * 4)) != cudaSuccess) return fail("cudaMalloc", e);
  if ((e = cudaMalloc(&h->d.counter, 32 * 4)) != cudaSuccess) return fail("cudaMalloc", e);
  if ((e = cudaMalloc(&h->d.bump, 2 * 4)) != cudaSuccess) return fail("cudaMalloc", e);
  if ((e = cudaMalloc(&h->d.stats, ST_NSTATS * 8)) != cudaSuccess) return fail("cudaMalloc", e);
  if ((e = cudaMalloc(&h->ctl_buf[0], 2 * sizeof(BatchCtl))) != cudaSuccess) return fail("cudaMalloc", e);
  cudaMemset(h->ctl_buf[0], 0, 2 * sizeof(BatchCtl));
  h->ctl_buf[1] = h->ctl_buf[0] + 1;
  h->ctl = h->ctl_buf[0];
  h->d.ctl = h->ctl;
  if ((e = cudaHostAlloc(&h->h_error, 4, cudaHostAllocMapped)) != cudaSuccess) return fail("cudaHostAlloc", e);
  *h->h_error = 0;
  if ((e = cudaHostGetDevicePointer(&h->d.error, h->h_error, 0)) != cudaSuccess) return fail("cudaHostGetDevicePointer", e);
  if ((e = cudaEventCreateWithFlags(&h->last, cudaEventDisableTiming)) != cudaSuccess) return fail("cudaEventCreate", e);
  if ((e = cudaHostAlloc(&h->h_bump, 8, cudaHostAllocMapped)) != cudaSuccess) return fail("cudaHostAlloc", e);
  h->h_bump[0] = 1;
  h->h_bump[1] = N - 1;
  if ((e = cudaHostGetDevicePointer(&h->d.bump_host, h->h_bump, 0)) != cudaSuccess) return fail("cudaHostGetDevicePointer", e);
  if ((e = cudaHostAlloc(&h->h_mut, 8, cudaHostAllocMapped)) != cudaSuccess) return fail("cudaHostAlloc", e);
  *h->h_mut = 0;
  if ((e = cudaHostGetDevicePointer(&h->d.mut_host, h->h_mut, 0)) != cudaSuccess) return fail("cudaHostGetDevicePointer", e);
  setup_l2_window(h);
  {
    RebuildBufs &b = h->rb;
    b.words = (uint32_t)((key_range + 2 + 31) / 32);
    b.blocks = (b.words + RB_BLOCK_WORDS - 1) / RB_BLOCK_WORDS;
    b.fill = N - 4;  // leaves 2 free DATA slots per rebuilt chunk for later raises
    if ((e = cudaMalloc(&b.bitmap, (size_t)b.words * 4)) != cudaSuccess) return fail("cudaMalloc(rebuild)", e);
    if ((e = cudaMalloc(&b.word_prefix, (size_t)b.words * 4)) != cudaSuccess) return fail("cudaMalloc(rebuild)", e);
    if ((e = cudaMalloc(&b.block_sum, (size_t)b.blocks * 4)) != cudaSuccess) return fail("cudaMalloc(rebuild)", e);
    if ((e = cudaMalloc(&b.order_key, ((size_t)cap_b + 16) * 4)) != cudaSuccess) return fail("cudaMalloc(rebuild)", e);  // + the search kernel's look-ahead (R38)
    if ((e = cudaMalloc(&b.order_chunk, (size_t)cap_b * 4)) != cudaSuccess) return fail("cudaMalloc(rebuild)", e);
    if ((e = cudaMalloc(&b.n1, 32)) != cudaSuccess) return fail("cudaMalloc(rebuild)", e);
    if ((e = cudaMalloc(&b.levels, sizeof(RbLevels))) != cudaSuccess) return fail("cudaMalloc(rebuild)", e);
    cudaMemset(b.bitmap, 0, (size_t)b.words * 4);
    cudaMemset(b.n1, 0, 32);
    h->d.dirty = b.n1 + 2;
    h->d.dir_oc = b.order_chunk;
    h->d.dir_ok = b.order_key;
    if ((e = cudaMalloc(&h->d.freelist, (size_t)cap_b * 8)) != cudaSuccess) return fail("cudaMalloc(freelist)", e);
    if ((e = cudaMalloc(&h->ghead, (size_t)cap_b * 4)) != cudaSuccess) return fail("cudaMalloc(ghead)", e);  // R40
    cudaMemset(h->ghead, 0xFF, (size_t)cap_b * 4);
    if ((e = cudaMalloc(&h->d.fl, 8 * 4)) != cudaSuccess) return fail("cudaMalloc(freelist)", e);
    if ((e = cudaMalloc(&h->rc_tiles, ((size_t)cap_b / RC_TILE + 2) * 4)) != cudaSuccess) return fail("cudaMalloc(reclaim)", e);
    cudaMemset(h->d.fl, 0, 8 * 4);
    // R27 / R27b: level-1 directory, about four buckets per level-1 key, at most
    // 2^GFSL_DIR_CAP_LOG2: one byte per bucket plus one 32-bit base per 32 buckets
    uint32_t dcap = 1024;
    while (dcap < (1u << GFSL_DIR_CAP_LOG2) && (uint64_t)dcap < key_range + 1) dcap <<= 1;
    {  // tests: a smaller directory (GFSL_DIR_CAP buckets, a power of two >= 1024) forces
       // the coarse-directory path (C5's 8-key min-key window) on small structures
      const char *dc = getenv("GFSL_DIR_CAP");
      if (dc && *dc) dcap = std::min<uint32_t>(dcap, std::max<uint32_t>(1024u, (uint32_t)atoi(dc)));
    }
    h->d.dir_cap = dcap;
#ifdef GFSL_DIR_U32
    if ((e = cudaMalloc(&h->d.dir, (size_t)dcap * 4)) != cudaSuccess) return fail("cudaMalloc(dir)", e);
#else  // room for either layout (R27b split, R27c sector; the rebuild chooses)
    if ((e = cudaMalloc(&h->d.dir, std::max<size_t>(dcap, ((size_t)dcap / DIR_SEC_BUCKETS + 2) * 32))) != cudaSuccess)
      return fail("cudaMalloc(dir)", e);
#endif
    if ((e = cudaMalloc(&h->d.dir_base, (size_t)dcap / 32 * 4)) != cudaSuccess) return fail("cudaMalloc(dir)", e);
    if ((e = cudaMalloc(&h->d.dir_hdr, 64 * 4)) != cudaSuccess) return fail("cudaMalloc(dir)", e);
    cudaMemset(h->d.dir_hdr, 0, 64 * 4);
    // R30: zombie marks, two bitmaps over every chunk index
    h->d.zwords = (uint32_t)(((uint64_t)h->d.cap_upper + h->d.cap_bottom + 31) / 32);
    if ((e = cudaMalloc(&h->d.zbits, (size_t)h->d.zwords * 8)) != cudaSuccess) return fail("cudaMalloc(zbits)", e);
    cudaMemset(h->d.zbits, 0, (size_t)h->d.zwords * 8);
#ifdef GFSL_DEBUG_TIMING
    if ((e = cudaMalloc(&h->d.debug_times, ((size_t)148 * 64 * 48 + 64) * 8)) != cudaSuccess) return fail("cudaMalloc", e);
    cudaMemset(h->d.debug_times, 0, ((size_t)148 * 64 * 48 + 64) * 8);
#endif
  }
  cudaMemset(h->d.head, 0xFF, 32 * 4);
  cudaMemset(h->d.counter, 0, 32 * 4);
  cudaMemset(h->d.stats, 0, ST_NSTATS * 8);
  init_pool_kernel<<<h->sms * 8, 256>>>(h->d.pool, total_entries, N);
  init_heads_kernel<<<1, 32>>>(h->d, N);
  if ((e = cudaGetLastError()) != cudaSuccess) return fail("init kernels", e);
  if ((e = cudaDeviceSynchronize()) != cudaSuccess) return fail("init sync", e);

  apply_launch_shape(h);
  // The per-batch lists for batches of up to min(capacity, 2^21) ops, and a stream-ordered
  // pool that keeps what the bulk path frees (no OS round trip per bulk batch): neither a
  // handle's first batches nor its bulk batches allocate inside a caller's timed region.
  if (ensure_lists(h, std::min<uint64_t>(capacity, 1ull << 21)) != GFSL_OK) {
    free_all(h);
    return nullptr;
  }
  {
    cudaMemPool_t mp;
    if (cudaDeviceGetDefaultMemPool(&mp, h->device) == cudaSuccess) {
      uint64_t thr = ~0ull;
      cudaMemPoolSetAttribute(mp, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    cudaGetLastError();
  }
  return h;
}

extern "C" gfsl_t gfsl_create(uint64_t key_range, uint64_t capacity) {
  return gfsl_create_ex(key_range, capacity, nullptr);
}

extern "C" gfsl_status gfsl_configure(gfsl_t h, const gfsl_config *cfg) {
  if (!h || !cfg) return GFSL_EINVAL;
  if (cfg->chunk_entries != 0 && cfg->chunk_entries != h->N) {
    set_last_error("gfsl_configure: chunk_entries cannot change");
    return GFSL_EINVAL;
  }
  const uint32_t team = cfg->contains_team ? cfg->contains_team : (h->N == 32 ? 4 : h->N == 16 ? 2 : h->N);
  if (!valid_team(h->N, team)) {
    set_last_error("gfsl_configure: unsupported contains_team");
    return GFSL_EINVAL;
  }
  h->cfg = *cfg;
  h->cfg.chunk_entries = h->N;
  h->d.p_chunk_q32 = cfg->p_chunk_q32;
  h->cfg.contains_team = team;
  h->team = team;
  apply_launch_shape(h);
  setup_l2_window(h);
  return GFSL_OK;
}

extern "C" void gfsl_destroy(gfsl_t h) {
  if (!h) return;
  cudaDeviceSynchronize();
  free_all(h);
}

// bits of the combining sort: internal keys are in [1, key_range]; the all-ones key of
// Contains / invalid ops must compare above every real key within the sorted bits
static int sort_bits_for(uint64_t key_range) {
  int b = 1;
  while (b < 32 && (1ull << b) - 1 <= key_range) ++b;
  return b;
}

// ------------------------------------------------------------------------------------
// batch

static gfsl_status sticky(gfsl *h) {
  if (h->sticky_cuda) return GFSL_ECUDA;
  const uint32_t e = *(volatile uint32_t *)h->h_error;
  if (e & ERR_POOL) {
    set_last_error("chunk pool exhausted (sticky)");
    return GFSL_EPOOL;
  }
  if (e & ERR_HANG) {
    set_last_error("device watchdog fired: structure corrupt (sticky)");
    h->sticky_cuda = true;
    return GFSL_ECUDA;
  }
  return GFSL_OK;
}

static gfsl_status ensure_lists(gfsl *h, uint64_t n) {
  h->region_cap = region_cap_for(h, n);
  // mut_of is indexed by op; records and paths by region slot
  n = std::max<uint64_t>(n, (uint64_t)BatchCtl::MUT_REGIONS * h->region_cap);
  if (n <= h->list_cap) return GFSL_OK;
  cudaDeviceSynchronize();
  cudaFree(h->plan_path);
  cudaFree(h->mut_of);
  cudaFree(h->mut_rec);
  cudaFree(h->gnext);
  h->plan_path = nullptr;
  h->mut_of = nullptr;
  h->mut_rec = nullptr;
  h->gnext = nullptr;
  h->list_cap = 0;
  const uint64_t cap = std::max<uint64_t>(n, 1024);
  CK(cudaMalloc(&h->plan_path, cap * 4 * PLAN_LEVELS));
  CK(cudaMalloc(&h->mut_of, cap * 4));
  CK(cudaMalloc(&h->mut_rec, cap * 16 * REC_STRIDE));
  CK(cudaMalloc(&h->gnext, cap * 4));
  h->list_cap = cap;
  return GFSL_OK;
}

// Combining-mode buffers (R26), grown on demand like the lists.
static gfsl_status ensure_combine(gfsl *h, uint64_t n) {
  h->sort_bits = sort_bits_for(h->key_range);
  const uint64_t n_sort = n;
  n = std::max<uint64_t>(n, (uint64_t)BatchCtl::MUT_REGIONS * h->region_cap);  // net records
  size_t need = 0;
  {
    cub::DoubleBuffer<uint32_t> kb(nullptr, nullptr), vb(nullptr, nullptr);
    CK(cub::DeviceRadixSort::SortPairs(nullptr, need, kb, vb, (int)std::max<uint64_t>(n_sort, h->comb_cap), 0, h->sort_bits));
  }
  if (n <= h->comb_cap && need <= h->cub_bytes) return GFSL_OK;
  cudaDeviceSynchronize();
  if (n > h->comb_cap) {
    for (int b = 0; b < 2; ++b) {
      cudaFree(h->ck[b]);
      cudaFree(h->cw[b]);
      h->ck[b] = h->cw[b] = nullptr;
    }
    cudaFree(h->net_rec);
    cudaFree(h->net_path);
    cudaFree(h->vw);
    h->net_rec = nullptr;
    h->net_path = nullptr;
    h->vw = nullptr;
    h->comb_cap = 0;
    const uint64_t cap = std::max<uint64_t>(n, 1024);
    for (int b = 0; b < 2; ++b) {
      CK(cudaMalloc(&h->ck[b], cap * 4));
      CK(cudaMalloc(&h->cw[b], cap * 4));
    }
    CK(cudaMalloc(&h->net_rec, cap * 16 * REC_STRIDE));
    CK(cudaMalloc(&h->net_path, cap * 4 * PLAN_LEVELS));
    CK(cudaMalloc(&h->vw, cap * 8));
    h->comb_cap = cap;
  }
  if (need > h->cub_bytes) {
    cudaFree(h->cub_tmp);
    h->cub_tmp = nullptr;
    h->cub_bytes = 0;
    CK(cudaMalloc(&h->cub_tmp, need));
    h->cub_bytes = need;
  }
  return GFSL_OK;
}

// ---- key-ordered intake (R39) ----
// With level 0 in key order (R38), ops taken in key order make the search phase's chunk
// gathers walk level 0 (and the sorted min keys, the directory) nearly sequentially: the
// teams in flight at one time cover a narrow key window, so chunks are shared in L1/L2 and
// DRAM sees near-sequential rows instead of random ones.  The intake sorts (key, op index)
// on the key's top 16 bits (CUB onesweep, 2 passes); results still go to the input order.
// Measured in one gpurun call (R39): the sort costs more than the locality saves
// (C5 7670 -> 7019, C4-16 15598 -> 12826 Mops/s), so it is off unless GFSL_KEY_ORDER=1 is in
// the environment at gfsl_create; never in serial / combining mode or for device counts.
static bool use_key_order(const gfsl *h, uint64_t n) {
  if (h->cfg.serial_updates || h->cfg.combine || n == 0) return false;
  return h->key_order == 1;
}
static void key_order_bits(const gfsl *h, int &lo, int &hi) {
  hi = 1;
  while (hi < 32 && (1ull << hi) < h->key_range) ++hi;
  lo = std::max(0, hi - 16);
}
static gfsl_status ensure_key_order(gfsl *h, uint64_t n) {
  h->ko_now = use_key_order(h, n);
  if (!h->ko_now) return GFSL_OK;
  int lo, hi;
  key_order_bits(h, lo, hi);
  size_t need = 0;
  CK(cub::DeviceRadixSort::SortPairs(nullptr, need, (const uint32_t *)nullptr, (uint32_t *)nullptr,
                                     (const uint32_t *)nullptr, (uint32_t *)nullptr,
                                     (int)std::max<uint64_t>(n, h->ko_cap), lo, hi));
  if (n <= h->ko_cap && need <= h->ko_bytes) return GFSL_OK;
  cudaDeviceSynchronize();
  if (n > h->ko_cap) {
    cudaFree(h->ko_key);
    cudaFree(h->ko_w[0]);
    cudaFree(h->ko_w[1]);
    h->ko_key = h->ko_w[0] = h->ko_w[1] = nullptr;
    h->ko_cap = 0;
    CK(cudaMalloc(&h->ko_key, n * 4));
    CK(cudaMalloc(&h->ko_w[0], n * 4));
    CK(cudaMalloc(&h->ko_w[1], n * 4));
    h->ko_cap = n;
  }
  if (need > h->ko_bytes) {
    cudaFree(h->ko_tmp);
    h->ko_tmp = nullptr;
    h->ko_bytes = 0;
    CK(cudaMalloc(&h->ko_tmp, need));
    h->ko_bytes = need;
  }
  return GFSL_OK;
}
// the sort's payload: op index | op code (capped at 3 = invalid) << 29
__global__ void key_order_pack_kernel(const uint8_t *ops, uint32_t n, uint32_t *w) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    w[i] = i | ((uint32_t)min(ops[i], (uint8_t)3) << 29);
}
static gfsl_status enqueue_key_order(gfsl *h, BatchIn &in, cudaStream_t s) {
  int lo, hi;
  key_order_bits(h, lo, hi);
  const int grid = (int)std::min<uint64_t>((in.n + 255) / 256, (uint64_t)h->sms * 8);
  key_order_pack_kernel<<<grid, 256, 0, s>>>(in.ops, in.n, h->ko_w[0]);
  h->launches += 1;
  size_t bytes = h->ko_bytes;
  CK(cub::DeviceRadixSort::SortPairs(h->ko_tmp, bytes, in.keys, h->ko_key, h->ko_w[0], h->ko_w[1],
                                     (int)in.n, lo, hi, s));
  h->lib_launches += 1 + (uint64_t)(hi - lo + 7) / 8;  // onesweep: histogram + one pass per digit
  in.skey = h->ko_key;
  in.sw = h->ko_w[1];
  return GFSL_OK;
}

// R26: sort the batch's (key, op) pairs so that each key's Insert/Delete chain is
// contiguous and in input order (LSD radix sort is stable), then reduce the chains.
static gfsl_status enqueue_combine(gfsl *h, const BatchIn &in, cudaStream_t s) {
  cub::DoubleBuffer<uint32_t> kb(h->ck[0], h->ck[1]), vb(h->cw[0], h->cw[1]);
  size_t bytes = h->cub_bytes;
  CK(cub::DeviceRadixSort::SortPairs(h->cub_tmp, bytes, kb, vb, (int)in.n, 0, h->sort_bits, s));
  h->lib_launches += 1 + (uint64_t)(h->sort_bits + 7) / 8;  // onesweep: histogram + one pass per 8-bit digit
  h->launches += 1;  // combine_kernel
  cudaLaunchConfig_t lc{};
  cudaLaunchAttribute attr[1];
  set_pdl(h, attr[0]);
  lc.attrs = attr;
  lc.numAttrs = 1;
  lc.stream = s;
  lc.blockDim = dim3(256);
  lc.gridDim = dim3((unsigned)std::min<uint64_t>((in.n + 255) / 256, (uint64_t)h->sms * 8));
  CK(cudaLaunchKernelEx(&lc, combine_kernel, in, h->ctl, (const uint32_t *)kb.Current(),
                        (const uint32_t *)vb.Current(), search_out(h), update_in(h), h->vw));
  return GFSL_OK;
}

static gfsl_status enqueue_batch(gfsl *h, const uint8_t *ops, const uint32_t *keys,
                                 const uint32_t *vals, uint8_t *res, uint64_t n, cudaStream_t s,
                                 const uint32_t *n_dev = nullptr, uint64_t n_policy = 0) {
  CK(cudaStreamWaitEvent(s, h->last, 0));
  {
    // R36: level-0 loads evict_first, except when level 0 spills the L2 while the upper
    // levels fit it (C4-like: measured 4% slower with the hint; C3 +11%, C5 +3%).  Sizes
    // from the bump counters of the previous batch (pinned copy; a heuristic only).
    const double l2 = 126.0 * (1 << 20);
    const double l0 = (double)h->h_bump[0] * h->N * 8, up = (double)h->h_bump[1] * h->N * 8;
#ifdef GFSL_L0_EVICT_FIRST_ALWAYS
    h->d.l0_evict_first = 1u;
    (void)up;
#else
    h->d.l0_evict_first = (l0 > l2 && up <= l2) ? 0u : 1u;
#endif
    h->idle_skip = l0 > l2;
    h->d.upd_prefetch = l0 > l2 ? 0u : 1u;
  }
  // R37: enter level 0 straight from the directory (Contains, and the Insert/Delete of lazy
  // batches); GFSL_NO_L0_ENTRY (environment, read at gfsl_create) keeps R27's level-1 entry
  h->d.l0_entry = h->l0_entry;
  h->n_policy = n_dev ? n_policy : n;
  h->d.zparity = (uint32_t)(h->batches & 1);  // R30: this batch's zombie-mark bitmap
#ifdef GFSL_NO_LAZY_UPPER  // ablation
  h->d.lazy_upper = 0;
#else
  h->d.lazy_upper = (!h->cfg.serial_updates && h->cfg.rebuild_every != GFSL_REBUILD_NEVER) ? 1u : 0u;  // R33
#endif
  if (h->d.lazy_upper) {
    h->upper_stale = true;
    h->d.zparity = 0;  // R33: the marks of all lazy batches since the last rebuild
  }
  // R40: chunk-grouped mutations in lazy concurrent batches (the update paths that take
  // them: update_multi at N = 16 / 32)
  h->group_now = h->d.lazy_upper && !h->cfg.combine && !h->cfg.serial_updates && h->cfg.group == GFSL_GROUP_ON &&
                 (h->N == 16 || h->N == 32) && GFSL_UPD_SEG != 16 && GFSL_UPD_SEG_SMALL != 16;
  // R41: the update paths that derive a record's path (update_multi at N = 16 / 32)
  h->derive_now = GFSL_DERIVE_PATH && h->derive_ok && h->d.lazy_upper && !h->cfg.combine && !h->cfg.serial_updates &&
                  (h->N == 16 || h->N == 32) && GFSL_UPD_SEG != 16 && GFSL_UPD_SEG_SMALL != 16;
  std::array<cudaEvent_t, 5> ev{};
  const bool prof = h->cfg.profile_phases != 0;
  if (prof) {
    for (auto &e : ev) CK(cudaEventCreate(&e));
    CK(cudaEventRecord(ev[0], s));
  }
  {
    const int cur = h->ctl_cur;
    h->ctl = h->ctl_buf[cur];
    h->d.ctl = h->ctl;
    // normally zeroed by the previous batch's update kernel; after a failed batch, here
    if (!h->ctl_clean[cur]) CK(cudaMemsetAsync(h->ctl, 0, sizeof(BatchCtl), s));
    h->ctl_clean[cur] = false;
  }
  if (prof) CK(cudaEventRecord(ev[1], s));
  BatchIn in{ops, keys, vals, res, (uint32_t)n, h->key_range, n_dev, nullptr, nullptr};
  {
    const bool ko = !n_dev && h->ko_now;
    const char *sp = getenv("GFSL_KO_SPREAD");
    h->spread_now = ko && sp && *sp == '1';
    if (ko) {
      gfsl_status ks = enqueue_key_order(h, in, s);
      if (ks != GFSL_OK) return ks;
    }
  }
  // small batches: search + barrier + update in one cooperative kernel
  const bool fused = !h->cfg.serial_updates && !h->cfg.combine && !h->cfg.count_reads && !h->ko_now && !n_dev &&
                     !h->group_now &&
                     h->small_grid && n <= h->small_max && launch_small(h, in, s);
  bool ok = fused || dispatch_contains(h, in, s);
  if (!ok) {
    set_last_error("no contains kernel for this (N, team)");
    return GFSL_EINVAL;
  }
  if (h->cfg.combine) {
    gfsl_status cs = enqueue_combine(h, in, s);
    if (cs != GFSL_OK) return cs;
  }
  if (prof) CK(cudaEventRecord(ev[2], s));
  switch (h->N) {
    case 32: launch_update<32>(h, in, s, prof ? ev[3] : nullptr, fused); break;
    case 16: launch_update<16>(h, in, s, prof ? ev[3] : nullptr, fused); break;
    case 12: launch_update<12>(h, in, s, prof ? ev[3] : nullptr, fused); break;
    case 6: launch_update<6>(h, in, s, prof ? ev[3] : nullptr, fused); break;
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    h->sticky_cuda = true;
    set_last_error(std::string("kernel launch: ") + cudaGetErrorString(e));
    return GFSL_ECUDA;
  }
  if (prof) {
    CK(cudaEventRecord(ev[4], s));
    h->phase_ev.push_back(ev);
  }
  CK(cudaEventRecord(h->last, s));
  h->ctl_cur ^= 1;
  h->batches++;
  h->ops += h->n_policy;
  h->live_ub = std::min(h->capacity, h->live_ub + n);
  return GFSL_OK;
}

// ------------------------------------------------------------------------------------
// the bulk path (gfsl_bulk.cuh, R34): a batch much larger than the structure

struct MaxU32 {  // (the bulk path's group-start scan)
  __device__ __forceinline__ uint32_t operator()(uint32_t a, uint32_t b) const { return a > b ? a : b; }
};

static bool bulk_wanted(const gfsl *h, uint64_t n) {
  if (h->cfg.serial_updates || h->cfg.combine || h->cfg.bulk == GFSL_BULK_OFF) return false;
  if (h->cfg.bulk == GFSL_BULK_ALWAYS) return true;
  const uint64_t U = std::min(h->capacity, h->live_ub);
  return n >= GFSL_BULK_MIN_OPS && n >= (uint64_t)GFSL_BULK_RATIO * U;
}

template <int N>
static gfsl_status enqueue_bulk(gfsl *h, const uint8_t *ops, const uint32_t *keys, const uint32_t *vals,
                                uint8_t *res, uint64_t n, cudaStream_t s) {
  CK(cudaStreamWaitEvent(s, h->last, 0));
  CK(cudaEventSynchronize(h->last));  // the bump counters after the previous batch
  uint32_t hb[2];
  CK(cudaMemcpy(hb, h->d.bump, 8, cudaMemcpyDeviceToHost));
  const uint32_t used_b = std::min(hb[0], h->d.cap_bottom);
  const uint64_t M = n + (uint64_t)used_b * (N - 2);
  const int bits = sort_bits_for(h->key_range);
  uint32_t *sk0, *sk1, *hd, *gs, *fi, *fd, *ck;
  uint64_t *pl0, *pl1, *cp;
  uint8_t *has_e, *keep;
  unsigned long long *cnt;  // [0] selected, [1] mutations
  void *tmp = nullptr;
  size_t b_sort = 0, b_scan = 0, b_sel = 0, b_sel2 = 0;
  {
    cub::DoubleBuffer<uint32_t> kb(nullptr, nullptr);
    cub::DoubleBuffer<uint64_t> vb(nullptr, nullptr);
    CK(cub::DeviceRadixSort::SortPairs(nullptr, b_sort, kb, vb, (int64_t)M, 0, bits, s));
    CK(cub::DeviceScan::InclusiveScan(nullptr, b_scan, (const uint32_t *)nullptr, (uint32_t *)nullptr, MaxU32(),
                                      (int64_t)M, s));
    CK(cub::DeviceSelect::Flagged(nullptr, b_sel, (const uint32_t *)nullptr, (const uint8_t *)nullptr,
                                  (uint32_t *)nullptr, (unsigned long long *)nullptr, (int64_t)M, s));
    CK(cub::DeviceSelect::Flagged(nullptr, b_sel2, (const uint64_t *)nullptr, (const uint8_t *)nullptr,
                                  (uint64_t *)nullptr, (unsigned long long *)nullptr, (int64_t)M, s));
  }
  const size_t b_tmp = std::max(std::max(b_sort, b_scan), std::max(b_sel, b_sel2));
  char *arena = nullptr;
  const size_t a4 = ((M * 4 + 255) / 256) * 256, a8 = ((M * 8 + 255) / 256) * 256, a1 = ((M + 255) / 256) * 256;
  const size_t total = 7 * a4 + 3 * a8 + 2 * a1 + 256 + b_tmp;
  if (cudaMallocAsync((void **)&arena, total, s) != cudaSuccess) {
    cudaGetLastError();
    set_last_error("bulk path: out of device memory");
    return GFSL_ENOMEM;
  }
  char *q = arena;
  auto take = [&](size_t b) { char *r = q; q += b; return r; };
  sk0 = (uint32_t *)take(a4); sk1 = (uint32_t *)take(a4); hd = (uint32_t *)take(a4); gs = (uint32_t *)take(a4);
  fi = (uint32_t *)take(a4); fd = (uint32_t *)take(a4); ck = (uint32_t *)take(a4);
  pl0 = (uint64_t *)take(a8); pl1 = (uint64_t *)take(a8); cp = (uint64_t *)take(a8);
  has_e = (uint8_t *)take(a1); keep = (uint8_t *)take(a1);
  cnt = (unsigned long long *)take(256);
  tmp = take(b_tmp);
  CK(cudaMemsetAsync(cnt, 0, 16, s));
  const int grid = h->sms * 8;
  bulk_collect_kernel<N><<<grid, 256, 0, s>>>(h->d, ops, keys, vals, res, (uint32_t)n, h->key_range, used_b, sk0, pl0);
  cub::DoubleBuffer<uint32_t> kb(sk0, sk1);
  cub::DoubleBuffer<uint64_t> vb(pl0, pl1);
  size_t bytes = b_tmp;
  CK(cub::DeviceRadixSort::SortPairs(tmp, bytes, kb, vb, (int64_t)M, 0, bits, s));
  const uint32_t *sk = kb.Current();
  const uint64_t *pl = vb.Current();
  bulk_head_kernel<<<grid, 256, 0, s>>>(sk, M, hd, fi, fd, has_e);
  bytes = b_tmp;
  CK(cub::DeviceScan::InclusiveScan(tmp, bytes, (const uint32_t *)hd, gs, MaxU32(), (int64_t)M, s));
  bulk_group_kernel<<<grid, 256, 0, s>>>(sk, pl, gs, M, fi, fd, has_e);
  bulk_result_kernel<<<grid, 256, 0, s>>>(sk, pl, gs, M, fi, fd, has_e, res, keep, cnt + 1);
  bytes = b_tmp;
  CK(cub::DeviceSelect::Flagged(tmp, bytes, sk, keep, ck, cnt, (int64_t)M, s));
  bytes = b_tmp;
  CK(cub::DeviceSelect::Flagged(tmp, bytes, pl, keep, cp, cnt + 2, (int64_t)M, s));
  bulk_write_kernel<N><<<grid, 256, 0, s>>>(h->d, ck, cp, cnt, used_b, cnt + 1);
  CK(cudaGetLastError());
  CK(cudaFreeAsync(arena, s));
  h->launches += 6;
  h->lib_launches += 4 + (uint64_t)(bits + 7) / 8 + 2;  // sort, scan, 2 selects (estimated)
  // the upper levels from the new level 0 (R24, R27); the zombies are gone already
  h->upkeep_pending = false;
  launch_rebuild<N>(h, s);
  CK(cudaGetLastError());
  CK(cudaMemcpyAsync(h->h_bump, h->d.bump, 8, cudaMemcpyDeviceToHost, s));
  CK(cudaEventRecord(h->last, s));
  h->batches++;
  h->bulk_batches++;
  h->ops += n;
  h->live_ub = std::min(h->capacity, h->live_ub + n);
  h->ops_since_rebuild = 0;
  h->ops_at_rebuild = h->ops;
  h->muts_at_rebuild = *(volatile unsigned long long *)h->h_mut;
  return GFSL_OK;
}

static gfsl_status enqueue_bulk_any(gfsl *h, const uint8_t *ops, const uint32_t *keys, const uint32_t *vals,
                                    uint8_t *res, uint64_t n, cudaStream_t s) {
  switch (h->N) {
    case 32: return enqueue_bulk<32>(h, ops, keys, vals, res, n, s);
    case 16: return enqueue_bulk<16>(h, ops, keys, vals, res, n, s);
    case 12: return enqueue_bulk<12>(h, ops, keys, vals, res, n, s);
    case 6: return enqueue_bulk<6>(h, ops, keys, vals, res, n, s);
  }
  return GFSL_EINVAL;
}

extern "C" gfsl_status gfsl_rebuild(gfsl_t h, void *stream) {
  if (!h) {
    set_last_error("NULL handle");
    return GFSL_EINVAL;
  }
  gfsl_status st = sticky(h);
  if (st != GFSL_OK) return st;
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaStreamWaitEvent(s, h->last, 0));
  switch (h->N) {
    case 32: launch_rebuild<32>(h, s); break;
    case 16: launch_rebuild<16>(h, s); break;
    case 12: launch_rebuild<12>(h, s); break;
    case 6: launch_rebuild<6>(h, s); break;
  }
  CK(cudaGetLastError());
  CK(cudaEventRecord(h->last, s));
  h->ops_since_rebuild = 0;
  h->ops_at_rebuild = h->ops;
  h->muts_at_rebuild = *(volatile unsigned long long *)h->h_mut;
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_batch(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                                  const uint32_t *values, uint8_t *results, uint64_t n,
                                  void *stream) {
  if (!h) {
    set_last_error("NULL handle");
    return GFSL_EINVAL;
  }
  gfsl_status st = sticky(h);
  if (st != GFSL_OK) return st;
  if (n == 0) return GFSL_OK;
  if (!op_types || !keys || !results || n > GFSL_MAX_BATCH) {
    set_last_error("bad batch arguments");
    return GFSL_EINVAL;
  }
  if (bulk_wanted(h, n)) return enqueue_bulk_any(h, op_types, keys, values, results, n, (cudaStream_t)stream);
  if ((st = ensure_lists(h, n)) != GFSL_OK) return st;
  if (h->cfg.combine && (st = ensure_combine(h, n)) != GFSL_OK) return st;
  if ((st = ensure_key_order(h, n)) != GFSL_OK) return st;
  return enqueue_batch(h, op_types, keys, values, results, n, (cudaStream_t)stream);
}

extern "C" gfsl_status gfsl_batch_dn(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                                     const uint32_t *values, uint8_t *results, uint64_t n_max,
                                     const uint32_t *n_dev, uint64_t n_hint, void *stream) {
  if (!h) {
    set_last_error("NULL handle");
    return GFSL_EINVAL;
  }
  gfsl_status st = sticky(h);
  if (st != GFSL_OK) return st;
  if (n_max == 0) return GFSL_OK;
  if (!op_types || !keys || !results || !n_dev || n_max > GFSL_MAX_BATCH) {
    set_last_error("bad batch arguments");
    return GFSL_EINVAL;
  }
  if (h->cfg.combine || h->cfg.serial_updates) {
    set_last_error("gfsl_batch_dn: not available in combining or serial mode");
    return GFSL_EINVAL;
  }
  if ((st = ensure_lists(h, n_max)) != GFSL_OK) return st;
  h->ko_now = false;
  return enqueue_batch(h, op_types, keys, values, results, n_max, (cudaStream_t)stream, n_dev,
                       n_hint ? std::min(n_hint, n_max) : n_max);
}

static gfsl_status ensure_staging(gfsl *h, uint64_t n) {
  if (!h->copy_stream) {
    CK(cudaStreamCreateWithFlags(&h->copy_stream, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&h->exec_stream, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&h->d2h_stream, cudaStreamNonBlocking));
    for (int b = 0; b < 2; ++b) {
      CK(cudaEventCreateWithFlags(&h->ev_in[b], cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&h->ev_used[b], cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&h->ev_out[b], cudaEventDisableTiming));
    }
  }
  if (n <= h->st_cap) return GFSL_OK;
  cudaDeviceSynchronize();
  h->st_cap = 0;
  for (int b = 0; b < 2; ++b) {
    cudaFree(h->st_op[b]);
    cudaFree(h->st_res[b]);
    cudaFree(h->st_key[b]);
    cudaFree(h->st_val[b]);
    h->st_op[b] = h->st_res[b] = nullptr;
    h->st_key[b] = h->st_val[b] = nullptr;
  }
  for (int b = 0; b < 2; ++b) {
    CK(cudaMalloc(&h->st_op[b], n));
    CK(cudaMalloc(&h->st_res[b], n));
    CK(cudaMalloc(&h->st_key[b], n * 4));
    CK(cudaMalloc(&h->st_val[b], n * 4));
  }
  h->st_cap = n;
  return GFSL_OK;
}

// The host-buffer batch, asynchronous, on three library streams: the inputs go to staging
// slot b on the copy stream (after the kernels of the batch that last used the slot have
// read it), the kernels run on the exec stream once they have arrived (and once the
// slot's previous results have left), the results come back on the d2h stream, and
// `stream` waits for them.  With pinned host memory the copy-in of the next batch and
// the copy-out of the previous one both overlap this batch's kernels (the kernels of
// batch i+1 do not queue behind the copy-out of batch i, as they would on `stream`).
// Batches of one handle stay ordered by the handle's own event (enqueue_batch).
static gfsl_status batch_host_async(gfsl *h, const uint8_t *op_types, const uint32_t *keys,
                                    const uint32_t *values, uint8_t *results, uint64_t n,
                                    cudaStream_t s) {
  gfsl_status st = sticky(h);
  if (st != GFSL_OK) return st;
  if (n == 0) return GFSL_OK;
  if (!op_types || !keys || !results || n > GFSL_MAX_BATCH) {
    set_last_error("bad batch arguments");
    return GFSL_EINVAL;
  }
  if ((st = ensure_staging(h, n)) != GFSL_OK) return st;
  if ((st = ensure_lists(h, n)) != GFSL_OK) return st;
  if (h->cfg.combine && (st = ensure_combine(h, n)) != GFSL_OK) return st;
  if ((st = ensure_key_order(h, n)) != GFSL_OK) return st;
  const int b = h->st_slot;
  h->st_slot ^= 1;
  const bool bulk = bulk_wanted(h, n);
  // Zero-copy values (opt-in, GFSL_ZC_VALUES=1 at gfsl_create): an Insert's value is the
  // only one any kernel reads (the search kernel loads it when the Insert becomes current),
  // so with a mapped pinned value buffer the kernel can read those values over PCIe instead
  // of the whole array being copied.  Measured: with 10% Inserts the PCIe reads
  // on the search kernel's path cost more than the copy (C5 e2e 5589 -> 3712 Mops/s).  Not
  // for the bulk path or combining mode.
  const uint32_t *vals_in = nullptr;
  if (values && h->zc_values && !bulk && !h->cfg.combine) {
    cudaPointerAttributes pa{};
    if (cudaPointerGetAttributes(&pa, values) == cudaSuccess && pa.type == cudaMemoryTypeHost && pa.devicePointer)
      vals_in = (const uint32_t *)pa.devicePointer;
    cudaGetLastError();
  }
  cudaStream_t c = h->copy_stream;
  CK(cudaStreamWaitEvent(c, h->ev_used[b], 0));  // the slot's previous batch has read it
  CK(cudaMemcpyAsync(h->st_op[b], op_types, n, cudaMemcpyHostToDevice, c));
  CK(cudaMemcpyAsync(h->st_key[b], keys, n * 4, cudaMemcpyHostToDevice, c));
  if (values && !vals_in) {
    CK(cudaMemcpyAsync(h->st_val[b], values, n * 4, cudaMemcpyHostToDevice, c));
    vals_in = h->st_val[b];
  } else if (vals_in) {
    h->zc_batches++;
  }
  CK(cudaEventRecord(h->ev_in[b], c));
  cudaStream_t k = h->exec_stream, o = h->d2h_stream;
  CK(cudaStreamWaitEvent(k, h->ev_in[b], 0));
  CK(cudaStreamWaitEvent(k, h->ev_out[b], 0));  // the slot's previous results have left
  st = bulk ? enqueue_bulk_any(h, h->st_op[b], h->st_key[b], vals_in, h->st_res[b], n, k)
            : enqueue_batch(h, h->st_op[b], h->st_key[b], vals_in, h->st_res[b], n, k);
  if (st != GFSL_OK) return st;
  CK(cudaEventRecord(h->ev_used[b], k));
  CK(cudaStreamWaitEvent(o, h->ev_used[b], 0));
  CK(cudaMemcpyAsync(results, h->st_res[b], n, cudaMemcpyDeviceToHost, o));
  CK(cudaEventRecord(h->ev_out[b], o));
  CK(cudaStreamWaitEvent(s, h->ev_out[b], 0));
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_batch_host(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                                       const uint32_t *values, uint8_t *results, uint64_t n,
                                       void *stream) {
  if (!h) {
    set_last_error("NULL handle");
    return GFSL_EINVAL;
  }
  cudaStream_t s = (cudaStream_t)stream;
  gfsl_status st = batch_host_async(h, op_types, keys, values, results, n, s);
  if (st != GFSL_OK) return st;
  CK(cudaStreamSynchronize(s));
  return sticky(h);
}

extern "C" gfsl_status gfsl_batch_host_async(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                                             const uint32_t *values, uint8_t *results, uint64_t n,
                                             void *stream) {
  if (!h) {
    set_last_error("NULL handle");
    return GFSL_EINVAL;
  }
  return batch_host_async(h, op_types, keys, values, results, n, (cudaStream_t)stream);
}

#ifdef GFSL_DEBUG_TIMING
extern "C" gfsl_status gfsl_debug_times(gfsl_t h, unsigned long long *out, uint64_t n) {
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(out, h->d.debug_times, std::min<uint64_t>(n, (uint64_t)148 * 64 * 48 + 64) * 8, cudaMemcpyDeviceToHost));
  return GFSL_OK;
}
#endif

extern "C" gfsl_status gfsl_get_stats(gfsl_t h, gfsl_stats *out) {
  if (!h || !out) return GFSL_EINVAL;
  unsigned long long s[ST_NSTATS];
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(s, h->d.stats, sizeof(s), cudaMemcpyDeviceToHost));
  memset(out, 0, sizeof(*out));
  out->batches = h->batches;
  out->ops = h->ops;
  out->restarts = s[ST_RESTARTS];
  out->splits = s[ST_SPLITS];
  out->merges = s[ST_MERGES];
  out->zombie_unlinks = s[ST_ZOMBIE_UNLINKS];
  out->lock_retries = s[ST_LOCK_RETRIES];
  out->contains_reads = s[ST_CREADS];
  out->contains_reads_l0 = s[ST_CREADS_L0];
  out->contains_ops = s[ST_COPS];
  out->mutations = s[ST_MUTATIONS];
  out->grouped = s[ST_GROUPED];
  out->zero_copy_batches = h->zc_batches;
  out->kernel_launches = h->launches;
  out->library_launches = h->lib_launches;
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_phase_times(gfsl_t h, double *ms, uint64_t *batches) {
  if (!h || !ms) return GFSL_EINVAL;
  CK(cudaDeviceSynchronize());
  double acc[5] = {0, 0, 0, 0, 0};
  for (auto &ev : h->phase_ev) {
    float a = 0, b = 0, c = 0, u = 0, t = 0;
    CK(cudaEventElapsedTime(&a, ev[0], ev[1]));
    CK(cudaEventElapsedTime(&b, ev[1], ev[2]));
    CK(cudaEventElapsedTime(&c, ev[2], ev[3]));
    CK(cudaEventElapsedTime(&u, ev[3], ev[4]));
    CK(cudaEventElapsedTime(&t, ev[0], ev[4]));
    acc[0] += a;
    acc[1] += b;
    acc[2] += c;
    acc[3] += u;
    acc[4] += t;
    for (auto &e : ev) cudaEventDestroy(e);
  }
  for (int i = 0; i < 5; ++i) ms[i] = acc[i];
  if (batches) *batches = h->phase_ev.size();
  h->phase_ev.clear();
  return GFSL_OK;
}

// ------------------------------------------------------------------------------------
// dump / load (test-only)

static gfsl_status read_meta(gfsl *h, gfsl_meta *m) {
  memset(m, 0, sizeof(*m));
  uint32_t bump[2];
  CK(cudaMemcpy(m->head, h->d.head, 32 * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(m->counters, h->d.counter, 32 * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(bump, h->d.bump, 8, cudaMemcpyDeviceToHost));
  m->used_bottom = std::min(bump[0], h->d.cap_bottom);
  m->used_upper = std::min(bump[1], h->d.cap_upper);
  m->cap_bottom = h->d.cap_bottom;
  m->cap_upper = h->d.cap_upper;
  m->chunk_entries = h->N;
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_dump(gfsl_t h, gfsl_meta *meta, uint64_t *entries, uint64_t max_entries) {
  if (!h) return GFSL_EINVAL;
  CK(cudaDeviceSynchronize());
  gfsl_meta m;
  gfsl_status st = read_meta(h, &m);
  if (st != GFSL_OK) return st;
  if (meta) *meta = m;
  if (entries) {
    const uint64_t total = ((uint64_t)h->d.cap_bottom + h->d.cap_upper) * h->N;
    CK(cudaMemcpy(entries, h->d.pool, std::min(total, max_entries) * 8, cudaMemcpyDeviceToHost));
  }
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_load(gfsl_t h, const gfsl_meta *meta, const uint64_t *entries,
                                 uint64_t n_entries) {
  if (!h || !meta || !entries) return GFSL_EINVAL;
  const uint64_t total = ((uint64_t)h->d.cap_bottom + h->d.cap_upper) * h->N;
  if (n_entries != total || meta->chunk_entries != h->N || meta->cap_bottom != h->d.cap_bottom ||
      meta->cap_upper != h->d.cap_upper) {
    set_last_error("gfsl_load: image does not match the handle's pool geometry");
    return GFSL_EINVAL;
  }
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(h->d.pool, entries, total * 8, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(h->d.head, meta->head, 32 * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(h->d.counter, meta->counters, 32 * 4, cudaMemcpyHostToDevice));
  uint32_t bump[2] = {meta->used_bottom, meta->used_upper};
  CK(cudaMemcpy(h->d.bump, bump, 8, cudaMemcpyHostToDevice));
  CK(cudaMemset(h->d.dir_hdr, 0, 64 * 4));  // the directory describes the old structure
  CK(cudaMemset(h->d.zbits, 0, (size_t)h->d.zwords * 8));
  return GFSL_OK;
}

// ------------------------------------------------------------------------------------
// validate (a6): copy the used part of the pool and walk it.  Invariants:
//  V1 non-zombie chunks sorted, EMPTY grouped at the end
//  V2 non-last chunk: max == largest key; last: max = next = inf
//  V3 consecutive non-zombie chunks: max(c) < min(next)
//  V4 level l+1 keys are a subset of level l keys
//  V5 the down pointer of k at level l+1 reaches k laterally
//  V7 no lock held at quiescence
//  V8 the last chunk of a level is not a zombie
//  V9 the head reaches a first non-zombie chunk holding -inf at index 0
//  V10 keys are valid internal keys; -inf only first
//  V12 every reachable chunk index is allocated
//  (V13 of SURVEY 8(c), min fill floor(DSIZE/3), is NOT an invariant: a splitRemove can
//   leave the new chunk with cntF - DSIZE/2 < DSIZE/3 entries; it is reported as a count)
//  V14 counter[l] = #non-zombie chunks if level l holds a real key, else 0 (R9/R17)

namespace {
struct HostPool {
  uint32_t N, cap_u, cap_b, used_u, used_b;
  std::vector<uint64_t> up, bot;
  bool allocated(uint32_t c) const {
    if (c < cap_u) return c < used_u;
    return c >= cap_u && (uint64_t)c < (uint64_t)cap_u + used_b;
  }
  const uint64_t *chunk(uint32_t c) const {
    if (c < cap_u) return &up[(size_t)c * N];
    return &bot[(size_t)(c - cap_u) * N];
  }
};
inline uint32_t klo(uint64_t e) { return (uint32_t)e; }
inline uint32_t khi(uint64_t e) { return (uint32_t)(e >> 32); }
}  // namespace

extern "C" gfsl_status gfsl_validate(gfsl_t h, gfsl_report *rep_out, uint32_t *keys_out,
                                     uint32_t *vals_out, uint64_t cap, uint64_t *count) {
  if (!h) return GFSL_EINVAL;
  CK(cudaDeviceSynchronize());
  gfsl_status st = sticky(h);
  if (st != GFSL_OK) return st;
  gfsl_meta m;
  if ((st = read_meta(h, &m)) != GFSL_OK) return st;
  HostPool P;
  P.N = h->N;
  P.cap_u = m.cap_upper;
  P.cap_b = m.cap_bottom;
  P.used_u = m.used_upper;
  P.used_b = m.used_bottom;
  P.up.resize((size_t)P.used_u * P.N);
  P.bot.resize((size_t)P.used_b * P.N);
  CK(cudaMemcpy(P.up.data(), h->d.pool, P.up.size() * 8, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(P.bot.data(), h->d.pool + (size_t)P.cap_u * P.N, P.bot.size() * 8, cudaMemcpyDeviceToHost));

  gfsl_report rep;
  memset(&rep, 0, sizeof(rep));
  const uint32_t N = P.N, DS = N - 2, NX = N - 2, LK = N - 1;
  rep.chunk_entries = N;
  uint32_t viol = 0;
  auto V = [&](int v) { viol |= 1u << (v - 1); };
  int height = 0;
  for (uint32_t l = 1; l < N; ++l)
    if (m.counters[l] > 0) height = (int)l;
  rep.height = height;
  for (uint32_t l = 0; l < N && l < 32; ++l) rep.counters[l] = m.counters[l];
  rep.pool_used[0] = P.used_b;
  rep.pool_used[1] = P.used_u;
  rep.pool_cap[0] = P.cap_b;
  rep.pool_cap[1] = P.cap_u;

  // per level: ordered list of (non-zombie chunk index), and key -> chunk map (sorted)
  std::vector<std::vector<uint32_t>> chunks(N);
  std::vector<std::vector<std::pair<uint32_t, uint32_t>>> keymap(N);  // (key, value) per level
  std::vector<std::vector<uint32_t>> keychunk(N);                     // chunk holding that key
  const uint64_t step_cap = (uint64_t)P.used_u + P.used_b + 16;
  for (uint32_t l = 0; l < N; ++l) {
    uint32_t c = m.head[l];
    bool seen_first = false;
    uint64_t steps = 0;
    uint32_t prev_max = 0;
    bool have_prev = false;
    while (c != NULL_CHUNK) {
      if (!P.allocated(c) || ++steps > step_cap) {
        V(12);
        break;
      }
      const uint64_t *ch = P.chunk(c);
      const uint32_t state = klo(ch[LK]);
      const uint32_t next = khi(ch[NX]);
      const uint32_t mx = klo(ch[NX]);
      if (state == LOCK_ZOMBIE) {
        rep.zombies[l]++;
        if (next == NULL_CHUNK) V(8);
        c = next;
        continue;
      }
      if (state != LOCK_FREE) V(7);
      rep.chunks[l]++;
      chunks[l].push_back(c);
      // V1 sortedness / EMPTY grouping; count
      uint32_t cnt = 0;
      bool empty_seen = false;
      uint32_t last_key = 0;
      for (uint32_t i = 0; i < DS; ++i) {
        const uint32_t k = klo(ch[i]);
        if (k == KEY_EMPTY) {
          empty_seen = true;
          if (ch[i] != EMPTY_ENTRY) V(1);
          continue;
        }
        if (empty_seen) V(1);
        if (cnt > 0 && k <= last_key) V(1);
        if (k == KEY_NEG_INF) {
          if (seen_first || i != 0) V(10);
        } else {
          if (k > h->d.key_max) V(10);
          keymap[l].push_back({k, khi(ch[i])});
          keychunk[l].push_back(c);
        }
        last_key = k;
        ++cnt;
      }
      if (!seen_first) {
        if (cnt == 0 || klo(ch[0]) != KEY_NEG_INF) V(9);
      }
      // V2
      if (next == NULL_CHUNK) {
        if (mx != KEY_POS_INF) V(2);
      } else {
        if (cnt == 0 || mx != last_key) V(2);
        if (cnt < std::max<uint32_t>(1, DS / 3)) rep.underfull++;  // underfull (not an invariant)
      }
      // V3
      if (have_prev && cnt > 0) {
        const uint32_t first_real = klo(ch[0]);
        if (!(prev_max < first_real)) V(3);
      }
      if (cnt > 0) {
        prev_max = last_key;
        have_prev = true;
      }
      seen_first = true;
      c = next;
    }
    if (!seen_first) V(9);
    rep.level_keys[l] = keymap[l].size();
    // V14 counters
    const int64_t expect = keymap[l].empty() ? 0 : (int64_t)rep.chunks[l];
    if (N >= 12 && m.counters[l] != expect) V(14);
    if (N < 12 && !keymap[l].empty() && m.counters[l] <= 0 && l >= 1) V(14);
  }
  // V4 + V5
  for (uint32_t l = 0; l + 1 < N; ++l) {
    const auto &lo = keymap[l];
    const auto &up = keymap[l + 1];
    for (size_t i = 0; i < up.size(); ++i) {
      const uint32_t k = up[i].first;
      auto it = std::lower_bound(lo.begin(), lo.end(), std::make_pair(k, 0u),
                                 [](auto a, auto b) { return a.first < b.first; });
      uint32_t target;
      if (it == lo.end() || it->first != k) {
        // R33: after lazy batches a level-1 key may be a stale separator (deleted from
        // level 0 since the last rebuild); its down pointer must still reach, laterally,
        // the level-0 chunk that encloses k (the chunk of the next larger key, or the last)
        if (!(h->upper_stale && l == 0) || chunks[0].empty()) {
          V(4);
          continue;
        }
        // k above every key (or level 0 empty): the last chunk of the level
        target = it == lo.end() ? chunks[0].back() : keychunk[l][it - lo.begin()];
      } else {
        target = keychunk[l][it - lo.begin()];
      }
      // walk laterally from the down pointer to the chunk holding k
      uint32_t c = up[i].second;
      uint64_t steps = 0;
      bool ok = false;
      while (c != NULL_CHUNK && P.allocated(c) && ++steps <= step_cap) {
        if (c == target) {
          ok = true;
          break;
        }
        c = khi(P.chunk(c)[NX]);
      }
      if (!ok) V(5);
    }
  }
  // the -inf down pointers must also reach the level below laterally
  rep.keys = keymap[0].size();
  rep.violations = viol;
  for (int v = 1; v <= 32; ++v)
    if (viol & (1u << (v - 1))) {
      rep.first_violation = v;
      break;
    }
  unsigned long long s[ST_NSTATS];
  CK(cudaMemcpy(s, h->d.stats, sizeof(s), cudaMemcpyDeviceToHost));
  rep.restarts = s[ST_RESTARTS];
  if (rep_out) *rep_out = rep;
  if (count) *count = rep.keys;
  if (keys_out || vals_out) {
    const uint64_t n = std::min<uint64_t>(cap, keymap[0].size());
    for (uint64_t i = 0; i < n; ++i) {
      if (keys_out) keys_out[i] = keymap[0][i].first - 1u;  // user key
      if (vals_out) vals_out[i] = keymap[0][i].second;
    }
  }
  if (viol) {
    char buf[128];
    snprintf(buf, sizeof(buf), "invariant violation mask 0x%x (first V%u)", viol, rep.first_violation);
    set_last_error(buf);
    return GFSL_ECORRUPT;
  }
  return GFSL_OK;
}

// ------------------------------------------------------------------------------------
// B4: device-side structural check and bottom-level export (gfsl_check.cuh)

template <int N>
static gfsl_status check_impl(gfsl *h, gfsl_report *rep_out, uint32_t flags) {
  gfsl_meta m;
  gfsl_status st = read_meta(h, &m);
  if (st != GFSL_OK) return st;
  CheckBufs b{};
  b.used_u = m.used_upper;
  b.used_b = m.used_bottom;
  b.stale_ok = h->upper_stale ? 1u : 0u;
  const bool cross = (flags & GFSL_CHECK_CROSS) && h->snap_max && h->snap_rebuilds == h->rebuilds;
  if (cross) {
    b.snap_max = h->snap_max;
    b.snap_zh = h->snap_zh;
    b.snap_used_u = h->snap_used_u;
    b.snap_used_b = h->snap_used_b;
  }
  const size_t total = (size_t)b.used_u + b.used_b;
  CK(cudaMalloc(&b.indeg, std::max<size_t>(total, 1) * 4));
  CK(cudaMalloc(&b.cnt, CC_NCNT * 8 + 8));
  b.viol = (uint32_t *)(b.cnt + CC_NCNT);
  CK(cudaMemset(b.indeg, 0, std::max<size_t>(total, 1) * 4));
  CK(cudaMemset(b.cnt, 0, CC_NCNT * 8 + 8));
  const int grid = h->sms * 8;
  check_chunks_kernel<N><<<grid, 256>>>(h->d, b);
  check_indeg_kernel<N><<<grid, 256>>>(h->d, b);
  CK(cudaGetLastError());
  unsigned long long cnt[CC_NCNT + 1];
  CK(cudaMemcpy(cnt, b.cnt, sizeof(cnt), cudaMemcpyDeviceToHost));
  uint32_t viol = (uint32_t)cnt[CC_NCNT];
  cudaFree(b.indeg);
  cudaFree(b.cnt);
  auto V = [&](int v) { viol |= 1u << (v - 1); };
  // chain shape: one first and one last live chunk per level, no merging NEXT chains
  if (cnt[CC_SRC_B] != 1 || cnt[CC_LAST_B] != 1 || cnt[CC_FIRST_B] != 1) V(9);
  if (cnt[CC_SRC_U] != N - 1 || cnt[CC_LAST_U] != N - 1 || cnt[CC_FIRST_U] != N - 1) V(9);
  if (cnt[CC_MULTI]) V(3);
  // the head array leads (through zombies) to the first live chunk holding -inf
  std::vector<uint64_t> hc(N);
  for (uint32_t l = 0; l < N; ++l) {
    uint32_t c = m.head[l];
    for (int hops = 0; hops < 4096 && c != NULL_CHUNK; ++hops) {
      CK(cudaMemcpy(hc.data(), h->d.pool + (size_t)c * N, N * 8, cudaMemcpyDeviceToHost));
      if ((uint32_t)hc[N - 1] != LOCK_ZOMBIE) break;
      c = (uint32_t)(hc[N - 2] >> 32);
    }
    if (c == NULL_CHUNK || (uint32_t)hc[N - 1] != LOCK_FREE || (uint32_t)hc[0] != KEY_NEG_INF ||
        (l == 0) != (c >= m.cap_upper))
      V(9);
  }
  const uint64_t keys = cnt[CC_KEYS_B];
  if (N >= 12 && m.counters[0] != (keys ? (int64_t)cnt[CC_LIVE_B] : 0)) V(14);
  gfsl_report rep;
  memset(&rep, 0, sizeof(rep));
  rep.keys = keys;
  rep.chunk_entries = N;
  for (uint32_t l = 1; l < N; ++l)
    if (m.counters[l] > 0) rep.height = l;
  for (uint32_t l = 0; l < N; ++l) rep.counters[l] = m.counters[l];
  rep.chunks[0] = cnt[CC_LIVE_B];
  rep.chunks[1] = cnt[CC_LIVE_U];  // all upper levels together (the check is chunk-parallel)
  rep.zombies[0] = cnt[CC_ZOMBIE_B];
  rep.zombies[1] = cnt[CC_ZOMBIE_U];
  rep.level_keys[0] = keys;
  rep.pool_used[0] = m.used_bottom;
  rep.pool_used[1] = m.used_upper;
  rep.pool_cap[0] = m.cap_bottom;
  rep.pool_cap[1] = m.cap_upper;
  rep.underfull = cnt[CC_UNDERFULL];
  rep.reserved[0] = cnt[CC_STALE];      // level-1 stale separators (R33)
  rep.reserved[1] = cross ? 1u : 0u;    // 1 = V6 / V11 were checked against a snapshot
  unsigned long long sstat[ST_NSTATS];
  CK(cudaMemcpy(sstat, h->d.stats, sizeof(sstat), cudaMemcpyDeviceToHost));
  rep.restarts = sstat[ST_RESTARTS];
  rep.violations = viol;
  for (int v = 1; v <= 32; ++v)
    if (viol & (1u << (v - 1))) {
      rep.first_violation = v;
      break;
    }
  if (flags & GFSL_CHECK_SNAPSHOT) {
    cudaFree(h->snap_max);
    cudaFree(h->snap_zh);
    h->snap_max = nullptr;
    h->snap_zh = nullptr;
    CK(cudaMalloc(&h->snap_max, std::max<size_t>(total, 1) * 4));
    CK(cudaMalloc(&h->snap_zh, std::max<size_t>(total, 1) * 8));
    check_snapshot_kernel<N><<<grid, 256>>>(h->d, b.used_u, b.used_b, h->snap_max, h->snap_zh);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    h->snap_used_u = b.used_u;
    h->snap_used_b = b.used_b;
    h->snap_rebuilds = h->rebuilds;
  }
  if (rep_out) *rep_out = rep;
  if (viol) {
    char buf[128];
    snprintf(buf, sizeof(buf), "invariant violation mask 0x%x (first V%u)", viol, rep.first_violation);
    set_last_error(buf);
    return GFSL_ECORRUPT;
  }
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_check(gfsl_t h, gfsl_report *rep, uint32_t flags) {
  if (!h) return GFSL_EINVAL;
  CK(cudaDeviceSynchronize());
  gfsl_status st = sticky(h);
  if (st != GFSL_OK) return st;
  switch (h->N) {
    case 32: return check_impl<32>(h, rep, flags);
    case 16: return check_impl<16>(h, rep, flags);
    case 12: return check_impl<12>(h, rep, flags);
    case 6: return check_impl<6>(h, rep, flags);
  }
  return GFSL_EINVAL;
}

template <int N>
static gfsl_status export_impl(gfsl *h, uint32_t *keys_out, uint32_t *vals_out, uint64_t cap,
                               uint64_t *count) {
  gfsl_meta m;
  gfsl_status st = read_meta(h, &m);
  if (st != GFSL_OK) return st;
  const uint64_t slots = std::max<uint64_t>((uint64_t)m.used_bottom * (N - 2), 1);
  unsigned long long *d_cnt = nullptr;
  uint32_t *k0 = nullptr, *v0 = nullptr, *k1 = nullptr, *v1 = nullptr, *viol = nullptr;
  void *tmp = nullptr;
  gfsl_status rs = GFSL_OK;
  auto cleanup = [&]() {
    cudaFree(d_cnt); cudaFree(k0); cudaFree(v0); cudaFree(k1); cudaFree(v1); cudaFree(tmp);
  };
  CK(cudaMalloc(&d_cnt, 16));
  viol = (uint32_t *)(d_cnt + 1);
  CK(cudaMemset(d_cnt, 0, 16));
  if (!keys_out && !vals_out) {  // count only
    export_count_kernel<N><<<h->sms * 8, 256>>>(h->d, m.used_bottom, d_cnt);
    uint64_t cnt = 0;
    CK(cudaMemcpy(&cnt, d_cnt, 8, cudaMemcpyDeviceToHost));
    cleanup();
    if (count) *count = cnt;
    return GFSL_OK;
  }
  if (cudaMalloc(&k0, slots * 4) != cudaSuccess || cudaMalloc(&v0, slots * 4) != cudaSuccess ||
      cudaMalloc(&k1, slots * 4) != cudaSuccess || cudaMalloc(&v1, slots * 4) != cudaSuccess) {
    cleanup();
    set_last_error("gfsl_export: out of device memory");
    return GFSL_ENOMEM;
  }
  export_collect_kernel<N><<<h->sms * 8, 256>>>(h->d, m.used_bottom, k0, v0, d_cnt);
  uint64_t n = 0;
  CK(cudaMemcpy(&n, d_cnt, 8, cudaMemcpyDeviceToHost));
  if (n) {
    cub::DoubleBuffer<uint32_t> kb(k0, k1), vb(v0, v1);
    size_t bytes = 0;
    CK(cub::DeviceRadixSort::SortPairs(nullptr, bytes, kb, vb, (int64_t)n, 0, 32));
    if (cudaMalloc(&tmp, bytes) != cudaSuccess) {
      cleanup();
      set_last_error("gfsl_export: out of device memory");
      return GFSL_ENOMEM;
    }
    CK(cub::DeviceRadixSort::SortPairs(tmp, bytes, kb, vb, (int64_t)n, 0, 32));
    const uint64_t w = std::min(n, cap);
    export_finish_kernel<<<h->sms * 8, 256>>>(kb.Current(), vb.Current(), w, keys_out, vals_out, viol);
    CK(cudaGetLastError());
    uint32_t v = 0;
    CK(cudaMemcpy(&v, viol, 4, cudaMemcpyDeviceToHost));
    if (v) {
      set_last_error("gfsl_export: a key is held by two live level-0 chunks (V3)");
      rs = GFSL_ECORRUPT;
    }
  }
  cleanup();
  if (count) *count = n;
  return rs;
}

extern "C" gfsl_status gfsl_export(gfsl_t h, uint32_t *keys, uint32_t *values, uint64_t cap,
                                   uint64_t *count) {
  if (!h) return GFSL_EINVAL;
  CK(cudaDeviceSynchronize());
  gfsl_status st = sticky(h);
  if (st != GFSL_OK) return st;
  switch (h->N) {
    case 32: return export_impl<32>(h, keys, values, cap, count);
    case 16: return export_impl<16>(h, keys, values, cap, count);
    case 12: return export_impl<12>(h, keys, values, cap, count);
    case 6: return export_impl<6>(h, keys, values, cap, count);
  }
  return GFSL_EINVAL;
}

// ------------------------------------------------------------------------------------
// multi-GPU routing (B5): stable partition of a batch by destination shard.

constexpr int ROUTE_TILE = 1024;  // ops per block tile (256 threads x 4)
constexpr int MAX_WORLD = 64;

__device__ __forceinline__ uint32_t route_dest(uint8_t op, uint32_t key, uint64_t key_range,
                                               uint64_t span, uint32_t world) {
  if (op > 2 || (uint64_t)key >= key_range) return 0;
  const uint64_t g = (uint64_t)key / span;
  return (uint32_t)(g < world ? g : world - 1);
}

// pass 1: per-tile histogram -> tile_counts[tile * world + g]
__global__ void route_hist_kernel(const uint8_t *ops, const uint32_t *keys, uint32_t n,
                                  uint64_t key_range, uint64_t span, uint32_t world,
                                  uint32_t *tile_counts) {
  __shared__ uint32_t hist[MAX_WORLD];
  for (uint32_t g = threadIdx.x; g < world; g += blockDim.x) hist[g] = 0;
  __syncthreads();
  const uint32_t base = blockIdx.x * ROUTE_TILE;
  for (uint32_t i = base + threadIdx.x; i < min(n, base + ROUTE_TILE); i += blockDim.x)
    atomicAdd(&hist[route_dest(ops[i], keys[i], key_range, span, world)], 1u);
  __syncthreads();
  for (uint32_t g = threadIdx.x; g < world; g += blockDim.x) tile_counts[blockIdx.x * world + g] = hist[g];
}

// pass 2: one block per destination g scans its column of tile counts (tiles in input
// order) with a carry: tile_counts[t * world + g] = ops for g in tiles before t; counts[g]
// = the column total.  The destination-major base (the ops of the destinations before g)
// is added by the scatter kernel, which reads counts.
__global__ void __launch_bounds__(1024) route_scan_kernel(uint32_t *tile_counts, uint32_t tiles, uint32_t world,
                                                         unsigned long long *counts) {
  __shared__ uint32_t warp_tot[32];
  __shared__ uint32_t carry;
  const uint32_t g = blockIdx.x;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (uint32_t t0 = 0; t0 < tiles; t0 += blockDim.x) {
    const uint32_t t = t0 + threadIdx.x;
    const uint32_t v = t < tiles ? tile_counts[(size_t)t * world + g] : 0u;
    uint32_t incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
      if (lane >= o) incl += y;
    }
    if (lane == 31) warp_tot[warp] = incl;
    __syncthreads();
    if (warp == 0) {
      const uint32_t wt = lane < (int)(blockDim.x >> 5) ? warp_tot[lane] : 0u;
      uint32_t wi = wt;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, wi, o);
        if (lane >= o) wi += y;
      }
      warp_tot[lane] = wi - wt;  // exclusive prefix of the warp totals
    }
    __syncthreads();
    const uint32_t base = carry;
    if (t < tiles) tile_counts[(size_t)t * world + g] = base + warp_tot[warp] + incl - v;
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry = base + warp_tot[warp] + incl;
    __syncthreads();
  }
  if (threadIdx.x == 0) counts[g] = carry;
}

// pass 3: stable scatter of op indices; ranks within a tile follow input order.
__global__ void route_scatter_kernel(const uint8_t *ops, const uint32_t *keys, uint32_t n,
                                     uint64_t key_range, uint64_t span, uint32_t world,
                                     const uint32_t *tile_offsets, const unsigned long long *counts,
                                     uint32_t *perm) {
  __shared__ uint32_t base_g[MAX_WORLD];
  __shared__ uint32_t warp_counts[8][MAX_WORLD];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t tile0 = blockIdx.x * ROUTE_TILE;
  if (threadIdx.x == 0) {  // destination-major base: the ops of the destinations before g
    uint32_t run = 0;
    for (uint32_t g = 0; g < world; ++g) {
      base_g[g] = run + tile_offsets[(size_t)blockIdx.x * world + g];
      run += (uint32_t)counts[g];
    }
  }
  __syncthreads();
  // the tile is processed 256 consecutive ops at a time, in input order
  for (uint32_t off = 0; off < ROUTE_TILE; off += 256) {
    for (uint32_t x = threadIdx.x; x < 8 * MAX_WORLD; x += blockDim.x) (&warp_counts[0][0])[x] = 0;
    __syncthreads();
    const uint32_t i = tile0 + off + threadIdx.x;
    const bool live = i < n;
    const uint32_t g = live ? route_dest(ops[i], keys[i], key_range, span, world) : 0xFFFFFFFFu;
    const uint32_t same = __match_any_sync(0xFFFFFFFFu, g);
    if (live && lane == __ffs(same) - 1) warp_counts[warp][g] = __popc(same);
    __syncthreads();
    if (live) {
      uint32_t pos = base_g[g];
      for (int w = 0; w < warp; ++w) pos += warp_counts[w][g];
      pos += __popc(same & ((1u << lane) - 1u));
      perm[pos] = i;
    }
    __syncthreads();
    for (uint32_t d = threadIdx.x; d < world; d += blockDim.x) {
      uint32_t t = 0;
      for (int w = 0; w < 8; ++w) t += warp_counts[w][d];
      base_g[d] += t;
    }
    __syncthreads();
  }
}

// Packs op j of the routed order; a valid op's key is rebased to its destination shard's
// local key space (key - g * span), so every shard is a GFSL over [0, its width).
__global__ void route_pack_kernel(const uint32_t *perm, const uint8_t *ops, const uint32_t *keys,
                                  const uint32_t *vals, uint32_t n, uint64_t key_range, uint64_t span,
                                  uint32_t world, uint8_t *so, uint32_t *sk, uint32_t *sv) {
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    const uint32_t i = perm[j];
    const uint8_t op = ops[i];
    const uint32_t key = keys[i];
    so[j] = op;
    sk[j] = (op <= 2 && (uint64_t)key < key_range)
                ? (uint32_t)(key - (uint64_t)route_dest(op, key, key_range, span, world) * span)
                : key;
    sv[j] = vals ? vals[i] : 0u;
  }
}

__global__ void route_unpack_kernel(const uint32_t *perm, const uint8_t *rr, uint32_t n, uint8_t *res) {
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x)
    res[perm[j]] = rr[j];
}

// Route plan with a caller-provided workspace of gfsl_internal_route_ws_bytes() (used by
// gfsl_xroute.cu, whose batches must not allocate: a stream-ordered allocation may wait on
// another shard's stream, which can be spinning in an exchange barrier).
size_t gfsl_internal_route_ws_bytes(uint64_t n, uint32_t world) {
  return (size_t)((n + ROUTE_TILE - 1) / ROUTE_TILE) * world * 4;
}
gfsl_status gfsl_internal_route_plan(const uint8_t *op_types, const uint32_t *keys, uint64_t n,
                                     uint64_t key_range, uint32_t world, uint64_t *counts,
                                     uint32_t *perm, uint32_t *tile_counts, cudaStream_t s) {
  if (n == 0) {
    CK(cudaMemsetAsync(counts, 0, world * 8, s));
    return GFSL_OK;
  }
  const uint64_t span = (key_range + world - 1) / world;
  const uint32_t tiles = (uint32_t)((n + ROUTE_TILE - 1) / ROUTE_TILE);
  route_hist_kernel<<<tiles, 256, 0, s>>>(op_types, keys, (uint32_t)n, key_range, span, world, tile_counts);
  route_scan_kernel<<<world, 1024, 0, s>>>(tile_counts, tiles, world, (unsigned long long *)counts);
  route_scatter_kernel<<<tiles, 256, 0, s>>>(op_types, keys, (uint32_t)n, key_range, span, world,
                                             tile_counts, (const unsigned long long *)counts, perm);
  CK(cudaGetLastError());
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_route_plan(const uint8_t *op_types, const uint32_t *keys, uint64_t n,
                                       uint64_t key_range, uint32_t world, uint64_t *counts,
                                       uint32_t *perm, void *stream) {
  if (world == 0 || world > MAX_WORLD || n > 0xFFFFFFFFull || !counts || (n && (!op_types || !keys || !perm))) {
    set_last_error("gfsl_route_plan: bad arguments");
    return GFSL_EINVAL;
  }
  cudaStream_t s = (cudaStream_t)stream;
  if (n == 0) {
    CK(cudaMemsetAsync(counts, 0, world * 8, s));
    return GFSL_OK;
  }
  const uint32_t tiles = (uint32_t)((n + ROUTE_TILE - 1) / ROUTE_TILE);
  uint32_t *tile_counts = nullptr;
  CK(cudaMallocAsync(&tile_counts, (size_t)tiles * world * 4, s));
  gfsl_status st = gfsl_internal_route_plan(op_types, keys, n, key_range, world, counts, perm, tile_counts, s);
  CK(cudaFreeAsync(tile_counts, s));
  return st;
}

extern "C" gfsl_status gfsl_route_pack(const uint32_t *perm, const uint8_t *op_types,
                                       const uint32_t *keys, const uint32_t *values, uint64_t n,
                                       uint64_t key_range, uint32_t world,
                                       uint8_t *send_op, uint32_t *send_key, uint32_t *send_val,
                                       void *stream) {
  if (n > 0xFFFFFFFFull || world == 0 || world > MAX_WORLD || key_range == 0) return GFSL_EINVAL;
  if (n == 0) return GFSL_OK;
  const uint64_t span = (key_range + world - 1) / world;
  const int grid = (int)std::min<uint64_t>((n + 255) / 256, 148 * 16);
  route_pack_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(perm, op_types, keys, values, (uint32_t)n,
                                                            key_range, span, world, send_op, send_key,
                                                            send_val);
  CK(cudaGetLastError());
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_route_unpack(const uint32_t *perm, const uint8_t *recv_res, uint64_t n,
                                         uint8_t *results, void *stream) {
  if (n > 0xFFFFFFFFull) return GFSL_EINVAL;
  if (n == 0) return GFSL_OK;
  const int grid = (int)std::min<uint64_t>((n + 255) / 256, 148 * 16);
  route_unpack_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(perm, recv_res, (uint32_t)n, results);
  CK(cudaGetLastError());
  return GFSL_OK;
}

// ------------------------------------------------------------------------------------
// B6 roofline microbenchmarks; measurement only, not part of a batch.

extern "C" gfsl_status gfsl_ubench(uint32_t block_bytes, uint64_t buffer_bytes, double *gather_gbps,
                                   double *chase_ns) {
  if ((block_bytes != 256 && block_bytes != 128) || buffer_bytes < (1ull << 24)) return GFSL_EINVAL;
  int dev = 0, sms = 148;
  CK(cudaGetDevice(&dev));
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  void *buf = nullptr;
  uint32_t *sink = nullptr;
  CK(cudaMalloc(&buf, buffer_bytes));
  CK(cudaMalloc(&sink, 4096 * 4));
  uint64_t nblocks = 1;
  while (nblocks * 2 * block_bytes <= buffer_bytes) nblocks *= 2;  // power of two
  ubench_fill_chase<<<sms * 8, 256>>>((uint32_t *)buf, nblocks, block_bytes / 4, 12345u);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const uint32_t iters = 256;
  const uint32_t teams_per_block = 256 / (block_bytes == 256 ? 4 : 2);
  double best_gbps = 0;
  // sweep the gathers in flight per team (4 / 8 / 16) and keep the best rate
  auto run = [&](auto kern) -> gfsl_status {
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, 256, 0);
    const int grid = sms * std::max(occ, 1);
    float best = 1e30f;
    for (int rep = 0; rep < 4; ++rep) {
      cudaEventRecord(a);
      kern<<<grid, 256>>>((const uint4 *)buf, nblocks, iters, 77u + rep, sink);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      float ms = 0;
      cudaEventElapsedTime(&ms, a, b);
      if (rep > 0) best = std::min(best, ms);
    }
    const double bytes = (double)grid * teams_per_block * iters * block_bytes;
    best_gbps = std::max(best_gbps, bytes / (best * 1e-3) / 1e9);
    return GFSL_OK;
  };
  gfsl_status rs = GFSL_OK;
  if (block_bytes == 256) {
    if ((rs = run(ubench_gather<256, 4, 4>)) != GFSL_OK) return rs;
    if ((rs = run(ubench_gather<256, 4, 8>)) != GFSL_OK) return rs;
    if ((rs = run(ubench_gather<256, 4, 16>)) != GFSL_OK) return rs;
  } else {
    if ((rs = run(ubench_gather<128, 2, 4>)) != GFSL_OK) return rs;
    if ((rs = run(ubench_gather<128, 2, 8>)) != GFSL_OK) return rs;
    if ((rs = run(ubench_gather<128, 2, 16>)) != GFSL_OK) return rs;
  }
  if (gather_gbps) *gather_gbps = best_gbps;
  // dependent chase: one warp, 2000 steps
  const uint32_t steps = 2000;
  float cms = 0;
  cudaEventRecord(a);
  if (block_bytes == 256) ubench_chase<256><<<1, 32>>>((const uint32_t *)buf, 1u, steps, sink);
  else ubench_chase<128><<<1, 32>>>((const uint32_t *)buf, 1u, steps, sink);
  cudaEventRecord(b);
  CK(cudaEventSynchronize(b));
  cudaEventElapsedTime(&cms, a, b);
  if (chase_ns) *chase_ns = cms * 1e6 / steps;
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFree(buf);
  cudaFree(sink);
  CK(cudaGetLastError());
  return GFSL_OK;
}
