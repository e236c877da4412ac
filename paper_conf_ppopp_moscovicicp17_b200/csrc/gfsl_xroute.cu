// gfsl_xroute.cu -- fused multi-GPU exchange over peer memory.
//
// The key space is range-partitioned: shard g owns [g*ceil(R/G),
// (g+1)*ceil(R/G)), and each rank holds one slice of every global batch.  The NCCL router
// (router.py) packs each op into a send buffer, exchanges counts, ops, keys and values with
// four all-to-alls and the results with a fifth, every payload passing through HBM twice.
// Here each rank owns one WINDOW (one cudaMalloc, shared with the peers through CUDA IPC
// on one node), and the route kernels move the payload themselves:
//
//   route_plan (gfsl.cu)    per-op destination, stable destination-major order
//   xr_counts_kernel        this rank's count row into every peer's count matrix; arrive
//   xr_wait_counts_kernel   wait; n_recv = this rank's column of the matrix (read back)
//   xr_push_kernel          each op is stored ONCE, straight from the caller's arrays into
//                           its destination's receive arrays (NVLink stores), at the offset
//                           the replicated count matrix gives (sources in rank order); arrive
//   xr_wait_kernel          everyone's pushes are complete
//   gfsl_batch              the local shard runs on its receive arrays (S1 on the shard)
//   xr_arrive_kernel        this rank's results are written
//   xr_wait_kernel          everyone's results are written
//   xr_pull_kernel          each rank loads its ops' results from the destinations' result
//                           arrays (NVLink loads) straight into the caller's order
//
// The barriers are split-phase (arrive and wait are separate launches, so one process can
// drive several shards in phase order even when its streams share one hardware queue).
// No host round trip: the received count stays on the device (the window's n_recv word),
// and the local shard runs gfsl_batch_dn, whose kernels read their op count from there.
// Keys arrive rebased to the destination's local key space (key - g * span), so each shard
// is a GFSL over [0, its width) with bitmaps and directory sized for its own range.  Every
// barrier spin is bounded by a timeout (%globaltimer); on expiry the rank raises a sticky
// error flag, the remaining kernels of the batch do nothing (n_recv = 0, results INVALID),
// and a later host call returns GFSL_ETIMEOUT (gfsl_xr_status checks at once).
//
// Reuse of the windows across batches: a rank writes a peer's receive arrays only after
// the first barrier of the next batch, which every rank reaches only after its pull of the
// previous batch; the count matrix is double-buffered by batch parity, because a peer may
// still be pulling (and reading its matrix) while a fast rank writes the next counts.
#include "../../include/gfsl.h"

#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <string>

// gfsl.cu
void gfsl_internal_set_error(const std::string &s);
size_t gfsl_internal_route_ws_bytes(uint64_t n, uint32_t world);
gfsl_status gfsl_internal_route_plan(const uint8_t *op_types, const uint32_t *keys, uint64_t n,
                                     uint64_t key_range, uint32_t world, uint64_t *counts,
                                     uint32_t *perm, uint32_t *tile_counts, cudaStream_t s);
extern "C" gfsl_status gfsl_batch_dn(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                                     const uint32_t *values, uint8_t *results, uint64_t n_max,
                                     const uint32_t *n_dev, uint64_t n_hint, void *stream);

#define XCK(call)                                                                     \
  do {                                                                                \
    cudaError_t e_ = (call);                                                          \
    if (e_ != cudaSuccess) {                                                          \
      gfsl_internal_set_error(std::string(#call) + ": " + cudaGetErrorString(e_));    \
      return GFSL_ECUDA;                                                              \
    }                                                                                 \
  } while (0)

namespace {

constexpr uint32_t XR_MAX_WORLD = 64;  // as the route kernels (gfsl.cu MAX_WORLD)

// Window layout; identical on every rank (same world and max_slice).
struct Layout {
  size_t flags;   // u64[XR_MAX_WORLD]: flags[s] = the last barrier epoch rank s arrived at
  size_t cnt;     // u32[2][world][world]: cnt[parity][s][g] = ops rank s sends to rank g
  size_t misc;    // u64 n_recv; u32 err; u32 n_recv (the local batch's device count)
  size_t op, key, val, res;  // receive arrays, cap = world * max_slice entries each
  size_t total;
};

inline size_t up256(size_t x) { return (x + 255) & ~(size_t)255; }

Layout make_layout(uint32_t world, uint64_t cap) {
  Layout L{};
  size_t o = 0;
  L.flags = o; o = up256(o + XR_MAX_WORLD * 8);
  L.cnt = o;   o = up256(o + (size_t)2 * world * world * 4);
  L.misc = o;  o = up256(o + 16);
  L.op = o;    o = up256(o + cap);
  L.key = o;   o = up256(o + cap * 4);
  L.val = o;   o = up256(o + cap * 4);
  L.res = o;   o = up256(o + cap);
  L.total = o;
  return L;
}

struct XrArgs {
  char *const *peer;  // device table: window base of every rank (own included)
  uint64_t key_range, span;  // the global key space and the shard width ceil(R / world)
  uint32_t rank, world, parity;
  uint64_t epoch;      // epoch of THIS barrier (counts / barrier kernels)
  uint64_t timeout_ns;
  Layout L;
};

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_sys_u32(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_sys_u8(const uint8_t *p) {
  uint16_t v;
  asm volatile("ld.relaxed.sys.global.u8 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ uint32_t *err_word(const XrArgs &a, char *base) {
  return (uint32_t *)(base + a.L.misc + 8);
}
__device__ __forceinline__ uint32_t *cnt_of(const XrArgs &a, char *base) {
  return (uint32_t *)(base + a.L.cnt) + (size_t)a.parity * a.world * a.world;
}

// Split-phase device barrier.  Arrive (release: everything this rank wrote before, in this
// or an earlier kernel of the stream, is visible to a peer that observes the flag) and wait
// (acquire) are separate launches, so that one process may drive several shards through
// streams that the hardware serialises: every wait is enqueued after every matching arrive.
__device__ void xr_arrive(const XrArgs &a) {
  if (threadIdx.x < a.world) st_release_sys((uint64_t *)(a.peer[threadIdx.x] + a.L.flags) + a.rank, a.epoch);
}
// Threads t < world each wait for rank t; bounded by the timeout.  Returns false (for the
// calling thread) if the exchange has failed.
__device__ bool xr_wait(const XrArgs &a) {
  char *own = a.peer[a.rank];
  const uint32_t t = threadIdx.x;
  if (t < a.world) {
    const uint64_t *f = (const uint64_t *)(own + a.L.flags) + t;
    const uint64_t t0 = globaltimer();
    while (ld_acquire_sys(f) < a.epoch) {
      if (*(volatile uint32_t *)err_word(a, own) != 0 || globaltimer() - t0 > a.timeout_ns) {
        atomicOr(err_word(a, own), 1u << (t & 31));
        break;
      }
      __nanosleep(256);
    }
  }
  return *(volatile uint32_t *)err_word(a, own) == 0;
}

// (1) this rank's count row into every peer's matrix, then arrive
__global__ void xr_counts_kernel(XrArgs a, const unsigned long long *counts) {
  __shared__ uint32_t c[XR_MAX_WORLD];
  if (threadIdx.x < a.world) c[threadIdx.x] = (uint32_t)counts[threadIdx.x];
  __syncthreads();
  for (uint32_t x = threadIdx.x; x < a.world * a.world; x += blockDim.x) {
    const uint32_t p = x / a.world, g = x % a.world;
    cnt_of(a, a.peer[p])[a.rank * a.world + g] = c[g];
  }
  __syncthreads();
  if (threadIdx.x == 0) __threadfence_system();
  __syncthreads();
  xr_arrive(a);
}

// (2) wait for every count row; n_recv = column `rank` of the matrix (0 if the exchange
// failed: the local batch then has no ops)
__global__ void xr_wait_counts_kernel(XrArgs a) {
  const bool ok = xr_wait(a);
  __syncthreads();
  if (threadIdx.x == 0) {
    char *own = a.peer[a.rank];
    uint64_t n = 0;
    const uint32_t *m = cnt_of(a, own);
    if (ok && *(volatile uint32_t *)err_word(a, own) == 0)
      for (uint32_t s = 0; s < a.world; ++s) n += ld_relaxed_sys_u32(m + s * a.world + a.rank);
    *(unsigned long long *)(own + a.L.misc) = n;
    *(uint32_t *)(own + a.L.misc + 12) = (uint32_t)n;
  }
}

__global__ void xr_arrive_kernel(XrArgs a) {
  if (threadIdx.x == 0) __threadfence_system();
  __syncthreads();
  xr_arrive(a);
}

__global__ void xr_wait_kernel(XrArgs a) { xr_wait(a); }

// Per-block tables of the routed order: seg[g] = first routed position of destination g
// (this rank's counts), dst[g] = where this rank's ops start in g's receive arrays (the
// counts of the lower ranks to g).  Returns false if the exchange already failed.
__device__ bool xr_tables(const XrArgs &a, uint32_t *seg, uint32_t *dst) {
  char *own = a.peer[a.rank];
  const uint32_t *m = cnt_of(a, own);
  if (threadIdx.x == 0) {
    uint32_t run = 0;
    for (uint32_t g = 0; g < a.world; ++g) {
      seg[g] = run;
      run += ld_relaxed_sys_u32(m + a.rank * a.world + g);
      uint32_t d = 0;
      for (uint32_t s = 0; s < a.rank; ++s) d += ld_relaxed_sys_u32(m + s * a.world + g);
      dst[g] = d;
    }
    seg[a.world] = run;
  }
  __syncthreads();
  return *(volatile uint32_t *)err_word(a, own) == 0;
}

__device__ __forceinline__ uint32_t seg_of(const uint32_t *seg, uint32_t world, uint32_t j) {
  uint32_t lo = 0, hi = world;  // seg[lo] <= j < seg[hi]
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (seg[mid] <= j) lo = mid; else hi = mid;
  }
  return lo;
}

// (4) push: routed position j -> destination g, slot dst[g] + (j - seg[g]) of g's arrays
__global__ void __launch_bounds__(256) xr_push_kernel(XrArgs a, const uint32_t *perm, uint32_t n,
                                                      const uint8_t *op, const uint32_t *key,
                                                      const uint32_t *val) {
  __shared__ uint32_t seg[XR_MAX_WORLD + 1], dst[XR_MAX_WORLD];
  __shared__ char *base[XR_MAX_WORLD];
  if (threadIdx.x < a.world) base[threadIdx.x] = a.peer[threadIdx.x];
  if (!xr_tables(a, seg, dst)) return;
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    const uint32_t g = seg_of(seg, a.world, j);
    const size_t slot = (size_t)dst[g] + (j - seg[g]);
    const uint32_t i = perm[j];
    char *b = base[g];
    const uint8_t o = op[i];
    const uint32_t k = key[i];
    ((uint8_t *)(b + a.L.op))[slot] = o;
    // a valid op's key in its shard's local key space; invalid ones (routed to shard 0)
    // stay out of range there
    ((uint32_t *)(b + a.L.key))[slot] = (o <= 2 && (uint64_t)k < a.key_range) ? (uint32_t)(k - (uint64_t)g * a.span) : k;
    ((uint32_t *)(b + a.L.val))[slot] = val ? val[i] : 0u;
  }
  __threadfence_system();
}

// (6) pull: results[perm[j]] = g's result slot of routed position j
__global__ void __launch_bounds__(256) xr_pull_kernel(XrArgs a, const uint32_t *perm, uint32_t n,
                                                      uint8_t *res) {
  __shared__ uint32_t seg[XR_MAX_WORLD + 1], dst[XR_MAX_WORLD];
  __shared__ char *base[XR_MAX_WORLD];
  if (threadIdx.x < a.world) base[threadIdx.x] = a.peer[threadIdx.x];
  const bool ok = xr_tables(a, seg, dst);
  for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
    const uint32_t g = seg_of(seg, a.world, j);
    const size_t slot = (size_t)dst[g] + (j - seg[g]);
    res[perm[j]] = ok ? (uint8_t)ld_relaxed_sys_u8((const uint8_t *)(base[g] + a.L.res) + slot)
                      : (uint8_t)GFSL_RESULT_INVALID;
  }
}

}  // namespace

struct gfsl_xr {
  int device = 0;
  int sms = 148;
  uint32_t rank = 0, world = 1;
  uint64_t key_range = 0, max_slice = 0, cap = 0;
  uint64_t timeout_ns = 0;
  Layout L{};
  char *win = nullptr;
  char *peer[XR_MAX_WORLD] = {};
  bool ipc_opened[XR_MAX_WORLD] = {};
  char **d_peer = nullptr;
  unsigned long long *d_counts = nullptr;
  uint32_t *d_perm = nullptr;
  uint32_t *d_tiles = nullptr;           // route-plan workspace
  unsigned long long *h_misc = nullptr;  // pinned: n_recv, err
  cudaEvent_t ev_counts = nullptr;
  uint64_t epoch = 0;
  uint64_t batches = 0;
  uint64_t n_cur = 0;
  const uint8_t *in_op = nullptr;
  const uint32_t *in_key = nullptr, *in_val = nullptr;
  int stage = 0;  // 0 idle, 1 sent, 2 pushed, 3 received, 4 done
  bool sticky = false;
};

static gfsl_status upload_table(gfsl_xr *x);

static XrArgs xr_args(gfsl_xr *x, uint64_t epoch) {
  XrArgs a{};
  a.peer = x->d_peer;
  a.key_range = x->key_range;
  a.span = (x->key_range + x->world - 1) / x->world;
  a.rank = x->rank;
  a.world = x->world;
  a.parity = (uint32_t)(x->batches & 1);
  a.epoch = epoch;
  a.timeout_ns = x->timeout_ns;
  a.L = x->L;
  return a;
}

extern "C" gfsl_xr_t gfsl_xr_create(uint32_t rank, uint32_t world, uint64_t key_range,
                                    uint64_t max_slice, uint64_t timeout_ms) {
  if (world == 0 || world > XR_MAX_WORLD || rank >= world || key_range == 0 ||
      key_range > 0xFFFFFFFEull || max_slice == 0 || max_slice > GFSL_MAX_BATCH ||
      (uint64_t)world * max_slice > GFSL_MAX_BATCH) {  // the local batch takes them all
    gfsl_internal_set_error("gfsl_xr_create: bad arguments");
    return nullptr;
  }
  gfsl_xr *x = new gfsl_xr();
  x->rank = rank;
  x->world = world;
  x->key_range = key_range;
  x->max_slice = max_slice;
  x->cap = (uint64_t)world * max_slice;
  x->timeout_ns = (timeout_ms ? timeout_ms : 60000ull) * 1000000ull;
  x->L = make_layout(world, x->cap);
  auto fail = [&](const char *what, cudaError_t e) -> gfsl_xr_t {
    gfsl_internal_set_error(std::string("gfsl_xr_create: ") + what + ": " + cudaGetErrorString(e));
    gfsl_xr_destroy(x);
    return nullptr;
  };
  cudaError_t e;
  if ((e = cudaGetDevice(&x->device)) != cudaSuccess) return fail("cudaGetDevice", e);
  cudaDeviceGetAttribute(&x->sms, cudaDevAttrMultiProcessorCount, x->device);
  if ((e = cudaMalloc(&x->win, x->L.total)) != cudaSuccess) return fail("window", e);
  if ((e = cudaMemset(x->win, 0, x->L.misc + 16)) != cudaSuccess) return fail("memset", e);
  if ((e = cudaMalloc(&x->d_peer, XR_MAX_WORLD * sizeof(char *))) != cudaSuccess) return fail("peer table", e);
  if ((e = cudaMalloc(&x->d_counts, XR_MAX_WORLD * 8)) != cudaSuccess) return fail("counts", e);
  if ((e = cudaMalloc(&x->d_perm, max_slice * 4)) != cudaSuccess) return fail("perm", e);
  if ((e = cudaMalloc(&x->d_tiles, gfsl_internal_route_ws_bytes(max_slice, world))) != cudaSuccess)
    return fail("route workspace", e);
  if ((e = cudaMallocHost(&x->h_misc, 16)) != cudaSuccess) return fail("pinned", e);
  memset(x->h_misc, 0, 16);
  if ((e = cudaEventCreateWithFlags(&x->ev_counts, cudaEventDisableTiming)) != cudaSuccess) return fail("event", e);
  if ((e = cudaDeviceSynchronize()) != cudaSuccess) return fail("sync", e);
  x->peer[rank] = x->win;
  if (upload_table(x) != GFSL_OK) return fail("peer table", cudaGetLastError());
  return x;
}

extern "C" void gfsl_xr_destroy(gfsl_xr_t x) {
  if (!x) return;
  cudaDeviceSynchronize();
  for (uint32_t p = 0; p < XR_MAX_WORLD; ++p)
    if (x->ipc_opened[p]) cudaIpcCloseMemHandle(x->peer[p]);
  cudaFree(x->win);
  cudaFree(x->d_peer);
  cudaFree(x->d_counts);
  cudaFree(x->d_perm);
  cudaFree(x->d_tiles);
  if (x->h_misc) cudaFreeHost(x->h_misc);
  if (x->ev_counts) cudaEventDestroy(x->ev_counts);
  delete x;
}

// The device copy of the window table is written here, at setup, never inside a batch: a
// synchronous copy waits for every blocking stream of the context, and another shard's
// stream of this process may be spinning in an exchange barrier then.
static gfsl_status upload_table(gfsl_xr *x) {
  XCK(cudaMemcpy(x->d_peer, x->peer, sizeof(x->peer), cudaMemcpyHostToDevice));
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_xr_export(gfsl_xr_t x, void *handle) {
  if (!x || !handle) return GFSL_EINVAL;
  static_assert(sizeof(cudaIpcMemHandle_t) <= GFSL_XR_HANDLE_BYTES, "IPC handle size");
  cudaIpcMemHandle_t h;
  XCK(cudaIpcGetMemHandle(&h, x->win));
  memset(handle, 0, GFSL_XR_HANDLE_BYTES);
  memcpy(handle, &h, sizeof(h));
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_xr_attach(gfsl_xr_t x, uint32_t peer, const void *handle) {
  if (!x || !handle || peer >= x->world || peer == x->rank || x->stage != 0) return GFSL_EINVAL;
  if (x->ipc_opened[peer]) {
    cudaIpcCloseMemHandle(x->peer[peer]);
    x->ipc_opened[peer] = false;
  }
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof(h));
  void *p = nullptr;
  XCK(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
  x->peer[peer] = (char *)p;
  x->ipc_opened[peer] = true;
  return upload_table(x);
}

extern "C" gfsl_status gfsl_xr_attach_local(gfsl_xr_t x, uint32_t peer, gfsl_xr_t other) {
  if (!x || !other || peer >= x->world || other->rank != peer || other->world != x->world ||
      other->max_slice != x->max_slice || x->stage != 0)
    return GFSL_EINVAL;
  if (other->device != x->device) {
    cudaError_t e = cudaDeviceEnablePeerAccess(other->device, 0);
    if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) XCK(e);
    cudaGetLastError();
  }
  x->peer[peer] = other->win;
  return upload_table(x);
}

static gfsl_status xr_sticky(gfsl_xr *x) {
  if (!x->sticky && ((volatile const uint32_t *)x->h_misc)[2] != 0) x->sticky = true;
  if (x->sticky) {
    gfsl_internal_set_error("gfsl_xr: an earlier exchange timed out (sticky)");
    return GFSL_ETIMEOUT;
  }
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_xr_send(gfsl_xr_t x, const uint8_t *op_types, const uint32_t *keys,
                                    const uint32_t *values, uint64_t n, void *stream) {
  if (!x || x->stage != 0 || n > x->max_slice || (n && (!op_types || !keys))) {
    gfsl_internal_set_error("gfsl_xr_send: bad arguments or call order");
    return GFSL_EINVAL;
  }
  gfsl_status st = xr_sticky(x);
  if (st != GFSL_OK) return st;
  for (uint32_t p = 0; p < x->world; ++p)
    if (!x->peer[p]) {
      gfsl_internal_set_error("gfsl_xr_send: peer window not attached");
      return GFSL_EINVAL;
    }
  cudaStream_t s = (cudaStream_t)stream;
  st = gfsl_internal_route_plan(op_types, keys, n, x->key_range, x->world, (uint64_t *)x->d_counts,
                                x->d_perm, x->d_tiles, s);
  if (st != GFSL_OK) return st;
  xr_counts_kernel<<<1, 256, 0, s>>>(xr_args(x, ++x->epoch), x->d_counts);
  XCK(cudaGetLastError());
  x->n_cur = n;
  x->in_op = op_types;
  x->in_key = keys;
  x->in_val = values;
  x->stage = 1;
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_xr_push(gfsl_xr_t x, void *stream) {
  if (!x || x->stage != 1) {
    gfsl_internal_set_error("gfsl_xr_push: call order");
    return GFSL_EINVAL;
  }
  cudaStream_t s = (cudaStream_t)stream;
  xr_wait_counts_kernel<<<1, 64, 0, s>>>(xr_args(x, x->epoch));
  if (x->n_cur) {
    const int grid = (int)std::min<uint64_t>((x->n_cur + 255) / 256, (uint64_t)x->sms * 8);
    xr_push_kernel<<<grid, 256, 0, s>>>(xr_args(x, x->epoch), x->d_perm, (uint32_t)x->n_cur, x->in_op,
                                        x->in_key, x->in_val);
  }
  xr_arrive_kernel<<<1, 64, 0, s>>>(xr_args(x, ++x->epoch));
  XCK(cudaGetLastError());
  x->stage = 2;
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_xr_recv(gfsl_xr_t x, const uint8_t **op_types, const uint32_t **keys,
                                    const uint32_t **values, uint8_t **results, uint64_t *n_cap,
                                    const uint32_t **n_dev, void *stream) {
  if (!x || x->stage != 2 || !n_cap || !n_dev) {
    gfsl_internal_set_error("gfsl_xr_recv: bad arguments or call order");
    return GFSL_EINVAL;
  }
  xr_wait_kernel<<<1, 64, 0, (cudaStream_t)stream>>>(xr_args(x, x->epoch));
  XCK(cudaGetLastError());
  x->stage = 3;
  *n_cap = x->cap;
  *n_dev = (const uint32_t *)(x->win + x->L.misc + 12);
  if (op_types) *op_types = (const uint8_t *)(x->win + x->L.op);
  if (keys) *keys = (const uint32_t *)(x->win + x->L.key);
  if (values) *values = (const uint32_t *)(x->win + x->L.val);
  if (results) *results = (uint8_t *)(x->win + x->L.res);
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_xr_done(gfsl_xr_t x, void *stream) {
  if (!x || x->stage != 3) {
    gfsl_internal_set_error("gfsl_xr_done: call order");
    return GFSL_EINVAL;
  }
  xr_arrive_kernel<<<1, 64, 0, (cudaStream_t)stream>>>(xr_args(x, ++x->epoch));
  XCK(cudaGetLastError());
  x->stage = 4;
  return GFSL_OK;
}

extern "C" gfsl_status gfsl_xr_finish(gfsl_xr_t x, uint8_t *results, void *stream) {
  if (!x || x->stage != 4 || (x->n_cur && !results)) {
    gfsl_internal_set_error("gfsl_xr_finish: bad arguments or call order");
    return GFSL_EINVAL;
  }
  cudaStream_t s = (cudaStream_t)stream;
  xr_wait_kernel<<<1, 64, 0, s>>>(xr_args(x, x->epoch));
  if (x->n_cur) {
    const int grid = (int)std::min<uint64_t>((x->n_cur + 255) / 256, (uint64_t)x->sms * 8);
    xr_pull_kernel<<<grid, 256, 0, s>>>(xr_args(x, x->epoch), x->d_perm, (uint32_t)x->n_cur, results);
  }
  // the error word goes to pinned host memory asynchronously: a timeout of this batch makes
  // a later call fail (gfsl_xr_status checks synchronously)
  XCK(cudaMemcpyAsync(x->h_misc, x->win + x->L.misc, 16, cudaMemcpyDeviceToHost, s));
  XCK(cudaGetLastError());
  x->batches += 1;
  x->stage = 0;
  return xr_sticky(x);
}

extern "C" gfsl_status gfsl_xr_status(gfsl_xr_t x) {
  if (!x) return GFSL_EINVAL;
  if (!x->sticky) {
    uint32_t err = 0;
    XCK(cudaMemcpy(&err, x->win + x->L.misc + 8, 4, cudaMemcpyDeviceToHost));
    if (err) x->sticky = true;
  }
  return xr_sticky(x);
}

extern "C" gfsl_status gfsl_xr_local(gfsl_xr_t x, gfsl_t local, uint64_t n_hint, void *stream) {
  if (!x || !local || x->stage != 3) {
    gfsl_internal_set_error("gfsl_xr_local: bad arguments or call order");
    return GFSL_EINVAL;
  }
  uint8_t *rr = (uint8_t *)(x->win + x->L.res);
  gfsl_status st = gfsl_batch_dn(local, (const uint8_t *)(x->win + x->L.op), (const uint32_t *)(x->win + x->L.key),
                                 (const uint32_t *)(x->win + x->L.val), rr, x->cap,
                                 (const uint32_t *)(x->win + x->L.misc + 12), n_hint ? n_hint : 1, stream);
  if (st != GFSL_OK) {
    // the peers still pull their results from this window: answer them INVALID; the caller
    // then takes part in the remaining barriers (done, finish) so no peer waits for it
    cudaMemsetAsync(rr, 0xFF, x->cap, (cudaStream_t)stream);
  }
  return st;
}

extern "C" gfsl_status gfsl_xr_batch(gfsl_xr_t x, gfsl_t local, const uint8_t *op_types,
                                     const uint32_t *keys, const uint32_t *values, uint8_t *results,
                                     uint64_t n, void *stream) {
  if (!x || !local) return GFSL_EINVAL;
  gfsl_status st = gfsl_xr_send(x, op_types, keys, values, n, stream);
  if (st != GFSL_OK) return st;
  const uint8_t *ro;
  const uint32_t *rk, *rv, *nd;
  uint8_t *rr;
  uint64_t cap = 0;
  if ((st = gfsl_xr_push(x, stream)) != GFSL_OK) return st;
  if ((st = gfsl_xr_recv(x, &ro, &rk, &rv, &rr, &cap, &nd, stream)) != GFSL_OK) return st;
  // the local shard; the expected count (this rank's own slice) paces its rebuild policy
  const gfsl_status local_st = gfsl_xr_local(x, local, n, stream);
  if ((st = gfsl_xr_done(x, stream)) != GFSL_OK) return st;
  st = gfsl_xr_finish(x, results, stream);
  return local_st != GFSL_OK ? local_st : st;
}

extern "C" gfsl_status gfsl_xr_window(gfsl_xr_t x, void **base, uint64_t *bytes) {
  if (!x) return GFSL_EINVAL;
  if (base) *base = x->win;
  if (bytes) *bytes = x->L.total;
  return GFSL_OK;
}
