/*
 * gfsl.h -- C ABI of the B200-native GFSL (GPU-Friendly SkipList) hot path.
 *
 * GFSL is the chunked skiplist of Moscovici, Cohen & Petrank (PPoPP'17 / PACT'17),
 * /root/reference/PAPER.md ("P:n" = PAPER.md line n).  It is an ordered map over
 * 32-bit unsigned keys and values (Table 4.1) with three operations:
 *   Contains(k)  -> bool                     Alg 4.1
 *   Insert(k, v) -> false iff k is present  Alg 4.5
 *   Delete(k)    -> false iff k is absent   Alg 4.11
 * and work arrives as an array of (op type, key).
 *
 * Plain C: no CUDA or torch types.  Streams are passed as `void*` holding a
 * cudaStream_t (NULL = the legacy default stream).  All functions are host functions;
 * a handle is bound to the CUDA device that was current when it was created and must
 * be used from a single host thread at a time.
 *
 * Batch semantics (reading R1, "S1 snapshot batch"): for every op of a batch
 * the result is computed against the map as it was BEFORE the batch; the map after the
 * batch is  M + {successful inserts} - {successful deletes}.  Contract: at most one
 * mutating op (Insert/Delete) per key per batch.  Outside the contract every result is
 * still the result of SOME linearization of the batch, but parity with the
 * oracle is only promised inside it -- unless the handle runs in combining mode
 * (gfsl_config.combine, reading R26), which is exact for any batch.
 *
 * Keys are valid in [0, key_range), key_range <= 2^32 - 2 (the two extremes of the
 * 32-bit internal key space are the -inf / +inf sentinels of P:203).  Any uint32 is a
 * valid value.  Invalid ops (op code > 2, or key >= key_range) get result
 * GFSL_RESULT_INVALID and have no effect.
 */
#ifndef GFSL_H_
#define GFSL_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct gfsl gfsl;
typedef gfsl *gfsl_t;

typedef enum gfsl_status {
  GFSL_OK = 0,
  GFSL_EINVAL = 1,   /* bad host argument (NULL handle, bad size, ...) */
  GFSL_ENOMEM = 2,   /* device or host allocation failed */
  GFSL_EPOOL = 3,    /* chunk pool exhausted: sticky; the structure is undefined */
  GFSL_ECUDA = 4,    /* a CUDA runtime call failed: sticky */
  GFSL_ECORRUPT = 5, /* gfsl_validate found an invariant violation */
  GFSL_ETIMEOUT = 6  /* gfsl_xr_*: a peer did not reach an exchange barrier in time: sticky */
} gfsl_status;

/* Default upper-level rebuild policy (rebuild_every = 0; R29): rebuild after the
 * batch at which the ops submitted since the last rebuild reach GFSL_REBUILD_DEFAULT_WEAR x
 * L, L = min(capacity, ops submitted up to the last rebuild) -- an upper bound on the live
 * keys, so a structure growing from empty is rebuilt at geometrically spaced sizes.  In
 * steady state with the paper's [10,10,80] mix at half fill this is about two mutations
 * per live key (every 8 batches at C1-C3, every 40 at C5). */
#define GFSL_REBUILD_DEFAULT_WEAR 5
#define GFSL_REBUILD_NEVER 0xFFFFFFFFu

/* Largest batch (ops per gfsl_batch call): the op index shares a 32-bit word with three
 * flag bits on the device.  Larger batches are split by the caller. */
#define GFSL_MAX_BATCH ((1u << 29) - 1u)

/* Op codes (the "operation type" of the op array). */
enum { GFSL_CONTAINS = 0, GFSL_INSERT = 1, GFSL_DELETE = 2 };
/* Per-op result codes. */
enum { GFSL_RESULT_FALSE = 0, GFSL_RESULT_TRUE = 1, GFSL_RESULT_INVALID = 0xFF };

typedef struct gfsl_config {
  uint32_t chunk_entries;   /* N: 16 (128-B chunks) or 32 (256-B chunks).
                               0 = 16 (fastest on B200).  MAX_LEVEL = N (path held one level per lane,
                               P:493-495). */
  uint32_t contains_team;   /* lanes per Contains team (a power of two dividing N, >= 4);
                               0 = the tuned default.  P:205 allows teams <= a warp. */
  uint32_t contains_blocks_per_sm; /* launch shape of the Contains kernel; 0 = default */
  uint32_t update_blocks_per_sm;   /* launch shape of the update kernel; 0 = default */
  uint32_t serial_updates;  /* 1 = one team applies the updates strictly in op order
                               (deterministic structure; test mode).  0 = concurrent. */
  uint32_t count_reads;     /* 1 = Contains kernel counts its chunk reads (gfsl_stats);
                               measurement builds only, slower */
  uint32_t profile_phases;  /* 1 = record CUDA events between the phases of every batch
                               (read with gfsl_phase_times) */
  uint32_t l2_window;       /* 1 = launch the search kernel with an L2 access-policy window
                               marking the upper-level pool persisting (opt-in; see
                               DESIGN.md §9 for why it is off by default) */
  uint32_t no_pdl;          /* 1 = launch the kernels of a batch without programmatic
                               dependent launch (ablation) */
  uint32_t rebuild_every;   /* after every k-th batch, rebuild the levels >= 1 from level 0
                               (R24: "compact the structure between kernel
                               launches").  0 = the default wear policy
                               (GFSL_REBUILD_DEFAULT_WEAR, R29); GFSL_REBUILD_NEVER = the
                               paper's structure dynamics only */
  uint32_t combine;         /* 1 = combining mode (R26): exact
                               for ANY batch, with no <=1-mutation-per-key contract.  The
                               Contains of a batch still see the map before the batch (S1);
                               the Insert/Delete ops are linearized in input order, so each
                               one's result follows the paper's Insert (false iff present,
                               Alg 4.5 l.2-4; no overwrite) and Delete (false iff absent,
                               Alg 4.11 l.3-5) applied one after another.  Each key's chain
                               is reduced to at most one net structural op (or an in-place
                               value write) before the update kernel.  Costs a radix sort of
                               the batch's keys.  0 = the contract mode of R1. */
  uint32_t p_chunk_q32;     /* p_chunk, the probability that a split raises a key to the
                               level above (isKeyRaised; swept in P:1068-1072), as a
                               32-bit fraction p * 2^32.  0 = p_chunk = 1, the paper's best
                               and the default (R16, R28).  The draw is a hash of
                               (raised key, level), so runs are reproducible.  The periodic
                               upper-level rebuild (rebuild_every) replaces what the raises
                               built; combine with GFSL_REBUILD_NEVER to study p_chunk. */
  uint32_t bulk;            /* the bulk path (R34; "compact the structure
                               between kernel launches"): a batch of n >= GFSL_BULK_MIN_OPS
                               ops on a map of at most U live keys with n >= GFSL_BULK_RATIO x U
                               (U = min(capacity, ops ever submitted)) is applied by sorting
                               the level-0 entries and the ops together and writing level 0
                               anew (then the upper levels are rebuilt): same S1 results, no
                               lock contention on a small structure.  0 = that rule (default),
                               GFSL_BULK_OFF = never (the paper's per-op path only),
                               GFSL_BULK_ALWAYS = every batch.  Not in serial or combining
                               mode. */
  uint32_t group;           /* chunk-grouped mutations (R40; opt-in): in concurrent
                               batches with the lazy upper levels, the Insert/Delete ops of a
                               batch that target the same bottom chunk are applied together in
                               one lock session of that chunk (one read, one merged write, one
                               split / merge decision, one release) instead of one session per
                               op.  Same results.  0 = off (default: one lock session per op,
                               the paper's protocol; measured faster on B200),
                               GFSL_GROUP_ON = grouped. */
} gfsl_config;
#define GFSL_GROUP_ON 1u
#define GFSL_BULK_OFF 1u
#define GFSL_BULK_ALWAYS 2u
#define GFSL_BULK_MIN_OPS 4096u
#define GFSL_BULK_RATIO 16u

/*
 * Create an empty GFSL (one unlocked chunk per level holding -inf with a pointer
 * to the level below; head array; per-level counters = 0).
 *   key_range : keys are valid in [0, key_range); 1 <= key_range <= 2^32 - 2.
 *   capacity  : the maximum number of live keys the caller will store; 0 = key_range.
 *               The library sizes the pre-allocated chunk pools from it.
 * Returns NULL on failure (see gfsl_last_error()).
 */
gfsl_t gfsl_create(uint64_t key_range, uint64_t capacity);
gfsl_t gfsl_create_ex(uint64_t key_range, uint64_t capacity, const gfsl_config *cfg);

/*
 * Change the run-time options of a live handle: contains_team, the blocks-per-SM launch
 * shapes, serial_updates, count_reads, profile_phases.  cfg->chunk_entries must be 0 or
 * equal to the handle's.  Takes effect for the next batch.  GFSL_EINVAL if unsupported.
 */
gfsl_status gfsl_configure(gfsl_t h, const gfsl_config *cfg);

/* Release every device resource of the handle (synchronizes the device first). */
void gfsl_destroy(gfsl_t h);

/*
 * Run one batch of n ops, asynchronously on `stream`.
 *   op_types : device pointer, n x uint8  (GFSL_CONTAINS / _INSERT / _DELETE)
 *   keys     : device pointer, n x uint32
 *   values   : device pointer, n x uint32 (read for inserts only; may be NULL, = 0)
 *   results  : device pointer, n x uint8  (written: GFSL_RESULT_*), in input order
 * All arrays belong to the caller, must be on the handle's device, and must stay valid
 * until `stream` reaches the end of the batch.  Batches on one handle are serialized in
 * issue order (the handle makes each batch wait for the previous one).
 * n <= GFSL_MAX_BATCH.
 * Returns GFSL_EINVAL for bad host arguments, or a sticky error (GFSL_EPOOL, GFSL_ECUDA)
 * raised by an earlier batch; on error nothing is enqueued.
 */
gfsl_status gfsl_batch(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                       const uint32_t *values, uint8_t *results, uint64_t n,
                       void *stream);

/*
 * gfsl_batch with the op count in DEVICE memory (no host round trip; e.g. the received
 * count of a multi-GPU exchange, gfsl_xr_recv): the batch has min(*n_dev, n_max) ops,
 * read by the kernels when they run.  n_max sizes the launch and the per-batch lists;
 * n_hint (0 = n_max) is the op count the default rebuild policy (R29) counts for this
 * batch.  The arrays must hold n_max entries.  Not available in combining or serial mode
 * (GFSL_EINVAL).  Otherwise as gfsl_batch.
 */
gfsl_status gfsl_batch_dn(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                          const uint32_t *values, uint8_t *results, uint64_t n_max,
                          const uint32_t *n_dev, uint64_t n_hint, void *stream);

/*
 * Same batch through HOST buffers (pageable or pinned): copies the ops in, runs the
 * batch, copies the results out, and returns when `results` holds them (synchronous).
 * This is the end-to-end entry point; the copies go through library-owned pinned
 * staging buffers on `stream`.
 */
gfsl_status gfsl_batch_host(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                            const uint32_t *values, uint8_t *results, uint64_t n,
                            void *stream);

/*
 * The same, asynchronous: returns once the copies and kernels are enqueued.  The inputs
 * are copied on a library-owned copy stream into one of two device staging slots, the
 * kernels run on a library-owned exec stream and the results come back on a
 * library-owned copy-out stream, so the copy-in of the next batch and the copy-out of
 * the previous one overlap the kernels of this one.  `stream` is made to wait for the
 * copy-out: `results` holds the answers once `stream` has reached this point (e.g.
 * after cudaStreamSynchronize).  The batch itself does not wait for earlier work on
 * `stream` (its inputs are host memory); it is ordered after the handle's earlier
 * batches, as every batch is.  The host buffers must stay
 * valid and unmodified until then, and must be pinned (page-locked) for the copies to
 * be asynchronous (pageable buffers still work, with synchronous copies).  `values` may
 * be NULL (all values 0; nothing copied) -- only Inserts read a value.  With
 * GFSL_ZC_VALUES=1 in the environment at gfsl_create and a mapped pinned `values`, the
 * search kernel reads each Insert's value from it directly instead of the array being
 * copied (faster only when Inserts are rare).
 */
gfsl_status gfsl_batch_host_async(gfsl_t h, const uint8_t *op_types, const uint32_t *keys,
                                  const uint32_t *values, uint8_t *results, uint64_t n,
                                  void *stream);

/* Result of gfsl_validate: the invariants of PAPER.md §4.3 and P:203. */
typedef struct gfsl_report {
  uint64_t keys;                /* live keys (bottom level, non-zombie chunks) */
  uint32_t height;              /* highest level with counter > 0 */
  uint32_t chunk_entries;       /* N */
  uint64_t chunks[32];          /* non-zombie chunks reachable per level */
  uint64_t zombies[32];         /* zombie chunks still linked per level */
  uint64_t level_keys[32];      /* real keys per level */
  int64_t  counters[32];        /* the per-level counters as stored */
  uint64_t pool_used[2];        /* chunks allocated: [0] bottom pool, [1] upper pool */
  uint64_t pool_cap[2];
  uint32_t violations;          /* bitmask: bit v-1 set = invariant Vv violated */
  uint32_t first_violation;     /* lowest violated invariant number, 0 if none */
  uint64_t restarts;            /* Contains/search restarts so far */
  uint64_t underfull;           /* non-last chunks with < floor(DSIZE/3) entries (info) */
  uint64_t reserved[3];
} gfsl_report;

/*
 * Synchronous structural check and export.  Waits for all batches, walks every level
 * from its head and checks V1-V12.  If keys_out/vals_out are
 * non-NULL (host pointers), writes up to `cap` live (key, value) pairs in ascending key
 * order and sets *count to the number of live keys.  rep and count may be NULL.
 * Returns GFSL_OK, GFSL_ECORRUPT (rep->violations says which), or an error.
 */
/*
 * Rebuild the upper levels now (R24: "compact the structure between kernel
 * launches"; with the zombie reclamation of R25 and the level-1 directory of R27), e.g.
 * after a bulk load.  A no-op if no batch mutated the structure since the last rebuild.
 * Asynchronous on `stream`, ordered after the handle's previous batch; restarts the default
 * policy's count.  Returns a sticky error of an earlier batch, if any.
 */
gfsl_status gfsl_rebuild(gfsl_t h, void *stream);

gfsl_status gfsl_validate(gfsl_t h, gfsl_report *rep, uint32_t *keys_out,
                          uint32_t *vals_out, uint64_t cap, uint64_t *count);

/*
 * Device-side structural check (B4), chunk-parallel, for structures
 * too large for the host walk of gfsl_validate (seconds at C5's 500M keys).  Synchronous.
 * Checks V1-V5, V7-V9, V12, V14 and the chain shape of every level (one live chain per
 * level from its head: one first and one last live chunk per level, every other live
 * chunk with exactly one live predecessor); with GFSL_CHECK_CROSS also V6 (no max field
 * grew) and V11 (zombie bytes unchanged) against the snapshot taken by an
 * earlier call with GFSL_CHECK_SNAPSHOT, if no upper-level rebuild (and so no reclamation)
 * ran in between.  rep (may be NULL): keys, counters, chunks[0] / zombies[0] = live /
 * zombie level-0 chunks, chunks[1] / zombies[1] = the same over all upper levels,
 * underfull, reserved[0] = level-1 stale separators (R33), reserved[1] = 1 if V6 / V11
 * were checked.  Returns GFSL_OK or GFSL_ECORRUPT (rep->violations says which).
 */
#define GFSL_CHECK_SNAPSHOT 1u
#define GFSL_CHECK_CROSS 2u
gfsl_status gfsl_check(gfsl_t h, gfsl_report *rep, uint32_t flags);

/*
 * The bottom level's live (key, value) pairs in ascending key order, into DEVICE buffers
 * keys[cap] / values[cap] (either may be NULL; both NULL = count only, no allocation).
 * *count = the number of live keys.  Collects every live level-0 chunk's entries and sorts
 * them on the device (temporary device memory ~16 B per slot); a key found in two live
 * chunks makes it return GFSL_ECORRUPT.  Synchronous.
 */
gfsl_status gfsl_export(gfsl_t h, uint32_t *keys, uint32_t *values, uint64_t cap,
                        uint64_t *count);

/* Human-readable description of the last error on this thread. */
const char *gfsl_last_error(void);

/* Counters since creation (debug statistics). */
typedef struct gfsl_stats {
  uint64_t batches, ops;
  uint64_t restarts;        /* traversal restarts (Alg 4.2 l.25) */
  uint64_t splits, merges;  /* Alg 4.9 / Alg 4.12 */
  uint64_t zombie_unlinks;  /* Alg 4.6 l.10-20 redirects */
  uint64_t lock_retries;    /* failed CAS / waits in findAndLockEnclosing (Alg 4.8) */
  uint64_t contains_reads;  /* chunk reads by Contains traversals (count_reads=1) */
  uint64_t contains_reads_l0; /* ... of which on the bottom level */
  uint64_t contains_ops;    /* Contains ops counted (count_reads=1) */
  uint64_t mutations;       /* Insert/Delete ops that changed the map */
  uint64_t kernel_launches; /* libgfsl kernels enqueued by gfsl_batch calls so far */
  uint64_t library_launches;/* library (CUB radix sort, combining mode) kernels, estimated */
  uint64_t grouped;         /* Insert/Delete ops applied in a chunk group of >= 2 (R40) */
  uint64_t zero_copy_batches; /* host-path batches whose Insert values the kernel read from
                               the caller's mapped pinned buffer (no copy) */
} gfsl_stats;
gfsl_status gfsl_get_stats(gfsl_t h, gfsl_stats *out);

/*
 * Per-phase device time of the batches enqueued since the last call (profile_phases=1):
 * ms[0] intake (memset + classify), ms[1] search kernel, ms[2] update kernel,
 * ms[3] upkeep + upper-level rebuild, ms[4] whole batches (ms must hold 5 doubles);
 * *batches = how many.  Synchronizes the device; resets the sums.
 */
gfsl_status gfsl_phase_times(gfsl_t h, double *ms, uint64_t *batches);

/* ---- test-only: raw pool access (T2 byte parity, worked-example fixtures) ----
 * Pool image layout (host memory, little endian):
 *   uint64 entries[(cap_bottom + cap_upper) * N]   chunk c at entries[c*N .. c*N+N)
 * Chunk indices [0, cap_upper) are the upper pool, [cap_upper, cap_upper+cap_bottom)
 * the bottom pool.  The meta block is: head[N] (uint32), counters[N] (int32),
 * used_bottom, used_upper (uint32).  Internal key = user key + 1; 0 = -inf;
 * 0xFFFFFFFF = +inf = EMPTY = null pointer. */
typedef struct gfsl_meta {
  uint32_t head[32];
  int32_t counters[32];
  uint32_t used_bottom, used_upper;
  uint32_t cap_bottom, cap_upper;
  uint32_t chunk_entries;
  uint32_t reserved[3];
} gfsl_meta;
gfsl_status gfsl_dump(gfsl_t h, gfsl_meta *meta, uint64_t *entries, uint64_t max_entries);
gfsl_status gfsl_load(gfsl_t h, const gfsl_meta *meta, const uint64_t *entries,
                      uint64_t n_entries);

/* ---- multi-GPU range routing (B5) ----
 * Shard g owns keys [g*ceil(R/G), min(R, (g+1)*ceil(R/G))).  The collective exchange
 * between these calls is done by the caller (torch.distributed / NCCL).
 *
 * gfsl_route_plan: per-op destination and stable order.  Writes counts[G] (device,
 *   uint64, number of ops for each destination) and perm[n] (device, uint32: perm[j] =
 *   input index of the j-th op in destination-major, input-stable order).  Invalid keys
 *   are routed to shard 0, which reports them invalid.
 * gfsl_route_pack: packs ops in perm order into send_op/send_key/send_val; a valid op's
 *   key is rebased to its destination's LOCAL key space (key - g * ceil(key_range/world)),
 *   so shard g is a GFSL created over [0, its width); invalid ops keep their key.
 * gfsl_route_unpack: results[perm[j]] = recv_res[j].
 */
gfsl_status gfsl_route_plan(const uint8_t *op_types, const uint32_t *keys, uint64_t n,
                            uint64_t key_range, uint32_t world, uint64_t *counts,
                            uint32_t *perm, void *stream);
gfsl_status gfsl_route_pack(const uint32_t *perm, const uint8_t *op_types,
                            const uint32_t *keys, const uint32_t *values, uint64_t n,
                            uint64_t key_range, uint32_t world,
                            uint8_t *send_op, uint32_t *send_key, uint32_t *send_val,
                            void *stream);
gfsl_status gfsl_route_unpack(const uint32_t *perm, const uint8_t *recv_res, uint64_t n,
                              uint8_t *results, void *stream);

/* ---- fused multi-GPU exchange over peer memory ----
 * The same range partition as above, without NCCL on the data path: every rank owns one
 * device WINDOW (receive arrays for world * max_slice ops, a double-buffered count matrix,
 * barrier flags) that the peers map through CUDA IPC (one node, NVLink/NVSwitch).  The
 * push kernel stores each routed op once, straight from the caller's arrays into its
 * destination's window, its key rebased to the destination's local key space (as
 * gfsl_route_pack: shard g's GFSL is created over [0, its width)); the local shard runs
 * gfsl_batch_dn on its window with the received count read on the device (no host
 * synchronisation anywhere in a batch); the pull kernel loads every result straight from
 * the destination's window into the caller's order.
 * Ranks synchronise with device-side barriers (release/acquire flags at system scope),
 * each spin bounded by `timeout_ms`; an expired barrier makes the handle sticky-failed
 * (GFSL_ETIMEOUT) and the batch's results GFSL_RESULT_INVALID.  The semantics are those of
 * gfsl_batch on one map holding every shard (S1 per shard = S1 globally: a key lives on one
 * shard and every op touches one key).
 *
 * gfsl_xr_create: this rank's window on the current device.  rank < world <= 64;
 *   key_range as gfsl_create; max_slice = the largest n any rank will pass (the receive
 *   arrays hold world * max_slice <= GFSL_MAX_BATCH ops, all of which the local batch may
 *   receive); timeout_ms 0 = 60 s.  NULL on failure.
 * gfsl_xr_export: writes the window's CUDA IPC handle (GFSL_XR_HANDLE_BYTES bytes, host).
 * gfsl_xr_attach: maps peer `peer`'s window from its exported handle (another process).
 * gfsl_xr_attach_local: uses the window of another handle of THIS process (one process
 *   driving several shards, e.g. on one GPU; a handle on another device gets peer access).
 *   Every rank must attach every peer before its first batch.
 * A batch is collective over all ranks.  Each rank makes these calls in this order; one
 * process driving several shards makes each call for every shard before the next call
 * (the barriers are split into arrive and wait launches, so this order never waits on a
 * launch that is not yet enqueued):
 *   gfsl_xr_send(ops of this rank's slice, n <= max_slice, stream): route plan, count row
 *     into every peer, arrive.  Enqueue only; the caller's arrays must stay valid until the
 *     stream passes the batch.
 *   gfsl_xr_push(stream): wait for all counts, push the ops into the peers' windows, arrive.
 *   gfsl_xr_recv(..., stream): enqueues the wait for everyone's pushes and returns (without
 *     waiting) the window's receive arrays (device pointers, owned by the handle, valid
 *     until gfsl_xr_finish): op/key/val to feed the local shard, `results` for its answers,
 *     their capacity *n_cap and *n_dev, the device word that holds the received count once
 *     the stream has passed the count exchange.
 *   gfsl_xr_local(local, n_hint, stream): the local shard's batch on the window
 *     (gfsl_batch_dn with the device count; n_hint = the expected count, e.g. this rank's
 *     slice size, paces the rebuild policy).  If it fails (e.g. a sticky GFSL_EPOOL) the
 *     received ops are answered GFSL_RESULT_INVALID and its error is returned; the caller
 *     must still make the remaining calls, so that no peer waits for this rank.
 *   gfsl_xr_done(stream): arrive (this shard's results are written).
 *   gfsl_xr_finish(results[n] of the slice, device, stream): wait, then the pull.
 * gfsl_xr_batch: all of the above, for one shard per process; a local failure is returned
 *   after the exchange has completed.
 * An expired barrier is reported by a later call on the handle (the error word reaches
 * host memory asynchronously); gfsl_xr_status checks synchronously: GFSL_ETIMEOUT once any
 * barrier of this handle has expired.
 * gfsl_xr_window: the window's base pointer and size (tests). */
typedef struct gfsl_xr gfsl_xr;
typedef gfsl_xr *gfsl_xr_t;
#define GFSL_XR_HANDLE_BYTES 64
gfsl_xr_t gfsl_xr_create(uint32_t rank, uint32_t world, uint64_t key_range, uint64_t max_slice,
                         uint64_t timeout_ms);
void gfsl_xr_destroy(gfsl_xr_t x);
gfsl_status gfsl_xr_export(gfsl_xr_t x, void *handle);
gfsl_status gfsl_xr_attach(gfsl_xr_t x, uint32_t peer, const void *handle);
gfsl_status gfsl_xr_attach_local(gfsl_xr_t x, uint32_t peer, gfsl_xr_t other);
gfsl_status gfsl_xr_send(gfsl_xr_t x, const uint8_t *op_types, const uint32_t *keys,
                         const uint32_t *values, uint64_t n, void *stream);
gfsl_status gfsl_xr_push(gfsl_xr_t x, void *stream);
gfsl_status gfsl_xr_recv(gfsl_xr_t x, const uint8_t **op_types, const uint32_t **keys,
                         const uint32_t **values, uint8_t **results, uint64_t *n_cap,
                         const uint32_t **n_dev, void *stream);
gfsl_status gfsl_xr_local(gfsl_xr_t x, gfsl_t local, uint64_t n_hint, void *stream);
gfsl_status gfsl_xr_done(gfsl_xr_t x, void *stream);
gfsl_status gfsl_xr_finish(gfsl_xr_t x, uint8_t *results, void *stream);
gfsl_status gfsl_xr_batch(gfsl_xr_t x, gfsl_t local, const uint8_t *op_types,
                          const uint32_t *keys, const uint32_t *values, uint8_t *results,
                          uint64_t n, void *stream);
gfsl_status gfsl_xr_status(gfsl_xr_t x);
gfsl_status gfsl_xr_window(gfsl_xr_t x, void **base, uint64_t *bytes);

/* ---- measurement: the roofline denominators of SURVEY 8(d) (B6) ----
 * gfsl_ubench: random aligned `block_bytes` (256 or 128) gathers over a fresh device buffer
 * of `buffer_bytes` (choose >> L2), issued like the search kernel's chunk reads (teams of
 * 4 / 2 lanes, 32-B vector loads), many independent gathers per warp: *gather_gbps =
 * R_rand(block).  *chase_ns = the latency of one dependent block gather.  Synchronous;
 * allocates and frees the buffer itself. */
gfsl_status gfsl_ubench(uint32_t block_bytes, uint64_t buffer_bytes, double *gather_gbps,
                        double *chase_ns);

#ifdef __cplusplus
}
#endif
#endif /* GFSL_H_ */
