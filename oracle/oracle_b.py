"""Oracle-B: the GFSL algorithm of PAPER.md §4, step by step, one team, no concurrency.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Plain Python, written from the paper
and the readings R1-R22 of DESIGN.md §3; it shares no code with the CUDA path.  It exists
because the exact *structure* (not only the results) is defined for a single team: the
GPU's serial mode (one team applies the batch's updates in op order) must produce the
same pool, entry for entry, except the lock versions (test_gpu_structure.py).

Pinned by (tests/test_oracle_b.py, tests/test_oracle_b_pins.py): the worked examples of
Fig 4.1-4.6 on the
fixtures of SURVEY Appendix B, including the restart of Contains(70) under two injected
Deletes and the printed intermediate state of the merge write order
(F = [24, 26, EMPTY, 26]); a hand-worked splitRemove; Oracle-A's results
and final sets on random sequences; the invariants V1-V12 after every op; the special
case "one chunk holds everything" (a sorted array).  The B200 design's between-batch
steps (upkeep R23, rebuild R24, reclamation R25) are pinned by properties checked
against plain re-derivations written in the tests (not by this model's own code).

What this model does NOT contain: any scheduling policy of the GPU library (the wear
rule R29 is a GPU-side policy; the model rebuilds only on a fixed period or on demand),
and any kernel shortcut (a Delete checks every level from the current height, Alg 4.11
l.12-16, instead of the kernel's start at the level where its snapshot saw k).

Layout (Fig 3.1): chunk = N entries of 64 bits; DATA i = key | value << 32,
NEXT = max | next << 32, LOCK = state | version << 32.  Internal key = user key + 1;
-inf = 0; +inf = EMPTY = null = 0xFFFFFFFF (R3).  Level-0 chunks come from the bottom
pool, chunks of levels >= 1 from the upper pool (R18); every pool chunk starts in the
allocated state of P:237 (all +inf, locked).
"""
from __future__ import annotations

NEG_INF = 0
INF = 0xFFFFFFFF
EMPTY = 0xFFFFFFFFFFFFFFFF
NULL = 0xFFFFFFFF
FREE, HELD, ZOMBIE = 0, 1, 2
PLAN_LEVELS = 16


def K(e):  # key (or max / lock state) half of an entry
    return e & 0xFFFFFFFF


def V(e):  # value (or next / version) half of an entry
    return e >> 32


def E(k, v):
    return (k & 0xFFFFFFFF) | ((v & 0xFFFFFFFF) << 32)


class PoolExhausted(Exception):
    pass


def raise_draw(rkey: int, level: int) -> int:
    """isKeyRaised's random draw: a counter-based 32-bit
    hash of (raised key, level of the split) -- the murmur3 finalizer of
    rkey ^ level * 0x9E3779B9 ^ 0x2545F491.  The key is raised iff the draw < p * 2^32."""
    x = (rkey ^ (level * 0x9E3779B9) ^ 0x2545F491) & 0xFFFFFFFF
    x ^= x >> 16
    x = (x * 0x85EBCA6B) & 0xFFFFFFFF
    x ^= x >> 13
    x = (x * 0xC2B2AE35) & 0xFFFFFFFF
    x ^= x >> 16
    return x


class GFSLModel:
    def __init__(self, N: int, key_range: int, cap_bottom: int, cap_upper: int,
                 rebuild_every: int = 0, p_chunk_q32: int = 0):
        assert N >= 6
        # p_chunk as a 32-bit fraction; 0 = p_chunk = 1 (R16)
        self.p_chunk_q32 = p_chunk_q32
        # R24: rebuild the upper levels after every k-th batch (0 = never); the GPU's
        # default wear rule (R29) is a library policy and is not modelled here
        self.rebuild_every = rebuild_every
        self.batches = 0
        self.rebuilds = 0       # upper-level rebuilds so far (R24)
        self.dirty = False
        self.free, self.free_taken = [], 0  # R25 free list of reclaimed level-0 chunks
        self.N, self.DSIZE, self.NEXT, self.LOCK, self.MAXL = N, N - 2, N - 2, N - 1, N
        self.key_range = key_range
        self.cap_bottom, self.cap_upper = cap_bottom, cap_upper
        # every chunk is allocated locked with +inf everywhere
        self.pool = [[EMPTY] * (N - 1) + [HELD] for _ in range(cap_upper + cap_bottom)]
        self.head = [NULL] * 32
        self.counter = [0] * 32
        # one unlocked chunk per level holding -inf with a pointer to the level below
        for l in range(N):
            c = cap_upper if l == 0 else l - 1
            below = 0 if l == 0 else (cap_upper if l == 1 else l - 2)
            ch = self.pool[c]
            ch[0] = E(NEG_INF, below)
            ch[self.NEXT] = E(INF, NULL)
            ch[self.LOCK] = E(FREE, 0)
            self.head[l] = c
        self.bump = [1, N - 1]  # [bottom pool, upper pool]
        self.trace = None       # chunks read by the last search (for the worked examples)
        self.wtrace = None      # list -> every entry write is appended as (chunk, index, entry)
        self.merges = 0         # merges of the current batch (-> upkeep)
        self.restarts = 0       # searchDown restarts (Alg 4.2 l.25; only under injection)
        self.check_each_op = False  # run check_invariants() after every op of a batch
        self.reset_log = set()  # chunks reset to the allocated state since the last snapshot

    # ---- chunk accessors ----------------------------------------------------------------
    def w(self, c, i, e):
        """One atomic 64-bit entry write (AtomicWrite of Alg 4.7 / 4.9 / 4.12)."""
        self.pool[c][i] = e
        if self.wtrace is not None:
            self.wtrace.append((c, i, e))

    def keys(self, c):
        return [K(e) for e in self.pool[c][: self.DSIZE]]

    def mx(self, c):
        return K(self.pool[c][self.NEXT])

    def nxt(self, c):
        return V(self.pool[c][self.NEXT])

    def state(self, c):
        return K(self.pool[c][self.LOCK])

    def zombie(self, c):
        return self.state(c) == ZOMBIE

    def count(self, c):  # numNonEmpty (Alg 4.12 l.3): -inf counts (R8)
        return sum(1 for k in self.keys(c) if k != INF)

    def eq_idx(self, c, k):  # isTidWithEqualKey (Alg 4.4)
        ks = self.keys(c)
        for i in range(self.DSIZE - 1, -1, -1):
            if ks[i] == k:
                return i
        return None

    def le_idx(self, c, k):  # highest DATA index with key <= k (Alg 4.3, DATA votes)
        ks = self.keys(c)
        for i in range(self.DSIZE - 1, -1, -1):
            if ks[i] <= k:
                return i
        return None

    def height(self):  # getHeight
        h = 0
        for l in range(1, self.N):
            if self.counter[l] > 0:
                h = l
        return h

    # ---- locks (serial: a lock is never found held by someone else) ---------------------
    def lock(self, c):
        assert self.state(c) == FREE
        ch = self.pool[c]
        ch[self.LOCK] = E(HELD, V(ch[self.LOCK]))
        if self.wtrace is not None:
            self.wtrace.append((c, self.LOCK, ch[self.LOCK]))

    def unlock(self, c, state=FREE):
        ch = self.pool[c]
        ch[self.LOCK] = E(state, V(ch[self.LOCK]) + 1)
        if self.wtrace is not None:
            self.wtrace.append((c, self.LOCK, ch[self.LOCK]))

    def alloc(self, level):  # bump a counter, the chunk is already +inf and locked
        if level == 0 and self.free_taken < len(self.free):  # R25: reclaimed chunks first
            c = self.free[self.free_taken]
            self.free_taken += 1
            return c
        p = 1 if level > 0 else 0
        cap = self.cap_upper if p else self.cap_bottom
        i = self.bump[p]
        if i >= cap:
            raise PoolExhausted
        self.bump[p] += 1
        return i if p else self.cap_upper + i

    # ---- search phase (Alg 4.1-4.4 and searchSlow's path, on the snapshot; R1, R21) ------
    def search(self, k, hook=None):
        """searchDown + searchLateral (Alg 4.2-4.4) with searchSlow's path (Alg 4.6).
        Returns (found, path{level: chunk}, top level that held k).  `hook(chunk)` (tests
        only) runs before every chunk read, so a test can interleave other operations as a
        concurrent team would; a backtrack with no prevKv then restarts the traversal from
        the top (Alg 4.2 l.25), counted in self.restarts.  Within a batch the
        search runs on the quiescent snapshot (R1) and never restarts."""
        while True:
            r = self._search_once(k, hook)
            if r is not None:
                return r
            self.restarts += 1

    def _search_once(self, k, hook):
        height = self.height()                        # getHeight
        cur, level = self.head[height], height
        bt = bt_c = None
        top = 0
        path = {}
        trace = self.trace = []                       # chunks read by this pass
        while True:
            if hook is not None:
                hook(cur)
                self.trace = trace
            trace.append(cur)
            if self.zombie(cur):                      # Alg 4.2 l.9-11
                cur = self.nxt(cur)
                continue
            w = self.le_idx(cur, k) if level > 0 else None
            if self.mx(cur) < k:                      # lateral step (l.15-18)
                if level > 0:
                    bt = None if w is None else V(self.pool[cur][w])
                    bt_c = cur
                cur = self.nxt(cur)
                continue
            if level == 0:                            # searchLateral result (Alg 4.4)
                path[0] = cur
                return self.eq_idx(cur, k) is not None, path, top
            if w is not None:                         # down step (l.19-23)
                path[level] = cur
                if self.keys(cur)[w] == k and top == 0:
                    top = level
                cur = V(self.pool[cur][w])
            elif bt is not None:                      # backtrack (l.24-28, 33-38)
                path[level] = bt_c
                cur = bt
            else:                                     # restart (l.25): prevKv is null
                return None
            level -= 1
            bt = bt_c = None

    def search_down_to_level(self, L, k):  # Alg 4.10 l.4
        height = self.height()
        if height <= L:
            return self.head[L]
        cur, level, prev = self.head[height], height, None
        while level > L:
            if self.zombie(cur):
                cur = self.nxt(cur)
                continue
            if self.mx(cur) < k:
                prev = cur
                cur = self.nxt(cur)
                continue
            w = self.le_idx(cur, k)
            if w is not None:
                cur = V(self.pool[cur][w])
            else:
                assert prev is not None
                cur = V(self.pool[prev][self.le_idx(prev, k)])
            level -= 1
            prev = None
        return cur

    # ---- findAndLockEnclosing (Alg 4.8) with the lazy zombie redirect (Alg 4.6, R15, R21) -
    def first_non_zombie(self, z):
        c = self.nxt(z)
        while self.zombie(c):
            c = self.nxt(c)
        return c

    def redirect_zombie(self, prev, z, fnz):  # Alg 4.6 l.13-14 (try-lock succeeds serially)
        if self.zombie(prev) or self.nxt(prev) != z or self.state(prev) != FREE:
            return
        self.lock(prev)
        if self.nxt(prev) == z:
            self.w(prev, self.NEXT, E(self.mx(prev), fnz))
        self.unlock(prev)

    def find_and_lock_enclosing(self, c, k, level):
        prev = None
        while True:
            if self.state(c) == FREE:                 # optimistic lock, validated under it
                self.lock(c)
                if self.mx(c) < k:                    # l.17-21
                    nx = self.nxt(c)
                    self.unlock(c)
                    prev, c = c, nx
                    continue
                return c
            if self.zombie(c):
                fnz = self.first_non_zombie(c)
                if prev is not None:
                    self.redirect_zombie(prev, c, fnz)
                elif level >= 0 and c == self.head[level]:
                    self.head[level] = fnz            # updateHeadArray (Alg 4.6 l.15)
                c = fnz
            if self.mx(c) < k:                        # chunkNotEnclosing (l.5-8)
                prev, c = c, self.nxt(c)
                continue
            assert self.state(c) == FREE, "serial model: lock held"

    def lock_next_chunk(self, c):  # Alg 4.9 l.17 / Alg 4.12 l.9
        n = self.nxt(c)
        skipped = False
        while n != NULL:
            if self.zombie(n):
                n = self.nxt(n)
                skipped = True
                continue
            if skipped:  # unlink the zombies from c's NEXT (we hold c)
                self.w(c, self.NEXT, E(self.mx(c), n))
            self.lock(n)
            return n
        return None

    # ---- the chunk operations ---------------------------------------------------------
    def execute_insert(self, c, k, v):  # Alg 4.7, Fig 4.3: shift right from insertIdx
        ch = self.pool[c]
        ks = self.keys(c)
        idx = sum(1 for x in ks if x < k)             # insertion index (l.3)
        old = ch[:]
        for t in range(self.DSIZE - 1, idx - 1, -1):  # l.7-10: from DSIZE-1 down to idx
            ins = E(k, v) if t == idx else old[t - 1]  # l.2: each lane takes its left neighbour
            if K(ins) != INF:
                self.w(c, t, ins)

    def execute_remove_no_merge(self, c, k):  # P:900-902, Fig 4.6, R13
        ch = self.pool[c]
        idx = self.eq_idx(c, k)
        cnt = self.count(c)
        last = self.nxt(c) == NULL
        old = ch[:]
        if idx == cnt - 1 and not last:  # k was the max: the max field goes first
            self.w(c, self.NEXT, E(K(old[idx - 1]), V(old[self.NEXT])))
        for t in range(idx, cnt - 1):    # lanes idx+1 .. cnt-1 write leftwards, ascending
            self.w(c, t, old[t + 1])
        self.w(c, cnt - 1, EMPTY)        # the vacated last slot (Q20)

    def split(self, level, c):  # Alg 4.9 preSplit + splitCopy (also splitRemove)
        HALF = self.DSIZE // 2
        pnext = self.lock_next_chunk(c)               # preSplit (l.16-21)
        pnew = self.alloc(level)
        ch = self.pool[c]
        cnt = self.count(c)
        thresh = K(ch[HALF - 1])
        oldmax = self.mx(c)
        self.w(pnew, self.NEXT, E(oldmax, NULL if pnext is None else pnext))  # new -> next
        for t in range(cnt - HALF):                   # splitCopy l.27-28: lanes >= DSIZE/2
            self.w(pnew, t, ch[t + HALF])
        self.w(c, self.NEXT, E(thresh, pnew))         # l.30: one 64-bit write links it
        for t in range(HALF, cnt):
            self.w(c, t, EMPTY)                       # l.32 setMovedValsEmpty
        if pnext is not None:
            self.unlock(pnext)
        self.counter[level] += 1                      # Alg 4.5 l.42 / 4.12 l.18 (R9)
        return pnew

    def update_down_ptrs(self, level, moved, lower):  # Alg 4.10, R14
        if level + 1 >= self.MAXL or not moved:
            return
        moved = list(moved)
        upper = self.search_down_to_level(level + 1, moved[0])
        lc = lower
        while moved:
            km0 = moved[0]
            while self.zombie(upper) or self.mx(upper) < km0:
                upper = self.nxt(upper)
            umax = self.mx(upper)
            here = [km for km in moved if km <= umax]
            moved = [km for km in moved if km > umax]
            if not any(self.eq_idx(upper, km) is not None for km in here):
                continue
            upper = self.find_and_lock_enclosing(upper, km0, level + 1)
            for j, km in enumerate(here):
                if km > self.mx(upper):
                    moved = here[j:] + moved
                    break
                ui = self.eq_idx(upper, km)
                if ui is None:
                    continue
                while self.zombie(lc) or self.mx(lc) < km:
                    lc = self.nxt(lc)
                if self.eq_idx(lc, km) is not None and V(self.pool[upper][ui]) != lc:
                    self.w(upper, ui, E(km, lc))
            self.unlock(upper)

    # ---- Insert (Alg 4.5) ---------------------------------------------------------------
    def insert_to_level(self, level, pe, k, v):
        """Returns (ok, pins, pextra, raise, rkey, rptr); pins (and pextra) stay locked."""
        pe = self.find_and_lock_enclosing(pe, k, level)   # l.30
        if self.eq_idx(pe, k) is not None:                # l.32
            return False, pe, None, False, 0, 0
        if self.count(pe) < self.DSIZE:                   # l.35
            first = self.keys(pe)[0] == NEG_INF
            self.execute_insert(pe, k, v)                 # l.36
            if first and self.counter[level] == 0:        # l.37-38 (R9: every level)
                self.counter[level] = 1
            return True, pe, None, False, 0, 0
        HALF = self.DSIZE // 2
        moved = self.keys(pe)[HALF:self.count(pe)]
        thresh = self.keys(pe)[HALF - 1]
        pnew = self.split(level, pe)
        minK = self.keys(pnew)[0]
        if k < thresh:                                    # insertNewData (Alg 4.9 l.4)
            self.execute_insert(pe, k, v)
            pins, other = pe, pnew
        else:
            self.execute_insert(pnew, k, v)
            pins, other = pnew, pe
        if level == 0:                                    # keyForNextLevel
            rkey, rptr = max(k, minK), pnew               # R10
            hold = pins != pnew                           # R11
        else:
            rkey, rptr, hold = k, pins, False
        pextra = other if hold else None
        if not hold:
            self.unlock(other)                            # Alg 4.9 l.6-9
        self.update_down_ptrs(level, moved, pnew)         # Alg 4.9 l.12
        # isKeyRaised (Alg 4.5 l.15): always at p_chunk = 1 (R16), else with
        # probability p_chunk (the counter-based draw of R28)
        up = self.p_chunk_q32 == 0 or raise_draw(rkey, level) < self.p_chunk_q32
        return True, pins, pextra, up, rkey, rptr

    def insert(self, k, v, path):
        ok, pins, pextra, raise_, rkey, rptr = self.insert_to_level(0, path[0], k, v)
        if not ok:
            self.unlock(pins)
            return False
        level = 1
        while raise_ and level < self.MAXL:               # Alg 4.5 l.15-22
            ok2, p2, _, r2, rk2, rp2 = self.insert_to_level(level, path[level], rkey, rptr)
            self.unlock(p2)
            raise_ = ok2 and r2                           # R19
            rkey, rptr = rk2, rp2
            level += 1
        if pextra is not None:
            self.unlock(pextra)
        self.unlock(pins)
        return True

    # ---- Delete (Alg 4.11-4.12) -----------------------------------------------------------
    def execute_remove_merge(self, e, f, k):  # P:947-951, Fig 4.5c
        """Every value of e but k moves to f's low slots and f's own entries move right;
        f is written serially in DESCENDING index order, so after the first write
        of Fig 4.5c F reads [24, 26, EMPTY, 26]."""
        idx = self.eq_idx(e, k)
        eent = [x for i, x in enumerate(self.pool[e][: self.count(e)]) if i != idx]
        fent = self.pool[f][: self.count(f)]
        merged = eent + fent
        for t in range(len(merged) - 1, -1, -1):
            self.w(f, t, merged[t])

    def remove_from_chunk(self, level, pe, k):
        cnt = self.count(pe)
        only_neg_inf_after = cnt == 2 and self.keys(pe)[0] == NEG_INF
        if cnt > self.DSIZE // 3:                         # l.4-7 (R8)
            last = self.nxt(pe) == NULL
            self.execute_remove_no_merge(pe, k)
            if only_neg_inf_after and last:               # R17
                self.counter[level] -= 1
            self.unlock(pe)
            return
        pnext = self.lock_next_chunk(pe)                  # l.9
        if pnext is None:                                 # l.10-13
            self.execute_remove_no_merge(pe, k)
            if only_neg_inf_after:
                self.counter[level] -= 1
            self.unlock(pe)
            return
        pg = None
        g_moved = []
        nf = self.count(pnext)
        if nf + cnt - 1 > self.DSIZE:                     # l.16-19 splitRemove
            HALF = self.DSIZE // 2
            g_moved = self.keys(pnext)[HALF:nf]
            pg = self.split(level, pnext)
            self.unlock(pg)
            nf = HALF
        e_moved = [x for x in self.keys(pe)[:cnt] if x != k]
        self.execute_remove_merge(pe, pnext, k)           # l.21
        self.unlock(pe, ZOMBIE)                           # l.22 markAsZombie (R6)
        self.counter[level] -= 1                          # l.24
        self.merges += 1
        if nf + cnt - 1 == 1 and self.nxt(pnext) == NULL and self.keys(pe)[0] == NEG_INF:
            self.counter[level] -= 1                      # R17
        self.unlock(pnext)                                # l.25
        self.update_down_ptrs(level, e_moved, pnext)      # l.27
        if pg is not None:
            self.update_down_ptrs(level, g_moved, pg)

    def search_lateral(self, k, c):  # Alg 4.4 (exact: no concurrency here)
        while self.zombie(c) or self.mx(c) < k:
            c = self.nxt(c)
        return self.eq_idx(c, k) is not None

    def delete(self, k, path, top=None):
        """Alg 4.11.  `top` (the highest level where the snapshot search saw k) is not
        used: the paper checks every level from the current height down (l.12-16)."""
        pb = self.find_and_lock_enclosing(path[0], k, 0)  # l.8
        if self.eq_idx(pb, k) is None:                    # l.9-10 (R15: unlock first)
            self.unlock(pb)
            return False
        height = self.height()                            # l.12 rereadHeightAndUpdatePath
        for i in range(height, 0, -1):                    # l.13-20
            if not self.search_lateral(k, path[i]):       # l.15: containment before locking
                continue
            pe = self.find_and_lock_enclosing(path[i], k, i)  # l.18
            self.remove_from_chunk(i, pe, k)              # l.19
        self.remove_from_chunk(0, pb, k)                  # l.22
        return True

    # ---- a batch (R1: search phase on the snapshot, then the mutations in op order) -----
    def batch(self, ops, keys, vals=None):
        n = len(ops)
        res = [0xFF] * n
        snap_h = self.height()
        plans = []
        for i in range(n):
            op, key = int(ops[i]), int(keys[i])
            if op > 2 or key >= self.key_range:
                continue
            k = key + 1
            found, path, top = self.search(k)
            if op == 0:
                res[i] = int(found)
            else:
                mut = (not found) if op == 1 else found
                res[i] = int(mut)
                if mut:
                    plans.append((i, op, k, path, top))
        head_at_start = list(self.head)  # levels above the snapshot height start at head[l]
        self.merges = 0
        for i, op, k, path, top in plans:
            full = [path[l] if l <= snap_h else head_at_start[l]
                    for l in range(self.N)]
            if op == 1:
                r = self.insert(k, 0 if vals is None else int(vals[i]), full)
            else:
                r = self.delete(k, full, top)
            if not r:
                res[i] = 0
            if self.check_each_op:
                bad = self.check_invariants()
                assert not bad, f"after op {i} ({'insert' if op == 1 else 'delete'} {k - 1}): {bad[:5]}"
        if self.merges:
            self.upkeep()
        if plans:
            self.dirty = True  # a mutating batch since the last rebuild
        due = bool(n and self.rebuild_every and (self.batches + 1) % self.rebuild_every == 0)
        if due and self.dirty:
            self.rebuild()
            self.reclaim()
            self.dirty = False
        if n:
            self.batches += 1
        return res

    def reclaim(self):
        """R25: after a rebuild no pointer reaches a zombie; reset them to the allocated
        state and append them (ascending) after the unused part of the free list."""
        zombies = [self.cap_upper + i for i in range(self.bump[0]) if self.zombie(self.cap_upper + i)]
        for c in zombies:
            self.pool[c] = [EMPTY] * (self.N - 1) + [HELD]
            self.reset_log.add(c)
        self.free = self.free[self.free_taken:] + zombies
        self.free_taken = 0

    def rebuild_now(self):
        """gfsl_rebuild: rebuild now if a batch mutated the structure since the last
        rebuild."""
        if self.dirty:
            self.rebuild()
            self.reclaim()
            self.dirty = False

    def rebuild(self):
        """R24: re-derive levels >= 1 from level 0 between batches ("compact the
        structure between kernel launches").  Level 1 = [-inf -> head[0]] + (min key of C
        -> C) for every live non-first level-0 chunk C holding a key, in key order, F per
        chunk; level l+1 = [-inf -> first chunk of level l] + (first key of chunk j -> chunk
        j); chunks of level l: the head chunk l-1, then the next free upper indices."""
        N, F = self.N, self.N - 4
        live = []
        for i in range(self.bump[0]):
            c = self.cap_upper + i
            k0 = K(self.pool[c][0])
            if not self.zombie(c) and k0 not in (NEG_INF, INF):
                live.append((k0, c))
        live.sort()
        n1 = len(live)
        m, base, pw = {}, {}, {}
        length, b, p, top = n1 + 1, N - 1, 1, N - 1
        for l in range(1, N):
            m[l], base[l], pw[l] = -(-length // F), b, p
            b += m[l] - 1
            if m[l] == 1:
                top = l
                for q in range(l + 1, N):
                    m[q], base[q], pw[q] = 1, b, p * F
                break
            length, p = m[l], p * F

        def chunk(l, j):
            return l - 1 if j == 0 else base[l] + j - 1

        self.rebuilds += 1
        head0, old_used = self.head[0], self.bump[1]
        for l in range(1, N):
            length = 1 if l > top else (n1 + 1 if l == 1 else m[l - 1])
            for j in range(m[l]):
                ch = self.pool[chunk(l, j)]
                last_key = 0
                for e in range(self.DSIZE):
                    i = j * F + e
                    if e < F and i < length:
                        if i == 0:
                            key, val = NEG_INF, (head0 if l == 1 else l - 2)
                        else:
                            key = live[i * pw[l] - 1][0]
                            val = live[i - 1][1] if l == 1 else chunk(l - 1, i)
                        ch[e] = E(key, val)
                        last_key = key
                    else:
                        ch[e] = EMPTY
                last = j + 1 == m[l]
                ch[self.NEXT] = E(INF, NULL) if last else E(last_key, chunk(l, j + 1))
                ch[self.LOCK] = E(FREE, 0)
        for l in range(1, N):
            self.head[l] = l - 1
            real = (n1 > 0) if l == 1 else (m[l - 1] > 1)
            self.counter[l] = m[l] if (l <= top and real) else 0
        new_used = base[N - 1] + (m[N - 1] - 1 if top == N - 1 else 0)
        self.bump[1] = new_used
        for c in range(new_used, old_used):  # back to the allocated state of P:237
            self.pool[c] = [EMPTY] * (N - 1) + [HELD]

    def upkeep(self):
        """R23: between batches, point every live chunk past the zombie chains that follow
        it and move zombie first chunks out of the head array ("compact the structure
        between kernel launches"; the values are those of Alg 4.6's lazy redirect)."""
        used = list(range(self.bump[1])) + [self.cap_upper + i for i in range(self.bump[0])]
        for c in used:
            if self.zombie(c):
                continue
            n = self.nxt(c)
            if n == NULL or not self.zombie(n):
                continue
            while self.zombie(n):
                n = self.nxt(n)
            self.pool[c][self.NEXT] = E(self.mx(c), n)
        for l in range(self.N):
            h = self.head[l]
            while self.zombie(h):
                h = self.nxt(h)
            self.head[l] = h

    # ---- views ------------------------------------------------------------------------
    def level_chain(self, l):
        out, c = [], self.head[l]
        while c != NULL:
            out.append(c)
            c = self.nxt(c)
        return out

    def level_keys(self, l, with_values=False):
        out = []
        for c in self.level_chain(l):
            if self.zombie(c):
                continue
            for e in self.pool[c][: self.DSIZE]:
                if K(e) not in (INF, NEG_INF):
                    out.append((K(e) - (1 if l == 0 else 0), V(e)) if with_values else K(e))
        return out

    def export(self):
        kv = self.level_keys(0, with_values=True)
        return [k for k, _ in kv], [v for _, v in kv]

    def snapshot(self):
        """State for the cross-batch invariants V6 / V11: every used
        chunk's max field and the bytes of every zombie."""
        self.reset_log = set()
        used = list(range(self.bump[1])) + [self.cap_upper + i for i in range(self.bump[0])]
        return {"max": {c: self.mx(c) for c in used},
                "zombie": {c: list(self.pool[c][: self.LOCK]) for c in used if self.zombie(c)},
                "upper_gen": self.rebuilds}

    def reachable(self):
        """Every chunk index reachable from the head array through NEXT and down pointers."""
        seen, stack = set(), [(self.head[l], l) for l in range(self.N)]
        while stack:
            c, l = stack.pop()
            if c == NULL or (c, l) in seen:
                continue
            seen.add((c, l))
            stack.append((self.nxt(c), l))
            if l > 0:
                for e in self.pool[c][: self.DSIZE]:
                    if K(e) != INF:
                        stack.append((V(e), l - 1))
        return {c for c, _ in seen}

    def check_invariants(self, prev=None):
        """The structural invariants of P:203 and §4.3, numbered as in
        DESIGN.md: V1 sorted chunks, V2 max fields, V3 order between chunks, V4 level l+1
        keys within level l, V5 down pointers reach their key laterally, V7 no
        lock held, V8 the last chunk is not a zombie, V9 head chunks start with
        -inf, V12 every reachable chunk index is allocated; with `prev` (a snapshot()):
        V6 a max field never increases and V11 a zombie never changes.
        Returns a list of violations."""
        bad = []
        for l in range(self.N):
            chain = self.level_chain(l)
            nz = [c for c in chain if not self.zombie(c)]
            if chain and self.zombie(chain[-1]):
                bad.append(f"V8 L{l}")
            if not nz or self.keys(nz[0])[0] != NEG_INF:
                bad.append(f"V9 L{l}")
            prev_max = None
            for c in nz:
                ks = [k for k in self.keys(c) if k != INF]
                if self.keys(c)[: len(ks)] != ks or sorted(set(ks)) != ks:
                    bad.append(f"V1 L{l} c{c}")
                if self.state(c) != FREE:
                    bad.append(f"V7 L{l} c{c}")
                if self.nxt(c) == NULL:
                    if self.mx(c) != INF:
                        bad.append(f"V2 L{l} c{c}")
                elif not ks or self.mx(c) != ks[-1]:
                    bad.append(f"V2 L{l} c{c}")
                if ks and prev_max is not None and not prev_max < ks[0]:
                    bad.append(f"V3 L{l} c{c}")
                if ks:
                    prev_max = ks[-1]
            if l + 1 < self.N:
                lower = set(self.level_keys(l))
                for k in self.level_keys(l + 1):
                    if k not in lower:
                        bad.append(f"V4 L{l + 1} k{k}")
            if l > 0:                                     # V5
                for c in nz:
                    for e in self.pool[c][: self.DSIZE]:
                        k = K(e)
                        if k == INF:
                            continue
                        d, hops = V(e), 0
                        while d != NULL and hops <= self.bump[0] + self.bump[1] and (
                                self.zombie(d) or self.mx(d) < k):
                            d, hops = self.nxt(d), hops + 1
                        if d == NULL or self.eq_idx(d, k) is None:
                            bad.append(f"V5 L{l} k{k}")
        used_hi = {0: self.cap_upper + self.bump[0], 1: self.bump[1]}
        for c in self.reachable():                        # V12
            if c >= self.cap_upper + self.cap_bottom or (
                    c >= self.cap_upper and c >= used_hi[0]) or (c < self.cap_upper and c >= used_hi[1]):
                bad.append(f"V12 c{c}")
        if prev is not None:
            same_upper = prev["upper_gen"] == self.rebuilds
            for c, m in prev["max"].items():              # V6
                if c in self.reset_log or (c < self.cap_upper and not same_upper):
                    continue
                if self.mx(c) > m:
                    bad.append(f"V6 c{c}")
            for c, b in prev["zombie"].items():           # V11
                if c in self.reset_log or (c < self.cap_upper and not same_upper):
                    continue
                if list(self.pool[c][: self.LOCK]) != b or not self.zombie(c):
                    bad.append(f"V11 c{c}")
        return bad
