/*
 * oracle_a.c -- Oracle-A: the plain CPU definition of what a GFSL batch computes.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this file's shared library.  The
 * product path (paper_conf_ppopp_moscovicicp17_b200/) never imports, links or calls it,
 * and this file shares no code, header, constant or helper with the CUDA path.
 *
 * What it computes
 * ----------------
 * GFSL is a concurrent ordered map over 32-bit unsigned keys and values
 * (Table 4.1) with three operations:
 *   contains(k)   -> true iff k is in the map               (Alg 4.1)
 *   insert(k, v)  -> false if k is present, else adds (k,v) (Alg 4.5 l.2-4, P:503-510;
 *                    the value of a present key is not overwritten)
 *   delete(k)     -> false if k is absent, else removes k   (Alg 4.11 l.3-5)
 * Work arrives as an array of (op type, key).  The paper runs the array
 * concurrently, so any linearization is a correct answer.  The
 * build fixes one: S1, the "snapshot batch" (reading R1 = SURVEY 8(c) C-1):
 *   for every op i of the batch, its result is computed against the map M as it
 *   was BEFORE the batch; then M' = M + {successful inserts} - {successful deletes}.
 * Contract: at most one mutating (insert/delete) op per key per batch.  Under it the
 * second pass is order independent.  oa_batch() returns OA_ECONTRACT if violated.
 * Invalid ops (op code > 2 or key >= key_range) get result 0xFF and no effect
 * (reading R5).
 *
 * oa_batch_seq() is the combining semantics of SURVEY 8(f) NEXT-1 (R26), exact
 * for ANY batch: every Contains is answered against M (as in S1); then the mutating ops
 * are applied one by one in input order, each answered against the map as it is at that
 * point.  Under the contract it equals oa_batch() (the mutations of distinct keys
 * commute).
 *
 * How: a sequential Pugh skiplist (levels of sorted linked lists, each a
 * random sublist of the one below, a node's height drawn with p = 1/2), MAX_LEVEL 32,
 * xorshift64 RNG.  This is the textbook structure of P:191, not GFSL: the two share
 * no code.  Written for obviousness, not speed; never tuned.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OA_MAX_LEVEL 32

enum { OA_OK = 0, OA_ECONTRACT = 1, OA_ENOMEM = 2 };
enum { OA_CONTAINS = 0, OA_INSERT = 1, OA_DELETE = 2 };
enum { OA_FALSE = 0, OA_TRUE = 1, OA_INVALID = 0xFF };

typedef struct oa_node {
  uint32_t key;
  uint32_t val;
  int height;
  struct oa_node *next[]; /* next[0..height-1] */
} oa_node;

typedef struct oa_map {
  oa_node *head;   /* sentinel, height OA_MAX_LEVEL, smaller than every key */
  int level;       /* number of levels in use (>= 1) */
  uint64_t size;   /* number of keys */
  uint64_t rng;    /* xorshift64 state */
} oa_map;

static oa_node *oa_node_new(int height, uint32_t key, uint32_t val) {
  oa_node *n = (oa_node *)malloc(sizeof(oa_node) + sizeof(oa_node *) * (size_t)height);
  if (!n) return NULL;
  n->key = key;
  n->val = val;
  n->height = height;
  for (int i = 0; i < height; i++) n->next[i] = NULL;
  return n;
}

/* Pugh's randomLevel with p = 1/2. */
static int oa_random_level(oa_map *m) {
  int lvl = 1;
  for (;;) {
    uint64_t x = m->rng;
    x ^= x << 13;
    x ^= x >> 7;
    x ^= x << 17;
    m->rng = x;
    if ((x >> 63) == 0 || lvl >= OA_MAX_LEVEL) break; /* coin flip */
    lvl++;
  }
  return lvl;
}

oa_map *oa_create(uint64_t seed) {
  oa_map *m = (oa_map *)calloc(1, sizeof(oa_map));
  if (!m) return NULL;
  m->head = oa_node_new(OA_MAX_LEVEL, 0, 0);
  if (!m->head) { free(m); return NULL; }
  m->level = 1;
  m->size = 0;
  m->rng = seed ? seed : 0x9E3779B97F4A7C15ull;
  return m;
}

void oa_destroy(oa_map *m) {
  if (!m) return;
  oa_node *n = m->head->next[0];
  while (n) { oa_node *nx = n->next[0]; free(n); n = nx; }
  free(m->head);
  free(m);
}

uint64_t oa_size(const oa_map *m) { return m->size; }

/* Search: walk each level right while the next key is < k, then step down. */
static oa_node *oa_find_ge(const oa_map *m, uint32_t k, oa_node **update) {
  oa_node *x = m->head;
  for (int i = m->level - 1; i >= 0; i--) {
    while (x->next[i] && x->next[i]->key < k) x = x->next[i];
    if (update) update[i] = x;
  }
  return x->next[0]; /* first node with key >= k, or NULL */
}

int oa_contains(const oa_map *m, uint32_t k) {
  oa_node *x = oa_find_ge(m, k, NULL);
  return x && x->key == k;
}

/* Returns 1 and writes *v if present. */
int oa_get(const oa_map *m, uint32_t k, uint32_t *v) {
  oa_node *x = oa_find_ge(m, k, NULL);
  if (x && x->key == k) { if (v) *v = x->val; return 1; }
  return 0;
}

/* Returns 1 if inserted, 0 if k was present (value not overwritten), -1 on ENOMEM. */
int oa_insert(oa_map *m, uint32_t k, uint32_t v) {
  oa_node *update[OA_MAX_LEVEL];
  oa_node *x = oa_find_ge(m, k, update);
  if (x && x->key == k) return 0;
  int lvl = oa_random_level(m);
  if (lvl > m->level) {
    for (int i = m->level; i < lvl; i++) update[i] = m->head;
    m->level = lvl;
  }
  oa_node *n = oa_node_new(lvl, k, v);
  if (!n) return -1;
  for (int i = 0; i < lvl; i++) {
    n->next[i] = update[i]->next[i];
    update[i]->next[i] = n;
  }
  m->size++;
  return 1;
}

/* Returns 1 if removed, 0 if absent. */
int oa_erase(oa_map *m, uint32_t k) {
  oa_node *update[OA_MAX_LEVEL];
  oa_node *x = oa_find_ge(m, k, update);
  if (!x || x->key != k) return 0;
  for (int i = 0; i < m->level; i++) {
    if (update[i]->next[i] != x) break;
    update[i]->next[i] = x->next[i];
  }
  free(x);
  while (m->level > 1 && m->head->next[m->level - 1] == NULL) m->level--;
  m->size--;
  return 1;
}

/* Sorted export of the bottom level.  Returns the number of keys; writes at most cap. */
uint64_t oa_export(const oa_map *m, uint32_t *keys, uint32_t *vals, uint64_t cap) {
  uint64_t c = 0;
  for (oa_node *n = m->head->next[0]; n; n = n->next[0]) {
    if (c < cap) {
      if (keys) keys[c] = n->key;
      if (vals) vals[c] = n->val;
    }
    c++;
  }
  return c;
}

/* ---- contract check: open-addressing set of the batch's mutating keys ---- */
static uint64_t oa_mix(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull;
  x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull;
  x ^= x >> 33; return x;
}

static int oa_valid(uint8_t op, uint32_t key, uint64_t key_range) {
  return op <= OA_DELETE && (uint64_t)key < key_range;
}

/*
 * S1 batch (R1).  Pass 1: every result from the pre-batch map.  Pass 2: the
 * successful mutations, in input order.  Returns OA_OK, OA_ECONTRACT (two mutating ops
 * on one key; nothing is applied) or OA_ENOMEM.
 */
int oa_batch(oa_map *m, const uint8_t *op, const uint32_t *key, const uint32_t *val,
             uint8_t *res, uint64_t n, uint64_t key_range) {
  /* contract check first, so a violating batch leaves the map untouched */
  uint64_t nmut = 0;
  for (uint64_t i = 0; i < n; i++)
    if (oa_valid(op[i], key[i], key_range) && op[i] != OA_CONTAINS) nmut++;
  if (nmut) {
    uint64_t cap = 16;
    while (cap < 2 * nmut) cap <<= 1;
    uint64_t *tab = (uint64_t *)malloc(cap * sizeof(uint64_t));
    if (!tab) return OA_ENOMEM;
    memset(tab, 0xff, cap * sizeof(uint64_t)); /* empty slot = all ones */
    int bad = 0;
    for (uint64_t i = 0; i < n && !bad; i++) {
      if (!oa_valid(op[i], key[i], key_range) || op[i] == OA_CONTAINS) continue;
      uint64_t s = oa_mix(key[i]) & (cap - 1);
      for (;;) {
        if (tab[s] == ~0ull) { tab[s] = key[i]; break; }
        if (tab[s] == key[i]) { bad = 1; break; }
        s = (s + 1) & (cap - 1);
      }
    }
    free(tab);
    if (bad) return OA_ECONTRACT;
  }
  /* pass 1: results against the snapshot */
  for (uint64_t i = 0; i < n; i++) {
    if (!oa_valid(op[i], key[i], key_range)) { res[i] = OA_INVALID; continue; }
    int present = oa_contains(m, key[i]);
    switch (op[i]) {
      case OA_CONTAINS: res[i] = present ? OA_TRUE : OA_FALSE; break;
      case OA_INSERT:   res[i] = present ? OA_FALSE : OA_TRUE; break;
      default:          res[i] = present ? OA_TRUE : OA_FALSE; break;
    }
  }
  /* pass 2: apply the successful mutations */
  for (uint64_t i = 0; i < n; i++) {
    if (res[i] != OA_TRUE || op[i] == OA_CONTAINS) continue;
    if (op[i] == OA_INSERT) {
      if (oa_insert(m, key[i], val ? val[i] : 0) < 0) return OA_ENOMEM;
    } else {
      oa_erase(m, key[i]);
    }
  }
  return OA_OK;
}

/*
 * Combining batch (R26): pass 1 answers the Contains ops
 * against the pre-batch map; pass 2 applies every valid Insert/Delete sequentially in
 * input order, each result taken from the map at that moment.  No contract.
 */
int oa_batch_seq(oa_map *m, const uint8_t *op, const uint32_t *key, const uint32_t *val,
                 uint8_t *res, uint64_t n, uint64_t key_range) {
  for (uint64_t i = 0; i < n; i++) {
    if (!oa_valid(op[i], key[i], key_range)) { res[i] = OA_INVALID; continue; }
    if (op[i] == OA_CONTAINS) res[i] = oa_contains(m, key[i]) ? OA_TRUE : OA_FALSE;
  }
  for (uint64_t i = 0; i < n; i++) {
    if (!oa_valid(op[i], key[i], key_range) || op[i] == OA_CONTAINS) continue;
    if (op[i] == OA_INSERT) {
      int r = oa_insert(m, key[i], val ? val[i] : 0);
      if (r < 0) return OA_ENOMEM;
      res[i] = r ? OA_TRUE : OA_FALSE;
    } else {
      res[i] = oa_erase(m, key[i]) ? OA_TRUE : OA_FALSE;
    }
  }
  return OA_OK;
}
