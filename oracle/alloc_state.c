/*
 * oracle/alloc_state.c -- O2 plumbing shared by O2-P (alloc_paper.c) and O2-R
 * (alloc_runs.c): lifecycle, the class geometry, the ring queue, the live-
 * allocation map behind the invariant checks, the structural check, the
 * canonical image and the exported entry points.  No policy decision is made
 * here.  TEST INFRASTRUCTURE ONLY (see alloc_paper.c).
 */
#include <stdlib.h>
#include <string.h>

#include "alloc_state.h"

#define IMAGE_MAGIC 0x47414C4C494D4731ULL

/* ---------------------------------------------------------- geometry --- */
uint64_t ceil_log2(uint64_t x) { uint64_t r = 0; while ((1ULL << r) < x) r++; return r; }
uint32_t nb_of(uint32_t t) { return MAX_BLOCKS_PER_SEGMENT >> t; }
uint64_t block_bytes(uint32_t t) { return SEGMENT_BYTES / nb_of(t); }         /* 64 KB << t */
/* linear block index (segment * nb + block) -> global block id (segment * 256 + block) */
uint32_t gid_of(uint32_t t, uint64_t linear) {
    return (uint32_t)((linear / nb_of(t)) * MAX_BLOCKS_PER_SEGMENT + linear % nb_of(t));
}

/* A-1..A-4: kind 0 = slice of class c, 1 = whole block of tree
 * t (A-2), 2 = k segments (A-3); returns the usable bytes. */
uint64_t class_usable(uint64_t size, uint32_t *kind, uint32_t *cls) {
    if (size <= MAX_SLICE) {
        uint64_t c = ceil_log2(size); c = c < 4 ? 0 : c - 4;
        *kind = 0; *cls = (uint32_t)c; return MIN_SLICE << c;
    }
    if (size < SEGMENT_BYTES) {
        uint64_t t = ceil_log2(size); t = t < 16 ? 0 : t - 16;
        *kind = 1; *cls = (uint32_t)t; return block_bytes((uint32_t)t);
    }
    uint64_t k = (size + SEGMENT_BYTES - 1) / SEGMENT_BYTES;
    *kind = 2; *cls = (uint32_t)k; return k * SEGMENT_BYTES;
}

uint64_t o2_usable_size(uint64_t size) {
    if (size == 0) return 0;
    uint32_t kind, cls;
    return class_usable(size, &kind, &cls);
}

/* ------------------------------------------------ ring queue --- */
uint16_t ring_pop(ring_t *r) {
    uint16_t j = r->e[r->head];
    r->e[r->head] = 0xFFFF;
    r->head = (r->head + 1) & 255; r->count--;
    return j;
}
void ring_push(ring_t *r, uint16_t j) {
    r->e[(r->head + r->count) & 255] = j;
    r->count++;
}
void ring_clear(ring_t *r) {
    r->head = 0; r->count = 0;
    for (int i = 0; i < 256; i++) r->e[i] = 0xFFFF;
}

/* ------------------------------------------------ live-allocation map --- */
static uint64_t mix(uint64_t x) { x ^= x >> 33; x *= 0xff51afd7ed558ccdULL; x ^= x >> 33; return x; }
static void live_grow(o2_t *a);
static void live_put(o2_t *a, uint64_t k, uint64_t v) {
    if (2 * (a->live_n + 1) > a->live_cap) live_grow(a);
    uint64_t m = a->live_cap - 1, i = mix(k) & m;
    while (a->live[i].key != NONE64) i = (i + 1) & m;
    a->live[i].key = k; a->live[i].val = v; a->live_n++;
}
static void live_grow(o2_t *a) {
    kv_t *old = a->live; uint64_t oc = a->live_cap;
    a->live_cap = oc ? oc * 2 : 1024;
    a->live = (kv_t *)malloc(a->live_cap * sizeof(kv_t));
    for (uint64_t i = 0; i < a->live_cap; i++) a->live[i].key = NONE64;
    a->live_n = 0;
    for (uint64_t i = 0; i < oc; i++) if (old[i].key != NONE64) live_put(a, old[i].key, old[i].val);
    free(old);
}
static int live_take(o2_t *a, uint64_t k, uint64_t *v) {
    if (!a->live_cap) return 0;
    uint64_t m = a->live_cap - 1, i = mix(k) & m;
    while (a->live[i].key != NONE64) {
        if (a->live[i].key == k) {
            *v = a->live[i].val;
            uint64_t j = i;                                   /* backward-shift deletion */
            for (;;) {
                j = (j + 1) & m;
                if (a->live[j].key == NONE64) break;
                uint64_t h = mix(a->live[j].key) & m;
                if ((j > i && (h <= i || h > j)) || (j < i && (h <= i && h > j))) {
                    a->live[i] = a->live[j]; i = j;
                }
            }
            a->live[i].key = NONE64; a->live_n--;
            return 1;
        }
        i = (i + 1) & m;
    }
    return 0;
}

/* invariants on a new allocation: inside the heap, aligned to its class */
void note_malloc(o2_t *a, uint64_t off, uint64_t usable) {
    if (off + usable > a->nseg * SEGMENT_BYTES) a->violations |= V_HEAP;
    uint64_t align = usable < SEGMENT_BYTES ? usable : SEGMENT_BYTES;
    if (off % align) a->violations |= V_ALIGN;
    live_put(a, off, usable);
    a->usable_live += usable;
}
void note_free(o2_t *a, uint64_t off) {
    uint64_t usable;
    if (live_take(a, off, &usable)) a->usable_live -= usable;
    else a->violations |= V_BAD_FREE;
}

/* ---------------------------------------------------------- lifecycle --- */
static o2_t *create(uint64_t nseg, unsigned slot_base, unsigned slot_min) {
    if (nseg < 1 || nseg > (1ULL << 14) || slot_base < 1) return NULL;
    o2_t *a = (o2_t *)calloc(1, sizeof(o2_t));
    a->nseg = nseg;
    unsigned off = 0;
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        unsigned n = slot_base >> c;                          /* halving per class */
        if (n < slot_min) n = slot_min;                       /* "capped at four"  */
        if (n < 1) n = 1;
        a->nslot[c] = n; a->slot_off[c] = off; off += n;
    }
    a->nslot_total = off;
    a->tree = (uint32_t *)malloc(nseg * sizeof(uint32_t));
    a->avail = (int32_t *)calloc(nseg, sizeof(int32_t));
    a->ring = (ring_t *)calloc(nseg, sizeof(ring_t));
    a->freecnt = (uint32_t *)calloc(nseg * MAX_BLOCKS_PER_SEGMENT, sizeof(uint32_t));
    unsigned k = (unsigned)ceil_log2(nseg); if (k < 1) k = 1;
    a->segfree = oracle_veb_create(k);
    for (unsigned t = 0; t < NUM_BLOCK_TREES; t++) a->btree[t] = oracle_veb_create(k);
    for (uint64_t s = 0; s < nseg; s++) {
        a->tree[s] = TREE_FREE; oracle_veb_insert(a->segfree, s);
        ring_clear(&a->ring[s]);
    }
    a->slot = (uint64_t *)malloc(a->nslot_total * sizeof(uint64_t));
    a->next = (uint64_t *)malloc(a->nslot_total * sizeof(uint64_t));
    for (unsigned i = 0; i < a->nslot_total; i++) a->slot[i] = a->next[i] = SLOT_EMPTY;
    return a;
}

/* O2-P: the paper's policy (P:195 block buffer of one-block slots). */
o2_t *o2_create_paper(uint64_t nseg, unsigned slot_base, unsigned slot_min) {
    return create(nseg, slot_base, slot_min);
}

/* O2-R: the deviation model (DESIGN.md Deviations 5). */
o2_t *o2_create_runs(uint64_t nseg, unsigned slot_base, unsigned slot_min, unsigned run_max, uint64_t run_bytes,
                     unsigned format_ahead, unsigned run_init, unsigned prefetch, unsigned run_grow,
                     unsigned prefill) {
    if (run_grow < 1 || run_grow > 8 || run_max < 1 || run_max > 512) return NULL;
    o2_t *a = create(nseg, slot_base, slot_min);
    if (!a) return NULL;
    a->runs = 1;
    a->run_max = run_max; a->run_bytes = run_bytes; a->format_ahead = format_ahead;
    a->run_init = run_init < 1 ? 1 : run_init;
    a->prefetch = prefetch;
    a->run_grow = run_grow;
    if (prefill) runs_prefill(a);                             /* R7 */
    return a;
}

void o2_destroy(o2_t *a) {
    if (!a) return;
    free(a->tree); free(a->avail); free(a->ring); free(a->freecnt);
    oracle_veb_destroy(a->segfree);
    for (unsigned t = 0; t < NUM_BLOCK_TREES; t++) oracle_veb_destroy(a->btree[t]);
    free(a->slot); free(a->next); free(a->live);
    free(a);
}

unsigned o2_nslot(const o2_t *a, unsigned c) { return c < NUM_BLOCK_TREES ? a->nslot[c] : 0; }
uint64_t o2_errors(const o2_t *a) { return a->err; }
uint64_t o2_violations(const o2_t *a) { return a->violations; }
uint64_t o2_live_count(const o2_t *a) { return a->live_n; }
uint64_t o2_usable_live(const o2_t *a) { return a->usable_live; }

/* ------------------------------------------------------ entry points --- */
uint64_t o2_malloc(o2_t *a, uint64_t size, uint64_t key) {
    return a->runs ? runs_malloc(a, size, key) : pol_malloc(a, size, key);
}
void o2_free(o2_t *a, uint64_t off) { pol_free(a, off); }
void o2_drain(o2_t *a) { if (a->runs) runs_drain(a); else pol_drain(a); }

/* Replay: kinds[i] 0 = malloc(args[i]) with slot key keys[i], out[i] = offset
 * (UINT64_MAX = NULL); 1 = free(out[args[i]]); 2 = drain. */
void o2_replay(o2_t *a, const uint8_t *kinds, const uint64_t *args, const uint64_t *keys,
               uint64_t n, uint64_t *out) {
    for (uint64_t i = 0; i < n; i++) {
        if (kinds[i] == 0) out[i] = o2_malloc(a, args[i], keys[i]);
        else if (kinds[i] == 1) { o2_free(a, out[args[i]]); out[i] = 0; }
        else { o2_drain(a); out[i] = 0; }
    }
}

/* Timing helpers (one thread, in order): malloc every size with key
 * i / keydiv (the request's warp), then free every offset in order. */
void o2_malloc_batch(o2_t *a, const uint64_t *sizes, uint64_t n, uint64_t keydiv, uint64_t *out) {
    for (uint64_t i = 0; i < n; i++) out[i] = o2_malloc(a, sizes[i], keydiv ? i / keydiv : 0);
}
void o2_free_batch(o2_t *a, const uint64_t *offs, uint64_t n) {
    for (uint64_t i = 0; i < n; i++) o2_free(a, offs[i]);
}

/* -------------------------------------------------- invariant check --- */
static int cmp_kv(const void *x, const void *y) {
    const kv_t *p = (const kv_t *)x, *q = (const kv_t *)y;
    return p->key < q->key ? -1 : p->key > q->key;
}

/* Full structural check; returns the accumulated violation mask. */
uint64_t o2_check(o2_t *a) {
    kv_t *v = (kv_t *)malloc((a->live_n + 1) * sizeof(kv_t));
    uint64_t n = 0, sum = 0;
    for (uint64_t i = 0; i < a->live_cap; i++) if (a->live[i].key != NONE64) v[n++] = a->live[i];
    qsort(v, n, sizeof(kv_t), cmp_kv);
    for (uint64_t i = 0; i < n; i++) {                       /* live allocations never overlap */
        sum += v[i].val;
        if (i + 1 < n && v[i].key + v[i].val > v[i + 1].key) a->violations |= V_OVERLAP;
    }
    free(v);
    if (sum != a->usable_live) a->violations |= V_ACCOUNT;
    for (uint64_t s = 0; s < a->nseg; s++) {                  /* trees agree with the table */
        uint32_t t = a->tree[s];
        if (oracle_veb_member(a->segfree, s) != (t == TREE_FREE)) a->violations |= V_TREES;
        for (uint32_t b = 0; b < NUM_BLOCK_TREES; b++)
            if (oracle_veb_member(a->btree[b], s) != ((t == b) && a->avail[s] > 0)) a->violations |= V_TREES;
        if (t < NUM_BLOCK_TREES) {
            ring_t *r = &a->ring[s];
            if (r->count != (uint32_t)a->avail[s] || a->avail[s] < 0 || (uint32_t)a->avail[s] > nb_of(t))
                a->violations |= V_RING;
            uint8_t seen[256] = {0};
            for (uint32_t q = 0; q < r->count; q++) {
                uint16_t j = r->e[(r->head + q) & 255];
                if (j >= nb_of(t) || seen[j]++) a->violations |= V_RING;
            }
        } else if (a->avail[s] != 0) {
            a->violations |= V_RING;
        }
    }
    return a->violations;
}

/* ------------------------------------------------------------- image --- */
static uint64_t tree_words(uint64_t nbits, uint64_t *wpl, unsigned *levels) {
    uint64_t w = (nbits + 63) / 64, total = 0;
    unsigned L = 0;
    for (;;) { wpl[L++] = w; total += w; if (w == 1) break; w = (w + 63) / 64; }
    *levels = L;
    return total;
}

/* a set as bitmap levels: leaf bit x = member, summary bit = child word != 0 */
static void tree_image(const oracle_veb *t, uint64_t nbits, uint64_t *out) {
    uint64_t wpl[16]; unsigned L;
    uint64_t total = tree_words(nbits, wpl, &L);
    memset(out, 0, total * sizeof(uint64_t));
    for (uint64_t x = oracle_veb_successor(t, 0); x != NONE64 && x < nbits; x = oracle_veb_successor(t, x + 1))
        out[x >> 6] |= 1ULL << (x & 63);
    uint64_t bp = 0, b = wpl[0];
    for (unsigned l = 1; l < L; l++) {
        for (uint64_t c = 0; c < wpl[l - 1]; c++) if (out[bp + c]) out[b + (c >> 6)] |= 1ULL << (c & 63);
        bp = b; b += wpl[l];
    }
}

uint64_t o2_image_words(const o2_t *a) {
    uint64_t wpl[16]; unsigned L;
    uint64_t W = tree_words(a->nseg, wpl, &L);
    return 8 + 10 * W + a->nseg * (1 + 65 + 128) + 2ULL * a->nslot_total;
}

/* Canonical image; layout documented in include/gallatin.h ("Snapshot image"). */
uint64_t o2_image(const o2_t *a, uint64_t *out, uint64_t cap) {
    uint64_t need = o2_image_words(a);
    if (cap < need) return 0;
    uint64_t wpl[16]; unsigned L;
    uint64_t W = tree_words(a->nseg, wpl, &L);
    uint64_t *p = out;
    p[0] = IMAGE_MAGIC; p[1] = a->nseg; p[2] = L; p[3] = W; p[4] = a->nslot_total;
    p[5] = a->err; p[6] = 0; p[7] = 0;
    p += 8;
    tree_image(a->segfree, a->nseg, p); p += W;
    for (unsigned t = 0; t < NUM_BLOCK_TREES; t++) { tree_image(a->btree[t], a->nseg, p); p += W; }
    for (uint64_t s = 0; s < a->nseg; s++) *p++ = ((uint64_t)a->tree[s] << 32) | (uint32_t)a->avail[s];
    for (uint64_t s = 0; s < a->nseg; s++) {
        const ring_t *r = &a->ring[s];
        *p++ = r->count;
        uint16_t e[256];
        for (uint32_t q = 0; q < 256; q++) e[q] = q < r->count ? r->e[(r->head + q) & 255] : 0xFFFF;
        for (uint32_t q = 0; q < 64; q++)
            *p++ = (uint64_t)e[4 * q] | ((uint64_t)e[4 * q + 1] << 16) |
                   ((uint64_t)e[4 * q + 2] << 32) | ((uint64_t)e[4 * q + 3] << 48);
    }
    for (uint64_t g = 0; g < a->nseg * MAX_BLOCKS_PER_SEGMENT; g += 2)
        *p++ = (uint64_t)a->freecnt[g] | ((uint64_t)a->freecnt[g + 1] << 32);
    for (unsigned i = 0; i < a->nslot_total; i++) *p++ = a->slot[i];
    for (unsigned i = 0; i < a->nslot_total; i++) *p++ = a->next[i];
    return need;
}
