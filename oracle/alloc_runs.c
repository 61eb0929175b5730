/*
 * oracle/alloc_runs.c -- O2-R: the deviation model, sequential.
 *
 * TEST INFRASTRUCTURE ONLY (see alloc_paper.c for who may load it).  It is
 * the paper's policy (alloc_paper.c, whose primitives it calls for segment
 * claims, formats, block returns, large claims and frees) with the policy
 * changes of DESIGN.md "Deviations" 5 and 8 that the CUDA path's serialized
 * replay reproduces exactly:
 *   R1 runs: a block-buffer slot holds a RUN of m consecutive blocks (one
 *      address range), handed out slice by slice in order; the first run has
 *      max(run_init >> c, min(run_init, 8)) blocks (at most one segment and
 *      the class cap), each refill takes 2^run_grow times the last, capped at
 *      run_max blocks and run_bytes bytes.  Slot index k of a run maps to
 *      block first + k / 4096, slice k mod 4096 (P:220 with consecutive
 *      blocks).  run_max = run_init = 1 is the paper's one-block buffer;
 *   R2 a run of < nb blocks comes from the lowest segment of the block tree
 *      (up to m of its ring entries: the longest run of consecutive block
 *      indices among them is kept, lowest start on ties, the rest re-enqueued
 *      in ascending order) or from one fresh segment whose other blocks are
 *      published; a run of >= nb blocks takes whole free segments privately
 *      (the lowest free one and the free ones right after it, no ring, no
 *      block tree) -- also when the block tree has a segment but with fewer
 *      than m blocks available, as long as a segment is free (a partly
 *      returned segment would give a short run: the warm-state refills);
 *   R3 format-ahead: the reservation that takes a segment below nb/4
 *      available blocks formats one more segment for the tree when no higher
 *      segment of the tree has blocks;
 *   R4 prefetch: the request drawing the middle of a run fetches the next run
 *      (never trimming other slots) into the slot's second word, which the
 *      run's replacement takes first;
 *   R5 before "no memory" (Deviations 8): every slot, class-major and slot-
 *      ascending, keeps the ceil(issued / 4096) blocks of its run requests
 *      have drawn from and gives the rest back whole (a prefetched run
 *      entirely); if that gave anything back the request is retried for ONE
 *      block; a large request retries its claim once after the trims;
 *   R6 segments formatted ahead and never used (all blocks home) go back to
 *      the segment tree before a segment claim reports "all in use", and in
 *      the drain after the slots are retired;
 *   R7 prefill (knob): the initial state holds every slot's first run, laid
 *      out class by class from the front ("always populated").
 * Not modelled: the exhaustion record (Deviations 11) -- a concurrency
 * device, checked on the GPU by invariants and by the paper-policy replays
 * (where it is state-neutral); the serialized replays of this model run the
 * CUDA path with the record off.  Pins per function: DESIGN.md 11.
 */
#include <stdlib.h>
#include <string.h>

#include "alloc_state.h"

/* largest run (blocks of tree t) a slot may hold: run_max blocks, run_bytes bytes */
static uint32_t run_cap(const o2_t *a, uint32_t t) {
    uint64_t by = a->run_bytes / block_bytes(t);
    uint64_t m = a->run_max < by ? a->run_max : by;
    return m < 1 ? 1 : (uint32_t)m;
}

/* R6: formatted segments with every block home go back, in segment order */
static uint64_t retire_idle_all(o2_t *a) {
    uint64_t n = 0;
    for (uint64_t s = 0; s < a->nseg; s++) {
        uint32_t t = a->tree[s];
        if (t < NUM_BLOCK_TREES && (uint32_t)a->avail[s] == nb_of(t)) {
            a->tree[s] = TREE_FREE; a->avail[s] = 0;
            ring_clear(&a->ring[s]);
            oracle_veb_delete(a->btree[t], s);
            oracle_veb_insert(a->segfree, s);
            n++;
        }
    }
    return n;
}

static uint64_t claim_front(o2_t *a) {
    uint64_t s = pol_claim_front(a);
    if (s == NONE64 && retire_idle_all(a)) s = pol_claim_front(a);
    return s;
}

/* format segment s for tree t and hand blocks [0, keep) to the caller: the
 * paper's initSegment followed by `keep` ring dequeues */
static void format_keep(o2_t *a, uint64_t s, uint32_t t, uint32_t keep) {
    pol_format_segment(a, s, t);
    for (uint32_t q = 0; q < keep; q++) ring_pop(&a->ring[s]);
    a->avail[s] -= (int32_t)keep;
    if (a->avail[s] == 0) oracle_veb_delete(a->btree[t], s);
}

/* R2: up to want / nb consecutive free segments from the front, privately */
static uint32_t take_segments(o2_t *a, uint32_t t, uint32_t want, uint32_t *first) {
    uint32_t nb = nb_of(t);
    uint64_t s0 = claim_front(a);
    if (s0 == NONE64) return 0;
    uint32_t k = 1;
    while (k < want / nb && s0 + k < a->nseg && oracle_veb_member(a->segfree, s0 + k)) {
        oracle_veb_delete(a->segfree, s0 + k);
        k++;
    }
    for (uint32_t q = 0; q < k; q++) format_keep(a, s0 + q, t, nb);
    *first = (uint32_t)(s0 * nb);
    return k * nb;
}

/* R2/R3: a run of up to `want` consecutive blocks of tree t (Alg.2 for a
 * run).  Returns its length (0 = no memory), its first block's linear index
 * in *first. */
static uint32_t get_run_once(o2_t *a, uint32_t t, uint32_t want, uint32_t *first) {
    uint32_t nb = nb_of(t);
    uint64_t s = oracle_veb_successor(a->btree[t], 0);              /* findSegment */
    if (s != NONE64 && want >= nb && (uint32_t)a->avail[s] < want &&
        oracle_veb_successor(a->segfree, 0) != NONE64)              /* R2: whole segments first */
        return take_segments(a, t, want, first);
    if (s != NONE64) {
        uint32_t av = (uint32_t)a->avail[s];
        uint32_t got = want < av ? want : av;                       /* reserve */
        a->avail[s] -= (int32_t)got;
        if (a->avail[s] == 0) oracle_veb_delete(a->btree[t], s);
        if (a->format_ahead && av >= nb / 4 && av - got < nb / 4 &&
            oracle_veb_successor(a->btree[t], s + 1) == NONE64) {   /* R3 */
            uint64_t f = claim_front(a);
            if (f != NONE64) pol_format_segment(a, f, t);
        }
        uint8_t in[256] = {0};
        for (uint32_t q = 0; q < got; q++) in[ring_pop(&a->ring[s])] = 1;
        uint32_t bs = 0, bl = 0, len = 0;                           /* longest consecutive run */
        for (uint32_t j = 0; j <= nb; j++) {
            if (j < nb && in[j]) { len++; continue; }
            if (len > bl) { bl = len; bs = j - len; }
            len = 0;
        }
        for (uint32_t j = 0; j < nb; j++)                           /* the rest back, ascending */
            if (in[j] && (j < bs || j >= bs + bl)) pol_return_block(a, s, j, t);
        *first = (uint32_t)(s * nb + bs);
        return bl;
    }
    if (want >= nb) return take_segments(a, t, want, first);
    uint64_t s1 = claim_front(a);                                   /* Alg.2 -> getSegment */
    if (s1 == NONE64) return 0;
    format_keep(a, s1, t, want);
    *first = (uint32_t)(s1 * nb);
    return want;
}

/* R5: slots give back their undrawn blocks; returns the blocks given back */
static uint64_t trim_slots(o2_t *a) {
    uint64_t back = 0;
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        for (unsigned q = 0; q < a->nslot[c]; q++) {
            unsigned i = a->slot_off[c] + q;
            uint64_t cnt = slot_cnt(a->slot[i]);
            uint32_t m = slot_run(a->slot[i]), first = slot_first(a->slot[i]);
            if (cnt < SLICES_PER_BLOCK * (uint64_t)m) {
                uint32_t m2 = (uint32_t)((cnt + SLICES_PER_BLOCK - 1) / SLICES_PER_BLOCK);
                a->slot[i] = m2 == 0 ? SLOT_EMPTY : slot_make(cnt, m2, first);
                for (uint32_t k = m2; k < m; k++) pol_block_freed(a, gid_of(c, (uint64_t)first + k), SLICES_PER_BLOCK);
                back += m - m2;
            }
            if (a->prefetch) {
                uint32_t nm = slot_run(a->next[i]), nf = slot_first(a->next[i]);
                a->next[i] = SLOT_EMPTY;
                for (uint32_t k = 0; k < nm; k++) pol_block_freed(a, gid_of(c, (uint64_t)nf + k), SLICES_PER_BLOCK);
                back += nm;
            }
        }
    }
    return back;
}

static uint32_t get_run(o2_t *a, uint32_t t, uint32_t want, uint32_t *first) {
    uint32_t got = get_run_once(a, t, want, first);
    if (!got && trim_slots(a)) got = get_run_once(a, t, 1, first);
    return got;
}

/* R1: the first run of an empty slot of class c */
uint32_t runs_first_run(const o2_t *a, uint32_t c) {
    uint32_t fl = a->run_init < 8 ? a->run_init : 8;
    uint32_t fr = (a->run_init >> c) > fl ? (a->run_init >> c) : fl;
    if (fr > nb_of(c)) fr = nb_of(c);
    uint32_t cap = run_cap(a, c);
    return fr < cap ? fr : cap;
}

/* R1/R4: Alg.3 with a run per slot */
static uint64_t malloc_slice(o2_t *a, uint32_t c, uint64_t key) {
    unsigned i = a->slot_off[c] + (unsigned)(key % a->nslot[c]);
    uint32_t cap = run_cap(a, c);
    for (;;) {
        uint64_t cnt = slot_cnt(a->slot[i]);
        uint32_t m = slot_run(a->slot[i]), first = slot_first(a->slot[i]);
        uint32_t grow = (m << a->run_grow) < cap ? (m << a->run_grow) : cap;
        if (cnt < SLICES_PER_BLOCK * m) {                           /* valid index */
            a->slot[i] = slot_make(cnt + 1, m, first);
            if (a->prefetch && cnt == SLICES_PER_BLOCK * m / 2 && a->next[i] == SLOT_EMPTY) {
                uint32_t nf, ng = get_run_once(a, c, grow, &nf);    /* R4 */
                if (ng) a->next[i] = slot_make(0, ng, nf);
            }
            return (uint64_t)first * block_bytes(c) + cnt * (MIN_SLICE << c);
        }
        if (a->next[i] != SLOT_EMPTY) {                             /* the prefetched run */
            a->slot[i] = a->next[i];
            a->next[i] = SLOT_EMPTY;
            continue;
        }
        uint32_t want = m == 0 ? runs_first_run(a, c) : grow;
        uint32_t got = get_run(a, c, want, &first);
        if (!got) { a->slot[i] = SLOT_EMPTY; return NONE64; }       /* nullptr */
        a->slot[i] = slot_make(0, got, first);
    }
}

/* ---------------------------------------------------------- prefill --- */
/* R7 prefill ("each block buffer is always populated", reading A-19):
 * the initial state has every slot, class-major and slot-ascending, holding
 * a run of r[c] consecutive blocks of its class: the blocks of the class's
 * current segment in ring order (a fresh segment when it has none left), or
 * r[c] / nb whole fresh segments.  r[c] starts at the largest power of two
 * <= the first run (R1); while the segments this takes exceed nseg / 8, the
 * class holding the most segments (lowest class on ties) whose r[c] is above
 * max(1, nb >> run_grow) is halved (so the slot's first refill still grows
 * to whole segments); if none can be and it does not fit, the slots start
 * empty. */
static uint64_t prefill_segs(const o2_t *a, const uint32_t *r, unsigned c) {
    return ((uint64_t)a->nslot[c] * r[c] + nb_of(c) - 1) / nb_of(c);
}

void runs_prefill(o2_t *a) {
    uint32_t r[NUM_BLOCK_TREES];
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        uint32_t fr = runs_first_run(a, c);
        r[c] = 1;
        while (r[c] * 2 <= fr) r[c] *= 2;
    }
    for (;;) {
        uint64_t total = 0;
        for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) total += prefill_segs(a, r, c);
        if (total <= a->nseg / 8) break;
        int big = -1;
        for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
            uint32_t floor_ = nb_of(c) >> a->run_grow;
            if (floor_ < 1) floor_ = 1;
            if (r[c] > floor_ && (big < 0 || prefill_segs(a, r, c) > prefill_segs(a, r, (unsigned)big))) big = (int)c;
        }
        if (big < 0) return;                                        /* does not fit: slots start empty */
        r[big] /= 2;
    }
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        uint32_t nb = nb_of(c);
        uint64_t s = NONE64;
        for (unsigned q = 0; q < a->nslot[c]; q++) {
            uint64_t first = 0;
            if (r[c] >= nb) {                                       /* whole segments, all blocks out */
                for (uint32_t k = 0; k < r[c] / nb; k++) {
                    uint64_t x = pol_claim_front(a);
                    pol_format_segment(a, x, c);
                    for (uint32_t j = 0; j < nb; j++) ring_pop(&a->ring[x]);
                    a->avail[x] = 0;
                    oracle_veb_delete(a->btree[c], x);
                    if (k == 0) first = x * nb;
                }
            } else {                                                /* r[c] divides nb */
                if (s == NONE64 || a->avail[s] == 0) {
                    s = pol_claim_front(a);
                    pol_format_segment(a, s, c);
                }
                first = s * nb + a->ring[s].e[a->ring[s].head];
                for (uint32_t j = 0; j < r[c]; j++) ring_pop(&a->ring[s]);
                a->avail[s] -= (int32_t)r[c];
                if (a->avail[s] == 0) oracle_veb_delete(a->btree[c], s);
            }
            a->slot[a->slot_off[c] + q] = slot_make(0, r[c], (uint32_t)first);
        }
    }
}

uint64_t runs_malloc(o2_t *a, uint64_t size, uint64_t key) {
    if (size == 0) return NONE64;
    uint32_t kind, cls;
    uint64_t usable = class_usable(size, &kind, &cls), off;
    if (kind == 0) {
        off = malloc_slice(a, cls, key);
    } else if (kind == 1) {
        uint32_t first;
        if (!get_run(a, cls, 1, &first)) return NONE64;
        a->freecnt[gid_of(cls, first)] = SLICES_PER_BLOCK - 1;     /* A-2 */
        off = (uint64_t)first * block_bytes(cls);
    } else {
        uint64_t i = pol_claim_multiple(a, cls);
        if (i == NONE64 && trim_slots(a)) i = pol_claim_multiple(a, cls);   /* R5 */
        off = i == NONE64 ? NONE64 : i * SEGMENT_BYTES;
    }
    if (off != NONE64) note_malloc(a, off, usable);
    return off;
}

/* Drain: every slot (class-major, slot-ascending) counts the unissued rest of
 * each block of its run as freed; a prefetched run comes back whole; then the
 * idle formatted segments retire (R6). */
void runs_drain(o2_t *a) {
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        for (unsigned q = 0; q < a->nslot[c]; q++) {
            unsigned i = a->slot_off[c] + q;
            uint64_t cnt = slot_cnt(a->slot[i]);
            uint32_t m = slot_run(a->slot[i]), first = slot_first(a->slot[i]);
            a->slot[i] = SLOT_EMPTY;
            for (uint32_t k = 0; k < m; k++) {
                uint64_t lo = SLICES_PER_BLOCK * k;
                uint64_t issued = cnt <= lo ? 0 : (cnt - lo > SLICES_PER_BLOCK ? SLICES_PER_BLOCK : cnt - lo);
                if (issued < SLICES_PER_BLOCK)
                    pol_block_freed(a, gid_of(c, (uint64_t)first + k), (uint32_t)(SLICES_PER_BLOCK - issued));
            }
            uint32_t nm = slot_run(a->next[i]), nf = slot_first(a->next[i]);
            a->next[i] = SLOT_EMPTY;
            for (uint32_t k = 0; k < nm; k++) pol_block_freed(a, gid_of(c, (uint64_t)nf + k), SLICES_PER_BLOCK);
        }
    }
    retire_idle_all(a);
}
