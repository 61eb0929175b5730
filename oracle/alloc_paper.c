/*
 * oracle/alloc_paper.c -- O2-P: the paper's allocator policy POL, sequential.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this code.  It
 * shares no code, header, table or constant with the CUDA path and never
 * calls it.  Its trees are O1 textbook vEB trees (veb_oracle.c).
 *
 * One request at a time, in the paper's order (P = /root/reference/PAPER.md
 * line, A-n = the reading in SURVEY.md 8(c) / DESIGN.md 2):
 *   - the heap is a row of 16 MB segments in a segment tree, bit = 1
 *     <=> free; block segments come from the FRONT: successor(0)
 *     (Alg.1);
 *   - one block tree per block size (A-1: 4096-slice blocks of 64 KB
 *     .. 16 MB, nb(t) = 256 >> t per segment); a segment formatted for
 *     tree t puts its blocks in a per-segment ring queue (A-15: FIFO)
 *     and joins block tree t ("broadcast availability"); GetBlock
 *     (Alg.2) takes the lowest segment of the tree and the ring's
 *     head; the segment leaves the tree when its last block goes and
 *     rejoins when one comes back (A-16: avail 0 -> 1);
 *   - slices (Alg.3): class c = ceil(log2 size) - 4;
 *     block buffer of NSLOT(c) = max(slot_min, slot_base >> c) one-block slots
 *     (A-5), slot = key mod NSLOT(c) (A-6); a counter hands out the
 *     block's 4096 slices in order, valid iff idx < 4096,
 *     address offset(blockId * 4096 + idx); the request that finds no
 *     valid index replaces the block (A-7); exhaustion -> NULL
 *     (P:118);
 *   - (4 KB, 16 MB): one whole block of tree max(0, ceil(log2 size) - 16),
 *     its free counter preset to 4095 so Alg.4's rule returns it on its one
 *     free (A-2); >= 16 MB: k = ceil(size / 16 MB) segments from the END, the
 *     highest start with k free (A-17), tree id 9 + k
 *     (P:143), the others CONT (A-18);
 *   - free (Alg.4): segment = offset >> 24 (A-10); tree id <
 *     9: block = offset in segment >> log2(block bytes) (A-11), count
 *     the free, the 4096th returns the block (A-14) and the segment
 *     goes back to the segment tree once all its blocks are home (P:178,
 *     P:237); a large allocation's k segments rejoin the tree;
 *   - drain (A15, R-1): retire every slot; the unissued rest of its block
 *     counts as freed.
 * There is no trim, exhaustion record, run or prefetch here (those are
 * alloc_runs.c, the deviation model).  Pins: tests/test_oracle_alloc.py and
 * the brute-force POL simulation tests/pol_sim.py.
 */
#include <stdlib.h>
#include <string.h>

#include "alloc_state.h"

/* ------------------------------------------ Alg.1 GetSegment (front) --- */
/* successor(0) + claimIndex.  Front first: every segment
 * below the claimed one is in use. */
uint64_t pol_claim_front(o2_t *a) {
    uint64_t s = oracle_veb_successor(a->segfree, 0);
    if (s == NONE64 || s >= a->nseg) return NONE64;                 /* "All segments in use" */
    for (uint64_t i = 0; i < s; i++)
        if (a->tree[i] == TREE_FREE) a->violations |= V_FRONT_FIRST;
    oracle_veb_delete(a->segfree, s);
    return s;
}

/* initSegment for tree t: all nb(t) blocks into the ring, in order,
 * and the segment joins block tree t. */
void pol_format_segment(o2_t *a, uint64_t s, uint32_t t) {
    a->tree[s] = t;
    a->avail[s] = (int32_t)nb_of(t);
    ring_clear(&a->ring[s]);
    for (uint32_t j = 0; j < nb_of(t); j++) ring_push(&a->ring[s], (uint16_t)j);
    oracle_veb_insert(a->btree[t], s);
}

/* ------------------------------------------------- Alg.2 GetBlock --- */
/* Returns the block's linear index (segment * nb + block) or NONE64. */
static uint64_t get_block(o2_t *a, uint32_t t) {
    uint64_t s = oracle_veb_successor(a->btree[t], 0);              /* findSegment */
    if (s == NONE64) {
        s = pol_claim_front(a);
        if (s == NONE64) return NONE64;                             /* "No allocations left" */
        pol_format_segment(a, s, t);
    }
    uint32_t j = ring_pop(&a->ring[s]);                             /* getBlock */
    if (--a->avail[s] == 0) oracle_veb_delete(a->btree[t], s);
    return s * nb_of(t) + j;
}

/* ----------------------------------------- block / segment return --- */
/* ring enqueue; all blocks home -> the segment tree;
 * avail 0 -> 1 -> back in the block tree (A-16). */
void pol_return_block(o2_t *a, uint64_t s, uint32_t j, uint32_t t) {
    ring_push(&a->ring[s], (uint16_t)j);
    a->avail[s]++;
    if ((uint32_t)a->avail[s] == nb_of(t)) {
        a->tree[s] = TREE_FREE;
        a->avail[s] = 0;
        ring_clear(&a->ring[s]);
        oracle_veb_delete(a->btree[t], s);
        oracle_veb_insert(a->segfree, s);
    } else if (a->avail[s] == 1) {
        oracle_veb_insert(a->btree[t], s);
    }
}

/* count frees of block gid; the free completing 4096 returns it (A-14) */
void pol_block_freed(o2_t *a, uint32_t gid, uint32_t count) {
    a->freecnt[gid] += count;
    if (a->freecnt[gid] == SLICES_PER_BLOCK) {
        a->freecnt[gid] = 0;
        uint64_t s = gid / MAX_BLOCKS_PER_SEGMENT;
        pol_return_block(a, s, gid % MAX_BLOCKS_PER_SEGMENT, a->tree[s]);
    }
}

/* ------------------------------------------- claimMultiple (back) --- */
/* Highest start i with [i, i+k) all free, walking down with predecessor
 * (A-17).  Returns i or NONE64. */
uint64_t pol_claim_multiple(o2_t *a, uint64_t k) {
    if (k > a->nseg) return NONE64;
    uint64_t x = a->nseg - 1;
    for (;;) {
        uint64_t y = oracle_veb_predecessor(a->segfree, x);
        if (y == NONE64) return NONE64;
        uint64_t run = 1;                                           /* free run ending at y */
        while (run < k && y >= run && oracle_veb_member(a->segfree, y - run)) run++;
        if (run >= k) {
            uint64_t i = y - k + 1;
            for (uint64_t j = i + 1; j + k <= a->nseg; j++) {       /* no free window above i */
                uint64_t m = 0;
                while (m < k && a->tree[j + m] == TREE_FREE) m++;
                if (m == k) a->violations |= V_BACK_FIRST;
            }
            for (uint64_t m = 0; m < k; m++) oracle_veb_delete(a->segfree, i + m);
            a->tree[i] = NUM_BLOCK_TREES + (uint32_t)k;
            for (uint64_t m = 1; m < k; m++) a->tree[i + m] = TREE_CONT;   /* A-18 */
            return i;
        }
        if (y < run + 1) return NONE64;                             /* nothing below y - run */
        x = y - run - 1;
    }
}

/* --------------------------------------------- Alg.3 MALLOC.Slice --- */
static uint64_t malloc_slice(o2_t *a, uint32_t c, uint64_t key) {
    uint64_t *w = &a->slot[a->slot_off[c] + key % a->nslot[c]];
    if (*w == SLOT_EMPTY || slot_cnt(*w) == SLICES_PER_BLOCK) {      /* no valid index: replace */
        uint64_t b = get_block(a, c);
        if (b == NONE64) { *w = SLOT_EMPTY; return NONE64; }        /* nullptr */
        *w = slot_make(0, 1, (uint32_t)b);
    }
    uint64_t idx = slot_cnt(*w);
    *w = slot_make(idx + 1, 1, slot_first(*w));
    return (uint64_t)slot_first(*w) * block_bytes(c) + idx * (MIN_SLICE << c);
}

uint64_t pol_malloc(o2_t *a, uint64_t size, uint64_t key) {
    if (size == 0) return NONE64;                                   /* A-4 */
    uint32_t kind, cls;
    uint64_t usable = class_usable(size, &kind, &cls), off;
    if (kind == 0) {
        off = malloc_slice(a, cls, key);
    } else if (kind == 1) {                                         /* whole block (A-2) */
        uint64_t b = get_block(a, cls);
        if (b == NONE64) return NONE64;
        a->freecnt[gid_of(cls, b)] = SLICES_PER_BLOCK - 1;
        off = b * block_bytes(cls);
    } else {                                                        /* k segments */
        uint64_t i = pol_claim_multiple(a, cls);
        off = i == NONE64 ? NONE64 : i * SEGMENT_BYTES;
    }
    if (off != NONE64) note_malloc(a, off, usable);
    return off;
}

/* ------------------------------------------------------ Alg.4 FREE --- */
void pol_free(o2_t *a, uint64_t off) {
    if (off == NONE64) return;                                      /* free(NULL) */
    if (off >= a->nseg * SEGMENT_BYTES) { a->err++; return; }
    note_free(a, off);
    uint64_t s = off / SEGMENT_BYTES;
    uint32_t t = a->tree[s];
    if (t < NUM_BLOCK_TREES) {
        uint32_t j = (uint32_t)((off % SEGMENT_BYTES) / block_bytes(t));
        pol_block_freed(a, (uint32_t)(s * MAX_BLOCKS_PER_SEGMENT + j), 1);
    } else if (t != TREE_FREE && t != TREE_CONT) {
        for (uint64_t m = 0; m < t - NUM_BLOCK_TREES; m++) {
            a->tree[s + m] = TREE_FREE;
            oracle_veb_insert(a->segfree, s + m);
        }
    } else {
        a->err++;                                                   /* A-27 */
    }
}

/* ------------------------------------------------------------ drain --- */
/* Retire every slot, class-major and slot-ascending: the 4096 - issued
 * slices of its block no request drew count as freed (R-1). */
void pol_drain(o2_t *a) {
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        for (unsigned q = 0; q < a->nslot[c]; q++) {
            uint64_t *w = &a->slot[a->slot_off[c] + q];
            if (*w != SLOT_EMPTY && slot_cnt(*w) < SLICES_PER_BLOCK)
                pol_block_freed(a, gid_of(c, slot_first(*w)), (uint32_t)(SLICES_PER_BLOCK - slot_cnt(*w)));
            *w = SLOT_EMPTY;
        }
    }
}
