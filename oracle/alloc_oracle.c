/*
 * oracle/alloc_oracle.c -- O2: the SEQUENTIAL Gallatin allocator (CPU).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this code.  It
 * shares no code, header, table or constant with the CUDA path and never
 * calls it.  Its trees are O1 textbook vEB trees (veb_oracle.c).
 *
 * It implements, one request at a time and in the paper's order, the policy
 * of PAPER.md S4-S5 (P = /root/reference/PAPER.md line):
 *   - heap of 16 MB segments; segment tree, bit=1 <=> free;
 *     segments for blocks taken from the FRONT by successor(0);
 *   - one block tree per block size; a segment formatted for tree t
 *     holds nb(t) = 256 >> t blocks (256 blocks at 16 B slices,
 *     128 at 32 B); blocks leave and return through a constant-size
 *     per-segment ring queue, i.e. FIFO; the segment leaves its block
 *     tree when its last block is handed out and rejoins when a block comes
 *     back (reading A-16: on avail 0 -> 1); when every block is back
 *     the segment returns to the segment tree;
 *   - slices: a block holds 4096 slices of 1/4096 of the block, slice
 *     sizes 16 B..4096 B, tree id = log2(size) - log2(16);
 *     slices are handed out in order by a counter (Alg.3 P:212-
 *     213: valid = idx < 4096), address offset(blockId*4096 + idx);
 *   - block buffer: NSLOT(c) = max(slot_min, slot_base >> c) slots per class
 *     (P:195), slot chosen by the request's key mod NSLOT(c) (reading A-6); an
 *     exhausted slot is refilled by the request that finds it exhausted
 *     (Alg.3, reading A-7).
 *   - [ours, DESIGN.md "Deviations"] a slot holds a RUN of m consecutive
 *     blocks (a contiguous address range) handed out slice by slice in order;
 *     m starts at run_init-derived length and grows 2^run_grow-fold on each
 *     refill of the slot up to a cap.  With cap 1 and format_ahead off this is
 *     exactly the paper's one-block buffer.  A run comes from the lowest
 *     segment of the block tree (up to m of its ring entries, keeping the
 *     longest run of consecutive block indices among them and re-enqueueing
 *     the rest in ascending order), else from fresh segments (privately when
 *     m covers whole segments, else one segment is formatted with the run's
 *     blocks removed and the rest published).  Before "no memory", every slot
 *     gives back the blocks of its run no request has drawn from.
 *     format_ahead: the reservation that takes a segment below nb/4 available
 *     blocks formats one more segment for the tree.
 *   - requests in (4 KB, 16 MB): one whole block of tree max(0, ceil(log2
 *     size) - 16) whose free counter is preset to 4095 so that Alg.4's rule
 *      returns it on its one free (reading A-2);
 *   - requests >= 16 MB: k = ceil(size / 16 MB) contiguous segments from the
 *     END of the segment tree, first fit via predecessor search (P:111-113,
 *     P:138, reading A-17: the highest start), tree id = 9 + k;
 *   - free (Alg.4): segment = offset / 16 MB (reading A-10);
 *     tree id < 9: block = (offset in segment) >> log2(block size) (P:239,
 *     reading A-11), free counter += 1, the free that completes 4096 returns
 *     the block (reading A-14); otherwise the k segments are
 *     re-inserted into the segment tree.
 *   - [ours, DESIGN.md Deviations 11] exhaustion record: a run request of
 *     tree t that fails (after the slot trims) records "t exhausted"; later
 *     run requests of t fail at once while the record stands.  Every step
 *     that puts blocks or segments back where a search could find them clears
 *     all records: a block return to a segment with no block available (it
 *     rejoins its block tree), a segment freed, a segment formatted into a
 *     block tree, and the give-backs inside a run request (an over-reservation
 *     of a segment's blocks, the re-enqueued blocks outside the kept run, the
 *     free segments of a claim window past its consecutive prefix).
 *   - drain (reading A-15/SURVEY A15, R-1): retire every block-buffer slot,
 *     the unissued remainder of its run counted as freed; then retire the
 *     segments whose blocks are all home.
 *
 * Canonical metadata image: see include/gallatin.h, "Snapshot image"; this
 * file writes the same documented layout from its own state.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---- O1 (veb_oracle.c) ---- */
typedef struct oracle_veb oracle_veb;
oracle_veb *oracle_veb_create(unsigned k);
void oracle_veb_destroy(oracle_veb *h);
int oracle_veb_member(const oracle_veb *h, uint64_t x);
int oracle_veb_insert(oracle_veb *h, uint64_t x);
int oracle_veb_delete(oracle_veb *h, uint64_t x);
uint64_t oracle_veb_successor(const oracle_veb *h, uint64_t x);
uint64_t oracle_veb_predecessor(const oracle_veb *h, uint64_t x);

#define NONE64 UINT64_MAX
/* The paper's constants, restated (not shared with the CUDA path). */
#define SEGMENT_BYTES (16ULL << 20)   /* P:134 "16MB regions"              */
#define SLICES_PER_BLOCK 4096ULL
#define MIN_SLICE 16ULL               /* P:184 "16 B"                     */
#define MAX_SLICE 4096ULL             /* P:184 "4096 B"                   */
#define NUM_BLOCK_TREES 9u            /* 16 B..4 KB slices -> 64 KB..16 MB blocks (A-1) */
#define MAX_BLOCKS_PER_SEGMENT 256u
#define TREE_FREE 0xFFFFFFFFu         /* segment in the segment tree       */
#define TREE_CONT 0xFFFFFFFEu         /* non-first segment of a large alloc */
#define GID_NONE 0xFFFFFFFFu
#define IMAGE_MAGIC 0x47414C4C494D4731ULL

static uint64_t ceil_log2(uint64_t x) { uint64_t r = 0; while ((1ULL << r) < x) r++; return r; }
static uint32_t nb_of(uint32_t t) { return MAX_BLOCKS_PER_SEGMENT >> t; }
static uint64_t block_bytes(uint32_t t) { return SEGMENT_BYTES / nb_of(t); }

typedef struct { uint16_t e[256]; uint32_t head, count; } ring_t;   /* FIFO */
typedef struct { uint64_t key, val; } kv_t;

typedef struct o2 {
    uint64_t nseg;
    unsigned slot_base, slot_min, run_max, format_ahead, run_init;
    uint64_t run_bytes;
    unsigned nslot[NUM_BLOCK_TREES], slot_off[NUM_BLOCK_TREES], nslot_total;
    uint32_t *tree;               /* memoryTable.ids           */
    int32_t *avail;               /* blocks currently in the ring       */
    ring_t *ring;
    uint32_t *freecnt;            /* per block free counter     */
    oracle_veb *segfree;          /* segment tree               */
    oracle_veb *btree[NUM_BLOCK_TREES];  /* block trees         */
    uint64_t *slot;               /* cnt << 32 | m << 22 | first block  */
    uint64_t *next;               /* prefetched run (m << 22 | first) or empty */
    unsigned prefetch;
    unsigned run_grow;            /* a refill takes m << run_grow blocks        */
    uint64_t err;                 /* out-of-heap / non-allocated segment frees */
    uint32_t oom_rec;             /* [ours] bit t: tree t recorded exhausted    */
    uint64_t oom_fast;            /* run requests failed by the record          */
    /* oracle-only bookkeeping for the invariant checks */
    kv_t *live; uint64_t live_cap, live_n;
    uint64_t usable_live;
    uint64_t violations;          /* bit mask, see o2_violations()      */
} o2_t;

enum { V_FRONT_FIRST = 1, V_BACK_FIRST = 2, V_BAD_FREE = 4, V_OVERLAP = 8,
       V_ALIGN = 16, V_HEAP = 32, V_ACCOUNT = 64, V_TREES = 128, V_RING = 256, V_OOM_RECORD = 512 };

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
            /* backward-shift deletion */
            uint64_t j = i;
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

/* ---------------------------------------------------------- lifecycle --- */
#define RUN_NONE 0x3FFFFFu                          /* 22-bit first block */
#define RUN_SHIFT 22                                /* 10-bit run length  */
#define SLOT_EMPTY ((uint64_t)RUN_NONE)            /* cnt 0, m 0: refill on first use */
static uint64_t slot_make(uint64_t cnt, uint32_t m, uint32_t first) {
    return (cnt << 32) | ((uint64_t)m << RUN_SHIFT) | first;
}

o2_t *o2_create(uint64_t nseg, unsigned slot_base, unsigned slot_min, unsigned run_max,
                uint64_t run_bytes, unsigned format_ahead, unsigned run_init, unsigned prefetch,
                unsigned run_grow) {
    if (run_grow < 1 || run_grow > 8) return NULL;
    if (nseg < 1 || nseg > (1ULL << 14) || slot_base < 1 || run_max < 1 || run_max > 512) return NULL;
    o2_t *a = (o2_t *)calloc(1, sizeof(o2_t));
    a->nseg = nseg; a->slot_base = slot_base; a->slot_min = slot_min;
    a->run_max = run_max; a->run_bytes = run_bytes; a->format_ahead = format_ahead;
    a->run_init = run_init < 1 ? 1 : run_init;
    a->prefetch = prefetch;
    a->run_grow = run_grow;
    unsigned off = 0;
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        unsigned n = slot_base >> c;                  /* halving per class */
        if (n < slot_min) n = slot_min;               /* "capped at four"  */
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
        for (int i = 0; i < 256; i++) a->ring[s].e[i] = 0xFFFF;
    }
    a->slot = (uint64_t *)malloc(a->nslot_total * sizeof(uint64_t));
    a->next = (uint64_t *)malloc(a->nslot_total * sizeof(uint64_t));
    for (unsigned i = 0; i < a->nslot_total; i++) a->slot[i] = a->next[i] = SLOT_EMPTY;
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
uint64_t o2_oom_fast(const o2_t *a) { return a->oom_fast; }
uint64_t o2_live_count(const o2_t *a) { return a->live_n; }
uint64_t o2_usable_live(const o2_t *a) { return a->usable_live; }

/* Largest run (in blocks of tree t) a slot may hold: run_max blocks and
 * run_bytes bytes, at least one block. */
static uint32_t run_cap(const o2_t *a, uint32_t t) {
    uint64_t by = a->run_bytes / block_bytes(t);
    uint64_t m = a->run_max < by ? a->run_max : by;
    return m < 1 ? 1 : (uint32_t)m;
}

/* ------------------------------------------------ ring queue --- */
static uint16_t ring_pop(ring_t *r) {
    uint16_t j = r->e[r->head];
    r->e[r->head] = 0xFFFF;
    r->head = (r->head + 1) & 255; r->count--;
    return j;
}
static void ring_push(ring_t *r, uint16_t j) {
    r->e[(r->head + r->count) & 255] = j;
    r->count++;
}

/* --------------------------------------------- Alg.1 getSegment (front) --- */
/* successor(0) on the segment tree and claimIndex; front-first
 * invariant: every segment below the claimed one is in use. */
/* A formatted segment whose blocks are all home goes back to the segment
 * tree, in segment order (used by drain, and before reporting that every
 * segment is in use). Returns how many were retired. */
static uint64_t retire_idle_all(o2_t *a) {
    uint64_t n = 0;
    for (uint64_t s = 0; s < a->nseg; s++) {
        uint32_t t = a->tree[s];
        if (t < NUM_BLOCK_TREES && (uint32_t)a->avail[s] == nb_of(t)) {
            ring_t *r = &a->ring[s];
            a->tree[s] = TREE_FREE; a->avail[s] = 0;
            r->head = 0; r->count = 0;
            for (int i = 0; i < 256; i++) r->e[i] = 0xFFFF;
            oracle_veb_delete(a->btree[t], s);
            oracle_veb_insert(a->segfree, s);
            a->oom_rec = 0;
            n++;
        }
    }
    return n;
}

static uint64_t claim_front(o2_t *a) {
    uint64_t s = oracle_veb_successor(a->segfree, 0);
    if (s == NONE64 && retire_idle_all(a)) s = oracle_veb_successor(a->segfree, 0);
    if (s == NONE64 || s >= a->nseg) return NONE64;        /* "All segments in use" */
    for (uint64_t i = 0; i < s; i++) if (a->tree[i] == TREE_FREE) a->violations |= V_FRONT_FIRST;
    oracle_veb_delete(a->segfree, s);
    return s;
}

/* initSegment for tree t: blocks [keep, nb) go into the ring and the
 * segment joins block tree t ("broadcast availability"); blocks
 * [0, keep) are handed to the caller. */
static void format_segment(o2_t *a, uint64_t s, uint32_t t, uint32_t keep) {
    uint32_t nb = nb_of(t);
    a->tree[s] = t;
    a->avail[s] = (int32_t)(nb - keep);
    ring_t *r = &a->ring[s];
    r->head = 0; r->count = 0;
    for (uint32_t j = 0; j < 256; j++) r->e[j] = 0xFFFF;
    for (uint32_t j = keep; j < nb; j++) ring_push(r, (uint16_t)j);
    if (a->avail[s] > 0) oracle_veb_insert(a->btree[t], s);
}

/* ------------------------------------------ block / segment return --- */
static void return_block(o2_t *a, uint64_t s, uint32_t j, uint32_t t) {
    if (a->avail[s] == 0) a->oom_rec = 0;                  /* the segment becomes findable */
    ring_push(&a->ring[s], (uint16_t)j);                   /* ring enqueue       */
    a->avail[s]++;
    if ((uint32_t)a->avail[s] == nb_of(t)) {               /* every block back  */
        ring_t *r = &a->ring[s];
        a->tree[s] = TREE_FREE; a->avail[s] = 0;
        r->head = 0; r->count = 0;
        for (int i = 0; i < 256; i++) r->e[i] = 0xFFFF;
        oracle_veb_delete(a->btree[t], s);
        oracle_veb_insert(a->segfree, s);                   /* back to segment tree */
        a->oom_rec = 0;
    } else if (a->avail[s] == 1) {
        oracle_veb_insert(a->btree[t], s);                  /* re-added (A-16)    */
    }
}

static void block_freed(o2_t *a, uint32_t gid, uint32_t count) {
    a->freecnt[gid] += count;
    if (a->freecnt[gid] == SLICES_PER_BLOCK) {              /* P:250 (== 4095 before) */
        a->freecnt[gid] = 0;
        uint64_t s = gid / MAX_BLOCKS_PER_SEGMENT;
        return_block(a, s, gid % MAX_BLOCKS_PER_SEGMENT, a->tree[s]);
    }
}

/* [ours] the run covers whole segments: take up to want/nb consecutive free
 * segments from the front, privately (no ring, no block tree).  Returns the
 * blocks taken, 0 if no segment is free. */
static uint32_t take_segments(o2_t *a, uint32_t t, uint32_t want, uint32_t *first) {
    uint32_t nb = nb_of(t);
    uint64_t s0 = claim_front(a);
    if (s0 == NONE64) return 0;
    uint32_t k = 1;
    const uint64_t kmax = want / nb;
    while (k < kmax && s0 + k < a->nseg && oracle_veb_member(a->segfree, s0 + k)) {
        oracle_veb_delete(a->segfree, s0 + k);
        k++;
    }
    /* [ours] the CUDA claim takes every free segment of a window [x, end) --
     * end = min(x + segments still wanted, x's word end, nseg), words of 64 --
     * and gives back those past the consecutive prefix; a window that the
     * prefix fills up to a word end continues in the next word */
    for (uint64_t x = s0;;) {
        uint64_t end = x + (kmax - (x - s0)), wend = (x | 63) + 1;
        if (end > wend) end = wend;
        if (end > a->nseg) end = a->nseg;
        if (s0 + k < end) {
            for (uint64_t y = s0 + k + 1; y < end; y++)
                if (oracle_veb_member(a->segfree, y)) { a->oom_rec = 0; break; }
            break;
        }
        if (k >= kmax || end >= a->nseg || (end & 63)) break;
        x = end;
    }
    for (uint32_t q = 0; q < k; q++) format_segment(a, s0 + q, t, nb);
    *first = (uint32_t)(s0 * nb);
    return k * nb;
}

static uint32_t gid_of(uint32_t t, uint64_t linear) {
    uint32_t nb = nb_of(t);
    return (uint32_t)((linear / nb) * MAX_BLOCKS_PER_SEGMENT + linear % nb);
}

/* --------------------------------------------------- Alg.2 getBlock --- */
/* A run of up to `want` consecutive blocks of tree t.  Returns the number of
 * blocks (0 = no memory) and the first block's linear index in *first
 * (segment * nb + block). */
static uint32_t get_run_once(o2_t *a, uint32_t t, uint32_t want, uint32_t *first) {
    uint32_t nb = nb_of(t);
    uint64_t s = oracle_veb_successor(a->btree[t], 0);     /* findSegment */
    if (s != NONE64) {
        ring_t *r = &a->ring[s];
        uint32_t av = (uint32_t)a->avail[s];
        uint32_t got = want < av ? want : av;              /* reserve */
        uint32_t low = nb / 4;
        if (av < want) a->oom_rec = 0;                      /* over-reservation given back */
        a->avail[s] -= (int32_t)got;
        if (a->avail[s] == 0) oracle_veb_delete(a->btree[t], s);   /* no over-subscription */
        if (a->format_ahead && av >= low && av - got < low &&
            oracle_veb_successor(a->btree[t], s + 1) == NONE64) {
            uint64_t f = claim_front(a);                      /* format one segment ahead */
            if (f != NONE64) { format_segment(a, f, t, 0); a->oom_rec = 0; }
        }
        uint8_t in[256] = {0};
        for (uint32_t q = 0; q < got; q++) in[ring_pop(r)] = 1;     /* getBlock */
        /* [ours] keep the longest run of consecutive block indices among them
         * (lowest start on ties); the others go back in ascending order */
        uint32_t bs = 0, bl = 0, len = 0;
        for (uint32_t j = 0; j <= nb; j++) {
            if (j < nb && in[j]) { len++; continue; }
            if (len > bl) { bl = len; bs = j - len; }
            len = 0;
        }
        for (uint32_t j = 0; j < nb; j++)
            if (in[j] && (j < bs || j >= bs + bl)) return_block(a, s, j, t);
        if (bl < got) a->oom_rec = 0;                       /* re-enqueued: clears the record */
        *first = (uint32_t)(s * nb + bs);
        return bl;
    }
    if (want >= nb) return take_segments(a, t, want, first);  /* 0: "No allocations left" */
    uint64_t s1 = claim_front(a);                             /* Alg.2 -> getSegment */
    if (s1 == NONE64) return 0;
    format_segment(a, s1, t, want);
    a->oom_rec = 0;
    *first = (uint32_t)(s1 * nb);
    return want;
}


/* [ours, DESIGN.md Deviations 5] Before "no memory": every slot, class-major
 * and slot-ascending, keeps only the ceil(issued / 4096) blocks of its run that
 * requests have drawn from (an undrawn slot becomes empty); the other blocks
 * come back whole, in block order, then a prefetched next run comes back
 * whole.  Returns the number of blocks given back. */
static uint64_t trim_slots(o2_t *a) {
    uint64_t back = 0;
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        for (unsigned q = 0; q < a->nslot[c]; q++) {
            unsigned i = a->slot_off[c] + q;
            uint64_t cnt = a->slot[i] >> 32;
            uint32_t m = (uint32_t)(a->slot[i] >> RUN_SHIFT) & 0x3FF;
            uint32_t first = (uint32_t)a->slot[i] & RUN_NONE;
            if (cnt < SLICES_PER_BLOCK * (uint64_t)m) {
                uint32_t m2 = (uint32_t)((cnt + SLICES_PER_BLOCK - 1) / SLICES_PER_BLOCK);
                a->slot[i] = m2 == 0 ? SLOT_EMPTY : slot_make(cnt, m2, first);
                for (uint32_t k = m2; k < m; k++) block_freed(a, gid_of(c, (uint64_t)first + k), SLICES_PER_BLOCK);
                back += m - m2;
            }
            if (a->prefetch) {
                uint32_t nm = (uint32_t)(a->next[i] >> RUN_SHIFT) & 0x3FF;
                uint32_t nf = (uint32_t)a->next[i] & RUN_NONE;
                a->next[i] = SLOT_EMPTY;
                for (uint32_t k = 0; k < nm; k++) block_freed(a, gid_of(c, (uint64_t)nf + k), SLICES_PER_BLOCK);
                back += nm;
            }
        }
    }
    return back;
}

/* A run of up to `want` blocks (get_run_once); on "no memory" the slots give
 * back their undrawn blocks and the request is retried once, for a single
 * block: memory is scarce, so no slot hoards a run of it (DESIGN.md
 * Deviations 5, "near exhaustion"). */
/* Check of the exhaustion record, without changing any state: would the full
 * search for one block of tree t (get_run_once, then the slot trims and a
 * retry) succeed?  It succeeds iff tree t holds a segment, a segment is free
 * or formatted with all blocks home, or the blocks the trims would give back
 * include one of tree t or complete a segment's blocks. */
static int search_would_succeed(const o2_t *a, uint32_t t) {
    if (oracle_veb_successor(a->btree[t], 0) != NONE64) return 1;
    if (oracle_veb_successor(a->segfree, 0) != NONE64) return 1;
    for (uint64_t s = 0; s < a->nseg; s++)
        if (a->tree[s] < NUM_BLOCK_TREES && (uint32_t)a->avail[s] == nb_of(a->tree[s])) return 1;
    uint32_t *back = (uint32_t *)calloc(a->nseg, sizeof(uint32_t));
    int ok = 0;
    for (unsigned c = 0; c < NUM_BLOCK_TREES && !ok; c++) {
        for (unsigned q = 0; q < a->nslot[c] && !ok; q++) {
            unsigned i = a->slot_off[c] + q;
            uint64_t cnt = a->slot[i] >> 32;
            uint32_t m = (uint32_t)(a->slot[i] >> RUN_SHIFT) & 0x3FF, first = (uint32_t)a->slot[i] & RUN_NONE;
            uint32_t m2 = cnt < SLICES_PER_BLOCK * (uint64_t)m ? (uint32_t)((cnt + SLICES_PER_BLOCK - 1) / SLICES_PER_BLOCK) : m;
            uint32_t nm = a->prefetch ? (uint32_t)(a->next[i] >> RUN_SHIFT) & 0x3FF : 0;
            uint32_t nf = (uint32_t)a->next[i] & RUN_NONE;
            for (uint32_t k = 0; k < (m - m2) + nm && !ok; k++) {
                uint32_t gid = k < m - m2 ? gid_of(c, (uint64_t)first + m2 + k) : gid_of(c, (uint64_t)nf + k - (m - m2));
                uint64_t s = gid / MAX_BLOCKS_PER_SEGMENT;
                if (a->freecnt[gid] != 0) continue;             /* not whole: the trim does not return it */
                if (c == t) ok = 1;
                else if ((uint32_t)a->avail[s] + ++back[s] == nb_of(c)) ok = 1;
            }
        }
    }
    free(back);
    return ok;
}

static uint32_t get_run(o2_t *a, uint32_t t, uint32_t want, uint32_t *first) {
    if ((a->oom_rec >> t) & 1) {                              /* [ours] exhaustion record */
        if (search_would_succeed(a, t)) a->violations |= V_OOM_RECORD;
        a->oom_fast++;
        return 0;
    }
    uint32_t got = get_run_once(a, t, want, first);
    if (!got && trim_slots(a)) got = get_run_once(a, t, 1, first);
    if (!got) a->oom_rec |= 1u << t;
    return got;
}

/* ------------------------------------------ claimMultiple (back) --- */
/* Highest start i with [i, i+k) all free: walk down with predecessor (P:112,
 * P:138, reading A-17). */
static uint64_t claim_multiple(o2_t *a, uint64_t k) {
    if (k > a->nseg) return NONE64;
    uint64_t x = a->nseg - 1;
    for (;;) {
        uint64_t y = oracle_veb_predecessor(a->segfree, x);
        if (y == NONE64) return NONE64;
        uint64_t run = 1;
        while (run < k && y >= run && oracle_veb_member(a->segfree, y - run)) run++;
        if (run >= k) {
            uint64_t i = y - k + 1;
            /* back-first invariant: no free window starts above i */
            for (uint64_t j = i + 1; j + k <= a->nseg; j++) {
                uint64_t m = 0;
                while (m < k && a->tree[j + m] == TREE_FREE) m++;
                if (m == k) a->violations |= V_BACK_FIRST;
            }
            for (uint64_t m = 0; m < k; m++) oracle_veb_delete(a->segfree, i + m);
            a->tree[i] = NUM_BLOCK_TREES + (uint32_t)k;
            for (uint64_t m = 1; m < k; m++) a->tree[i + m] = TREE_CONT;   /* A-18 */
            return i;
        }
        if (y < run + 1) return NONE64;
        x = y - run - 1;  /* y - run is in use; continue below it */
        if (x == NONE64) return NONE64;
    }
}

/* ------------------------------------------------------------ malloc --- */
/* offset(blockId*4096 + idx): slices of a run are consecutive; the
 * run's first block has linear index `first` in units of the class's block. */
static uint64_t slice_addr(uint32_t first, uint32_t c, uint64_t idx) {
    return (uint64_t)first * block_bytes(c) + idx * (MIN_SLICE << c);
}

static uint64_t malloc_slice(o2_t *a, uint32_t c, uint64_t key) {
    unsigned i = a->slot_off[c] + (unsigned)(key % a->nslot[c]);
    for (;;) {
        uint64_t cnt = a->slot[i] >> 32;
        uint32_t m = (uint32_t)(a->slot[i] >> RUN_SHIFT) & 0x3FF;
        uint32_t first = (uint32_t)a->slot[i] & RUN_NONE;
        uint32_t cap = run_cap(a, c);
        uint32_t grow = (m << a->run_grow) < cap ? (m << a->run_grow) : cap;   /* [ours] x 2^run_grow */
        if (cnt < SLICES_PER_BLOCK * m) {                   /* valid = idx < 4096 (per block) */
            a->slot[i] = slot_make(cnt + 1, m, first);
            uint64_t off = slice_addr(first, c, cnt);
            if (a->prefetch && cnt == SLICES_PER_BLOCK * m / 2 && a->next[i] == SLOT_EMPTY) {
                uint32_t nf;                                  /* [ours] prefetch the next run */
                uint32_t ng = get_run_once(a, c, grow, &nf);   /* never trims other slots */
                if (ng) a->next[i] = slot_make(0, ng, nf);
            }
            return off;
        }
        /* exhausted: this request replaces the run (Alg.3) */
        if (a->next[i] != SLOT_EMPTY) {                       /* the prefetched run */
            a->slot[i] = a->next[i];
            a->next[i] = SLOT_EMPTY;
            continue;
        }
        /* empty slot: max(run_init >> c, min(run_init, 8)) blocks, at most one
           segment (256 >> c blocks) and the class cap [ours, DESIGN.md Deviations 5] */
        uint32_t fl = a->run_init < 8 ? a->run_init : 8;
        uint32_t fr = (a->run_init >> c) > fl ? (a->run_init >> c) : fl;
        if (fr > (256u >> c)) fr = 256u >> c;
        uint32_t first_run = fr < cap ? fr : cap;
        uint32_t want = m == 0 ? first_run : grow;
        uint32_t got = get_run(a, c, want, &first);
        if (!got) {
            a->slot[i] = SLOT_EMPTY;
            return NONE64;                                   /* nullptr */
        }
        a->slot[i] = slot_make(0, got, first);
    }
}

static uint64_t class_usable(uint64_t size, uint32_t *kind, uint32_t *cls) {
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

/* Usable bytes a request of `size` receives (A-1..A-4); 0 for size 0. */
uint64_t o2_usable_size(uint64_t size) {
    if (size == 0) return 0;
    uint32_t kind, cls;
    return class_usable(size, &kind, &cls);
}

uint64_t o2_malloc(o2_t *a, uint64_t size, uint64_t key) {
    if (size == 0) return NONE64;                            /* reading A-4 */
    uint32_t kind, cls;
    uint64_t usable = class_usable(size, &kind, &cls);
    uint64_t off;
    if (kind == 0) {
        off = malloc_slice(a, cls, key);
    } else if (kind == 1) {
        uint32_t first;
        if (!get_run(a, cls, 1, &first)) return NONE64;
        uint32_t gid = gid_of(cls, first);
        a->freecnt[gid] = SLICES_PER_BLOCK - 1;              /* one free returns it (A-2) */
        off = (uint64_t)first * block_bytes(cls);
    } else {
        uint64_t i = claim_multiple(a, cls);
        if (i == NONE64 && trim_slots(a)) i = claim_multiple(a, cls);   /* [ours] as get_run */
        if (i == NONE64) return NONE64;
        off = i * SEGMENT_BYTES;
    }
    if (off == NONE64) return NONE64;
    /* invariants on the new allocation */
    if (off + usable > a->nseg * SEGMENT_BYTES) a->violations |= V_HEAP;
    uint64_t align = usable < SEGMENT_BYTES ? usable : SEGMENT_BYTES;
    if (off % align) a->violations |= V_ALIGN;
    live_put(a, off, usable);
    a->usable_live += usable;
    return off;
}

/* ------------------------------------------------------- Alg.4 free --- */
void o2_free(o2_t *a, uint64_t off) {
    if (off == NONE64) return;                               /* free(NULL) */
    if (off >= a->nseg * SEGMENT_BYTES) { a->err++; return; }
    uint64_t usable;
    if (live_take(a, off, &usable)) a->usable_live -= usable;
    else a->violations |= V_BAD_FREE;
    uint64_t s = off / SEGMENT_BYTES;
    uint32_t t = a->tree[s];
    if (t < NUM_BLOCK_TREES) {
        uint32_t j = (uint32_t)((off % SEGMENT_BYTES) / block_bytes(t));
        block_freed(a, (uint32_t)(s * MAX_BLOCKS_PER_SEGMENT + j), 1);
    } else if (t != TREE_FREE && t != TREE_CONT) {
        uint64_t k = t - NUM_BLOCK_TREES;
        a->oom_rec = 0;
        for (uint64_t m = 0; m < k; m++) {
            a->tree[s + m] = TREE_FREE; a->avail[s + m] = 0;
            oracle_veb_insert(a->segfree, s + m);
        }
    } else {
        a->err++;
    }
}

/* Retire every block-buffer slot in class-major, slot-ascending order: the
 * unissued remainder of each block of its run is counted as freed.  Then
 * every segment whose blocks are all home (formatted ahead and never used)
 * goes back to the segment tree, in segment order. */
void o2_drain(o2_t *a) {
    for (unsigned c = 0; c < NUM_BLOCK_TREES; c++) {
        for (unsigned q = 0; q < a->nslot[c]; q++) {
            unsigned i = a->slot_off[c] + q;
            uint64_t cnt = a->slot[i] >> 32;
            uint32_t m = (uint32_t)(a->slot[i] >> RUN_SHIFT) & 0x3FF;
            uint32_t first = (uint32_t)a->slot[i] & RUN_NONE;
            a->slot[i] = SLOT_EMPTY;
            for (uint32_t k = 0; k < m; k++) {
                uint64_t lo = SLICES_PER_BLOCK * k;
                uint64_t issued = cnt <= lo ? 0 : (cnt - lo > SLICES_PER_BLOCK ? SLICES_PER_BLOCK : cnt - lo);
                if (issued < SLICES_PER_BLOCK)
                    block_freed(a, gid_of(c, (uint64_t)first + k), (uint32_t)(SLICES_PER_BLOCK - issued));
            }
            /* a prefetched run was never issued from: all of it comes back */
            uint32_t nm = (uint32_t)(a->next[i] >> RUN_SHIFT) & 0x3FF;
            uint32_t nf = (uint32_t)a->next[i] & RUN_NONE;
            a->next[i] = SLOT_EMPTY;
            for (uint32_t k = 0; k < nm; k++) block_freed(a, gid_of(c, (uint64_t)nf + k), (uint32_t)SLICES_PER_BLOCK);
        }
    }
    retire_idle_all(a);
}

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

/* Bulk helpers for timing the oracle on a workload (one thread, in order):
 * malloc every size (key = i / keydiv, i.e. the request's warp), then free
 * every returned offset in the same order. */
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
    /* live allocations never overlap (sort and scan) */
    kv_t *v = (kv_t *)malloc((a->live_n + 1) * sizeof(kv_t));
    uint64_t n = 0, sum = 0;
    for (uint64_t i = 0; i < a->live_cap; i++) if (a->live[i].key != NONE64) v[n++] = a->live[i];
    qsort(v, n, sizeof(kv_t), cmp_kv);
    for (uint64_t i = 0; i < n; i++) {
        sum += v[i].val;
        if (i + 1 < n && v[i].key + v[i].val > v[i + 1].key) a->violations |= V_OVERLAP;
    }
    free(v);
    if (sum != a->usable_live) a->violations |= V_ACCOUNT;
    /* trees agree with the memory table */
    for (uint64_t s = 0; s < a->nseg; s++) {
        uint32_t t = a->tree[s];
        int fr = oracle_veb_member(a->segfree, s);
        if (fr != (t == TREE_FREE)) a->violations |= V_TREES;
        for (uint32_t b = 0; b < NUM_BLOCK_TREES; b++) {
            int want = (t == b) && a->avail[s] > 0;
            if (oracle_veb_member(a->btree[b], s) != want) a->violations |= V_TREES;
        }
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

static void tree_image(const oracle_veb *t, uint64_t nbits, uint64_t *out) {
    uint64_t wpl[16]; unsigned L;
    uint64_t total = tree_words(nbits, wpl, &L);
    memset(out, 0, total * sizeof(uint64_t));
    for (uint64_t x = oracle_veb_successor(t, 0); x != NONE64 && x < nbits;
         x = oracle_veb_successor(t, x + 1))
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

/* Canonical image; layout documented in include/gallatin.h. */
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
