/*
 * oracle/alloc_state.h -- state shared by the two O2 models (TEST
 * INFRASTRUCTURE ONLY; see alloc_paper.c).  Internal to oracle/: the CUDA
 * path never includes it and it includes nothing of the CUDA path.
 *
 *   alloc_state.c  lifecycle, live-allocation map, invariant check, image
 *   alloc_paper.c  O2-P: the paper's policy POL (Alg. 1-4, one-block buffer)
 *   alloc_runs.c   O2-R: the deviation model (runs of blocks, format-ahead,
 *                  prefetch, slot trims before "no memory"), built on O2-P's
 *                  primitives
 */
#ifndef GALLATIN_ORACLE_ALLOC_STATE_H
#define GALLATIN_ORACLE_ALLOC_STATE_H
#include <stdint.h>

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
#define SEGMENT_BYTES (16ULL << 20)   /* P:134 "16MB regions"                      */
#define SLICES_PER_BLOCK 4096ULL
#define MIN_SLICE 16ULL               /* P:184 "16 B"                              */
#define MAX_SLICE 4096ULL             /* P:184 "4096 B"                            */
#define NUM_BLOCK_TREES 9u            /* 16 B..4 KB slices -> 64 KB..16 MB blocks (A-1) */
#define MAX_BLOCKS_PER_SEGMENT 256u
#define TREE_FREE 0xFFFFFFFFu         /* segment in the segment tree               */
#define TREE_CONT 0xFFFFFFFEu         /* non-first segment of a large allocation   */

/* A block-buffer slot word (same layout as the image documents):
 * issued slices << 32 | run length (blocks) << 22 | first block (linear index
 * segment * nb + block, in units of the class's block).  EMPTY = no run. */
#define RUN_NONE 0x3FFFFFu
#define RUN_SHIFT 22
#define SLOT_EMPTY ((uint64_t)RUN_NONE)

typedef struct { uint16_t e[256]; uint32_t head, count; } ring_t;   /* FIFO ring queue */
typedef struct { uint64_t key, val; } kv_t;

typedef struct o2 {
    uint64_t nseg;
    int runs;                     /* 0: O2-P (alloc_paper.c), 1: O2-R (alloc_runs.c) */
    unsigned nslot[NUM_BLOCK_TREES], slot_off[NUM_BLOCK_TREES], nslot_total;
    /* O2-R knobs (DESIGN.md Deviations 5); unused by O2-P */
    unsigned run_max, format_ahead, run_init, prefetch, run_grow;
    uint64_t run_bytes;
    /* the allocator */
    uint32_t *tree;               /* memoryTable.ids                  */
    int32_t *avail;               /* blocks in the segment's ring             */
    ring_t *ring;
    uint32_t *freecnt;            /* per block free counter           */
    oracle_veb *segfree;          /* segment tree, bit = free         */
    oracle_veb *btree[NUM_BLOCK_TREES];   /* block trees              */
    uint64_t *slot;               /* block buffer                     */
    uint64_t *next;               /* O2-R: prefetched run, else SLOT_EMPTY    */
    uint64_t err;                 /* frees of pointers outside live segments  */
    /* oracle-only bookkeeping for the invariant checks */
    kv_t *live; uint64_t live_cap, live_n;
    uint64_t usable_live;
    uint64_t violations;          /* bit mask, see alloc_state.c               */
} o2_t;

enum { V_FRONT_FIRST = 1, V_BACK_FIRST = 2, V_BAD_FREE = 4, V_OVERLAP = 8,
       V_ALIGN = 16, V_HEAP = 32, V_ACCOUNT = 64, V_TREES = 128, V_RING = 256 };

/* geometry */
uint64_t ceil_log2(uint64_t x);
uint32_t nb_of(uint32_t t);
uint64_t block_bytes(uint32_t t);
uint32_t gid_of(uint32_t t, uint64_t linear);
uint64_t class_usable(uint64_t size, uint32_t *kind, uint32_t *cls);
static inline uint64_t slot_make(uint64_t cnt, uint32_t m, uint32_t first) {
    return (cnt << 32) | ((uint64_t)m << RUN_SHIFT) | first;
}
static inline uint64_t slot_cnt(uint64_t w) { return w >> 32; }
static inline uint32_t slot_run(uint64_t w) { return (uint32_t)(w >> RUN_SHIFT) & 0x3FF; }
static inline uint32_t slot_first(uint64_t w) { return (uint32_t)w & RUN_NONE; }

/* ring queue */
uint16_t ring_pop(ring_t *r);
void ring_push(ring_t *r, uint16_t j);
void ring_clear(ring_t *r);

/* invariant bookkeeping (alloc_state.c) */
void note_malloc(o2_t *a, uint64_t off, uint64_t usable);
void note_free(o2_t *a, uint64_t off);

/* O2-P primitives (alloc_paper.c), also used by O2-R */
uint64_t pol_claim_front(o2_t *a);
void pol_format_segment(o2_t *a, uint64_t s, uint32_t t);
void pol_return_block(o2_t *a, uint64_t s, uint32_t j, uint32_t t);
void pol_block_freed(o2_t *a, uint32_t gid, uint32_t count);
uint64_t pol_claim_multiple(o2_t *a, uint64_t k);
void pol_free(o2_t *a, uint64_t off);
uint64_t pol_malloc(o2_t *a, uint64_t size, uint64_t key);
void pol_drain(o2_t *a);

/* O2-R (alloc_runs.c) */
uint64_t runs_malloc(o2_t *a, uint64_t size, uint64_t key);
void runs_drain(o2_t *a);
uint32_t runs_first_run(const o2_t *a, uint32_t c);
void runs_prefill(o2_t *a);

#endif
