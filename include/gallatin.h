/*
 * gallatin.h -- C-ABI of libgallatin.so, the B200 (sm_100a) Gallatin hot path.
 *
 * Source of the operations: "Gallatin: A General-Purpose GPU Memory Manager",
 * McCoy & Pandey, PPoPP'24 (PAPER.md; P:n = line n).  The paper gives "a
 * standard malloc/free interface" over one cudaMalloc'd heap,
 * excluded-from-timing construction, a reset between runs,
 * nullptr on exhaustion and a concurrent vEB tree with
 * insert / delete / successor / predecessor / query.
 *
 * Conventions (every entry point):
 *   - Return value: GALLATIN_OK (0) or a negative GALLATIN_ERR_* code.  Device
 *     pointer arguments are not dereferenced on the host; bad device pointers
 *     surface as GALLATIN_ERR_CUDA from a later call (asynchronous errors).
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  Bulk calls are asynchronous on it and return after the launch.
 *   - "d_" arrays are caller-owned DEVICE memory, "h_" arrays caller-owned
 *     HOST memory (pinned or pageable).  Sizes are element counts.
 *   - The library owns the heap and all metadata.  A pointer returned by the
 *     allocator is owned by the caller until it is freed.
 *   - One allocator per process (the paper's global variant), on the
 *     device current at gallatin_init.  Host calls are thread-compatible, not
 *     thread-safe.  Device calls (bulk kernels, device header) are fully
 *     concurrent with each other.
 */
#ifndef GALLATIN_H_
#define GALLATIN_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
    GALLATIN_OK = 0,
    GALLATIN_ERR_INVALID = -1,   /* bad argument (size, count, universe, NULL)       */
    GALLATIN_ERR_CUDA = -2,      /* a CUDA runtime call or kernel launch failed       */
    GALLATIN_ERR_STATE = -3,     /* not initialized / already initialized             */
    GALLATIN_ERR_NOMEM = -4      /* cudaMalloc of heap/metadata failed (init only)    */
};

/* ------------------------------------------------------------ allocator --- */

/* Tuning knobs (all optional: zero selects the default).
 *   heap_bytes : rounded DOWN to a multiple of 16 MiB, >= 1 segment.
 *   slot_base  : block-buffer slots of the 16 B class; class c gets
 *                max(slot_min, slot_base >> c).  Default = #SMs (148).
 *   slot_min   : lower cap; the paper caps at four; default
 *                clamp(nseg / 32, 4, 32) (more slots for the big classes on big heaps).
 *   run_max    : a slot holds a RUN of up to run_max consecutive blocks (1..512,
 *                default 256); the run starts at run_init blocks and grows
 *                2^run_grow-fold on every refill of the slot.  1 = the paper's
 *                one-block buffer.  Before a run request reports "no memory",
 *                every slot gives back the blocks of its run no request has
 *                drawn from, and the request is retried once.
 *   run_bytes  : and at most run_bytes per run (default min(256 MiB, heap/64)).
 *   format_ahead: 1 (default) = the reservation that leaves a segment with
 *                fewer than nb/4 blocks formats the next segment of its tree;
 *                2 = off (the paper: format on demand).
 *   fence_free : 1 (default) = a release fence per freeing team before its
 *                free-counter atomic; 2 = none
 *                (measurement only: frees then do not order user data).
 * (run_max = 1, format_ahead = 2 reproduce the paper's policy exactly; the
 *  run/format-ahead policy is DESIGN.md "Deviations" 5.) */
typedef struct gallatin_config {
    uint64_t heap_bytes;
    uint64_t run_bytes;
    uint32_t slot_base;
    uint32_t slot_min;
    uint32_t run_max;
    uint32_t format_ahead;
    uint32_t fence_free;
    uint32_t bulk_items;   /* bulk kernels: 0 = auto (4 from 606,208 requests on, else 1); 1 = one request per
                              thread and one slot RMW per warp team (k_bulk_malloc<1> / k_bulk_free<1>); 4 = four
                              per thread (eight in the malloc), one slot RMW per class per 1024-request CTA tile (k_bulk_malloc_cta) and
                              the warp-team free with 32-bit block ids (k_bulk_free_w) */
    uint32_t run_init;     /* first run of an empty slot of class c: min(max(run_init >> c, min(run_init, 8)), 256 >> c) blocks (default: the largest power of two <= 256 whose first runs over all slots fit in half the heap) */
    uint32_t prefetch;     /* 1 = fetch the next run at the middle of the current one; 0/2 = off (default) */
    uint32_t run_grow;     /* a refilled run is 2^run_grow times the last one, up to the cap: 1..8 (default 3) */
    uint32_t demand_hint;  /* bulk malloc: 0/1 = a refill takes at least the blocks this slot's share of the launch
                              needs (the CTA's per-class count x CTAs / slots; DESIGN.md Deviations 10), up to the
                              run cap (default); 2 = off (runs grow 2^run_grow-fold per refill only) */
    uint32_t oom_record;   /* 0/1 = exhaustion record on (default; DESIGN.md Deviations 11): a run request of a
                              block tree confirmed exhausted fails in O(1) until memory comes back; 2 = off (every
                              request repeats the full search with slot trims -- the policy oracle/alloc_runs.c
                              replays exactly) */
    uint32_t prefill;      /* 0/1 = prefilled block buffer (default; "each block buffer is always
                              populated"): gallatin_init / gallatin_reset leave every slot holding its first run,
                              laid out class by class from segment 0 (slot q of class c: blocks
                              [q*r, (q+1)*r) of the class's segments, r = its first-run length; the class's partly
                              used last segment keeps its other blocks in its ring and block tree) -- when those
                              runs fit in half the heap, else the slots start empty and fill on first use (reading
                              A-19); 2 = off.  gallatin_drain empties the slots (the pristine image). */
} gallatin_config_t;

int gallatin_init(uint64_t heap_bytes);                 /* defaults for the rest */
int gallatin_init_ex(const gallatin_config_t *cfg);
int gallatin_destroy(void);                             /* frees heap + metadata; every
                                                           outstanding pointer dies   */
int gallatin_is_initialized(void);                      /* 1 / 0 */

/* Bulk malloc (Alg. 3 -> 2 -> 1): d_ptrs[i] = malloc(d_sizes[i]) by
 * one GPU thread per request.  Size 0 and exhaustion give NULL.  Sizes
 * <= 4096 B are slices (16 B .. 4 KB powers of two); (4 KB, 16 MB)
 * whole blocks; >= 16 MB whole contiguous segments.
 * From 606,208 requests on the call is two kernels on `stream`: the bulk
 * kernel, and a one-CTA batch kernel that serves the launch's whole-block and
 * segment requests together (DESIGN.md Deviations 21; a launch running
 * concurrently with another one's batch serves its own inline).  Every
 * d_ptrs[i] is written when the stream reaches the end of the call. */
int gallatin_malloc(const uint64_t *d_sizes, void **d_ptrs, uint64_t n, void *stream);

/* Bulk free (Alg. 4).  NULL entries are ignored.  A pointer outside
 * the heap or into an unallocated segment increments the device error counter
 * (gallatin_stats); other foreign, interior or double frees are undefined. */
int gallatin_free(void *const *d_ptrs, uint64_t n, void *stream);

/* Same two calls with HOST arrays: copies the inputs to the device, runs the
 * kernel on `stream`, copies the results back and synchronizes the stream. */
int gallatin_malloc_host(const uint64_t *h_sizes, uint64_t *h_ptrs, uint64_t n, void *stream);
int gallatin_free_host(const uint64_t *h_ptrs, uint64_t n, void *stream);

/* The initial state (the paper resets before every run): the pristine
 * image, or with the prefill knob every slot holding its first run.
 * Invalidates every outstanding pointer.  Asynchronous on `stream`. */
int gallatin_reset(void *stream);

/* Quiescent only (no malloc/free in flight): retire every block-buffer slot
 * (sequentially, class-major slot order) -- the unissued remainder of every
 * block of its run is freed -- then return every formatted segment whose
 * blocks are all home to the segment tree.  After every user pointer is freed,
 * drain restores the pristine image. */
int gallatin_drain(void *stream);

/* Serialized replay (test hook, one GPU thread, in order): kinds[i] 0 =
 * malloc(args[i]) with block-buffer slot key keys[i] (instead of %smid); 1 =
 * free(result of op args[i]); 2 = drain.  d_out[i] = pointer OFFSET from the
 * heap base for mallocs (UINT64_MAX = NULL), 0 otherwise. */
int gallatin_replay(const uint8_t *d_kinds, const uint64_t *d_args, const uint64_t *d_keys,
                    uint64_t n, uint64_t *d_out, void *stream);

typedef struct gallatin_stats {
    uint64_t heap_base;          /* device address of segment 0 (16 MiB aligned)   */
    uint64_t heap_bytes;
    uint64_t num_segments;
    uint64_t free_segments;      /* bits set in the segment tree                    */
    uint64_t tree_segments[9];   /* segments formatted for each block tree          */
    uint64_t large_segments;     /* segments held by >= 16 MB allocations           */
    uint64_t errors;             /* device error counter (bad frees)                */
    uint64_t run_bytes;          /* effective configuration ...                     */
    uint32_t nslot[9];           /* block-buffer slots per class                    */
    uint32_t run_cap[9];         /* max blocks per run per class                    */
    uint32_t slot_base, slot_min, run_max, format_ahead, fence_free, run_init, formatters, prefetch;
    uint32_t run_grow, demand_hint, oom_record;
    uint32_t prefill_segments;   /* segments a reset carves into prefilled slot runs (0 = none) */
} gallatin_stats_t;
int gallatin_stats(gallatin_stats_t *out);               /* synchronizes the device */

/* Snapshot image (synchronizes the device).  A flat array of uint64 words:
 *   [0] magic 0x47414C4C494D4731  [1] nseg  [2] tree levels L  [3] W = words
 *   per tree  [4] S = total slots  [5] error counter  [6] number of segments
 *   whose read-mostly tree-id copy disagrees with the table (always 0)  [7] 0
 *   then: segment tree (W words: level 0 first; bit = segment free)
 *         9 block trees (9*W; bit s of tree t = segment s formatted for t
 *           with blocks available)
 *         memory table (nseg words: tree id << 32 | (uint32) available blocks;
 *           tree id 0..8 block tree, 9+k first of k segments, 0xFFFFFFFE
 *           continuation, 0xFFFFFFFF free)
 *         ring queues (nseg x 65 words: [count] then 256 uint16 block ids in
 *           FIFO order, 0xFFFF padded, 4 per word little-endian)
 *         block free counters (nseg*256 uint32, 2 per word)
 *         block-buffer slots (S words, class-major: issued count << 32 |
 *           run length << 22 | first block of the run as a linear index in
 *           units of the class's block size; empty = 0x00000000003FFFFF)
 *         prefetched next run per slot (S words, same layout, count 0)
 * gallatin_snapshot_words() gives the length. */
int gallatin_snapshot_words(uint64_t *words);
int gallatin_snapshot(uint64_t *h_out, uint64_t cap_words, uint64_t *len_words);

/* Device view for the header-only device API (include/gallatin/device.cuh). */
struct gallatin_device_view;
int gallatin_get_device_view(struct gallatin_device_view *out, uint64_t out_bytes);
uint64_t gallatin_device_view_bytes(void);

/* Test harness kernels (not timed by the paper; "checks the correctness
 * of allocated memory"):
 *   stamp  : every request i writes the uint32 value i over ceil(size/4) words.
 *   verify : separate launch, L1-bypassing loads; adds the number of words not
 *            equal to i to *d_bad (uint64).
 *   usable : for every non-NULL pointer, the usable size read from the memory
 *            table (slice 16<<t, block 64K<<t, or k segments); adds the sum to
 *            *d_sum and the count of pointers whose table entry contradicts
 *            their request (wrong class, not aligned, outside the heap) to
 *            *d_bad. d_usable (nullable) receives the per-pointer value. */
int gallatin_stamp(void *const *d_ptrs, const uint64_t *d_sizes, uint64_t n, void *stream);
int gallatin_verify(void *const *d_ptrs, const uint64_t *d_sizes, uint64_t n,
                    uint64_t *d_bad, void *stream);
int gallatin_usable(void *const *d_ptrs, const uint64_t *d_sizes, uint64_t n,
                    uint64_t *d_usable, uint64_t *d_sum, uint64_t *d_bad, void *stream);

/* ------------------------------------------------------ standalone vEB --- */
/* The paper's GPU vEB tree: 64-bit bitmap nodes, no min/max, a
 * fixed height ceil(log64 u); a concurrent set over [0, 2^universe_log2).
 * Every node operation is one 64-bit atomic.  Keys >= 2^universe_log2 are
 * ignored by insert/delete (out 0) and have no successor (UINT64_MAX). */
typedef struct veb veb_t;
int veb_create(uint32_t universe_log2 /* 1..32 */, veb_t **out);
int veb_destroy(veb_t *h);
int veb_clear(veb_t *h, void *stream);
/* d_out[i] = 1 iff key i was newly added / was present (exactly one of several
 * equal keys in a batch reports 1).  d_out may be NULL. */
int veb_insert(veb_t *h, const uint64_t *d_keys, uint8_t *d_out, uint64_t n, void *stream);
int veb_delete(veb_t *h, const uint64_t *d_keys, uint8_t *d_out, uint64_t n, void *stream);
int veb_member(veb_t *h, const uint64_t *d_keys, uint8_t *d_out, uint64_t n, void *stream);
/* succ(x) = min{y in S, y >= x}; pred(x) = max{y in S, y <= x};
 * UINT64_MAX when none.  By default query batches (member / successor /
 * predecessor) read the tree through the read-only path: no insert/delete may
 * run on the same tree concurrently (different streams) with a query batch. */
int veb_successor(veb_t *h, const uint64_t *d_q, uint64_t *d_out, uint64_t n, void *stream);
int veb_predecessor(veb_t *h, const uint64_t *d_q, uint64_t *d_out, uint64_t n, void *stream);
/* on = 1: later query batches read the tree with coherent loads
 * (ld.relaxed.gpu) and MAY overlap insert/delete batches on other streams
 * (SURVEY 8(f)3 concurrent mixed batches).  A query then sees each key that
 * stays present throughout it, and reports only keys present at some moment
 * during it (bt_successor restarts past a summary bit whose child emptied).
 * on = 0 (default) = the read-only path, quiescent trees only.  Host-side
 * flag: takes effect for batches launched after the call. */
int veb_set_concurrent(veb_t *h, int on);
/* Image (all levels, level 0 first; bit = element / child non-empty); syncs. */
int veb_words(const veb_t *h, uint64_t *words);
int veb_snapshot(const veb_t *h, uint64_t *h_out, uint64_t cap_words, uint64_t *len_words);

/* ------------------------------------------------------ measurement ----- */
/* Peak probes (DESIGN.md 5 "Roofline"): persistent
 * microkernels over all SMs (148 x 8 CTAs x 256 threads) looping over about
 * `n` operations; each returns the time of one launch in *ms (CUDA events on
 * `stream`, after an untimed warm-up launch) and the operations it performed
 * in *ops.  `param` per kind: */
enum {
    GALLATIN_PROBE_ATOM_U64_RANDOM = 1,    /* PK1 atom.add.u64 with return, random over param words        */
    GALLATIN_PROBE_ATOM_HOT = 2,           /* PK2 atom.add.u64 with return by one lane per warp on param
                                              128 B lines chosen by %smid (the block-buffer pattern)    */
    GALLATIN_PROBE_RED_HOT = 3,            /* PK3 as 2 with red.add (no return)                             */
    GALLATIN_PROBE_BUMP_WARP = 4,          /* PK5a one team atomicAdd per warp + 16 B I/O per request, n
                                              requests, param lines (RegEff-AW analogue)         */
    GALLATIN_PROBE_FENCE_ACQ_REL = 5,      /* PK7 fence.acq_rel.gpu per warp (ops = fences)                 */
    GALLATIN_PROBE_HBM_COPY = 6,           /* PK6 HBM copy of param bytes (ops = bytes read + written)      */
    GALLATIN_PROBE_ATOM_U32_RANDOM = 7,    /* PK1 atom.add.u32, random over param words                     */
    GALLATIN_PROBE_ATOM_U64_COALESCED = 8, /* PK1 atom.add.u64, thread-consecutive words                    */
    GALLATIN_PROBE_ATOM_U32_COALESCED = 9, /* PK1 atom.add.u32, thread-consecutive words                    */
    GALLATIN_PROBE_CAS_HOT = 10,           /* PK4 atom.cas on param hot lines (every CAS counted)           */
    GALLATIN_PROBE_BUMP_CTA = 11,          /* PK5b the bulk CTA kernel's structure without the allocator:
                                              one RMW per class per 512-request tile, 16 B I/O per
                                              request; n requests of 16 B, param slot lines           */
    GALLATIN_PROBE_FENCE_SC = 12,          /* PK7 fence.sc.gpu per warp                                     */
    GALLATIN_PROBE_LOAD_RANDOM = 13        /* PK6 random 8 B loads over param words (L2-resident at 16 MB,
                                              HBM random sectors beyond L2)                             */
};
int gallatin_probe(int kind, uint64_t n, uint64_t param, double *ms, double *ops, void *stream);

const char *gallatin_version(void);
const char *gallatin_error_string(int code);

#ifdef __cplusplus
}
#endif
#endif /* GALLATIN_H_ */
