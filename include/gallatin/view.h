/*
 * gallatin/view.h -- the device view: where every piece of allocator state
 * lives in HBM.  A plain C struct, passed by value to the bulk kernels and
 * copied into __constant__ memory by the device-header binding.
 *
 * Layout (P = PAPER.md line):
 *   heap        nseg x 16 MiB, base aligned to 16 MiB
 *   seg_tree    W words: 64-ary bitmap levels, level 0 first, bit = free
 *   block_trees 9 x W words (tree t at t*W): bit s = segment s formatted for
 *               tree t with blocks available
 *   seg_word    nseg x u64 {tree id:32 | available blocks + 2^31:32}: the
 *               memory table's ids fused with the ring's
 *               reservation count
 *   seg_tid     nseg x u32: a copy of each table word's tree id, written only
 *               when a segment changes owner, so frees can read it through L1
 *   q_head/tail nseg x u32 ring counters; q_entries nseg x 256 x u16 block ids
 *               (the per-segment ring queue)
 *   block_free  nseg x 256 x u32 free counters
 *   slots       S x 128 B lines: word 0 = {issued count:32 | run length:10 |
 *               first block:22} (block buffer; a run = consecutive
 *               blocks, first block as a linear index in units of the class's
 *               block size), word 1 = the prefetched next run (same layout),
 *               word 2 = 1 if the slot's last refill found no memory
 *   fmt_token   9 x 128 B lines: one formatter per block tree
 *   err         u64 error counter (bad frees)
 *   oom         one 128 B line: word 0 = {epoch:32 | searchers:22 | flag:10}
 *               (the exhaustion record, DESIGN.md Deviations 11), word 1 + t =
 *               epoch + 1 at which block tree t was confirmed exhausted
 *   bigq        the whole-block and segment requests a bulk malloc launch
 *               defers to its batch kernel (k_big): bigq_cap x {&ptrs[i],
 *               size}; bigq_ctl = {owner tag, count} (one line)
 */
#ifndef GALLATIN_VIEW_H_
#define GALLATIN_VIEW_H_
#include <stdint.h>

#define GALLATIN_NUM_TREES 9
#define GALLATIN_MAX_LEVELS 8

struct gallatin_device_view {
    uint64_t heap;              /* device address of segment 0                */
    uint64_t nseg;
    uint64_t *seg_tree;
    uint64_t *block_trees;
    uint64_t *seg_word;
    uint32_t *seg_tid;          /* tree id of each segment (read-mostly copy) */
    uint32_t *q_head;
    uint32_t *q_tail;
    uint16_t *q_entries;
    uint32_t *block_free;
    uint64_t *slots;            /* 16 words (128 B) per slot                  */
    uint32_t *fmt_token;        /* 32 words (128 B) per tree                  */
    unsigned long long *err;
    uint64_t *oom;              /* exhaustion record (1 line)                  */
    uint64_t *bigq;             /* bulk launches' deferred whole-block / segment requests:
                                   bigq_cap pairs {&ptrs[i], size} (DESIGN.md Deviations 20) */
    uint32_t *bigq_ctl;         /* one 128 B line: [0] owner launch tag (0 = free), [1] entries */
    uint32_t tree_levels;       /* L                                           */
    uint32_t tree_words;        /* W                                           */
    uint32_t level_off[GALLATIN_MAX_LEVELS];
    uint32_t nslot[GALLATIN_NUM_TREES];
    uint32_t slot_off[GALLATIN_NUM_TREES];
    float nslot_rcp[GALLATIN_NUM_TREES];  /* 1 / nslot (bulk demand estimates) */
    uint32_t nslot_total;
    uint32_t run_cap[GALLATIN_NUM_TREES];  /* max blocks per slot run, per class */
    uint32_t format_ahead;      /* 1 = format the next segment at nb/4 left   */
    uint32_t fence_free;        /* 1 = release fence per freeing team, 2 = none */
    uint32_t formatters;        /* concurrent segment formatters per tree      */
    uint32_t run_init;          /* run length of an empty slot's first refill  */
    uint32_t prefetch;          /* 1 = fetch the next run at the run's middle  */
    uint32_t run_grow;          /* log2 of the run growth factor per refill    */
    uint32_t demand_hint;       /* 1 = bulk refills sized to the launch's demand */
    uint32_t oom_record;        /* 1 = exhaustion record on (DESIGN.md Deviations 11) */
    uint32_t nsm;               /* SMs of the device (slot keys are %smid mod nslot) */
    uint32_t bigq_cap;
    /* prefilled block buffer ("always populated"; reading A-19):
     * 0 segments = reset leaves every slot empty; else class c's slots hold
     * runs of pf_run[c] blocks laid out from segment pf_base[c] on, slot q at
     * linear block pf_base[c] * nb(c) + q * pf_run[c]; pf_last[c] is the class's
     * partly used last segment (0xFFFFFFFF: none), pf_used[c] its blocks in runs */
    uint32_t pf_segs;
    uint32_t pf_base[GALLATIN_NUM_TREES];
    uint32_t pf_run[GALLATIN_NUM_TREES];
    uint32_t pf_last[GALLATIN_NUM_TREES];
    uint32_t pf_used[GALLATIN_NUM_TREES];
};
typedef struct gallatin_device_view gallatin_device_view_t;

#endif
