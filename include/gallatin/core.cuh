// gallatin/core.cuh -- the allocator's device code (one copy, used by the bulk
// kernels of libgallatin.so and by user kernels through gallatin/device.cuh).
//
// PAPER.md (P = line): segments of 16 MB in a segment tree (S4.1, P:132-143,
// Alg. 1), blocks of 4096 slices in per-size block trees (S4.2, P:170-180,
// Alg. 2), slices handed out by a counter from a per-SM block buffer with
// warp coalescing (S4.3, Alg. 3), frees through per-block counters
// and segment re-insertion (S5, Alg. 4).  Differences from the
// paper's own GPU design are listed in DESIGN.md ("Deviations") and marked
// [dev] here.
#pragma once
#include <stdint.h>

#include "gallatin/bittree.cuh"
#include "gallatin/ptx.cuh"
#include "gallatin/view.h"

namespace gallatin {
namespace core {

using View = gallatin_device_view;

constexpr uint32_t kSegLog2 = 24;                   // 16 MB segments
constexpr uint64_t kSegBytes = 1ull << kSegLog2;
constexpr uint32_t kSlices = 4096;                  // slices per block
constexpr uint32_t kSliceLog2 = 12;
constexpr uint32_t kMinSliceLog2 = 4;               // 16 B
constexpr uint64_t kMaxSlice = 4096;                // 4096 B
constexpr uint32_t kTrees = GALLATIN_NUM_TREES;     // block trees 64 KB..16 MB
constexpr uint32_t kMaxBlocks = 256;                // blocks per segment
constexpr uint32_t kTreeFree = 0xFFFFFFFFu;
constexpr uint32_t kTreeCont = 0xFFFFFFFEu;
constexpr uint32_t kGidNone = 0xFFFFFFFFu;
constexpr uint32_t kAvailBias = 0x80000000u;
constexpr uint16_t kRingEmpty = 0xFFFF;
constexpr uint32_t kMaxRun = 512;                   // blocks per slot run (10-bit field)
constexpr uint32_t kRunShift = 22;                  // slot word: issued:32 | run:10 | first:22

__device__ __forceinline__ uint32_t nb_of(uint32_t t) { return kMaxBlocks >> t; }

// ---- memory-table word {tree id : 32 | available blocks + 2^31 : 32} --------
// [dev] The paper keeps the tree id and the ring queue separately and
// re-checks the id with ldcv after taking a block (Alg.2).  Packing
// the id with the ring's reservation count lets one fetch-add reserve a block
// and validate the id at once; every update of the word is a fetch-add (or
// the one CAS that retires a full segment), so concurrent updates commute.
__device__ __forceinline__ uint32_t sw_tree(uint64_t w) { return (uint32_t)(w >> 32); }
__device__ __forceinline__ int32_t sw_avail(uint64_t w) { return (int32_t)((uint32_t)w - kAvailBias); }
__device__ __forceinline__ uint64_t sw_make(uint32_t tree, int32_t avail) {
    return ((uint64_t)tree << 32) | (uint32_t)((uint32_t)avail + kAvailBias);
}
__device__ __forceinline__ uint64_t sw_retree(uint32_t from, uint32_t to) {
    return (uint64_t)(uint32_t)(to - from) << 32;
}
// block tree t holds segment s  <=>  s is formatted for t and has a block
__device__ __forceinline__ bool sw_in_tree(uint64_t w, uint32_t t) { return sw_tree(w) == t && sw_avail(w) > 0; }

__device__ __forceinline__ BitTree seg_tree(const View &v) {
    BitTree b;
    b.w = v.seg_tree;
    b.nbits = v.nseg;
    b.levels = v.tree_levels;
#pragma unroll
    for (int i = 0; i < kMaxLevels; i++) b.off[i] = v.level_off[i];
    return b;
}
__device__ __forceinline__ BitTree block_tree(const View &v, uint32_t t) {
    BitTree b = seg_tree(v);
    b.w = v.block_trees + (uint64_t)t * v.tree_words;
    return b;
}

// Make block-tree t's bit for segment s equal its predicate (the derived-bit
// reconcile loop of DESIGN.md "Quiescent exactness").
__device__ inline __noinline__ void btree_reconcile(const View &v, uint32_t t, uint64_t s) {
    const BitTree bt = block_tree(v, t);
    uint64_t *leaf = bt.w + bt.off[0] + (s >> 6);
    const uint64_t bit = 1ull << (s & 63);
    bool flipped = false;
    ptx::fence_acq_rel();
    for (;;) {
        const bool in = sw_in_tree(ptx::ld_relaxed(v.seg_word + s), t);
        const uint64_t old = in ? ptx::atom_or(leaf, bit) : ptx::atom_and(leaf, ~bit);
        flipped |= in ? (old == 0) : (old == bit);
        ptx::fence_acq_rel();
        if (sw_in_tree(ptx::ld_relaxed(v.seg_word + s), t) == in) break;
    }
    if (flipped) bt_reconcile_up(bt, 0, s >> 6);
}

__device__ inline __noinline__ bool try_free_segment(const View &v, uint64_t s, uint32_t t);

// ---- exhaustion record [dev] (DESIGN.md Deviations 11) ----------------------
// Without it every request that finds the heap exhausted repeats the whole
// confirmation (slot trims, table scans) before reporting NULL: a bulk call
// asking 2x the heap took minutes.  A request whose run search for tree t
// failed announces itself (searchers + 1), repeats the search to the end and,
// if that fails too, records "tree t exhausted in epoch e" -- unless an epoch
// bump happened meanwhile.  Every RMW that makes blocks or segments available
// (block return, segment free, format, give-backs of reservations and claim
// windows) is followed by oom_notify: a fence.sc, then -- only if a search is
// in flight or a record exists -- one epoch bump.  The fence pair (the
// searcher's after its announce, the notifier's after its RMW) forbids the
// store-buffer outcome in which neither sees the other, so a record is never
// left standing for memory that became available after the search began.
// Later requests of tree t fail in O(1) while the record's epoch is current.
constexpr uint64_t kOomFlagMask = 0x3FFull;               // bits 0..9: tree t recorded this epoch
constexpr uint64_t kOomOne = 1ull << 10;                  // searchers: bits 10..31
constexpr uint64_t kOomEpoch = 1ull << 32;

__device__ __forceinline__ bool oom_match(uint64_t r, uint64_t rec, uint32_t t) {
    return (r & (1ull << t)) && rec == (r >> 32) + 1;
}
__device__ __forceinline__ bool oom_known(const View &v, uint32_t t) {
    return oom_match(ptx::ld_relaxed(v.oom), ptx::ld_relaxed(v.oom + 1 + t), t);
}
constexpr uint32_t kOomFast = 0xFFFFFFFFu;                // *first of a run request failed by the record

__device__ inline __noinline__ void oom_notify_slow(const View &v, uint64_t w) {
    while (w & 0xFFFFFFFFull) {                              // a search in flight or a record
        const uint64_t o = ptx::atom_cas(v.oom, w, (w + kOomEpoch) & ~kOomFlagMask);
        if (o == w || (o >> 32) != (w >> 32)) return;         // bumped (by us or after our fence)
        w = o;
    }
}
__device__ __forceinline__ void oom_notify(const View &v) {
    ptx::fence_sc();
    const uint64_t w = ptx::ld_relaxed(v.oom);
    if (w & 0xFFFFFFFFull) oom_notify_slow(v, w);
}

// announce a confirming search
__device__ __forceinline__ void oom_enter(const View &v) {
    ptx::atom_add(v.oom, kOomOne);
    ptx::fence_sc();
}
// the epoch a search step starts in (acquire: it sees every RMW whose notify
// bumped the epoch up to this value)
__device__ __forceinline__ uint64_t oom_epoch(const View &v) {
    const uint64_t e = ptx::ld_relaxed(v.oom) >> 32;
    ptx::fence_acq_rel();
    return e;
}
// the search of tree t in epoch e failed: record it unless the epoch moved;
// then leave the searchers
__device__ inline __noinline__ void oom_leave(const View &v, uint32_t t, uint64_t e, bool failed) {
    if (failed) {
        uint64_t w = ptx::ld_relaxed(v.oom);
        while ((w >> 32) == e && !(w & (1ull << t))) {
            const uint64_t o = ptx::atom_cas(v.oom, w, w | (1ull << t));
            if (o == w) { w |= 1ull << t; break; }
            w = o;
        }
        if ((w >> 32) == e) ptx::st_relaxed(v.oom + 1 + t, e + 1);
    }
    ptx::atom_add(v.oom, (uint64_t)(-(int64_t)kOomOne));
}

// Every thread whose RMW on seg_word[s] changed a block-tree predicate repairs
// that bit; the RMW that brings a segment back to "all blocks home" retires it
// -- first: if its retiring CAS succeeds no RMW came between, and the retire
// reconciles the bit itself (one reconcile instead of two on the free path's
// tail).  Returns whether the segment was retired.
__device__ __forceinline__ bool seg_after_rmw(const View &v, uint64_t s, uint64_t old, uint64_t now) {
    const uint32_t to = sw_tree(old), tn = sw_tree(now);
    if (tn < kTrees && tn == to && sw_avail(now) == (int32_t)nb_of(tn) && sw_avail(old) < sw_avail(now) &&
        try_free_segment(v, s, tn))
        return true;
    if (to < kTrees && sw_in_tree(old, to) != sw_in_tree(now, to)) btree_reconcile(v, to, s);
    if (tn < kTrees && tn != to && sw_in_tree(old, tn) != sw_in_tree(now, tn)) btree_reconcile(v, tn, s);
    return false;
}

// "When all blocks are returned, the segment is freed and re-added to the
// segment tree".
__device__ inline __noinline__ bool try_free_segment(const View &v, uint64_t s, uint32_t t) {
    const uint64_t full = sw_make(t, (int32_t)nb_of(t));
    if (ptx::atom_cas(v.seg_word + s, full, sw_make(kTreeFree, 0)) != full) return false;
    ptx::st_relaxed(v.seg_tid + s, kTreeFree);
    // No block of s is out or in flight: reset its ring.
    ptx::st_relaxed(v.q_head + s, 0u);
    ptx::st_relaxed(v.q_tail + s, 0u);
    uint4 *e = reinterpret_cast<uint4 *>(v.q_entries + s * kMaxBlocks);
#pragma unroll 4
    for (int i = 0; i < (int)(kMaxBlocks * sizeof(uint16_t) / sizeof(uint4)); i++)
        e[i] = make_uint4(0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu);
    ptx::fence_acq_rel();
    btree_reconcile(v, t, s);
    bt_insert(seg_tree(v), s);
    oom_notify(v);
    return true;
}

// Every formatted segment whose blocks are all home goes back to the segment
// tree (formatted ahead and never used); returns how many.
__device__ inline __noinline__ uint32_t reclaim_idle(const View &v) {
    uint32_t n = 0;
    for (uint64_t s = 0; s < v.nseg; s++) {
        const uint64_t w = ptx::ld_relaxed(v.seg_word + s);
        const uint32_t t = sw_tree(w);
        if (t < kTrees && sw_avail(w) == (int32_t)nb_of(t)) {
            try_free_segment(v, s, t);
            n++;
        }
    }
    return n;
}

// [dev] A claimer that lost the race for a bit of leaf word `old` retries at a
// pseudo-random bit among the free bits its failed RMW returned (seeded by the
// thread and the attempt) instead of the next one up: k simultaneous claimers
// -- every slot refilling at a launch's start -- then collide O(1) times each
// instead of walking the word one loss at a time, and they stay in the lowest
// word with free segments (front-first packing).  kNone if the word
// had no free bit.
__device__ __forceinline__ uint64_t claim_retry_hint(uint64_t wi, uint64_t old, uint32_t attempt) {
    if (old == 0) return kNone;
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t h = (tid * 0x9E3779B1u) ^ (attempt * 0x85EBCA6Bu);
    h ^= h >> 15;
    uint32_t r = h % (uint32_t)__popcll((long long)old);
    uint64_t m = old;
    for (; r; r--) m &= m - 1;                                // drop r lowest free bits
    return (wi << 6) + (uint64_t)(__ffsll((long long)m) - 1);
}

// ---- Alg. 1 GetSegment(treeId < numBlockTrees) ----------------
// [dev] A claimer that has already lost a race (attempt > 0) and moves on to
// the next word does not aim at its lowest free bit -- every other loser
// aims there too, and a launch's first burst of refills (one per slot, all
// at once) then takes one segment per round -- but at a pseudo-random bit at
// or above it in that word; the RMW tells whether it was free.
// A window claim of kmax segments aims at a window boundary (kmax rounded up
// to a power of two, at most a word), so concurrent windows do not overlap.
__device__ __forceinline__ uint32_t claim_align(uint32_t kmax) {
    return kmax >= 64 ? 64u : (kmax <= 1 ? 1u : 1u << (32 - __clz(kmax - 1)));
}
__device__ __forceinline__ uint64_t claim_spread(uint64_t s, uint32_t attempt, uint32_t kmax = 1) {
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t h = (tid * 0x27D4EB2Fu) ^ (attempt * 0x165667B1u);
    h ^= h >> 15;
    const uint32_t lo = (uint32_t)(s & 63);
    uint32_t b = (lo + h % (64u - lo)) & ~(claim_align(kmax) - 1);
    if (b < lo) b = lo;
    return (s & ~63ull) | b;
}

// [dev] RUN claims only (claim_front_run: a slot's run of whole segments, a
// deviation of ours): the FIRST loss means every concurrent claimer aimed at
// the same lowest free window (a launch's burst of refills); the loser then
// aims at a pseudo-random window boundary of the next kSpreadWords + kmax/2
// leaf words -- the RMW tells whether it was free -- instead of queueing on
// one word.  The paper's GetSegment (claim_front: formats) stays in the
// lowest word with free segments (claim_retry_hint).  Serially no claim
// loses.
constexpr uint32_t kSpreadWords = 4;
__device__ __forceinline__ uint64_t claim_first_loss(const View &v, uint64_t wi, uint32_t kmax = 1) {
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    uint32_t h = tid * 0x9E3779B1u;
    h ^= h >> 13;
    h *= 0x85EBCA6Bu;
    h ^= h >> 16;
    const uint32_t words = kSpreadWords + kmax / 2;            // room for the windows of every claimer
    const uint64_t s = ((wi + h % words) << 6) | (((h >> 8) & 63) & ~(claim_align(kmax) - 1));
    return s < v.nseg ? s : v.nseg - 1;
}

// successor(0) on the segment tree + claimIndex, front first
// (P:138).  Returns the claimed segment or kNone when every segment is in use.
// A claimer that loses the race retries elsewhere (claim_retry_hint,
// claim_spread; serially the first attempt always wins, so this is
// successor(0)).
__device__ inline __noinline__ uint64_t claim_front(const View &v) {
    const BitTree st = seg_tree(v);
    uint64_t from = 0, hint = kNone;
    uint32_t attempt = 0;
    for (;;) {
        uint64_t s = hint != kNone ? hint : bt_successor<false>(st, from);
        if (hint == kNone && attempt > 0 && s != kNone) {
            s = claim_spread(s, attempt);
            if (s >= v.nseg) s = v.nseg - 1;
        }
        hint = kNone;
        if (s == kNone) {
            if (from != 0) { from = 0; continue; }
            s = bt_scan_first(st);                         // confirm before failing
            if (s == kNone) {
                // [dev] before failing, return idle formatted segments (all blocks home)
                if (!reclaim_idle(v)) return kNone;            // "All segments in use"
                continue;
            }
        }
        uint64_t *leaf = st.w + st.off[0] + (s >> 6);
        const uint64_t bit = 1ull << (s & 63);
        const uint64_t old = ptx::atom_and(leaf, ~bit);
        if (old & bit) {
            if (old == bit) bt_reconcile_up(st, 0, s >> 6);       // the word emptied
            ptx::fence_acq_rel();
            return s;
        }
        hint = claim_retry_hint(s >> 6, old, ++attempt);   // a free bit the lost RMW saw, same word
        from = ((s >> 6) + 1) << 6;
    }
}

// [dev] claim a run of up to kmax consecutive free segments starting at the
// lowest free one, with one atomicAnd on the leaf word: the window
// [s, s+kmax) within that word is taken at once, the consecutive prefix from
// s is kept and the rest given back.  Concurrent claimers then get disjoint
// windows instead of interleaving single segments.  *k = segments claimed
// (serially: s = successor(0) and the free segments that follow it).
__device__ inline __noinline__ uint64_t claim_front_run(const View &v, uint32_t kmax, uint32_t *k) {
    const BitTree st = seg_tree(v);
    uint64_t from = 0, hint = kNone;
    uint32_t attempt = 0;
    for (;;) {
        uint64_t s = hint != kNone ? hint : bt_successor<false>(st, from);
        if (hint == kNone && attempt > 0 && s != kNone) {
            s = claim_spread(s, attempt, kmax);
            if (s >= v.nseg) s = v.nseg - 1;
        }
        hint = kNone;
        if (s == kNone) {
            if (from != 0) { from = 0; continue; }
            s = bt_scan_first(st);
            if (s == kNone) {
                if (!reclaim_idle(v)) return kNone;
                continue;
            }
        }
        const uint64_t wi = s >> 6;
        const uint32_t lo = (uint32_t)(s & 63);
        uint64_t hi = lo + (uint64_t)kmax;
        if (hi > 64) hi = 64;
        if ((wi << 6) + hi > v.nseg) hi = v.nseg - (wi << 6);
        const uint64_t mask = bit_range(lo, (uint32_t)hi);
        uint64_t *leaf = st.w + st.off[0] + wi;
        const uint64_t old = ptx::atom_and(leaf, ~mask);
        const uint64_t got = old & mask;
        const uint64_t inv = ~(got >> lo);                 // 0 only if all 64 bits of a word were taken
        const uint32_t run = inv ? (uint32_t)__ffsll((long long)inv) - 1 : 64u;   // 0 if s was lost
        const uint64_t extra = got & ~bit_range(lo, lo + run);
        bool flip = old != 0 && (old & ~mask) == 0;
        if (extra) flip |= ptx::atom_or(leaf, extra) == 0;
        if (flip) bt_reconcile_up(st, 0, wi);
        if (extra) oom_notify(v);
        if (run == 0) {
            // a free bit the lost RMW saw, at a window boundary if one is free
            // (concurrent windows then do not overlap); a run claim's first
            // loss spreads over the next words (claim_first_loss)
            const uint32_t al = claim_align(kmax);
            const uint64_t fr = old & ~mask, at = fr & (al >= 64 ? 1ull : ~0ull / ((1ull << al) - 1));
            hint = ++attempt == 1 ? claim_first_loss(v, wi, kmax) : claim_retry_hint(wi, at ? at : fr, attempt);
            from = (wi + 1) << 6;
            continue;
        }
        ptx::fence_acq_rel();
        *k = run | (attempt << 16);                        // attempts: traced builds read them
        return s;
    }
}

// initSegment for tree t: blocks [keep, nb) go into the ring in order
// and the segment joins block tree t ("broadcast availability");
// blocks [0, keep) belong to the caller.
__device__ inline __noinline__ void format_segment(const View &v, uint64_t s, uint32_t t, uint32_t keep) {
    const uint32_t nb = nb_of(t);
    uint16_t *e = v.q_entries + s * kMaxBlocks;
    const uint32_t cnt = nb - keep;                       // entries at positions 0 .. cnt-1
    uint64_t *e4 = reinterpret_cast<uint64_t *>(e);
    uint32_t q = 0;
    for (; q + 4 <= cnt; q += 4) {
        const uint64_t j = keep + q;
        e4[q / 4] = j | ((j + 1) << 16) | ((j + 2) << 32) | ((j + 3) << 48);
    }
    for (; q < cnt; q++) e[q] = (uint16_t)(keep + q);
    ptx::st_relaxed(v.q_head + s, 0u);
    ptx::st_relaxed(v.q_tail + s, nb - keep);
    ptx::st_relaxed(v.seg_tid + s, t);
    ptx::fence_acq_rel();
    const uint64_t delta = sw_retree(kTreeFree, t) + (nb - keep);
    const uint64_t old = ptx::atom_add(v.seg_word + s, delta);
    seg_after_rmw(v, s, old, old + delta);
    oom_notify(v);
}

// ---- block return (Alg.4; ring enqueue P:178) --------------------
// [dev] A segment of one block (4 KB slices: 16 MB blocks) whose block comes
// back is home at once: one CAS {t, 0 available} -> FREE retires it without
// the ring enqueue, the table fetch-add and the block-tree repair that the
// general path runs (its block-tree bit was never set: no RMW ever saw it
// with a block available).  The same final state as the general path; a
// failed CAS (a refiller's transient reservation on the word) falls back.
__device__ __forceinline__ bool return_whole_segment(const View &v, uint64_t s, uint32_t t) {
    if (ptx::atom_cas(v.seg_word + s, sw_make(t, 0), sw_make(kTreeFree, 0)) != sw_make(t, 0)) return false;
    ptx::st_relaxed(v.seg_tid + s, kTreeFree);
    ptx::fence_acq_rel();                                    // table + tree-id copy before the tree bit
    bt_insert(seg_tree(v), s);
    oom_notify(v);
    return true;
}

__device__ inline __noinline__ void return_block(const View &v, uint32_t gid) {
    const uint64_t s = gid / kMaxBlocks;
    const uint32_t tid = ptx::ld_relaxed(v.seg_tid + s);
    if (tid == kTrees - 1 && return_whole_segment(v, s, tid)) return;
    const uint32_t pos = atomicAdd(v.q_tail + s, 1u) & (kMaxBlocks - 1);
    uint16_t *slotp = v.q_entries + s * kMaxBlocks + pos;
    ptx::Backoff wb(3, (s << 32) | pos);
    while (ptx::ld_relaxed(slotp) != kRingEmpty) wb.pause();   // previous lap's dequeue in flight
    ptx::st_relaxed(slotp, (uint16_t)(gid % kMaxBlocks));
    ptx::fence_acq_rel();
    const uint64_t old = ptx::atom_add(v.seg_word + s, 1ull);
    const bool retired = seg_after_rmw(v, s, old, old + 1);   // all blocks home: try_free_segment notified
    // a search can newly find the segment only if it had no block available
    if (!retired && sw_avail(old) == 0) oom_notify(v);
}

// n slices of block gid came back; the team completing 4096 returns it
// (reading A-14 of "== 4095").
__device__ __forceinline__ void block_freed(const View &v, uint32_t gid, uint32_t n) {
    const uint32_t old = atomicAdd(v.block_free + gid, n);
    if (old + n == kSlices) {
        atomicExch(v.block_free + gid, 0u);
        ptx::fence_acq_rel();
        return_block(v, gid);
    }
}

__device__ __forceinline__ uint32_t gid_of(uint32_t t, uint64_t linear) {
    const uint32_t sh = 8 - t;                              // log2 nb(t)
    return (uint32_t)(((linear >> sh) << 8) | (linear & ((1u << sh) - 1)));
}

// [dev] formatter tokens: at most v.formatters threads format segments for
// one tree at a time (the paper lets every waiting thread format, P:151-155;
// one at a time would serialize the bursts in which every slot refills).
__device__ __forceinline__ bool token_try(uint32_t *tok, uint32_t limit) {
    if (atomicAdd(tok, 1u) < limit) return true;
    atomicSub(tok, 1u);
    return false;
}
__device__ __forceinline__ void token_release(uint32_t *tok) {
    ptx::fence_acq_rel();
    atomicSub(tok, 1u);
}

// [dev] format one more segment for tree t when the current one runs low, so
// that refills rarely wait for a format (skipped if every token is busy).
__device__ inline __noinline__ void format_ahead(const View &v, uint32_t t) {
    uint32_t *tok = v.fmt_token + t * 32;
    if (!token_try(tok, v.formatters)) return;
    const uint64_t s = claim_front(v);
    if (s != kNone) format_segment(v, s, t, 0);
    token_release(tok);
}

// [dev] A run covering whole segments takes up to want/nb fresh segments
// privately (no ring, no block tree): the lowest free one and the free ones
// that follow it.  Returns the blocks taken (0 if no segment is free).
__device__ inline __noinline__ uint32_t take_segments(const View &v, uint32_t t, uint32_t want, uint32_t *first) {
    const uint32_t nb = nb_of(t);
    uint32_t k = 0;
    const uint32_t kmax = want / nb;
#ifdef GALLATIN_TRACE
    const uint64_t tr0 = ptx::globaltimer();
#endif
    const uint64_t s0 = claim_front_run(v, kmax, &k);
    if (s0 == kNone) return 0;
#ifdef GALLATIN_TRACE
    const uint32_t attempts = k >> 16;
#endif
    k &= 0xFFFFu;
#ifdef GALLATIN_TRACE
    const uint64_t tr1 = ptx::globaltimer();
    ptx::trace(tr0, tr1, (1ull << 60) | ((uint64_t)attempts << 32) | ((uint64_t)t << 24) | k);
#endif
    const BitTree st = seg_tree(v);
    // extend with the following free segments: one atomicAnd per leaf
    // word claims the whole window, the consecutive prefix is kept and
    // the rest given back (serially: the next free segments in order)
    while (k < kmax && s0 + k < v.nseg && ((s0 + k) & 63) == 0) {
        const uint64_t x = s0 + k, wi = x >> 6;
        const uint32_t lo = (uint32_t)(x & 63);
        uint64_t hi = lo + (uint64_t)(kmax - k);
        if (hi > 64) hi = 64;
        if ((wi << 6) + hi > v.nseg) hi = v.nseg - (wi << 6);
        const uint64_t mask = bit_range(lo, (uint32_t)hi);
        uint64_t *leaf = st.w + st.off[0] + wi;
        const uint64_t old = ptx::atom_and(leaf, ~mask);
        const uint64_t got = old & mask;
        const uint64_t inv = ~(got >> lo);                 // 0 only if all 64 bits of a word were taken
        const uint32_t run = inv ? (uint32_t)__ffsll((long long)inv) - 1 : 64u;   // prefix length
        const uint64_t extra = got & ~bit_range(lo, lo + run);
        bool flip = old != 0 && (old & ~mask) == 0;
        if (extra) flip |= ptx::atom_or(leaf, extra) == 0;
        if (flip) bt_reconcile_up(st, 0, wi);
        if (extra) oom_notify(v);
        k += run;
        if (lo + run < hi) break;                         // the free run ended here
    }
    // tree ids (table words and the read-mostly copies) for the free path;
    // both are read only through a pointer this run hands out, so one fence
    // before the run is published (refill_slot's exchange) orders them all
    for (uint32_t q = 0; q < k; q++) ptx::st_relaxed(v.seg_tid + s0 + q, t);
    for (uint32_t q = 0; q < k; q++) ptx::atom_add(v.seg_word + s0 + q, sw_retree(kTreeFree, t));
    ptx::fence_acq_rel();
#ifdef GALLATIN_TRACE
    ptx::trace(tr1, ptx::globaltimer(), (2ull << 60) | ((uint64_t)t << 24) | k);
#endif
    *first = (uint32_t)(s0 * nb);
    return k * nb;
}

// [dev] Blocks of tree t that are reserved past their segment's available
// count (a negative count: a refiller's give-back of its excess is in
// flight) will be available again in a moment; a refill about to report "no
// memory" checks for them (one pass over the table, near exhaustion only) and
// retries instead.
constexpr uint32_t kFluxRetries = 64;
__device__ inline __noinline__ bool flux_pending(const View &v, uint32_t t) {
    for (uint64_t s = 0; s < v.nseg; s++) {
        const uint64_t w = ptx::ld_relaxed(v.seg_word + s);
        if (sw_tree(w) == t && sw_avail(w) < 0) return true;
    }
    return false;
}

// ---- Alg. 2 GetBlock(treeId), for a RUN of blocks [dev] --------
// Returns the number of consecutive blocks obtained (0 = exhausted) and the
// first one's linear index (segment * nb + block) in *first.
// check_oom: fail at once (*first = kOomFast) if tree t is recorded exhausted
// -- checked only once the block tree came up empty, with the record loaded
// at entry, so a refill that finds blocks pays no extra round trip.
__device__ inline __noinline__ uint32_t get_run_once(const View &v, uint32_t t, uint32_t want, uint32_t *first,
                                                     bool check_oom = false) {
    const uint64_t oom_r = check_oom ? ptx::ld_relaxed(v.oom) : 0, oom_rec = check_oom ? ptx::ld_relaxed(v.oom + 1 + t) : 0;
    const BitTree bt = block_tree(v, t);
    const uint32_t nb = nb_of(t);
    ptx::Backoff bo(4, t);
    uint64_t from = 0, hint = kNone;
    uint32_t attempt = 0, flux_retries = 0;
    bool flux = false;            // saw blocks of tree t reserved beyond the available count
    for (;;) {
        // findSegment; after a lost race, a random other candidate
        const uint64_t s = hint != kNone ? hint : bt_successor<false>(bt, from);
        hint = kNone;
        // [dev] a run of whole segments takes fresh ones while any is free
        // rather than a short run from a partly returned segment (the
        // warm-state refills); serially exact with O2-R's R2
        if (s != kNone && want >= nb && sw_avail(ptx::ld_relaxed(v.seg_word + s)) < (int32_t)want &&
            bt_successor<false>(seg_tree(v), 0) != kNone) {
            const uint32_t k = take_segments(v, t, want, first);
            if (k) return k;
        }
        if (s != kNone) {
            // reserve up to `want` blocks of s and validate its tree id in one RMW
            const uint64_t dec = (uint64_t)(-(int64_t)want);
            const uint64_t old = ptx::atom_add(v.seg_word + s, dec);
            const int32_t a = sw_avail(old);
            if (sw_tree(old) == t && a > 0) {
                const uint32_t got = (uint32_t)a < want ? (uint32_t)a : want;
                if (got < want) {
                    // give back the excess at once, then repair the block-tree
                    // bit once for both RMWs: the over-reservation must not
                    // drop s from the tree while other refillers search it
                    const uint64_t o2 = ptx::atom_add(v.seg_word + s, (uint64_t)(want - got));
                    if (sw_in_tree(old, t) != sw_in_tree(old + dec, t) ||
                        sw_in_tree(o2, t) != sw_in_tree(o2 + (want - got), t))
                        btree_reconcile(v, t, s);
                    oom_notify(v);
                } else {
                    seg_after_rmw(v, s, old, old + dec);
                }
                const uint32_t low = nb / 4;
                if (v.format_ahead && (uint32_t)a >= low && (uint32_t)a - got < low &&
                    bt_successor<false>(bt, s + 1) == kNone)
                    format_ahead(v, t);
                // getBlock from the segment's ring queue
                const uint32_t pos = atomicAdd(v.q_head + s, got);
                uint16_t *ring = v.q_entries + s * kMaxBlocks;
                uint64_t bm[4] = {0, 0, 0, 0};                   // the dequeued blocks (nb <= 256)
                // 16 independent loads in flight per batch (not one round trip per entry)
                for (uint32_t b = 0; b < got; b += 16) {
                    uint16_t r[16];
#pragma unroll
                    for (int u = 0; u < 16; u++)
                        if (b + u < got) r[u] = ptx::ld_relaxed(ring + ((pos + b + u) & (kMaxBlocks - 1)));
#pragma unroll
                    for (int u = 0; u < 16; u++) {
                        const uint32_t q = b + u;
                        if (q >= got) break;
                        uint16_t *ep = ring + ((pos + q) & (kMaxBlocks - 1));
                        uint16_t j = r[u];
                        ptx::Backoff wb(2, (s << 32) | ((pos + q) & 0xFFFFFFFFu));
                        while (j == kRingEmpty) {                 // enqueue in flight
                            wb.pause();
                            j = ptx::ld_relaxed(ep);
                        }
                        ptx::st_relaxed(ep, kRingEmpty);
                        bm[j >> 6] |= 1ull << (j & 63);
                    }
                }
                ptx::fence_acq_rel();
                // [dev] keep the longest run of consecutive blocks among them
                // (lowest start on ties): blocks come back in free order, so
                // the FIFO prefix alone would shrink runs to a block or two
                uint32_t bs = 0, bl = 0;
                for (uint32_t j = 0, len = 0; j <= nb; j++) {
                    if (j < nb && ((bm[j >> 6] >> (j & 63)) & 1)) { len++; continue; }
                    if (len > bl) { bl = len; bs = j - len; }
                    len = 0;
                }
                for (uint32_t j = bs; j < bs + bl; j++) bm[j >> 6] &= ~(1ull << (j & 63));
                if (bl < got) {                                   // the rest goes back, ascending: one enqueue
                    const uint32_t r = got - bl;
                    const uint32_t tp = atomicAdd(v.q_tail + s, r);
                    uint32_t q = 0;
                    for (uint32_t wv = 0; wv < 4; wv++) {
                        for (uint64_t w = bm[wv]; w; w &= w - 1, q++) {
                            uint16_t *ep = ring + ((tp + q) & (kMaxBlocks - 1));
                            ptx::Backoff wb(3, (s << 32) | ((tp + q) & 0xFFFFFFFFu));
                            while (ptx::ld_relaxed(ep) != kRingEmpty) wb.pause();   // previous lap's dequeue
                            ptx::st_relaxed(ep, (uint16_t)(wv * 64 + __ffsll((long long)w) - 1));
                        }
                    }
                    ptx::fence_acq_rel();
                    const uint64_t o3 = ptx::atom_add(v.seg_word + s, (uint64_t)r);
                    seg_after_rmw(v, s, o3, o3 + r);
                    oom_notify(v);
                }
                *first = (uint32_t)(s * nb + bs);
                return bl;
            }
            // stale hint (P:158-161's failure case): undo, repair, look further;
            // a negative count means another refiller's give-back is in flight
            if (sw_tree(old) == t && a < 0) flux = true;
            seg_after_rmw(v, s, old, old + dec);
            const uint64_t o2 = ptx::atom_add(v.seg_word + s, (uint64_t)want);
            seg_after_rmw(v, s, o2, o2 + want);
            btree_reconcile(v, t, s);
            oom_notify(v);
            from = s + 1;
            hint = claim_retry_hint(s >> 6, ptx::ld_relaxed(bt.w + bt.off[0] + (s >> 6)) & ~(1ull << (s & 63)),
                                    ++attempt);
            continue;
        }
        if (from != 0) {                                      // re-scan from the front once more
            from = 0;
            bo.pause();
            continue;
        }
        if (check_oom && oom_match(oom_r, oom_rec, t)) {      // [dev] exhaustion record
            *first = kOomFast;
            return 0;
        }
        // [dev] before reporting "no memory", wait out blocks that are only
        // transiently unavailable (an over-reservation being given back)
        if (flux && flux_retries < kFluxRetries) {
            flux = false;
            flux_retries++;
            bo.pause();
            continue;
        }
        if (want >= nb) {
            const uint32_t k = take_segments(v, t, want, first);
            if (k || !flux_pending(v, t) || flux_retries >= kFluxRetries) return k;   // 0: "No allocations left"
            flux_retries++;
            bo.pause();
            continue;
        }
        // Alg.2: format a segment; [dev] bounded formatters per tree
        uint32_t *tok = v.fmt_token + t * 32;
        if (token_try(tok, v.formatters)) {
            if (bt_successor<false>(bt, 0) != kNone) {        // someone published meanwhile
                token_release(tok);
                continue;
            }
            const uint64_t s1 = claim_front(v);
            if (s1 != kNone) format_segment(v, s1, t, want);
            token_release(tok);
            if (s1 == kNone) {
                if (bt_scan_first(bt) == kNone) {
                    if (!flux_pending(v, t) || flux_retries >= kFluxRetries) return 0;   // "No allocations left"
                    flux_retries++;
                    bo.pause();
                }
                continue;
            }
            *first = (uint32_t)(s1 * nb);
            return want;
        }
        while (ptx::ld_relaxed(tok) >= v.formatters && bt_successor<false>(bt, 0) == kNone) bo.pause();
    }
}

// ---- addresses -------------------------------------------------------------
__device__ __forceinline__ uint64_t *slot_word(const View &v, uint32_t si) { return v.slots + (uint64_t)si * 16; }

constexpr uint32_t kRunNone = 0x3FFFFFu;
constexpr uint64_t kSlotEmpty = kRunNone;                 // issued 0, run 0: refill on first use
__device__ __forceinline__ uint32_t run_len(uint64_t w) { return (uint32_t)(w >> kRunShift) & 0x3FFu; }

// [dev] Before reporting "no memory", every slot gives back the blocks of its
// run that no request has drawn from (class-major, slot-ascending): one CAS
// shrinks the run to ceil(issued / 4096) blocks -- issued and run share the
// word, so a draw racing the CAS makes it fail and retry, and no draw can land
// in a dropped block afterwards -- and the dropped blocks return whole.  A
// prefetched next run returns entirely.  Returns the number of blocks given back.
__device__ inline __noinline__ uint32_t trim_slots(const View &v) {
    uint32_t back = 0;
    for (uint32_t c = 0; c < kTrees; c++) {
        for (uint32_t q = 0; q < v.nslot[c]; q++) {
            uint64_t *sw = slot_word(v, v.slot_off[c] + q);
            uint64_t w = ptx::ld_relaxed(sw);
            for (;;) {
                const uint64_t cnt = w >> 32;
                const uint32_t m = run_len(w);
                if (cnt >= ((uint64_t)m << kSliceLog2)) break;            // exhausted or empty
                const uint32_t m2 = (uint32_t)((cnt + kSlices - 1) >> kSliceLog2);
                const uint64_t nw = m2 == 0 ? kSlotEmpty
                                            : (w & ~(0x3FFull << kRunShift)) | ((uint64_t)m2 << kRunShift);
                const uint64_t o = ptx::atom_cas(sw, w, nw);
                if (o != w) { w = o; continue; }
                for (uint32_t k = m2; k < m; k++) block_freed(v, gid_of(c, (w & kRunNone) + k), kSlices);
                back += m - m2;
                break;
            }
            {                                                    // a prefetched run (not one in flight)
                const uint64_t nx = ptx::ld_relaxed(sw + 1);
                if (run_len(nx) != 0 && ptx::atom_cas(sw + 1, nx, kSlotEmpty) == nx) {
                    for (uint32_t k = 0; k < run_len(nx); k++) block_freed(v, gid_of(c, (nx & kRunNone) + k), kSlices);
                    back += run_len(nx);
                }
            }
        }
    }
    return back;
}

// A run of up to `want` blocks of tree t (get_run_once); on "no memory" the
// slots' undrawn blocks are given back and the request retried for a SINGLE
// block (memory is scarce: no slot should hoard a run of it).  Under
// concurrency the retry repeats while trims still find blocks, and once
// more after an empty trim: a concurrent refiller's trim may just have given
// the blocks back.  Serially this is one trim and one retry.
__device__ inline __noinline__ uint32_t get_run(const View &v, uint32_t t, uint32_t want, uint32_t *first) {
    const bool rec = v.oom_record != 0;
#ifdef GALLATIN_TRACE
    const uint64_t tr0 = ptx::globaltimer();
    uint32_t got = get_run_once(v, t, want, first, rec);
    ptx::trace(tr0, ptx::globaltimer(), (3ull << 60) | ((uint64_t)t << 24) | (want << 12) | got);
#else
    uint32_t got = get_run_once(v, t, want, first, rec);
#endif
    if (got || (rec && *first == kOomFast)) return got;       // [dev] exhaustion record
    oom_enter(v);
    uint64_t e = 0;
    for (uint32_t r = 0; got == 0 && r < 8; r++) {
        const uint32_t back = trim_slots(v);                  // its block returns bump the epoch
        e = oom_epoch(v);
        got = get_run_once(v, t, 1, first);
        if (back == 0 && r >= 1) break;
    }
    oom_leave(v, t, e, rec && got == 0);
    return got;
}

// Replace an exhausted run (Alg.3): the run doubles up to the class cap.
// [dev] `hint` (bulk calls only): the blocks this slot's share of the launch
// needs (DESIGN.md Deviations 10); the run is at least that long, up to the cap.
// The length of a slot's next run: the first run (halves per class, floor
// min(run_init, 8), at most one segment) or 2^run_grow times the last, up to
// the class cap; [dev] at least `hint` blocks (the launch's demand, bulk
// calls only), rounded up to whole segments above one segment.
__device__ __forceinline__ uint32_t refill_want(const View &v, uint32_t c, uint32_t m_prev, uint32_t hint) {
    const uint32_t cap = v.run_cap[c];
    const uint32_t fl = v.run_init < 8 ? v.run_init : 8u;
    const uint32_t fs = (v.run_init >> c) > fl ? (v.run_init >> c) : fl;
    const uint32_t fr = fs < (256u >> c) ? fs : (256u >> c);
    const uint32_t first_run = fr < cap ? fr : cap;
    const uint32_t grow = m_prev << v.run_grow;
    uint32_t want = m_prev == 0 ? first_run : (grow < cap ? grow : cap);
    if (hint > want) {
        // whole segments once the hint exceeds one (a run of more than nb
        // blocks is taken in whole segments: 111 blocks would get 64)
        const uint32_t nb = nb_of(c);
        const uint32_t h = hint > nb ? (hint + nb - 1) / nb * nb : hint;
        want = h < cap ? h : cap;
    }
    return want;
}

// slot word 1 while a demand prefetch is fetching the run (run length 0: the
// drain and the trims see no blocks in it)
constexpr uint64_t kSlotPending = 0x3FFFFEull;

// Replace an exhausted run (Alg.3): the prefetched run if one is
// waiting in word 1 (or being fetched: wait for it), else a new run.
__device__ inline __noinline__ bool refill_slot(const View &v, uint32_t si, uint32_t c, uint32_t m_prev,
                                                uint32_t hint = 0) {
    {                                                         // [dev] the prefetched run, if any
#ifdef GALLATIN_TRACE
        const uint64_t ts0 = ptx::globaltimer();
#endif
        uint64_t *w1 = slot_word(v, si) + 1;
        uint64_t nx = ptx::ld_relaxed(w1);
        ptx::Backoff bo(6, si);
        while (nx == kSlotPending) {
            bo.pause();
            nx = ptx::ld_relaxed(w1);
        }
        if (run_len(nx) != 0 && ptx::atom_cas(w1, nx, kSlotEmpty) == nx) {
            ptx::st_relaxed(slot_word(v, si) + 2, 0ull);
            ptx::atom_exch(slot_word(v, si), nx);               // {issued 0, run, first}
#ifdef GALLATIN_TRACE
            ptx::trace(ts0, ptx::globaltimer(), (11ull << 60) | ((uint64_t)si << 32) | run_len(nx));
#endif
            return true;
        }
    }
    const uint32_t want = refill_want(v, c, m_prev, hint);
    uint32_t first = 0;
#ifdef GALLATIN_TRACE
    const uint64_t t0 = ptx::globaltimer();
    const uint32_t got = get_run(v, c, want, &first);
    ptx::trace(t0, ptx::globaltimer(), ((uint64_t)si << 32) | (c << 24) | (want << 12) | got);
#else
    const uint32_t got = get_run(v, c, want, &first);
#endif
    if (got == 0) {
        ptx::st_relaxed(slot_word(v, si) + 2, 1ull);        // waiters then consult the exhaustion record
        ptx::atom_exch(slot_word(v, si), kSlotEmpty);
        return false;
    }
    ptx::st_relaxed(slot_word(v, si) + 2, 0ull);
    ptx::atom_exch(slot_word(v, si), ((uint64_t)got << kRunShift) | first);
    return true;
}

// [dev] the request that draws the middle of a run fetches the next run
// (twice as long, up to the cap) into the slot's second word, so that the
// refill at the end of the run is one exchange.
__device__ inline __noinline__ void prefetch_slot(const View &v, uint32_t si, uint32_t c, uint32_t m) {
    if (ptx::ld_relaxed(slot_word(v, si) + 1) != kSlotEmpty) return;   // a run is already waiting
    const uint32_t cap = v.run_cap[c];
    const uint32_t grow = m << v.run_grow;
    const uint32_t want = grow < cap ? grow : cap;
    uint32_t first = 0;
    const uint32_t got = get_run_once(v, c, want, &first);         // never trims other slots
    if (got == 0) return;
    const uint64_t run = ((uint64_t)got << kRunShift) | first;
    if (ptx::atom_cas(slot_word(v, si) + 1, kSlotEmpty, run) != kSlotEmpty)
        for (uint32_t k = 0; k < got; k++) block_freed(v, gid_of(c, (uint64_t)first + k), kSlices);   // raced: give back
}

// [dev] Demand prefetch (bulk CTA kernel, DESIGN.md Deviations 19): a tile
// whose slot RMW leaves the run shorter than the launch's estimated demand
// on the slot fetches the next run into word 1 after its own stores -- one
// tile per slot wins the EMPTY -> PENDING CAS -- so the run's end swaps it
// in instead of stalling every CTA of the slot on a refill.
__device__ inline __noinline__ void demand_prefetch(const View &v, uint32_t si, uint32_t c, uint32_t m,
                                                    uint32_t hint) {
    uint64_t *w1 = slot_word(v, si) + 1;
    if (ptx::atom_cas(w1, kSlotEmpty, kSlotPending) != kSlotEmpty) return;
    uint32_t first = 0;
    const uint32_t got = get_run_once(v, c, refill_want(v, c, m, hint), &first);   // never trims other slots
    ptx::atom_exch(w1, got ? (((uint64_t)got << kRunShift) | first) : kSlotEmpty);
}

__device__ __forceinline__ void *slice_ptr(const View &v, uint32_t c, uint64_t first, uint64_t idx) {
    // offset(blockId*4096 + idx) with the run's blocks contiguous
    return reinterpret_cast<void *>(v.heap + (first << (16 + c)) + (idx << (kMinSliceLog2 + c)));
}

__device__ __forceinline__ uint32_t slice_class(uint64_t size) {
    return size <= 16 ? 0u : (uint32_t)(64 - __clzll((long long)(size - 1))) - kMinSliceLog2;
}
__device__ __forceinline__ uint32_t block_class(uint64_t size) {
    return size <= 65536 ? 0u : (uint32_t)(64 - __clzll((long long)(size - 1))) - 16;
}

// After a team RMW returned `old` and this lane drew idx >= the run's end:
// refill (the lane that drew exactly the end) or wait for the refill.
// Returns false if the refill found no memory.
__device__ inline __noinline__ bool slot_exhausted(const View &v, uint32_t si, uint32_t c, uint64_t old, uint32_t idx) {
    const uint32_t m = run_len(old);
    if (idx == (m << kSliceLog2)) return refill_slot(v, si, c, m);
    ptx::Backoff bo(1, si);
#ifdef GALLATIN_TRACE
    const uint64_t tw0 = ptx::globaltimer();
    struct TraceEnd {
        uint64_t t0, si;
        __device__ ~TraceEnd() {
            if ((threadIdx.x & 31) == (uint32_t)(__ffs((int)__activemask()) - 1))
                ptx::trace(t0, ptx::globaltimer(), (10ull << 60) | (si << 32));
        }
    } trace_end{tw0, si};
#endif
    for (;;) {
        // the slot word and its failed-refill flag share a sector (one round trip)
        const uint64_t w = ptx::ld_relaxed(slot_word(v, si));
        const uint64_t failed = ptx::ld_relaxed(slot_word(v, si) + 2);
        if ((uint32_t)(w >> 32) <= (run_len(w) << kSliceLog2)) return true;
        // the last refill found no memory: if tree c is still recorded
        // exhausted, the pending refill cannot succeed either [dev]
        if (failed && oom_known(v, c)) return false;
        bo.note(w);
        bo.pause();
    }
}

// ---- Alg. 3 MALLOC.Slice ---------------------------------------
// The lanes of a warp asking the same slot form a team (reading A-8);
// the leader does ONE atomicAdd on the slot word {issued:32 | run:8 |
// first:24} that returns the run and the first slice index together [dev: the
// paper reads the buffer, then adds on the block's counter]; __shfl_sync
// broadcasts it; lane r takes index old+r, valid iff < 4096 * run.
// The lane that draws the end replaces the run (reading A-7);
// lanes past it wait for the replacement and retry.
__device__ inline void *malloc_slice(const View &v, uint32_t c, uint32_t key) {
    const uint32_t si = v.slot_off[c] + key % v.nslot[c];
    uint64_t *sw = slot_word(v, si);
    const uint32_t lane = ptx::lane_id();
    for (;;) {
        const unsigned act = __activemask();
        const unsigned peers = __match_any_sync(act, si);
        const uint32_t leader = (uint32_t)__ffs((int)peers) - 1;
        const uint32_t rank = (uint32_t)__popc(peers & ptx::lanemask_lt());
        uint64_t old = 0;
        if (lane == leader) old = ptx::atom_add(sw, (uint64_t)__popc(peers) << 32);
        old = __shfl_sync(peers, old, (int)leader);
        const uint32_t cnt = (uint32_t)(old >> 32), limit = run_len(old) << kSliceLog2;
        const uint32_t idx = cnt + rank;
        if (idx < limit) {
            if (v.prefetch && idx == (limit >> 1)) prefetch_slot(v, si, c, run_len(old));
            return slice_ptr(v, c, old & kRunNone, idx);
        }
        const uint32_t n = (uint32_t)__popc(peers);
        if (cnt <= limit && limit < cnt + n) {
            // The refiller is in this team: its team-mates past the end wait at
            // a warp barrier, not in a sleep loop that would stall the
            // refiller's own diverged path.
            unsigned waiters = peers;
            for (uint32_t k = limit - cnt; k; k--) waiters &= waiters - 1;   // drop the valid lanes
            bool ok = true;
            if (idx == limit) ok = refill_slot(v, si, c, run_len(old));
            ok = __shfl_sync(waiters, ok, __ffs((int)waiters) - 1);
            if (!ok) return nullptr;            // nullptr: the team's refill found no memory
            continue;
        }
        // refill is another warp's; false: tree c is recorded exhausted [dev]
        if (!slot_exhausted(v, si, c, old, idx)) return nullptr;
    }
}

// (4 KB, 16 MB): one whole block of the smallest fitting tree; its counter is
// preset to 4095 so that Alg.4's rule returns it on its one free (reading A-2).
// [dev] The lanes of a warp asking the same block tree form a team (the
// paper's coalescing, applied to whole blocks): the team's lowest
// unserved lane asks GetBlock for as many blocks as lanes remain and the run
// it gets is dealt out in lane order, until every lane has a block or the
// tree is exhausted.  A lone request is exactly GetBlock(t) (serial replay).
__device__ inline __noinline__ void *malloc_block(const View &v, uint32_t t) {
    const unsigned peers = __match_any_sync(__activemask(), t);
    const uint32_t lane = ptx::lane_id();
    unsigned pending = peers;
    void *res = nullptr;
    while (pending) {
        const uint32_t leader = (uint32_t)__ffs((int)pending) - 1;
        uint32_t first = 0, got = 0;
        if (lane == leader) got = get_run(v, t, (uint32_t)__popc(pending), &first);
        got = __shfl_sync(peers, got, (int)leader);
        first = __shfl_sync(peers, first, (int)leader);
        if (got == 0) break;                                   // "No allocations left"
        const uint32_t r = (uint32_t)__popc(pending & ptx::lanemask_lt());
        if (((pending >> lane) & 1) && r < got) {
            atomicExch(v.block_free + gid_of(t, (uint64_t)first + r), kSlices - 1);
            res = reinterpret_cast<void *>(v.heap + (((uint64_t)first + r) << (16 + t)));
        }
        unsigned served = pending;                            // the lowest `got` pending lanes
        for (uint32_t k = got; k < (uint32_t)__popc(pending); k++) served &= ~(1u << (31 - __clz((int)served)));
        pending &= ~served;
    }
    return res;
}

// >= 16 MB: Alg.1 with treeId >= numBlockTrees: claimMultiple from the back
// (P:110-113); tree id = numBlockTrees + numSegments.
__device__ inline __noinline__ void *malloc_large(const View &v, uint64_t k) {
    if (k > v.nseg) return nullptr;
    const BitTree st = seg_tree(v);
    ptx::Backoff bo(5, k);
    uint64_t i;
    int misses = 0;
    bool trimmed = false;
    uint64_t below = kNone;
    uint32_t lost = 0;
    for (;;) {
        i = bt_find_highest_run(st, k, below);
        if (i == kNone && below != kNone) {                   // nothing lower: search everything again
            below = kNone;
            continue;
        }
        if (i == kNone) {
            if (!trimmed) {                                   // [dev] as get_run: slots give back first
                trimmed = true;
                if (trim_slots(v)) continue;
            }
            if (++misses > 2) return nullptr;
            bo.pause();
            continue;
        }
        if (bt_claim_range(st, i, k)) break;
        oom_notify(v);                                        // the claim's rollback gave segments back
        // [dev] concurrent claimers of one size all found the same run: the
        // loser looks below it, a pseudo-random number of k-runs down (whole
        // runs, so equal-size claims stay packed from the top: the heap still
        // holds floor(nseg / k) of them); serially no claim loses: the
        // highest run
        {
            const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
            uint32_t h = (tid * 0x9E3779B1u) ^ (++lost * 0x85EBCA6Bu);
            h ^= h >> 15;
            const uint64_t jit = k * (uint64_t)(h % (128u * (lost < 8 ? lost : 8u)));   // widens with each loss
            below = i > jit ? i - jit : 0;
        }
    }
    ptx::fence_acq_rel();
    ptx::st_relaxed(v.seg_tid + i, kTrees + (uint32_t)k);
    for (uint64_t m = 1; m < k; m++) ptx::st_relaxed(v.seg_tid + i + m, kTreeCont);
    ptx::atom_add(v.seg_word + i, sw_retree(kTreeFree, kTrees + (uint32_t)k));
    for (uint64_t m = 1; m < k; m++) ptx::atom_add(v.seg_word + i + m, sw_retree(kTreeFree, kTreeCont));
    ptx::fence_acq_rel();
    return reinterpret_cast<void *>(v.heap + (i << kSegLog2));
}

// Classify (A1): slices 16 B..4 KB by ceil(log2), blocks, segments.
__device__ inline void *malloc_impl(const View &v, uint64_t size, uint32_t key) {
    if (size == 0) return nullptr;
    if (size <= kMaxSlice) return malloc_slice(v, slice_class(size), key);
    if (size < kSegBytes) return malloc_block(v, block_class(size));
    const uint64_t k = (size >> kSegLog2) + ((size & (kSegBytes - 1)) != 0);
    return malloc_large(v, k);
}

// segment allocation: return the k segments to the segment tree
__device__ inline __noinline__ void free_large(const View &v, uint64_t s, uint32_t t) {
    const uint64_t k = t - kTrees;
    ptx::fence_acq_rel();
    ptx::atom_add(v.seg_word + s, sw_retree(t, kTreeFree));
    for (uint64_t m = 1; m < k; m++) ptx::atom_add(v.seg_word + s + m, sw_retree(kTreeCont, kTreeFree));
    for (uint64_t m = 0; m < k; m++) ptx::st_relaxed(v.seg_tid + s + m, kTreeFree);
    ptx::fence_acq_rel();
    bt_insert_range(seg_tree(v), s, k);
    oom_notify(v);
}

// ---- Alg. 4 FREE -----------------------------------------------
__device__ inline void free_impl(const View &v, void *p) {
    if (p == nullptr) return;
    const uint64_t off = reinterpret_cast<uint64_t>(p) - v.heap;
    if (off >= (v.nseg << kSegLog2)) { atomicAdd(v.err, 1ull); return; }
    const uint64_t s = off >> kSegLog2;
    const uint32_t t = sw_tree(ptx::ld_relaxed(v.seg_word + s));   // ldcv(ids[segment])
    if (t < kTrees) {
        // locateBlock; frees of one block coalesce
        const uint32_t gid = (uint32_t)(s * kMaxBlocks + ((off & (kSegBytes - 1)) >> (16 + t)));
        const unsigned act = __activemask();
        const unsigned peers = __match_any_sync(act, gid);
        const uint32_t leader = (uint32_t)__ffs((int)peers) - 1;
        if (v.fence_free != 2) __syncwarp(peers);
        if (ptx::lane_id() == leader) {
            if (v.fence_free != 2) ptx::fence_acq_rel();     // release the team's writes
            block_freed(v, gid, (uint32_t)__popc(peers));
        }
        return;
    }
    if (t == kTreeFree || t == kTreeCont) { atomicAdd(v.err, 1ull); return; }
    free_large(v, s, t);
}

// Quiescent drain, part 1 (one thread): retire every slot in class-major
// order; the unissued remainder of every block of its run counts as freed.
__device__ inline void drain_slots(const View &v) {
    for (uint32_t c = 0; c < kTrees; c++) {
        for (uint32_t q = 0; q < v.nslot[c]; q++) {
            const uint64_t w = ptx::atom_exch(slot_word(v, v.slot_off[c] + q), kSlotEmpty);
            const uint64_t cnt = w >> 32;
            const uint32_t m = run_len(w);
            const uint64_t first = w & kRunNone;
            for (uint32_t k = 0; k < m; k++) {
                const uint64_t lo = (uint64_t)k << kSliceLog2;
                const uint64_t issued = cnt <= lo ? 0 : (cnt - lo > kSlices ? kSlices : cnt - lo);
                if (issued < kSlices) block_freed(v, gid_of(c, first + k), (uint32_t)(kSlices - issued));
            }
            // a prefetched run was never issued from: all of it comes back
            const uint64_t nx = ptx::atom_exch(slot_word(v, v.slot_off[c] + q) + 1, kSlotEmpty);
            for (uint32_t k = 0; k < run_len(nx); k++) block_freed(v, gid_of(c, (nx & kRunNone) + k), kSlices);
        }
    }
}

// Quiescent drain, part 2: a segment whose blocks are all home (formatted
// ahead, never used) goes back to the segment tree.
__device__ inline void retire_idle(const View &v, uint64_t s) {
    const uint64_t w = ptx::ld_relaxed(v.seg_word + s);
    const uint32_t t = sw_tree(w);
    if (t < kTrees && sw_avail(w) == (int32_t)nb_of(t)) try_free_segment(v, s, t);
}

}  // namespace core
}  // namespace gallatin
