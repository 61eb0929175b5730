// gallatin/bittree.cuh -- the paper's GPU van Emde Boas tree.
//
// PAPER.md S3.2: "we fix the size of each node to 64 bits, and we remove the
// min and max values ... every vEB node operation [is] performed in one atomic
// operation"; the height is bounded by a small constant: ceil(log64 u).
// Level 0 word i bit b  <=>  element 64*i+b is in S.
// Level l word i bit b  <=>  level l-1 word 64*i+b is non-zero (a summary).
// Bits at or beyond the universe are always 0.
//
// Concurrency: insert/delete change a leaf
// with one atomicOr/atomicAnd; the thread whose RMW flips a word between empty
// and non-empty reconciles the parent bit with the loop
//     read child; set/clear parent bit to match; fence.sc; re-read child;
//     repeat if the child's emptiness changed
// so that, at quiescence, every summary bit equals "child non-empty".
// Successor/predecessor tolerate transient stale summaries: a set summary bit
// over an empty child restarts the search just past that child.
#pragma once
#include <stdint.h>

#include "gallatin/ptx.cuh"

namespace gallatin {

constexpr uint64_t kNone = ~0ull;
constexpr int kMaxLevels = 8;

struct BitTree {
    uint64_t *w;          // all levels, level 0 first
    uint64_t nbits;       // universe size
    uint32_t levels;
    uint32_t off[kMaxLevels];
};

// Geometry: level 0 has ceil(nbits/64) words, each next level ceil(prev/64),
// the last level is the first with one word.  Returns the total word count.
__host__ __device__ inline uint64_t bittree_geometry(uint64_t nbits, uint32_t *levels, uint32_t *off) {
    uint64_t w = (nbits + 63) / 64, total = 0;
    uint32_t L = 0;
    for (;;) {
        off[L++] = (uint32_t)total;
        total += w;
        if (w <= 1) break;
        w = (w + 63) / 64;
    }
    *levels = L;
    return total;
}

template <bool NC>
__device__ __forceinline__ uint64_t bt_load(const uint64_t *p) {
    if constexpr (NC) return ptx::ld_nc(p);
    else return ptx::ld_relaxed(p);
}

// Make the level-(lvl+1) bit of word `idx` agree with that word's emptiness,
// walking up while our RMWs flip a parent between empty and non-empty.
__device__ inline void bt_reconcile_up(const BitTree &t, uint32_t lvl, uint64_t idx) {
    while (lvl + 1 < t.levels) {
        const uint64_t *child = t.w + t.off[lvl] + idx;
        uint64_t *parent = t.w + t.off[lvl + 1] + (idx >> 6);
        const uint64_t bit = 1ull << (idx & 63);
        bool flipped = false;
        ptx::fence_sc();
        for (;;) {
            const bool ne = ptx::ld_relaxed(child) != 0;
            const uint64_t old = ne ? ptx::atom_or(parent, bit) : ptx::atom_and(parent, ~bit);
            flipped |= ne ? (old == 0) : (old == bit);
            ptx::fence_sc();
            if ((ptx::ld_relaxed(child) != 0) == ne) break;
        }
        if (!flipped) return;
        lvl++;
        idx >>= 6;
    }
}

// The setting half of the reconcile: the thread whose RMW made level-lvl word
// idx non-empty sets its parent bit with a release fence before the RMW, and
// climbs while its RMWs flip parents from empty.  No re-read loop is needed on
// this side: if a clearer's RMW on the parent bit comes after ours in the
// bit's coherence order, it read our release, so the clearer's re-read (after
// its fence.sc, bt_reconcile_up) sees our child RMW and sets the bit again.
// One fence.acq_rel per level instead of two fence.sc and a re-read.
__device__ inline void bt_set_up(const BitTree &t, uint32_t lvl, uint64_t idx) {
    while (lvl + 1 < t.levels) {
        ptx::fence_acq_rel();
        const uint64_t old = ptx::atom_or(t.w + t.off[lvl + 1] + (idx >> 6), 1ull << (idx & 63));
        if (old != 0) return;
        lvl++;
        idx >>= 6;
    }
}

// insert(x): S <- S u {x}.  Returns true iff x was newly added.
__device__ inline bool bt_insert(const BitTree &t, uint64_t x) {
    if (x >= t.nbits) return false;
    const uint64_t bit = 1ull << (x & 63);
    const uint64_t old = ptx::atom_or(t.w + t.off[0] + (x >> 6), bit);
    if (old == 0) bt_set_up(t, 0, x >> 6);
    return !(old & bit);
}

// delete(x): S <- S \ {x}.  Returns true iff x was present -- which is
// also the paper's claimIndex: exactly one thread removes a bit.
__device__ inline bool bt_delete(const BitTree &t, uint64_t x) {
    if (x >= t.nbits) return false;
    const uint64_t bit = 1ull << (x & 63);
    const uint64_t old = ptx::atom_and(t.w + t.off[0] + (x >> 6), ~bit);
    if (old == bit) bt_reconcile_up(t, 0, x >> 6);
    return (old & bit) != 0;
}

template <bool NC>
__device__ inline bool bt_member(const BitTree &t, uint64_t x) {
    if (x >= t.nbits) return false;
    return (bt_load<NC>(t.w + t.off[0] + (x >> 6)) >> (x & 63)) & 1;
}

// succ(x) = min{y in S : y >= x}, kNone if none.  The recursion of P:87
// flattened onto 64-ary levels: mask the leaf at x, else climb the summaries
// looking strictly right of the current child, then descend by lowest bits.
template <bool NC>
__device__ inline uint64_t bt_successor(const BitTree &t, uint64_t x) {
    for (;;) {
        if (x >= t.nbits) return kNone;
        uint64_t idx = x >> 6;
        // allocator trees (coherent loads, mostly-empty leaves): the leaf and
        // the first summary word on the path are independent loads, issued
        // together (one round trip, not two); bulk queries (NC) load lazily
        const uint64_t w0 = bt_load<NC>(t.w + t.off[0] + idx);
        const uint64_t s1 = (!NC && t.levels > 1) ? bt_load<NC>(t.w + t.off[1] + (idx >> 6)) : 0;
        const uint64_t w = w0 & (~0ull << (x & 63));
        if (w) return (idx << 6) + (uint64_t)(__ffsll((long long)w) - 1);
        uint32_t lvl = 1;
        for (; lvl < t.levels; lvl++) {
            const uint32_t pos = (uint32_t)(idx & 63);
            const uint64_t p = idx >> 6;
            const uint64_t m = pos == 63 ? 0 : (~0ull << (pos + 1));
            const uint64_t s = m ? (((!NC && lvl == 1) ? s1 : bt_load<NC>(t.w + t.off[lvl] + p)) & m) : 0;
            idx = p;
            if (s) { idx = (p << 6) + (uint64_t)(__ffsll((long long)s) - 1); break; }
        }
        if (lvl >= t.levels) return kNone;
        bool stale = false;
        for (int d = (int)lvl - 1; d >= 0; d--) {
            const uint64_t v = bt_load<NC>(t.w + t.off[d] + idx);
            if (v == 0) {                      // stale summary: resume past this child
                x = (idx + 1) << (6 * (d + 1));
                stale = true;
                break;
            }
            idx = (idx << 6) + (uint64_t)(__ffsll((long long)v) - 1);
        }
        if (!stale) return idx;
    }
}

// pred(x) = max{y in S : y <= x}, kNone if none; x beyond the universe
// is clamped (pred is then max S).
template <bool NC>
__device__ inline uint64_t bt_predecessor(const BitTree &t, uint64_t x) {
    if (t.nbits == 0) return kNone;
    if (x >= t.nbits) x = t.nbits - 1;
    for (;;) {
        uint64_t idx = x >> 6;
        const uint32_t pos0 = (uint32_t)(x & 63);
        const uint64_t m0 = pos0 == 63 ? ~0ull : ((2ull << pos0) - 1);
        uint64_t w = bt_load<NC>(t.w + t.off[0] + idx) & m0;
        if (w) return (idx << 6) + 63 - (uint64_t)__clzll((long long)w);
        uint32_t lvl = 1;
        for (; lvl < t.levels; lvl++) {
            const uint32_t pos = (uint32_t)(idx & 63);
            const uint64_t p = idx >> 6;
            const uint64_t m = pos == 0 ? 0 : ((1ull << pos) - 1);
            const uint64_t s = m ? (bt_load<NC>(t.w + t.off[lvl] + p) & m) : 0;
            idx = p;
            if (s) { idx = (p << 6) + 63 - (uint64_t)__clzll((long long)s); break; }
        }
        if (lvl >= t.levels) return kNone;
        bool stale = false;
        for (int d = (int)lvl - 1; d >= 0; d--) {
            const uint64_t v = bt_load<NC>(t.w + t.off[d] + idx);
            if (v == 0) {                      // stale summary: resume below this child
                const uint64_t first = idx << (6 * (d + 1));
                if (first == 0) return kNone;
                x = first - 1;
                stale = true;
                break;
            }
            idx = (idx << 6) + 63 - (uint64_t)__clzll((long long)v);
        }
        if (!stale) return idx;
    }
}

// First set bit by a linear scan of the leaves, ignoring the summaries: the
// confirmation step before reporting exhaustion (summaries may lag).
__device__ inline uint64_t bt_scan_first(const BitTree &t) {
    const uint64_t nw = (t.nbits + 63) / 64;
    for (uint64_t i = 0; i < nw; i++) {
        const uint64_t v = ptx::ld_relaxed(t.w + t.off[0] + i);
        if (v) return (i << 6) + (uint64_t)(__ffsll((long long)v) - 1);
    }
    return kNone;
}

// Mask of bits [lo, hi) within one 64-bit word (0 <= lo < hi <= 64).
__device__ __forceinline__ uint64_t bit_range(uint32_t lo, uint32_t hi) {
    const uint64_t upper = hi == 64 ? ~0ull : ((1ull << hi) - 1);
    return upper & (~0ull << lo);
}

// Insert [i, i+k) (the paper's segmentTree.insert(segment, numSegments)).
__device__ inline void bt_insert_range(const BitTree &t, uint64_t i, uint64_t k) {
    uint64_t x = i, end = i + k;
    while (x < end) {
        const uint64_t wi = x >> 6;
        const uint32_t lo = (uint32_t)(x & 63);
        const uint32_t hi = (uint32_t)((end - (wi << 6)) < 64 ? (end - (wi << 6)) : 64);
        const uint64_t old = ptx::atom_or(t.w + t.off[0] + wi, bit_range(lo, hi));
        if (old == 0) bt_set_up(t, 0, wi);
        x = (wi << 6) + hi;
    }
}

// Claim [i, i+k) -- all bits must be set; on a conflict every bit this call
// cleared is restored and false is returned (the paper's claimMultiple).
__device__ inline bool bt_claim_range(const BitTree &t, uint64_t i, uint64_t k) {
    uint64_t x = i, end = i + k;
    bool ok = true;
    while (x < end) {
        const uint64_t wi = x >> 6;
        const uint32_t lo = (uint32_t)(x & 63);
        const uint32_t hi = (uint32_t)((end - (wi << 6)) < 64 ? (end - (wi << 6)) : 64);
        const uint64_t m = bit_range(lo, hi);
        const uint64_t old = ptx::atom_and(t.w + t.off[0] + wi, ~m);
        if ((old & m) != m) {
            // give back what this call took in this word, then roll back the rest
            const uint64_t took = old & m;
            if (took) {
                const uint64_t o2 = ptx::atom_or(t.w + t.off[0] + wi, took);
                if (o2 == 0) bt_reconcile_up(t, 0, wi);
            }
            if (old != 0 && (old & ~m) == 0) bt_reconcile_up(t, 0, wi);
            ok = false;
            end = x;                  // roll back [i, x)
            break;
        }
        if ((old & ~m) == 0) bt_reconcile_up(t, 0, wi);   // the word became empty
        x = (wi << 6) + hi;
    }
    if (!ok && end > i) bt_insert_range(t, i, end - i);
    return ok;
}

// Highest start i such that [i, i+k) is all set (first fit from the back,
// P:138 / reading A-17), by a top-down walk over the leaf words; kNone if no
// such run is visible.  Leaf reads are relaxed: the claim re-validates.
// `below`: only runs entirely below this index (kNone: the whole tree).
// The leaf words are loaded 8 at a time (independent loads in flight) and
// walked from the top down in registers.
__device__ inline uint64_t bt_find_highest_run(const BitTree &t, uint64_t k, uint64_t below = kNone) {
    if (k == 0 || k > t.nbits) return kNone;
    const uint64_t lim = below < t.nbits ? below : t.nbits;
    if (lim < k) return kNone;
    const uint64_t nw = (lim + 63) / 64;
    const uint64_t top_mask = (lim & 63) ? ((1ull << (lim & 63)) - 1) : ~0ull;   // bits < lim in the top word
    uint64_t run = 0;   // length of the set run just above the current word
    uint64_t top = 0;   // highest element of that run
    uint64_t batch[8];
    for (uint64_t wi = nw; wi-- > 0;) {
        const uint32_t slot = (uint32_t)((nw - 1 - wi) & 7);
        if (slot == 0) {                                      // next 8 words down, loads in flight together
#pragma unroll
            for (int q = 0; q < 8; q++)
                batch[q] = wi >= (uint64_t)q ? ptx::ld_relaxed(t.w + t.off[0] + wi - q) : 0ull;
        }
        uint64_t v = batch[slot];
        if (wi == nw - 1) v &= top_mask;
        const uint64_t base = wi << 6;
        if (v == ~0ull) {
            if (run == 0) top = base + 63;
            run += 64;
            if (run >= k) return top - k + 1;
            continue;
        }
        // leading ones (from bit 63 down) extend the run from above
        const uint32_t lead = (uint32_t)__clzll((long long)~v);
        if (lead) {
            if (run == 0) top = base + 63;
            run += lead;
            if (run >= k) return top - k + 1;
        }
        // runs strictly inside the word, high to low
        uint64_t rest = lead ? (v & ~bit_range(64 - lead, 64)) : v;
        while (rest) {
            const uint32_t hi = 63 - (uint32_t)__clzll((long long)rest);
            // number of consecutive ones from bit hi downward
            const uint64_t shifted = rest << (63 - hi);
            const uint32_t len = (uint32_t)__clzll((long long)~shifted);
            if (len >= k) return base + hi - k + 1;
            if (hi + 1 == len) {      // run touches bit 0: continues into the word below
                break;
            }
            rest &= ~bit_range(hi + 1 - len, hi + 1);
        }
        // the run at the bottom of this word continues downward
        const uint32_t trail = (uint32_t)__ffsll((long long)~v) - 1;   // v != ~0
        if (trail && !(lead && trail + lead >= 64)) {
            run = trail;
            top = base + trail - 1;
        } else {
            run = 0;
        }
    }
    return kNone;
}

}  // namespace gallatin
