/*
 * oracle/veb_oracle.c -- O1: the TEXTBOOK van Emde Boas tree (CPU, sequential).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this code.  It
 * shares no code, header, table or constant with the CUDA path
 * (paper_conf_ppopp_mccoyp24_b200/csrc) and never calls it.
 *
 * What it follows (PAPER.md = /root/reference/PAPER.md, "Gallatin", PPoPP'24):
 *   - P:71-79 (S3 "Preliminary"): the set operations over U = {0..u-1}:
 *       insert(x): S <- S u {x};  delete(x): S <- S \ {x};  query(x): x in S?
 *       succ(x) = min{ y in S : y >= x };  pred(x) = max{ y in S : y <= x };
 *       "x in U but x need not be in S".
 *   - P:83-87 (S3.1 "vEB tree design"): the recursive node = (min, max,
 *     summary bit-array over sqrt(U) children, sqrt(U) subtrees); insert and
 *     delete recurse and maintain min/max; successor checks max, then min,
 *     then recurses into the cluster or the summary.  The recursion is the
 *     CLRS (3rd ed., S20.3) formulation the paper describes: min is NOT
 *     stored inside a cluster; the upper root is 2^ceil(k/2), the lower
 *     root 2^floor(k/2).
 *   - P:76 uses ">= x" for succ (CLRS uses "> x"); succ_ge(x) is therefore
 *     member(x) ? x : succ_gt(x)  (reading A-21).  "None" is
 *     returned as UINT64_MAX (reading A-21: the paper's -1).
 *
 * The canonical bitmap-level image (oracle_veb_image) is the DEFINITION of
 * the words the GPU's 64-ary bitmap tree must hold at quiescence:
 * level 0 word i bit b = [64*i + b in S]; level l>0 word i bit b = [level l-1
 * word 64*i + b != 0]; levels stop at the first level with one word; bits at
 * or beyond the universe are 0 (reading A-22).  It is produced here from the
 * membership of S only (enumerated through succ), not from any GPU layout.
 *
 * Batches are applied sequentially in index order.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define NIL (-1LL)
#define NONE UINT64_MAX

typedef struct vnode {
    unsigned k;               /* universe of this node is 2^k, k >= 1      */
    int64_t min, max;         /* NIL when the subtree is empty        */
    struct vnode *summary;    /* universe 2^hi: which clusters are non-empty */
    struct vnode **cluster;   /* 2^hi clusters, each of universe 2^lo       */
} vnode;

static unsigned hi_bits(unsigned k) { return (k + 1) / 2; } /* upper sqrt exponent */
static unsigned lo_bits(unsigned k) { return k / 2; }       /* lower sqrt exponent */
static int64_t high(const vnode *v, int64_t x) { return x >> lo_bits(v->k); }
static int64_t low(const vnode *v, int64_t x) { return x & ((1LL << lo_bits(v->k)) - 1); }
static int64_t index_of(const vnode *v, int64_t h, int64_t l) { return (h << lo_bits(v->k)) | l; }

static vnode *vnode_new(unsigned k) {
    vnode *v = (vnode *)calloc(1, sizeof(vnode));
    v->k = k;
    v->min = v->max = NIL;
    if (k > 1) v->cluster = (vnode **)calloc((size_t)1 << hi_bits(k), sizeof(vnode *));
    return v;
}

static void vnode_free(vnode *v) {
    if (!v) return;
    if (v->k > 1) {
        size_t nc = (size_t)1 << hi_bits(v->k);
        for (size_t i = 0; i < nc; i++) vnode_free(v->cluster[i]);
        free(v->cluster);
        vnode_free(v->summary);
    }
    free(v);
}

/* Lazily created children keep the O(u) textbook structure affordable. */
static vnode *get_summary(vnode *v) {
    if (!v->summary) v->summary = vnode_new(hi_bits(v->k));
    return v->summary;
}
static vnode *get_cluster(vnode *v, int64_t h) {
    if (!v->cluster[h]) v->cluster[h] = vnode_new(lo_bits(v->k));
    return v->cluster[h];
}
static int64_t vmin(const vnode *v) { return v ? v->min : NIL; }
static int64_t vmax(const vnode *v) { return v ? v->max : NIL; }

static int member(const vnode *v, int64_t x) {
    if (x == v->min || x == v->max) return 1;
    if (v->k == 1) return 0;
    const vnode *c = v->cluster[high(v, x)];
    return c ? member(c, low(v, x)) : 0;
}

/* CLRS VEB-TREE-SUCCESSOR: smallest element strictly greater than x. */
static int64_t succ_gt(const vnode *v, int64_t x) {
    if (v->k == 1) {
        if (x == 0 && v->max == 1) return 1;
        return NIL;
    }
    if (v->min != NIL && x < v->min) return v->min;
    const vnode *c = v->cluster[high(v, x)];
    int64_t max_low = vmax(c);
    if (max_low != NIL && low(v, x) < max_low) {
        int64_t off = succ_gt(c, low(v, x));
        return index_of(v, high(v, x), off);
    }
    if (!v->summary) return NIL;
    int64_t sc = succ_gt(v->summary, high(v, x));
    if (sc == NIL) return NIL;
    return index_of(v, sc, vmin(v->cluster[sc]));
}

/* CLRS VEB-TREE-PREDECESSOR: largest element strictly less than x. */
static int64_t pred_lt(const vnode *v, int64_t x) {
    if (v->k == 1) {
        if (x == 1 && v->min == 0) return 0;
        return NIL;
    }
    if (v->max != NIL && x > v->max) return v->max;
    const vnode *c = v->cluster[high(v, x)];
    int64_t min_low = vmin(c);
    if (min_low != NIL && low(v, x) > min_low) {
        int64_t off = pred_lt(c, low(v, x));
        return index_of(v, high(v, x), off);
    }
    int64_t pc = v->summary ? pred_lt(v->summary, high(v, x)) : NIL;
    if (pc == NIL) {
        if (v->min != NIL && x > v->min) return v->min;
        return NIL;
    }
    return index_of(v, pc, vmax(v->cluster[pc]));
}

static void empty_insert(vnode *v, int64_t x) { v->min = v->max = x; }

/* CLRS VEB-TREE-INSERT (x not in S). P:85: recurse, maintain min/max. */
static void insert(vnode *v, int64_t x) {
    if (v->min == NIL) { empty_insert(v, x); return; }
    if (x < v->min) { int64_t t = x; x = v->min; v->min = t; }
    if (v->k > 1) {
        vnode *c = get_cluster(v, high(v, x));
        if (c->min == NIL) {
            insert(get_summary(v), high(v, x));
            empty_insert(c, low(v, x));
        } else {
            insert(c, low(v, x));
        }
    }
    if (x > v->max) v->max = x;
}

/* CLRS VEB-TREE-DELETE (x in S). */
static void delete_(vnode *v, int64_t x) {
    if (v->min == v->max) { v->min = v->max = NIL; return; }
    if (v->k == 1) {
        v->min = (x == 0) ? 1 : 0;
        v->max = v->min;
        return;
    }
    if (x == v->min) {
        int64_t first = vmin(v->summary);
        x = index_of(v, first, vmin(v->cluster[first]));
        v->min = x;
    }
    vnode *c = v->cluster[high(v, x)];
    delete_(c, low(v, x));
    if (c->min == NIL) {
        delete_(v->summary, high(v, x));
        if (x == v->max) {
            int64_t smax = vmax(v->summary);
            if (smax == NIL) v->max = v->min;
            else v->max = index_of(v, smax, vmax(v->cluster[smax]));
        }
    } else if (x == v->max) {
        v->max = index_of(v, high(v, x), c->max);
    }
}

/* ---------------------------------------------------------------- API --- */
typedef struct oracle_veb {
    unsigned k;      /* universe u = 2^k */
    uint64_t u;
    uint64_t n;      /* |S| */
    vnode *root;
} oracle_veb;

oracle_veb *oracle_veb_create(unsigned k) {
    if (k < 1 || k > 40) return NULL;
    oracle_veb *h = (oracle_veb *)calloc(1, sizeof(oracle_veb));
    h->k = k;
    h->u = 1ULL << k;
    h->root = vnode_new(k);
    return h;
}

void oracle_veb_destroy(oracle_veb *h) {
    if (!h) return;
    vnode_free(h->root);
    free(h);
}

uint64_t oracle_veb_size(const oracle_veb *h) { return h->n; }

int oracle_veb_member(const oracle_veb *h, uint64_t x) {
    if (x >= h->u) return 0;
    return member(h->root, (int64_t)x);
}

/* returns 1 iff x was newly added */
int oracle_veb_insert(oracle_veb *h, uint64_t x) {
    if (x >= h->u) return 0;
    if (member(h->root, (int64_t)x)) return 0;
    insert(h->root, (int64_t)x);
    h->n++;
    return 1;
}

/* returns 1 iff x was present */
int oracle_veb_delete(oracle_veb *h, uint64_t x) {
    if (x >= h->u) return 0;
    if (!member(h->root, (int64_t)x)) return 0;
    delete_(h->root, (int64_t)x);
    h->n--;
    return 1;
}

/* succ(x) = min{y in S : y >= x}; NONE if there is no such y. */
uint64_t oracle_veb_successor(const oracle_veb *h, uint64_t x) {
    if (x >= h->u) return NONE;
    if (member(h->root, (int64_t)x)) return x;
    int64_t y = succ_gt(h->root, (int64_t)x);
    return y == NIL ? NONE : (uint64_t)y;
}

/* pred(x) = max{y in S : y <= x}; NONE if there is no such y.
 * For x beyond the universe this is max(S) (the definition, unclamped). */
uint64_t oracle_veb_predecessor(const oracle_veb *h, uint64_t x) {
    if (x >= h->u) return h->root->max == NIL ? NONE : (uint64_t)h->root->max;
    if (member(h->root, (int64_t)x)) return x;
    int64_t y = pred_lt(h->root, (int64_t)x);
    return y == NIL ? NONE : (uint64_t)y;
}

uint64_t oracle_veb_min(const oracle_veb *h) { return h->root->min == NIL ? NONE : (uint64_t)h->root->min; }
uint64_t oracle_veb_max(const oracle_veb *h) { return h->root->max == NIL ? NONE : (uint64_t)h->root->max; }

/* Op codes for oracle_veb_apply: one batch applied in index order. */
enum { OV_INSERT = 0, OV_DELETE = 1, OV_MEMBER = 2, OV_SUCC = 3, OV_PRED = 4 };

void oracle_veb_apply(oracle_veb *h, const uint8_t *ops, const uint64_t *keys,
                      uint64_t n, uint64_t *out) {
    for (uint64_t i = 0; i < n; i++) {
        uint64_t r = 0;
        switch (ops[i]) {
        case OV_INSERT: r = (uint64_t)oracle_veb_insert(h, keys[i]); break;
        case OV_DELETE: r = (uint64_t)oracle_veb_delete(h, keys[i]); break;
        case OV_MEMBER: r = (uint64_t)oracle_veb_member(h, keys[i]); break;
        case OV_SUCC: r = oracle_veb_successor(h, keys[i]); break;
        case OV_PRED: r = oracle_veb_predecessor(h, keys[i]); break;
        default: r = NONE;
        }
        if (out) out[i] = r;
    }
}

/* Homogeneous batches: same op for every key, in index order. */
void oracle_veb_batch(oracle_veb *h, int op, const uint64_t *keys, uint64_t n, uint64_t *out) {
    for (uint64_t i = 0; i < n; i++) {
        uint8_t o = (uint8_t)op;
        oracle_veb_apply(h, &o, keys + i, 1, out ? out + i : NULL);
    }
}

/* Geometry of the canonical bitmap image: number of levels and the word
 * count of level l.  Level 0 has ceil(u/64) words; each next level has
 * ceil(prev/64) words; the last level is the first with exactly one word. */
unsigned oracle_veb_image_levels(unsigned k, uint64_t *words_per_level /* >= 8 */) {
    uint64_t u = 1ULL << k;
    uint64_t w = (u + 63) / 64;
    unsigned L = 0;
    for (;;) {
        words_per_level[L++] = w;
        if (w == 1) break;
        w = (w + 63) / 64;
    }
    return L;
}

/* Writes the canonical image (all levels concatenated, level 0 first) to
 * out[0..total), returns total words, or 0 if cap is too small. */
uint64_t oracle_veb_image(const oracle_veb *h, uint64_t *out, uint64_t cap) {
    uint64_t wpl[16];
    unsigned L = oracle_veb_image_levels(h->k, wpl);
    uint64_t total = 0;
    for (unsigned l = 0; l < L; l++) total += wpl[l];
    if (cap < total) return 0;
    memset(out, 0, total * sizeof(uint64_t));
    /* level 0: membership of S, enumerated through succ */
    uint64_t x = oracle_veb_min(h);
    while (x != NONE) {
        out[x >> 6] |= 1ULL << (x & 63);
        x = (x + 1 < h->u) ? oracle_veb_successor(h, x + 1) : NONE;
    }
    /* level l: bit b of word i says "child word 64*i+b is non-empty" */
    uint64_t base_prev = 0, base = wpl[0];
    for (unsigned l = 1; l < L; l++) {
        for (uint64_t c = 0; c < wpl[l - 1]; c++)
            if (out[base_prev + c]) out[base + (c >> 6)] |= 1ULL << (c & 63);
        base_prev = base;
        base += wpl[l];
    }
    return total;
}
