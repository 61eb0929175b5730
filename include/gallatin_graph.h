/*
 * gallatin_graph.h -- the streaming-graph workload of BASELINE configs[4] on
 * the device-side allocator (libgallatin.so).  PAPER.md S6.12:
 * "graphs are stored in memory as edge lists, with an edge list for a given
 * vertex malloc the next largest power of two region of memory"; the
 * operations are initialization, (bulk) edge insertion, (bulk) deletion and
 * expansion.
 *
 * Every per-vertex list is allocated, grown, shrunk and freed by GPU threads
 * through the device API (include/gallatin/device.cuh); the host only
 * launches kernels.  Policy (reading A-29), evaluated once per batch
 * per vertex: a list holds `size` uint32 destination ids in `cap` slots,
 * cap = next power of two >= max(size, 4); a batch that makes size > cap
 * reallocates to the new cap (malloc, copy, free); a delete batch that leaves
 * size <= cap/4 reallocates down, and size 0 frees the list (cap 0).
 *
 * Requires gallatin_init.  Arrays are caller-owned DEVICE memory; batch calls
 * are asynchronous on `stream`.  Errors: GALLATIN_ERR_* (gallatin.h); an
 * allocation that returned NULL inside a kernel is counted in
 * gallatin_graph_counters()[2]; an edge or expansion entry whose source vertex
 * id is >= num_vertices is ignored (no list is touched) and counted in
 * gallatin_graph_counters()[3].
 */
#ifndef GALLATIN_GRAPH_H_
#define GALLATIN_GRAPH_H_
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct gallatin_graph gallatin_graph_t;

/* An empty graph over vertices [0, num_vertices); library-owned state. */
int gallatin_graph_create(uint32_t num_vertices, gallatin_graph_t **out);
/* Frees every list (device API) and the graph state. */
int gallatin_graph_destroy(gallatin_graph_t *g, void *stream);

/* One bulk insert batch: append d_dst[i] to the list of d_src[i]. */
int gallatin_graph_insert(gallatin_graph_t *g, const uint32_t *d_src, const uint32_t *d_dst, uint64_t n, void *stream);
/* One bulk delete batch: remove ONE instance of d_dst[i] from the list of
 * d_src[i] for every i (edges not present are ignored). */
int gallatin_graph_delete(gallatin_graph_t *g, const uint32_t *d_src, const uint32_t *d_dst, uint64_t n, void *stream);
/* One expansion round ("graph expansion"): every vertex in d_v (distinct)
 * appends max(size, 4) edges; edge j of vertex v gets destination
 * (v + size_before + j + 1) mod num_vertices. */
int gallatin_graph_expand(gallatin_graph_t *g, const uint32_t *d_v, uint64_t n, void *stream);

/* Single-edge operations ("edge updates" / "edge deletes", as opposed
 * to the bulk batches above): one GPU thread per edge, each under its source
 * vertex's lock.  insert_edges appends d_dst[i] to the list of d_src[i]; a
 * full list (size == cap) is reallocated to 2*cap (4 if empty) at that edge.
 * delete_edges removes ONE instance of d_dst[i] from the list of d_src[i] if
 * present (the newest such entry; the last entry fills the hole); after each removal size 0 frees
 * the list and size <= cap/4 (cap > 4) reallocates it to nextpow2(max(size, 4)).
 * Final sizes, capacities and adjacency multisets are independent of the
 * thread order (reading A-29 per edge).  Asynchronous on `stream`. */
int gallatin_graph_insert_edges(gallatin_graph_t *g, const uint32_t *d_src, const uint32_t *d_dst, uint64_t n,
                                void *stream);
int gallatin_graph_delete_edges(gallatin_graph_t *g, const uint32_t *d_src, const uint32_t *d_dst, uint64_t n,
                                void *stream);

/* Per-vertex size, capacity and list pointer (any may be NULL). */
int gallatin_graph_export(const gallatin_graph_t *g, uint32_t *d_size, uint32_t *d_cap, uint64_t *d_list, void *stream);
/* CSR copy: d_out[d_offsets[v] + k] = list_v[k] for k < size_v (caller gives
 * the exclusive prefix sum of the sizes). */
int gallatin_graph_gather(const gallatin_graph_t *g, const uint64_t *d_offsets, uint32_t *d_out, void *stream);
/* Device counters: [0] mallocs, [1] frees, [2] failed mallocs, [3] ignored
 * entries with a vertex id >= num_vertices (synchronizes). */
int gallatin_graph_counters(const gallatin_graph_t *g, uint64_t out[4]);

#ifdef __cplusplus
}
#endif
#endif
