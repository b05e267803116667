/*
 * ecl_cc.h — C ABI of the B200-native ECL-CC connected-components library (libecl_cc.so).
 *
 * The operation (PAPER.md = /root/reference/PAPER.md; "P:Lnnn" = its line nnn):
 *   Given an undirected graph G = (V, E) in CSR form (§4: each undirected edge is
 *   stored as two directed entries), "label each vertex with the ID of the component to
 *   which it belongs" (§1).  The label written is the minimum vertex ID of the
 *   component (the convention of P:L61 §1 / Fig. 1; reading R1) — the unique
 *   fixed point the ECL-CC method (§3) reaches, so results are deterministic
 *   and bit-exact across runs, launch configurations and GPU counts.
 *
 * Method (all on the GPU, hand-written CUDA for sm_100a):
 *   init  : Init3 — parent[v] = first neighbour in adjacency order with a smaller ID,
 *           else v (§3); vertices are binned by degree into a double-sided
 *           worklist (§3: <=16 thread, 17..352 warp, >352 block).
 *   hook  : asynchronous, lock-free union-find over every edge once, in one direction
 *           (v > u), on representatives found with intermediate pointer jumping
 *           (Fig. 5, Fig. 6).
 *   final : single pointer jumping, parent[v] = root(v) (Fini3, §5.1).
 *
 * Conventions for every entry point:
 *   - Vertex IDs are int32 in [0, n).  Offsets (nindex) are int32 (ecl_cc_run) or int64
 *     (ecl_cc_run_i64); nindex has n+1 entries, nindex[0] == 0, nindex[n] == m, and is
 *     non-decreasing.  nlist has m entries.
 *   - Unless a name ends in _host, every pointer is a CUDA device pointer on the handle's
 *     device.  The caller owns all of them; the library never frees them and keeps no
 *     reference after the call returns.
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  Device
 *     entry points only ENQUEUE work: no host synchronisation, no device->host copies.
 *     Results are valid once the stream reaches that point.
 *   - The graph must be symmetric (every (a,b) entry has a matching (b,a) entry); this is
 *     a precondition, not checked by the run calls (R9).  ecl_cc_validate is the
 *     opt-in checker.  Self-loops, duplicate entries and unsorted rows are accepted.
 *   - Errors: argument errors return ECL_CC_ERR_INVALID_ARG before anything is enqueued;
 *     CUDA launch/allocation errors return ECL_CC_ERR_CUDA / ECL_CC_ERR_OOM and the CUDA
 *     error text is available from ecl_cc_last_error(h).  n == 0 is a no-op returning OK.
 *   - A handle may be used by one host thread at a time.  It owns device scratch (the
 *     double-sided worklist and counters, O(n)), allocated stream-ordered on first use,
 *     grown on demand, and released by ecl_cc_destroy.  Calls on one handle are ordered:
 *     a call enqueued on a stream other than the previous call's first makes its stream
 *     wait (cudaStreamWaitEvent) for the previous call, since they share the scratch.
 */
#ifndef ECL_CC_H
#define ECL_CC_H

#include <stdint.h>

#if defined(__GNUC__)
#define ECL_CC_API __attribute__((visibility("default")))
#else
#define ECL_CC_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct ecl_cc_ctx *ecl_cc_handle;

typedef enum {
    ECL_CC_OK = 0,
    ECL_CC_ERR_INVALID_ARG = 1,
    ECL_CC_ERR_CUDA = 2,
    ECL_CC_ERR_OOM = 3,
    ECL_CC_ERR_INVALID_GRAPH = 4 /* only returned by ecl_cc_validate */
} ecl_cc_status;

/* Create a handle bound to CUDA device `device` (queries SM count / occupancy; no large
 * allocations).  *out is set to NULL on failure. */
ECL_CC_API ecl_cc_status ecl_cc_create(ecl_cc_handle *out, int device);

/* Release the handle and its scratch.  NULL is a no-op.  No device-wide synchronisation:
 * the scratch is freed stream-ordered after the handle's most recent call, and the host
 * waits only for that (the handle's own work), not for other work on the device. */
ECL_CC_API ecl_cc_status ecl_cc_destroy(ecl_cc_handle h);

/* Connected components of the whole graph (int32 offsets; requires m <= INT32_MAX).
 *   n          number of vertices (>= 0)
 *   m          number of directed CSR entries (== nindex[n])
 *   nindex     n+1 offsets (device)
 *   nlist      m neighbour IDs (device)
 *   nstat_out  n labels out (device); also used as the union-find parent array during
 *              the run, so it must not alias nindex/nlist.
 * On completion nstat_out[v] = min{ w : w reachable from v }.
 * Asynchrony: only enqueues work on `stream` (no host sync, no D2H); with the default
 * kernel order (ECL_CC_OPT_ORDER 2) hook_block runs on a handle-owned side stream forked
 * from and joined back into `stream` with events.  After one warm-up call has grown the
 * handle's scratch for this graph size, a call can be captured into a CUDA graph and
 * replayed (tests/test_gpu_parity.py::test_cuda_graph_capture_replay). */
ECL_CC_API ecl_cc_status ecl_cc_run(ecl_cc_handle h, int32_t n, int64_t m, const int32_t *nindex,
                         const int32_t *nlist, int32_t *nstat_out, void *stream);

/* Same with int64 offsets (graphs with m > INT32_MAX, e.g. Graph500 scale 27). */
ECL_CC_API ecl_cc_status ecl_cc_run_i64(ecl_cc_handle h, int32_t n, int64_t m, const int64_t *nindex,
                             const int32_t *nlist, int32_t *nstat_out, void *stream);

/* End-to-end convenience call on HOST buffers: copies nindex/nlist host->device into
 * handle-owned device buffers, runs, copies the labels device->host, and synchronises
 * `stream` before returning.  index_bytes is 4 (int32 offsets) or 8 (int64 offsets).
 * Host buffers should be pinned (cudaHostAlloc / cudaHostRegister) for full PCIe speed. */
ECL_CC_API ecl_cc_status ecl_cc_run_host(ecl_cc_handle h, int32_t n, int64_t m, const void *nindex_host,
                              int index_bytes, const int32_t *nlist_host,
                              int32_t *labels_host, void *stream);

/* Connected components plus a spanning forest (the union-find use the
 * paper names next).  Labels are written to labels_out exactly as ecl_cc_run
 * does.  For every vertex x that is not its component's minimum, (tree_a[x], tree_b[x])
 * is a CSR edge, and these n - #components edges form a spanning forest of the graph
 * (one spanning tree per component); for component minima both entries are -1.
 * The edges are the Init edges (x, parent[x]) of the initialisation plus, for
 * every successful hook CAS of Fig. 6 (lines 9/14) that made a root x a child, the edge
 * being hooked — it joins exactly the two trees the CAS merges.  The forest is one
 * valid answer of many (it depends on the race order); the labels are unique.
 *   index_bytes  4 (nindex is int32, m <= INT32_MAX) or 8 (int64)
 *   tree_a/b     n int32 each (device), caller-owned.
 * Same errors and asynchrony as ecl_cc_run. */
ECL_CC_API ecl_cc_status ecl_cc_spanning_forest(ecl_cc_handle h, int32_t n, int64_t m,
                                                const void *nindex, int index_bytes,
                                                const int32_t *nlist, int32_t *labels_out,
                                                int32_t *tree_a, int32_t *tree_b, void *stream);

/* ---- input preparation beside the hot path ----------------------------
 * ecl_cc_build_csr: the symmetric CSR ECL-CC consumes, built on the GPU from an undirected
 * edge list the way the paper prepared its inputs (§4): self-loops are removed,
 * multiple edges between the same two vertices are merged, missing back edges are added,
 * and each undirected edge becomes two directed entries.  Rows come out ascending.
 *   n              number of vertices; every src/dst ID must be in [0, n)
 *   num_edges      pairs in src/dst (device, int32 each); (a,b) and (b,a) are the same edge
 *   nindex_out     n+1 int64 offsets (device, caller-owned)
 *   nlist_out      int32 entries (device, caller-owned), room for nlist_capacity entries;
 *                  2*num_edges always suffices
 *   m_out          HOST int64: entries written (== nindex_out[n])
 * Synchronises `stream` (the entry count is returned to the host).  Scratch (2 x 16 bytes
 * per pair + CUB temp) is owned by the handle, grow-only.  Errors: INVALID_GRAPH if an ID
 * is out of range; INVALID_ARG (with *m_out = the needed count) if nlist_capacity is too
 * small.  The sort and duplicate removal use CUB (cub::DeviceRadixSort, DeviceSelect). */
ECL_CC_API ecl_cc_status ecl_cc_build_csr(ecl_cc_handle h, int32_t n, int64_t num_edges,
                                          const int32_t *src, const int32_t *dst,
                                          int64_t *nindex_out, int32_t *nlist_out,
                                          int64_t nlist_capacity, int64_t *m_out, void *stream);

/* Host readers (no handle, no GPU): an undirected edge list in malloc'ed host arrays
 * (*src_out, *dst_out; release each with ecl_cc_free_host).  Edges are returned as stored
 * (loops / duplicates / one direction only); pass them to ecl_cc_build_csr.
 * ecl_cc_read_mtx: MatrixMarket "coordinate" files (SMC / SuiteSparse, the source of most
 *   of Table 2's graphs); 1-based (i, j) entries become 0-based edges, any value
 *   columns are ignored, n = max(rows, cols).
 * ecl_cc_read_edgelist: whitespace-separated "a b" lines, '#' or '%' comment lines (SNAP);
 *   0-based IDs, n = 1 + the largest ID.
 * Errors: INVALID_ARG (null argument / unreadable file), INVALID_GRAPH (malformed file or
 * index out of range), OOM; the message is available from ecl_cc_io_last_error() (per
 * host thread). */
ECL_CC_API ecl_cc_status ecl_cc_read_mtx(const char *path, int32_t *n_out, int64_t *num_edges_out,
                                         int32_t **src_out, int32_t **dst_out);
ECL_CC_API ecl_cc_status ecl_cc_read_edgelist(const char *path, int32_t *n_out,
                                              int64_t *num_edges_out, int32_t **src_out,
                                              int32_t **dst_out);
ECL_CC_API void ecl_cc_free_host(void *p);
ECL_CC_API const char *ecl_cc_io_last_error(void);

/* ---- multi-GPU building blocks (the transport is the caller's NCCL process group) ----
 * ecl_cc_run_rows: local forest of the rows [row_lo, row_hi) of a graph with n vertices.
 *   m_rows       entries of the slice (== nindex_rows[row_hi-row_lo])
 *   nindex_rows  row_hi-row_lo+1 int64 offsets into nlist_rows, rebased so
 *                nindex_rows[0] == 0 (device)
 *   nlist_rows   the concatenated adjacency of those rows (device)
 *   parent       n entries out (device): flattened min-ID labels of the subgraph formed by
 *                the edges stored in these rows (every vertex outside them labels itself
 *                unless joined through an edge).  Each undirected edge (a,b), a > b, is
 *                hooked by the owner of row a only (Fig. 6 line 1 "if (v > u)").  With
 *                ECL_CC_OPT_STOP_AFTER = 2 the forest is left unflattened: parent[v] <= v
 *                is some vertex of v's tree, enough to be a peer of ecl_cc_merge.
 * ecl_cc_merge: hook the edges (v, peer_labels[v - v_lo]) for v in [v_lo, v_hi) into the
 *   forest `parent` (every v whose peer entry differs from v).  peer_labels is any forest
 *   of the peer's subgraph with peer_labels[v] <= v in v's peer tree: a flattened min-ID
 *   labelling or an unflattened parent array (the pairs (v, peer[v]) span the same trees,
 *   P:L161-L163).  Does NOT flatten; call ecl_cc_finalize once after the last merge.
 * ecl_cc_finalize: parent[v] = root(v) for all v (Fini3). */
ECL_CC_API ecl_cc_status ecl_cc_run_rows(ecl_cc_handle h, int32_t n, int32_t row_lo, int32_t row_hi,
                              int64_t m_rows, const int64_t *nindex_rows,
                              const int32_t *nlist_rows, int32_t *parent, void *stream);
ECL_CC_API ecl_cc_status ecl_cc_merge(ecl_cc_handle h, int32_t n, int32_t v_lo, int32_t v_hi,
                           const int32_t *peer_labels, int32_t *parent, void *stream);
ECL_CC_API ecl_cc_status ecl_cc_finalize(ecl_cc_handle h, int32_t n, int32_t *parent, void *stream);

/* ---- encoded forest exchange and P2P merge (not in the paper) ----------
 * ecl_cc_forest_encode: encode a forest `labels` (n entries with labels[x] <= x in x's
 *   tree: a flattened labelling, or an unflattened forest such as ecl_cc_run_rows with
 *   STOP_AFTER 2 leaves — each vertex's root is then found by a read-only walk) as the
 *   relation it spans: D = root(anchor) (pick a vertex of the largest component, e.g. the
 *   highest-degree row; anchor = -1: no bitmap class, every non-root becomes a pair;
 *   with ECL_CC_OPT_MERGE_FILTER set and an R21 bitmap in this handle's most recent run,
 *   which must be the run that built `labels`, that run's anchor replaces `anchor` and its
 *   bitmap proves most vertices' class without a walk), bits[v / 32] bit v % 32 set iff
 *   root(v) == D, and the pairs (v, root(v)) of every other v with root(v) != v.
 *   The edges {(v, D) : bit v} u {(v, root(v)) : pairs} span exactly the classes of
 *   `labels`, so merging them is exact (hook-once sufficiency).
 *     bits   (n + 31) / 32 uint32 words out (device)
 *     pairs  2 x cap int32 out (device): pair i is (pairs[2i], pairs[2i+1]); the order is
 *            unspecified.  cap = n always suffices.
 *     meta   2 uint64 out (device): meta[0] = number of pairs (may exceed cap: then only
 *            cap pairs were written and the caller must retry with a larger cap),
 *            meta[1] = D.
 *   Enqueues only (the counts stay on the device).
 * ecl_cc_merge_encoded: hook the relations of npeers (0..8) encodings into the forest
 *   `parent` (n entries; does NOT flatten: call ecl_cc_finalize after the last merge).
 *   bits / pairs / meta / caps are HOST arrays of npeers entries; the buffers they point
 *   to are device memory readable from the handle's device — local copies, or another
 *   GPU's buffers mapped with ecl_cc_ipc_open (NVLink peer reads: the transfer happens
 *   inside the merge kernels).  caps[i] bounds the pairs read from peer i.  The peer
 *   buffers must stay valid and unchanged until the merge has run on `stream`.
 * ecl_cc_ipc_export: the ECL_CC_IPC_HANDLE_BYTES-byte handle of a device pointer (CUDA IPC
 *   handle of its allocation + the pointer's offset in it), for another process.
 * ecl_cc_ipc_open: map such a handle on `device` (peer access enabled lazily); returns a
 *   device pointer usable by that process's kernels.  ecl_cc_ipc_close unmaps it.
 * Errors: INVALID_ARG for bad arguments, ECL_CC_ERR_CUDA when CUDA IPC fails. */
#define ECL_CC_IPC_HANDLE_BYTES 72
ECL_CC_API ecl_cc_status ecl_cc_forest_encode(ecl_cc_handle h, int32_t n, const int32_t *labels,
                                              int32_t anchor, uint32_t *bits, int32_t *pairs,
                                              int64_t cap, uint64_t *meta, void *stream);
ECL_CC_API ecl_cc_status ecl_cc_merge_encoded(ecl_cc_handle h, int32_t n, int npeers,
                                              const uint32_t *const *bits,
                                              const int32_t *const *pairs,
                                              const uint64_t *const *meta, const int64_t *caps,
                                              int32_t *parent, void *stream);
ECL_CC_API ecl_cc_status ecl_cc_ipc_export(const void *dev_ptr, void *handle_out);
ECL_CC_API ecl_cc_status ecl_cc_ipc_open(int device, const void *handle, void **dev_ptr_out);
ECL_CC_API ecl_cc_status ecl_cc_ipc_close(void *dev_ptr);

/* Debug checker (synchronises the stream): offsets monotone with nindex[0]==0 and
 * nindex[n]==m, neighbour IDs in range, graph symmetric.  Returns ECL_CC_OK or
 * ECL_CC_ERR_INVALID_GRAPH.  index_bytes is 4 or 8. */
ECL_CC_API ecl_cc_status ecl_cc_validate(ecl_cc_handle h, int32_t n, int64_t m, const void *nindex,
                              int index_bytes, const int32_t *nlist, void *stream);

/* ---- options (apply to later runs on this handle) ----------------------------------- */
typedef enum {
    ECL_CC_OPT_THRESH_THREAD = 1, /* max degree of the thread bin (paper: 16)           */
    ECL_CC_OPT_THRESH_WARP = 2,   /* max degree of the warp bin (paper: 352)            */
    ECL_CC_OPT_GRID_BLOCKS = 3,   /* override blocks per launch (0 = auto); race shaking */
    ECL_CC_OPT_STOP_AFTER = 4,    /* debug: 1 = stop after init (nstat_out = Init3
                                     parents), 2 = stop before finalize, 0 = full run    */
    ECL_CC_OPT_LOAD_MODE = 5,     /* parent[] loads: bit 0 set = weak L1-cacheable loads,
                                     clear = ld.relaxed.gpu (R7); bit 1 = L2
                                     policies (parent evict_last, adjacency evict_first) */
    ECL_CC_OPT_TIMING = 6,        /* 1 = record CUDA events between the phase kernels of
                                     every run (read with ecl_cc_get_timing)             */
    ECL_CC_OPT_TTAS = 7,          /* 1 (default) = load-test the target before every hook
                                     CAS (test-and-test-and-set); 0 = bare CAS (Fig. 6)  */
    ECL_CC_OPT_L2_FETCH = 8,      /* cudaLimitMaxL2FetchGranularity hint in bytes (32, 64,
                                     128) for the device; 0 = leave unchanged.  NOTE: a
                                     device-wide setting that outlives the handle.       */
    ECL_CC_OPT_OCC_THREAD = 9,    /* blocks per SM of hook_thread (0 = max occupancy);
                                     with ORDER 2 it caps hook_warp as well (both run
                                     on the caller's stream next to hook_block)         */
    ECL_CC_OPT_OCC_RANGE = 10,    /* blocks per SM of hook_warp / hook_block (0 = max);
                                     with ORDER 2: of hook_block only (0 = 3/4 of max)  */
    /* paper ablations; defaults are ECL-CC's */
    ECL_CC_OPT_INIT = 11,         /* 3 = Init3 first smaller neighbour (default),
                                     2 = Init2 smallest neighbour, 1 = Init1 own ID      */
    ECL_CC_OPT_JUMP = 12,         /* 4 = intermediate (halving, default), 1 = multiple,
                                     2 = single, 3 = none                                */
    ECL_CC_OPT_FINI = 13,         /* 3 = single (default), 1 = intermediate, 2 = multiple */
    ECL_CC_OPT_BATCH = 14,        /* 1 (default) = batched two-hop gathers with early exit
                                     at v_rep (R16/R19); 0 = one find per edge */
    ECL_CC_OPT_FILTER = 15,       /* anchor-tree membership bitmap (R21): 0 off,
                                     1 on, 2 (default) = on when 4n > 128 MB             */
    ECL_CC_OPT_ORDER = 16,        /* order of the three independent hook kernels: 0 =
                                     thread, warp, block (paper); 1 = block,
                                     warp, thread (hubs first); 2 (default) = block on a
                                     handle-owned side stream (forked from and joined
                                     back into the run's stream with events) capped at
                                     OCC_RANGE blocks/SM (0 = 3/4 of the SM), thread
                                     then warp on the run's stream with full grids that
                                     take the SM slots hook_block leaves or retires.
                                     Labels are the same in every order (R13).         */
    ECL_CC_OPT_PREJUMP = 17,      /* pointer-doubling passes between init and the hook
                                     kernels (R23; Jump's pointer jumping,
                                     P:L245, as synchronous passes): 0 off, 1 always,
                                     2 (default) only when a sample of the Init3
                                     forest is deep (meshes, road-like graphs).
                                     Labels are unchanged (R13).                       */
    ECL_CC_OPT_FLATTEN_PASSES = 18, /* ecl_cc_finalize only: run R23's pointer-jumping
                                     passes before the finalize kernel: 0 (default) off,
                                     1 always, 2 when a depth probe finds the forest deep.
                                     For merged multi-GPU forests, whose former roots
                                     form long chains that Fini3 would walk per vertex. */
    ECL_CC_OPT_FUSE_INIT = 19,    /* Init3 folded into the hook kernels (R28):
                                     the init kernel only bins rows by degree and writes
                                     parent[v] = v; the kernel that owns a row's start
                                     CASes parent[v] from v to the first smaller
                                     neighbour (Init3's value) if v is still a root.
                                     0 off (separate Init3 pass), 1 on, 2 (default)
                                     auto: off when m >= 16 n, else decided on the
                                     device by a one-block probe of 256 rows (on when
                                     their first smaller neighbours are mostly far
                                     from the row's ID, i.e. random vertex IDs; off
                                     for meshes / road-like graphs, whose Init3 chains
                                     the R23 passes shorten).  ecl_cc_get_run_info
                                     reports the decision.  Applies with INIT 3 and STOP_AFTER
                                     != 1 (the Init3 stage then uses the separate pass);
                                     the R23 passes are skipped.  Labels unchanged (R13);
                                     the worklists then hold every row of their degree
                                     range, not only rows with a smaller neighbour.    */
    ECL_CC_OPT_MERGE_FILTER = 20  /* multi-GPU: 1 = ecl_cc_forest_encode,
                                     ecl_cc_merge_encoded and
                                     ecl_cc_finalize treat `parent` as the forest this
                                     handle's most recent run built and use that run's
                                     R21 bitmap (anchor-tree membership proofs) to skip
                                     walks; merge_encoded extends the bitmap with the
                                     vertices it joins to the anchor's tree.  0 (default)
                                     = no such assumption.                             */,
    ECL_CC_OPT_VEC = 21           /* 1 = hook_warp and hook_block stream the adjacency
                                     as aligned 16-byte quads (R31; used when
                                     nlist is 16-byte aligned and m < 2^33, else
                                     four-byte loads), 2 (default) = hook_warp only and
                                     only with int32 offsets (quads help its multi-row
                                     rounds, not the hubs' single-row rounds; measured
                                     slower with int64 offsets), 0 = four-byte loads
                                     everywhere.  Labels unchanged.                    */,
    ECL_CC_OPT_FUSED = 22         /* R33: the whole path as ONE cooperative
                                     launch (grid barriers between init, the R23
                                     passes, the three hook kernels and finalize):
                                     0 off, 1 on, 2 (default) for graphs with at most
                                     2^20 rows and 2^22 entries.  Not used by
                                     ecl_cc_run_rows or with ECL_CC_OPT_TIMING (no
                                     per-phase events inside one kernel); the kernel
                                     ORDER option does not apply to it.  Labels
                                     unchanged.                                        */
} ecl_cc_option;
ECL_CC_API ecl_cc_status ecl_cc_set_option(ecl_cc_handle h, int option, int64_t value);

/* Debug: copy the worklist of the most recent run (device->device, synchronises).
 * front receives the warp-bin vertices, back the block-bin vertices (unordered sets);
 * *nfront / *nback receive the counts.  Either buffer may be NULL to query counts only. */
ECL_CC_API ecl_cc_status ecl_cc_get_worklist(ecl_cc_handle h, int32_t *front, int64_t *nfront,
                                  int32_t *back, int64_t *nback);

/* Debug counters, only non-zero in the ECL_CC_STATS build (libecl_cc_stats.so):
 * [0] successful hook CASes, [1] failed hook CASes, [2] find_repres steps,
 * [3] path-halving stores.  Synchronises; counters reset at the start of every run. */
ECL_CC_API ecl_cc_status ecl_cc_get_stats(ecl_cc_handle h, int64_t out[4]);

/* The same counters and the edge-filter breakdown of the batched hook path (count <= 16):
 * [4] entries with v > u (Fig. 6 line 1), [5] of those skipped as same-tree by R15
 * (u == parent[v] or u == v_rep), [6] checked against the R21 bitmap, [7] skipped by the
 * bitmap, [8] hop-1 gathers parent[u], [9] hop-2 gathers, [10] bitmap marks,
 * [11] non-empty edge windows (process_window calls), [12] edges deferred to the R22
 * hook queue, and the path lengths of the find_repres walks (Table 4 analogue,
 * P:L329-L337; length = parent pointers followed from the walk's start to where it
 * stopped — the root, or v_rep under the early exit; walks from a root are not counted,
 * nor edges the R21/R22 probe settles without a walk): [13] sum of lengths, [14] walks,
 * [15] maximum length. */
ECL_CC_API ecl_cc_status ecl_cc_get_stats_ex(ecl_cc_handle h, int64_t *out, int count);

/* Debug: what the most recent run decided (synchronises it); count <= 4:
 * [0] 1 if Init3 ran inside the hook kernels (R28), [1] 1 if the R23 depth probe found a
 * deep forest (the pointer-jumping passes ran), [2] 1 if the R21 bitmap filter was on,
 * [3] the R21 anchor vertex (-1 if none), [4] 1 if the run took the R33 single-launch
 * path.  count <= 5. */
ECL_CC_API ecl_cc_status ecl_cc_get_run_info(ecl_cc_handle h, int64_t *out, int count);

/* Debug: the handle's R21 anchor-tree membership bitmap (R21) as left by the
 * most recent run — *bits (device, NULL if no run used the filter), *words (uint32 words
 * allocated, >= (n+31)/32), *anchor (the anchor vertex X, -1 if none).  A set bit v is a
 * proof that v is in X's tree.  Synchronises the last run's stream. */
ECL_CC_API ecl_cc_status ecl_cc_get_filter(ecl_cc_handle h, const uint32_t **bits,
                                           int64_t *words, int32_t *anchor);

/* Per-phase device time of the most recent full run with ECL_CC_OPT_TIMING set
 * (synchronises on it): ms[0] init_bin (incl. the counter memset), ms[1] hook_thread,
 * ms[2] hook_warp (worklist front), ms[3] hook_block (worklist back), ms[4] finalize.
 * With ECL_CC_OPT_ORDER 2 each hook kernel's span is measured on its own stream; the
 * spans overlap, so ms[1] + ms[2] + ms[3] exceeds the hook phase of the run. */
ECL_CC_API ecl_cc_status ecl_cc_get_timing(ecl_cc_handle h, float ms[5]);

/* 1 if this build counts statistics (ECL_CC_STATS), else 0. */
ECL_CC_API int ecl_cc_stats_enabled(void);

ECL_CC_API const char *ecl_cc_status_string(ecl_cc_status s);
ECL_CC_API const char *ecl_cc_last_error(ecl_cc_handle h);
ECL_CC_API const char *ecl_cc_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ECL_CC_H */
