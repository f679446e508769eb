/*
 * nulpa.h -- C ABI of the B200-native nu-LPA hot path.
 *
 * nu-LPA (PAPER.md, Sahu): asynchronous label propagation with a per-vertex
 * open-addressing hashtable (float32 values, hybrid quadratic-double
 * probing), the Pick-Less rule every rho iterations, vertex pruning, and a
 * tolerance-based stop (Algorithm 1; Algorithm 2,
 * PAPER.md:368-406), plus modularity (Eq. 1).
 *
 * Conventions for every entry point
 *   - Return value: NULPA_OK (0) on success, a positive NULPA_E* code on
 *     failure; nulpa_last_error() then describes the failure (thread-local
 *     string owned by the library, valid until the next call on the thread).
 *     No entry point aborts the process or falls back to the CPU.
 *   - Graphs are CSR: offsets[n_rows+1] int64 (offsets[0]
 *     must be 0), indices[M] int32 global vertex IDs in [0, n_global),
 *     weights[M] float32 >= 0 or NULL for unit weights.
 *     Undirected graphs store both directions.  Self-loops are skipped when
 *     accumulating.
 *   - `memkind` says where a pointer lives: NULPA_MEM_HOST (pageable or
 *     pinned host memory) or NULPA_MEM_DEVICE (CUDA device memory on the
 *     current device).
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  All device work of a handle is enqueued on the stream given
 *     to nulpa_create; calls that return host results synchronise it.
 *   - Labels are int32 community IDs; after nulpa_run they are vertex IDs.
 */
#ifndef NULPA_H
#define NULPA_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define NULPA_OK 0
#define NULPA_EINVAL 1   /* bad argument (null pointer, size, range)        */
#define NULPA_ECUDA 2    /* a CUDA runtime call or kernel launch failed      */
#define NULPA_ENOMEM 3   /* device or pinned-host allocation failed          */
#define NULPA_ESTATE 4   /* call not valid in the handle's current state     */

#define NULPA_MEM_HOST 0
#define NULPA_MEM_DEVICE 1

#define NULPA_ASYNC 0    /* production mode: one label vector, in-place writes (PAPER.md:173 (1)) */
#define NULPA_SYNC 1     /* deterministic Jacobi mode: reads previous sweep's labels (north star) */

typedef struct nulpa_graph nulpa_graph;

/* Parameters of nulpa_run / nulpa_sweep.  nulpa_default_params() fills the
 * paper's values: tau = 0.05, 20 iterations, Pick-Less every 4 iterations
 * (PAPER.md:173), asynchronous mode, B200 switch degrees. */
typedef struct nulpa_params {
    double tolerance;            /* tau: stop when not PL and dN/N < tau      */
    int32_t max_iterations;      /* MAX_ITERATIONS                            */
    int32_t pickless_period;     /* rho: PL when l mod rho == 0; <= 0 disables PL (R10)       */
    int32_t mode;                /* NULPA_ASYNC or NULPA_SYNC                                 */
    int32_t switch_degree;       /* degree >= this -> warp-per-vertex instead of thread-per-vertex
                                    (the paper's SWITCH_DEGREE; B200 default 16) */
    int32_t block_degree;        /* degree >= this -> block-per-vertex (shared-memory table)  */
    int32_t giant_degree;        /* degree >= this -> multi-CTA, global-memory table          */
    int32_t reset;               /* 1: C <- [0..N) and all vertices unprocessed first;
                                    0: continue from the current labels / flags               */
    int32_t timing;              /* 1: time every kernel with CUDA events (nulpa_get_stats)   */
    int32_t tie_rule;            /* order among labels of equal weight (R6): must be
                                    NULPA_TIE_SMALLEST (0) -- the smallest label wins (north
                                    star "ties broken by smallest label"; "the
                                    first label with the highest associated weight").  Any other
                                    value is rejected with NULPA_EINVAL                          */
    int32_t bin_order;           /* 4 (default, auto): 3 if the warp bin holds >= 2/3 of the
                                    CSR entries, else 1.  3: thread bin, then the warp bin on a
                                    high-priority stream and block + giant on a low-priority
                                    stream released after the warp-bin frontier (they fill the
                                    warp bin's tail); 1: thread, warp, block, giant bins in
                                    that order within a sweep (hubs last); 0: giant, block,
                                    warp, thread; 2: block + giant on a second stream,
                                    concurrent with thread + warp                             */
    int32_t wide_degree;         /* within the block bin: degree < this -> one warp per vertex
                                    with a warp-private 1023-slot shared-memory table (load
                                    <= 1/2 at 512); degree >= this -> one CTA per vertex.
                                    Range [1, 1024] (distinct labels <= D <= 1023 = p1, so R5's
                                    linear continuation always finds a slot); <= block_degree
                                    sends the whole bin to the CTA kernel.  B200 default 512    */
    int32_t first_sweep_block;   /* warp-bin schedule of the first sweep after a reset.
                                    0 (default): each warp owns one contiguous range of the
                                    bin's 32-vertex record groups and walks it in ID order;
                                    warps that run dry steal the far half of the most-loaded
                                    of 32 sampled ranges (labels propagate along ID order within
                                    a run as in the sequential Algorithm 1 -- modularity -- and
                                    the end of the sweep is balanced; DESIGN.md "Quality
                                    notes").  1: static strided; > 1: guided chunks of up to
                                    this many groups from a global counter.  Range [0, 1024]   */
    int32_t sweep_block;         /* the same for every later sweep; default 4 (guided)          */
    int32_t device_loop;         /* 1 (default): when timing == 0, nulpa_run launches sweep 0 and
                                    then ONE CUDA graph whose conditional while node runs sweeps
                                    1.. and Algorithm 1's stop test on the device
                                    -- no host synchronisation per iteration; the graph is built
                                    once per handle and parameter set, from the handle's second
                                    nulpa_run on (the first run of a handle takes the host loop:
                                    building a graph costs more than one run of a small graph
                                    saves).  0 (or timing == 1): the host loop, one
                                    synchronisation per iteration                              */
} nulpa_params;

#define NULPA_TIE_SMALLEST 0

/* Statistics of the last nulpa_run (or accumulated nulpa_sweep calls since
 * the last reset).  Bins: 0 thread, 1 warp, 2 block, 3 giant. */
typedef struct nulpa_stats {
    int32_t iterations;                /* iterations performed by the last nulpa_run   */
    int32_t converged;                 /* 1 if stopped by the tolerance test           */
    int64_t changed[64];               /* dN of iteration l (l < 64)                   */
    int64_t vertices_processed[4];     /* per bin, summed over iterations              */
    int64_t edges_scanned[4];          /* per bin, summed over iterations              */
    int64_t vertices_changed[4];       /* per bin, summed over iterations              */
    int64_t changed_edges[4];          /* per bin: CSR entries of changed vertices      */
    double kernel_ms[4];               /* per bin, summed (timing=1 only)              */
    int32_t launches[4];               /* kernel launches per bin                      */
    int32_t other_launches;            /* init / copy / bookkeeping kernels            */
    int64_t bin_vertices[4];           /* vertices in each degree bin                  */
    int64_t bin_edges[4];              /* CSR entries of the vertices in each bin      */
    double run_ms;                     /* wall time of nulpa_run on the stream (events) */
    /* per iteration l < 64 and bin b (the totals above split by iteration):  */
    double iter_kernel_ms[64][4];      /* bin b's event span in iteration l (timing=1)  */
    int64_t iter_processed[64][4];
    int64_t iter_edges[64][4];
    int64_t iter_changed[64][4];
    int64_t iter_changed_edges[64][4];
} nulpa_stats;

void nulpa_default_params(nulpa_params *p);

/* Create a handle over a CSR graph or a row shard of one.
 *   offsets  : n_rows+1 int64 prefix sums into indices/weights (offsets[0]==0)
 *   indices  : offsets[n_rows] int32 neighbour IDs (global, < n_global)
 *   weights  : offsets[n_rows] float32 (>= 0, R12) or NULL for unit weights
 *   n_rows   : rows in this CSR (= vertices this handle sweeps)
 *   n_global : vertices of the whole graph (length of the label array);
 *              single-GPU: n_global == n_rows
 *   row_begin: global ID of row 0 (shards: rows are vertices
 *              [row_begin, row_begin+n_rows)); single-GPU: 0
 *   memkind  : where offsets/indices/weights live.  DEVICE arrays are
 *              BORROWED (the caller keeps them alive and unchanged until
 *              nulpa_destroy); HOST arrays are copied to device memory owned
 *              by the handle (copy enqueued on `stream`; the host arrays may
 *              be reused once nulpa_create returns).
 *   stream   : cudaStream_t for all work of this handle.
 * Errors: NULPA_EINVAL for null/inconsistent sizes, offsets[0] != 0, or any
 * weight that is negative, NaN or infinite (R12: one device pass checks
 * them); NULPA_ENOMEM / NULPA_ECUDA from allocation / copies.
 * Builds the degree-binned frontier (row a1) with the default switch degrees;
 * nulpa_run rebuilds it if other switch degrees are requested.
 * Labels start as C = [0..n_global), all vertices unprocessed. */
int nulpa_create(const int64_t *offsets, const int32_t *indices, const float *weights,
                 int64_t n_rows, int64_t n_global, int64_t row_begin, int memkind,
                 void *stream, nulpa_graph **out);

/* Use caller-owned device buffers for the label vector (n_global int32) and
 * the "unprocessed" flags (n_global uint8, nonzero = unprocessed) instead of
 * the handle's own (multi-GPU driver: the replicated label array is a torch
 * tensor exchanged by NCCL).  Their contents are adopted as the current
 * state.  Borrowed until nulpa_destroy. */
int nulpa_bind_state(nulpa_graph *g, int32_t *labels_device, uint8_t *flags_device);

/* Run Algorithm 1's lpa() loop with `params` (NULL =
 * defaults) and fill *stats (may be NULL).  With params->device_loop (and no
 * timing) the stop test runs on the device and the stream is synchronised
 * once at the end; otherwise once per iteration (the tolerance test then
 * needs dN on the host). */
int nulpa_run(nulpa_graph *g, const nulpa_params *params, nulpa_stats *stats);

/* One lpaMove over this handle's rows with Pick-Less on
 * or off; *changed receives dN (may be NULL: then the call does not
 * synchronise).  params supplies mode and switch degrees (NULL = defaults). */
int nulpa_sweep(nulpa_graph *g, int pickless, const nulpa_params *params, int64_t *changed);

/* Reset to C = [0..n_global), all unprocessed. */
int nulpa_reset(nulpa_graph *g);

/* Copy the current labels (n_global int32) to `out` in `memkind` memory. */
int nulpa_labels(nulpa_graph *g, int32_t *out, int memkind);

/* Overwrite the labels (n_global int32 from `in` in `memkind` memory) and
 * the unprocessed flags (n_global uint8, or NULL = all unprocessed).
 * NULPA_EINVAL (state unchanged) if any label is outside [0, n_global). */
int nulpa_set_labels(nulpa_graph *g, const int32_t *in, const uint8_t *flags, int memkind);

/* Copy the unprocessed flags (n_global uint8) to `out`. */
int nulpa_flags(nulpa_graph *g, uint8_t *out, int memkind);

/* Modularity Q of `labels` (n_global int32 in [0, n_global), memkind; NULL =
 * the handle's current labels), Eq. 1 second form (R11), float64
 * accumulation.  Requires a whole graph (n_rows == n_global).  NULPA_EINVAL
 * if any label is outside [0, n_global) (labels index the community sums). */
int nulpa_modularity(nulpa_graph *g, const int32_t *labels, int memkind, double *q);

/* Shard pieces of the modularity for the multi-GPU driver: adds this
 * shard's intra-community weight to *sigma_intra, its total weight to
 * *two_m, and K_i into Sigma_device[labels[i]] (n_global float64, device). */
int nulpa_modularity_partial(nulpa_graph *g, const int32_t *labels_device, double *sigma_intra,
                             double *two_m, double *Sigma_device);
/* Q = sigma_intra/two_m - sum_c (Sigma_c/two_m)^2 over a device Sigma. */
int nulpa_modularity_finish(nulpa_graph *g, const double *Sigma_device, double sigma_intra,
                            double two_m, double *q);

/* Multi-GPU exchange primitives (distributed.py; the bulk-synchronous
 * label / mark exchange after every lpaMove of a row shard, north star
 * "changed labels are exchanged per iteration").  All pointers are device
 * memory; work is enqueued on the handle's stream.
 *
 * nulpa_pack_changed: for every row r of this shard whose current label
 * differs from prev_device[r] (the shard's labels saved before the sweep,
 * n_rows int32), write one pair (vertex << 32) | label into pairs_device
 * (capacity n_rows int64; order arbitrary); *count = pairs written
 * (synchronises the stream). */
int nulpa_pack_changed(nulpa_graph *g, const int32_t *prev_device, long long *pairs_device, int64_t *count);
/* Apply n pairs to the label vector (pairs < 0 are padding, skipped). */
int nulpa_apply_pairs(nulpa_graph *g, const long long *pairs_device, int64_t n);
/* Pack the unprocessed flags of every rank's row range q = [bounds[q],
 * bounds[q+1]) (bounds_device: P+1 int64) into bits_device[q*words ..]
 * (words uint32 per range, bit t of word w = flag of row bounds[q]+32w+t),
 * then clear the flags outside this shard's rows. */
int nulpa_pack_flag_bits(nulpa_graph *g, const int64_t *bounds_device, int P, int64_t words, uint32_t *bits_device);
/* This shard's flags = OR over P received bitmaps of its own range
 * (bits_device: P*words uint32, words*32 >= n_rows). */
int nulpa_or_flag_bits(nulpa_graph *g, const uint32_t *bits_device, int P, int64_t words);

int nulpa_get_stats(nulpa_graph *g, nulpa_stats *out);

/* Return the device memory that destroyed handles left in the library's
 * stream-ordered pool on the current device to the driver.  Handles keep
 * their memory in a per-device pool that retains up to 48 GB after
 * nulpa_destroy (so create/destroy cycles of the same size reuse it instead
 * of paying cudaMalloc/cudaFree of the CSR copy); call this before handing
 * the memory to another allocator.  Live handles are unaffected. */
int nulpa_release_memory(void);

/* Device pointers of the current label / flag vectors (for zero-copy
 * wrapping by the binding).  Valid until the next nulpa_* call. */
int nulpa_state_pointers(nulpa_graph *g, int32_t **labels_device, uint8_t **flags_device);

int nulpa_destroy(nulpa_graph *g);

const char *nulpa_last_error(void);

/* Library version string ("nulpa <semver> sm_100a"). */
const char *nulpa_version(void);

#ifdef __cplusplus
}
#endif
#endif /* NULPA_H */
