/*
 * glp.h -- C ABI of libglp.so, the B200-native hot path of GLP
 *          (Ye, Li, He, Li, Sun, "GPU-Accelerated Graph Label Propagation for
 *          Real-Time Fraud Detection", SIGMOD '21).
 *
 * Citations: [P:n §s] = line n of the paper text, section s.
 * Readings R1..R18 (where the paper is silent/garbled) are listed in DESIGN.md.
 *
 * What the library computes (one LP run, §2.1 [P:68] and §3.1
 * [P:97-119]):  every vertex starts with a label (PickLabel [P:99, P:109]);
 * each bulk-synchronous iteration [P:48] every active vertex gathers the labels
 * of its CSR neighbours (LoadNeighbor [P:110]), counts them and takes the label
 * of maximum score (LabelScore [P:111]; most frequent label = MFL [P:68]) with
 * the smallest label winning ties (R4), writing it to Lnext [P:143]
 * (UpdateVertex [P:101, P:112]).  Three fixed variants ([P:116-119], [P:33]):
 *   CLASSIC  score(l) = k(l)                                   [P:118]
 *   SEEDED   CLASSIC from black-listed seeds; non-seeds start UNLABELED (-1),
 *            -1 neighbours do not vote, seeds never change     [P:33, P:335], R12
 *   LLP      score(l) = k - gamma * (V(l) - k), in double, V(l) = number of
 *            vertices holding l at the previous iteration      [P:119], R10, R11
 * Only vertices with a neighbour that changed in the previous iteration are
 * recomputed (active-vertex frontier; exact for CLASSIC/SEEDED, R9).
 *
 * Conventions for every entry point:
 *  - returns glp_status; never aborts or throws across the ABI; on error the
 *    thread-local glp_last_error() holds a one-line message and the graph is
 *    left in its previous state;
 *  - every pointer argument is either a HOST pointer or a DEVICE pointer as
 *    documented; "borrowed" means the caller keeps ownership and must keep the
 *    memory alive and unmodified for the graph's lifetime;
 *  - all work runs on the graph's CUDA stream; calls are host-synchronous on
 *    return unless stated otherwise.
 *  - distinct graphs may be used from distinct threads; one graph is not
 *    thread-safe.
 */
#ifndef GLP_H_
#define GLP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct glp_graph glp_graph; /* opaque; owned by the library */

typedef enum {
  GLP_OK = 0,
  GLP_ERR_INVALID_ARGUMENT = 1, /* bad scalar / pointer / seed / params      */
  GLP_ERR_INVALID_GRAPH = 2,    /* malformed CSR (validate=1)                */
  GLP_ERR_OUT_OF_MEMORY = 3,    /* device or host allocation failed          */
  GLP_ERR_CUDA = 4,             /* CUDA runtime error (message has the name)  */
  GLP_ERR_NCCL = 5,             /* NCCL error (multi-GPU)                    */
  GLP_ERR_UNSUPPORTED = 6,      /* no CUDA device / non-sm_100 device         */
  GLP_ERR_STATE = 7             /* call out of order (e.g. labels before run) */
} glp_status;

typedef enum {
  GLP_VARIANT_CLASSIC = 0,
  GLP_VARIANT_SEEDED = 1,
  GLP_VARIANT_LLP = 2,
  GLP_VARIANT_SLP = 3  /* speaker-listener LP [P:120]: each vertex keeps up to
                          slp_max_labels candidate labels; per iteration its
                          speaker label (the most frequent candidate) is what
                          the neighbours count, and the MFL heard joins the
                          candidates (R19).  Runs exactly max_iters iterations;
                          glp_labels_get returns the speaker labels,
                          glp_slp_memory_get the candidates                   */
} glp_variant;

typedef enum {
  GLP_STOP_MAX_ITERS = 0,   /* ran max_iters iterations                        */
  GLP_STOP_FIXED_POINT = 1, /* an iteration changed no label (it is counted)   */
  GLP_STOP_TWO_CYCLE = 2    /* L_t == L_{t-2} with changes (R8)                */
} glp_stop_reason;

#define GLP_UNLABELED (-1)

/* CSR of the OWNED rows [v_begin, v_end) with GLOBAL column ids
 * ("Graph" structure in CSR format [P:97]; row v lists N(v) [P:68], R1).
 * Single GPU: v_begin = 0, v_end = n_global. */
typedef struct {
  int64_t n_global;            /* number of vertices, 0 <= n_global < 2^31    */
  int64_t v_begin, v_end;      /* owned row range, 0 <= v_begin <= v_end <= n */
  int64_t nnz_local;           /* arcs of the owned rows                       */
  const int64_t *row_offsets;  /* v_end-v_begin+1 entries, [0]==0,
                                  last==nnz_local, non-decreasing              */
  const int32_t *col_idx;      /* nnz_local entries in [0, n_global); a row
                                  may list a neighbour twice (two votes, R3)   */
  int32_t on_device;           /* 1: device pointers, BORROWED for the graph's
                                     lifetime (e.g. torch tensors); their
                                     contents must be complete when create is
                                     called, or be produced on the stream
                                     passed in glp_dist.cuda_stream;
                                  0: host pointers, copied during create       */
  int32_t symmetric;           /* 1: caller asserts the global graph is
                                  symmetric (u in N(v) <=> v in N(u)); the
                                  frontier push then walks the CSR itself.
                                  0: the frontier is disabled (full sweeps)    */
  const uint32_t *weights;     /* NULL, or nnz_local arc weights in [1, 2^31)
                                  (LoadNeighbor's weight [P:110, P:145]): a
                                  label's frequency is the SUM of the weights
                                  of the arcs carrying it (weighted LP,
                                  CLASSIC / SEEDED; LLP -> UNSUPPORTED).
                                  Same memory space as col_idx; copied into
                                  the library's layout during create.  Every
                                  row's weight total must be < 2^31
                                  (GLP_ERR_INVALID_GRAPH otherwise)            */
} glp_csr;

/* In-process rank group: P ranks (P graphs, one host thread each) in ONE
 * process exchange labels through each other's device buffers instead of NCCL
 * (glp_local_group_create).  Used to run the partitioned path on one GPU. */
typedef struct glp_local_group glp_local_group;

/* Multi-GPU placement (1-D vertex-range partition, one process per GPU, or P
 * ranks of one local group).  NULL = single GPU, device = current device.
 * Creating and running a partitioned graph are COLLECTIVE: every rank calls
 * glp_graph_create / glp_run with the same arguments (except its own rows),
 * concurrently (separate processes or separate host threads). */
typedef struct {
  int32_t rank, nranks;        /* this process's rank and the world size      */
  int32_t device;              /* CUDA ordinal for this rank                   */
  const void *nccl_unique_id;  /* 128 bytes from glp_nccl_unique_id() on rank 0,
                                  broadcast by the caller; NULL if nranks == 1
                                  or local_group is set                        */
  void *cuda_stream;           /* cudaStream_t to run on, or NULL = a stream
                                  owned by the library                         */
  glp_local_group *local_group;/* non-NULL: exchange through this in-process
                                  group (borrowed; must outlive the graph)     */
} glp_dist;

/* Run parameters.  Zero-initialise, set struct_size = sizeof(glp_params),
 * then override fields; NULL params = all defaults. */
typedef struct {
  uint32_t struct_size;        /* must equal sizeof(glp_params)                */
  double gamma;                /* LLP gamma, finite and >= 0 (default 0)       */
  int32_t frontier;            /* -1 auto (default), 0 always full sweeps,
                                  1 force frontier (not allowed for LLP)       */
  int32_t stop_on_2cycle;      /* 1 (default) / 0                              */
  int32_t validate;            /* create-time CSR validation, default 1        */
  int32_t profile;             /* 1: time each kernel with CUDA events
                                  (glp_kernel_stats); default 0                */
  int32_t dense_divisor;       /* go dense when sum_{changed} deg > nnz/this;
                                  0 = default (4)                              */
  int32_t debug_pred_cap;      /* testing only: clamp each row's predicted
                                  distinct-label count (forces the overflow /
                                  re-queue paths; results are unchanged); 0 off */
  int32_t llp_hist;            /* LLP label histogram with nranks > 1:
                                  0 default (= 2), 1 replicated (every rank
                                  counts all n labels after the label
                                  all-gather), 2 sharded (each rank counts its
                                  own rows, the counts are all-reduced, and the
                                  (label, V) pairs of the owned rows are
                                  all-gathered instead of the labels)          */
  int32_t host_arcs;           /* create only.  1: CPU-GPU hybrid mode for
                                  graphs whose arcs exceed device memory
                                  [P:103]: the library's arc array lives in
                                  pinned, mapped HOST memory and every
                                  iteration streams it over the host link;
                                  labels, counters and tables stay on the
                                  device.  Needs a host CSR (on_device = 0),
                                  whose col_idx is registered (pinned) during
                                  create.  Results are identical.  Default 0 */
  int32_t tail_cms;            /* 1: L rows (long, many labels) count with the
                                  paper's HT + Count-Min Sketch single scan
                                  [P:132-182 §4.1]; the HT's best is taken
                                  only when it beats every sketch estimate
                                  strictly, else the row is recounted exactly
                                  (results never change).  Default 0 */
  int32_t cms_ht_slots;        /* tail_cms: HT capacity h (power of two <=
                                  8192; 0 = 8192).  Testing / analysis        */
  int32_t cms_depth;           /* tail_cms: sketch rows d (1..8, width =
                                  8192 / d; 0 = 4)                             */
  int32_t slp_max_labels;      /* SLP: candidate labels per vertex K, 1..16
                                  (0 = 5 [P:270])                              */
  double slp_threshold;        /* SLP: after iteration t a candidate whose count
                                  is < slp_threshold * (t + 1) is dropped
                                  (never the most frequent one); >= 0, default 0 */
  int32_t sparse_exchange;     /* nranks > 1, CLASSIC / SEEDED (§8(f)1): replace
                                  the label all-gather by an exchange of the
                                  changed vertices' (id, label) pairs of t-1
                                  and t.  -1 auto (default: when changed at
                                  t-1 < n / (4 nranks)), 0 never, 1 always     */
} glp_params;

typedef struct {
  int32_t iterations;          /* executed iterations t                         */
  int32_t stop_reason;         /* glp_stop_reason                               */
  int64_t changed_last;        /* changed_t of the last iteration               */
  int64_t arcs_processed;      /* sum over iterations of scanned arcs           */
  double elapsed_ms;           /* device time of the run (CUDA events)          */
  int64_t kernel_launches;     /* CUDA kernels the run launched                 */
} glp_run_info;

/* Per-iteration statistics of the last run (host copies). */
typedef struct {
  int64_t changed;             /* #{v : L_t[v] != L_{t-1}[v]}                   */
  int64_t d2;                  /* #{v : L_t[v] != L_{t-2}[v]} (t >= 2)          */
  int64_t active_vertices;     /* vertices scanned (superset of the frontier)   */
  int64_t active_arcs;         /* arcs scanned                                  */
  int32_t dense;               /* 1 if the iteration was a full sweep           */
  int32_t exchange;            /* nranks > 1: 1 label all-gather, 2 sparse
                                  (changed pairs), 3 (label, V) all-gather     */
  double ms;                   /* device time of the iteration                  */
  int64_t cms_rows;            /* tail_cms: L rows whose scan used the sketch   */
  int64_t cms_rescans;         /* ... of those, rows rescanned for estimates    */
  int64_t cms_fallbacks;       /* ... of those, rows recounted exactly          */
} glp_iter_stat;

/* Per-kernel totals of the last run with params.profile = 1. */
typedef struct {
  char name[32];
  int64_t launches;
  double ms;                   /* summed CUDA-event duration                    */
  double bytes;                /* algorithmic bytes       */
  double arcs;                 /* arcs processed                                */
} glp_kernel_stat;

/* In-process group of nranks ranks (1 <= nranks <= 16); owned by the caller,
 * destroyed after every graph that uses it.  A rank that fails inside a
 * collective aborts the group: the other ranks' calls then return
 * GLP_ERR_STATE instead of waiting (and the group cannot be reused). */
glp_status glp_local_group_create(int32_t nranks, glp_local_group **out);
glp_status glp_local_group_destroy(glp_local_group *grp); /* NULL-safe */

/* 128-byte NCCL unique id; rank 0 calls it and broadcasts the bytes. */
glp_status glp_nccl_unique_id(uint8_t out[128]);

/* Row ranges for nranks: bounds_out[r] = first row of rank r, [nranks] = n.
 * edge_balanced = 0: equal vertex counts; 1: equal arc counts (row_offsets of
 * the whole graph, host).  row_offsets_host may be NULL when edge_balanced = 0. */
glp_status glp_partition(const int64_t *row_offsets_host, int64_t n, int32_t nranks,
                         int32_t edge_balanced, int64_t *bounds_out);

/* Build the device graph: copy (on_device=0) or borrow (on_device=1) the CSR,
 * validate it (if params->validate), bin vertices by degree (low <= 32 packed
 * warps [P:227-234 §4.2]; mid; high/huge block-per-vertex [P:132 §4.1]),
 * allocate label buffers and scratch.  params may be NULL (defaults). */
glp_status glp_graph_create(const glp_csr *csr, const glp_dist *dist, const glp_params *params,
                            glp_graph **out);

/* Run LP from PickLabel: CLASSIC/LLP start from L[v] = v [P:68]; SEEDED from
 * L[s] = s for s in seeds, else -1 (R12).  seeds: HOST array of n_seeds global
 * ids in [0, n_global) (duplicates ignored); must be NULL/0 unless SEEDED.
 * Stops at a fixed point, a two-cycle (if stop_on_2cycle) or max_iters >= 0.
 * info may be NULL.  Labels stay on the device (glp_labels_get). */
glp_status glp_run(glp_graph *g, glp_variant variant, int32_t max_iters, const int32_t *seeds,
                   int64_t n_seeds, const glp_params *params, glp_run_info *info);

/* SLP candidates of the last SLP run, in original vertex order, for this
 * rank's rows [v_begin, v_end): labels_out / counts_out hold K entries per
 * vertex (K = the run's slp_max_labels; -1 / 0 = empty slot), out_len >=
 * (v_end - v_begin) * K; out_on_device as for glp_labels_get. */
glp_status glp_slp_memory_get(const glp_graph *g, int32_t *labels_out, int32_t *counts_out, int64_t out_len,
                              int32_t out_on_device);

/* Copy all n_global labels of the last run into out (out_on_device = 0: host
 * buffer, 1: device buffer), out_len >= n_global. */
glp_status glp_labels_get(const glp_graph *g, int32_t *out, int64_t out_len,
                          int32_t out_on_device);

/* Copy up to max_entries per-iteration stats of the last run; *n_out = count. */
glp_status glp_iter_stats(const glp_graph *g, glp_iter_stat *out, int32_t max_entries,
                          int32_t *n_out);

/* Copy up to max_entries per-kernel stats of the last profiled run. */
glp_status glp_kernel_stats(const glp_graph *g, glp_kernel_stat *out, int32_t max_entries,
                            int32_t *n_out);

/* Graph facts: n_global, nnz_local, and vertex/arc counts of the degree bins
 * (out[0..]: n, nnz, then for bins {isolated, low, mid, high, huge}:
 * vertices, arcs), at most max_entries values written. */
glp_status glp_graph_info(const glp_graph *g, int64_t *out, int32_t max_entries);

glp_status glp_graph_destroy(glp_graph *g); /* NULL-safe */

/* ABI self-check for bindings: out[0..5] = sizeof(glp_csr), sizeof(glp_dist),
 * sizeof(glp_params), sizeof(glp_run_info), sizeof(glp_iter_stat),
 * sizeof(glp_kernel_stat) (at most max_entries written).  Host only. */
glp_status glp_struct_sizes(int64_t *out, int32_t max_entries);

const char *glp_last_error(void);  /* thread-local, never NULL */
const char *glp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GLP_H_ */
