/*
 * rap.h — C ABI of the B200-native RAP fused DLRM input-preprocessing library
 * (librap.so).  Paper: Wang et al., "RAP: Resource-aware Automated GPU Sharing
 * for Multi-GPU Recommendation Model Training and Input Preprocessing",
 * ASPLOS '24 (PAPER.md, cited L<line>).
 *
 * The calls follow the paper's problem statement: a plan is built once from
 * "the computational graph of data preprocessing" plus the hardware and the
 * co-running budget (L840-846 §4); each batch, one call turns the raw batch
 * into the "input tensors" consumed by training (L466-469 §2.1); the budget
 * can be changed between batches so the fused kernel fits the remaining GPU
 * capacity (resource-aware sharding, L1351-1366 §6.2).
 *
 * Conventions (all entry points):
 *  - Plain C types only; every pointer documented as HOST or DEVICE.
 *  - Ownership: rap_plan_create deep-copies the graph and parameters (the
 *    caller may free them on return).  The plan owns its device program blob,
 *    descriptor table, scan-state and staging workspaces.  The caller owns
 *    every raw-batch and output buffer and the CUDA stream.
 *  - Errors: functions return rap_status; rap_last_error() gives a
 *    thread-local human-readable detail of the last failure.  Asynchronous
 *    device faults surface through the CUDA stream as usual.
 *  - Concurrency: a plan is not re-entrant — use one plan per stream that
 *    runs concurrently.  Results never depend on the SM budget.
 *  - Operator semantics: DESIGN.md §3 (readings R1-R20 of Table 1).
 */
#ifndef RAP_H
#define RAP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  RAP_OK = 0,
  RAP_ERR_INVALID_ARGUMENT = 1, /* null pointer, negative size, bad param index, bad budget */
  RAP_ERR_INVALID_GRAPH = 2,    /* cycle, bad reference, unknown op, type mismatch (R20) */
  RAP_ERR_INVALID_PARAM = 3,    /* operator parameter out of its domain (R20) */
  RAP_ERR_CAPACITY = 4,         /* output buffer smaller than the host-computed bound */
  RAP_ERR_UNSUPPORTED = 5,      /* valid graph outside what the kernel lowers (nested NGram) */
  RAP_ERR_CUDA = 6,             /* a CUDA runtime call failed */
  RAP_ERR_OUT_OF_MEMORY = 7
} rap_status;

/* Operators of PAPER.md Table 1 (L440-463). */
typedef enum {
  RAP_OP_FILLNULL = 0,   /* L462: "Fill NA/NaN values using the specified value"        (R10) */
  RAP_OP_LOGIT = 1,      /* L446: "Logit transform for normalization"                   (R11) */
  RAP_OP_BOXCOX = 2,     /* L448: "BoxCox transform for normalization"                  (R12) */
  RAP_OP_ONEHOT = 3,     /* L449: "Apply one hot encoding to normalize dense features"  (R9)  */
  RAP_OP_SIGRIDHASH = 4, /* L452: "Compute hash value to normalize list of sparse features" (R1-R3) */
  RAP_OP_BUCKETIZE = 5,  /* L458: "Shard features based on bucket borders"              (R4)  */
  RAP_OP_FIRSTX = 6,     /* L454: "List truncation of sparse features"                  (R5)  */
  RAP_OP_CLAMP = 7,      /* L455: "Clamp the sparse input based on the upper and lower bound" (R6) */
  RAP_OP_NGRAM = 8,      /* L459 + footnote L181-182: n-gram across multiple sparse features (R7) */
  RAP_OP_MAPID = 9       /* L460: "Maps feature IDs to fixed values"                    (R8)  */
} rap_op_type;

/* Node input encoding: a value >= 0 is a node index; raw columns are encoded
 * with these macros (dense column c is an f32 scalar per row, sparse column c
 * an Arrow list<int64>). */
#define RAP_RAW_DENSE(c) (-1 - 2 * (c))
#define RAP_RAW_SPARSE(c) (-2 - 2 * (c))

/* One DAG node (§2.3: a feature's preprocessing is a DAG).
 * HOST memory.  `inputs` has n_inputs entries (1, or 1..8 for NGram);
 * `param` indexes the rap_op_param array passed to rap_plan_create. */
typedef struct {
  int32_t op;            /* rap_op_type */
  int32_t n_inputs;
  const int32_t* inputs; /* node indices or RAP_RAW_* */
  int32_t param;
} rap_node;

/* The whole preprocessing graph.  HOST memory.  Outputs are emitted in this
 * order: Dense nodes as 1 dense column, OneHot nodes as K dense columns, Ids
 * nodes as one jagged sparse feature (R17). */
typedef struct {
  int32_t n_dense_in, n_sparse_in, n_nodes;
  const rap_node* nodes;
  int32_t n_outputs;
  const int32_t* output_nodes;
} rap_graph;

/* Operator parameters.  HOST memory; only the fields of the node's op are
 * read.  `borders` is f32[n_borders] when Bucketize reads a Dense value and
 * int64[n_borders] when it reads an id list. */
typedef struct {
  float f_fill, eps, lambda;
  int64_t i_fill, lo, hi, x, max_value, map_default;
  uint64_t salt;
  int32_t n, k_width, n_borders;
  const void* borders;
  int64_t map_size;
  const int64_t* map_keys;
  const int64_t* map_vals;
} rap_op_param;

/* One raw columnar batch (Arrow layout: columnar data
 * loaded to the GPU).  The pointer ARRAYS are HOST memory; the column buffers
 * they point to are DEVICE memory for rap_preprocess and HOST memory for
 * rap_preprocess_host.
 *   dense[c]       f32[n_rows]
 *   dense_valid[c] u32 bitmap, bit (b&31) of word b>>5, 1 = valid; the array
 *                  itself or an entry may be NULL = all valid (R19)
 *   sp_offsets[c]  int32[n_rows+1], absolute, non-decreasing (off[0] may be > 0)
 *   sp_values[c]   int64 child values
 *   sp_valid[c]    bitmap as above (NULL = all valid)
 *   sp_nnz         HOST int64[n_sparse_in]: sp_offsets[c][n_rows] - sp_offsets[c][0]
 *                  (used only for the host-side capacity bound and H2D sizes) */
typedef struct {
  int64_t n_rows;
  const float* const* dense;
  const uint32_t* const* dense_valid;
  const int32_t* const* sp_offsets;
  const int64_t* const* sp_values;
  const uint32_t* const* sp_valid;
  const int64_t* sp_nnz;
} rap_raw_batch;

/* Output "input tensors" (R17).  DEVICE memory for rap_preprocess, HOST for
 * rap_preprocess_host.
 *   dense_out  f32[n_rows * dense_ld], row-major, dense_ld >= d_out_cols
 *   lengths    int32[n_sparse_out * n_rows], feature-major
 *   offsets    int64[n_sparse_out * n_rows + 1] (may be NULL when
 *              n_sparse_out == 0; if given, offsets[0] = 0 is written)
 *   values     int64[values_capacity]; values_capacity must be >= the bound
 *              returned by rap_plan_output_shape, else RAP_ERR_CAPACITY. */
typedef struct {
  float* dense_out;
  int64_t dense_ld;
  int32_t* lengths;
  int64_t* offsets;
  int64_t* values;
  int64_t values_capacity;
  int32_t flags;         /* 0, RAP_OUT_CHAIN, RAP_OUT_VALUES_I32 */
  int32_t reserved;
} rap_output;

/* rap_output.flags: a chained launch continues a jagged output that a
 * preceding launch (or rap_jagged_append) on the same stream wrote into the
 * same buffers.  `offsets` then points at the slot holding that running total
 * (the previous piece's last offset, a DEVICE value read when the launch
 * starts, never by the host); every offset this launch writes is that total
 * plus its own exclusive scan and its ids go to values[total ...].  `lengths`
 * points at the first row slot of this launch.  Used to stitch multi-GPU
 * residual pieces. */
#define RAP_OUT_CHAIN 1
/* Cast (Table 1; reading R13): the values are emitted as
 * int32 -- `values` points to int32[values_capacity] and every id is cast by
 * two's-complement truncation ((int32_t)id, torch's .to(torch.int32)).
 * rap_preprocess only (the host-buffer entries and chained launches take
 * int64 values: RAP_ERR_UNSUPPORTED). */
#define RAP_OUT_VALUES_I32 2

struct rap_plan;
typedef struct rap_plan rap_plan;

/* Read-only description of a plan (HOST).  The kernel fields describe the
 * last launch: kernel_last = RAP_KERNEL_TILED or RAP_KERNEL_ROWS; for the
 * row-block kernel rb_row_blocks x rb_feature_groups CTAs of rb_rows rows. */
typedef struct {
  int32_t device, sm_count, sm_budget, ctas_per_sm, threads_per_cta, grid;
  int32_t n_dense_out_cols, n_sparse_out, n_dense_groups, rows_per_dense_desc;
  int32_t max_rows_per_sparse_desc, min_rows_per_sparse_desc;
  int64_t n_descriptors_last, n_launches;
  int64_t smem_bytes;
  int32_t kernel_mode, kernel_last, rows_ctas_per_sm, rows_smem_bytes;
  int32_t rb_row_blocks, rb_feature_groups, rb_rows, rb_memo_slots;
  int64_t partition_uploads;  /* work partitions uploaded (tiled kernel), cumulative */
  int32_t jit_state;          /* generated kernel: 0 not built yet, 1 built, -1 failed (see rap_last_error) */
  int32_t jit_ctas_per_sm;
  double jit_compile_seconds; /* NVRTC compile + load time of the generated kernel */
} rap_plan_info;

/* Which fused kernel rap_preprocess launches.  Both compute
 * the same outputs (R1-R20); they differ in how work maps to threads.
 *   RAP_KERNEL_AUTO  (default) the row-block kernel when the plan fits it
 *                    (<= 64 raw sparse / 32 raw dense columns, <= 1024 sparse
 *                    outputs) and every raw sparse column's mean list length
 *                    in this batch is <= 2 (Criteo-shaped) -- its generated
 *                    form when the batch runs as one feature group -- else
 *                    the tiled kernel
 *   RAP_KERNEL_TILED (feature, 128-row) tiles, element-parallel for long
 *                    multi-hot lists (rap_kernel.cu)
 *   RAP_KERNEL_ROWS  row blocks x feature groups, one row per thread, each
 *                    output interpreted from its record (rap_rows.cu);
 *                    RAP_ERR_UNSUPPORTED if the plan does not fit it
 *   RAP_KERNEL_JIT   the row-block kernel with every output's chain generated
 *                    as straight-line CUDA for this plan and compiled by NVRTC
 *                    for sm_100a on the first launch that uses it (seconds of
 *                    host time, cached per process); batches
 *                    that split the outputs into several feature groups run
 *                    the interpreted form.  If NVRTC fails the plan keeps the
 *                    interpreted form (rap_plan_info.jit_state = -1). */
#define RAP_KERNEL_AUTO 0
#define RAP_KERNEL_TILED 1
#define RAP_KERNEL_ROWS 2
#define RAP_KERNEL_JIT 3

/* Build a plan (the a0 row of DESIGN.md §1): validate the DAG and parameters
 * (R20, same checks and codes as the oracle), lower every output to a device
 * op program, precompute H(salt), sort MapId tables, size the descriptor
 * geometry, query occupancy and set grid = f(sm_budget).  sm_budget in
 * [1, #SMs] (the SMs' worth of CTA slots the kernel may hold, §6.2);
 * 0 = all SMs.  `device` is a CUDA ordinal.  *out receives the plan. */
rap_status rap_plan_create(const rap_graph* graph, const rap_op_param* params, int32_t n_params,
                           int32_t device, int32_t sm_budget, rap_plan** out);

/* Shapes for a batch of n_rows rows.  sp_nnz: HOST int64[n_sparse_in] (may be
 * NULL when n_rows == 0).  Outputs (HOST, any may be NULL): dense output
 * columns, sparse output features, an upper bound on values written. */
rap_status rap_plan_output_shape(const rap_plan* plan, int64_t n_rows, const int64_t* sp_nnz,
                                 int64_t* d_out_cols, int64_t* n_sparse_out, int64_t* values_upper_bound);

/* Enqueue one fused preprocessing launch on `stream` (a cudaStream_t; NULL =
 * legacy default stream).  Device buffers.  No allocation and no host reads
 * of device data.  A batch whose shape (rows, grid, quantised mean list
 * lengths) is new uploads its per-warp work partition (async, pinned); the
 * plan caches 8 shapes and only evicting one synchronises `stream`.  Outputs
 * are valid when the stream reaches this point.
 * CUDA-graph capture: a captured call bakes in its shape's cached partition
 * slot, which is then pinned for the plan's lifetime (later eager calls never
 * overwrite what a replay reads).  A replay must see the same batch shape it
 * was captured with (rows; sp_nnz may vary within the cached shape).  A shape
 * first seen during capture takes a free slot; when none is left (8 shapes
 * cached) the call returns RAP_ERR_UNSUPPORTED instead of evicting -- launch
 * each shape once before capturing. */
rap_status rap_preprocess(rap_plan* plan, const rap_raw_batch* raw, const rap_output* out, void* stream);

/* Same as rap_preprocess with HOST raw and output buffers (pinned memory makes
 * the copies asynchronous): copies the batch into plan-owned device staging,
 * launches, copies dense/lengths/offsets and the values back, and
 * synchronises `stream` before returning.  When every input column is pinned
 * (device-mapped) host memory, one gather kernel reads all of them across
 * PCIe into the staging buffers (one launch instead of a copy per column);
 * otherwise each column is a cudaMemcpyAsync (RAP_H2D_COPIES=1 forces that).  When `values` is pinned host
 * memory, a copy kernel moves exactly offsets[end] ids into it (no host sync,
 * no padding over PCIe); pageable memory receives the first
 * values_upper_bound ids.  Host values beyond offsets[end] are unspecified. */
rap_status rap_preprocess_host(rap_plan* plan, const rap_raw_batch* raw, const rap_output* out, void* stream);

/* rap_preprocess_host without the final synchronisation: H2D copies, the
 * launch and the D2H copies are enqueued on `stream` and the call returns.
 * The host buffers must stay alive and unmodified, and the outputs are valid,
 * once the stream reaches this point.  The plan's device staging is reused by
 * its next call, so use one plan per stream in flight: with two plans on two
 * streams, batch i+1's H2D copies and kernel overlap batch i's D2H copies
 * (inter-batch pipelining, §6.3). */
rap_status rap_preprocess_host_async(rap_plan* plan, const rap_raw_batch* raw, const rap_output* out, void* stream);

/* Change the SM budget for the next rap_preprocess (resource-aware sharding,
 * L1351-1366).  sm_budget in [1, #SMs]; 0 = all SMs. */
rap_status rap_set_budget(rap_plan* plan, int32_t sm_budget);

/* Co-running cost model (§5, L871-879 and L1138-1143):
 * predicted standalone latency P (microseconds) of one rap_preprocess for a
 * batch of n_rows under sm_budget, replacing the paper's XGBoost predictor
 * (L1037-1057) with a structural model of the launch the plan would make:
 * P = t0[kernel] + c[kernel] * (busiest CTA's predicted work) + bytes / BW,
 * its constants fitted on B200.  sp_nnz as in
 * rap_plan_output_shape. */
rap_status rap_predict_latency_us(const rap_plan* plan, int64_t n_rows, const int64_t* sp_nnz,
                                  int32_t sm_budget, double* latency_us);

/* The latency model's inputs for a launch of n_rows at sm_budget (0 = all
 * SMs), as rap_predict_latency_us evaluates them: terms[0] the kernel it
 * takes (RAP_KERNEL_TILED / _ROWS / _JIT), terms[1] its grid (CTAs),
 * terms[2] the busiest CTA's predicted sparse work (cost units), terms[3]
 * the algorithmic bytes, terms[4] its dense work (the generated kernel: its
 * dense warp's), terms[5] its (sparse output, row) pairs.  terms: HOST
 * double[6].  For refitting the model. */
rap_status rap_predict_terms(const rap_plan* plan, int64_t n_rows, const int64_t* sp_nnz, int32_t sm_budget,
                             double* terms);

/* Smallest budget whose predicted exposed latency T_delta = P - OC is <= 0
 * for the given overlapping capacity OC (microseconds of training slack),
 * L1138-1152; if none fits, the budget minimising T_delta (all SMs).
 * Writes the budget and T_delta (HOST). */
rap_status rap_choose_budget(const rap_plan* plan, int64_t n_rows, const int64_t* sp_nnz,
                             double overlap_capacity_us, int32_t* sm_budget, double* t_delta_us);

rap_status rap_plan_info_get(const rap_plan* plan, rap_plan_info* info);

/* A stream whose kernels run on a dedicated partition of the device's SMs (a
 * CUDA green context): the SM budget enforced by the hardware instead of by a
 * CTA-slot cap (§6.2; a capped grid is spread by the block
 * scheduler over up to ctas_per_sm x budget SMs).  n_sms is rounded up to the
 * architecture's granularity (sm_100: multiples of 8); *sms_out (HOST, may be
 * NULL) receives the partition's SM count.  priority as cudaStreamCreateWithPriority.
 * Launch rap_preprocess on it with the plan's budget set to *sms_out.
 * RAP_ERR_UNSUPPORTED without driver support.  Destroy with
 * rap_sm_partition_stream_destroy (after the work on it completed). */
rap_status rap_sm_partition_stream(int32_t device, int32_t n_sms, int32_t priority, void** stream_out,
                                   int32_t* sms_out);
rap_status rap_sm_partition_stream_destroy(void* stream);

/* Select the kernel of the following rap_preprocess calls (RAP_KERNEL_*). */
rap_status rap_set_kernel(rap_plan* plan, int32_t mode);

/* Development aid (no device needed): validate and lower the graph, write the
 * CUDA source the code generator emits for it into HOST buf[cap] (NUL
 * terminated, truncated to fit) and, if compile != 0, compile it with NVRTC for
 * sm_100a (no load); *ok = 1 if it compiled.  NVRTC's log goes to
 * rap_last_error().  RAP_ERR_UNSUPPORTED if the plan does not fit the
 * row-block kernel. */
rap_status rap_debug_jit_source(const rap_graph* graph, const rap_op_param* params, int32_t n_params, char* buf,
                                int64_t cap, int32_t compile, int32_t* ok);

/* Device-side capacity overflow of the launches since the last query: a
 * kernel that found more output ids than values_capacity (possible only when
 * sp_nnz understated the batch) stores none past the capacity and raises a
 * flag.  Synchronises the plan's device, writes *overflow (HOST, 0 or 1) and
 * clears the flag. */
rap_status rap_check_overflow(rap_plan* plan, int32_t* overflow);

/* ---- Multi-GPU (§7.2; hybrid parallelism L488-499) ----
 * Table-wise: each sparse output ("table") is preprocessed over the FULL
 * global batch on the GPU that owns its embedding table (locality rule,
 * L1526-1534); dense outputs are batch-sharded (each rank produces the rows of
 * its own MLP mini-batch).  Only a residual row range of an overloaded rank's
 * feature moves (L1594-1600), shipped back over NCCL by the caller.
 */
typedef enum {
  RAP_PLACE_BALANCED = 0,    /* LPT on predicted cost (largest first to the least loaded rank) */
  RAP_PLACE_ROUND_ROBIN = 1, /* output j -> rank j mod world */
  RAP_PLACE_SKEWED = 2       /* rank 0 takes ~2x the mean load (Fig 12's skew, L2317-2318), LPT for the rest */
} rap_place_mode;

/* A residual move: rows [split_row, n_rows) of sparse output `output` are
 * preprocessed on `helper` instead of its owner and shipped to the owner.
 * split_row is a multiple of 128 in [128, n_rows).  output = -1: none. */
typedef struct {
  int32_t output, owner, helper, pad;
  int64_t split_row;
} rap_residual;

/* Rows of `rank`'s batch shard: [*row0, *row0 + *rows).  Boundaries are
 * multiples of 128 rows (so validity bitmaps and 16-byte staging stay
 * aligned); the last rank takes the remainder.  world = 1: the whole batch. */
rap_status rap_shard_rows(int64_t n_rows, int32_t rank, int32_t world, int64_t* row0, int64_t* rows);

/* Predicted cost (model units per batch, the cost model of the fused kernel's
 * partition) of each sparse output of `plan` for a batch of
 * n_rows.  cost: HOST double[n_sparse_out]. */
rap_status rap_plan_output_costs(const rap_plan* plan, int64_t n_rows, const int64_t* sp_nnz, double* cost);

/* Place n sparse outputs on `world` ranks (host only, no device).
 *   cost[n]      HOST, per-output predicted cost (rap_plan_output_costs)
 *   colocate[n]  HOST, may be NULL; -1 or the index of an earlier output this
 *                one must share a rank with (an NGram table with its first
 *                source's table)
 *   owner_out[n] HOST, rank of each output
 *   load_out     HOST double[world] or NULL: resulting predicted load per rank
 *   residual     HOST or NULL.  Non-NULL: when the most loaded rank exceeds
 *                the mean by more than imbalance_tol (relative), move the
 *                row range [split_row, n_rows) of its costliest output to
 *                the least loaded rank so their loads about meet, and report
 *                it (load_out includes the move).  One move per call. */
rap_status rap_place(const double* cost, const int32_t* colocate, int32_t n, int32_t world, int32_t mode,
                     int64_t n_rows, double imbalance_tol, int32_t* owner_out, double* load_out,
                     rap_residual* residual);

/* Communication model of a residual move (§7.2: move
 * only when the balance gain beats the added communication). */
typedef struct {
  double us_per_unit;      /* microseconds per cost unit (a measured kernel time / its predicted cost) */
  double link_gbs;         /* owner <-> helper point-to-point bandwidth, GB/s (NVLink 5 / NVSwitch) */
  double link_latency_us;  /* fixed cost of one exchange (send/recv launch and synchronisation) */
  const double* row_bytes; /* HOST double[n]: bytes one row of output j moves (its raw input row to
                              the helper plus its output row back to the owner) */
} rap_comm_model;

/* rap_place with a costed residual move: with h the most and l the least
 * loaded rank (loads L_h > L_l, cost units), f h's costliest output (p cost
 * units per row) and t(m) = (link_latency_us + m * row_bytes[f] /
 * (1e3 * link_gbs)) / us_per_unit the exchange of m rows, the helper finishes
 * the piece at L_l + m p and the owner holds its KJT at
 * max(L_h - m p, L_l + m p + t(m)).  m balances the two
 * (m = (L_h - L_l - t(0)) / (2 p + t(1) - t(0))), rounded down to whole
 * 128-row tiles; the move is made only if that finish time is below L_h
 * (a gain after communication), whatever imbalance_tol.  comm NULL:
 * rap_place.  load_out: compute loads after the move. */
rap_status rap_place_comm(const double* cost, const int32_t* colocate, int32_t n, int32_t world, int32_t mode,
                          int64_t n_rows, const rap_comm_model* comm, int32_t* owner_out, double* load_out,
                          rap_residual* residual);

/* Joint preprocessing-graph mapping (§7.2): start from
 * the data-locality mapping (every output on the rank that consumes it,
 * home[j]; home[j] = -1: a row-wise sharded table whose input every rank
 * needs, so its graph is duplicated on every rank, L1526-1533), evaluate it
 * with the co-running cost model, then repeatedly substitute: move one
 * preprocessing graph (an output with its colocated outputs) from the rank
 * with the highest cost to the one with the lowest, when that lowers the
 * mapping's cost after charging the move's input communication (the raw
 * rows to the new rank and the output rows back to the consumer,
 * comm->row_bytes[j] per row over comm->link_gbs plus link_latency_us), until
 * no substitution helps (L1592-1602).
 *   cost[n]       HOST, per-output predicted cost units (rap_plan_output_costs)
 *   colocate[n]   HOST or NULL, as rap_place
 *   home[n]       HOST, consumer rank of each output, or -1 (duplicated)
 *   n_rows        batch rows (row_bytes * n_rows = one output's traffic)
 *   comm          HOST, the link model (us_per_unit converts cost units)
 *   oc_us         overlap capacity of the training step per rank (us): the
 *                 cost of a mapping is the largest exposed preprocessing
 *                 time max_r max(0, T_r - oc_us), ties broken by max_r T_r,
 *                 with T_r the rank's compute time plus its exchanges
 *   owner_out[n]  HOST, the rank that evaluates each output (-1: every rank)
 *   time_out      HOST double[world] or NULL: T_r of the final mapping (us)
 *   n_moves       HOST or NULL: substitutions made */
rap_status rap_place_joint(const double* cost, const int32_t* colocate, const int32_t* home, int32_t n,
                           int32_t world, int64_t n_rows, const rap_comm_model* comm, double oc_us,
                           int32_t* owner_out, double* time_out, int32_t* n_moves);

/* A sharded plan: the graph restricted to its dense outputs (evaluated over
 * this rank's batch shard, rap_shard_rows) and the sparse outputs j with
 * sparse_owner[j] == rank (j counts the graph's sparse outputs in order),
 * evaluated over the full batch.  sparse_owner: HOST int32[#sparse outputs],
 * each in [-1, world); -1 = in no rank's main plan (a residual output that
 * its owner and helper run as row-range pieces).
 * Output shapes: rap_plan_output_shape's d_out_cols with shard rows. */
rap_status rap_plan_create_sharded(const rap_graph* graph, const rap_op_param* params, int32_t n_params,
                                   int32_t device, int32_t sm_budget, const int32_t* sparse_owner,
                                   int32_t rank, int32_t world, rap_plan** out);

/* Append a jagged piece (n rows: lengths int32[n], its own offsets int64[n+1]
 * starting at src_offsets[0], values indexed by those offsets) to a chained
 * output (see RAP_OUT_CHAIN): dst_offsets[0] holds the running total T (DEVICE);
 * writes dst_lengths[0..n), dst_offsets[1..n] = T + src_offsets[i] -
 * src_offsets[0] and values to dst_values[T ..].  All pointers DEVICE;
 * values_bound (HOST) bounds the piece's value count (launch sizing only);
 * dst_capacity guards dst_values.  Enqueued on `stream`, no host sync. */
rap_status rap_jagged_append(const int32_t* lengths, const int64_t* src_offsets, const int64_t* values, int64_t n,
                             int64_t values_bound, int32_t* dst_lengths, int64_t* dst_offsets, int64_t* dst_values,
                             int64_t dst_capacity, void* stream);

/* Profiling aid.  enable = 1: the following rap_preprocess calls record 24
 * uint64 stamps per CTA (slots 0..4 = %globaltimer at the phase boundaries,
 * 5 = sparse tile range, 6 = SM id, 7 = partition rank, 8..23 = clock64
 * inside the first sparse tile / dense block) for up to `cap` CTAs.
 * enable = 0: synchronise the device and copy the stamps of the last call to
 * HOST host_out (uint64[cap * 24]);
 * *n_desc receives that call's CTA count.  enable = -1: stop recording and
 * free the buffer. */
rap_status rap_debug_trace(rap_plan* plan, int32_t enable, uint64_t* host_out, int64_t cap, int64_t* n_desc);
void rap_plan_destroy(rap_plan* plan);

const char* rap_status_string(rap_status status);
const char* rap_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* RAP_H */
