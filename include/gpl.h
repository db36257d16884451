/*
 * gpl.h — C ABI of the B200-native GPL hot path (pipelined scan -> probe ->
 * aggregate over columnar in-memory relations).
 *
 * Paper: J. Paul, J. He, B. He, "GPL: A GPU-based Pipelined Query Processing
 * Engine", SIGMOD'16 (PAPER.md; cited as P:<line>).
 *
 * The calls follow the paper's problem statement:
 *   - a query plan over columnar in-memory relations is split into segments,
 *     each ending at a blocking kernel; hash build is blocking, probe is not
 *     (§3.1 "segments", §3.2 "Hash join ... requires a blocking
 *     barrier after hash build");
 *   - the input of a segment is processed tile by tile, the tile size coming
 *     from a cost model (§3.1, §3.3, §4 Eqs 1-9);
 *   - only the outputs of blocking kernels are materialised in global memory
 *     (P:135); the rest passes through on-chip channels (P:179-189
 *     §3.4), here shared-memory rings inside one fused sm_100a kernel;
 *   - data is resident on the device (App. A).
 *
 * Conventions
 *   - Every call returns gpl_status (0 = GPL_OK). No C++ exception crosses the
 *     ABI; the message of the last failure is gpl_last_error(ctx).
 *   - One context = one CUDA device + one stream, used by one host thread at a
 *     time. All device work is enqueued on that stream, in call order; stream
 *     order is the "blocking barrier" between segments.
 *   - Types: keys, dates (int32 yyyymmdd) and dictionary codes are int32;
 *     decimals are scaled int64 (scale stated per column). Sums are exact:
 *     int64 on chip, int128 in the partials and the result.
 *   - Plan texts: see DESIGN.md §4 (grammar) and paper_conf_sigmod_paulhh16_b200/plans/.
 */
#ifndef GPL_H
#define GPL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t gpl_status;
enum {
  GPL_OK = 0,
  GPL_E_ARG = 1,       /* bad argument (NULL, type, alignment, size)                */
  GPL_E_CUDA = 2,      /* CUDA runtime error (message has the CUDA error string)    */
  GPL_E_NOMEM = 3,     /* device allocation failed                                  */
  GPL_E_STATE = 4,     /* missing table / hash table / no run to fetch              */
  GPL_E_DUPKEY = 5,    /* build key not unique (all paper joins are FK->PK)         */
  GPL_E_CAPACITY = 6,  /* caller buffer too small (n_groups / nbytes set)           */
  GPL_E_OVERFLOW = 7,  /* a value bound exceeds exact int64 arithmetic              */
  GPL_E_DOMAIN = 8,    /* a row's group value fell outside the declared domain      */
  GPL_E_NODEV = 9,     /* operation needs a device but the context has none         */
  GPL_E_PLAN = 10      /* plan text: syntax or semantic error                        */
};

/* Column types. */
enum { GPL_I32 = 1, GPL_I64 = 2, GPL_DATE32 = 3, GPL_DEC64 = 4, GPL_DICT32 = 5 };

/* gpl_load_columns flags */
enum { GPL_COPY = 0, GPL_BORROW = 1 };

typedef struct {
  const char* name;       /* column name, unique within the table                          */
  int32_t type;           /* GPL_I32 .. GPL_DICT32                                           */
  int32_t scale;          /* decimal scale (informational; 0 for non-decimals)              */
  const void* data;       /* host or device pointer to nrows values                          */
  int32_t on_device;      /* 1: data is a device pointer on the context's device            */
  int32_t reserved;
  int64_t capacity_rows;  /* BORROW only: rows allocated behind data (0 = nrows).           */
} gpl_column;

typedef struct gpl_ctx gpl_ctx;

/* Statistics of the last gpl_run_plan (filled by gpl_fetch_result). */
typedef struct {
  int64_t rows_scanned;        /* fact rows streamed through the pipeline                        */
  int64_t tile_rows_used;      /* Δ actually used (rows per scheduling claim)                    */
  int32_t stage_rows;          /* rows per TMA stage                                              */
  int32_t ring_depth;          /* stages in the shared-memory ring ("channels")            */
  int32_t consumer_warps;      /* consumer warps per CTA                                          */
  int32_t grid;                /* persistent CTAs                                                 */
  int32_t n_ops;               /* entries used in op_pass                                         */
  int32_t probe_split;         /* probes run before the survivor queue (-1: none)                */
  int64_t op_pass[16];         /* rows passing each operator in plan order (filters, probes, where) */
  double kernel_ms;            /* fused pipeline kernel time (CUDA events on the ctx stream)      */
  double predicted_ms;         /* A9 model estimate for this run                                   */
  double bytes_scanned;        /* the fused kernel's own HBM bytes: rows x bytes/row of TMA-staged */
                               /* columns + the clustered probe's table cells + per lazy column   */
                               /* min(rows reaching its first use x 32 B sector, rows x width)     */
  int32_t agg_mode;            /* 0 registers (1 group), 1 smem table, 2 global int128 atomics,  */
                               /* 3 hash group-by (global open-addressing table, int64 sums)      */
  int32_t kbe;                 /* 1 if produced by gpl_run_plan_kbe                               */
  int32_t jit;                 /* 1 if the plan-specialised (NVRTC) kernel ran, 0 the generic one */
  int32_t reserved;
  double intermediate_bytes;   /* bytes of operator outputs materialised in HBM (fused path: 0)   */
  double bytes_full_scan;      /* rows x bytes/row of EVERY column the plan reads (no late        */
                               /* materialisation): the logical scan; >= bytes_scanned            */
  int32_t lazy_columns;        /* columns gathered per surviving row instead of TMA-staged        */
  int32_t packets;             /* 128-row packets per consumer iteration                          */
  int64_t groups_total;        /* hash group-by: distinct groups (the result may be LIMITed)      */
  int64_t hash_slots;          /* hash group-by: slots of the aggregation table                    */
  int32_t drain_warps;         /* of consumer_warps, those that only drain hand-off packets (NEXT-1) */
  int32_t launches;            /* kernels one graph-replayed gpl_run_query step launched (its graph's */
                               /* kernel nodes: clear, builds, fused run, result steps); 0 otherwise */
} gpl_stats;

/* Result of the last run. Arrays are CALLER-owned with capacity cap_groups. */
typedef struct {
  int32_t cap_groups;          /* in: rows the arrays can hold                                    */
  int32_t n_groups;            /* out: non-empty groups (1 row when the plan has no GROUP BY);   */
                               /* with 'order'/'limit' (A10): rows in ORDER BY order      */
                               /* (ties: decoded key tuple ascending), at most the limit         */
                               /* (hash group-by: stats.groups_total = all distinct groups)      */
  int32_t n_keys;              /* out: group key columns                                          */
  int32_t n_aggs;              /* out: aggregates per row; agg 0 is COUNT(*)                      */
  int32_t* keys;               /* out: [cap_groups][n_keys] key values (after the plan's 'decode' */
                               /* maps, e.g. nation key -> n_name code); rows sorted by key       */
                               /* unless the plan has 'order'                                     */
  int64_t* aggs;               /* out: [cap_groups][n_aggs][2] int128 as (lo, hi) little-endian   */
  gpl_stats stats;             /* out */
  int32_t n_ratios;            /* out: ratio columns of the plan ('ratio [C *] agg I / agg J')    */
  int32_t reserved;
  double* ratios;              /* out (optional, may be NULL): [cap_groups][n_ratios] C*num/den    */
                               /* as doubles (P:634-635 mkt_share, P:682-685 promo_revenue);      */
                               /* NaN = SQL NULL (den = 0)                                         */
} gpl_result;

/* A9 model report (gpl_choose_tile_rows). */
typedef struct {
  int64_t tile_rows;
  int32_t stage_rows, ring_depth, consumer_warps, grid;
  double predicted_ms;
  double t_stream_ms, t_probe_ms, t_tail_ms, t_launch_ms;
  double bw_gbs;               /* effective HBM bandwidth the model used                           */
  int32_t smem_bytes;
  int32_t feasible;
  int32_t ctas_per_sm;
  int32_t candidates;          /* gpl_autotune: shapes measured                                    */
  double measured_ms;          /* gpl_autotune: median kernel time of the chosen shape            */
  int32_t probe_split;         /* probes run before the survivor queue (autotune: measured best)  */
  int32_t builds_tuned;        /* gpl_autotune: pipelined (DIRECT) build segments measured         */
  double build_ms_model;       /* gpl_autotune: Σ median build time at the model's shapes          */
  double build_ms;             /* gpl_autotune: Σ median build time at the pinned (best) shapes    */
} gpl_model_report;

/* Create a context on CUDA device `device` enqueuing on `cuda_stream` (a
 * cudaStream_t, e.g. torch.cuda.current_stream().cuda_stream; NULL = the
 * library creates its own non-blocking stream). device = -1 creates a
 * HOST-ONLY context (no CUDA calls): plans can be parsed/validated and the
 * cost model queried; gpl_build_hash only validates and registers the
 * table's shape (no data), run/fetch return GPL_E_NODEV. Platform facts (SMs,
 * shared memory, L2) are queried from the device.
 * Errors: GPL_E_ARG (out == NULL), GPL_E_CUDA (bad device). */
gpl_status gpl_create(int device, void* cuda_stream, gpl_ctx** out);

/* Free every ctx-owned device allocation (copied columns, hash tables,
 * partials). Borrowed column memory is untouched. NULL is a no-op. */
void gpl_destroy(gpl_ctx* ctx);

/* Place a table's columns in HBM (SoA). Replaces an
 * existing table of that name and invalidates hash tables built from it.
 *   GPL_COPY:   data may be host or device memory; the ctx owns a padded
 *               (64-row, zero-filled) 256-B-aligned copy.
 *   GPL_BORROW: data must be device memory, 16-B aligned, with
 *               capacity_rows >= nrows rounded up to 4 rows; the caller keeps
 *               it alive and unchanged while any run may read it.
 * Per-column min/max and sortedness are computed on the device with the load
 * (validator bounds, clustered probes). The call does NOT synchronise: the
 * copies and the min/max pass are enqueued on the ctx stream, and the first
 * later call that validates, plans or runs (gpl_check_plan, gpl_build_hash,
 * gpl_run_*, gpl_autotune, gpl_compile_plan, gpl_choose_tile_rows,
 * gpl_fetch_result, gpl_sync) waits for all pending loads at once. So a
 * GPL_COPY source in pinned host or device memory must stay allocated and
 * unchanged until such a call (pageable host memory is staged by the CUDA
 * runtime before this call returns).
 * Errors: GPL_E_ARG (type, alignment, duplicate name, nrows < 0), GPL_E_NOMEM. */
gpl_status gpl_load_columns(gpl_ctx* ctx, const char* table, int64_t nrows, int32_t ncols,
                            const gpl_column* cols, uint32_t flags);

/* Run one BUILD segment (scan -> filter -> probe earlier hash tables ->
 * insert): open addressing, linear probing, power-of-two slots sized
 * exactly from a device-side count pass (load <= 0.5). Asynchronous; later
 * segments see the table by stream order. *ht_id receives the table's id
 * (also addressable by name from plan texts). A table of the same name is
 * replaced. Errors: GPL_E_PLAN, GPL_E_STATE (unknown table/column/hash table).
 * Duplicate keys are detected on device and reported by the next
 * gpl_fetch_result (GPL_E_DUPKEY) or gpl_sync(). */
gpl_status gpl_build_hash(gpl_ctx* ctx, const char* build_segment, int32_t* ht_id);

/* Run the PROBE segment (the fused pipeline: TMA-staged tiles -> filter ->
 * survivor queue -> probe(s) -> where -> group-by aggregate; no
 * inter-operator HBM traffic). tile_rows = 0 lets the A9 cost model choose
 * Δ; otherwise it is rounded up to a multiple of the stage rows.
 * Asynchronous on the ctx stream. Errors: GPL_E_PLAN, GPL_E_STATE,
 * GPL_E_OVERFLOW (value bound not provably exact). */
gpl_status gpl_run_plan(gpl_ctx* ctx, const char* probe_segment, int64_t tile_rows);

/* Whole query in one call: `plan` holds the build segments followed by the
 * probe segment (split at 'build NAME' / 'run TABLE' lines); equivalent to
 * gpl_build_hash for each build segment then gpl_run_plan. Once every segment
 * is prepared and profiled, the sequence (hash builds + fused kernel) is
 * recorded as a CUDA graph and later calls replay it with a single
 * cudaGraphLaunch while the tables, hash tables and options are unchanged
 * (any change falls back to the per-segment path and re-records). Fetch with
 * gpl_fetch_result. Errors: as gpl_build_hash / gpl_run_plan. */
gpl_status gpl_run_query(gpl_ctx* ctx, const char* plan, int64_t tile_rows);

/* Same plan, executed kernel-at-a-time with every operator's output
 * materialised in HBM: the paper's KBE baseline (§2.2, Fig 7): per
 * operator a map kernel, a prefix sum and a scatter, the host reading each
 * output cardinality to size the next buffers (so this call synchronises).
 * Same result contract (bit-identical results); stats.kbe = 1 and
 * stats.intermediate_bytes = bytes materialised between operators (flags,
 * positions, payload and compacted columns). For comparison only (config 5).
 * With option "kbe_tile_rows" = T > 0 the same sequence runs tile by tile
 * (T rows at a time, materialising per tile): the paper's GPL (w/o CE)
 * variant, tiling without concurrent kernels or channels (P:337, P:382,
 * P:564); its buffers are sized for T rows and every operator's cardinality
 * stays on the device (the kernels read it), so the tiles run back to back
 * with no host round trip (one synchronise at the end for the byte count);
 * stats.tile_rows_used = T. */
gpl_status gpl_run_plan_kbe(gpl_ctx* ctx, const char* probe_segment);

/* Synchronise the stream and return the last run's result: the A10 finalize
 * step ("ORDER BY is blocking") — host decode of the
 * int128 partials, empty groups dropped, group keys mapped through the plan's
 * 'decode key I TABLE KEYCOL -> OUTCOL' tables, the plan's ORDER BY ('order
 * agg I|key I [asc|desc], ...'; ties by the key tuple ascending) else key
 * order, 'limit K', and the 'ratio [C *] agg I / agg J' columns (into
 * out->ratios when non-NULL; den = 0 gives NaN). Errors: as below, plus
 * GPL_E_STATE when a decode table misses a group key. Device error
 * flags latched during builds/run are returned here (GPL_E_DUPKEY,
 * GPL_E_DOMAIN, GPL_E_OVERFLOW). GPL_E_CAPACITY if out->cap_groups is too
 * small (out->n_groups then holds the needed rows). */
gpl_status gpl_fetch_result(gpl_ctx* ctx, gpl_result* out);

/* Raw dense partial aggregates of the last run, for a cross-GPU merge:
 * n_groups_declared x n_aggs int128 (lo, hi), row-major. Copied
 * (stream-ordered, asynchronous) into `dst` (device pointer if
 * dst_on_device, else host; then the call synchronises). *nbytes = size.
 * GPL_E_CAPACITY if cap_bytes is too small. */
gpl_status gpl_fetch_partials(gpl_ctx* ctx, void* dst, int32_t dst_on_device, size_t cap_bytes,
                              size_t* nbytes);

/* Decode merged partials (host memory, the layout above, for the plan of the
 * context's last run) into out, exactly like gpl_fetch_result. */
gpl_status gpl_decode_partials(gpl_ctx* ctx, const void* host_partials, size_t nbytes,
                               gpl_result* out);

/* Fixed-order exact int128 sum of `nranks` partial vectors laid out back to
 * back in host memory (the all-gather output): out[i] = sum_r in[r][i].
 * Pure host function (no context). */
gpl_status gpl_merge_partials(const void* gathered, int32_t nranks, size_t nbytes_each, void* out);

/* Synchronise the ctx stream; returns latched device errors. */
gpl_status gpl_sync(gpl_ctx* ctx);

/* A9: the B200 re-derivation of the paper's model (Eqs 2-9) for
 * `probe_segment` over n_rows fact rows (n_rows <= 0: the loaded table).
 * Fills the chosen configuration and its predicted time. */
gpl_status gpl_choose_tile_rows(gpl_ctx* ctx, const char* probe_segment, int64_t n_rows,
                                gpl_model_report* out);

/* Calibrate the pipeline shape of a query by measurement (the paper profiles
 * the first tile and then searches its model): runs the plan's
 * build segments, takes the A9 model's best configuration for every
 * (CTAs per SM, stage rows) shape (at most max_candidates) under every probe
 * split (how many probes run before the survivor queue), times each on the
 * device with L2 flushed (median of 3), and pins the fastest for this probe
 * segment; later gpl_run_plan / gpl_run_query calls with tile_rows = 0 use
 * it until gpl_set_option is called. Every build segment that runs as a
 * pipeline (DIRECT tables) is tuned the same way: the model's per-shape
 * candidates are timed on a rebuild of the table (identical contents) and
 * the fastest is pinned for that segment. Synchronises. out (optional)
 * receives the chosen shape, its model estimate and its measured time, and
 * the build segments' summed times at the model's and the pinned shapes. */
gpl_status gpl_autotune(gpl_ctx* ctx, const char* plan, int32_t max_candidates, gpl_model_report* out);

/* One point of the channel calibration Γ (Eq 1; the
 * producer -> consumer chain of P:83): the throughput of the fused kernel's
 * shared-memory ring for one shape (ring depth = the "number of channels",
 * stage rows = the packet analog, CTAs per SM) at one data size. */
typedef struct {
  int32_t ring_depth, stage_rows, ctas_per_sm, consumer_warps;
  int64_t rows;    /* rows streamed (16 B each: 2 int32 + 1 int64 columns)             */
  double bytes;    /* rows x 16                                                         */
  double ms;       /* median kernel time, L2 flushed before each repetition             */
  double t0_ms;    /* the same shape over an empty input (launch + prologue)            */
  double gbs;      /* Γ = bytes / (ms - t0_ms) / 1e9                                    */
} gpl_gamma_point;

/* Calibrate Γ: for every ring shape (depth {2,3,4} x
 * stage rows {1024,2048,4096} x CTAs/SM {1,2}; shapes that do not fit shared
 * memory are skipped) and every size in rows[0..n_rows) (NULL/0: 2^19..2^26
 * rows), stream a synthetic zero table through the pipeline kernel and time
 * it on the device. The points replace the copy bandwidth in the A9 model
 * (predict: Γ of the candidate shape at d = rows x bytes/row; t0 as its
 * launch term) until gpl_set_calibration / gpl_set_option("use_gamma", 0).
 * Options, tables and hash tables of the context are left as they were.
 * out (optional, capacity cap) receives the points; *n_out their count
 * (GPL_E_CAPACITY if cap is too small — the calibration is still applied).
 * Synchronises; takes seconds (one plan-specialised compile per shape). */
gpl_status gpl_calibrate(gpl_ctx* ctx, const int64_t* rows, int32_t n_rows, gpl_gamma_point* out, int32_t cap,
                         int32_t* n_out);

/* Load a saved calibration (points as gpl_calibrate returned them; n = 0
 * clears it: the model falls back to the copy bandwidth). Host only. */
gpl_status gpl_set_calibration(gpl_ctx* ctx, const gpl_gamma_point* pts, int32_t n);

/* Tuning knobs (tests / sweeps): "stage_rows", "ring_depth",
 * "consumer_warps", "ctas_per_sm", "probe_split" (-1 = auto), "hash_load_pct",
 * "jit" (1 = plan-specialised kernels, default; 0 = generic kernel),
 * "build_pipeline" (1 = DIRECT build segments run through the fused pipeline
 * with an insert sink, default; 0 = the standalone build kernels),
 * "kbe_tile_rows" (gpl_run_plan_kbe tile size; 0 = whole input),
 * "kbe_graph" (1 = GPL (w/o CE)'s tile loop replayed as one captured CUDA graph, default; 0 = launched),
 * "autotune_probe" (1 = gpl_autotune measures the build segments and the probe segment, default; 0 = the
 * build segments only, the probe segment keeping the A9 model's pick; changing it keeps pinned shapes),
 * "use_gamma" (1 = the model uses the Γ calibration when loaded, default),
 * "drain_warps" (operator-specialised consumer warps, NEXT-1: of the
 * consumer warps, this many only run the queue phase of survivor packets the
 * others hand over; -1 = the model's choice from {0, 1, 2}, default),
 * "graph_branches" (1 = gpl_run_query's graph runs build segments that do
 * not depend on each other on two lanes, default; 0 = one chain),
 * "hash_slots_log2" (hash group-by table of 2^v slots; 0 = sized from the
 * plan's last run, default), "use_profile" (1 = the model fits its consumer cost to the plan's first
 * timed run after its λ profile, Table 2 "profiling input", default),
 * "dense_build" (1 = a DIRECT build keyed by a strictly increasing column writes
 * its cell ranges densely, default; 0 = atomic inserts into a cleared table),
 * "nibble_cells" (1 = DIRECT payloads of at most 15 values in 4-bit cells; 0 =
 * byte cells, default), "lazy_columns" (late materialisation: -1 = from the
 * plan's pass fractions, default; 0 = off; 1 = every eligible column).
 * Builds take "probe_split" too (a DIRECT build's probes and insert in the
 * stage phase or the queue phase; gpl_autotune measures both).
 * value < 0 restores automatic selection. */
gpl_status gpl_set_option(gpl_ctx* ctx, const char* key, int64_t value);

/* Validate a plan segment against the loaded tables (host only). */
gpl_status gpl_check_plan(gpl_ctx* ctx, const char* segment);

/* Compile (NVRTC, sm_100a) the plan-specialised build of the fused kernel for
 * this probe segment and cache it, so the first gpl_run_plan does not pay the
 * compile. The shape depends on the loaded tables, hash tables, options and
 * the A9 configuration for tile_rows. On a host-only context it compiles
 * without loading (a build check). GPL_E_STATE if NVRTC is unavailable or
 * the compile fails (message in gpl_last_error); gpl_run_plan then uses the
 * generic precompiled kernel. Disable with gpl_set_option("jit", 0).
 * A build segment is accepted too: a DIRECT build compiles its pipelined
 * (insert-sink) kernel; other builds use precompiled kernels (no-op). */
gpl_status gpl_compile_plan(gpl_ctx* ctx, const char* probe_segment, int64_t tile_rows);

/* Hash group-by across ranks (SURVEY §8(f) NEXT-4 with §8(e)): the rows of the
 * last run of a 'group hash' plan — [packed key, acc 0 .. nagg-1] int64 words
 * per row (key = k0 << 32 | k1 for two keys; *row_words = 1 + nagg) — into
 * caller-owned host memory (cap_rows rows):
 * the LIMIT rows in ORDER BY order, else every group. *n_rows is set even when
 * cap_rows is too small (GPL_E_CAPACITY). Synchronises. */
gpl_status gpl_fetch_groups(gpl_ctx* ctx, int64_t* rows, int64_t cap_rows, int64_t* n_rows, int32_t* row_words);

/* Merge the rows of several ranks (concatenated gpl_fetch_groups outputs,
 * e.g. all-gathered over NCCL): exact int128 sums per key, then the probe
 * segment's ORDER BY / LIMIT (else key order), into `out` as gpl_fetch_result
 * fills it (stats.groups_total = distinct merged groups). A LIMIT plan is exact
 * when every rank ships all its groups, or when the group key contains the
 * shard key (TPC-H Q3: l_orderkey; disjoint groups). Host only. */
gpl_status gpl_merge_groups(gpl_ctx* ctx, const char* probe_segment, const int64_t* rows, int64_t n_rows,
                            gpl_result* out);

/* Message of the last failed call on ctx (ctx-owned, valid until the next
 * call). gpl_last_error(NULL) reports gpl_create failures. */
const char* gpl_last_error(const gpl_ctx* ctx);

/* "gpl-b200 <version> sm_100a". */
const char* gpl_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GPL_H */
