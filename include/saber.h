/*
 * saber.h -- C ABI of the B200-native windowed-query hot path
 * (SABER, Koliousis et al., SIGMOD'16; PAPER.md = /root/reference/PAPER.md).
 *
 * One query q = (window function ω, operator function f^q, stream function φ^q)
 * (§2.4) is created once, fed a stream of row-major tuples
 * through saber_task_submit*, and its window results are read back in window
 * order through saber_results_poll.  Internally the submitted stream is cut
 * into fixed-size query tasks of φ = task_bytes bytes that are independent of
 * the window definition (§3, §4.1); each task runs on the
 * GPU as: window-boundary/pane assignment → σ/π with stream compaction or
 * pane (window-fragment) partial aggregation → window assembly → result stage
 * (§4.3).  There is no CPU execution path: every step of a task
 * runs in this library's sm_100a kernels; without a CUDA device every
 * compute entry point returns SABER_ECUDA.
 *
 * Conventions for every function:
 *   - all functions return saber_status (0 = OK, < 0 = error) unless noted;
 *   - no C++ types and no exceptions cross this boundary;
 *   - a query is used by ONE submitting thread (the paper's single-inserter
 *     rule, L745-748); poll/release may run on one other thread;
 *   - after a data error (non-monotone or negative timestamp, out-of-domain
 *     key, table overflow) the query is sticky-failed: every later call
 *     returns the same status and saber_last_error() says why.
 */
#ifndef SABER_H
#define SABER_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  SABER_OK = 0,
  SABER_EINVAL = -22,     /* invalid argument / query / schema                       */
  SABER_ENOMEM = -12,     /* device or pinned allocation failed, result slot too small */
  SABER_EAGAIN = -11,     /* poll timed out / no result ready                        */
  SABER_EORDER = -1001,   /* timestamps not non-decreasing       */
  SABER_ECUDA = -1002,    /* CUDA runtime error or no device                         */
  SABER_ENCCL = -1003,    /* reserved: the cross-GPU exchange runs in torch.distributed
                             (NCCL) above this ABI                     */
  SABER_ECLOSED = -1004,  /* submit after finish                                     */
  SABER_ETS = -1005,      /* negative timestamp (time domain is {0,1,..}, L349-350)  */
  SABER_EKEY = -1006,     /* GROUP BY key outside its declared domain [0, domain)    */
  SABER_ECAPACITY = -1007 /* pane hash table or pane ring overflow   */
} saber_status;

typedef enum { SABER_I32 = 0, SABER_I64 = 1, SABER_F32 = 2, SABER_F64 = 3 } saber_type;

/* Row-major byte tuples (L744-745, L1207-1213).  tuple_bytes must be a
 * multiple of 16 (128-bit loads); columns are naturally aligned; ts_col is an
 * I64 column holding τ(t) (§2.4).  The arrays are copied at create. */
typedef struct {
  int32_t ncols;
  const saber_type *types;
  const int32_t *offsets;
  int32_t tuple_bytes;
  int32_t ts_col;
} saber_schema;

/* ω(size, slide): count-based (tuples) or time-based (timestamp units),
 * sliding (slide < size) or tumbling (slide == size) (L366-376).  Time windows
 * are W_j = [origin + j·slide, origin + j·slide + size) (reading A1).
 * slide > size is rejected (the paper defines l <= s only, L375). */
typedef enum { SABER_WIN_COUNT = 0, SABER_WIN_TIME = 1 } saber_window_kind;
typedef struct {
  saber_window_kind kind;
  int64_t size, slide, origin;
} saber_window;

typedef enum { SABER_LT = 0, SABER_LE, SABER_GT, SABER_GE, SABER_EQ, SABER_NE } saber_cmp;
/* σ term `col op const` (conjunction of up to 64 terms, L1320-1322; SELECT_n).  The constant
 * is ival for integer columns and fval for float columns.  In HAVING, col is
 * the index of an aggregate and the constant is ival for integer results
 * (COUNT, SUM/MIN/MAX of int columns) and fval otherwise. */
typedef struct { int32_t col; saber_cmp op; int64_t ival; double fval; } saber_pred;

typedef enum { SABER_SUM = 0, SABER_COUNT, SABER_AVG, SABER_MIN, SABER_MAX } saber_aggfn;
typedef struct { saber_aggfn fn; int32_t col; } saber_agg;   /* COUNT ignores col */

/* GROUP BY key expression: key = col / div (C truncating division; LRB1's
 * position/5280, L2721).  domain > 0 declares key values in [0, domain) and
 * lets the planner use a dense per-pane table; a value outside the declared
 * domain is a data error (SABER_EKEY).  domain == 0: arbitrary values, hashed. */
typedef struct { int32_t col; int32_t div; int64_t domain; } saber_keyexpr;

/* Operator function f^q.  Either σ/π (nagg == 0; IStream output of projected
 * tuples, L395-405) or α with optional σ, GROUP BY (≤ 4 integer key columns)
 * and HAVING (RStream output of one result relation per window). */
typedef struct {
  int32_t npred;  const saber_pred *where;
  int32_t nproj;  const int32_t *proj;
  int32_t nagg;   const saber_agg *aggs;
  int32_t nkeys;  const saber_keyexpr *group_by;
  int32_t nhave;  const saber_pred *having;
} saber_operator;

typedef enum { SABER_RESULTS_HOST = 0, SABER_RESULTS_DEVICE = 1 } saber_result_mode;

/* Runtime configuration.  Zero fields take defaults (in brackets).
 *  device           CUDA device ordinal [current device]
 *  task_bytes       φ, the query task size (L485-498)            [64 MiB]
 *  pipeline_depth   task/result slots in flight (Fig. 6)  [4]
 *  result_mode      HOST: results are DMA'd into pinned host memory and poll
 *                   returns host pointers; DEVICE: poll returns device
 *                   pointers, nothing is copied              [HOST]
 *  result_bytes     capacity of one result slot (rows + headers) [auto]
 *  hash_capacity    slots per pane hash table (power of two)   [auto]
 *  max_panes        pane ring capacity bound (time windows)    [auto]
 *  base_index       global position of the first submitted tuple (count
 *                   windows; used by task partitioning across GPUs) [0]
 *  first_window     windows with id < first_window are not emitted (they
 *                   belong to the previous partition)           [0]
 *  emit_on_finish   1: finish() closes windows up to the watermark; 0: the
 *                   partition's tail windows are left to its successor [1]
 *  result_slots     result slices held until released (the paper's circular
 *                   result buffer, L1044-1058); a submit that needs more free
 *                   slots than exist returns SABER_EAGAIN without consuming [8]
 *  profile          1: bracket each task's kernels with CUDA events on the
 *                   query's stream and accumulate per-phase device time in
 *                   saber_stats (read at poll)                  [0] */
typedef struct {
  int32_t device;
  int64_t task_bytes;
  int32_t pipeline_depth;
  int32_t result_mode;
  int64_t result_bytes;
  int64_t hash_capacity;
  int64_t max_panes;
  int64_t base_index;
  int64_t first_window;
  int32_t emit_on_finish;
  int32_t result_slots;
  int32_t profile;
  int32_t reserved[5];
} saber_config;

typedef struct saber_query saber_query;

/* Create a query.  All argument arrays are copied; nothing is borrowed.
 * Errors: SABER_EINVAL (validation), SABER_ECUDA (no
 * device), SABER_ENOMEM.  On success *out owns device memory, pinned memory,
 * streams and events until saber_query_destroy. */
saber_status saber_query_create(const saber_schema *schema, const saber_operator *op,
                                const saber_window *window, const saber_config *cfg,
                                saber_query **out);

/* Append nbytes (a multiple of tuple_bytes) of host tuples to the stream.
 * Unregistered (pageable) bytes are borrowed only for the call: they are
 * copied into the pinned ingest ring (the paper's copyin stage, §5.2
 * L1220-1259).  Whole tasks inside a range registered with
 * saber_register_host are DMA'd straight from it, asynchronously: submit
 * returns once the copy is enqueued, and the caller must not modify those
 * bytes until the result slice of the task holding them has been polled (or
 * saber_query_sync returned) -- the movein of task i+1 overlaps the kernels of
 * task i and the moveout of task i-1 (Fig. 6).  The dispatcher cuts φ-byte
 * tasks (§4.1); a partial task waits for more data or for finish().
 * Blocks only while a pinned staging buffer is still being copied (copyin
 * path); returns SABER_EAGAIN, consuming nothing, when the result-ring slots
 * the new tasks need are not all free. */
saber_status saber_task_submit(saber_query *q, const void *host_tuples, size_t nbytes);

/* Append tuples already resident in device memory.  No copy: the bytes must
 * stay valid and unmodified until the work enqueued by this call completes;
 * the library orders itself after all prior work on `cuda_stream` (a
 * cudaStream_t, NULL = legacy default stream) and makes `cuda_stream` wait for
 * its reads, so stream order protects the buffer.  The range is cut into
 * tasks of at most φ bytes (a short last task is processed immediately). */
saber_status saber_task_submit_device(saber_query *q, const void *dev_tuples, size_t nbytes,
                                      void *cuda_stream);

/* Page-lock a caller host range so later submits from it are DMA'd without
 * a staging copy (the paper's copyin stage disappears).  Unregistered at
 * destroy. */
saber_status saber_register_host(saber_query *q, void *p, size_t nbytes);

/* End of stream: flush the partial task; for time windows close every window
 * whose end <= watermark (INT64_MIN: τ_last + 1; reading A3).  After finish,
 * submits return SABER_ECLOSED. */
saber_status saber_query_finish(saber_query *q, int64_t watermark);

typedef struct {
  int64_t window_id;   /* j: windows are numbered 0,1,.. from the stream start  */
  int64_t ts;          /* time: origin + j·slide; count: τ of position j·slide  */
  int64_t row_offset;  /* first row of this window inside the slice             */
  int32_t nrows;       /* rows of this window (0 allowed, reading A6)           */
  int32_t flags;       /* reserved, 0                                            */
} saber_win_hdr;

/* One result slice = all windows closed by one task, in window order.
 * Aggregation (RStream): nwindows headers + nrows rows stored column-wise:
 * cols[0..nkeys) are the GROUP BY key values (I32 key column → int32, I64 →
 * int64), cols[nkeys..nkeys+nagg) the aggregates (COUNT int64; SUM int64 for
 * integer columns and double for float columns; AVG double; MIN/MAX int64
 * for integer and double for float columns).  Rows inside a window have no
 * specified order (relation semantics, L381-382).
 * σ/π (IStream): tuples = ntuples projected rows (projected columns packed in
 * projection order, tuple_bytes each), in stream order.
 * Pointers are host pointers (HOST mode) or device pointers (DEVICE mode)
 * and stay valid until saber_results_release. */
typedef struct {
  int64_t task_id;
  int64_t first_window, nwindows;
  const saber_win_hdr *hdr;
  int64_t nrows;
  int32_t ncols;
  int32_t on_device;
  const void *cols[12];
  int32_t col_bytes[12];
  const void *tuples;
  int32_t tuple_bytes;
  int32_t reserved;
  int64_t ntuples;
} saber_results;

/* Return the next result slice in task order (the paper's ordered output
 * stream, L1092-1099).  timeout_us < 0 waits forever, 0 polls.  Returns
 * SABER_EAGAIN if no slice is ready in time (or nothing is pending).  In HOST
 * mode the slice's D2H was issued by the query's moveout thread as soon as the
 * task finished; poll only waits for that copy. */
saber_status saber_results_poll(saber_query *q, saber_results *out, int32_t timeout_us);
/* Hand a polled slice back; its slot is reused by a later task. */
saber_status saber_results_release(saber_query *q, const saber_results *r);

typedef struct {
  int64_t tasks, tuples, bytes_in;
  int64_t windows, rows, out_tuples;
  int64_t tasks_pending;
  /* window-fragment classes of the last task */
  int64_t last_complete, last_opening, last_closing, last_pending;
  /* device work: kernels launched, and (profile = 1) accumulated device time of
   * the pane/selection pass (K1+σ+K2/K4 or K1+K3) and of window assembly +
   * result stage (K5/K6), over the tasks polled so far */
  int64_t kernel_launches;
  int64_t scan_launches;        /* launches of the fused scan kernel (pane or select) */
  double scan_ms, assemble_ms;
  /* kernels the plan runs: scan 0 k_select, 1 k_pane_agg, 2 k_pane_cnt,
   * 3 k_pane_bucket; window assembly 0 none (σ/π), 1 k_vh_build + k_win_packed/fused,
   * 2 k_win_block, 3 bucket (k_bkt_count + k_win_scan + k_bkt_emit), 4 hash, 5 slab,
   * 6 k_vh_build + k_win_wide */
  int32_t scan_kind, window_kind;
  /* CTAs per launch of the scan kernel and of the main window-assembly kernel */
  int32_t scan_grid, window_grid;
  /* 1 if window assembly of a task overlaps the next task's scan (SABER_OVERLAP=1) */
  int32_t overlap, reserved;
  /* effective task size φ in tuples: task_bytes / tuple_bytes, lowered for count
   * windows when a task's worst-case rows would not fit one result slot */
  int64_t task_tuples;
} saber_stats;
saber_status saber_query_stats(const saber_query *q, saber_stats *out);

/* Block until all enqueued work of q is complete (results stay pending). */
saber_status saber_query_sync(saber_query *q);
/* Restart q on a new stream with the same plan and buffers (nothing is
 * reallocated).  Every polled slice must have been released (else
 * SABER_EAGAIN); results not yet polled are discarded; the sticky error and
 * the statistics are cleared.  base_index / first_window as in saber_config. */
saber_status saber_query_reset(saber_query *q, int64_t base_index, int64_t first_window);
/* Make `cuda_stream` (a cudaStream_t; NULL = legacy default stream) wait for
 * all work enqueued on q so far, without blocking the host (stream-ordered
 * completion, e.g. for CUDA-event timing around a whole query). */
saber_status saber_query_record(saber_query *q, void *cuda_stream);

void saber_query_destroy(saber_query *q);
/* Human-readable reason for the last error of q (q may be NULL: global). */
const char *saber_last_error(const saber_query *q);

/* ---- task partitioning across GPUs (one process per GPU) -------------------
 * For a contiguous partition [begin, begin+n) of the global stream held in
 * device memory, compute (a) how many windows are closed by the partition's
 * last tuple (all windows with id < *closed_windows end inside or before it)
 * and (b) the first global tuple position its successor needs as a halo:
 * the first tuple of window *closed_windows.  Runs on the GPU (binary search
 * over τ for time windows).  tuples == NULL is allowed for count windows. */
saber_status saber_partition_plan(const saber_schema *schema, const saber_window *window,
                                  const void *dev_tuples, int64_t begin, int64_t n,
                                  int64_t *closed_windows, int64_t *halo_first);

/* ---- windowed θ-join of two streams ----------------------
 * The n-ary query task v = (f^q, <b1, b2>) of PAPER.md §3 L415-422 with the
 * θ-join operator (§2.4; JOIN_r, Table 1), RStream (L401-405).
 * Both streams use the same COUNT window ω(size, slide) (reading A26): window j
 * of the join is W1_j ⋈θ W2_j, W_j = [j·slide, j·slide+size) on each stream,
 * closed once both streams hold j·slide+size tuples.  θ is a conjunction of
 * `S1.col1 op S2.col2` (both integer columns: int64 compare, else double).
 * Every matching pair (a, b) emits one row π1(t1[a]) ++ π2(t2[b]) (projected
 * columns packed in projection order); rows of a window are in (a, b) order;
 * headers as for aggregation (ts = τ of S1's first tuple of the window, A7).
 * Executed as in §5.4: count the matches per (window, row of S1),
 * scan, then write the pairs at their offsets (no quadratic buffers). */
typedef struct { int32_t col1; saber_cmp op; int32_t col2; } saber_join_pred;
typedef struct {
  int32_t npred;  const saber_join_pred *theta;    /* <= 64 terms                    */
  int32_t nproj1; const int32_t *proj1;            /* S1 columns of an output row    */
  int32_t nproj2; const int32_t *proj2;            /* S2 columns (nproj1+nproj2 >= 1) */
} saber_join_op;
typedef struct saber_join saber_join;

/* Create a θ-join.  cfg: device, task_bytes (batch capacity per stream, bytes of
 * S1 tuples) [32 MiB], result_mode, result_bytes (rows per slot) [256 MiB],
 * result_slots [4]; other fields ignored.  Errors: SABER_EINVAL (time windows,
 * bad columns/terms), SABER_ECUDA, SABER_ENOMEM. */
saber_status saber_join_create(const saber_schema *s1, const saber_schema *s2, const saber_join_op *op,
                               const saber_window *window, const saber_config *cfg, saber_join **out);
/* One query task: ntuples tuples of each stream (device pointers, 16-B aligned),
 * ordered after `cuda_stream`'s prior work, which then waits for the task's
 * reads.  SABER_EAGAIN (nothing consumed) when the task's result slot is busy. */
saber_status saber_join_submit_device(saber_join *j, const void *dev1, const void *dev2, size_t ntuples,
                                      void *cuda_stream);
/* The same from host memory (copied before return). */
saber_status saber_join_submit(saber_join *j, const void *host1, const void *host2, size_t ntuples);
/* Next task's slice in task order: nwindows headers, ntuples pair rows of
 * tuple_bytes each in `tuples` (host or device pointers, valid until release).
 * SABER_ENOMEM if the task's pairs exceed result_bytes. */
saber_status saber_join_poll(saber_join *j, saber_results *out, int32_t timeout_us);
saber_status saber_join_release(saber_join *j, const saber_results *r);
void saber_join_destroy(saber_join *j);
const char *saber_join_last_error(const saber_join *j);

/* Library version string. */
const char *saber_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SABER_H */
