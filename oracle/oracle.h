/*
 * oracle.h -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU evaluation of one windowed streaming
 * query, written from the paper's definitions (§2.4):
 * every window is enumerated literally and recomputed from scratch; there are
 * no panes, fragments, tasks or incremental reuse.  Only tests/, the
 * __graft_entry__.smoke() check and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  It shares no code with the CUDA path
 * (paper_conf_sigmod_koliousiswfwcp16_b200/), which never links or calls it.
 *
 * Conventions (readings of the paper):
 *   positions are 0-based; τ is the int64 at ts_off; windows:
 *     count ω(s,l): W_j = [j·l, j·l+s) for j·l+s <= N            (L370-372)
 *     time  ω(s,l): W_j = {i : T0+j·l <= τ_i < T0+j·l+s},
 *                   for T0+j·l+s <= wm (wm = τ_{N-1}+1 by default) (L372-376, A1-A3)
 *   aggregation → RStream (one result relation per window, L392-405)
 *   σ/π         → IStream (tuples of W_j not in W_{j-1}, position identity, A9)
 */
#ifndef SABER_ORACLE_H
#define SABER_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum { OQ_I32 = 0, OQ_I64 = 1, OQ_F32 = 2, OQ_F64 = 3 };
enum { OQ_LT = 0, OQ_LE = 1, OQ_GT = 2, OQ_GE = 3, OQ_EQ = 4, OQ_NE = 5 };
enum { OQ_SUM = 0, OQ_COUNT = 1, OQ_AVG = 2, OQ_MIN = 3, OQ_MAX = 4 };
enum { OQ_COUNTWIN = 0, OQ_TIMEWIN = 1 };
enum { OQ_OK = 0, OQ_EORDER = -1, OQ_EINVAL = -22, OQ_EOVERFLOW = -75 };

typedef struct { int32_t off, type; } oq_col;
typedef struct { int32_t off, type, op; int32_t pad; int64_t ival; double fval; } oq_pred;
typedef struct { int32_t fn, off, type; int32_t pad; } oq_agg;      /* COUNT: off ignored */
typedef struct { int32_t off, type; int64_t div; } oq_key;
typedef struct { int32_t agg, op; int64_t ival; double fval; } oq_have;

typedef struct {
  int32_t tuple_bytes, ts_off;
  int32_t win_kind; int32_t pad;
  int64_t size, slide, origin;
  int32_t npred;  oq_pred pred[64];
  int32_t nproj;  oq_col  proj[16];
  int32_t nagg;   oq_agg  agg[8];
  int32_t nkeys;  oq_key  key[4];
  int32_t nhave;  oq_have have[8];
} oq_query;

typedef struct {
  int32_t error;
  int64_t nwin;
  int64_t *win_id, *win_ts, *win_nrows, *win_rowoff;   /* per window          */
  int64_t nrows;
  int64_t *keys;                                      /* nrows * nkeys       */
  uint64_t *vals;                                     /* nrows * nagg (bits) */
  int32_t val_is_float[8];                            /* per agg: 1 = double */
  int64_t out_bytes;                                  /* IStream bytes       */
  uint8_t *out;
  int64_t row_bytes;                                  /* IStream row width   */
} oq_result;

/* Evaluate the query over tuples[0..n).  watermark is used only for time
 * windows when has_wm != 0, otherwise wm = τ_{n-1}+1.  If window_ids != NULL,
 * only those windows (which must exist) are evaluated, in the given order.
 * nthreads parallelises across windows only; results never depend on it. */
int32_t oq_run(const oq_query *q, const uint8_t *tuples, int64_t n,
               int64_t watermark, int32_t has_wm,
               const int64_t *window_ids, int64_t nids, int32_t nthreads,
               oq_result *out);
/* Number of closed windows (count / time rules above); -1 on error. */
int64_t oq_num_windows(const oq_query *q, const uint8_t *tuples, int64_t n,
                       int64_t watermark, int32_t has_wm);
void oq_free(oq_result *r);

/* Windowed θ-join of two streams (§2.4 L377-383 θ-join per window,
 * RStream L401-405; n-ary query tasks §3; JOIN_r, Table 1).
 * Reading A26: both streams use the same count window ω(s,l);
 * window j of the join is W1_j ⋈θ W2_j with W_j = [j·l, j·l+s) on each stream,
 * for j·l+s <= min(n1, n2); θ is a conjunction of `S1.col1 op S2.col2`
 * (compared as int64 when both columns are integers, else as double); every
 * matching pair (a, b) emits π1(t1[a]) ++ π2(t2[b]), pairs in (a, b) order;
 * the window header ts is τ of t1[j·l] (reading A7). */
typedef struct { int32_t off1, type1, op, off2, type2, pad; } oq_jpred;
typedef struct {
  int32_t tuple_bytes1, tuple_bytes2, ts_off1, pad;
  int64_t size, slide;
  int32_t npred;  oq_jpred pred[64];
  int32_t nproj1; oq_col proj1[16];
  int32_t nproj2; oq_col proj2[16];
} oq_join;
/* out: win_id/win_ts/win_nrows/win_rowoff per window, out/out_bytes the
 * concatenated pair rows, row_bytes their width (nrows = pairs). */
int32_t oq_join_run(const oq_join *q, const uint8_t *t1, int64_t n1, const uint8_t *t2, int64_t n2,
                    int32_t nthreads, oq_result *out);

#ifdef __cplusplus
}
#endif
#endif
