// runtime.cu -- host runtime behind include/saber.h.
//
//   planner     query → Plan (pane length g = gcd(s,l), key regime, table sizes)
//   dispatcher  cuts the submitted byte stream into φ-byte query tasks with
//               monotone task ids (§4.1)
//   ingest      pinned staging ring + H2D on a copy stream, event-chained to the
//               compute stream (the paper's copyin/movein stages, §5.2)
//   moveout     HOST result mode: a mover thread per query issues each finished
//               task's D2H (exact sizes, from its slot metadata) on a second copy
//               stream as soon as the task completes, so result copies overlap the
//               next tasks' H2D and kernels (the moveout stage of Fig. 6)
//   result ring result slot = task id mod slots; poll hands slices out in task
//               order (the ordered output stream of §4.3)
// Every step of a task executes in kernels.cu; nothing here touches tuple data.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <condition_variable>
#include <deque>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../../include/saber.h"
#include "kernels.h"
#include "plan.h"

using namespace sb;

namespace {

thread_local std::string g_last_error;

enum SlotState { SLOT_FREE = 0, SLOT_BUSY = 1, SLOT_POLLED = 2 };

struct Slot {
  SlotDev dev{};
  unsigned char *h_rows = nullptr;
  saber_win_hdr *h_hdr = nullptr;
  SlotMeta *h_meta = nullptr;
  cudaEvent_t done = nullptr;
  cudaEvent_t moved = nullptr;          // HOST mode: the slice's D2H on the moveout stream
  int mstate = 0;                       // HOST mode: 0 not moved, 1 D2H issued, 2 task failed (mv_mu)
  cudaEvent_t scan_done = nullptr;      // overlap plans: the task's scan + epilogue on cs
  cudaEvent_t prof[3] = {nullptr, nullptr, nullptr};
  bool profiled = false, scanned = false;
  int64_t task_id = -1;
  int state = SLOT_FREE;
  SlotMeta meta{};
};

struct Stage {
  unsigned char *h = nullptr;   // pinned
  unsigned char *d = nullptr;   // device
  cudaEvent_t free_ev = nullptr;     // the task reading d[] is done (device buffer reusable)
  cudaEvent_t h2d_ev = nullptr;      // the H2D out of h[] is done (pinned staging reusable)
  bool used = false;
};

constexpr int64_t kDenseMaxPlan = 8192;   // declared key domains up to this use dense pane tables
bool getenv_flag(const char *name) {
  const char *v = std::getenv(name);
  return v && *v && *v != '0';
}
int64_t gcd64(int64_t a, int64_t b) { while (b) { int64_t t = a % b; a = b; b = t; } return a; }
int64_t next_pow2(int64_t x) { int64_t p = 1; while (p < x) p <<= 1; return p; }
int64_t floor_pow2(int64_t x) { int64_t p = 1; while (p * 2 <= x) p <<= 1; return p; }
int type_bytes(int t) { return (t == T_I32 || t == T_F32) ? 4 : 8; }
bool is_float(int t) { return t == T_F32 || t == T_F64; }

}  // namespace

struct saber_query {
  Plan plan{};
  int ncols_schema = 0;
  std::vector<int> col_type, col_off;
  saber_window win{};
  saber_config cfg{};
  int device = 0, nsm = 148;
  int nsm_hint = 148;           // SM count known at planning time
  cudaStream_t cs = nullptr, h2d = nullptr, d2h = nullptr;
  cudaStream_t ws = nullptr;    // overlap plans: window phases (Plan::overlap)
  QueryDev qd{};
  std::vector<Slot> slots;
  std::vector<Stage> stages;
  int cur_stage = 0;
  int64_t stage_fill = 0;       // bytes in stages[cur_stage]
  int64_t task_tuples = 0;
  int64_t next_task = 0, next_poll = 0;
  int p1_grid = 0, p2_grid = 0, sel_grid = 0, win_chunk = 32;
  Plan plan_lane{};             // plan.lane_alt: the same plan with lane-private tables
  int p1_grid_lane = 0;
  bool use_lane = false;        // completed tasks showed long panes (set in poll)
  bool closed = false;
  saber_status sticky = SABER_OK;
  std::string err;
  saber_stats stats{};
  std::vector<std::pair<void *, size_t>> registered;
  std::vector<void *> prereg;   // registered by someone else: never unregistered here
  std::mutex mu;
  // moveout (HOST result mode): task ids whose slices the mover thread copies out
  std::thread mover;
  std::mutex mv_mu;
  std::condition_variable mv_cv;
  std::deque<int64_t> mq;
  int mv_busy = 0;
  bool mv_stop = false;
  int64_t *d_tmp = nullptr;
  int64_t epoch_base = 0;       // look-back epoch offset across saber_query_reset
  int64_t nbegin = 0;           // k_task_begin launches since the last reset (one epoch each)
};

static saber_status fail(saber_query *q, saber_status s, const std::string &msg) {
  if (q) q->err = msg;
  g_last_error = msg;
  return s;
}

#define CK(call)                                                                                 \
  do {                                                                                           \
    cudaError_t e_ = (call);                                                                     \
    if (e_ != cudaSuccess) {                                                                     \
      return fail(q, SABER_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_));          \
    }                                                                                            \
  } while (0)

static saber_status status_from_err(int e) {
  if (e & ERR_ORDER) return SABER_EORDER;
  if (e & ERR_TS) return SABER_ETS;
  if (e & ERR_KEY) return SABER_EKEY;
  if (e & (ERR_CAPACITY | ERR_CARRY)) return SABER_ECAPACITY;
  if (e & ERR_RESULT) return SABER_ENOMEM;
  return SABER_OK;
}
static const char *err_text(int e) {
  if (e & ERR_ORDER) return "timestamps are not non-decreasing (PAPER.md L347-349)";
  if (e & ERR_TS) return "negative timestamp (time domain is {0,1,...}, L349-350)";
  if (e & ERR_KEY) return "GROUP BY key outside its declared domain (or reserved key value)";
  if (e & ERR_CAPACITY) return "pane hash table / pane ring / window state capacity exceeded";
  if (e & ERR_CARRY) return "IStream carry (uncovered tail) exceeds its capacity";
  if (e & ERR_RESULT) return "task output exceeds the result slot capacity (raise result_bytes or lower task_bytes)";
  return "";
}

// ---------------------------------------------------------------------------
// planner
static saber_status build_plan(saber_query *q, const saber_schema *sc, const saber_operator *op,
                               const saber_window *w) {
  Plan &p = q->plan;
  std::memset(&p, 0, sizeof(p));
  if (!sc || !op || !w) return fail(q, SABER_EINVAL, "null argument");
  if (sc->ncols < 1 || !sc->types || !sc->offsets) return fail(q, SABER_EINVAL, "schema needs columns");
  if (sc->tuple_bytes % 16 || sc->tuple_bytes < 16 || sc->tuple_bytes > 64)
    return fail(q, SABER_EINVAL, "tuple_bytes must be 16, 32, 48 or 64");
  q->ncols_schema = sc->ncols;
  for (int c = 0; c < sc->ncols; ++c) {
    int t = sc->types[c], o = sc->offsets[c];
    if (t < 0 || t > 3) return fail(q, SABER_EINVAL, "unknown column type");
    int b = type_bytes(t);
    if (o < 0 || o % b || o + b > sc->tuple_bytes) return fail(q, SABER_EINVAL, "misaligned or out-of-range column");
    q->col_type.push_back(t);
    q->col_off.push_back(o);
  }
  if (sc->ts_col < 0 || sc->ts_col >= sc->ncols || sc->types[sc->ts_col] != SABER_I64)
    return fail(q, SABER_EINVAL, "ts_col must be an I64 column");
  if (w->size < 1 || w->slide < 1) return fail(q, SABER_EINVAL, "window size and slide must be >= 1");
  if (w->slide > w->size) return fail(q, SABER_EINVAL, "slide > size is not supported (PAPER.md L375)");
  if (w->kind != SABER_WIN_COUNT && w->kind != SABER_WIN_TIME) return fail(q, SABER_EINVAL, "window kind");
  if (w->kind == SABER_WIN_TIME && w->origin < 0) return fail(q, SABER_EINVAL, "negative origin");
  if (op->npred < 0 || op->npred > kMaxPred || (op->npred && !op->where)) return fail(q, SABER_EINVAL, "where");
  if (op->nagg < 0 || op->nagg > kMaxAgg || (op->nagg && !op->aggs)) return fail(q, SABER_EINVAL, "aggs");
  if (op->nkeys < 0 || op->nkeys > kMaxKey || (op->nkeys && !op->group_by)) return fail(q, SABER_EINVAL, "group_by");
  if (op->nproj < 0 || op->nproj > kMaxProj || (op->nproj && !op->proj)) return fail(q, SABER_EINVAL, "proj");
  if (op->nhave < 0 || op->nhave > kMaxHave || (op->nhave && !op->having)) return fail(q, SABER_EINVAL, "having");
  if (op->nagg == 0 && op->nproj == 0) return fail(q, SABER_EINVAL, "query needs aggregates or a projection");
  if (op->nagg > 0 && op->nproj > 0) return fail(q, SABER_EINVAL, "projection and aggregation are exclusive");
  if (op->nagg == 0 && (op->nkeys || op->nhave)) return fail(q, SABER_EINVAL, "GROUP BY / HAVING need aggregates");
  if (op->nkeys + op->nagg > kMaxCols) return fail(q, SABER_EINVAL, "too many output columns");

  auto colok = [&](int c) { return c >= 0 && c < sc->ncols; };
  p.tuple_bytes = sc->tuple_bytes;
  p.tuple_words = sc->tuple_bytes / 4;
  p.ts_word = sc->offsets[sc->ts_col] / 4;
  unsigned mask = 1u << (sc->offsets[sc->ts_col] / 16);
  auto use = [&](int c) { mask |= 1u << (sc->offsets[c] / 16); };
  p.win_kind = w->kind == SABER_WIN_TIME ? WK_TIME : WK_COUNT;
  p.s = w->size; p.l = w->slide; p.T0 = w->kind == SABER_WIN_TIME ? w->origin : 0;
  p.g = gcd64(p.s, p.l); p.K = p.s / p.g; p.L = p.l / p.g;
  p.g_inv = 1.0 / (double)p.g;
  p.g_shift = -1;
  if ((p.g & (p.g - 1)) == 0)
    for (int b = 0; b < 63; ++b)
      if ((1ll << b) == p.g) p.g_shift = b;
  // division by the invariant g (Granlund-Montgomery): l = ceil(log2 g),
  // m = floor(2^(32+l)/g) + 1 gives floor(x/g) = floor(x·m / 2^(32+l)) for x < 2^32
  p.g_magic = 0;
  p.g_mshift = 0;
  if (p.g < (1ll << 28)) {
    int lg = 0;
    while ((1ll << lg) < p.g) ++lg;
    p.g_mshift = 32 + lg;
    p.g_magic = (uint64_t)((((unsigned __int128)1) << p.g_mshift) / (unsigned __int128)p.g) + 1;
  }

  p.npred = op->npred;
  for (int i = 0; i < op->npred; ++i) {
    const saber_pred &pr = op->where[i];
    if (!colok(pr.col) || pr.op < SABER_LT || pr.op > SABER_NE) return fail(q, SABER_EINVAL, "bad predicate");
    p.pred[i].word = sc->offsets[pr.col] / 4;
    p.pred[i].type = sc->types[pr.col];
    p.pred[i].op = pr.op;
    p.pred[i].ival = pr.ival;
    p.pred[i].fval = pr.fval;
    use(pr.col);
  }
  p.nproj = op->nproj;
  int ow = 0;
  for (int i = 0; i < op->nproj; ++i) {
    int c = op->proj[i];
    if (!colok(c)) return fail(q, SABER_EINVAL, "bad projection column");
    int nw = type_bytes(sc->types[c]) / 4;
    for (int k = 0; k < nw; ++k) p.proj_word[ow++] = sc->offsets[c] / 4 + k;
    use(c);
  }
  p.out_row_words = ow;

  // aggregates → accumulator fields (shared when equal)
  p.nagg = op->nagg;
  p.nf = 0;
  for (int a = 0; a < op->nagg; ++a) {
    const saber_agg &ag = op->aggs[a];
    if (ag.fn < SABER_SUM || ag.fn > SABER_MAX) return fail(q, SABER_EINVAL, "bad aggregate");
    AggOut &o = p.agg[a];
    o.fn = ag.fn;
    o.field = -1;
    if (ag.fn == SABER_COUNT) { o.is_float_col = 0; o.out_float = 0; continue; }
    if (!colok(ag.col)) return fail(q, SABER_EINVAL, "bad aggregate column");
    int t = sc->types[ag.col];
    use(ag.col);
    int kind = (ag.fn == SABER_MIN) ? FK_MIN : (ag.fn == SABER_MAX) ? FK_MAX : (is_float(t) ? FK_SUM_F : FK_SUM_I);
    int word = sc->offsets[ag.col] / 4;
    int f = -1;
    for (int i = 0; i < p.nf; ++i)
      if (p.field[i].kind == kind && p.field[i].word == word) f = i;
    if (f < 0) {
      if (p.nf == kMaxField) return fail(q, SABER_EINVAL, "too many accumulator fields");
      f = p.nf++;
      p.field[f].kind = kind; p.field[f].word = word; p.field[f].type = t;
    }
    o.field = f;
    o.is_float_col = is_float(t);
    o.out_float = (ag.fn == SABER_AVG) || is_float(t);
    if (kind == FK_MIN || kind == FK_MAX) p.has_minmax = 1;
  }
  // GROUP BY keys
  p.nkeys = op->nkeys;
  bool all_dom = op->nkeys > 0;
  long double prod = 1;
  for (int i = 0; i < op->nkeys; ++i) {
    const saber_keyexpr &k = op->group_by[i];
    if (!colok(k.col) || is_float(sc->types[k.col])) return fail(q, SABER_EINVAL, "GROUP BY needs integer columns");
    if (k.div == 0) return fail(q, SABER_EINVAL, "key divisor is 0");
    if (k.domain < 0) return fail(q, SABER_EINVAL, "negative key domain");
    p.key[i].word = sc->offsets[k.col] / 4;
    p.key[i].type = sc->types[k.col];
    p.key[i].div = k.div;
    p.key[i].inv = 1.0 / (double)k.div;
    p.key[i].domain = k.domain;
    all_dom &= k.domain > 0;
    prod *= (long double)(k.domain > 0 ? k.domain : 1);
    use(k.col);
  }
  const int64_t kDenseMax = kDenseMaxPlan;
  if (op->nkeys == 0) {
    p.key_mode = KM_GLOBAL; p.key_pack = KP_RADIX; p.G = 1;
  } else if (all_dom && prod < 4.0e18L) {
    p.key_pack = KP_RADIX;
    int64_t stride = 1;
    for (int i = op->nkeys - 1; i >= 0; --i) { p.key[i].stride = stride; stride *= p.key[i].domain; }
    p.G = stride;
    p.key_mode = (p.G <= kDenseMax) ? KM_DENSE : KM_HASH;
  } else if (op->nkeys == 1) {
    p.key_pack = KP_BIASED64; p.key_mode = KM_HASH; p.G = 0;
  } else if (op->nkeys == 2) {
    p.key_pack = KP_BIASED32X2; p.key_mode = KM_HASH; p.G = 0;
  } else {
    return fail(q, SABER_EINVAL, "more than two GROUP BY columns need declared domains");
  }
  p.nhave = op->nhave;
  for (int h = 0; h < op->nhave; ++h) {
    const saber_pred &hv = op->having[h];
    if (hv.col < 0 || hv.col >= op->nagg || hv.op < SABER_LT || hv.op > SABER_NE)
      return fail(q, SABER_EINVAL, "bad HAVING term");
    p.have[h].agg = hv.col; p.have[h].op = hv.op; p.have[h].ival = hv.ival; p.have[h].fval = hv.fval;
  }
  p.chunk_mask = (int)mask;
  p.first_window = q->cfg.first_window;
  if (p.first_window < 0) return fail(q, SABER_EINVAL, "first_window < 0");
  return SABER_OK;
}

static saber_status size_plan(saber_query *q) {
  Plan &p = q->plan;
  const saber_config &c = q->cfg;
  q->task_tuples = c.task_bytes / p.tuple_bytes;
  if (q->task_tuples < 1) return fail(q, SABER_EINVAL, "task_bytes smaller than one tuple");
  if (q->task_tuples > (1ll << 31)) return fail(q, SABER_EINVAL, "task_bytes too large (max 2^31 tuples)");
  const int64_t T = q->task_tuples;
  if (p.nagg > 0) {
    // entries per pane slot
    if (p.key_mode == KM_GLOBAL) p.C = 1;
    else if (p.key_mode == KM_DENSE) p.C = p.G;
    else {
      int64_t cap = c.hash_capacity;
      if (cap <= 0) {
        int64_t distinct = p.win_kind == WK_COUNT ? p.g : 4096;
        if (p.key_pack == KP_RADIX && p.G < distinct) distinct = p.G;
        cap = next_pow2(std::max<int64_t>(64, 2 * distinct));
        cap = std::min<int64_t>(cap, 1 << 16);
      }
      if (cap & (cap - 1)) return fail(q, SABER_EINVAL, "hash_capacity must be a power of two");
      p.C = cap;
      int b = 0; while ((1ll << b) < cap) ++b;
      p.hash_bits = b;
    }
    p.slot_words = (p.key_mode == KM_HASH ? p.C : 0) + p.C * (1 + p.nf);
    const int64_t slot_bytes = p.slot_words * 8;
    const int64_t budget = 2ll << 30;
    // time windows: the windows closed next to a time gap read up to K-1 panes past
    // the data while the open ones hold K+L (k_task_begin), so twice that at least
    int64_t need = p.win_kind == WK_TIME ? 2 * (p.K + p.L) + 2 : p.K + p.L + 2;
    int64_t R;
    if (c.max_panes > 0) R = next_pow2(c.max_panes + need);
    else if (p.win_kind == WK_COUNT) R = next_pow2(need + (T + p.g - 1) / p.g + 1);
    else R = std::min(next_pow2(need + (1 << 20)), floor_pow2(std::max<int64_t>(budget / slot_bytes, 1)));
    if (R < need + 16) R = next_pow2(need + 16);
    p.R = R;
    // phase-1 shared-memory tables, fields padded to the NF template:
    //   LANE   (C <= 8 keys): 8 KiB per warp, one column per lane, no atomics (2 CTAs/SM)
    //   DIRECT (small dense C): 2.5 KiB per warp, shared atomics (3 CTAs/SM)
    //   HASHED (large/unbounded C): 5 KiB per warp, one pane at a time (2 CTAs/SM)
    const int nft = p.nf <= 1 ? 1 : p.nf <= 2 ? 2 : p.nf <= 4 ? 4 : 8;
    const int ed = 4 + 8 * nft, eh = 12 + 8 * nft;
    const int lane_budget = 8 * 1024, direct_budget = 2560, hash_budget = 5 * 1024;
    // lane-private tables flush once per few panes: worth it for one key (no GROUP BY:
    // atomics would all hit one address) or count windows with long panes; time
    // windows of unknown rate with several keys take warp tables instead
    const bool lane_ok = p.C == 1 || (p.win_kind == WK_COUNT && p.g >= 64 * p.C);
    if (p.key_mode != KM_HASH && lane_ok && p.C * 2 * 32 * ed <= lane_budget) {
      p.local_mode = 0;
      p.local_pl = (int)std::min<int64_t>(1024, lane_budget / (32 * ed * p.C));
      p.local_entries = p.local_pl * (int)p.C;
      p.local_bytes = ((p.local_entries * 32 * ed) + 15) & ~15;
    } else if (p.key_mode != KM_HASH && p.C * 2 * ed <= direct_budget) {
      p.local_mode = 1;
      // time windows: switch to lane-private tables per task once completed tasks show
      // long panes (>= 64·C tuples per pane), see enqueue_task
      if (p.win_kind == WK_TIME && p.C * 2 * 32 * ed <= lane_budget) {
        p.lane_alt = 1;
        p.lane_pl = (int)std::min<int64_t>(1024, lane_budget / (32 * ed * p.C));
        p.lane_entries = p.lane_pl * (int)p.C;
        p.lane_bytes = ((p.lane_entries * 32 * ed) + 15) & ~15;
      }
      p.local_pl = (int)std::min<int64_t>(1024, direct_budget / (ed * p.C));
      p.local_entries = p.local_pl * (int)p.C;
      p.local_bytes = ((p.local_entries * ed) + 15) & ~15;
    } else if (p.key_mode != KM_HASH && p.C * 2 * ed <= 48 * 1024) {
      // one dense table per CTA, shared atomics (mid-size declared domains)
      const char *kb = std::getenv("SABER_SHARED_KB");
      // 24 KiB: one pane of C5a's 2,048 keys, 3 CTAs/SM (48 KiB gave 2: C5a scan 1.98 -> 2.49 TB/s)
      const int64_t tb = (kb ? std::max(1, std::atoi(kb)) : 24) * 1024;
      p.local_mode = 3;
      p.local_pl = (int)std::max<int64_t>(1, std::min<int64_t>(1024, tb / (ed * p.C)));
      p.local_entries = p.local_pl * (int)p.C;
      p.local_bytes = ((p.local_entries * ed) + 15) & ~15;
    } else {
      p.local_mode = 2;
      p.local_entries = (int)floor_pow2(hash_budget / eh);
      p.local_pl = 1;
      p.local_bytes = ((p.local_entries * eh) + 15) & ~15;
    }
    p.fx_agg = 0;
    {
      bool fast = p.nf <= 2;
      for (int f = 0; f < p.nf; ++f) fast &= p.field[f].kind == FK_SUM_F && p.field[f].type == T_F32;
      if (p.nkeys > 1) fast = false;
      if (p.nkeys == 1)
        fast &= p.key[0].type == T_I32 && p.key[0].div == 1 &&
                ((p.key_pack == KP_RADIX && p.key[0].domain < (1ll << 31)) || p.key_pack == KP_BIASED64);
      p.fast_path = fast ? 1 : 0;
      // generic scan: several radix-packed int32 keys (C5a's plug/household/house,
      // C5b's highway/direction/position÷5280) on the same fast path
      bool fk = p.nf <= 2;
      for (int f = 0; f < p.nf; ++f) fk &= p.field[f].kind == FK_SUM_F && p.field[f].type == T_F32;
      if (p.nkeys > 0 && p.key_pack == KP_RADIX)
        for (int i = 0; i < p.nkeys; ++i)
          fk &= p.key[i].type == T_I32 && p.key[i].div > 0 && p.key[i].domain < (1ll << 31);
      else if (p.nkeys > 0)
        fk &= p.fast_path != 0;
      p.fast_keys = (fk || p.fast_path) ? 1 : 0;
    }
    // k_pane_cnt's FX tables (count-window dense plans, f32 sums as u32 limbs): one
    // CTA-wide table of 6 KiB instead of per-warp copies.  The limbs take
    // fire-and-forget REDs, which never retry under cross-warp contention, so the copies
    // bought nothing but 8x the flush work; one table holds 8 panes of 64 keys, so a
    // flush comes every 8 panes instead of every 3 (C3 G=64 scan 0.788 -> 0.705 ms per
    // 4 GiB task; 24 KiB tables cost the 4th CTA per SM: 0.754).  SABER_CNT_SHARED_KB=0
    // keeps the per-warp tables.
    if (p.win_kind == WK_COUNT && p.key_mode != KM_HASH && p.local_mode == 1 && p1_cnt_fx_plan(p)) {
      const char *ckb = std::getenv("SABER_CNT_SHARED_KB");
      const int kb = ckb ? std::atoi(ckb) : 6;
      if (kb > 0) {
        p.local_mode = 3;
        p.local_pl = (int)std::max<int64_t>(1, std::min<int64_t>(1024, ((int64_t)kb * 1024) / (ed * p.C)));
        p.local_entries = p.local_pl * (int)p.C;
        p.local_bytes = ((p.local_entries * ed) + 15) & ~15;
      }
    }
    // time-window plans with few dense keys (C4): one CTA-wide 24 KiB table instead of
    // per-warp copies (and no lane-table switch) -- C4 R=4096 2.32 -> 2.09 ms, R=64
    // 2.62 -> 2.58 ms per 8 GiB step.  SABER_AGG_SHARED_KB=0 keeps the per-warp tables.
    {
      const char *akb = std::getenv("SABER_AGG_SHARED_KB");
      const int kb = akb ? std::atoi(akb) : 24;
      if (kb > 0 && p.win_kind == WK_TIME && p.key_mode != KM_HASH && p.local_mode == 1) {
        p.local_mode = 3;
        p.lane_alt = 0;
        p.local_pl = (int)std::max<int64_t>(1, std::min<int64_t>(1024, ((int64_t)kb * 1024) / (ed * p.C)));
        p.local_entries = p.local_pl * (int)p.C;
        p.local_bytes = ((p.local_entries * ed) + 15) & ~15;
      }
    }
    // k_pane_agg FX3 tables (atomic DIRECT / SHARED tables of f32 sums): three u32
    // limbs per sum instead of one fp64 word -- re-size the pane window for them
    if (p.fast_keys && p.nf >= 1 && p.nf <= 2 && (p.local_mode == 1 || p.local_mode == 3) &&
        !getenv_flag("SABER_NO_FX")) {
      bool sums = true;
      for (int f = 0; f < p.nf; ++f) sums &= p.field[f].kind == FK_SUM_F && p.field[f].type == T_F32;
      // k_pane_cnt's FX tables hold a u32 count and two u32 limbs (12 B per entry, more
      // panes per flush window); k_pane_agg's FX3 tables three limbs per field
      const int edx = p1_cnt_fx_plan(p) && !getenv_flag("SABER_FX16") ? 12 : 4 + 12 * p.nf;
      // SHARED: at least one pane of C entries, up to 48 KiB (3 CTAs/SM with the 32 KiB stage ring)
      const int64_t budget = p.local_mode == 1 ? direct_budget
                             : std::max<int64_t>(p.local_bytes, std::min<int64_t>(48 * 1024, (int64_t)edx * p.C));
      const int64_t pl = std::min<int64_t>(1024, budget / (edx * p.C));
      if (sums && pl >= 1) {
        p.fx_agg = 1;
        p.local_pl = (int)pl;
        p.local_entries = p.local_pl * (int)p.C;
        p.local_bytes = ((p.local_entries * edx) + 15) & ~15;
      }
    }
    // phase-2 geometry
    const int smem_budget = 96 * 1024;
    if (p.key_mode != KM_HASH) {
      p.GS = p.C <= 256 ? 32 : 256;
      const int gpb = 256 / p.GS;
      int sb = p.GS == 32 ? 256 : 2048;
      while (sb > 1 && (int64_t)gpb * sb * 8 * (1 + p.nf) > smem_budget) sb >>= 1;
      if (sb > p.C) sb = (int)p.C;
      p.SB = sb;
      p.S = (int)((p.C + sb - 1) / sb);
      p.p2_smem = 0;        // van Herk windows keep no state in shared memory
      (void)gpb; (void)smem_budget;
    } else {
      p.GS = 256;
      p.state_cap = (int)floor_pow2(smem_budget / (8 * (2 + 2 * p.nf) + 4));   // keys, counts, fields, compensation, occupancy list
      if (const char *hs = std::getenv("SABER_HASH_STATE")) p.state_cap = (int)floor_pow2(std::max(64, std::atoi(hs)));
      // keys a home slot contributes to an item: one per pane it is occupied in.  Sized for
      // an eighth of the pane slots occupied (hash capacities are planned at >= 2x a pane's
      // distinct keys); an item whose state still overflows restarts split into 2, 4, ...
      // sub-slabs (k_win_hash), so a denser stream costs time, not correctness (CM2: 4 -> 1 slab)
      const double A = (double)(p.K + q->win_chunk * p.L) / 8.0;
      const double B = p.key_pack == KP_RADIX ? (double)p.G / (double)p.C : 1e30;
      const double per_slot = std::max(1e-9, std::min(A, B));
      int64_t sb = floor_pow2(std::max<int64_t>(1, (int64_t)(p.state_cap / (2.0 * per_slot))));
      if (const char *hsb = std::getenv("SABER_HASH_SB")) sb = floor_pow2(std::max(1, std::atoi(hsb)));
      if (sb > p.C) sb = p.C;
      p.SB = (int)sb;
      p.S = (int)(p.C / sb);
      p.p2_smem = p.state_cap * (8 * (2 + 2 * p.nf) + 4);
      // radix-packed keys with a declared domain: key-range slabs with a dense
      // shared-memory state (48 KiB) over compacted pane buckets
      if (p.key_pack == KP_RADIX && p.G < (1ll << 31)) {
        const int64_t slab = floor_pow2((48 * 1024) / (8 * (1 + 2 * p.nf)));
        const int64_t S = (p.G + slab - 1) / slab;
        if (S <= 1024) {
          p.slab_mode = 1;
          q->win_chunk = 128;          // K-pane initialisation amortised over 128 windows
          p.SB = (int)slab;
          p.S = (int)S;
          p.p2_smem = (int)(slab * 8 * (1 + 2 * p.nf));
        }
      }
    }
    // bucket mode: count windows, one int32 key with a large declared domain,
    // fp64 sums of f32 columns, no HAVING (k_bucket.cu).  SB keys per slab so
    // that the slab state (u32 count + nf fp64 sums per key) fits one CTA.
    // Also for mid-size declared domains (1024 <= G <= 8192) when a pane has at least
    // G/4 tuples: dense pane tables would then be about as large as the input.
    // (Measured on B200, C3 1 GiB tasks: G = 256 dense 6.3 ms vs bucket 21.9 ms,
    // G = 512 7.9 vs 13.7, G = 1024 11.5 vs 9.7, G = 2048 21.7 vs 10.5.)
    const bool mid = p.key_mode == KM_DENSE && p.G >= 1024 && p.g * 4 >= p.G;
    if (p.win_kind == WK_COUNT && (p.key_mode == KM_HASH || mid) && p.key_pack == KP_RADIX && p.nkeys == 1 &&
        p.fast_path && p.nhave == 0 && p.nagg <= 4 && p.G >= 256 && p.G <= (1ll << 18) && p.g_magic != 0 &&
        p.g <= 65536 && !getenv_flag("SABER_NO_BUCKET")) {
      const char *sbe = std::getenv("SABER_BK_SB");      // tuning: max keys per slab
      int64_t sb = std::min<int64_t>(sbe ? std::max(256, std::atoi(sbe)) : 16384,
                                     floor_pow2((224 * 1024) / (6 + 8 * p.nf)));    // k_bkt_emit clean layout
      sb = std::min<int64_t>(sb, next_pow2(p.G));
      const int64_t S = (p.G + sb - 1) / sb;
      const int64_t st_max = 16384 / p.tuple_bytes;           // tuples per scan stage
      if (S <= 16 && (st_max / p.g + 2) * S <= 1024) {
        p.bucket_mode = 1;
        p.slab_mode = 0;
        p.SB = (int)sb;
        p.S = (int)S;
        p.bk_shift = 0;
        while ((1ll << p.bk_shift) < sb) ++p.bk_shift;
        p.C = S;
        p.slot_words = S;                                      // per-(pane, slab) fill counters
        const char *bte = std::getenv("SABER_BK_THREADS"), *bce = std::getenv("SABER_BK_CTAS");
        p.bk_threads = (int)std::min<int64_t>(bte ? std::atoi(bte) : 512, sb / 2);   // >= 64 slots per warp
        p.bk_ctas = bce ? std::max(1, std::atoi(bce)) : 1;       // emission CTAs per SM
        p.key_mode = KM_HASH;                                    // no dense pane tables
        // windows per assembly chunk: about one chunk per SM and slab per task
        const int64_t nwt = std::max<int64_t>(1, T / p.l);
        const int64_t per_slab = std::max<int64_t>(1, q->nsm_hint * p.bk_ctas / S);
        p.bk_W = (int)std::max<int64_t>(16, std::min<int64_t>(1024, (nwt + per_slab - 1) / per_slab));
        p.bk_vals = ((p.R * S * p.g * 2) + 255) & ~255ll;
        p.p2_smem = 0;
      }
    }
    // dense / global count-window plans overlap the window phase of a task with the
    // next task's scan (Plan::overlap): the ring then holds two tasks' panes
    if (!p.bucket_mode && !p.slab_mode && p.key_mode != KM_HASH && p.win_kind == WK_COUNT && c.max_panes <= 0 &&
        getenv_flag("SABER_OVERLAP")) {
      const int64_t R2 = next_pow2(2 * ((T + p.g - 1) / p.g + 2) + p.K + p.L + 2);
      if (R2 > p.R && R2 * slot_bytes <= (1ll << 30)) p.R = R2;
    }
    // output columns (keys then aggregates)
    p.ncols = p.nkeys + p.nagg;
    p.row_bytes = 0;
    for (int i = 0; i < p.nkeys; ++i) { p.col_bytes[i] = type_bytes(p.key[i].type); p.row_bytes += p.col_bytes[i]; }
    for (int a = 0; a < p.nagg; ++a) { p.col_bytes[p.nkeys + a] = 8; p.row_bytes += 8; }
    p.win_cap = p.win_kind == WK_COUNT ? T / p.l + 4 : p.R / p.L + 4;
    // time windows: a time gap closes many empty windows at once (headers only,
    // reading A6): room for 2^20 of them per slot, bounded by the per-(window,
    // slab) count array (<= 256 MiB per slot)
    if (p.win_kind == WK_TIME)
      p.win_cap = std::max<int64_t>(p.win_cap, std::min<int64_t>(1 << 20, (256ll << 20) / (8 * std::max(1, p.S))));
    int64_t rows_per_win = p.key_mode == KM_GLOBAL ? 1 : p.key_mode == KM_DENSE ? p.G
                           : p.bucket_mode ? std::min<int64_t>(p.s, p.G)
                           : (p.win_kind == WK_COUNT ? std::min<int64_t>(p.s, p.C * p.K) : p.C * p.K);
    int64_t rb = c.result_bytes;
    if (p.win_kind == WK_COUNT) {
      // a task must not close more rows than one result slot holds (else its
      // emission would fail with SABER_ENOMEM): the dispatcher cuts smaller
      // tasks when the worst case (rows_per_win rows in each of the T/l closed
      // windows) exceeds the slot -- the effective φ is saber_stats.task_tuples
      const int64_t cap = rb > 0 ? rb : (c.result_mode == SABER_RESULTS_DEVICE ? (4ll << 30) : (1ll << 30));
      const int64_t cap_rows = cap / p.row_bytes;
      const int64_t wmax = cap_rows / std::max<int64_t>(1, rows_per_win) - 4;
      if (p.win_cap * rows_per_win > cap_rows && wmax >= 1) {
        q->task_tuples = std::max<int64_t>(p.l, wmax * p.l);
        p.win_cap = q->task_tuples / p.l + 4;
      }
    }
    if (rb <= 0) {
      long double bound = (long double)p.win_cap * rows_per_win * p.row_bytes;
      // device-resident results may use up to 4 GiB per slot; pinned host mirrors stay <= 1 GiB
      const int64_t cap = c.result_mode == SABER_RESULTS_DEVICE ? (4ll << 30) : (1ll << 30);
      rb = (int64_t)std::min<long double>(std::max<long double>(bound, 1 << 20), (long double)cap);
    }
    p.rows_cap = std::max<int64_t>(1, rb / p.row_bytes);
    int64_t off = 0;
    for (int i = 0; i < p.ncols; ++i) {
      p.col_off[i] = off;
      off += ((p.rows_cap * p.col_bytes[i]) + 255) & ~255ll;
    }
  } else {
    // the uncovered tail is < s tuples (count) or spans < s time units (time,
    // rate unknown: sized generously, overflow is SABER_ECAPACITY)
    p.carry_cap = p.win_kind == WK_COUNT ? p.s + p.l + 16 : std::max<int64_t>(T, 1 << 20) + 16;
    p.rows_cap = T + p.carry_cap;
    p.win_cap = p.win_kind == WK_COUNT ? T / p.l + 4 : T + 4;
    p.S = 1;
  }
  return SABER_OK;
}

// ---------------------------------------------------------------------------
static void mover_main(saber_query *q);
static saber_status alloc_query(saber_query *q) {
  Plan &p = q->plan;
  CK(cudaSetDevice(q->device));
  CK(cudaStreamCreateWithFlags(&q->cs, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&q->h2d, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&q->d2h, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&q->ws, cudaStreamNonBlocking));
  CK(cudaMalloc(&q->qd.st, sizeof(State)));
  CK(cudaMalloc(&q->qd.tile_ctr, 64));
  CK(cudaMalloc(&q->d_tmp, 64));
  if (p.nagg > 0) {
    CK(cudaMalloc(&q->qd.table, (size_t)p.R * p.slot_words * 8 + (size_t)p.R * 32));   // + pane bitmaps
    CK(cudaMalloc(&q->qd.pane_ts, (size_t)p.R * 8));
    if (p.key_mode != KM_HASH) {
      CK(cudaMalloc(&q->qd.vh_pre, (size_t)p.R * p.slot_words * 8));
      CK(cudaMalloc(&q->qd.vh_suf, (size_t)p.R * p.slot_words * 8));
    }
    // look-back status of the fused window pass / the window scan: one entry per window chunk
    q->qd.tile_status_cap = p.win_cap + 16;
    CK(cudaMalloc(&q->qd.tile_status, (size_t)q->qd.tile_status_cap * 8));
    CK(cudaMemset(q->qd.tile_status, 0, (size_t)q->qd.tile_status_cap * 8));
    if (p.bucket_mode) {
      CK(cudaMalloc(&q->qd.bkt, (size_t)p.bk_vals + (size_t)p.R * p.S * p.nf * p.g * 4 + 256));
    }
    if (p.slab_mode) {
      CK(cudaMalloc(&q->qd.clist, (size_t)p.R * p.C * (1 + p.nf) * 8));
      CK(cudaMalloc(&q->qd.coff, (size_t)p.R * (p.S + 1) * 4));
    }
  } else {
    q->qd.carry_cap = p.carry_cap;
    CK(cudaMalloc(&q->qd.carry[0], (size_t)p.carry_cap * p.tuple_bytes));
    CK(cudaMalloc(&q->qd.carry[1], (size_t)p.carry_cap * p.tuple_bytes));
    CK(cudaMalloc(&q->qd.sel_stage, (size_t)p.rows_cap * p.out_row_words * 4 + 16));
    CK(cudaMalloc(&q->qd.cta_cnt, 8192 * sizeof(int64_t)));
    CK(cudaMalloc(&q->qd.cta_base, 8192 * sizeof(int64_t)));
    CK(cudaMalloc(&q->qd.ihdr_tmp, (size_t)(p.win_cap + 1) * sizeof(int64_t)));
    // τ at window starts j·l: windows from J0 up to the cover's end (< win_cap + s/l + 2)
    const int64_t nts = p.win_kind == WK_COUNT ? next_pow2(p.win_cap + p.s / p.l + 8) : 1;
    q->qd.ts_mask = nts - 1;
    CK(cudaMalloc(&q->qd.win_ts, (size_t)nts * sizeof(int64_t)));
  }
  const int nslots = q->cfg.result_slots > 0 ? q->cfg.result_slots : 8;
  q->slots.resize(nslots);
  const size_t rows_bytes = p.nagg > 0 ? (size_t)p.col_off[p.ncols - 1] + (((p.rows_cap * p.col_bytes[p.ncols - 1]) + 255) & ~255ll)
                                       : (size_t)p.rows_cap * p.out_row_words * 4;
  for (auto &s : q->slots) {
    CK(cudaMalloc(&s.dev.rows, rows_bytes ? rows_bytes : 16));
    CK(cudaMalloc(&s.dev.hdr, (size_t)p.win_cap * sizeof(saber_win_hdr)));
    // + per (window, 64-key slice) row offsets of k_win_block_reg (dense C <= 256; win_block
    // is decided after the slots exist)
    const int64_t wslices = (p.key_mode != KM_HASH && p.C <= 256) ? std::max<int64_t>(1, p.C / 64) : 1;
    CK(cudaMalloc(&s.dev.counts, (size_t)p.win_cap * std::max<int64_t>({1, p.S, wslices}) * 8));
    CK(cudaMalloc(&s.dev.meta, sizeof(SlotMeta)));
    CK(cudaMalloc(&s.dev.wst, sizeof(State)));
    CK(cudaMalloc(&s.dev.ticket, 64));
    CK(cudaEventCreateWithFlags(&s.scan_done, cudaEventDisableTiming));
    CK(cudaMallocHost(&s.h_meta, sizeof(SlotMeta)));
    if (q->cfg.result_mode == SABER_RESULTS_HOST) {
      CK(cudaMallocHost(&s.h_rows, rows_bytes ? rows_bytes : 16));
      CK(cudaMallocHost(&s.h_hdr, (size_t)p.win_cap * sizeof(saber_win_hdr)));
    }
    CK(cudaEventCreateWithFlags(&s.done, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&s.moved, cudaEventDisableTiming));
    if (q->cfg.profile)
      for (auto &e : s.prof) CK(cudaEventCreate(&e));
  }
  CK(cudaDeviceGetAttribute(&q->nsm, cudaDevAttrMultiProcessorCount, q->device));
  if (p.nagg > 0 && !p.bucket_mode && wb_usable(p) && !getenv_flag("SABER_NO_WINBLOCK")) p.win_block = 1;
  if (p.nagg > 0 && !p.win_block && ww_usable(p) && !getenv_flag("SABER_NO_WINWIDE")) p.win_wide = 1;
  CK(set_kernel_attributes(p));
  if (p.win_block) p.wb_grid = wb_blocks_per_sm(p) * q->nsm;
  // k_win_block_reg plans count rows from the scan's pane presence bitmaps
  if (p.win_block && wb_prepass(p) && p.win_kind == WK_COUNT && p.C % 32 == 0 && p.C <= 256 &&
      !getenv_flag("SABER_NO_PANE_BM"))
    p.pane_bm = 1;
  if (p.win_wide) p.ww_grid = ww_blocks_per_sm(p) * q->nsm;
  // overlap the window phase of task i with the scan of task i+1 (dense / global
  // pane tables): the ring must hold the panes of two tasks' windows at once
  // (opt-in: measured on B200, the concurrent window kernel slows the scan more
  // than it hides -- C3 G=64 3.00 -> 2.84 ms, C4/C5/SG1 10-35% slower)
  if (p.nagg > 0 && !p.bucket_mode && !p.slab_mode && p.key_mode != KM_HASH && getenv_flag("SABER_OVERLAP")) {
    const int64_t T = q->task_tuples;
    // count windows only: time windows run in rounds (gap windows, k_gap_hdr)
    const bool fits = p.win_kind == WK_COUNT && p.R >= 2 * ((T + p.g - 1) / p.g + 2) + p.K + p.L + 2;
    if (fits) p.overlap = 1;
  }
  if (p.overlap) {
    // the scan leaves room on every SM for the previous task's window kernel
    const char *sb = std::getenv("SABER_OVL_SCAN_BPS"), *wb = std::getenv("SABER_OVL_WIN_BPS");
    const int bps = p1_blocks_per_sm(p);
    const int scan_bps = sb ? std::max(1, std::atoi(sb)) : std::max(1, bps - 1);
    const int win_bps = wb ? std::max(1, std::atoi(wb)) : 1;
    q->p1_grid = std::min(bps, scan_bps) * q->nsm;
    q->p2_grid = win_bps * q->nsm;
    if (p.win_block) p.wb_grid = std::min(wb_blocks_per_sm(p), win_bps) * q->nsm;
  } else if (p.bucket_mode) {
    q->p1_grid = bk_scan_blocks_per_sm(p) * q->nsm;
    q->p2_grid = q->nsm;
  } else if (p.nagg > 0) {
    q->p1_grid = p1_blocks_per_sm(p) * q->nsm;
    q->p2_grid = p2_blocks_per_sm(p) * q->nsm * 2;
  } else {
    q->sel_grid = sel_blocks_per_sm(p) * q->nsm;
  }
  // time windows: a task runs in up to 2 rounds (State::round_off, k_task_begin) so
  // that a time gap wider than the pane ring never fails (reading A6)
  if (p.nagg > 0 && p.win_kind == WK_TIME && !p.overlap) {
    const char *re = std::getenv("SABER_ROUNDS");
    p.rounds = re ? std::max(1, std::atoi(re)) : 2;      // one time gap per task
  } else {
    p.rounds = 1;
  }
  if (p.lane_alt) {
    Plan &pl = q->plan_lane;
    pl = p;
    pl.local_mode = 0;
    pl.local_pl = p.lane_pl;
    pl.local_entries = p.lane_entries;
    pl.local_bytes = p.lane_bytes;
    pl.fx_agg = 0;
    CK(set_kernel_attributes(pl));
    const int lbps = p1_blocks_per_sm(pl);
    q->p1_grid_lane = (p.overlap ? std::max(1, lbps - 1) : lbps) * q->nsm;
  }
  CK(launch_init_state(p, q->qd, q->cfg.base_index, 0, q->cs));
  CK(cudaStreamSynchronize(q->cs));
  if (q->cfg.result_mode == SABER_RESULTS_HOST) q->mover = std::thread(mover_main, q);
  return SABER_OK;
}

// wait until the mover has processed every task enqueued so far
static void mover_drain(saber_query *q) {
  if (!q->mover.joinable()) return;
  std::unique_lock<std::mutex> lk(q->mv_mu);
  q->mv_cv.wait(lk, [&] { return q->mq.empty() && !q->mv_busy; });
}

static saber_status check_sticky(saber_query *q) {
  if (q->sticky != SABER_OK) return fail(q, q->sticky, q->err);
  return SABER_OK;
}

// the next n tasks take ring slots next_task .. next_task+n-1 (slot = task id mod
// slots); slices may be released in any order, so every one of those slots must
// be FREE before a submit consumes input (else EAGAIN without consuming)
static bool ring_free(saber_query *q, int64_t n) {
  const int64_t ns = (int64_t)q->slots.size();
  if (n > ns) return false;
  for (int64_t t = 0; t < n; ++t)
    if (q->slots[(q->next_task + t) % ns].state != SLOT_FREE) return false;
  return true;
}

// Moveout: for every enqueued task (task-id order), wait for it, read its slot
// metadata and issue the D2H of exactly its headers and rows into the slot's
// pinned mirror on the moveout stream; poll then only waits for that copy.
static void mover_main(saber_query *q) {
  cudaSetDevice(q->device);
  const Plan &p = q->plan;
  for (;;) {
    int64_t t;
    {
      std::unique_lock<std::mutex> lk(q->mv_mu);
      q->mv_cv.wait(lk, [&] { return q->mv_stop || !q->mq.empty(); });
      if (q->mq.empty()) return;
      t = q->mq.front();
      q->mq.pop_front();
      q->mv_busy = 1;
    }
    Slot &s = q->slots[t % (int64_t)q->slots.size()];
    cudaError_t e = cudaEventSynchronize(s.done);
    const SlotMeta m = *s.h_meta;
    if (e == cudaSuccess && !m.error) {
      if (m.nwindows)
        e = cudaMemcpyAsync(s.h_hdr, s.dev.hdr, (size_t)m.nwindows * sizeof(saber_win_hdr), cudaMemcpyDeviceToHost,
                            q->d2h);
      if (p.nagg > 0) {
        for (int c = 0; c < p.ncols && m.nrows && e == cudaSuccess; ++c)
          e = cudaMemcpyAsync(s.h_rows + p.col_off[c], s.dev.rows + p.col_off[c], (size_t)m.nrows * p.col_bytes[c],
                              cudaMemcpyDeviceToHost, q->d2h);
      } else if (m.ntuples && e == cudaSuccess) {
        e = cudaMemcpyAsync(s.h_rows, s.dev.rows, (size_t)m.ntuples * p.out_row_words * 4, cudaMemcpyDeviceToHost,
                            q->d2h);
      }
      if (e == cudaSuccess) e = cudaEventRecord(s.moved, q->d2h);
    }
    {
      std::lock_guard<std::mutex> lk(q->mv_mu);
      s.mstate = (e == cudaSuccess && !m.error) ? 1 : 2;
      q->mv_busy = 0;
    }
    q->mv_cv.notify_all();
  }
}

// enqueue one task (device-resident tuples) on the compute stream
static saber_status enqueue_task(saber_query *q, const void *dev, int64_t ntuples, int final_, int has_wm, int64_t wm) {
  Slot &s = q->slots[q->next_task % (int64_t)q->slots.size()];
  if (s.state != SLOT_FREE) return fail(q, SABER_EAGAIN, "no free result slot");
  // look-back status words carry 24 bits of the task epoch (common.cuh lb_pack):
  // when the field wraps, stale words of an older task could match, so they are
  // cleared first (flag 0 = unpublished), after every earlier window phase
  bool wraps = false;
  for (int r = 0; r < q->plan.rounds; ++r) wraps |= ((q->epoch_base + q->nbegin + r + 1) & 0xffffff) == 0;
  q->nbegin += q->plan.rounds;
  if (q->plan.nagg > 0 && wraps) {
    if (q->next_task >= 1) {
      Slot &o = q->slots[(q->next_task - 1) % (int64_t)q->slots.size()];
      CK(cudaStreamWaitEvent(q->cs, o.done, 0));
    }
    CK(cudaMemsetAsync(q->qd.tile_status, 0, (size_t)q->qd.tile_status_cap * 8, q->cs));
  }
  const bool lane = q->plan.lane_alt && q->use_lane;
  const Plan &p = lane ? q->plan_lane : q->plan;
  cudaError_t e;
  int launches = 0;
  cudaEvent_t *evs = q->cfg.profile ? s.prof : nullptr;
  cudaStream_t done_stream = q->cs;
  if (p.overlap) {
    // cs runs at most one task ahead of ws: task k's pane-slot initialisation may
    // reuse slots that the window phase of task k-2 read
    if (q->next_task >= 2) {
      Slot &o = q->slots[(q->next_task - 2) % (int64_t)q->slots.size()];
      CK(cudaStreamWaitEvent(q->cs, o.done, 0));
    }
    e = launch_agg_task_overlap(p, q->qd, s.dev, dev, ntuples, final_, has_wm, wm, q->cfg.emit_on_finish,
                                lane ? q->p1_grid_lane : q->p1_grid, q->p2_grid, q->cs, q->ws, s.scan_done,
                                evs, &launches);
    done_stream = q->ws;
  } else if (p.nagg > 0)
    e = launch_agg_task(p, q->qd, s.dev, dev, ntuples, final_, has_wm, wm, q->cfg.emit_on_finish,
                        lane ? q->p1_grid_lane : q->p1_grid,
                        q->p2_grid, q->win_chunk, q->cs, evs, &launches);
  else
    e = launch_select_task(p, q->qd, s.dev, dev, ntuples, final_, has_wm, wm, q->cfg.emit_on_finish, q->sel_grid,
                           q->cs, evs, &launches);
  q->stats.kernel_launches += launches;
  s.profiled = evs != nullptr;
  s.scanned = (p.nagg == 0) || ntuples > 0;
  if (s.scanned) q->stats.scan_launches += 1;
  if (e != cudaSuccess) return fail(q, SABER_ECUDA, std::string("kernel launch: ") + cudaGetErrorString(e));
  CK(cudaMemcpyAsync(s.h_meta, s.dev.meta, sizeof(SlotMeta), cudaMemcpyDeviceToHost, done_stream));
  CK(cudaEventRecord(s.done, done_stream));
  s.state = SLOT_BUSY;
  s.task_id = q->next_task++;
  if (q->mover.joinable()) {
    {
      std::lock_guard<std::mutex> lk(q->mv_mu);
      s.mstate = 0;
      q->mq.push_back(s.task_id);
    }
    q->mv_cv.notify_all();
  }
  q->stats.tasks += 1;
  q->stats.tuples += ntuples;
  q->stats.bytes_in += ntuples * p.tuple_bytes;
  // window-fragment classes of this task (count windows, host closed form)
  if (p.win_kind == WK_COUNT && ntuples > 0) {
    const int64_t b = q->stats.tuples - ntuples + q->cfg.base_index, e2 = b + ntuples;
    int64_t c = 0, o = 0, cl = 0, pe = 0;
    // windows with start in [b, e2) or end-1 in [b, e2) or spanning
    int64_t jlo = (b - p.s + 1) > 0 ? (b - p.s + 1 + p.l - 1) / p.l : 0;   // first window ending >= b
    int64_t jhi = (e2 - 1) / p.l;                                          // last window starting < e2
    for (int64_t j = std::max(jlo, p.first_window); j <= jhi && j - jlo < (1 << 20); ++j) {
      int64_t a = j * p.l, z = a + p.s - 1;
      bool si = a >= b && a < e2, ei = z >= b && z < e2;
      if (si && ei) ++c; else if (si) ++o; else if (ei) ++cl; else ++pe;
    }
    q->stats.last_complete = c; q->stats.last_opening = o; q->stats.last_closing = cl; q->stats.last_pending = pe;
  }
  return SABER_OK;
}

// ---------------------------------------------------------------------------
extern "C" {

const char *saber_version(void) { return "saber-b200 0.1 (sm_100a)"; }

const char *saber_last_error(const saber_query *q) {
  if (q) return q->err.c_str();
  return g_last_error.c_str();
}

saber_status saber_query_create(const saber_schema *schema, const saber_operator *op, const saber_window *window,
                                const saber_config *cfg, saber_query **out) {
  saber_query *q = nullptr;
  if (!out) return fail(nullptr, SABER_EINVAL, "out is NULL");
  *out = nullptr;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < 1) {
    cudaGetLastError();
    return fail(nullptr, SABER_ECUDA, "no CUDA device (there is no CPU path)");
  }
  q = new saber_query();
  if (cfg) q->cfg = *cfg;
  if (q->cfg.task_bytes <= 0) q->cfg.task_bytes = 64ll << 20;
  if (q->cfg.pipeline_depth <= 0) q->cfg.pipeline_depth = 3;
  if (!cfg) q->cfg.emit_on_finish = 1;
  if (q->cfg.result_mode != SABER_RESULTS_HOST && q->cfg.result_mode != SABER_RESULTS_DEVICE) {
    delete q;
    return fail(nullptr, SABER_EINVAL, "result_mode");
  }
  if (cfg && cfg->device >= 0) q->device = cfg->device;
  else cudaGetDevice(&q->device);
  if (q->device >= ndev) { delete q; return fail(nullptr, SABER_EINVAL, "device ordinal"); }
  q->win = *window;
  cudaDeviceGetAttribute(&q->nsm_hint, cudaDevAttrMultiProcessorCount, q->device);
  if (q->nsm_hint <= 0) q->nsm_hint = 148;
  saber_status st = build_plan(q, schema, op, window);
  if (st == SABER_OK) st = size_plan(q);
  if (st == SABER_OK) st = alloc_query(q);
  if (st != SABER_OK) {
    g_last_error = q->err;
    saber_query_destroy(q);
    return st;
  }
  *out = q;
  return SABER_OK;
}

void saber_query_destroy(saber_query *q) {
  if (!q) return;
  if (q->mover.joinable()) {
    {
      std::lock_guard<std::mutex> lk(q->mv_mu);
      q->mv_stop = true;
    }
    q->mv_cv.notify_all();
    q->mover.join();
  }
  cudaSetDevice(q->device);
  if (q->cs) cudaStreamSynchronize(q->cs);
  if (q->h2d) cudaStreamSynchronize(q->h2d);
  if (q->ws) cudaStreamSynchronize(q->ws);
  for (auto &s : q->slots) {
    cudaFree(s.dev.rows); cudaFree(s.dev.hdr); cudaFree(s.dev.counts); cudaFree(s.dev.meta);
    cudaFree(s.dev.wst); cudaFree(s.dev.ticket);
    if (s.scan_done) cudaEventDestroy(s.scan_done);
    cudaFreeHost(s.h_meta); cudaFreeHost(s.h_rows); cudaFreeHost(s.h_hdr);
    if (s.done) cudaEventDestroy(s.done);
    if (s.moved) cudaEventDestroy(s.moved);
    for (auto e : s.prof) if (e) cudaEventDestroy(e);
  }
  for (auto &g : q->stages) {
    cudaFreeHost(g.h); cudaFree(g.d);
    if (g.free_ev) cudaEventDestroy(g.free_ev);
    if (g.h2d_ev) cudaEventDestroy(g.h2d_ev);
  }
  for (auto &r : q->registered)
    if (std::find(q->prereg.begin(), q->prereg.end(), r.first) == q->prereg.end()) cudaHostUnregister(r.first);
  cudaFree(q->qd.st); cudaFree(q->qd.table); cudaFree(q->qd.vh_pre); cudaFree(q->qd.vh_suf);
  cudaFree(q->qd.clist); cudaFree(q->qd.coff); cudaFree(q->qd.bkt); cudaFree(q->qd.sel_stage); cudaFree(q->qd.cta_cnt); cudaFree(q->qd.cta_base); cudaFree(q->qd.ihdr_tmp); cudaFree(q->qd.win_ts); cudaFree(q->qd.pane_ts); cudaFree(q->qd.tile_status);
  cudaFree(q->qd.carry[0]); cudaFree(q->qd.carry[1]); cudaFree(q->qd.tile_ctr); cudaFree(q->d_tmp);
  if (q->cs) cudaStreamDestroy(q->cs);
  if (q->h2d) cudaStreamDestroy(q->h2d);
  if (q->d2h) cudaStreamDestroy(q->d2h);
  if (q->ws) cudaStreamDestroy(q->ws);
  cudaGetLastError();
  delete q;
}

saber_status saber_task_submit_device(saber_query *q, const void *dev_tuples, size_t nbytes, void *cuda_stream) {
  if (!q) return fail(nullptr, SABER_EINVAL, "null query");
  std::lock_guard<std::mutex> lk(q->mu);
  if (saber_status s = check_sticky(q)) return s;
  if (q->closed) return fail(q, SABER_ECLOSED, "submit after finish");
  const Plan &p = q->plan;
  if (nbytes % p.tuple_bytes) return fail(q, SABER_EINVAL, "nbytes is not a multiple of tuple_bytes");
  if (q->stage_fill) return fail(q, SABER_EINVAL, "device submit while host bytes of a partial task are staged");
  const int64_t n = (int64_t)(nbytes / p.tuple_bytes);
  if (n == 0) return SABER_OK;
  if (((uintptr_t)dev_tuples) & 15) return fail(q, SABER_EINVAL, "device tuples must be 16-byte aligned");
  const int64_t ntasks = (n + q->task_tuples - 1) / q->task_tuples;
  if (ntasks > (int64_t)q->slots.size()) return fail(q, SABER_EINVAL, "submit at most result_slots * task_bytes per call");
  if (!ring_free(q, ntasks)) return fail(q, SABER_EAGAIN, "result slots busy: poll and release first");
  CK(cudaSetDevice(q->device));
  cudaStream_t us = (cudaStream_t)cuda_stream;
  cudaEvent_t ev;
  CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  CK(cudaEventRecord(ev, us));
  CK(cudaStreamWaitEvent(q->cs, ev, 0));
  for (int64_t t = 0; t < ntasks; ++t) {
    const int64_t off = t * q->task_tuples;
    const int64_t cnt = std::min(q->task_tuples, n - off);
    saber_status s = enqueue_task(q, (const unsigned char *)dev_tuples + off * p.tuple_bytes, cnt, 0, 0, 0);
    if (s) { cudaEventDestroy(ev); return s; }
  }
  CK(cudaEventRecord(ev, q->cs));
  CK(cudaStreamWaitEvent(us, ev, 0));
  CK(cudaEventDestroy(ev));
  return SABER_OK;
}

static bool is_registered(saber_query *q, const void *p, size_t n) {
  for (auto &r : q->registered)
    if ((const char *)p >= (const char *)r.first && (const char *)p + n <= (const char *)r.first + r.second) return true;
  return false;
}

// device staging buffers are always needed for host submits; pinned host
// staging only for the copyin path (unregistered caller memory)
static saber_status ensure_stages(saber_query *q, bool need_host) {
  const size_t tb = (size_t)q->task_tuples * q->plan.tuple_bytes;
  if (q->stages.empty()) {
    q->stages.resize(q->cfg.pipeline_depth);
    for (auto &g : q->stages) {
      CK(cudaMalloc(&g.d, tb));
      CK(cudaEventCreateWithFlags(&g.free_ev, cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&g.h2d_ev, cudaEventDisableTiming));
    }
  }
  if (need_host)
    for (auto &g : q->stages)
      if (!g.h) CK(cudaMallocHost(&g.h, tb));
  return SABER_OK;
}

// H2D of one task from pinned memory `src` into stage g, then the task itself
static saber_status dispatch_host_task(saber_query *q, Stage &g, const void *src, int64_t ntuples, int final_,
                                       int has_wm, int64_t wm) {
  const size_t bytes = (size_t)ntuples * q->plan.tuple_bytes;
  if (bytes) {
    if (g.used) CK(cudaStreamWaitEvent(q->h2d, g.free_ev, 0));   // the previous task on g.d is done
    CK(cudaMemcpyAsync(g.d, src, bytes, cudaMemcpyHostToDevice, q->h2d));
    CK(cudaEventRecord(g.h2d_ev, q->h2d));
    CK(cudaStreamWaitEvent(q->cs, g.h2d_ev, 0));
  }
  saber_status s = enqueue_task(q, g.d, ntuples, final_, has_wm, wm);
  if (s) return s;
  CK(cudaEventRecord(g.free_ev, q->cs));   // stage reusable once the task's kernels are done
  // the H2D copy of the next task may start now; the copy stream waits for the stage to be free
  g.used = true;
  return SABER_OK;
}

saber_status saber_task_submit(saber_query *q, const void *host_tuples, size_t nbytes) {
  if (!q) return fail(nullptr, SABER_EINVAL, "null query");
  std::lock_guard<std::mutex> lk(q->mu);
  if (saber_status s = check_sticky(q)) return s;
  if (q->closed) return fail(q, SABER_ECLOSED, "submit after finish");
  const Plan &p = q->plan;
  if (nbytes % p.tuple_bytes) return fail(q, SABER_EINVAL, "nbytes is not a multiple of tuple_bytes");
  if (nbytes == 0) return SABER_OK;
  CK(cudaSetDevice(q->device));
  const int64_t tbytes = q->task_tuples * p.tuple_bytes;
  const int64_t whole = ((int64_t)nbytes + q->stage_fill) / tbytes;
  if (whole > (int64_t)q->slots.size())
    return fail(q, SABER_EINVAL, "submit at most result_slots * task_bytes per call");
  if (!ring_free(q, whole)) return fail(q, SABER_EAGAIN, "result slots busy: poll and release first");
  const bool reg = is_registered(q, host_tuples, nbytes);
  const bool copyin = !reg || q->stage_fill > 0 || (int64_t)nbytes % tbytes != 0;
  if (saber_status s = ensure_stages(q, copyin)) return s;
  const unsigned char *src = (const unsigned char *)host_tuples;
  int64_t left = (int64_t)nbytes;
  while (left > 0) {
    Stage &g = q->stages[q->cur_stage];
    if (reg && q->stage_fill == 0 && left >= tbytes) {
      // registered caller memory: DMA straight from it (no copyin stage, no host wait)
      saber_status s = dispatch_host_task(q, g, src, q->task_tuples, 0, 0, 0);
      if (s) return s;
      src += tbytes; left -= tbytes;
      q->cur_stage = (q->cur_stage + 1) % (int)q->stages.size();
      continue;
    }
    // copyin: the pinned stage is rewritten only after its previous H2D completed
    if (q->stage_fill == 0 && g.used) CK(cudaEventSynchronize(g.h2d_ev));
    const int64_t take = std::min(left, tbytes - q->stage_fill);
    std::memcpy(g.h + q->stage_fill, src, (size_t)take);   // copyin (pageable → pinned)
    q->stage_fill += take; src += take; left -= take;
    if (q->stage_fill == tbytes) {
      saber_status s = dispatch_host_task(q, g, g.h, q->task_tuples, 0, 0, 0);
      if (s) return s;
      q->stage_fill = 0;
      q->cur_stage = (q->cur_stage + 1) % (int)q->stages.size();
    }
  }
  return SABER_OK;
}

saber_status saber_register_host(saber_query *q, void *ptr, size_t nbytes) {
  if (!q || !ptr || !nbytes) return fail(q, SABER_EINVAL, "register_host arguments");
  std::lock_guard<std::mutex> lk(q->mu);
  CK(cudaSetDevice(q->device));
  cudaError_t e = cudaHostRegister(ptr, nbytes, cudaHostRegisterDefault);
  cudaPointerAttributes attr{};
  if (e != cudaSuccess && cudaPointerGetAttributes(&attr, ptr) == cudaSuccess && attr.type == cudaMemoryTypeHost)
    e = cudaErrorHostMemoryAlreadyRegistered;
  if (e == cudaErrorHostMemoryAlreadyRegistered) {   // already page-locked (e.g. torch pinned memory)
    cudaGetLastError();
    q->registered.emplace_back(nullptr, 0);
    q->registered.back() = {ptr, nbytes};
    q->prereg.push_back(ptr);
    return SABER_OK;
  }
  if (e != cudaSuccess) return fail(q, SABER_ECUDA, std::string("cudaHostRegister: ") + cudaGetErrorString(e));
  q->registered.emplace_back(ptr, nbytes);
  return SABER_OK;
}

saber_status saber_query_finish(saber_query *q, int64_t watermark) {
  if (!q) return fail(nullptr, SABER_EINVAL, "null query");
  std::lock_guard<std::mutex> lk(q->mu);
  if (saber_status s = check_sticky(q)) return s;
  if (q->closed) return fail(q, SABER_ECLOSED, "finish called twice");
  CK(cudaSetDevice(q->device));
  const int need = 1 + (q->stage_fill > 0);
  if (!ring_free(q, need)) return fail(q, SABER_EAGAIN, "result slots busy: poll and release first");
  const int has_wm = watermark != INT64_MIN;
  if (q->stage_fill > 0) {
    Stage &g = q->stages[q->cur_stage];
    saber_status s = dispatch_host_task(q, g, g.h, q->stage_fill / q->plan.tuple_bytes, 0, 0, 0);
    if (s) return s;
    q->stage_fill = 0;
    q->cur_stage = (q->cur_stage + 1) % (int)q->stages.size();
  }
  saber_status s = enqueue_task(q, nullptr, 0, 1, has_wm, watermark);
  if (s) return s;
  q->closed = true;
  return SABER_OK;
}

saber_status saber_results_poll(saber_query *q, saber_results *out, int32_t timeout_us) {
  if (!q || !out) return fail(q, SABER_EINVAL, "poll arguments");
  std::lock_guard<std::mutex> lk(q->mu);
  std::memset(out, 0, sizeof(*out));
  if (q->next_poll >= q->next_task) return fail(q, SABER_EAGAIN, "no pending task");
  Slot &s = q->slots[q->next_poll % (int64_t)q->slots.size()];
  if (s.state != SLOT_BUSY || s.task_id != q->next_poll) return fail(q, SABER_EINVAL, "result ring out of order");
  CK(cudaSetDevice(q->device));
  const auto t0 = std::chrono::steady_clock::now();
  auto left_us = [&]() -> int64_t {
    return timeout_us - std::chrono::duration_cast<std::chrono::microseconds>(std::chrono::steady_clock::now() - t0).count();
  };
  auto wait_ev = [&](cudaEvent_t ev) -> saber_status {
    if (timeout_us < 0) {
      CK(cudaEventSynchronize(ev));
      return SABER_OK;
    }
    for (;;) {
      cudaError_t e = cudaEventQuery(ev);
      if (e == cudaSuccess) return SABER_OK;
      if (e != cudaErrorNotReady) CK(e);
      cudaGetLastError();
      if (left_us() <= 0) return fail(q, SABER_EAGAIN, "poll timeout");
      std::this_thread::sleep_for(std::chrono::microseconds(20));
    }
  };
  if (saber_status w = wait_ev(s.done)) return w;
  const bool host_mv = q->cfg.result_mode == SABER_RESULTS_HOST && q->mover.joinable();
  if (host_mv) {
    // the mover issued (or skipped, for a failed task) this slice's D2H
    int ms;
    {
      std::unique_lock<std::mutex> lk(q->mv_mu);
      auto ready = [&] { return s.mstate != 0; };
      if (timeout_us < 0) q->mv_cv.wait(lk, ready);
      else if (!q->mv_cv.wait_for(lk, std::chrono::microseconds(std::max<int64_t>(0, left_us())), ready))
        return fail(q, SABER_EAGAIN, "poll timeout");
      ms = s.mstate;
    }
    if (ms == 1)
      if (saber_status w = wait_ev(s.moved)) return w;
  }
  s.meta = *s.h_meta;
  const Plan &p = q->plan;
  // pane density of large tasks picks the phase-1 table layout of later tasks
  if (p.lane_alt && s.meta.in_tuples >= (1 << 20) && s.meta.in_panes > 0)
    q->use_lane = s.meta.in_tuples >= 64 * p.C * s.meta.in_panes;
  if (s.profiled) {
    float a = 0, b = 0;
    if (cudaEventElapsedTime(&a, s.prof[0], s.prof[1]) == cudaSuccess && s.scanned) q->stats.scan_ms += a;
    if (cudaEventElapsedTime(&b, s.prof[1], s.prof[2]) == cudaSuccess) q->stats.assemble_ms += b;
    cudaGetLastError();
    s.profiled = false;
  }
  if (s.meta.error) {
    q->sticky = status_from_err(s.meta.error);
    return fail(q, q->sticky, err_text(s.meta.error));
  }
  out->task_id = s.task_id;
  out->first_window = s.meta.first_window;
  out->nwindows = s.meta.nwindows;
  out->nrows = s.meta.nrows;
  out->ntuples = s.meta.ntuples;
  const bool host = q->cfg.result_mode == SABER_RESULTS_HOST;
  out->on_device = !host;
  if (p.nagg > 0) {
    out->ncols = p.ncols;
    for (int c = 0; c < p.ncols; ++c) out->col_bytes[c] = p.col_bytes[c];
    unsigned char *rows = host ? s.h_rows : s.dev.rows;
    out->hdr = host ? s.h_hdr : (const saber_win_hdr *)s.dev.hdr;
    for (int c = 0; c < p.ncols; ++c) out->cols[c] = rows + p.col_off[c];
  } else {
    out->tuple_bytes = p.out_row_words * 4;
    out->tuples = host ? (const void *)s.h_rows : (const void *)s.dev.rows;
    // per-window headers: row_offset / nrows count projected tuples (reading A9)
    out->hdr = host ? s.h_hdr : (const saber_win_hdr *)s.dev.hdr;
  }
  q->stats.windows += s.meta.nwindows;
  q->stats.rows += s.meta.nrows;
  q->stats.out_tuples += s.meta.ntuples;
  s.state = SLOT_POLLED;
  q->next_poll++;
  return SABER_OK;
}

saber_status saber_results_release(saber_query *q, const saber_results *r) {
  if (!q || !r) return fail(q, SABER_EINVAL, "release arguments");
  std::lock_guard<std::mutex> lk(q->mu);
  Slot &s = q->slots[r->task_id % (int64_t)q->slots.size()];
  if (s.task_id != r->task_id || s.state != SLOT_POLLED) return fail(q, SABER_EINVAL, "slice not polled or released twice");
  s.state = SLOT_FREE;
  return SABER_OK;
}

saber_status saber_query_stats(const saber_query *q, saber_stats *out) {
  if (!q || !out) return SABER_EINVAL;
  *out = q->stats;
  out->tasks_pending = q->next_task - q->next_poll;
  const Plan &p = q->plan;
  out->scan_kind = p.nagg == 0 ? 0 : p.bucket_mode ? 3 : p1_is_cnt(p) ? 2 : 1;
  out->window_kind = p.nagg == 0 ? 0 : p.bucket_mode ? 3 : p.slab_mode ? 5 : p.key_mode == KM_HASH ? 4
                     : p.win_block ? 2 : p.win_wide ? 6 : 1;
  out->scan_grid = p.nagg == 0 ? q->sel_grid : (p.lane_alt && q->use_lane) ? q->p1_grid_lane : q->p1_grid;
  out->window_grid = p.win_block ? p.wb_grid : p.win_wide ? p.ww_grid : q->p2_grid;
  out->overlap = p.overlap;
  out->task_tuples = q->task_tuples;
  return SABER_OK;
}

saber_status saber_query_reset(saber_query *q, int64_t base_index, int64_t first_window) {
  if (!q || base_index < 0 || first_window < 0) return fail(q, SABER_EINVAL, "reset arguments");
  std::lock_guard<std::mutex> lk(q->mu);
  for (auto &s : q->slots)
    if (s.state == SLOT_POLLED) return fail(q, SABER_EAGAIN, "release every polled slice before reset");
  CK(cudaSetDevice(q->device));
  mover_drain(q);
  CK(cudaStreamSynchronize(q->h2d));
  CK(cudaStreamSynchronize(q->cs));
  CK(cudaStreamSynchronize(q->ws));
  CK(cudaStreamSynchronize(q->d2h));
  for (auto &s : q->slots) { s.state = SLOT_FREE; s.task_id = -1; s.profiled = false; s.mstate = 0; }
  for (auto &g : q->stages) g.used = false;
  q->cfg.base_index = base_index;
  q->cfg.first_window = first_window;
  q->plan.first_window = first_window;
  q->stage_fill = 0;
  q->cur_stage = 0;
  q->closed = false;
  q->sticky = SABER_OK;
  q->err.clear();
  q->stats = saber_stats{};
  // task ids restart at 0; look-back epochs continue past every task run so far
  q->epoch_base += q->nbegin + 1;
  q->nbegin = 0;
  q->next_task = q->next_poll = 0;
  CK(launch_init_state(q->plan, q->qd, base_index, q->epoch_base, q->cs));
  CK(cudaStreamSynchronize(q->cs));
  return SABER_OK;
}

saber_status saber_query_sync(saber_query *q) {
  if (!q) return SABER_EINVAL;
  CK(cudaSetDevice(q->device));
  CK(cudaStreamSynchronize(q->cs));
  CK(cudaStreamSynchronize(q->ws));
  return SABER_OK;
}

saber_status saber_query_record(saber_query *q, void *cuda_stream) {
  if (!q) return SABER_EINVAL;
  std::lock_guard<std::mutex> lk(q->mu);
  CK(cudaSetDevice(q->device));
  cudaEvent_t ev;
  CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  CK(cudaEventRecord(ev, q->cs));
  CK(cudaStreamWaitEvent((cudaStream_t)cuda_stream, ev, 0));
  CK(cudaEventRecord(ev, q->ws));
  CK(cudaStreamWaitEvent((cudaStream_t)cuda_stream, ev, 0));
  CK(cudaEventDestroy(ev));
  return SABER_OK;
}

saber_status saber_partition_plan(const saber_schema *schema, const saber_window *window, const void *dev_tuples,
                                  int64_t begin, int64_t n, int64_t *closed_windows, int64_t *halo_first) {
  saber_query *q = nullptr;
  if (!schema || !window || !closed_windows || !halo_first || n < 0 || begin < 0)
    return fail(nullptr, SABER_EINVAL, "partition_plan arguments");
  if (window->size < 1 || window->slide < 1 || window->slide > window->size)
    return fail(nullptr, SABER_EINVAL, "window");
  if (schema->ts_col < 0 || schema->ts_col >= schema->ncols) return fail(nullptr, SABER_EINVAL, "ts_col");
  const int ts_word = schema->offsets[schema->ts_col] / 4;
  if (window->kind == SABER_WIN_COUNT) {
    int64_t total = begin + n;
    *closed_windows = total >= window->size ? (total - window->size) / window->slide + 1 : 0;
    *halo_first = *closed_windows * window->slide;
    return SABER_OK;
  }
  if (n == 0) { *closed_windows = 0; *halo_first = begin; return SABER_OK; }
  if (!dev_tuples) return fail(nullptr, SABER_EINVAL, "time windows need the partition's tuples");
  int64_t *d = nullptr;
  CK(cudaMalloc(&d, 16));
  CK(launch_partition_plan(ts_word, schema->tuple_bytes / 4, 1, window->size, window->slide, window->origin,
                           dev_tuples, begin, n, d, 0));
  int64_t h[2];
  CK(cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost));
  cudaFree(d);
  if (h[0] < 0) return fail(nullptr, SABER_EINVAL, "partition is shorter than the window span");
  *closed_windows = h[0];
  *halo_first = h[1];
  return SABER_OK;
}

}  // extern "C"
