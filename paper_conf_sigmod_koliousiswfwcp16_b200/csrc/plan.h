// plan.h -- query plan and per-query device state shared by the host runtime
// (runtime.cu) and the kernels (kernels.cu).  Product code: nothing here is
// shared with oracle/.
//
// A plan is derived once per query at saber_query_create from the paper's
// query q = (ω, f^q, φ^q) (§2.4):
//   pane length g = gcd(s, l), K = s/g panes per window, L = l/g panes per
//   slide; window j covers panes [j·L, j·L+K)  (panes: L180-181, L1275-1280).
// Pane partials (the window-fragment results f_f of §3) live in a
// device ring of R pane slots indexed by pane id mod R; every slot holds a
// table of C accumulator entries (C = 1 without GROUP BY, G for a declared
// dense key domain, CAP for an open-addressing hash of arbitrary keys).
#pragma once
#include <stdint.h>

namespace sb {

constexpr int kMaxPred = 64, kMaxProj = 16, kMaxAgg = 8, kMaxKey = 4, kMaxField = 8, kMaxHave = 8;
constexpr int kMaxCols = 12;
constexpr int kMaxTupleWords = 64;      // tuples up to 256 bytes

enum { T_I32 = 0, T_I64 = 1, T_F32 = 2, T_F64 = 3 };
enum { OP_LT = 0, OP_LE, OP_GT, OP_GE, OP_EQ, OP_NE };
enum { AG_SUM = 0, AG_COUNT, AG_AVG, AG_MIN, AG_MAX };
enum { KM_GLOBAL = 0, KM_DENSE = 1, KM_HASH = 2 };
enum { KP_RADIX = 0, KP_BIASED64 = 1, KP_BIASED32X2 = 2 };
// accumulator fields (besides the count): fp64 sum, int64 sum, min, max.
// min/max hold an order-preserving u64 encoding of int64 / double values.
enum { FK_SUM_F = 0, FK_SUM_I = 1, FK_MIN = 2, FK_MAX = 3 };
enum { WK_COUNT = 0, WK_TIME = 1 };

// error bits in State::error (first one wins for the status)
enum {
  ERR_ORDER = 1, ERR_TS = 2, ERR_KEY = 4, ERR_CAPACITY = 8, ERR_RESULT = 16, ERR_CARRY = 32
};

struct Pred { int32_t word, type, op, pad; int64_t ival; double fval; };
struct Key  { int32_t word, type, div, pad; int64_t domain, stride; double inv; };   // inv = 1/div
struct Field { int32_t kind, word, type, pad; };
struct AggOut { int32_t fn, field, is_float_col, out_float; };
struct Have { int32_t agg, op, pad0, pad1; int64_t ival; double fval; };

struct Plan {
  // schema
  int32_t tuple_bytes, tuple_words, ts_word, chunk_mask;   // chunk = 16 bytes
  // window ω(s,l), panes
  int32_t win_kind, pad0;
  int64_t s, l, T0, g, K, L;
  double g_inv;                   // 1/g for the reciprocal division in K1
  int32_t g_shift, g_mshift;      // log2(g) if g is a power of two, else -1; magic shift
  uint64_t g_magic;               // floor(x/g) = (x·g_magic) >> g_mshift for 0 <= x < 2^30, g < 2^28
  // σ
  int32_t npred, pad1;
  Pred pred[kMaxPred];
  // π (IStream): output word i of a row comes from tuple word proj_word[i]
  int32_t nproj, out_row_words;
  int32_t proj_word[2 * kMaxProj];
  // α
  int32_t nagg, nf;
  AggOut agg[kMaxAgg];
  Field field[kMaxField];
  // γ
  int32_t nkeys, key_mode, key_pack, pad2;
  Key key[kMaxKey];
  int64_t G;                      // dense key count (DENSE), 1 (GLOBAL)
  int32_t nhave, pad3;
  Have have[kMaxHave];
  // pane ring geometry
  int64_t C;                      // entries per pane slot
  int64_t R;                      // ring slots (power of two)
  int64_t slot_words;             // 8-byte words per slot
  int32_t hash_bits, pad4;        // log2(C) in HASH mode
  // phase-1 warp-private table
  int32_t local_mode;             // 0 LANE (lane-private), 1 DIRECT (warp, atomics), 2 HASHED (one-pane hash)
  int32_t local_entries;          // entries per warp
  int32_t local_pl;               // panes per direct table
  int32_t local_bytes;            // bytes per warp
  int32_t lane_alt;               // DIRECT plan that may switch to LANE per task (time windows)
  int32_t lane_pl, lane_entries, lane_bytes;
  int32_t fast_path, pad6;        // all fields fp64 sums of f32 columns, <= 1 int32 key (div 1), nf <= 2
  int32_t fast_keys, pad7;        // k_pane_agg fast path: as fast_path but up to kMaxKey radix int32 keys, div > 0
  // phase-2 window assembly
  int32_t S, SB, GS, pad5;        // key slabs, slots per slab, threads per slab group
  int32_t state_cap, p2_smem;     // hash state entries per CTA, dynamic smem bytes
  int32_t has_minmax, has_inv;    // min/max fields present; invertible (count/sum) fields
  int32_t slab_mode, pad8;        // HASH + radix keys: compacted key-range buckets, dense slab state
  // output
  int32_t ncols, row_bytes;       // aggregation output columns, bytes per row
  int32_t col_bytes[kMaxCols];
  int64_t col_off[kMaxCols];      // byte offset of each column array in a result slot
  int64_t rows_cap;               // rows per result slot
  int64_t win_cap;                // windows per result slot
  int64_t first_window;           // windows < first_window are not emitted
  int64_t carry_cap;              // IStream: raw tail tuples kept between tasks
  // bucket mode (count windows, one radix key with a large declared domain, fp64
  // sums of f32 columns, no HAVING): the scan writes every tuple's (key offset,
  // values) into a per-(pane, key slab) bucket; window assembly slides a dense
  // per-slab state over the buckets (k_bucket.cu)
  int32_t bucket_mode, bk_shift;  // SB = 1 << bk_shift keys per slab (S = p.S slabs)
  int32_t bk_W, bk_threads;       // windows per assembly chunk, threads per assembly CTA
  int64_t bk_vals;                // byte offset of the value section in the bucket store
  int32_t bk_ctas, pad10;         // emission CTAs per SM
  int32_t win_block, wb_grid;     // short windows over few keys: k_win_block (k_winblock.cu), its grid
  // window phase of task i on a second stream, concurrent with the scan of task
  // i+1 (dense/global pane tables): window kernels read a per-slot snapshot of
  // State, and the pane ring keeps the previous task's windows live
  int32_t overlap, pad9;
  int32_t win_wide, ww_grid;       // many dense keys (256 < C <= 2048): k_win_wide (k_winwide.cu), its grid
  int32_t rounds, pad11;           // kernel rounds per task (State::round_off): time-window aggregation 2, else 1
  int32_t fx_agg, pad12;           // k_pane_agg FX3 tables: sums as three u32 limbs of x·2^32 (DIRECT / SHARED)
  // pane presence bitmaps (k_win_block_reg plans): 8 u32 per ring slot after the
  // table (pane_bm_words), bit k set iff the pane counted key k (flush_entry / flush_fx)
  int32_t pane_bm, pad13;
};

// Per-query device state, updated only by kernels on the query's stream.
struct State {
  int32_t error;                  // ERR_* bits, sticky
  int32_t has_tau;
  int64_t tau_last;               // time windows: last τ seen
  int64_t pos_next;               // global position of the next tuple
  int64_t J0;                     // first window not yet emitted
  int64_t J1;                     // windows closed after the current task
  int64_t zeroed_hi;              // pane slots for panes < zeroed_hi are initialised
  int64_t zero_lo, zero_hi;       // pane range to initialise for the current task
  int64_t pane_hi;                // highest pane touched so far
  int64_t max_probe;              // longest pane-hash probe (HASH mode)
  // current task
  int64_t task_pos, task_n;
  // IStream
  int64_t cover_lo, cover_hi;     // emitted positions of the current task: [cover_lo, cover_hi)
  int64_t carry_pos, carry_n;     // uncovered raw tail kept from earlier tasks
  int32_t carry_sel, first_task;  // which carry buffer is current; first task flag
  int64_t sel_rows;               // rows written by the compaction kernel
  int64_t tile_epoch;             // look-back epoch
  int64_t compacted_hi;           // slab mode: panes < compacted_hi have bucketed lists
  int64_t live_J0;                // overlap: first window of the task whose window phase may still run
  int64_t vh_pre_hi;              // van Herk block-prefix values are valid for panes < vh_pre_hi (k_vh_build_tile)
  // rounds (time-window aggregation): a task is processed as up to Plan::rounds
  // consecutive sub-ranges so that the pane ring never has to hold a time gap
  // (reading A6: the gap's windows still get headers); every round appends its
  // windows and rows to the task's result slot
  int64_t round_off, round_n;     // this round's tuples: [round_off, round_off + round_n) of the task
  int64_t slot_J0;                // first window of the task's result slot
  int64_t row_base, hdr_base;     // rows / windows the earlier rounds of the task wrote into the slot
  int64_t jgap_hi;                // time windows [J1, jgap_hi) are empty (they start after the last data)
};

// Per result slot metadata, copied to the host after a task.
struct SlotMeta {
  int64_t first_window, nwindows, nrows, ntuples;
  int32_t error, pad;
  int64_t pos_end, tau_last;
  int64_t in_tuples, in_panes;    // this task's input tuples and the panes they span
};

}  // namespace sb
