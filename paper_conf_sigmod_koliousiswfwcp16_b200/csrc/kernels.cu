// kernels.cu -- the sm_100a kernels of one SABER query task.
//
//   k_task_begin   scalar task prologue: window-closing rule, pane range, IStream cover
//   k_zero_panes   initialise the pane-ring slots a task is about to touch
//   k_pane_agg     K1+σ+K2/K4 fused: one pass over the task's tuples; each tuple
//                  gets its pane (count: position/g; time: (τ-T0)/g), is filtered
//                  by σ, keyed, pre-aggregated in a warp-private shared-memory
//                  table (warp match/shuffle dedup, no shared atomics) and the
//                  table is flushed into the device pane ring with L2 atomics
//   k_win_dense /  window assembly (the batch operator f_b, §3):
//   k_win_hash     sliding over pane partials (+new panes, -expired panes) for
//                  count/sum/avg, direct K-pane recompute for min/max; run twice,
//                  COUNT pass (rows per window) then EMIT pass (rows written)
//   k_win_scan     window headers + row offsets (result-stage ordering, §4.3)
//   k_task_end     publish slot metadata, advance the emitted-window cursor
//   k_select       σ/π with stream compaction (§5.4): ballot/popc,
//                  block scan, decoupled look-back across tiles, in-order scatter
//   k_carry        keep the uncovered raw tail (< one slide) for the next task
#include <cuda_runtime.h>
#include <stdint.h>

#include "device_util.cuh"
#include "kernels.h"

namespace sb {

struct WinHdr { int64_t window_id, ts, row_offset; int32_t nrows, flags; };

constexpr int kP1Threads = 256;
constexpr int kWarpTile = 1024;       // tuples per warp tile (32 iterations of 32 lanes)
constexpr int kP1Unroll = 4;
constexpr int kSelThreads = 256;
constexpr int kSelPer = 8;            // tuples per thread per tile
constexpr int kSelTile = kSelThreads * kSelPer;

// --------------------------------------------------------------------------
// generic tuple access
template <int NW>
__device__ __forceinline__ void load_tuple(const uint4 *t, unsigned mask, uint32_t (&w)[NW]) {
#pragma unroll
  for (int c = 0; c < NW / 4; ++c) {
    uint4 v = make_uint4(0, 0, 0, 0);
    if (mask & (1u << c)) v = ld_stream(t + c);
    w[4 * c + 0] = v.x; w[4 * c + 1] = v.y; w[4 * c + 2] = v.z; w[4 * c + 3] = v.w;
  }
}

template <int NW>
__device__ __forceinline__ bool eval_preds(const Plan &p, const uint32_t (&w)[NW]) {
  bool ok = true;
  for (int i = 0; i < p.npred; ++i) {
    const Pred &pr = p.pred[i];
    if (pr.type == T_F32 || pr.type == T_F64) ok &= cmp_op(get_float<NW>(w, pr.word, pr.type), pr.op, pr.fval);
    else ok &= cmp_op(get_int<NW>(w, pr.word, pr.type), pr.op, pr.ival);
  }
  return ok;
}

// GROUP BY key of a tuple (reading A17); flags ERR_KEY.
template <int NW>
__device__ __forceinline__ uint64_t make_key(const Plan &p, const uint32_t (&w)[NW], bool &valid, int &err) {
  if (p.key_mode == KM_GLOBAL) return 0;
  int64_t v[kMaxKey];
#pragma unroll
  for (int i = 0; i < kMaxKey; ++i) {
    v[i] = 0;
    if (i < p.nkeys) {
      v[i] = get_int<NW>(w, p.key[i].word, p.key[i].type);
      if (p.key[i].div != 1) v[i] /= p.key[i].div;
    }
  }
  uint64_t k = 0;
  bool bad = false;
  if (p.key_pack == KP_RADIX) {
#pragma unroll
    for (int i = 0; i < kMaxKey; ++i)
      if (i < p.nkeys) {
        bad |= (v[i] < 0) | (v[i] >= p.key[i].domain);
        k += (uint64_t)v[i] * (uint64_t)p.key[i].stride;
      }
  } else if (p.key_pack == KP_BIASED64) {
    k = (uint64_t)v[0] ^ 0x8000000000000000ull;
    bad = (k == kEmpty);
  } else {
    bad = (v[0] != (int32_t)v[0]) | (v[1] != (int32_t)v[1]);
    k = ((uint64_t)((uint32_t)v[0] ^ 0x80000000u) << 32) | (uint64_t)((uint32_t)v[1] ^ 0x80000000u);
    bad |= (k == kEmpty);
  }
  if (valid && bad) { err |= ERR_KEY; valid = false; }
  return k;
}

template <int NW>
__device__ __forceinline__ uint64_t field_value(const Field &f, const uint32_t (&w)[NW]) {
  bool fl = (f.type == T_F32 || f.type == T_F64);
  switch (f.kind) {
    case FK_SUM_F: return (uint64_t)__double_as_longlong(get_float<NW>(w, f.word, f.type));
    case FK_SUM_I: return (uint64_t)get_int<NW>(w, f.word, f.type);
    default: return fl ? enc_dbl(get_float<NW>(w, f.word, f.type)) : enc_int(get_int<NW>(w, f.word, f.type));
  }
}

__device__ __forceinline__ int64_t cnt_off(const Plan &p) { return p.key_mode == KM_HASH ? p.C : 0; }
__device__ __forceinline__ int64_t fld_off(const Plan &p, int f) { return cnt_off(p) + (int64_t)(1 + f) * p.C; }

// --------------------------------------------------------------------------
// task prologue (one warp)
__device__ __forceinline__ int64_t tau_at(const Plan &p, const unsigned char *t, int64_t i) {
  return *(const int64_t *)(t + i * p.tuple_bytes + 4 * p.ts_word);
}

// lower_bound over the concatenation [a (na tuples) ++ b (nb tuples)] of τ < key (warp-cooperative)
__device__ int64_t warp_lower_bound(const Plan &p, const unsigned char *a, int64_t na,
                                    const unsigned char *b, int64_t nb, int64_t key) {
  const int lane = threadIdx.x & 31;
  int64_t lo = 0, hi = na + nb;
  while (lo < hi) {
    int64_t span = hi - lo;
    int64_t idx = (span <= 32) ? lo + lane : lo + (span * lane) / 32;
    bool inb = idx < hi;
    int64_t t = 0;
    if (inb) t = idx < na ? tau_at(p, a, idx) : tau_at(p, b, idx - na);
    bool pred = inb && t < key;
    unsigned bal = __ballot_sync(kFull, pred);
    int c = __popc(bal);
    if (span <= 32) { lo = lo + c; break; }
    if (c == 0) { hi = lo; break; }
    int64_t prev = lo + (span * (c - 1)) / 32;
    int64_t next = (c < 32) ? lo + (span * c) / 32 : hi;
    lo = prev + 1;
    hi = next;
  }
  return lo;
}

__global__ void k_task_begin(const Plan p, State *st, const unsigned char *tup, int64_t n, int final_,
                             int has_wm, int64_t wm, int emit_on_finish, SlotMeta *meta,
                             const unsigned char *carry0, const unsigned char *carry1, int *tile_ctr) {
  const int lane = threadIdx.x;
  __shared__ int64_t sh[8];
  if (lane == 0) {
    int err = 0;
    const int64_t pos0 = st->pos_next;
    st->task_pos = pos0;
    st->task_n = n;
    int64_t J0 = st->J0, J1 = J0;
    int64_t plo = 0, phi = -1;
    if (n > 0) {
      int64_t tf = tau_at(p, tup, 0), tl = tau_at(p, tup, n - 1);
      if (tf < 0) err |= ERR_TS;
      if (st->has_tau && tf < st->tau_last) err |= ERR_ORDER;
      if (!st->has_tau || tl > st->tau_last) st->tau_last = tl;
      st->has_tau = 1;
    }
    if (p.win_kind == WK_TIME) {
      if (n > 0) {
        int64_t tf = tau_at(p, tup, 0), tl = tau_at(p, tup, n - 1);
        if (tl >= p.T0) {
          plo = tf >= p.T0 ? (tf - p.T0) / p.g : 0;
          phi = (tl - p.T0) / p.g;
        }
      }
      // window j = [T0+j·l, T0+j·l+s) is closed once a tuple with τ >= its end has
      // arrived (τ non-decreasing, L347-349) or the watermark passed it (reading A3)
      bool use_wm = final_ && emit_on_finish;
      int64_t B;
      bool haveB = true;
      if (use_wm && has_wm) B = wm;
      else if (use_wm) { B = st->tau_last + 1; haveB = st->has_tau; }
      else { B = st->tau_last; haveB = st->has_tau; }
      if (haveB && B - p.T0 - p.s >= 0) J1 = (B - p.T0 - p.s) / p.l + 1;
    } else {
      int64_t total = pos0 + n;   // count: W_j = [j·l, j·l+s) closes with position j·l+s-1
      if (total >= p.s) J1 = (total - p.s) / p.l + 1;
      if (n > 0) { plo = pos0 / p.g; phi = (total - 1) / p.g; }
    }
    if (J1 < J0) J1 = J0;
    st->pos_next = pos0 + n;
    st->J1 = J1;
    // pane ring: slots of panes [J0·L, phi] must coexist during this task
    int64_t live_lo = J0 * p.L;
    int64_t zlo = st->zeroed_hi > live_lo ? st->zeroed_hi : live_lo;
    int64_t zhi = zlo;
    if (phi >= 0 && p.nagg > 0) {
      if (phi - live_lo + 1 > p.R) err |= ERR_CAPACITY;
      else if (phi + 1 > zlo) zhi = phi + 1;
    }
    st->zero_lo = zlo;
    st->zero_hi = zhi;
    if (zhi > st->zeroed_hi) st->zeroed_hi = zhi;
    if (phi > st->pane_hi) st->pane_hi = phi;
    (void)plo;
    if (J1 - J0 > p.win_cap) err |= ERR_RESULT;
    meta->first_window = J0;
    meta->nwindows = J1 - J0;
    if (err) st->error |= err;
    st->tile_epoch += 1;
    st->sel_rows = 0;
    *tile_ctr = 0;
    sh[0] = J0; sh[1] = J1; sh[2] = pos0;
  }
  __syncwarp();
  if (p.nagg > 0) return;
  // ---- IStream cover (L395-400): emit selected tuples of window positions not
  // emitted before; the virtual input is [carry ++ task]
  const int64_t J0 = sh[0], J1 = sh[1], pos0 = sh[2];
  const unsigned char *carry = st->carry_sel ? carry1 : carry0;
  const int64_t cpos = st->carry_pos, cn = st->carry_n;
  int64_t cover_lo = st->cover_hi;
  int64_t cover_hi;
  if (p.win_kind == WK_COUNT) {
    if (st->first_task) cover_lo = J0 > 0 ? (J0 - 1) * p.l + p.s : 0;
    cover_hi = J1 > 0 ? (J1 - 1) * p.l + p.s : cover_lo;
  } else {
    if (st->first_task) {
      int64_t B = J0 > 0 ? p.T0 + (J0 - 1) * p.l + p.s : p.T0;
      cover_lo = cpos + warp_lower_bound(p, carry, cn, tup, n, B);
    }
    if (J1 > 0) {
      int64_t B = p.T0 + (J1 - 1) * p.l + p.s;
      cover_hi = cpos + warp_lower_bound(p, carry, cn, tup, n, B);
    } else {
      cover_hi = cover_lo;
    }
  }
  if (lane == 0) {
    if (cover_hi < cover_lo) cover_hi = cover_lo;
    const int64_t end = pos0 + n;
    if (cover_lo < cpos) cover_lo = cpos;
    if (cover_hi > end) cover_hi = end;
    st->cover_lo = cover_lo;
    st->cover_hi = cover_hi;
    st->first_task = 0;
    // the uncovered tail [max(cover_hi, cpos), end) is carried to the next task
    int64_t ncp = cover_hi > cpos ? cover_hi : cpos;
    st->zero_lo = ncp;            // reused: new carry position
    st->zero_hi = end - ncp;      // reused: new carry length
    if (end - ncp > p.carry_cap) st->error |= ERR_CARRY;
  }
}

// --------------------------------------------------------------------------
__global__ void k_zero_panes(const Plan p, const State *st, uint64_t *table) {
  const int64_t lo = st->zero_lo, hi = st->zero_hi;
  if (hi <= lo) return;
  const int64_t words = (hi - lo) * p.slot_words;
  const int64_t co = cnt_off(p);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < words;
       i += (int64_t)gridDim.x * blockDim.x) {
    int64_t pane = lo + i / p.slot_words;
    int64_t w = i % p.slot_words;
    uint64_t v;
    if (w < co) v = kEmpty;                               // hash keys
    else if (w < co + p.C) v = 0;                         // counts
    else v = field_identity(p.field[(w - co - p.C) / p.C].kind);
    table[(pane & (p.R - 1)) * p.slot_words + w] = v;
  }
}

// --------------------------------------------------------------------------
// phase 1: fused boundary scan + σ + pane partial aggregation
struct P1Warp {
  unsigned char *base;
  uint64_t *keys;     // hashed local table only
  uint64_t *f;        // [nf][TE]
  uint32_t *cnt;      // [TE]
  int TE;
};

__device__ __forceinline__ int64_t global_insert(const Plan &p, State *st, uint64_t *gkeys, uint64_t k, int &err) {
  const uint32_t mask = (uint32_t)p.C - 1;
  uint32_t h = (uint32_t)fmix64(k) & mask;
  for (int64_t probe = 0; probe < p.C; ++probe) {
    uint64_t cur = __ldcg((const unsigned long long *)&gkeys[h]);
    if (cur == k) return h;
    if (cur == kEmpty) {
      uint64_t old = atomicCAS((unsigned long long *)&gkeys[h], kEmpty, k);
      if (old == kEmpty || old == k) {
        if (probe > 0) atomicMax((unsigned long long *)&st->max_probe, (unsigned long long)probe);
        return h;
      }
    }
    h = (h + 1) & mask;
  }
  err |= ERR_CAPACITY;
  return -1;
}

// add one pre-aggregated (pane, key) entry into the device pane ring
__device__ __forceinline__ void flush_entry(const Plan &p, State *st, uint64_t *table, int64_t pane,
                                            uint64_t key, uint32_t c, const uint64_t *f, int stride, int &err) {
  uint64_t *base = table + (pane & (p.R - 1)) * p.slot_words;
  int64_t idx;
  if (p.key_mode == KM_HASH) {
    idx = global_insert(p, st, base, key, err);
    if (idx < 0) return;
  } else {
    idx = (int64_t)key;
  }
  atomicAdd((unsigned long long *)&base[cnt_off(p) + idx], (unsigned long long)c);
  for (int i = 0; i < p.nf; ++i) red_field(p.field[i].kind, &base[fld_off(p, i) + idx], f[i * stride]);
}

// leaders of each equal-key lane group receive the group's combined fields
__device__ __forceinline__ void warp_combine(const Plan &p, bool act, unsigned m, uint64_t (&fv)[kMaxField]) {
  const int lane = threadIdx.x & 31;
  const int leader = m ? __ffs(m) - 1 : -1;
  const int npeer = __popc(m);
  const int maxn = (int)__reduce_max_sync(kFull, act ? (unsigned)npeer : 0u);
  if (maxn <= 1) return;
  const unsigned lmask = __ballot_sync(kFull, act && leader == lane);
  const int ng = __popc(lmask);
  if (ng * 5 < maxn - 1) {
    // few groups with many members (e.g. no GROUP BY): one butterfly per group
    unsigned rem = lmask;
    while (rem) {
      const int L = __ffs(rem) - 1;
      rem &= rem - 1;
      const bool mine = act && leader == L;
      for (int i = 0; i < p.nf; ++i) {
        const int kind = p.field[i].kind;
        uint64_t v = mine ? fv[i] : field_identity(kind);
#pragma unroll
        for (int x = 16; x; x >>= 1) v = field_combine(kind, v, shfl_xor64(v, x));
        if (lane == L) fv[i] = v;
      }
    }
  } else {
    uint64_t acc[kMaxField];
#pragma unroll
    for (int i = 0; i < kMaxField; ++i) acc[i] = fv[i];
    unsigned rest = act ? (m & (m - 1)) : 0u;     // peers after the leader
    for (int k = 1; k < maxn; ++k) {
      const bool ok = rest != 0u;
      const int s = ok ? __ffs(rest) - 1 : lane;
      rest &= rest - 1;
#pragma unroll
      for (int i = 0; i < kMaxField; ++i) {
        if (i < p.nf) {
          uint64_t o = shfl64(fv[i], s);
          if (ok && leader == lane) acc[i] = field_combine(p.field[i].kind, acc[i], o);
        }
      }
    }
#pragma unroll
    for (int i = 0; i < kMaxField; ++i) fv[i] = acc[i];
  }
}

__device__ __forceinline__ void flush_direct(const Plan &p, State *st, uint64_t *table, P1Warp &t,
                                             int64_t pbase, int &err) {
  __syncwarp();
  const int lane = threadIdx.x & 31;
  const int C = (int)p.C;
  for (int e = lane; e < t.TE; e += 32) {
    uint32_t c = t.cnt[e];
    if (c) {
      flush_entry(p, st, table, pbase + e / C, (uint64_t)(e % C), c, t.f + e, t.TE, err);
      t.cnt[e] = 0;
      for (int i = 0; i < p.nf; ++i) t.f[i * t.TE + e] = field_identity(p.field[i].kind);
    }
  }
  __syncwarp();
}

__device__ __forceinline__ void flush_hashed(const Plan &p, State *st, uint64_t *table, P1Warp &t,
                                             int64_t pane, int &err) {
  __syncwarp();
  const int lane = threadIdx.x & 31;
  for (int e = lane; e < t.TE; e += 32) {
    uint64_t k = t.keys[e];
    if (k != kEmpty) {
      flush_entry(p, st, table, pane, k, t.cnt[e], t.f + e, t.TE, err);
      t.keys[e] = kEmpty;
      t.cnt[e] = 0;
      for (int i = 0; i < p.nf; ++i) t.f[i * t.TE + e] = field_identity(p.field[i].kind);
    }
  }
  __syncwarp();
}

template <int NW, bool DIRECT>
__global__ void __launch_bounds__(kP1Threads, 2)
k_pane_agg(const Plan p, State *__restrict__ st, const uint4 *__restrict__ tup, int64_t n,
           uint64_t *__restrict__ table, int64_t *__restrict__ pane_ts) {
  extern __shared__ __align__(16) unsigned char smem[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  P1Warp t;
  t.TE = p.local_entries;
  t.base = smem + (size_t)wid * p.local_bytes;
  t.keys = (uint64_t *)t.base;
  t.f = (uint64_t *)(t.base + (DIRECT ? 0 : 8 * t.TE));
  t.cnt = (uint32_t *)(t.base + (DIRECT ? 0 : 8 * t.TE) + (size_t)8 * t.TE * p.nf);
  for (int e = lane; e < t.TE; e += 32) {
    if (!DIRECT) t.keys[e] = kEmpty;
    t.cnt[e] = 0;
    for (int i = 0; i < p.nf; ++i) t.f[i * t.TE + e] = field_identity(p.field[i].kind);
  }
  __syncwarp();

  const int64_t pos0 = st->task_pos;
  const int64_t min_pane = st->J0 * p.L;
  const int64_t ntiles = (n + kWarpTile - 1) / kWarpTile;
  const int64_t g = p.g;
  const uint32_t g32 = (uint32_t)g;
  const bool g_small = g < (1ll << 30);
  const int PL = p.local_pl;
  const int C = (int)p.C;
  int err = 0;

  for (int64_t tile = (int64_t)blockIdx.x * (kP1Threads / 32) + wid; tile < ntiles;
       tile += (int64_t)gridDim.x * (kP1Threads / 32)) {
    const int64_t tb = tile * kWarpTile;
    int64_t prev_tau = (tb > 0) ? *(const int64_t *)((const unsigned char *)tup + (tb - 1) * p.tuple_bytes + 4 * p.ts_word)
                                : INT64_MIN;
    // pane of the tile's first tuple: one 64-bit division per tile
    int64_t pb0, rb0, tref;
    if (p.win_kind == WK_COUNT) {
      pb0 = (pos0 + tb) / g; rb0 = (pos0 + tb) - pb0 * g; tref = 0;
    } else {
      int64_t t0 = *(const int64_t *)((const unsigned char *)tup + tb * p.tuple_bytes + 4 * p.ts_word);
      tref = t0 > p.T0 ? t0 : p.T0;
      pb0 = (tref - p.T0) / g; rb0 = (tref - p.T0) - pb0 * g;
    }
    int64_t pbase = -1;
    int occ = 0;
    for (int it = 0; it < kWarpTile / 32; it += kP1Unroll) {
      uint32_t w[kP1Unroll][NW];
#pragma unroll
      for (int u = 0; u < kP1Unroll; ++u) {
        const int64_t i = tb + (it + u) * 32 + lane;
        if (i < n) load_tuple<NW>(tup + i * (NW / 4), (unsigned)p.chunk_mask, w[u]);
        else {
#pragma unroll
          for (int k = 0; k < NW; ++k) w[u][k] = 0;
        }
      }
#pragma unroll
      for (int u = 0; u < kP1Unroll; ++u) {
        const int off = (it + u) * 32 + lane;
        const int64_t i = tb + off;
        const bool inb = i < n;
        const int64_t tau = get_int<NW>(w[u], p.ts_word, T_I64);
        // K1: τ must be non-decreasing (L347-349) and non-negative (L349-350)
        int64_t up = (int64_t)shfl64((uint64_t)tau, (lane + 31) & 31);
        if (lane == 0) up = prev_tau;
        if (inb && tau < up) err |= ERR_ORDER;
        if (inb && tau < 0) err |= ERR_TS;
        prev_tau = (int64_t)shfl64((uint64_t)tau, 31);
        // K1: pane id of the tuple
        int64_t pane;
        bool valid = inb;
        if (p.win_kind == WK_COUNT) {
          const int64_t r = rb0 + off;
          const int64_t q = g_small ? (int64_t)((uint32_t)r / g32) : r / g;
          pane = pb0 + q;
          if (inb && r == q * g && pane >= min_pane) pane_ts[pane & (p.R - 1)] = tau;
        } else {
          valid &= tau >= p.T0;
          int64_t d = tau - tref + rb0;
          if (g == 1) pane = pb0 + d;
          else pane = pb0 + ((g_small && d >= 0 && d < (1ll << 32)) ? (int64_t)((uint32_t)d / g32) : d / g);
        }
        valid &= pane >= min_pane;
        // σ (selection inside the window, reading A5)
        if (p.npred) valid &= eval_preds<NW>(p, w[u]);
        const uint64_t key = make_key<NW>(p, w[u], valid, err);
        uint64_t fv[kMaxField];
#pragma unroll
        for (int f = 0; f < kMaxField; ++f) fv[f] = (f < p.nf) ? field_value<NW>(p.field[f], w[u]) : 0;

        bool todo = valid;
        while (__any_sync(kFull, todo)) {
          if (DIRECT) {
            const int64_t pm = warp_min64(todo ? pane : INT64_MAX);
            if (pbase < 0 || pm >= pbase + PL || pm < pbase) {
              if (pbase >= 0) flush_direct(p, st, table, t, pbase, err);
              pbase = pm;
            }
            bool act = todo && pane < pbase + PL;
            const int e = act ? (int)(pane - pbase) * C + (int)key : 0;
            const unsigned actm = __ballot_sync(kFull, act);
            const unsigned m = __match_any_sync(kFull, e) & actm;
            uint64_t fc[kMaxField];
#pragma unroll
            for (int f = 0; f < kMaxField; ++f) fc[f] = fv[f];
            warp_combine(p, act, m, fc);
            if (act && (__ffs(m) - 1) == lane) {
              t.cnt[e] += (uint32_t)__popc(m);
              for (int f = 0; f < p.nf; ++f) t.f[f * t.TE + e] = field_combine(p.field[f].kind, t.f[f * t.TE + e], fc[f]);
            }
            __syncwarp();
            todo = todo && !act;
          } else {
            const int64_t pm = warp_min64(todo ? pane : INT64_MAX);
            if (pbase != pm) {
              if (pbase >= 0) flush_hashed(p, st, table, t, pbase, err);
              pbase = pm;
              occ = 0;
            } else if (occ + 32 > t.TE / 2) {
              flush_hashed(p, st, table, t, pbase, err);
              occ = 0;
            }
            const bool act = todo && pane == pbase;
            const unsigned actm = __ballot_sync(kFull, act);
            const unsigned m = __match_any_sync(kFull, (unsigned long long)key) & actm;
            uint64_t fc[kMaxField];
#pragma unroll
            for (int f = 0; f < kMaxField; ++f) fc[f] = fv[f];
            warp_combine(p, act, m, fc);
            bool ins = false;
            if (act && (__ffs(m) - 1) == lane) {
              uint32_t h = (uint32_t)fmix64(key) & (uint32_t)(t.TE - 1);
              volatile uint64_t *vk = t.keys;
              for (;;) {
                uint64_t k = vk[h];
                if (k == key) break;
                if (k == kEmpty) {
                  uint64_t old = atomicCAS((unsigned long long *)&t.keys[h], kEmpty, key);
                  if (old == kEmpty) { ins = true; break; }
                  if (old == key) break;
                }
                h = (h + 1) & (uint32_t)(t.TE - 1);
              }
              t.cnt[h] += (uint32_t)__popc(m);
              for (int f = 0; f < p.nf; ++f) t.f[f * t.TE + h] = field_combine(p.field[f].kind, t.f[f * t.TE + h], fc[f]);
            }
            occ += __popc(__ballot_sync(kFull, ins));
            __syncwarp();
            todo = todo && !act;
          }
        }
      }
    }
    if (pbase >= 0) {
      if (DIRECT) flush_direct(p, st, table, t, pbase, err);
      else flush_hashed(p, st, table, t, pbase, err);
    }
  }
  if (err) atomicOr(&st->error, err);
}

// --------------------------------------------------------------------------
// window assembly helpers
struct AggVal { uint64_t bits; bool isf; };

__device__ __forceinline__ AggVal finalize(const Plan &p, int a, int64_t cnt, const uint64_t *fv) {
  const AggOut &o = p.agg[a];
  AggVal r;
  r.isf = o.out_float;
  switch (o.fn) {
    case AG_COUNT: r.bits = (uint64_t)cnt; break;
    case AG_SUM: r.bits = fv[o.field]; break;
    case AG_AVG: {
      double sum = (p.field[o.field].kind == FK_SUM_F) ? __longlong_as_double((long long)fv[o.field])
                                                      : (double)(int64_t)fv[o.field];
      r.bits = (uint64_t)__double_as_longlong(sum / (double)cnt);   // reading A11
      break;
    }
    default: {
      uint64_t u = fv[o.field];
      r.bits = o.is_float_col ? (uint64_t)__double_as_longlong(dec_dbl(u)) : (uint64_t)dec_int(u);
    }
  }
  return r;
}

__device__ __forceinline__ bool having_ok(const Plan &p, int64_t cnt, const uint64_t *fv) {
  for (int h = 0; h < p.nhave; ++h) {
    const Have &hv = p.have[h];
    AggVal v = finalize(p, hv.agg, cnt, fv);
    bool ok = v.isf ? cmp_op(__longlong_as_double((long long)v.bits), hv.op, hv.fval)
                    : cmp_op((int64_t)v.bits, hv.op, hv.ival);
    if (!ok) return false;
  }
  return true;
}

__device__ __forceinline__ void write_row(const Plan &p, unsigned char *rows, int64_t r, const int64_t *kv,
                                          int64_t cnt, const uint64_t *fv) {
  if (r >= p.rows_cap) return;
  for (int i = 0; i < p.nkeys; ++i) {
    unsigned char *c = rows + p.col_off[i];
    if (p.col_bytes[i] == 4) ((int32_t *)c)[r] = (int32_t)kv[i];
    else ((int64_t *)c)[r] = kv[i];
  }
  for (int a = 0; a < p.nagg; ++a) {
    AggVal v = finalize(p, a, cnt, fv);
    ((uint64_t *)(rows + p.col_off[p.nkeys + a]))[r] = v.bits;
  }
}

__device__ __forceinline__ void decode_key(const Plan &p, uint64_t k, int64_t *kv) {
  if (p.key_pack == KP_RADIX) {
    for (int i = 0; i < p.nkeys; ++i) kv[i] = (int64_t)((k / (uint64_t)p.key[i].stride) % (uint64_t)p.key[i].domain);
  } else if (p.key_pack == KP_BIASED64) {
    kv[0] = (int64_t)(k ^ 0x8000000000000000ull);
  } else {
    kv[0] = (int32_t)((uint32_t)(k >> 32) ^ 0x80000000u);
    kv[1] = (int32_t)((uint32_t)k ^ 0x80000000u);
  }
}

// exclusive scan over the threads of a group (GS = 32: warp; GS = 256: block)
__device__ __forceinline__ int group_excl_scan(int v, int GS, int *sm, int &total) {
  const int lane = threadIdx.x & 31;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int y = __shfl_up_sync(kFull, x, o);
    if (lane >= o) x += y;
  }
  if (GS == 32) {
    total = __shfl_sync(kFull, x, 31);
    return x - v;
  }
  const int wid = threadIdx.x >> 5;
  if (lane == 31) sm[wid] = x;
  __syncthreads();
  if (wid == 0) {
    int w = lane < (GS >> 5) ? sm[lane] : 0;
    int s = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(kFull, s, o);
      if (lane >= o) s += y;
    }
    if (lane < (GS >> 5)) sm[lane] = s - w;
    if (lane == (GS >> 5) - 1) sm[32] = s;
  }
  __syncthreads();
  int r = sm[wid] + x - v;
  total = sm[32];
  __syncthreads();
  return r;
}

// DENSE / GLOBAL: thread-owned slots of a key slab, state in shared memory
template <bool EMIT>
__global__ void __launch_bounds__(256)
k_win_dense(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ table,
            int64_t *__restrict__ counts, unsigned char *__restrict__ rows, int W) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ int scan_sm[40];
  const int GS = p.GS;
  const int gpb = blockDim.x / GS, grp = threadIdx.x / GS, gt = threadIdx.x % GS;
  const int SB = p.SB, S = p.S;
  const int64_t C = p.C;
  const size_t group_words = (size_t)SB * (1 + p.nf);
  int64_t *scnt = (int64_t *)(smem + grp * group_words * 8);
  uint64_t *sf = (uint64_t *)(scnt + SB);
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const int64_t nchunks = (nw + W - 1) / W;
  const int64_t nitems = nchunks * S;
  const int64_t co = cnt_off(p);
  for (int64_t item0 = (int64_t)blockIdx.x * gpb; item0 < nitems; item0 += (int64_t)gridDim.x * gpb) {
    const int64_t item = item0 + grp;
    const bool live = item < nitems;      // groups of one block stay in lockstep (GS=256 → 1 group)
    const int64_t chunk = live ? item / S : 0;
    const int slab = live ? (int)(item % S) : 0;
    const int64_t ja = J0 + chunk * W;
    const int64_t jb = live ? (ja + W < J1 ? ja + W : J1) : ja;
    const int64_t slot0 = (int64_t)slab * SB;
    const int nslot = (int)((C - slot0) < SB ? (C - slot0) : SB);
    for (int s = gt; s < SB; s += GS) {
      scnt[s] = 0;
      for (int f = 0; f < p.nf; ++f) sf[f * SB + s] = 0;
    }
    auto add_pane = [&](int64_t q, int sign) {
      const uint64_t *b = table + (q & (p.R - 1)) * p.slot_words;
      for (int s = gt; s < nslot; s += GS) {
        int64_t c = (int64_t)b[co + slot0 + s];
        if (!c) continue;
        scnt[s] += sign * c;
        for (int f = 0; f < p.nf; ++f) {
          const int kind = p.field[f].kind;
          uint64_t v = b[fld_off(p, f) + slot0 + s];
          if (kind == FK_SUM_F) {
            double d = __longlong_as_double((long long)sf[f * SB + s]) + sign * __longlong_as_double((long long)v);
            sf[f * SB + s] = (uint64_t)__double_as_longlong(d);
          } else if (kind == FK_SUM_I) {
            sf[f * SB + s] = (uint64_t)((int64_t)sf[f * SB + s] + sign * (int64_t)v);
          }
        }
        if (sign < 0 && scnt[s] == 0)
          for (int f = 0; f < p.nf; ++f) sf[f * SB + s] = 0;   // no fp64 residue in empty groups
      }
    };
    if (live)
      for (int64_t q = ja * p.L; q < ja * p.L + p.K; ++q) add_pane(q, +1);
    for (int64_t j = ja; j < ja + W; ++j) {
      const bool wl = live && j < jb;
      if (wl && j > ja) {
        for (int64_t q = (j - 1) * p.L + p.K; q < j * p.L + p.K; ++q) add_pane(q, +1);
        for (int64_t q = (j - 1) * p.L; q < j * p.L; ++q) add_pane(q, -1);
      }
      if (wl && p.has_minmax) {
        for (int s = gt; s < nslot; s += GS)
          for (int f = 0; f < p.nf; ++f) {
            const int kind = p.field[f].kind;
            if (kind != FK_MIN && kind != FK_MAX) continue;
            uint64_t m = field_identity(kind);
            for (int64_t q = j * p.L; q < j * p.L + p.K; ++q)
              m = field_combine(kind, m, table[(q & (p.R - 1)) * p.slot_words + fld_off(p, f) + slot0 + s]);
            sf[f * SB + s] = m;
          }
      }
      int my = 0;
      uint64_t fv[kMaxField];
      if (wl)
        for (int s = gt; s < nslot; s += GS) {
          if (scnt[s] <= 0) continue;
          for (int f = 0; f < p.nf; ++f) fv[f] = sf[f * SB + s];
          if (having_ok(p, scnt[s], fv)) ++my;
        }
      int total;
      int excl = group_excl_scan(my, GS, scan_sm, total);
      if (!wl) continue;
      const int64_t ci = (j - J0) * S + slab;
      if (!EMIT) {
        if (gt == 0) counts[ci] = total;
      } else {
        int64_t r = counts[ci] + excl;
        for (int s = gt; s < nslot; s += GS) {
          if (scnt[s] <= 0) continue;
          for (int f = 0; f < p.nf; ++f) fv[f] = sf[f * SB + s];
          if (!having_ok(p, scnt[s], fv)) continue;
          int64_t kv[kMaxKey];
          decode_key(p, (uint64_t)(slot0 + s), kv);
          write_row(p, rows, r++, kv, scnt[s], fv);
        }
      }
    }
  }
}

// HASH: block-wide state hash keyed by the group key; slab = home-slot range
template <bool EMIT>
__global__ void __launch_bounds__(256)
k_win_hash(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ table,
           int64_t *__restrict__ counts, unsigned char *__restrict__ rows, int W) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ int scan_sm[40];
  __shared__ int s_err;
  const int ST = p.state_cap, SB = p.SB, S = p.S;
  const uint32_t Cm = (uint32_t)p.C - 1;
  uint64_t *skeys = (uint64_t *)smem;
  int64_t *scnt = (int64_t *)(skeys + ST);
  uint64_t *sf = (uint64_t *)(scnt + ST);
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const int64_t maxprobe = (int64_t)st->max_probe;
  const int64_t span = (SB + maxprobe + 1) < p.C ? (SB + maxprobe + 1) : p.C;
  const int64_t nchunks = (nw + W - 1) / W;
  const int64_t nitems = nchunks * S;
  if (threadIdx.x == 0) s_err = 0;
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t chunk = item / S;
    const uint32_t slot0 = (uint32_t)((item % S) * SB);
    const int64_t ja = J0 + chunk * W;
    const int64_t jb = ja + W < J1 ? ja + W : J1;
    __syncthreads();
    for (int h = threadIdx.x; h < ST; h += blockDim.x) {
      skeys[h] = kEmpty;
      scnt[h] = 0;
      for (int f = 0; f < p.nf; ++f) sf[f * ST + h] = field_identity(p.field[f].kind);
    }
    __syncthreads();
    auto find = [&](uint64_t k) -> int {
      uint32_t h = (uint32_t)(fmix64(k) >> 32) & (uint32_t)(ST - 1);
      volatile uint64_t *vk = skeys;
      for (int probe = 0; probe < ST; ++probe) {
        uint64_t cur = vk[h];
        if (cur == k) return (int)h;
        if (cur == kEmpty) {
          uint64_t old = atomicCAS((unsigned long long *)&skeys[h], kEmpty, k);
          if (old == kEmpty || old == k) return (int)h;
        }
        h = (h + 1) & (uint32_t)(ST - 1);
      }
      s_err = 1;
      return -1;
    };
    // mode 0: add (+1) / subtract (-1) invertible fields; mode 2: min/max only
    auto visit_pane = [&](int64_t q, int sign, bool minmax) {
      const uint64_t *b = table + (q & (p.R - 1)) * p.slot_words;
      for (int64_t o = threadIdx.x; o < span; o += blockDim.x) {
        const uint32_t h = (slot0 + (uint32_t)o) & Cm;
        const uint64_t k = b[h];
        if (k == kEmpty) continue;
        const uint32_t home = (uint32_t)fmix64(k) & Cm;
        if (((home - slot0) & Cm) >= (uint32_t)SB) continue;
        const int s = find(k);
        if (s < 0) continue;
        if (!minmax) {
          atomicAdd((unsigned long long *)&scnt[s], (unsigned long long)(sign * (int64_t)b[p.C + h]));
        }
        for (int f = 0; f < p.nf; ++f) {
          const int kind = p.field[f].kind;
          const uint64_t v = b[fld_off(p, f) + h];
          if (!minmax && kind == FK_SUM_F) atomicAdd((double *)&sf[f * ST + s], sign * __longlong_as_double((long long)v));
          else if (!minmax && kind == FK_SUM_I) atomicAdd((unsigned long long *)&sf[f * ST + s], (unsigned long long)(sign * (int64_t)v));
          else if (minmax && kind == FK_MIN) atomicMin((unsigned long long *)&sf[f * ST + s], (unsigned long long)v);
          else if (minmax && kind == FK_MAX) atomicMax((unsigned long long *)&sf[f * ST + s], (unsigned long long)v);
        }
      }
    };
    for (int64_t q = ja * p.L; q < ja * p.L + p.K; ++q) visit_pane(q, +1, false);
    for (int64_t j = ja; j < jb; ++j) {
      if (j > ja) {
        for (int64_t q = (j - 1) * p.L + p.K; q < j * p.L + p.K; ++q) visit_pane(q, +1, false);
        for (int64_t q = (j - 1) * p.L; q < j * p.L; ++q) visit_pane(q, -1, false);
      }
      __syncthreads();
      for (int h = threadIdx.x; h < ST; h += blockDim.x)
        if (scnt[h] == 0)
          for (int f = 0; f < p.nf; ++f)
            if (p.field[f].kind == FK_SUM_F || p.field[f].kind == FK_SUM_I) sf[f * ST + h] = 0;
      if (p.has_minmax) {
        for (int h = threadIdx.x; h < ST; h += blockDim.x)
          for (int f = 0; f < p.nf; ++f)
            if (p.field[f].kind == FK_MIN || p.field[f].kind == FK_MAX) sf[f * ST + h] = field_identity(p.field[f].kind);
        __syncthreads();
        for (int64_t q = j * p.L; q < j * p.L + p.K; ++q) visit_pane(q, 0, true);
      }
      __syncthreads();
      int my = 0;
      uint64_t fv[kMaxField];
      for (int h = threadIdx.x; h < ST; h += blockDim.x) {
        if (skeys[h] == kEmpty || scnt[h] <= 0) continue;
        for (int f = 0; f < p.nf; ++f) fv[f] = sf[f * ST + h];
        if (having_ok(p, scnt[h], fv)) ++my;
      }
      int total;
      int excl = group_excl_scan(my, 256, scan_sm, total);
      const int64_t ci = (j - J0) * S + (item % S);
      if (!EMIT) {
        if (threadIdx.x == 0) counts[ci] = total;
      } else {
        int64_t r = counts[ci] + excl;
        for (int h = threadIdx.x; h < ST; h += blockDim.x) {
          if (skeys[h] == kEmpty || scnt[h] <= 0) continue;
          for (int f = 0; f < p.nf; ++f) fv[f] = sf[f * ST + h];
          if (!having_ok(p, scnt[h], fv)) continue;
          int64_t kv[kMaxKey];
          decode_key(p, skeys[h], kv);
          write_row(p, rows, r++, kv, scnt[h], fv);
        }
      }
      __syncthreads();
    }
  }
  __syncthreads();
  if (threadIdx.x == 0 && s_err) atomicOr(&st->error, ERR_CAPACITY);
}

// headers and row offsets of the windows closed by this task (one block)
__global__ void __launch_bounds__(1024)
k_win_scan(const Plan p, State *st, const int64_t *__restrict__ pane_ts, int64_t *__restrict__ counts,
           WinHdr *__restrict__ hdr, SlotMeta *meta) {
  __shared__ int64_t wsum[32];
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  const int S = p.S;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t per = (nw + blockDim.x - 1) / blockDim.x;
  const int64_t a = (int64_t)tid * per, b = (a + per < nw) ? a + per : nw;
  int64_t local = 0;
  for (int64_t j = a; j < b; ++j)
    for (int s = 0; s < S; ++s) local += counts[j * S + s];
  int64_t x = local;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int64_t y = (int64_t)__shfl_up_sync(kFull, (unsigned long long)x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[wid] = x;
  __syncthreads();
  if (wid == 0) {
    int64_t w = wsum[lane], s = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int64_t y = (int64_t)__shfl_up_sync(kFull, (unsigned long long)s, o);
      if (lane >= o) s += y;
    }
    wsum[lane] = s - w;
  }
  __syncthreads();
  int64_t run = wsum[wid] + x - local;
  for (int64_t j = a; j < b; ++j) {
    WinHdr h;
    h.window_id = J0 + j;
    h.ts = (p.win_kind == WK_TIME) ? p.T0 + (J0 + j) * p.l : pane_ts[((J0 + j) * p.L) & (p.R - 1)];
    h.row_offset = run;
    int64_t nr = 0;
    for (int s = 0; s < S; ++s) {
      int64_t c = counts[j * S + s];
      counts[j * S + s] = run;
      run += c;
      nr += c;
    }
    h.nrows = (int32_t)nr;
    h.flags = 0;
    hdr[j] = h;
  }
  if (tid == blockDim.x - 1) {
    meta->nrows = run;
    if (run > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
  }
}

__global__ void k_task_end(const Plan p, State *st, SlotMeta *meta) {
  if (threadIdx.x) return;
  meta->first_window = st->J0;
  meta->nwindows = st->J1 - st->J0;
  meta->error = st->error;
  meta->pos_end = st->pos_next;
  meta->tau_last = st->tau_last;
  if (p.nagg == 0) {
    meta->nrows = 0;
    meta->ntuples = st->sel_rows;
    st->carry_pos = st->zero_lo;
    st->carry_n = st->zero_hi;
    st->carry_sel ^= 1;
    st->zero_lo = st->zero_hi = 0;
  } else {
    meta->ntuples = 0;
  }
  st->J0 = st->J1;
}

// --------------------------------------------------------------------------
// σ/π with stream compaction (IStream)
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ void st_relaxed(uint64_t *p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v));
}
constexpr uint64_t kFlagA = 1, kFlagP = 2;
__device__ __forceinline__ uint64_t pack_status(uint64_t epoch, uint64_t flag, uint64_t v) {
  return ((epoch & 0xffffffull) << 40) | (flag << 38) | (v & ((1ull << 38) - 1));
}

template <int NW>
__global__ void __launch_bounds__(kSelThreads)
k_select(const Plan p, State *__restrict__ st, const uint4 *__restrict__ task,
         const uint4 *__restrict__ carry0, const uint4 *__restrict__ carry1,
         uint64_t *__restrict__ status, int *__restrict__ tile_ctr, unsigned char *__restrict__ rows) {
  __shared__ int s_cnt[kSelPer][kSelThreads / 32];
  __shared__ int s_off[kSelPer][kSelThreads / 32];
  __shared__ int64_t s_tile, s_excl;
  __shared__ int s_total;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t lo = st->cover_lo, hi = st->cover_hi;
  const int64_t tpos = st->task_pos, cpos = st->carry_pos;
  const uint4 *carry = st->carry_sel ? carry1 : carry0;
  const uint64_t epoch = (uint64_t)st->tile_epoch;
  const int64_t ntiles = (hi - lo + kSelTile - 1) / kSelTile;
  const int CW = NW / 4;
  int err = 0;
  for (;;) {
    if (tid == 0) s_tile = atomicAdd(tile_ctr, 1);
    __syncthreads();
    const int64_t t = s_tile;
    if (t >= ntiles) break;
    const int64_t base = lo + t * kSelTile;
    uint32_t w[kSelPer][NW];
    bool sel[kSelPer];
#pragma unroll
    for (int k = 0; k < kSelPer; ++k) {
      const int64_t pos = base + k * kSelThreads + tid;
      if (pos < hi) {
        const uint4 *src = pos < tpos ? carry + (pos - cpos) * CW : task + (pos - tpos) * CW;
        load_tuple<NW>(src, (unsigned)p.chunk_mask, w[k]);
      } else {
#pragma unroll
        for (int c = 0; c < NW; ++c) w[k][c] = 0;
      }
    }
#pragma unroll
    for (int k = 0; k < kSelPer; ++k) {
      const int64_t pos = base + k * kSelThreads + tid;
      const bool inb = pos < hi;
      const int64_t tau = get_int<NW>(w[k], p.ts_word, T_I64);
      int64_t up = (int64_t)shfl64((uint64_t)tau, (lane + 31) & 31);
      if (lane == 0 && pos > cpos && inb) {
        const int64_t pp = pos - 1;
        const unsigned char *src = pp < tpos ? (const unsigned char *)carry + (pp - cpos) * p.tuple_bytes
                                             : (const unsigned char *)task + (pp - tpos) * p.tuple_bytes;
        up = *(const int64_t *)(src + 4 * p.ts_word);
      } else if (lane == 0) {
        up = INT64_MIN;
      }
      if (inb && tau < up) err |= ERR_ORDER;
      if (inb && tau < 0) err |= ERR_TS;
      bool s = inb;
      if (p.win_kind == WK_TIME) s &= tau >= p.T0;
      if (p.npred) s &= eval_preds<NW>(p, w[k]);
      sel[k] = s;
      const unsigned bal = __ballot_sync(kFull, s);
      if (lane == 0) s_cnt[k][wid] = __popc(bal);
    }
    __syncthreads();
    if (wid == 0) {
      // 64 (k, warp) counts in order: lane holds 2 consecutive entries
      const int i0 = 2 * lane, i1 = 2 * lane + 1;
      const int c0 = s_cnt[i0 / 8][i0 % 8], c1 = s_cnt[i1 / 8][i1 % 8];
      int x = c0 + c1;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int y = __shfl_up_sync(kFull, x, o);
        if (lane >= o) x += y;
      }
      const int ex = x - c0 - c1;
      s_off[i0 / 8][i0 % 8] = ex;
      s_off[i1 / 8][i1 % 8] = ex + c0;
      if (lane == 31) s_total = x;
    }
    __syncthreads();
    if (tid == 0) {
      // decoupled look-back over tiles (single pass)
      const uint64_t total = (uint64_t)s_total;
      int64_t excl = 0;
      if (t == 0) {
        st_relaxed(&status[0], pack_status(epoch, kFlagP, total));
      } else {
        st_relaxed(&status[t], pack_status(epoch, kFlagA, total));
        int64_t i = t - 1;
        for (;;) {
          const uint64_t sv = ld_relaxed(&status[i]);
          const uint64_t flag = (sv >> 38) & 3ull;
          if ((sv >> 40) != (epoch & 0xffffffull) || flag == 0) continue;
          excl += (int64_t)(sv & ((1ull << 38) - 1));
          if (flag == kFlagP) break;
          --i;
        }
        st_relaxed(&status[t], pack_status(epoch, kFlagP, (uint64_t)excl + total));
      }
      s_excl = excl;
      if (t == ntiles - 1) st->sel_rows = excl + (int64_t)total;
    }
    __syncthreads();
    const int64_t excl = s_excl;
    const int ow = p.out_row_words;
    const unsigned lt = (1u << lane) - 1u;
#pragma unroll
    for (int k = 0; k < kSelPer; ++k) {
      const unsigned bal = __ballot_sync(kFull, sel[k]);
      if (sel[k]) {
        const int64_t r = excl + s_off[k][wid] + __popc(bal & lt);
        uint32_t *dst = (uint32_t *)(rows + r * (int64_t)ow * 4);
        if (r < p.rows_cap) {
          if ((ow & 3) == 0) {
            for (int c = 0; c < ow; c += 4)
              *(uint4 *)(dst + c) = make_uint4(sel_word<NW>(w[k], p.proj_word[c]), sel_word<NW>(w[k], p.proj_word[c + 1]),
                                               sel_word<NW>(w[k], p.proj_word[c + 2]), sel_word<NW>(w[k], p.proj_word[c + 3]));
          } else {
            for (int c = 0; c < ow; ++c) dst[c] = sel_word<NW>(w[k], p.proj_word[c]);
          }
        }
      }
    }
    __syncthreads();
  }
  if (tid == 0 && ntiles == 0) { /* sel_rows already 0 from k_task_begin */ }
  if (err) atomicOr(&st->error, err);
}

__global__ void k_carry(const Plan p, const State *st, const uint4 *task, const uint4 *carry0,
                        const uint4 *carry1, uint4 *dst0, uint4 *dst1) {
  const int64_t ncp = st->zero_lo, nn = st->zero_hi;
  if (nn <= 0 || nn > p.carry_cap) return;
  const int64_t tpos = st->task_pos, cpos = st->carry_pos;
  const uint4 *carry = st->carry_sel ? carry1 : carry0;
  uint4 *dst = st->carry_sel ? dst0 : dst1;
  const int CW = p.tuple_bytes / 16;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nn * CW; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t pos = ncp + i / CW;
    const int c = (int)(i % CW);
    dst[i] = pos < tpos ? carry[(pos - cpos) * CW + c] : task[(pos - tpos) * CW + c];
  }
}

__global__ void k_init_state(State *st, int64_t base_index, int64_t first_window, int64_t L) {
  if (threadIdx.x) return;
  State s = {};
  s.pos_next = base_index;
  s.J0 = first_window;
  s.J1 = first_window;
  s.zeroed_hi = first_window * L;
  s.pane_hi = -1;
  s.first_task = 1;
  s.carry_pos = base_index;
  *st = s;
}

__global__ void k_partition_plan(int ts_word, int tuple_bytes, int win_kind, int64_t s, int64_t l, int64_t T0,
                                 const unsigned char *tup, int64_t begin, int64_t n, int64_t *out) {
  Plan p;
  p.ts_word = ts_word;
  p.tuple_bytes = tuple_bytes;
  int64_t closed = 0, halo = begin;
  if (win_kind == WK_COUNT) {
    const int64_t total = begin + n;
    closed = total >= s ? (total - s) / l + 1 : 0;
    halo = closed * l;
  } else if (n > 0) {
    const int64_t tl = tau_at(p, tup, n - 1);
    closed = (tl - T0 - s >= 0) ? (tl - T0 - s) / l + 1 : 0;
    const int64_t B = T0 + closed * l;
    const int64_t idx = warp_lower_bound(p, tup, n, tup, 0, B);
    halo = begin + idx;
    if (idx == 0 && begin > 0 && tau_at(p, tup, 0) > B) closed = -1;   // window spans > partition
  }
  if (threadIdx.x == 0) { out[0] = closed; out[1] = halo; }
}

// ==========================================================================
// host launchers
int p1_smem_bytes(const Plan &p) { return p.local_bytes * (kP1Threads / 32); }

template <int NW, bool D>
static void *p1_fn() { return (void *)k_pane_agg<NW, D>; }

static void *p1_kernel(const Plan &p) {
  const bool d = p.local_direct;
  switch (p.tuple_words) {
    case 4: return d ? p1_fn<4, true>() : p1_fn<4, false>();
    case 8: return d ? p1_fn<8, true>() : p1_fn<8, false>();
    case 12: return d ? p1_fn<12, true>() : p1_fn<12, false>();
    default: return d ? p1_fn<16, true>() : p1_fn<16, false>();
  }
}
static void *sel_kernel(const Plan &p) {
  switch (p.tuple_words) {
    case 4: return (void *)k_select<4>;
    case 8: return (void *)k_select<8>;
    case 12: return (void *)k_select<12>;
    default: return (void *)k_select<16>;
  }
}

cudaError_t set_kernel_attributes(const Plan &p) {
  cudaError_t e = cudaSuccess;
  if (p.nagg > 0) {
    e = cudaFuncSetAttribute(p1_kernel(p), cudaFuncAttributeMaxDynamicSharedMemorySize, p1_smem_bytes(p));
    if (e) return e;
    const void *k2[4] = {(void *)k_win_dense<false>, (void *)k_win_dense<true>, (void *)k_win_hash<false>,
                         (void *)k_win_hash<true>};
    for (auto k : k2) {
      e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, p.p2_smem);
      if (e) return e;
    }
  }
  return e;
}

int p1_blocks_per_sm(const Plan &p) {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, p1_kernel(p), kP1Threads, p1_smem_bytes(p));
  return b > 0 ? b : 1;
}
int p2_blocks_per_sm(const Plan &p) {
  int b = 0;
  const void *k = p.key_mode == KM_HASH ? (void *)k_win_hash<true> : (void *)k_win_dense<true>;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, k, 256, p.p2_smem);
  return b > 0 ? b : 1;
}
int sel_blocks_per_sm(const Plan &p) {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, sel_kernel(p), kSelThreads, 0);
  return b > 0 ? b : 1;
}

cudaError_t launch_init_state(const Plan &p, const QueryDev &q, int64_t base_index, cudaStream_t s) {
  k_init_state<<<1, 32, 0, s>>>(q.st, base_index, p.first_window, p.L);
  return cudaGetLastError();
}

cudaError_t launch_agg_task(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int64_t n,
                            int final_, int has_wm, int64_t wm, int emit_on_finish, int p1_grid, int p2_grid,
                            int win_chunk, cudaStream_t st) {
  k_task_begin<<<1, 32, 0, st>>>(p, q.st, (const unsigned char *)tuples, n, final_, has_wm, wm, emit_on_finish,
                                 s.meta, nullptr, nullptr, q.tile_ctr);
  k_zero_panes<<<148 * 4, 256, 0, st>>>(p, q.st, q.table);
  if (n > 0) {
    const int64_t ntiles = (n + kWarpTile - 1) / kWarpTile;
    int64_t grid = (ntiles + (kP1Threads / 32) - 1) / (kP1Threads / 32);
    if (grid > p1_grid) grid = p1_grid;
    void *args[] = {(void *)&p, (void *)&q.st, (void *)&tuples, (void *)&n, (void *)&q.table, (void *)&q.pane_ts};
    cudaError_t e = cudaLaunchKernel(p1_kernel(p), dim3((unsigned)grid), dim3(kP1Threads), args,
                                     (size_t)p1_smem_bytes(p), st);
    if (e) return e;
  }
  if (p.key_mode == KM_HASH) {
    k_win_hash<false><<<p2_grid, 256, p.p2_smem, st>>>(p, q.st, q.table, s.counts, s.rows, win_chunk);
    k_win_scan<<<1, 1024, 0, st>>>(p, q.st, q.pane_ts, s.counts, (WinHdr *)s.hdr, s.meta);
    k_win_hash<true><<<p2_grid, 256, p.p2_smem, st>>>(p, q.st, q.table, s.counts, s.rows, win_chunk);
  } else {
    k_win_dense<false><<<p2_grid, 256, p.p2_smem, st>>>(p, q.st, q.table, s.counts, s.rows, win_chunk);
    k_win_scan<<<1, 1024, 0, st>>>(p, q.st, q.pane_ts, s.counts, (WinHdr *)s.hdr, s.meta);
    k_win_dense<true><<<p2_grid, 256, p.p2_smem, st>>>(p, q.st, q.table, s.counts, s.rows, win_chunk);
  }
  k_task_end<<<1, 32, 0, st>>>(p, q.st, s.meta);
  return cudaGetLastError();
}

cudaError_t launch_select_task(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int64_t n,
                               int final_, int has_wm, int64_t wm, int emit_on_finish, int sel_grid,
                               cudaStream_t st) {
  k_task_begin<<<1, 32, 0, st>>>(p, q.st, (const unsigned char *)tuples, n, final_, has_wm, wm, emit_on_finish,
                                 s.meta, q.carry[0], q.carry[1], q.tile_ctr);
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&tuples, (void *)&q.carry[0], (void *)&q.carry[1],
                  (void *)&q.tile_status, (void *)&q.tile_ctr, (void *)&s.rows};
  cudaError_t e = cudaLaunchKernel(sel_kernel(p), dim3(sel_grid), dim3(kSelThreads), args, 0, st);
  if (e) return e;
  k_carry<<<148, 256, 0, st>>>(p, q.st, (const uint4 *)tuples, (const uint4 *)q.carry[0], (const uint4 *)q.carry[1],
                               (uint4 *)q.carry[0], (uint4 *)q.carry[1]);
  k_task_end<<<1, 32, 0, st>>>(p, q.st, s.meta);
  return cudaGetLastError();
}

cudaError_t launch_partition_plan(int ts_word, int tuple_words, int win_kind, int64_t s, int64_t l, int64_t T0,
                                  const void *tuples, int64_t begin, int64_t n, int64_t *dev_out2, cudaStream_t st) {
  k_partition_plan<<<1, 32, 0, st>>>(ts_word, tuple_words * 4, win_kind, s, l, T0, (const unsigned char *)tuples,
                                     begin, n, dev_out2);
  return cudaGetLastError();
}

}  // namespace sb
