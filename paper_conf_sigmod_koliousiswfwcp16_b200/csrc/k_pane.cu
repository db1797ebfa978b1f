// k_pane.cu -- K1 + σ + K2/K4 fused: the one HBM pass of an aggregation task.
//
// Each CTA owns a contiguous range of the task's tuples (row-major byte records,
// PAPER.md L744-745) and streams it through shared memory with 1-D TMA bulk
// copies (cp.async.bulk + mbarrier transaction counts), kStages deep, so the
// HBM stream never waits on compute.  Per tuple, in shared memory:
//   K1  pane id: count windows position/g, time windows (τ-T0)/g (panes are
//       the window fragments of length g = gcd(s,l), L180-181, L1275-1280);
//       τ non-decreasing (L347-349) and non-negative are checked here
//   σ   conjunction of `col op const` (L1320-1322)
//   γ   GROUP BY key (dense radix index or packed 64-bit key)
//   α   fields of the accumulator (count, fp64/int64 sums, min/max)
// and is folded into a shared-memory table private to its warp (or lane):
//   LANE    tiny key counts: one table column per lane, plain read-modify-write
//   DIRECT  small dense key domains: per-warp table indexed (pane, key), shared
//           memory atomics (measured ~0.8 SM-cycles per update on B200)
//   HASHED  large / unbounded domains: per-warp open-addressing table of one
//           pane, key claimed by CAS (the paper's GPU hash, L1337-1349), atomics
// The CTA advances over a pane window [pbase, pbase+PL) that is uniform across
// its warps; leaving it flushes the tables into the device pane ring with L2
// atomics (RED), after summing the warp/lane copies of an entry (LANE, DIRECT)
// so each (pane, key) costs one set of REDs per CTA.
#include <cuda_runtime.h>
#include <climits>
#include <stdint.h>

#include <cstdlib>

#include "common.cuh"
#include "launch_internal.h"
#include "tma.cuh"

namespace sb {

constexpr int kP1Threads = 256, kP1Warps = kP1Threads / 32;
// stage geometry and DIRECT-table occupancy (compile-time; -D overrides for experiments)
#ifndef SB_P1_STAGE_KB
#define SB_P1_STAGE_KB 16
#endif
#ifndef SB_P1_STAGES
#define SB_P1_STAGES 2
#endif
#ifndef SB_P1_MATCH
#define SB_P1_MATCH 0
#endif
#ifndef SB_P1_DIRECT_BPS
#define SB_P1_DIRECT_BPS 4
#endif
constexpr int kStageBytes = SB_P1_STAGE_KB * 1024;   // 16 KiB: 512 32-B tuples, 2 iterations per warp per stage
constexpr int kStages = SB_P1_STAGES;
enum { TM_LANE = 0, TM_DIRECT = 1, TM_HASHED = 2, TM_SHARED = 3 };


// x / d for x >= 0 via a double reciprocal and exact integer correction
__device__ __forceinline__ int64_t fdiv(int64_t x, int64_t d, double inv) {
  if (d == 1) return x;
  if (x < (1ll << 52)) {
    int64_t q = (int64_t)((double)x * inv);
    int64_t r = x - q * d;
    while (r < 0) { --q; r += d; }
    while (r >= d) { ++q; r -= d; }
    return q;
  }
  return x / d;
}
// pane division: shift for power-of-two pane lengths, reciprocal otherwise
// trunc(v / d) for int32 v and 0 < d < 2^31 (C semantics), via the double
// reciprocal inv = 1/d and one exact integer correction
__device__ __forceinline__ int32_t div_trunc32(int32_t v, int32_t d, double inv) {
  const uint32_t a = v < 0 ? 0u - (uint32_t)v : (uint32_t)v;
  uint32_t q = (uint32_t)((double)a * inv);
  const int64_t r = (int64_t)a - (int64_t)q * d;
  if (r < 0) --q;
  else if (r >= d) ++q;
  return v < 0 ? -(int32_t)q : (int32_t)q;
}

__device__ __forceinline__ int64_t pdiv(const Plan &p, int64_t x) {
  return p.g_shift >= 0 ? (x >> p.g_shift) : fdiv(x, p.g, p.g_inv);
}

__device__ __forceinline__ uint64_t s_key(const Plan &p, const unsigned char *t, bool &valid, int &err) {
  if (p.key_mode == KM_GLOBAL) return 0;
  uint64_t k = 0;
  bool bad = false;
  if (p.key_pack == KP_RADIX) {
    for (int i = 0; i < p.nkeys; ++i) {
      int64_t v = s_int(t, p.key[i].word, p.key[i].type);
      if (p.key[i].div != 1) v /= p.key[i].div;
      bad |= (v < 0) | (v >= p.key[i].domain);
      k += (uint64_t)v * (uint64_t)p.key[i].stride;
    }
  } else if (p.key_pack == KP_BIASED64) {
    int64_t v = s_int(t, p.key[0].word, p.key[0].type);
    if (p.key[0].div != 1) v /= p.key[0].div;
    k = (uint64_t)v ^ 0x8000000000000000ull;
    bad = (k == kEmpty);
  } else {
    int64_t v0 = s_int(t, p.key[0].word, p.key[0].type), v1 = s_int(t, p.key[1].word, p.key[1].type);
    if (p.key[0].div != 1) v0 /= p.key[0].div;
    if (p.key[1].div != 1) v1 /= p.key[1].div;
    bad = (v0 != (int32_t)v0) | (v1 != (int32_t)v1);
    k = ((uint64_t)((uint32_t)v0 ^ 0x80000000u) << 32) | (uint64_t)((uint32_t)v1 ^ 0x80000000u);
    bad |= (k == kEmpty);
  }
  if (valid && bad) { err |= ERR_KEY; valid = false; }
  return k;
}

__device__ __forceinline__ uint64_t s_field(const Field &f, const unsigned char *t) {
  const bool fl = (f.type == T_F32 || f.type == T_F64);
  switch (f.kind) {
    case FK_SUM_F: return (uint64_t)__double_as_longlong(s_flt(t, f.word, f.type));
    case FK_SUM_I: return (uint64_t)s_int(t, f.word, f.type);
    default: return fl ? enc_dbl(s_flt(t, f.word, f.type)) : enc_int(s_int(t, f.word, f.type));
  }
}

__device__ __forceinline__ uint64_t fadd64(uint64_t a, uint64_t b) {
  return (uint64_t)__double_as_longlong(__longlong_as_double((long long)a) + __longlong_as_double((long long)b));
}

// shared-memory atomic update of one accumulator field
__device__ __forceinline__ void atom_field(int kind, uint64_t *addr, uint64_t v) {
  switch (kind) {
    case FK_SUM_F: atomicAdd((double *)addr, __longlong_as_double((long long)v)); break;
    case FK_SUM_I: atomicAdd((unsigned long long *)addr, (unsigned long long)v); break;
    case FK_MIN: atomicMin((unsigned long long *)addr, (unsigned long long)v); break;
    default: atomicMax((unsigned long long *)addr, (unsigned long long)v); break;
  }
}

// add one pre-aggregated (pane, key) entry into the device pane ring
template <int NF, bool BM = true>
__device__ __forceinline__ void flush_entry(const Plan &p, State *st, uint64_t *table, int64_t pane, uint64_t key,
                                            uint32_t c, const uint64_t (&fv)[NF], int &err) {
  uint64_t *base = table + (pane & (p.R - 1)) * p.slot_words;
  if (BM && p.pane_bm)                          // dense keys only (C <= 256): presence bit of (pane, key)
    atomicOr(pane_bm_words(p, table) + (pane & (p.R - 1)) * 8 + (key >> 5), 1u << (key & 31));
  int64_t idx;
  if (p.key_mode == KM_HASH) {
    idx = global_insert(p, st, base, key, err);
    if (idx < 0) return;
  } else {
    idx = (int64_t)key;
  }
  atomicAdd((unsigned long long *)&base[cnt_off(p) + idx], (unsigned long long)c);
#pragma unroll
  for (int i = 0; i < NF; ++i)
    if (i < p.nf) red_field(p.field[i].kind, &base[fld_off(p, i) + idx], fv[i]);
}

// sum the warp (and lane) copies of each table entry of the pane window starting
// at pbase, one set of L2 REDs per (pane, key) per CTA; CTA-collective
template <int MODE, int NF, bool FAST>
__device__ __forceinline__ void flush_tables(const Plan &p, State *st, uint64_t *table, unsigned char *tabs,
                                          uint64_t *tf, uint32_t *tcnt, int64_t pbase, int &err) {
  const int tid = threadIdx.x, lane = tid & 31;
  const int TE = p.local_entries;
  const int CW = MODE == TM_LANE ? 32 : 1;
  constexpr int NCOPY = MODE == TM_SHARED ? 1 : kP1Warps;
  const int C = (int)p.C;

  if (MODE == TM_LANE) {
    // each warp first folds its 32 lane columns into lane 0's copy (shuffles)
    __syncwarp();
    for (int e = 0; e < TE; ++e) {
      const int x = e * 32 + lane;
      const uint32_t cl = tcnt[x];
      if (!__any_sync(kFull, cl != 0)) continue;
      const uint32_t c = __reduce_add_sync(kFull, cl);
      if (lane == 0) tcnt[x] = c; else tcnt[x] = 0;
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        if (!FAST && f >= p.nf) break;
        const int kind = FAST ? FK_SUM_F : p.field[f].kind;
        uint64_t v = tf[f * TE * 32 + x];
#pragma unroll
        for (int o = 16; o; o >>= 1)
          v = FAST ? fadd64(v, shfl_xor64(v, o)) : field_combine(kind, v, shfl_xor64(v, o));
        tf[f * TE * 32 + x] = lane == 0 ? v : field_identity(kind);
      }
    }
    __syncwarp();
  }
  __syncthreads();
  for (int e = tid; e < TE; e += kP1Threads) {
    uint32_t c = 0;
    uint64_t fv[NF];
#pragma unroll
    for (int f = 0; f < NF; ++f) fv[f] = f < p.nf ? field_identity(p.field[f].kind) : 0;
    for (int w = 0; w < NCOPY; ++w) {
      uint64_t *of = (uint64_t *)(tabs + (size_t)w * p.local_bytes);
      uint32_t *oc = (uint32_t *)((unsigned char *)of + (size_t)8 * TE * CW * NF);
      for (int l = 0; l < (MODE == TM_LANE ? 1 : CW); ++l) {
        const int x = e * CW + l;                        // LANE: lane 0 holds the warp total
        const uint32_t cw = oc[x];
        if (!cw) continue;
        c += cw;
        oc[x] = 0;
#pragma unroll
        for (int f = 0; f < NF; ++f)
          if (f < p.nf) {
            fv[f] = field_combine(p.field[f].kind, fv[f], of[f * TE * CW + x]);
            of[f * TE * CW + x] = field_identity(p.field[f].kind);
          }
      }
    }
    if (c) flush_entry<NF>(p, st, table, pbase + e / C, (uint64_t)(e % C), c, fv, err);
  }
  __syncthreads();
}

// FX3 tables of k_pane_agg (Plan::fx_agg): a sum field is three u32 limbs taking
// the 16-bit chunks of X = x·2^32 for x in [0, 2^16) and a multiple of 2^-32
// (SG's 1000·u24, LRB speeds, u24 values), with fire-and-forget shared REDs; a
// limb takes <= 65,535 chunks of <= 0xffff between flushes (the CTA flushes every
// 2^16 - stage tuples), so it cannot wrap.  Other values go as fp64 straight to
// the pane ring (RED.ADD.F64).  Layout per warp (or CTA): [NF][3][TE] limbs, [TE] counts.
__device__ __forceinline__ bool fx48(uint32_t xb, uint64_t &X) {
  const uint32_t ex = (xb >> 23) & 0xffu;
  const uint32_t m = (xb & 0x7fffffu) | 0x800000u;
  X = 0;
  if (xb == 0u) return true;
  if ((xb >> 31) || ex >= 143u || ex == 0u) return false;
  if (ex >= 118u) { X = (uint64_t)m << (ex - 118u); return true; }
  const uint32_t sh = 118u - ex;
  if (sh > 23u || (m & ((1u << sh) - 1u))) return false;
  X = m >> sh;
  return true;
}
__device__ __forceinline__ void red_add_u32(uint32_t *p, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(p)), "r"(v) : "memory");
}
template <int MODE, int NF>
__device__ __forceinline__ void flush_fx3(const Plan &p, State *st, uint64_t *table, unsigned char *tabs,
                                          int64_t pbase, int &err) {
  const int tid = threadIdx.x;
  const int TE = p.local_entries;
  constexpr int NCOPY = MODE == TM_SHARED ? 1 : kP1Warps;
  const int C = (int)p.C;
  __syncthreads();
  for (int e = tid; e < TE; e += kP1Threads) {
    uint32_t c = 0;
    double sum[NF];
#pragma unroll
    for (int f = 0; f < NF; ++f) sum[f] = 0.0;
    for (int w = 0; w < NCOPY; ++w) {
      uint32_t *lm = (uint32_t *)(tabs + (size_t)w * p.local_bytes);
      uint32_t *oc = lm + 3 * NF * TE;
      const uint32_t cw = oc[e];
      if (!cw) continue;
      c += cw;
      oc[e] = 0;
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        uint32_t *l = lm + 3 * f * TE;
        sum[f] += (double)l[e] * 0x1p-32 + (double)l[TE + e] * 0x1p-16 + (double)l[2 * TE + e];
        l[e] = 0;
        l[TE + e] = 0;
        l[2 * TE + e] = 0;
      }
    }
    if (c) {
      uint64_t fv[NF];
#pragma unroll
      for (int f = 0; f < NF; ++f) fv[f] = (uint64_t)__double_as_longlong(sum[f]);
      flush_entry<NF>(p, st, table, pbase + e / C, (uint64_t)(e % C), c, fv, err);
    }
  }
  __syncthreads();
}

// NK >= 0 (FAST plans): exactly NK radix-packed int32 key columns, known at
// compile time (no per-tuple loop bounds and plan-field branches); -1: run time
template <int MODE, int WK, int NF, bool FAST, int NK = -1>
__global__ void __launch_bounds__(kP1Threads, MODE == TM_DIRECT ? SB_P1_DIRECT_BPS : 2)
k_pane_agg(const Plan p, State *__restrict__ st, const unsigned char *__restrict__ tup, int64_t n,
           uint64_t *__restrict__ table, int64_t *__restrict__ pane_ts) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ long long s_next;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int tb = p.tuple_bytes;
  const int ST = kStageBytes / tb;                       // tuples per stage
  unsigned char *stages = smem;
  uint64_t *full = (uint64_t *)(smem + kStages * kStageBytes);
  uint64_t *empty = full + kStages;
  unsigned char *tabs = (unsigned char *)(empty + kStages);
  // table geometry: TE entries per warp; LANE mode stores every entry once per lane
  const int TE = p.local_entries;
  const int CW = MODE == TM_LANE ? 32 : 1;               // copies of an entry (lanes)
  unsigned char *wt = tabs + (MODE == TM_SHARED ? 0 : (size_t)wid * p.local_bytes);
  uint64_t *tkeys = (uint64_t *)wt;                      // HASHED only
  uint64_t *tf = (uint64_t *)(wt + (MODE == TM_HASHED ? 8 * TE : 0));   // [NF][TE*CW]
  constexpr bool FXM = FAST && (MODE == TM_DIRECT || MODE == TM_SHARED);
  const bool fx = FXM && p.fx_agg;                       // CTA-uniform
  uint32_t *tlimb = (uint32_t *)wt;                      // fx: [NF][3][TE] limbs
  uint32_t *tcnt = (uint32_t *)((unsigned char *)tf + (size_t)(fx ? 12 : 8) * TE * CW * NF);   // [TE*CW]
  for (int e = (MODE == TM_SHARED ? tid : lane); e < TE * CW; e += (MODE == TM_SHARED ? kP1Threads : 32)) {
    if (MODE == TM_HASHED) tkeys[e] = kEmpty;
    tcnt[e] = 0;
    if (fx) {
#pragma unroll
      for (int f = 0; f < 3 * NF; ++f) tlimb[f * TE + e] = 0;
    } else {
#pragma unroll
      for (int f = 0; f < NF; ++f) tf[f * TE * CW + e] = f < p.nf ? field_identity(p.field[f].kind) : 0;
    }
  }
  int fx_since = 0;                                      // tuples since the last flush (limb bound)

  // rounds (Plan::rounds > 1): this launch scans the sub-range k_task_begin chose
  if (p.rounds > 1) {
    tup += st->round_off * tb;
    n = st->round_n;
  }
  // contiguous, stage-aligned range of this CTA
  const int64_t per = ((n + gridDim.x - 1) / gridDim.x + ST - 1) / ST * ST;
  const int64_t lo = (int64_t)blockIdx.x * per;
  const int64_t hi = lo + per < n ? lo + per : n;
  const int nst = hi > lo ? (int)((hi - lo + ST - 1) / ST) : 0;
  if (tid == 0) {
    for (int i = 0; i < kStages; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], kP1Warps); }
    fence_mbar_init();
  }
  __syncthreads();
  auto issue = [&](int k) {
    const int slot = k % kStages;
    const int64_t cnt = (hi - lo - (int64_t)k * ST) < ST ? (hi - lo - (int64_t)k * ST) : ST;
    const uint32_t bytes = (uint32_t)(cnt * tb);
    mbar_expect_tx(&full[slot], bytes);
    bulk_g2s(stages + slot * kStageBytes, tup + (lo + (int64_t)k * ST) * tb, bytes, &full[slot]);
  };
  if (tid == 0)
    for (int k = 0; k < kStages && k < nst; ++k) issue(k);

  const int64_t pos0 = st->task_pos;
  const int64_t min_pane = st->J0 * p.L;
  const int PL = MODE == TM_HASHED ? 1 : p.local_pl;
  const int C = (int)p.C;
  const int tsw = p.ts_word;
  int err = 0;
  int occ = 0;
  int64_t pbase = -1;      // CTA-uniform pane window [pbase, pbase + PL)
  int64_t prev_last = (lo > 0 && lo < hi) ? *(const int64_t *)(tup + (lo - 1) * tb + 4 * tsw) : INT64_MIN;
  const int per_warp = (ST + kP1Warps - 1) / kP1Warps;

  auto flush_shared = [&]() {
    if (FXM && fx) flush_fx3<MODE, NF>(p, st, table, tabs, pbase, err);
    else flush_tables<MODE, NF, FAST>(p, st, table, tabs, tf, tcnt, pbase, err);
    fx_since = 0;
  };
  auto flush_hashed = [&]() {      // warp-private table of one pane
    __syncwarp();
    for (int e = lane; e < TE; e += 32) {
      const uint64_t k = tkeys[e];
      if (k == kEmpty) continue;
      uint64_t fv[NF];
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        fv[f] = tf[f * TE + e];
        if (f < p.nf) tf[f * TE + e] = field_identity(p.field[f].kind);
      }
      flush_entry<NF>(p, st, table, pbase, k, tcnt[e], fv, err);
      tkeys[e] = kEmpty;
      tcnt[e] = 0;
    }
    __syncwarp();
    occ = 0;
  };

  // count windows: 32-bit pane arithmetic when a pane window spans < 2^30 positions
  const int g32 = (p.g * (int64_t)(PL + 2) < (1ll << 30)) ? (int)p.g : 0;
  const int range32 = (int)(hi - lo);                     // tuples of this CTA (< 2^31)
  int64_t spos = pos0 + lo;                               // global position of stage tuple 0
  int slot = 0;
  uint32_t phase = 0;
  for (int k = 0; k < nst; ++k, spos += ST) {
    mbar_wait(&full[slot], phase);
    const unsigned char *sb = stages + slot * kStageBytes;
    const int ntup = range32 - k * ST < ST ? range32 - k * ST : ST;
    int64_t pf, pl;                                        // stage pane range (CTA-uniform)
    if (WK == WK_COUNT) {
      pf = pdiv(p, spos);
      pl = pdiv(p, spos + ntup - 1);
    } else {
      const int64_t t0 = *(const int64_t *)(sb + 4 * tsw), t1 = *(const int64_t *)(sb + (ntup - 1) * tb + 4 * tsw);
      pf = t0 >= p.T0 ? pdiv(p, t0 - p.T0) : 0;
      pl = t1 >= p.T0 ? pdiv(p, t1 - p.T0) : -1;
    }
    if (pf < min_pane) pf = min_pane;
    const int ib = wid * per_warp;
    const int ie = ib + per_warp < ntup ? ib + per_warp : ntup;
    int64_t cur = pf;
    bool first_round = true;
    while (cur <= pl) {
      if (pbase < 0 || cur < pbase || cur >= pbase + PL) {
        if (pbase >= 0) {
          if (MODE == TM_HASHED) flush_hashed(); else flush_shared();
        }
        pbase = cur;
      }
      const int64_t wend = pbase + PL;
      const int64_t wlo = pbase > min_pane ? pbase : min_pane;
      const bool all_in = (pf >= wlo) & (pl < wend);    // CTA-uniform: no per-tuple window test
      const int lo_ofs = (int)(wlo - pbase);             // first live offset in the window
      // count windows: this lane's tuple as (pane offset from pbase, position in the pane)
      int po = 0, cr = 0;
      int64_t cp = 0;
      if (WK == WK_COUNT) {
        const int64_t pos = spos + ib + lane;
        if (g32) {
          const int r = (int)(pos - pbase * p.g);       // < 0 for tuples before the window (later rounds)
          po = p.g_shift >= 0 ? (r >> p.g_shift) : (r >= 0 ? r / g32 : -((g32 - 1 - r) / g32));
          cr = r - po * g32;                            // in [0, g): floor division
        } else {
          cp = pdiv(p, pos);
          cr = (int)(pos - cp * p.g);
        }
      }
#pragma unroll 2
      for (int i0 = ib; i0 < ie; i0 += 32) {
        const int i = i0 + lane;
        bool valid = i < ie;
        const unsigned char *t = sb + (valid ? i : ib) * tb;
        const int64_t tau = *(const int64_t *)(t + 4 * tsw);
        if (first_round) {
          // K1: τ non-decreasing (L347-349) and non-negative (L349-350); the
          // predecessor of lane 0 is the previous iteration's lane 31
          const int64_t up = i > 0 ? *(const int64_t *)(t - tb + 4 * tsw) : prev_last;   // predecessor τ
          if (valid & (tau < up)) err |= ERR_ORDER;
          if (valid & (tau < 0)) err |= ERR_TS;
        }
        int64_t pane;
        int pw;                                          // this tuple's pane offset from pbase
        if (WK == WK_COUNT && g32) {
          pw = po;
          pane = pbase + po;
          if (first_round && valid && cr == 0 && po >= lo_ofs) pane_ts[pane & (p.R - 1)] = tau;
          if (!all_in) valid &= (po >= lo_ofs) & (po < PL);
          cr += 32;
          while (cr >= g32) { cr -= g32; ++po; }
        } else {
          if (WK == WK_COUNT) {
            pane = cp;
            if (first_round && valid && cr == 0 && pane >= min_pane) pane_ts[pane & (p.R - 1)] = tau;
            cr += 32;
            while (cr >= (int)p.g) { cr -= (int)p.g; ++cp; }
          } else {
            valid &= tau >= p.T0;
            pane = tau >= p.T0 ? pdiv(p, tau - p.T0) : -1;
          }
          if (!all_in) valid &= (pane >= pbase) & (pane < wend) & (pane >= min_pane);
          pw = (int)(pane - pbase);
        }
        if (p.npred && valid) valid &= s_preds(p, t);
        uint64_t key;
        uint64_t fv[NF];
        if (FAST) {
          // all fields are fp64 sums of f32 columns; at most one int32 key column, div 1
          if (NK == 0 || (NK < 0 && p.key_mode == KM_GLOBAL)) key = 0;
          else if (NK > 0 || p.key_pack == KP_RADIX) {
            // radix-packed int32 key columns, each col / div (C truncation, A17)
            uint64_t kk = 0;
            bool bad = false;
#pragma unroll
            for (int kc = 0; kc < (NK > 0 ? NK : kMaxKey); ++kc) {
              if (NK > 0 || kc < p.nkeys) {
                int32_t v = *(const int32_t *)(t + 4 * p.key[kc].word);
                if (p.key[kc].div != 1) v = div_trunc32(v, p.key[kc].div, p.key[kc].inv);
                bad |= (uint32_t)v >= (uint32_t)p.key[kc].domain;     // domain < 2^31 on the fast path
                kk += (uint64_t)(uint32_t)v * (uint64_t)p.key[kc].stride;
              }
            }
            if (bad) {
              if (valid) err |= ERR_KEY;
              valid = false;
            }
            key = kk;
          } else {
            const int32_t v = *(const int32_t *)(t + 4 * p.key[0].word);
            key = (uint64_t)(int64_t)v ^ 0x8000000000000000ull;
          }
#pragma unroll
          for (int f = 0; f < NF; ++f)
            fv[f] = (uint64_t)__double_as_longlong((double)*(const float *)(t + 4 * p.field[f].word));
        } else {
          key = s_key(p, t, valid, err);
#pragma unroll
          for (int f = 0; f < NF; ++f) fv[f] = (f < p.nf) ? s_field(p.field[f], t) : 0;
        }
        if (MODE == TM_LANE) {
          if (valid) {       // this lane's own column: plain read-modify-write
            const int e = (pw * C + (int)key) * 32 + lane;
            tcnt[e] += 1u;
#pragma unroll
            for (int f = 0; f < NF; ++f)
              if (FAST) tf[f * TE * 32 + e] = fadd64(tf[f * TE * 32 + e], fv[f]);
              else if (f < p.nf)
                tf[f * TE * 32 + e] = field_combine(p.field[f].kind, tf[f * TE * 32 + e], fv[f]);
          }
        } else if (MODE == TM_DIRECT || MODE == TM_SHARED) {
          if (valid && FXM && fx) {
            const int e = pw * C + (int)key;
            red_add_u32(&tcnt[e], 1u);
#pragma unroll
            for (int f = 0; f < NF; ++f) {
              const float xf = (float)__longlong_as_double((long long)fv[f]);   // exact: an f32 widened
              uint64_t X;
              if (fx48(__float_as_uint(xf), X)) {
                uint32_t *l = tlimb + 3 * f * TE + e;
                red_add_u32(l, (uint32_t)X & 0xffffu);
                red_add_u32(l + TE, (uint32_t)(X >> 16) & 0xffffu);
                if (X >> 32) red_add_u32(l + 2 * TE, (uint32_t)(X >> 32));
              } else {
                atomicAdd((double *)&table[((pbase + pw) & (p.R - 1)) * p.slot_words + fld_off(p, f) + key],
                          __longlong_as_double((long long)fv[f]));
              }
            }
          } else if (valid) {
            const int e = pw * C + (int)key;
            atomicAdd(&tcnt[e], 1u);
#pragma unroll
            for (int f = 0; f < NF; ++f)
              if (FAST) atomicAdd((double *)&tf[f * TE + e], __longlong_as_double((long long)fv[f]));
              else if (f < p.nf) atom_field(p.field[f].kind, &tf[f * TE + e], fv[f]);
          }
        } else {
          if (occ + 32 > TE / 2) flush_hashed();     // keep the load factor <= 1/2
          bool ins = false;
          if (valid) {
            uint32_t h = (uint32_t)fmix64(key) & (uint32_t)(TE - 1);
            volatile uint64_t *vk = tkeys;
            for (;;) {
              const uint64_t kk = vk[h];
              if (kk == key) break;
              if (kk == kEmpty) {
                const uint64_t old = atomicCAS((unsigned long long *)&tkeys[h], kEmpty, key);
                if (old == kEmpty) { ins = true; break; }
                if (old == key) break;
              }
              h = (h + 1) & (uint32_t)(TE - 1);
            }
            atomicAdd(&tcnt[h], 1u);
#pragma unroll
            for (int f = 0; f < NF; ++f)
              if (FAST) atomicAdd((double *)&tf[f * TE + h], __longlong_as_double((long long)fv[f]));
              else if (f < p.nf) atom_field(p.field[f].kind, &tf[f * TE + h], fv[f]);
          }
          occ += __popc(__ballot_sync(kFull, ins));
        }
      }
      first_round = false;
      if (pl < wend) break;
      // next non-empty pane >= wend in this stage (time gaps, tiny panes)
      if (tid == 0) s_next = LLONG_MAX;
      __syncthreads();
      for (int i = ib + lane; i < ie; i += 32) {
        const unsigned char *t = sb + i * tb;
        int64_t pane;
        if (WK == WK_COUNT) pane = pdiv(p, spos + i);
        else {
          const int64_t tau = *(const int64_t *)(t + 4 * tsw);
          pane = tau >= p.T0 ? pdiv(p, tau - p.T0) : -1;
        }
        if (pane >= wend) atomicMin(&s_next, (long long)pane);
      }
      __syncthreads();
      cur = s_next;
      __syncthreads();
    }
    prev_last = *(const int64_t *)(sb + (ntup - 1) * tb + 4 * tsw);
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[slot]);
    if (tid == 0 && k + kStages < nst) {
      mbar_wait(&empty[slot], phase);
      issue(k + kStages);
    }
    if (++slot == kStages) { slot = 0; phase ^= 1u; }
    if (FXM && fx) {                                     // limbs take < 2^16 chunks between flushes
      fx_since += ntup;
      if (fx_since + ST >= 65535 && pbase >= 0) flush_shared();
    }
  }
  if (pbase >= 0) {
    if (MODE == TM_HASHED) flush_hashed(); else flush_shared();
  }
  if (err) atomicOr(&st->error, err);
}

// ---------------------------------------------------------------------------
// Count windows, fast path (no σ, fp64 sums of f32 columns, no key or one dense
// int32 key): the same pass as k_pane_agg with all per-stage and per-tuple pane
// arithmetic in 32 bits relative to the CTA's first pane P0 (division by g via
// the invariant-divisor multiply, Plan::g_magic), stage bytes read through
// 32-bit shared addresses, and no runtime key/predicate dispatch.  Count-window
// panes are contiguous, so a stage's panes [pf, pl] are all non-empty.
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ int64_t lds_s64(uint32_t a) {
  int64_t v;
  asm volatile("ld.shared.s64 %0, [%1];" : "=l"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ int divg(const Plan &p, int x) {     // floor(x / g), 0 <= x < 2^30
  return (int)(((uint64_t)(uint32_t)x * p.g_magic) >> p.g_mshift);
}

enum { KK_GLOBAL = 1, KK_RADIX = 2 };

__device__ __forceinline__ uint4 lds_v4(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t sel4(const uint4 &v, int w) {
  return w == 0 ? v.x : w == 1 ? v.y : w == 2 ? v.z : v.w;
}

// ONECH: τ, the key and every field lie in one 16-byte chunk of the tuple (Syn:
// chunk 0), so a tuple costs one 128-bit shared load instead of one 8-way
// bank-conflicted 32-bit load per field
// OC: 0 fields loaded one by one; 1 one 16-byte chunk, word positions chosen at
// run time; 2 one chunk with τ in words 0-1, the value in word 2 and the key in
// word 3 (the Syn layout, L1473-1476: ts, a1, a2), selected at compile time
// (the run-time word selects compile to branch trees in the hot loop)
template <int W>
__device__ __forceinline__ uint32_t sel4c(const uint4 &v) {
  return W == 0 ? v.x : W == 1 ? v.y : W == 2 ? v.z : v.w;
}

// FX tables (DIRECT / SHARED, one f32 sum column, pane length g < 2^16): a value
// x in [0, 1) that is a multiple of 2^-32 -- every u24 value of the Syn stream --
// is added exactly as the 32-bit integer X = x·2^32, split into two 16-bit
// chunks that go to two u32 limbs with fire-and-forget shared atomics
// (red.shared.add.u32 = ATOMS.ADD, no return value, no scoreboard wait) instead
// of an fp64 atomicAdd, which sm_100a executes as a CAS loop (ATOMS.CAST.SPIN.64;
// scripts/ubench_pane_accum.cu: 0.82 -> 0.30 SM-cycles per update).  A limb
// receives at most g chunks of <= 0xffff between flushes, so it cannot wrap.
// Any other value (negative, >= 1, finer than 2^-32, non-finite) is added in
// fp64 into a CTA-wide side table (shared CAS loop, a rare path), so every f32
// input is summed; the flush converts the limbs exactly (< 2^53) and adds the
// side word.
__device__ __forceinline__ bool fx32(uint32_t xb, uint32_t &X) {
  const uint32_t ex = (xb >> 23) & 0xffu;
  const uint32_t m = (xb & 0x7fffffu) | 0x800000u;
  X = 0;
  if (xb == 0u) return true;
  if ((xb >> 31) || ex >= 127u || ex == 0u) return false;
  if (ex >= 118u) { X = m << (ex - 118u); return true; }
  const uint32_t sh = 118u - ex;                 // 1 .. 117
  if (sh > 23u || (m & ((1u << sh) - 1u))) return false;
  X = m >> sh;
  return true;
}
// shared-memory address (u32, from __cvta_generic_to_shared once per kernel)
__device__ __forceinline__ void red_add_s(uint32_t saddr, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(saddr), "r"(v) : "memory");
}

// flush of FX tables: sum the copies' count and limbs of each entry, one set of
// L2 REDs per (pane, key) per CTA (as flush_tables); CTA-collective
// Panes wholly inside this CTA's tuples (selfzero, CTA-relative pane r with
// r·g - R0 in [0, range - g]) have no other writer: their slots are written with
// plain stores, zeros for absent keys included, so k_zero_panes skips them and no
// RED has to fetch their lines (k_zero_panes initialises only the panes that hold
// a CTA boundary).  side: per entry, the fp64 sum of the values the limbs cannot
// hold (added into the ring by the flush, never straight into the table).
template <int MODE>
__device__ __forceinline__ void flush_fx(const Plan &p, State *st, uint64_t *table, unsigned char *tabs,
                                         int64_t pbase, int &err, double *side, int selfzero, int64_t P0, int R0,
                                         int range, int minrel) {
  const int tid = threadIdx.x;
  const int TE = p.local_entries;
  constexpr int NCOPY = MODE == TM_SHARED ? 1 : kP1Warps;
  const int C = (int)p.C;
  const int64_t g = p.g, Rm = p.R - 1;
  __syncthreads();
  for (int e = tid; e < TE; e += kP1Threads) {
    uint32_t c = 0;
    uint64_t X = 0;
    for (int w = 0; w < NCOPY; ++w) {
      uint32_t *lm = (uint32_t *)(tabs + (size_t)w * p.local_bytes);
      uint32_t *oc = lm + 2 * TE;
      const uint32_t cw = oc[e];
      if (!cw) continue;
      c += cw;
      X += (uint64_t)lm[2 * e] + ((uint64_t)lm[2 * e + 1] << 16);
      oc[e] = 0;
      lm[2 * e] = 0;
      lm[2 * e + 1] = 0;
    }
    const double sx = side[e];
    side[e] = 0.0;
    const int64_t pane = pbase + e / C;
    const int64_t r = pane - P0, t0 = r * g - R0;
    const bool own = selfzero && r >= minrel && t0 >= 0 && t0 + g <= range;
    if (p.pane_bm) {                          // 32 consecutive entries: one pane, one 32-key chunk
      const unsigned bal = __ballot_sync(kFull, c != 0);
      uint32_t *bw = pane_bm_words(p, table) + (pane & Rm) * 8 + (e % C) / 32;
      if ((tid & 31) == 0) {
        if (own) *bw = bal;
        else if (bal) atomicOr(bw, bal);
      }
    }
    const double sum = (double)X * 0x1p-32 + sx;                                       // limbs exact: X < 2^53
    if (own) {
      uint64_t *base = table + (pane & Rm) * p.slot_words;
      base[e % C] = (uint64_t)c;
      base[C + e % C] = (uint64_t)__double_as_longlong(sum);
    } else if (c) {
      const uint64_t fv[1] = {(uint64_t)__double_as_longlong(sum)};
      flush_entry<1, false>(p, st, table, pane, (uint64_t)(e % C), c, fv, err);
    }
  }
  __syncthreads();
}

template <int MODE, int NF, int KK, int OC, bool FX = false>
__global__ void __launch_bounds__(kP1Threads, MODE == TM_DIRECT ? SB_P1_DIRECT_BPS : 2)
k_pane_cnt(const Plan p, State *__restrict__ st, const unsigned char *__restrict__ tup, int64_t n,
           uint64_t *__restrict__ table, int64_t *__restrict__ pane_ts, int selfzero) {
  constexpr bool ONECH = OC != 0;
  static_assert(OC != 2 || NF == 1, "fixed layout: one value column");
  extern __shared__ __align__(128) unsigned char smem[];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int tb = OC == 2 ? 32 : p.tuple_bytes;                 // the fixed layout is the 32-B Syn tuple
  const int ST = kStageBytes / tb;
  unsigned char *stages = smem;
  uint64_t *full = (uint64_t *)(smem + kStages * kStageBytes);
  uint64_t *empty = full + kStages;
  unsigned char *tabs = (unsigned char *)(empty + kStages);
  const int TE = p.local_entries;
  const int CW = MODE == TM_LANE ? 32 : 1;
  // FX: fp64 side table of values the limbs cannot hold, one word per entry (CTA-wide)
  double *side = (double *)(tabs + (size_t)(MODE == TM_SHARED ? 1 : kP1Warps) * p.local_bytes);
  if (FX)
    for (int e = tid; e < TE; e += kP1Threads) side[e] = 0.0;
  unsigned char *wt = tabs + (MODE == TM_SHARED ? 0 : (size_t)wid * p.local_bytes);
  uint64_t *tf = (uint64_t *)wt;                                    // [NF][TE*CW]
  uint32_t *tcnt = (uint32_t *)(wt + (size_t)8 * TE * CW * NF);     // [TE*CW]
  for (int e = (MODE == TM_SHARED ? tid : lane); e < TE * CW; e += (MODE == TM_SHARED ? kP1Threads : 32)) {
    tcnt[e] = 0;
#pragma unroll
    for (int f = 0; f < NF; ++f) tf[f * TE * CW + e] = 0;          // fp64 +0.0
  }
  const int64_t per = ((n + gridDim.x - 1) / gridDim.x + ST - 1) / ST * ST;
  const int64_t lo = (int64_t)blockIdx.x * per;
  const int64_t hi = lo + per < n ? lo + per : n;
  const int nst = hi > lo ? (int)((hi - lo + ST - 1) / ST) : 0;
  if (tid == 0) {
    for (int i = 0; i < kStages; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], kP1Warps); }
    fence_mbar_init();
  }
  __syncthreads();
  auto issue = [&](int k) {
    const int slot = k % kStages;
    const int64_t cnt = (hi - lo - (int64_t)k * ST) < ST ? (hi - lo - (int64_t)k * ST) : ST;
    const uint32_t bytes = (uint32_t)(cnt * tb);
    mbar_expect_tx(&full[slot], bytes);
    bulk_g2s(stages + slot * kStageBytes, tup + (lo + (int64_t)k * ST) * tb, bytes, &full[slot]);
  };
  if (tid == 0)
    for (int k = 0; k < kStages && k < nst; ++k) issue(k);

  // CTA-relative pane coordinates: global pane = P0 + rel, rel of local tuple x = (R0 + x) / g
  const int64_t gpos = st->task_pos + lo;
  const int64_t P0 = gpos / p.g;
  const int R0 = (int)(gpos - P0 * p.g);
  const int64_t mp = st->J0 * p.L - P0;                      // panes < min_pane are dropped
  const int minrel = mp <= 0 ? 0 : (mp > (1 << 30) ? (1 << 30) : (int)mp);
  const int PL = p.local_pl;
  const int C = (int)p.C;
  const int g = (int)p.g;
  const uint32_t tsoff = 4u * p.ts_word;
  const uint32_t koff = KK == KK_RADIX ? 4u * p.key[0].word : 0u;
  const uint32_t dom = KK == KK_RADIX ? (uint32_t)p.key[0].domain : 1u;
  uint32_t foff[NF];
#pragma unroll
  for (int f = 0; f < NF; ++f) foff[f] = 4u * p.field[f].word;      // fast path: NF == p.nf
  // ONECH: word indices inside the shared 16-byte chunk
  const int ch = p.ts_word >> 2, tw = p.ts_word & 3, kw = KK == KK_RADIX ? p.key[0].word & 3 : 0;
  int fw[NF];
#pragma unroll
  for (int f = 0; f < NF; ++f) fw[f] = p.field[f].word & 3;
  const int64_t Rm = p.R - 1;
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(stages);
  const uint32_t s_tcnt = (uint32_t)__cvta_generic_to_shared(tcnt), s_tf = (uint32_t)__cvta_generic_to_shared(tf);
  int err = 0;
  int prel = -1;                                             // CTA-uniform pane window [prel, prel+PL)
  int64_t prev_last = (lo > 0 && lo < hi) ? *(const int64_t *)(tup + (lo - 1) * tb + tsoff) : INT64_MIN;
  const int per_warp = (ST + kP1Warps - 1) / kP1Warps;
  const int ib = wid * per_warp;
  const int range32 = (int)(hi - lo);
  int slot = 0;
  uint32_t phase = 0;
  for (int k = 0; k < nst; ++k) {
    mbar_wait(&full[slot], phase);
    const uint32_t sb = sbase + (uint32_t)(slot * kStageBytes);
    const int xs = k * ST;                                   // local index of the stage's tuple 0
    const int ntup = range32 - xs < ST ? range32 - xs : ST;
    int pf = divg(p, R0 + xs);
    const int pl = divg(p, R0 + xs + ntup - 1);
    // τ of every pane's first tuple in this stage (header ts of count windows, A7)
    for (int qq = divg(p, R0 + xs + g - 1) + tid; qq * g < R0 + xs + ntup; qq += kP1Threads)
      if (qq >= minrel) pane_ts[(P0 + qq) & Rm] = lds_s64(sb + (uint32_t)((qq * g - R0 - xs) * tb) + tsoff);
    if (pf < minrel) pf = minrel;
    const int ie = ib + per_warp < ntup ? ib + per_warp : ntup;
    bool first_round = true;
    for (int cur = pf; cur <= pl;) {
      if (prel < 0 || cur < prel || cur >= prel + PL) {
        if (prel >= 0) {
          if (FX) flush_fx<MODE>(p, st, table, tabs, P0 + prel, err, side, selfzero, P0, R0, range32, minrel);
          else flush_tables<MODE, NF, true>(p, st, table, tabs, tf, tcnt, P0 + prel, err);
        }
        prel = cur;
      }
      const int wend = prel + PL;
      const int wlo = prel > minrel ? prel : minrel;
      const bool all_in = (pf >= wlo) & (pl < wend);
      const int lo_ofs = wlo - prel;
#pragma unroll 2
      for (int i0 = ib; i0 < ie; i0 += 32) {
        const int i = i0 + lane;
        bool valid = i < ie;
        const uint32_t t = sb + (uint32_t)((valid ? i : ib) * tb);
        const int rel = R0 + xs + i;
        const int q = divg(p, rel);
        uint4 v4 = make_uint4(0, 0, 0, 0);
        if (ONECH) v4 = lds_v4(t + 16u * (uint32_t)ch);
        if (first_round) {
          // K1: τ non-decreasing (L347-349) and non-negative (L349-350); every lane
          // reads its predecessor's τ from the stage (no shuffles, no lane-0 branch),
          // the stage's first tuple compares with the previous stage's last
          const int64_t tau = OC == 2 ? (int64_t)(((uint64_t)sel4c<1>(v4) << 32) | sel4c<0>(v4))
                              : ONECH ? (int64_t)(((uint64_t)sel4(v4, tw + 1) << 32) | sel4(v4, tw)) : lds_s64(t + tsoff);
          const int64_t up = i > 0 ? lds_s64(t - tb + tsoff) : prev_last;
          if (valid & (tau < up)) err |= ERR_ORDER;
          if (valid & (tau < 0)) err |= ERR_TS;
        }
        const int po = q - prel;
        if (!all_in) valid &= (po >= lo_ofs) & (po < PL);
        uint32_t key = 0;
        if (KK == KK_RADIX) {
          key = OC == 2 ? sel4c<3>(v4) : ONECH ? sel4(v4, kw) : lds_u32(t + koff);
          if (key >= dom) {
            if (valid) err |= ERR_KEY;
            valid = false;
          }
        }
#if SB_P1_MATCH
        const unsigned vmask = __ballot_sync(kFull, valid);
#endif
        if (valid) {
          double fv[NF];
#pragma unroll
          for (int f = 0; f < NF; ++f)                                   // NF == nf
            fv[f] = (double)__uint_as_float(OC == 2 ? sel4c<2>(v4) : ONECH ? sel4(v4, fw[f]) : lds_u32(t + foff[f]));
#if SB_P1_MATCH
          // warp-private DIRECT table: a lane whose entry no other lane of this
          // iteration touches updates it with plain loads/stores (no CAS loop)
          const int em = po * C + (int)key;
          const bool solo = MODE == TM_DIRECT && __match_any_sync(vmask, em) == (1u << lane);
          if (solo) {
            tcnt[em] += 1u;
#pragma unroll
            for (int f = 0; f < NF; ++f) {
              double *a = (double *)&tf[f * TE + em];
              *a = *a + fv[f];
            }
          } else
#endif
          if (MODE == TM_LANE) {
            const int e = (po * C + (int)key) * 32 + lane;
            tcnt[e] += 1u;
#pragma unroll
            for (int f = 0; f < NF; ++f) {
              double *a = (double *)&tf[f * TE * 32 + e];
              *a = *a + fv[f];
            }
          } else if (FX) {
            const int e = po * C + (int)key;
            const uint32_t xb = OC == 2 ? sel4c<2>(v4) : ONECH ? sel4(v4, fw[0]) : lds_u32(t + foff[0]);
            uint32_t X;
            red_add_s(s_tcnt + 4u * (uint32_t)e, 1u);
            if (fx32(xb, X)) {
              const uint32_t lm = s_tf + 8u * (uint32_t)e;
              red_add_s(lm, X & 0xffffu);
              red_add_s(lm + 4u, X >> 16);
            } else {
              atomicAdd(&side[e], fv[0]);
            }
          } else {
            const int e = po * C + (int)key;
            atomicAdd(&tcnt[e], 1u);
#pragma unroll
            for (int f = 0; f < NF; ++f) atomicAdd((double *)&tf[f * TE + e], fv[f]);
          }
        }
#if SB_P1_MATCH
        __syncwarp();                                        // plain table updates visible to the next iteration
#endif
      }
      first_round = false;
      if (pl < wend) break;
      cur = wend;                                            // count-window panes are contiguous
    }
    prev_last = lds_s64(sb + (uint32_t)((ntup - 1) * tb) + tsoff);
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[slot]);
    if (tid == 0 && k + kStages < nst) {
      mbar_wait(&empty[slot], phase);
      issue(k + kStages);
    }
    if (++slot == kStages) { slot = 0; phase ^= 1u; }
  }
  if (prel >= 0) {
    if (FX) flush_fx<MODE>(p, st, table, tabs, P0 + prel, err, side, selfzero, P0, R0, range32, minrel);
    else flush_tables<MODE, NF, true>(p, st, table, tabs, tf, tcnt, P0 + prel, err);
  }
  if (err) atomicOr(&st->error, err);
}

// ---------------------------------------------------------------- host side
int p1_nf_template(int nf) { return nf <= 1 ? 1 : nf <= 2 ? 2 : nf <= 4 ? 4 : 8; }

static bool p1_cnt_fx(const Plan &p);
int p1_smem_bytes(const Plan &p) {
  return kStages * kStageBytes + 2 * kStages * 8 + (p.local_mode == TM_SHARED ? 1 : kP1Warps) * p.local_bytes +
         (p1_cnt_fx(p) ? (p.local_entries * 8 + 15) / 16 * 16 : 0);     // FX side table
}

template <int M, int WK, int NK>
static void *p1_fast_nk(int nf) {
  return nf <= 1 ? (void *)k_pane_agg<M, WK, 1, true, NK> : (void *)k_pane_agg<M, WK, 2, true, NK>;
}
// compile-time key count for FAST time-window plans with dense/global tables
template <int M, int WK>
static void *p1_fast(const Plan &p) {
  if (WK == WK_TIME && M != TM_HASHED && !std::getenv("SABER_NO_NK")) {
    if (p.key_mode == KM_GLOBAL) return p1_fast_nk<M, WK, 0>(p.nf);
    if (p.key_pack == KP_RADIX && p.key_mode != KM_HASH) {
      if (p.nkeys == 1) return p1_fast_nk<M, WK, 1>(p.nf);
      if (p.nkeys == 2) return p1_fast_nk<M, WK, 2>(p.nf);
      if (p.nkeys == 3) return p1_fast_nk<M, WK, 3>(p.nf);
    }
  }
  return p1_fast_nk<M, WK, -1>(p.nf);
}
template <int M, int WK>
static void *p1_nf(const Plan &p, int nf, bool fast) {
  if (fast) return p1_fast<M, WK>(p);
  switch (p1_nf_template(nf)) {
    case 1: return (void *)k_pane_agg<M, WK, 1, false>;
    case 2: return (void *)k_pane_agg<M, WK, 2, false>;
    case 4: return (void *)k_pane_agg<M, WK, 4, false>;
    default: return (void *)k_pane_agg<M, WK, 8, false>;
  }
}
template <int WK>
static void *p1_mode(const Plan &p) {
  const bool f = p.fast_keys;
  switch (p.local_mode) {
    case TM_LANE: return p1_nf<TM_LANE, WK>(p, p.nf, f);
    case TM_DIRECT: return p1_nf<TM_DIRECT, WK>(p, p.nf, f);
    case TM_SHARED: return p1_nf<TM_SHARED, WK>(p, p.nf, f);
    default: return p1_nf<TM_HASHED, WK>(p, p.nf, f);
  }
}
static void *p1_generic(const Plan &p) {
  return p.win_kind == WK_COUNT ? p1_mode<WK_COUNT>(p) : p1_mode<WK_TIME>(p);
}
// τ, the key and all fields in one 16-byte chunk (τ must not straddle chunks)
static bool one_chunk(const Plan &p) {
  const int ch = p.ts_word >> 2;
  if ((p.ts_word & 3) == 3) return false;
  if (p.key_mode != KM_GLOBAL && (p.key[0].word >> 2) != ch) return false;
  for (int f = 0; f < p.nf; ++f)
    if ((p.field[f].word >> 2) != ch) return false;
  return true;
}
template <int M, int OC>
static void *p1_cnt_nf2(const Plan &p, int kk) {
  if (kk == KK_GLOBAL) return p.nf <= 1 ? (void *)k_pane_cnt<M, 1, KK_GLOBAL, OC> : (void *)k_pane_cnt<M, 2, KK_GLOBAL, OC>;
  return p.nf <= 1 ? (void *)k_pane_cnt<M, 1, KK_RADIX, OC> : (void *)k_pane_cnt<M, 2, KK_RADIX, OC>;
}
// τ in words 0-1, one value in word 2, the key (if any) in word 3 of one chunk
static bool syn_layout(const Plan &p, int kk) {
  return one_chunk(p) && p.tuple_bytes == 32 && (p.ts_word & 3) == 0 && p.nf == 1 && (p.field[0].word & 3) == 2 &&
         (kk == KK_GLOBAL || (p.key[0].word & 3) == 3) && !std::getenv("SABER_NO_FIXED_LAYOUT");
}
// FX tables: atomic (DIRECT / SHARED) tables of one f32 sum column, limbs safe for g < 2^16
static bool fx_ok(const Plan &p) {
  return (p.local_mode == TM_DIRECT || p.local_mode == TM_SHARED) && p.nf == 1 && p.field[0].kind == FK_SUM_F &&
         p.field[0].type == T_F32 && p.g < 65536 && !std::getenv("SABER_NO_FX");
}
template <int M>
static void *p1_cnt_nf(const Plan &p, int kk) {
  if (syn_layout(p, kk) && M != TM_LANE && fx_ok(p))
    return kk == KK_GLOBAL ? (void *)k_pane_cnt<M, 1, KK_GLOBAL, 2, true> : (void *)k_pane_cnt<M, 1, KK_RADIX, 2, true>;
  if (syn_layout(p, kk))
    return kk == KK_GLOBAL ? (void *)k_pane_cnt<M, 1, KK_GLOBAL, 2> : (void *)k_pane_cnt<M, 1, KK_RADIX, 2>;
  return one_chunk(p) ? p1_cnt_nf2<M, 1>(p, kk) : p1_cnt_nf2<M, 0>(p, kk);
}
// count-window fast kernel, or nullptr when the plan needs the generic one
static void *p1_cnt(const Plan &p) {
  if (p.win_kind != WK_COUNT || !p.fast_path || p.npred != 0 || p.g_magic == 0) return nullptr;
  int kk;
  if (p.key_mode == KM_GLOBAL) kk = KK_GLOBAL;
  else if (p.key_mode != KM_HASH && p.key_pack == KP_RADIX && p.nkeys == 1) kk = KK_RADIX;
  else return nullptr;
  switch (p.local_mode) {
    case TM_LANE: return p1_cnt_nf<TM_LANE>(p, kk);
    case TM_DIRECT: return p1_cnt_nf<TM_DIRECT>(p, kk);
    case TM_SHARED: return p1_cnt_nf<TM_SHARED>(p, kk);
    default: return nullptr;
  }
}
bool p1_is_cnt(const Plan &p) { return p1_cnt(p) != nullptr; }
// the count kernel p1_cnt picks is an FX instance (flush_fx: side table, plain
// stores into the panes a CTA owns)
static bool p1_cnt_fx(const Plan &p) {
  if (!p1_cnt(p) || (p.local_mode != TM_DIRECT && p.local_mode != TM_SHARED)) return false;
  const int kk = p.key_mode == KM_GLOBAL ? KK_GLOBAL : KK_RADIX;
  return syn_layout(p, kk) && fx_ok(p);
}
bool p1_cnt_fx_plan(const Plan &p) { return p1_cnt_fx(p); }
void *p1_kernel(const Plan &p) {
  void *k = p1_cnt(p);
  return k ? k : p1_generic(p);
}
cudaError_t p1_set_attributes(const Plan &p) {
  cudaError_t e = cudaFuncSetAttribute(p1_generic(p), cudaFuncAttributeMaxDynamicSharedMemorySize, p1_smem_bytes(p));
  if (e == cudaSuccess && p1_cnt(p))
    e = cudaFuncSetAttribute(p1_cnt(p), cudaFuncAttributeMaxDynamicSharedMemorySize, p1_smem_bytes(p));
  return e;
}

int p1_blocks_per_sm(const Plan &p) {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, p1_kernel(p), kP1Threads, p1_smem_bytes(p));
  return b > 0 ? b : 1;
}

// the scan kernel and grid of a task of n tuples; k_pane_cnt initialises the pane
// slots that lie wholly inside one CTA's tuples itself (*per = its tuples per CTA,
// 0 for the other kernels)
static void *p1_choose(const Plan &p, int64_t n, int grid, int *g, int64_t *per) {
  const int64_t stage_t = kStageBytes / p.tuple_bytes;
  int64_t need = (n + stage_t - 1) / stage_t;     // at least one stage per CTA
  *g = (int)(need < grid ? need : grid);
  if (*g < 1) *g = 1;
  // the fast count kernel keeps CTA-relative positions and panes in 32 bits
  void *k = p1_cnt(p);
  if (!k || (n / *g + stage_t + p.g) >= (1ll << 30)) k = nullptr;
  // the fixed Syn layout reads 32-B tuples (k_pane_cnt: tb = 32, ST = kStageBytes / 32)
  const int64_t st_t = kStageBytes / p.tuple_bytes;
  *per = k && p1_cnt_fx(p) && !p.overlap && !std::getenv("SABER_NO_SELFZERO")
             ? ((n + *g - 1) / *g + st_t - 1) / st_t * st_t : 0;
  return k ? k : p1_generic(p);
}
int64_t p1_selfzero_per(const Plan &p, int64_t n, int grid, int *g) {
  int64_t per;
  p1_choose(p, n, grid, g, &per);
  return n > 0 ? per : 0;
}
cudaError_t launch_pane_agg(const Plan &p, const QueryDev &q, const void *tuples, int64_t n, int grid,
                            cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  int g;
  int64_t per;
  void *k = p1_choose(p, n, grid, &g, &per);
  int sz = per > 0;
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&tuples, (void *)&n, (void *)&q.table, (void *)&q.pane_ts,
                  (void *)&sz};
  return cudaLaunchKernel(k, dim3(g), dim3(kP1Threads), args, (size_t)p1_smem_bytes(p), st);
}

}  // namespace sb
