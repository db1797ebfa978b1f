// common.cuh -- device helpers shared by the kernel translation units.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "device_util.cuh"
#include "plan.h"

// loops over the query's fields / key columns with compile-time bounds, so small
// per-thread arrays indexed by the loop variable stay in registers
#define FOR_F(f) _Pragma("unroll") for (int f = 0; f < kMaxField; ++f) if (f < p.nf)
#define FOR_K(i) _Pragma("unroll") for (int i = 0; i < kMaxKey; ++i) if (i < p.nkeys)

namespace sb {

struct WinHdr { int64_t window_id, ts, row_offset; int32_t nrows, flags; };

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

// field access straight from the shared-memory tuple (runtime byte offsets)
__device__ __forceinline__ int64_t s_int(const unsigned char *t, int word, int type) {
  return type == T_I32 ? (int64_t) * (const int32_t *)(t + 4 * word) : *(const int64_t *)(t + 4 * word);
}
__device__ __forceinline__ double s_flt(const unsigned char *t, int word, int type) {
  return type == T_F32 ? (double)*(const float *)(t + 4 * word) : *(const double *)(t + 4 * word);
}

__device__ __forceinline__ bool s_preds(const Plan &p, const unsigned char *t) {
  bool ok = true;
  for (int i = 0; i < p.npred; ++i) {
    const Pred &pr = p.pred[i];
    if (pr.type == T_F32 || pr.type == T_F64) ok &= cmp_op(s_flt(t, pr.word, pr.type), pr.op, pr.fval);
    else ok &= cmp_op(s_int(t, pr.word, pr.type), pr.op, pr.ival);
  }
  return ok;
}

__device__ __forceinline__ int64_t cnt_off(const Plan &p) { return p.key_mode == KM_HASH ? p.C : 0; }
// pane presence bitmaps (Plan::pane_bm): [R][8] u32 right after the ring's R slots
__device__ __forceinline__ uint32_t *pane_bm_words(const Plan &p, uint64_t *table) {
  return (uint32_t *)(table + p.R * p.slot_words);
}
__device__ __forceinline__ const uint32_t *pane_bm_words(const Plan &p, const uint64_t *table) {
  return (const uint32_t *)(table + p.R * p.slot_words);
}
__device__ __forceinline__ int64_t fld_off(const Plan &p, int f) { return cnt_off(p) + (int64_t)(1 + f) * p.C; }

// --------------------------------------------------------------------------
// task prologue (one warp)
__device__ __forceinline__ int64_t tau_at(const Plan &p, const unsigned char *t, int64_t i) {
  return *(const int64_t *)(t + i * p.tuple_bytes + 4 * p.ts_word);
}

// lower_bound over the concatenation [a (na tuples) ++ b (nb tuples)] of τ < key (warp-cooperative)
static __device__ int64_t warp_lower_bound(const Plan &p, const unsigned char *a, int64_t na,
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


// Compensated fp64 accumulation for window states that slide by adding entering
// and subtracting expiring values (bucket / hash / slab plans).  Plain fp64
// add/subtract leaves an error proportional to everything the state ever held
// (a key that once summed 1e12 and now sums 1e-3 would be off by ~1e-4); with
// Knuth's error-free TwoSum the rounding error of every update is kept in a
// second word, so the state's error is ~2^-106 of its history.
// No multiplications: nothing for FMA contraction to change.
__device__ __forceinline__ double two_sum(double a, double b, double &e) {
  const double s = a + b;
  const double bb = s - a;
  e = (a - (s - bb)) + (b - bb);
  return s;
}
// shared-memory version for concurrent updates: CAS on the sum word, the
// (exact) rounding error of the successful update goes to the compensation word
__device__ __forceinline__ void dd_atomic_add(double *hi, double *lo, double x) {
  unsigned long long *a = (unsigned long long *)hi;
  unsigned long long old = *(volatile unsigned long long *)a, assumed;
  double s, e;
  do {
    assumed = old;
    s = two_sum(__longlong_as_double((long long)assumed), x, e);
    old = atomicCAS(a, assumed, (unsigned long long)__double_as_longlong(s));
  } while (old != assumed);
  if (e != 0.0) atomicAdd(lo, e);
}

// decoupled look-back status words: epoch (24 bits) | flag (2: 1 aggregate, 2 inclusive) | value (38 bits)
__device__ __forceinline__ uint64_t lb_ld(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}
__device__ __forceinline__ void lb_st(uint64_t *p, uint64_t v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v));
}
__device__ __forceinline__ uint64_t lb_pack(uint64_t epoch, uint64_t flag, uint64_t v) {
  return ((epoch & 0xffffffull) << 40) | (flag << 38) | (v & ((1ull << 38) - 1));
}

// Decoupled look-back for tile t (called by all 32 lanes of one warp): publishes
// the tile's aggregate, then inspects 32 predecessors per step (lane i reads
// tile t-1-i-32·k); the lanes up to the nearest inclusive prefix must all be
// published before their aggregates are summed.  Returns the exclusive prefix
// (to every lane) and publishes the inclusive one.  A one-thread walk costs one
// dependent L2 round trip per predecessor: with hundreds of tiles in flight the
// chain of a wave's last tile was tens of microseconds.
// base0: the prefix before tile 0 (rows earlier rounds of the task already wrote).
// published = true: the caller already published tile t's aggregate (or, for
// t == 0, its inclusive prefix) -- the look-back only resolves.
__device__ __forceinline__ int64_t lookback_warp(uint64_t *status, int64_t t, uint64_t epoch, uint64_t total,
                                                 int64_t base0 = 0, bool published = false) {
  const int lane = threadIdx.x & 31;
  const uint64_t ep = epoch & 0xffffffull;
  const uint64_t vmask = (1ull << 38) - 1;
  if (t == 0) {
    if (lane == 0 && !published) lb_st(&status[0], lb_pack(epoch, 2, (uint64_t)base0 + total));
    return base0;
  }
  if (lane == 0 && !published) lb_st(&status[t], lb_pack(epoch, 1, total));
  int64_t excl = 0;
  for (int64_t i = t - 1;;) {
    const int64_t idx = i - lane;
    uint64_t sv = idx >= 0 ? lb_ld(&status[idx]) : lb_pack(epoch, 2, 0);   // before tile 0: inclusive 0
    const uint64_t flag = (sv >> 38) & 3ull;
    const bool ok = (sv >> 40) == ep && flag != 0;
    const unsigned incl = __ballot_sync(kFull, ok && flag == 2);
    const unsigned bad = __ballot_sync(kFull, !ok);
    const unsigned need = incl ? (((incl & (0u - incl)) << 1) - 1u) : kFull;   // lanes 0 .. first inclusive
    if (bad & need) continue;                                                // not all published yet
    uint64_t v = ((need >> lane) & 1u) ? (sv & vmask) : 0ull;
#pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(kFull, v, o);
    excl += (int64_t)v;
    if (incl) break;
    i -= 32;
  }
  if (lane == 0) lb_st(&status[t], lb_pack(epoch, 2, (uint64_t)excl + total));
  return excl;
}

// --------------------------------------------------------------------------
// window assembly helpers
struct AggVal { uint64_t bits; bool isf; };

// fv[i] for a runtime i without dynamic register indexing (no local-memory spill)
__device__ __forceinline__ uint64_t pick_field(const uint64_t *fv, int i) {
  uint64_t r = fv[0];
#pragma unroll
  for (int k = 1; k < kMaxField; ++k) r = (i == k) ? fv[k] : r;
  return r;
}

__device__ __forceinline__ AggVal finalize(const Plan &p, int a, int64_t cnt, const uint64_t *fv) {
  const AggOut &o = p.agg[a];
  AggVal r;
  r.isf = o.out_float;
  const uint64_t x = o.field >= 0 ? pick_field(fv, o.field) : 0;
  switch (o.fn) {
    case AG_COUNT: r.bits = (uint64_t)cnt; break;
    case AG_SUM: r.bits = x; break;
    case AG_AVG: {
      double sum = (p.field[o.field].kind == FK_SUM_F) ? __longlong_as_double((long long)x) : (double)(int64_t)x;
      r.bits = (uint64_t)__double_as_longlong(sum / (double)cnt);   // reading A11
      break;
    }
    default: {
      uint64_t u = x;
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
  FOR_K(i) {
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
    if (p.nkeys == 1) {
      kv[0] = (int64_t)k;                                   // single key: the packed key is the value
    } else if (p.G <= 0xffffffffll) {                         // 32-bit divisions
      FOR_K(i)
        kv[i] = (int64_t)(((uint32_t)k / (uint32_t)p.key[i].stride) % (uint32_t)p.key[i].domain);
    } else {
      FOR_K(i) kv[i] = (int64_t)((k / (uint64_t)p.key[i].stride) % (uint64_t)p.key[i].domain);
    }
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


}  // namespace sb
