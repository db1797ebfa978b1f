// k_window.cu -- window assembly: the batch operator f_b (§3)
// and the result stage's window construction (§4.3).
//
// A window j covers panes [j·L, j·L+K).  Windows closed by a task are built
// from the device pane ring, which still holds the fragments (pane partials)
// of earlier tasks, so windows spanning tasks are assembled in task order by
// the task that closes them.
//
// DENSE / GLOBAL keys: van Herk / Gil-Werman block decomposition over panes.
// Panes are grouped in blocks of K aligned to multiples of K; per block a
// prefix array P[q] = ⊕ partial[bK..q] and a suffix array S[q] = ⊕ partial[q..bK+K-1]
// are built (k_vh_build); then every (window, key) is independent:
//   window(a) = S[a]                 if a ≡ 0 (mod K)
//             = S[a] ⊕ P[a+K-1]      otherwise
// one combine per window and key for count/sum (exact for integers, no
// floating-point cancellation) and for min/max alike.
//
// HASH keys: per-pane tables place a key at different slots, so windows slide
// over key slabs with a shared-memory state hash (add entering panes, subtract
// expired panes; min/max recomputed).
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "launch_internal.h"

namespace sb {

// pane-slot word offsets in the van Herk arrays (no key section)
__device__ __forceinline__ int64_t vh_off(const Plan &p, int f) { return (int64_t)(1 + f) * p.C; }

__device__ __forceinline__ uint64_t combine_cnt_or_field(const Plan &p, int f, uint64_t a, uint64_t b) {
  return f < 0 ? a + b : field_combine(p.field[f].kind, a, b);
}

// one thread per (block of K panes, table word, direction): the DENSE/GLOBAL pane
// slot is [cnt C][f0 C][f1 C].., identical in the table and in the van Herk arrays
__global__ void __launch_bounds__(256)
k_vh_build(const Plan p, const State *__restrict__ st, const uint64_t *__restrict__ table,
           uint64_t *__restrict__ pre, uint64_t *__restrict__ suf) {
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  const int64_t lo = J0 * p.L, hi = (J1 - 1) * p.L + p.K - 1;
  const int64_t b0 = lo / p.K, b1 = hi / p.K;
  const int64_t words = p.slot_words;                 // C * (1 + nf)
  const int64_t items = (b1 - b0 + 1) * words * 2;
  const int64_t Rm = p.R - 1;
  for (int64_t it = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; it < items; it += (int64_t)gridDim.x * blockDim.x) {
    const int64_t w = it % words;
    const int64_t rest = it / words;
    const bool prefix = rest & 1;
    const int64_t b = b0 + (rest >> 1);
    const int f = (int)(w / p.C) - 1;                   // -1: count
    const int kind = f < 0 ? -1 : p.field[f].kind;
    const int64_t bs = b * p.K, be = (bs + p.K - 1 < hi) ? bs + p.K - 1 : hi;
    uint64_t acc = kind < 0 ? 0ull : field_identity(kind);
    // eight loads in flight per thread, then the dependent combines
    constexpr int U = 8;
    if (prefix) {
      if (bs < lo) continue;                             // prefixes are only read for blocks starting >= lo
      for (int64_t q0 = bs; q0 <= be; q0 += U) {
        uint64_t v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = q0 + u <= be ? table[((q0 + u) & Rm) * words + w] : 0ull;
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (q0 + u > be) break;
          acc = kind < 0 ? acc + v[u] : field_combine(kind, acc, v[u]);
          pre[((q0 + u) & Rm) * words + w] = acc;
        }
      }
    } else {
      const int64_t qlo = bs > lo ? bs : lo;
      for (int64_t q0 = be; q0 >= qlo; q0 -= U) {
        uint64_t v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = q0 - u >= qlo ? table[((q0 - u) & Rm) * words + w] : 0ull;
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (q0 - u < qlo) break;
          acc = kind < 0 ? acc + v[u] : field_combine(kind, acc, v[u]);
          suf[((q0 - u) & Rm) * words + w] = acc;
        }
      }
    }
  }
}

__device__ __forceinline__ uint64_t shfl_up64_n(uint64_t v, int o) {
  const uint32_t lo = __shfl_up_sync(kFull, (uint32_t)v, o), hi = __shfl_up_sync(kFull, (uint32_t)(v >> 32), o);
  return ((uint64_t)hi << 32) | lo;
}

// Long windows (K > 64 panes): one CTA per (block, table word, direction); the
// block's panes are split into 256 chunks, each thread scans its chunk, the CTA
// scans the chunk totals, and each thread re-walks its chunk adding its offset.
__global__ void __launch_bounds__(256)
k_vh_build_long(const Plan p, const State *__restrict__ st, const uint64_t *__restrict__ table,
                uint64_t *__restrict__ pre, uint64_t *__restrict__ suf) {
  __shared__ uint64_t s_tot[256];
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  const int64_t lo = J0 * p.L, hi = (J1 - 1) * p.L + p.K - 1;
  const int64_t b0 = lo / p.K, b1 = hi / p.K;
  const int64_t words = p.slot_words;
  const int64_t items = (b1 - b0 + 1) * words * 2;
  const int64_t Rm = p.R - 1;
  const int tid = threadIdx.x;
  for (int64_t it = blockIdx.x; it < items; it += gridDim.x) {
    const int64_t w = it % words;
    const int64_t rest = it / words;
    const bool prefix = rest & 1;
    const int64_t b = b0 + (rest >> 1);
    const int f = (int)(w / p.C) - 1;
    const int kind = f < 0 ? -1 : p.field[f].kind;
    const int64_t bs = b * p.K, be = (bs + p.K - 1 < hi) ? bs + p.K - 1 : hi;
    const int64_t qa = prefix ? bs : (bs > lo ? bs : lo);      // scanned pane range [qa, be]
    if (prefix && bs < lo) continue;                             // uniform across the CTA
    const uint64_t id = kind < 0 ? 0ull : field_identity(kind);
    const int64_t len = be - qa + 1;
    const int64_t ch = (len + 255) / 256;
    // chunk t covers positions [t*ch, (t+1)*ch) of the scan order
    const int64_t c0 = tid * ch, c1 = (c0 + ch < len) ? c0 + ch : len;
    auto pane_of = [&](int64_t k) { return prefix ? qa + k : be - k; };
    uint64_t acc = id;
    for (int64_t k = c0; k < c1; ++k) {
      const uint64_t v = table[(pane_of(k) & Rm) * words + w];
      acc = kind < 0 ? acc + v : field_combine(kind, acc, v);
    }
    s_tot[tid] = acc;
    __syncthreads();
    if (tid < 32) {                                   // exclusive scan of 256 chunk totals (warp 0)
      uint64_t v[8];
      uint64_t lt = id;
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        v[k] = s_tot[tid * 8 + k];
        lt = kind < 0 ? lt + v[k] : field_combine(kind, lt, v[k]);
      }
      uint64_t x = lt;                                // inclusive warp scan of lane totals
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint64_t y = shfl_up64_n(x, o);
        if (tid >= o) x = kind < 0 ? x + y : field_combine(kind, y, x);
      }
      uint64_t run = shfl_up64_n(x, 1);
      if (tid == 0) run = id;
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        s_tot[tid * 8 + k] = run;
        run = kind < 0 ? run + v[k] : field_combine(kind, run, v[k]);
      }
    }
    __syncthreads();
    acc = s_tot[tid];
    uint64_t *dst = prefix ? pre : suf;
    for (int64_t k = c0; k < c1; ++k) {
      const int64_t r = (pane_of(k) & Rm) * words + w;
      const uint64_t v = table[r];
      acc = kind < 0 ? acc + v : field_combine(kind, acc, v);
      dst[r] = acc;
    }
    __syncthreads();
  }
}

// Long windows, many table words: one warp per (block, word, direction), lane =
// chunk of the block's panes; no shared memory, no barriers.
__global__ void __launch_bounds__(256)
k_vh_build_warp(const Plan p, const State *__restrict__ st, const uint64_t *__restrict__ table,
                uint64_t *__restrict__ pre, uint64_t *__restrict__ suf) {
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  const int lane = threadIdx.x & 31;
  const int64_t lo = J0 * p.L, hi = (J1 - 1) * p.L + p.K - 1;
  const int64_t b0 = lo / p.K, b1 = hi / p.K;
  const int64_t words = p.slot_words;
  const int64_t items = (b1 - b0 + 1) * words * 2;
  const int64_t Rm = p.R - 1;
  const int64_t gw = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t it = gw; it < items; it += nwarps) {
    const int64_t w = it % words;                        // consecutive warps: consecutive words
    const int64_t rest = it / words;
    const bool prefix = rest & 1;
    const int64_t b = b0 + (rest >> 1);
    const int f = (int)(w / p.C) - 1;
    const int kind = f < 0 ? -1 : p.field[f].kind;
    const int64_t bs = b * p.K, be = (bs + p.K - 1 < hi) ? bs + p.K - 1 : hi;
    if (prefix && bs < lo) continue;                     // warp-uniform
    const int64_t qa = prefix ? bs : (bs > lo ? bs : lo);
    const uint64_t id = kind < 0 ? 0ull : field_identity(kind);
    const int64_t len = be - qa + 1;
    const int64_t ch = (len + 31) / 32;
    const int64_t c0 = lane * ch, c1 = (c0 + ch < len) ? c0 + ch : len;
    auto pane_of = [&](int64_t k) { return prefix ? qa + k : be - k; };
    uint64_t acc = id;
#pragma unroll 4
    for (int64_t k = c0; k < c1; ++k) {
      const uint64_t v = table[(pane_of(k) & Rm) * words + w];
      acc = kind < 0 ? acc + v : field_combine(kind, acc, v);
    }
    uint64_t x = acc;                                    // inclusive scan of chunk totals
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint64_t y = shfl_up64_n(x, o);
      if (lane >= o) x = kind < 0 ? x + y : field_combine(kind, y, x);
    }
    uint64_t run = shfl_up64_n(x, 1);
    if (lane == 0) run = id;
    uint64_t *dst = prefix ? pre : suf;
#pragma unroll 4
    for (int64_t k = c0; k < c1; ++k) {
      const int64_t r = (pane_of(k) & Rm) * words + w;
      run = kind < 0 ? run + table[r] : field_combine(kind, run, table[r]);
      dst[r] = run;
    }
  }
}

// Long windows, many table words: one CTA per (block, direction, group of 32
// consecutive words).  Lane = word (each warp load is 256 contiguous bytes of a
// pane slot), warp = one of 8 chunks of the block's panes: chunk totals, a scan
// of the 8 totals per word in shared memory, then each warp re-walks its chunk.
__global__ void __launch_bounds__(256)
k_vh_build_cta(const Plan p, const State *__restrict__ st, const uint64_t *__restrict__ table,
               uint64_t *__restrict__ pre, uint64_t *__restrict__ suf) {
  __shared__ uint64_t s_tot[8][32];
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t lo = J0 * p.L, hi = (J1 - 1) * p.L + p.K - 1;
  const int64_t b0 = lo / p.K, b1 = hi / p.K;
  const int64_t words = p.slot_words, groups = (words + 31) / 32;
  const int64_t items = (b1 - b0 + 1) * 2 * groups;
  const int64_t Rm = p.R - 1;
  for (int64_t it = blockIdx.x; it < items; it += gridDim.x) {
    const int64_t grp = it % groups, rest = it / groups;
    const bool prefix = rest & 1;
    const int64_t b = b0 + (rest >> 1);
    const int64_t w = grp * 32 + lane;
    const bool live = w < words;
    const int f = live ? (int)(w / p.C) - 1 : -1;
    const int kind = f < 0 ? -1 : p.field[f].kind;
    const uint64_t id = kind < 0 ? 0ull : field_identity(kind);
    const int64_t bs = b * p.K, be = (bs + p.K - 1 < hi) ? bs + p.K - 1 : hi;
    if (prefix && bs < lo) continue;                                 // uniform across the CTA
    const int64_t qa = prefix ? bs : (bs > lo ? bs : lo);
    const int64_t len = be - qa + 1;
    const int64_t ch = (len + 7) / 8;
    const int64_t c0 = warp * ch, c1 = (c0 + ch < len) ? c0 + ch : len;
    auto pane_of = [&](int64_t k) { return prefix ? qa + k : be - k; };
    auto ld = [&](int64_t k) { return live ? table[(pane_of(k) & Rm) * words + w] : 0ull; };
    constexpr int U = 8;
    uint64_t acc = id;
    for (int64_t k0 = c0; k0 < c1; k0 += U) {
      uint64_t v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = k0 + u < c1 ? ld(k0 + u) : id;
#pragma unroll
      for (int u = 0; u < U; ++u) acc = kind < 0 ? acc + v[u] : field_combine(kind, acc, v[u]);
    }
    s_tot[warp][lane] = acc;
    __syncthreads();
    uint64_t run = id;                                                // combine of the chunks before this warp's
    for (int c = 0; c < warp; ++c) run = kind < 0 ? run + s_tot[c][lane] : field_combine(kind, run, s_tot[c][lane]);
    uint64_t *dst = prefix ? pre : suf;
    for (int64_t k0 = c0; k0 < c1; k0 += U) {
      uint64_t v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = k0 + u < c1 ? ld(k0 + u) : id;
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (k0 + u >= c1) break;
        run = kind < 0 ? run + v[u] : field_combine(kind, run, v[u]);
        if (live) dst[(pane_of(k0 + u) & Rm) * words + w] = run;
      }
    }
    __syncthreads();
  }
}

// Long windows, many table words, built only where the task's windows read them
// and in one pass: items are (block, direction, group of 32 consecutive words),
// lane = word.  Suffixes S[a] are needed for the window starts a in [a0, a1]
// (walk each start block backward from its end down to max(block start, a0));
// prefixes P[e] for the ends e = a+K-1 in [e0, e1] of non-aligned windows, in
// blocks starting after a0, and only from vh_pre_hi on: the previous task built
// the prefixes below it, so a block's walk continues from P[start-1].  A CTA walks
// its range in tiles of 8 warps × kVhU panes: per-lane register scans, warp
// totals through shared memory, a running carry; the next tile's loads are
// issued before the current tile is combined.  One table read and one write per
// (pane, word) and direction (k_vh_build_cta read every word twice, for both
// directions over the whole pane range of the task).
constexpr int kVhU = 8;

// combine with the field kind fixed at compile time (OP >= 0) or per lane (OP < 0)
template <int OP>
__device__ __forceinline__ uint64_t vh_comb(int op, uint64_t a, uint64_t b) {
  if (OP == FK_SUM_I) return a + b;
  if (OP == FK_SUM_F) return (uint64_t)__double_as_longlong(__longlong_as_double((long long)a) + __longlong_as_double((long long)b));
  if (OP == FK_MIN) return a < b ? a : b;
  if (OP == FK_MAX) return a < b ? b : a;
  return field_combine_sel(op, a, b);
}

// one (block, direction, 32-word group) item: walk `len` panes from `start`
// (forward for prefixes, backward for suffixes) in tiles of 8 warps × kVhU panes
template <int OP>
__device__ __forceinline__ void vh_tile_walk(uint64_t (*s_tot)[32], const uint64_t *__restrict__ table,
                                             uint64_t *__restrict__ dst, int64_t start, int64_t len, bool prefix,
                                             int64_t Rm, int64_t words, int64_t w, bool live, int op,
                                             uint64_t id, uint64_t carry) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  auto slot = [&](int64_t k) { return ((prefix ? start + k : start - k) & Rm) * words + w; };
  uint64_t v[kVhU], vn[kVhU];
  auto load = [&](int64_t k0, uint64_t (&x)[kVhU]) {
#pragma unroll
    for (int u = 0; u < kVhU; ++u) {
      const int64_t k = k0 + warp * kVhU + u;
      x[u] = (live && k < len) ? table[slot(k)] : id;
    }
  };
  load(0, vn);
  for (int64_t k0 = 0; k0 < len; k0 += 8 * kVhU) {
#pragma unroll
    for (int u = 0; u < kVhU; ++u) v[u] = vn[u];
    if (k0 + 8 * kVhU < len) load(k0 + 8 * kVhU, vn);
    uint64_t acc = id;
#pragma unroll
    for (int u = 0; u < kVhU; ++u) {
      acc = vh_comb<OP>(op, acc, v[u]);
      v[u] = acc;
    }
    s_tot[warp][lane] = acc;
    __syncthreads();
    uint64_t run = carry, all = carry;
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const uint64_t x = s_tot[c][lane];
      if (c < warp) run = vh_comb<OP>(op, run, x);
      all = vh_comb<OP>(op, all, x);
    }
    carry = all;
    if (live) {
#pragma unroll
      for (int u = 0; u < kVhU; ++u) {
        const int64_t k = k0 + warp * kVhU + u;
        if (k < len) dst[slot(k)] = vh_comb<OP>(op, run, v[u]);
      }
    }
    __syncthreads();
  }
}

__global__ void __launch_bounds__(256, 3)
k_vh_build_tile(const Plan p, const State *__restrict__ st, const uint64_t *__restrict__ table,
                uint64_t *__restrict__ pre, uint64_t *__restrict__ suf) {
  __shared__ uint64_t s_tot[8][32];
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  const int lane = threadIdx.x & 31;
  const int64_t K = p.K, Rm = p.R - 1, words = p.slot_words, groups = (words + 31) / 32;
  const int64_t a0 = J0 * p.L, a1 = (J1 - 1) * p.L, e1 = a1 + K - 1;
  const int64_t sb0 = a0 / K, nS = a1 / K - sb0 + 1;             // suffix blocks
  const int64_t pb0 = a0 / K + 1, nP = e1 / K >= pb0 ? e1 / K - pb0 + 1 : 0;   // prefix blocks (start > a0)
  const int64_t pdone = st->vh_pre_hi;
  const int64_t items = (nS + nP) * groups;
  auto op_of = [&](int64_t w) {                                   // count words add as integers
    const int f = (int)(w / p.C) - 1;
    return f < 0 ? (int)FK_SUM_I : p.field[f].kind;
  };
  for (int64_t it = blockIdx.x; it < items; it += gridDim.x) {
    const int64_t grp = it % groups, seg = it / groups;
    const bool prefix = seg >= nS;
    const int64_t b = prefix ? pb0 + (seg - nS) : sb0 + seg;
    const int64_t bs = b * K, be = bs + K - 1;
    int64_t start, len;                                           // walk: pane(k) = start ± k
    if (prefix) {
      start = bs > pdone ? bs : pdone;
      const int64_t end = be < e1 ? be : e1;
      len = end - start + 1;
    } else {
      start = be;
      len = be - (bs > a0 ? bs : a0) + 1;
    }
    if (len <= 0) continue;                                       // uniform across the CTA
    const int64_t w = grp * 32 + lane;
    const bool live = w < words;
    const int op = live ? op_of(w) : FK_SUM_I;
    const uint64_t id = field_identity(op);
    uint64_t carry = id;
    if (prefix && start > bs && live) carry = pre[((start - 1) & Rm) * words + w];
    uint64_t *dst = prefix ? pre : suf;
    // the group's 32 words usually lie in one section (count or one field): the
    // combine is then fixed for the whole walk
    const int64_t wl = grp * 32, wh = (wl + 31 < words ? wl + 31 : words - 1);
    const int uop = op_of(wl) == op_of(wh) ? op_of(wl) : -1;
    switch (uop) {
      case FK_SUM_I: vh_tile_walk<FK_SUM_I>(s_tot, table, dst, start, len, prefix, Rm, words, w, live, op, id, carry); break;
      case FK_SUM_F: vh_tile_walk<FK_SUM_F>(s_tot, table, dst, start, len, prefix, Rm, words, w, live, op, id, carry); break;
      case FK_MIN: vh_tile_walk<FK_MIN>(s_tot, table, dst, start, len, prefix, Rm, words, w, live, op, id, carry); break;
      case FK_MAX: vh_tile_walk<FK_MAX>(s_tot, table, dst, start, len, prefix, Rm, words, w, live, op, id, carry); break;
      default: vh_tile_walk<-1>(s_tot, table, dst, start, len, prefix, Rm, words, w, live, op, id, carry);
    }
  }
}

// ---------------------------------------------------------------------------
// Single pass over the windows closed by a task (DENSE/GLOBAL): CTAs take window
// chunks in ticket order, count the rows of every (window, slab) item, obtain
// the chunk's output offset by decoupled look-back over earlier chunks, write
// the window headers and then the rows.  Replaces count pass + scan + emit pass.
constexpr int kFusedMaxItems = 256;

template <int GS>
__global__ void __launch_bounds__(256)
k_win_fused(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ pre, const uint64_t *__restrict__ suf,
            const int64_t *__restrict__ pane_ts, WinHdr *__restrict__ hdr, unsigned char *__restrict__ rows,
            uint64_t *__restrict__ status, int *__restrict__ ticket, int WC) {
  hdr += st->hdr_base;                         // windows earlier rounds of the task wrote
  constexpr int gpb = 256 / GS;
  __shared__ int s_cnt[kFusedMaxItems];
  __shared__ int s_off[kFusedMaxItems];
  __shared__ int s_scan[40];
  __shared__ int s_total;
  __shared__ int64_t s_base;
  __shared__ int s_t;
  const int grp = threadIdx.x / GS, gt = threadIdx.x % GS, lane = threadIdx.x & 31;
  const int SB = p.SB, S = p.S;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const uint64_t epoch = (uint64_t)st->tile_epoch;
  const int64_t nchunks = (nw + WC - 1) / WC;
  for (;;) {
    if (threadIdx.x == 0) s_t = atomicAdd(ticket, 1);
    __syncthreads();
    const int64_t t = s_t;
    if (t >= nchunks) break;
    const int64_t ja = J0 + t * WC;
    const int nwc = (int)((J1 - ja) < WC ? (J1 - ja) : WC);
    const int nitems = nwc * S;
    // pass 1: rows per (window, slab) item
    for (int it0 = 0; it0 < nitems; it0 += gpb) {
      const int it = it0 + grp;
      int my = 0;
      if (it < nitems) {
        const int64_t j = ja + it / S;
        const int slab = it % S;
        const int64_t slot0 = (int64_t)slab * SB;
        const int nslot = (int)((p.C - slot0) < SB ? (p.C - slot0) : SB);
        const int64_t a = j * p.L;
        const bool aligned = (a % p.K) == 0;
        const uint64_t *sa = suf + (a & (p.R - 1)) * p.slot_words + slot0;
        const uint64_t *pb = pre + ((a + p.K - 1) & (p.R - 1)) * p.slot_words + slot0;
        for (int s = gt; s < nslot; s += GS) {
          const int64_t c = (int64_t)sa[s] + (aligned ? 0 : (int64_t)pb[s]);
          if (c <= 0) continue;
          if (p.nhave) {
            uint64_t fv[kMaxField];
            FOR_F(f) {
              const uint64_t x = sa[vh_off(p, f) + s];
              fv[f] = aligned ? x : field_combine(p.field[f].kind, x, pb[vh_off(p, f) + s]);
            }
            if (!having_ok(p, c, fv)) continue;
          }
          ++my;
        }
      }
      if (GS == 32) {
#pragma unroll
        for (int o = 16; o; o >>= 1) my += __shfl_xor_sync(kFull, my, o);
        if (gt == 0 && it < nitems) s_cnt[it] = my;
      } else {
        my = __reduce_add_sync(kFull, (unsigned)my);
        __shared__ int s_part[8];
        if (lane == 0) s_part[threadIdx.x >> 5] = my;
        __syncthreads();
        if (threadIdx.x == 0 && it < nitems) {
          int sum = 0;
          for (int w = 0; w < 8; ++w) sum += s_part[w];
          s_cnt[it] = sum;
        }
        __syncthreads();
      }
    }
    __syncthreads();
    // exclusive scan of the chunk's item counts (warp 0)
    if (threadIdx.x < 32) {
      int run = 0;
      for (int b = 0; b < nitems; b += 32) {
        const int v = (b + lane < nitems) ? s_cnt[b + lane] : 0;
        int x = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(kFull, x, o);
          if (lane >= o) x += y;
        }
        if (b + lane < nitems) s_off[b + lane] = run + x - v;
        run += __shfl_sync(kFull, x, 31);
      }
      if (lane == 0) s_total = run;
    }
    __syncthreads();
    if (threadIdx.x < 32) {
      const uint64_t total = (uint64_t)s_total;
      const int64_t excl = lookback_warp(status, t, epoch, total, st->row_base);
      if (threadIdx.x == 0) {
        s_base = excl;
        if (t == nchunks - 1) {
          st->sel_rows = excl + (int64_t)total;
          if (excl + (int64_t)total > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
        }
      }
    }
    __syncthreads();
    const int64_t base = s_base;
    // window headers
    for (int w = threadIdx.x; w < nwc; w += blockDim.x) {
      const int64_t j = ja + w;
      WinHdr h;
      h.window_id = j;
      h.ts = (p.win_kind == WK_TIME) ? p.T0 + j * p.l : pane_ts[(j * p.L) & (p.R - 1)];
      h.row_offset = base + s_off[w * S];
      int nr = 0;
      for (int s = 0; s < S; ++s) nr += s_cnt[w * S + s];
      h.nrows = nr;
      h.flags = 0;
      hdr[j - J0] = h;
    }
    // pass 2: rows
    for (int it0 = 0; it0 < nitems; it0 += gpb) {
      const int it = it0 + grp;
      if (it >= nitems) continue;
      const int64_t j = ja + it / S;
      const int slab = it % S;
      const int64_t slot0 = (int64_t)slab * SB;
      const int nslot = (int)((p.C - slot0) < SB ? (p.C - slot0) : SB);
      const int64_t a = j * p.L;
      const bool aligned = (a % p.K) == 0;
      const uint64_t *sa = suf + (a & (p.R - 1)) * p.slot_words + slot0;
      const uint64_t *pb = pre + ((a + p.K - 1) & (p.R - 1)) * p.slot_words + slot0;
      int64_t r = base + s_off[it];
      auto value = [&](int s, int64_t &c, uint64_t (&fv)[kMaxField]) -> bool {
        c = (int64_t)sa[s] + (aligned ? 0 : (int64_t)pb[s]);
        if (c <= 0) return false;
        FOR_F(f) {
          const uint64_t x = sa[vh_off(p, f) + s];
          fv[f] = aligned ? x : field_combine(p.field[f].kind, x, pb[vh_off(p, f) + s]);
        }
        return !p.nhave || having_ok(p, c, fv);
      };
      if (GS == 32) {
        // warp: rows in slot (key) order, one ballot per 32 slots
        for (int s0 = 0; s0 < nslot; s0 += GS) {
          const int s = s0 + gt;
          int64_t c = 0;
          uint64_t fv[kMaxField];
          const bool present = s < nslot && value(s, c, fv);
          const unsigned bal = __ballot_sync(kFull, present);
          if (present) {
            int64_t kv[kMaxKey];
            decode_key(p, (uint64_t)(slot0 + s), kv);
            write_row(p, rows, r + __popc(bal & ((1u << lane) - 1u)), kv, c, fv);
          }
          r += __popc(bal);
        }
      } else {
        // block: each thread's present slots are contiguous rows (one block scan per item)
        int my = 0;
        for (int s = gt; s < nslot; s += GS) {
          int64_t c;
          uint64_t fv[kMaxField];
          my += value(s, c, fv);
        }
        int tot;
        r += group_excl_scan(my, 256, s_scan, tot);
        for (int s = gt; s < nslot; s += GS) {
          int64_t c;
          uint64_t fv[kMaxField];
          if (!value(s, c, fv)) continue;
          int64_t kv[kMaxKey];
          decode_key(p, (uint64_t)(slot0 + s), kv);
          write_row(p, rows, r++, kv, c, fv);
        }
      }
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------------------
// Few keys (C <= 256, one slab): Cp = C rounded up to a power of two.  Cp <= 32:
// a warp pass holds 32/Cp windows side by side, lane = (window, key slot), so no
// lane idles on a 4-key GROUP BY or a GLOBAL aggregate; Cp > 32: a window takes
// NB = Cp/32 consecutive passes of 32 slots.  Row order is window-major, key
// order inside a window, exactly as k_win_fused.  One ballot per (pass, warp)
// gives every window's row count and every row's offset.
constexpr int kPackU = 16;    // ballot passes per warp per chunk

template <bool F, int NF = kMaxField>
__device__ __forceinline__ bool win_value(const Plan &p, const uint64_t *__restrict__ pre,
                                          const uint64_t *__restrict__ suf, int64_t j, int s, int64_t &c,
                                          uint64_t (&fv)[kMaxField]) {
  const int64_t a = j * p.L;
  const bool aligned = (a % p.K) == 0;
  const uint64_t *sa = suf + (a & (p.R - 1)) * p.slot_words;
  const uint64_t *pb = pre + ((a + p.K - 1) & (p.R - 1)) * p.slot_words;
  c = (int64_t)sa[s] + (aligned ? 0 : (int64_t)pb[s]);
  if (c <= 0) return false;
  if constexpr (F) {
#pragma unroll
    for (int f = 0; f < NF; ++f)
      if (f < p.nf) {
        const uint64_t x = sa[vh_off(p, f) + s];
        fv[f] = aligned ? x : field_combine(p.field[f].kind, x, pb[vh_off(p, f) + s]);
      }
    return !p.nhave || having_ok(p, c, fv);
  }
  return true;
}

template <int NF>
__global__ void __launch_bounds__(256)
k_win_packed(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ pre, const uint64_t *__restrict__ suf,
             const int64_t *__restrict__ pane_ts, WinHdr *__restrict__ hdr, unsigned char *__restrict__ rows,
             uint64_t *__restrict__ status, int *__restrict__ ticket, int cshift) {
  hdr += st->hdr_base;                         // windows earlier rounds of the task wrote
  __shared__ int s_wcnt[8];
  __shared__ int64_t s_base;
  __shared__ int s_t;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int cs = cshift < 5 ? cshift : 5, nbs = cshift - cs;     // NB = 1 << nbs passes per window
  const int WPW = 32 >> cs;                                       // windows per warp pass
  const int wsub = lane >> cs, sl = lane & ((1 << cs) - 1);
  const unsigned seg_lt = (1u << (wsub << cs)) - 1u;              // lanes of earlier windows
  const unsigned seg = cs == 5 ? kFull : (((1u << (1 << cs)) - 1u) << (wsub << cs));
  const unsigned lt = (1u << lane) - 1u;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const uint64_t epoch = (uint64_t)st->tile_epoch;
  const int WW = (kPackU >> nbs) * WPW;                           // windows per warp per chunk
  const int WC = 8 * WW;
  const int64_t nchunks = (nw + WC - 1) / WC;
  auto win_of = [&](int u) { return (int64_t)((u >> nbs) * WPW + wsub); };
  auto slot_of = [&](int u) { return ((u & ((1 << nbs) - 1)) << 5) + sl; };
  for (;;) {
    if (threadIdx.x == 0) s_t = atomicAdd(ticket, 1);
    __syncthreads();
    const int64_t t = s_t;
    if (t >= nchunks) break;
    const int64_t wb = J0 + t * WC + (int64_t)warp * WW;
    unsigned bal[kPackU];
    int wtot = 0;
#pragma unroll
    for (int u = 0; u < kPackU; ++u) {
      const int64_t j = wb + win_of(u);
      const int slot = slot_of(u);
      bool present = false;
      if (j < J1 && slot < p.C) {
        int64_t c;
        uint64_t fv[kMaxField];
        present = p.nhave ? win_value<true, NF>(p, pre, suf, j, slot, c, fv) : win_value<false, NF>(p, pre, suf, j, slot, c, fv);
      }
      bal[u] = __ballot_sync(kFull, present);
      wtot += __popc(bal[u]);
    }
    if (lane == 0) s_wcnt[warp] = wtot;
    __syncthreads();
    if (threadIdx.x < 32) {
      const int v = lane < 8 ? s_wcnt[lane] : 0;       // exclusive offsets of the 8 warps
      int x = v;
#pragma unroll
      for (int o = 1; o < 8; o <<= 1) {
        const int y = __shfl_up_sync(kFull, x, o);
        if (lane >= o) x += y;
      }
      const uint64_t total = (uint64_t)__shfl_sync(kFull, x, 7);
      __syncwarp();
      if (lane < 8) s_wcnt[lane] = x - v;
      const int64_t excl = lookback_warp(status, t, epoch, total, st->row_base);
      if (lane == 0) {
        s_base = excl;
        if (t == nchunks - 1) {
          st->sel_rows = excl + (int64_t)total;
          if (excl + (int64_t)total > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
        }
      }
    }
    __syncthreads();
    int64_t r = s_base + s_wcnt[warp];
    int64_t w_off = 0;
    int w_rows = 0;
#pragma unroll
    for (int u = 0; u < kPackU; ++u) {
      const int64_t j = wb + win_of(u);
      const int slot = slot_of(u);
      const int part = u & ((1 << nbs) - 1);
      if (part == 0) { w_off = r + __popc(bal[u] & seg_lt); w_rows = 0; }
      w_rows += __popc(bal[u] & seg);
      if (j < J1) {
        if (sl == 0 && part == (1 << nbs) - 1) {
          WinHdr h;
          h.window_id = j;
          h.ts = (p.win_kind == WK_TIME) ? p.T0 + j * p.l : pane_ts[(j * p.L) & (p.R - 1)];
          h.row_offset = w_off;
          h.nrows = w_rows;
          h.flags = 0;
          hdr[j - J0] = h;
        }
        if ((bal[u] >> lane) & 1u) {
          int64_t c;
          uint64_t fv[kMaxField];
          win_value<true, NF>(p, pre, suf, j, slot, c, fv);
#pragma unroll
          for (int f = NF; f < kMaxField; ++f) fv[f] = 0;
          int64_t kv[kMaxKey];
          decode_key(p, (uint64_t)slot, kv);
          write_row(p, rows, r + __popc(bal[u] & lt), kv, c, fv);
        }
      }
      r += __popc(bal[u]);
    }
    __syncthreads();
  }
}

// (window, slab) items; a group of GS threads owns the slots of one item
template <bool EMIT>
__global__ void __launch_bounds__(256)
k_win_vh(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ pre, const uint64_t *__restrict__ suf,
         int64_t *__restrict__ counts, unsigned char *__restrict__ rows) {
  __shared__ int scan_sm[40];
  const int GS = p.GS;
  const int gpb = blockDim.x / GS, grp = threadIdx.x / GS, gt = threadIdx.x % GS;
  const int SB = p.SB, S = p.S;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const int64_t nitems = nw * S;
  for (int64_t item0 = (int64_t)blockIdx.x * gpb; item0 < nitems; item0 += (int64_t)gridDim.x * gpb) {
    const int64_t item = item0 + grp;
    const bool live = item < nitems;
    const int64_t j = J0 + (live ? item / S : 0);
    const int slab = live ? (int)(item % S) : 0;
    const int64_t slot0 = (int64_t)slab * SB;
    const int nslot = live ? (int)((p.C - slot0) < SB ? (p.C - slot0) : SB) : 0;
    const int64_t a = j * p.L;
    const bool aligned = (a % p.K) == 0;
    const uint64_t *sa = suf + (a & (p.R - 1)) * p.slot_words + slot0;
    const uint64_t *pb = pre + ((a + p.K - 1) & (p.R - 1)) * p.slot_words + slot0;
    int my = 0;
    for (int s = gt; s < nslot; s += GS) {
      int64_t c = (int64_t)sa[s] + (aligned ? 0 : (int64_t)pb[s]);
      if (c <= 0) continue;
      uint64_t fv[kMaxField];
      FOR_F(f) {
        const uint64_t x = sa[vh_off(p, f) + s];
        fv[f] = aligned ? x : field_combine(p.field[f].kind, x, pb[vh_off(p, f) + s]);
      }
      if (having_ok(p, c, fv)) ++my;
    }
    int total;
    const int excl = group_excl_scan(my, GS, scan_sm, total);
    if (!live) continue;
    const int64_t ci = (j - J0) * S + slab;
    if (!EMIT) {
      if (gt == 0) counts[ci] = total;
      continue;
    }
    int64_t r = counts[ci] + excl;
    for (int s = gt; s < nslot; s += GS) {
      int64_t c = (int64_t)sa[s] + (aligned ? 0 : (int64_t)pb[s]);
      if (c <= 0) continue;
      uint64_t fv[kMaxField];
      FOR_F(f) {
        const uint64_t x = sa[vh_off(p, f) + s];
        fv[f] = aligned ? x : field_combine(p.field[f].kind, x, pb[vh_off(p, f) + s]);
      }
      if (!having_ok(p, c, fv)) continue;
      int64_t kv[kMaxKey];
      decode_key(p, (uint64_t)(slot0 + s), kv);
      write_row(p, rows, r++, kv, c, fv);
    }
  }
}

// HASH: block-wide state hash keyed by the group key; slab = home-slot range
constexpr int kHashMaxChunk = 128;      // windows per item (win_chunk <= 128)
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
  double *sc = (double *)(sf + (size_t)p.nf * ST);     // TwoSum compensation of FK_SUM_F fields
  // occupied state slots of the item, in insertion order: keys are never removed
  // within an item, so windows scan only these instead of all ST slots
  int *occ = (int *)(sc + (size_t)p.nf * ST);
  __shared__ int s_nocc;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const int64_t maxprobe = (int64_t)st->max_probe;
  const int64_t nchunks = (nw + W - 1) / W;
  const int64_t nitems = nchunks * S;
  if (threadIdx.x == 0) s_err = 0;
  // An item is (window chunk, key slab).  If its state overflows (more distinct keys
  // than ST), the item restarts with its slab split into 2, 4, ... sub-slabs of home
  // slots, each slid on its own; the count and emit passes overflow on the same key
  // sets, so both pick the same split (rows of a window stay inside its (window,
  // slab) range, sub-slab after sub-slab -- row order inside a window is free, A8).
  __shared__ int s_ovf;
  __shared__ int64_t s_wrun[kHashMaxChunk];            // rows of earlier sub-slabs per window
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t chunk = item / S;
    const uint32_t slab0 = (uint32_t)((item % S) * SB);
    const int64_t ja = J0 + chunk * W;
    const int64_t jb = ja + W < J1 ? ja + W : J1;
    for (int nsub = 1;; nsub *= 2) {
      const int SBs = SB / nsub;
      bool overflow = false;
      for (int sub = 0; sub < nsub && !overflow; ++sub) {
        const uint32_t slot0 = slab0 + (uint32_t)(sub * SBs);
        __syncthreads();
        for (int h = threadIdx.x; h < ST; h += blockDim.x) {
          skeys[h] = kEmpty;
          scnt[h] = 0;
          FOR_F(f) { sf[f * ST + h] = field_identity(p.field[f].kind); sc[f * ST + h] = 0.0; }
        }
        if (threadIdx.x == 0) { s_nocc = 0; s_ovf = 0; }
        for (int x = threadIdx.x; x < (int)(jb - ja); x += blockDim.x)
          if (sub == 0) s_wrun[x] = 0;
        __syncthreads();
        auto find = [&](uint64_t k) -> int {
          uint32_t h = (uint32_t)(fmix64(k) >> 32) & (uint32_t)(ST - 1);
          volatile uint64_t *vk = skeys;
          for (int probe = 0; probe < ST; ++probe) {
            uint64_t cur = vk[h];
            if (cur == k) return (int)h;
            if (cur == kEmpty) {
              uint64_t old = atomicCAS((unsigned long long *)&skeys[h], kEmpty, k);
              if (old == kEmpty) occ[atomicAdd(&s_nocc, 1)] = (int)h;
              if (old == kEmpty || old == k) return (int)h;
            }
            h = (h + 1) & (uint32_t)(ST - 1);
          }
          s_ovf = 1;
          return -1;
        };
        // mode 0: add (+1) / subtract (-1) invertible fields; mode 2: min/max only
        auto visit_pane = [&](int64_t q, int sign, bool minmax) {
          const uint64_t *b = table + (q & (p.R - 1)) * p.slot_words;
          const int64_t sp = (SBs + maxprobe + 1) < p.C ? (SBs + maxprobe + 1) : p.C;
          for (int64_t o = threadIdx.x; o < sp; o += blockDim.x) {
            const uint32_t h = (slot0 + (uint32_t)o) & Cm;
            const uint64_t k = b[h];
            if (k == kEmpty) continue;
            const uint32_t home = (uint32_t)fmix64(k) & Cm;
            if (((home - slot0) & Cm) >= (uint32_t)SBs) continue;
            const int s = find(k);
            if (s < 0) continue;
            if (!minmax) {
              atomicAdd((unsigned long long *)&scnt[s], (unsigned long long)(sign * (int64_t)b[p.C + h]));
            }
            FOR_F(f) {
              const int kind = p.field[f].kind;
              const uint64_t v = b[fld_off(p, f) + h];
              if (!minmax && kind == FK_SUM_F)
                dd_atomic_add((double *)&sf[f * ST + s], &sc[f * ST + s], sign * __longlong_as_double((long long)v));
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
          if (s_ovf) { overflow = true; break; }          // block-uniform (read after the barrier)
          const int nocc = s_nocc;
          for (int x = threadIdx.x; x < nocc; x += blockDim.x) {
            const int h = occ[x];
            if (scnt[h] == 0)
              FOR_F(f)
                if (p.field[f].kind == FK_SUM_F || p.field[f].kind == FK_SUM_I) { sf[f * ST + h] = 0; sc[f * ST + h] = 0.0; }
          }
          if (p.has_minmax) {
            for (int x = threadIdx.x; x < nocc; x += blockDim.x)
              FOR_F(f)
                if (p.field[f].kind == FK_MIN || p.field[f].kind == FK_MAX)
                  sf[f * ST + occ[x]] = field_identity(p.field[f].kind);
            __syncthreads();
            for (int64_t q = j * p.L; q < j * p.L + p.K; ++q) visit_pane(q, 0, true);
          }
          __syncthreads();
          if (s_ovf) { overflow = true; break; }
          int my = 0;
          uint64_t fv[kMaxField];
          const int nocc2 = s_nocc;                         // the min/max visit may have added keys
          for (int x = threadIdx.x; x < nocc2; x += blockDim.x) {
            const int h = occ[x];
            if (skeys[h] == kEmpty || scnt[h] <= 0) continue;
            FOR_F(f) fv[f] = p.field[f].kind == FK_SUM_F ? (uint64_t)__double_as_longlong(
                __longlong_as_double((long long)sf[f * ST + h]) + sc[f * ST + h]) : sf[f * ST + h];
            if (having_ok(p, scnt[h], fv)) ++my;
          }
          int total;
          int excl = group_excl_scan(my, 256, scan_sm, total);
          const int64_t ci = (j - J0) * S + (item % S);
          const int wi = (int)(j - ja);
          if (!EMIT) {
            if (threadIdx.x == 0) counts[ci] = (sub == 0 ? 0 : counts[ci]) + total;
          } else {
            int64_t r = counts[ci] + s_wrun[wi] + excl;
            for (int x = threadIdx.x; x < nocc2; x += blockDim.x) {
              const int h = occ[x];
              if (skeys[h] == kEmpty || scnt[h] <= 0) continue;
              FOR_F(f) fv[f] = p.field[f].kind == FK_SUM_F ? (uint64_t)__double_as_longlong(
                __longlong_as_double((long long)sf[f * ST + h]) + sc[f * ST + h]) : sf[f * ST + h];
              if (!having_ok(p, scnt[h], fv)) continue;
              int64_t kv[kMaxKey];
              decode_key(p, skeys[h], kv);
              write_row(p, rows, r++, kv, scnt[h], fv);
            }
          }
          __syncthreads();
          if (threadIdx.x == 0) s_wrun[wi] += total;
        }
      }
      if (!overflow) break;
      if (SB / (2 * nsub) < 1) {                          // one home slot and still too many keys
        if (threadIdx.x == 0) s_err = 1;
        break;
      }
    }
  }
  __syncthreads();
  if (threadIdx.x == 0 && s_err) atomicOr(&st->error, ERR_CAPACITY);
}


}  // namespace sb

namespace sb {

void *p2_kernel(const Plan &p) {
  return p.key_mode == KM_HASH ? (void *)k_win_hash<true> : (void *)k_win_vh<true>;
}

cudaError_t launch_windows(const Plan &p, const QueryDev &q, const SlotDev &s, bool emit, int grid, int win_chunk,
                           cudaStream_t st) {
  if (p.key_mode == KM_HASH) {
    if (emit) k_win_hash<true><<<grid, 256, p.p2_smem, st>>>(p, q.st, q.table, s.counts, s.rows, win_chunk);
    else k_win_hash<false><<<grid, 256, p.p2_smem, st>>>(p, q.st, q.table, s.counts, s.rows, win_chunk);
  } else {
    if (!emit) {
      k_vh_build<<<148 * 8, 256, 0, st>>>(p, q.st, q.table, q.vh_pre, q.vh_suf);
      k_win_vh<false><<<grid, 256, 0, st>>>(p, q.st, q.vh_pre, q.vh_suf, s.counts, s.rows);
    } else {
      k_win_vh<true><<<grid, 256, 0, st>>>(p, q.st, q.vh_pre, q.vh_suf, s.counts, s.rows);
    }
  }
  return cudaGetLastError();
}

// DENSE/GLOBAL: van Herk arrays, then one fused count + look-back + emit pass
cudaError_t launch_windows_fused(const Plan &p, const QueryDev &q, const SlotDev &s, int grid, cudaStream_t st) {
  // long windows: a CTA per (block, word) when there are few words (no GROUP BY),
  // a warp per (block, word) otherwise; short windows: a thread per (block, word)
  if (p.K > 64 && p.slot_words < 64) k_vh_build_long<<<148 * 8, 256, 0, st>>>(p, q.st, q.table, q.vh_pre, q.vh_suf);
  else if (p.K > 64 && p.win_wide) k_vh_build_tile<<<148 * 8, 256, 0, st>>>(p, q.st, q.table, q.vh_pre, q.vh_suf);
  else if (p.K > 64) k_vh_build_cta<<<148 * 8, 256, 0, st>>>(p, q.st, q.table, q.vh_pre, q.vh_suf);
  else k_vh_build<<<148 * 8, 256, 0, st>>>(p, q.st, q.table, q.vh_pre, q.vh_suf);
  if (p.win_wide) return launch_windows_wide(p, q, s, p.ww_grid, st);
  if (p.S == 1 && p.C <= 256) {
    int cshift = 0;
    while ((1 << cshift) < p.C) ++cshift;
    void (*k)(const Plan, State *, const uint64_t *, const uint64_t *, const int64_t *, WinHdr *, unsigned char *,
              uint64_t *, int *, int) = p.nf <= 1 ? k_win_packed<1> : p.nf <= 2 ? k_win_packed<2>
                                     : p.nf <= 4 ? k_win_packed<4> : k_win_packed<8>;
    k<<<grid, 256, 0, st>>>(p, q.st, q.vh_pre, q.vh_suf, q.pane_ts, (WinHdr *)s.hdr, s.rows, q.tile_status,
                            q.tile_ctr, cshift);
    return cudaGetLastError();
  }
  const int gpb = 256 / p.GS;
  int wc = gpb * 8 / p.S;
  if (wc * p.S > kFusedMaxItems) wc = kFusedMaxItems / p.S;
  if (wc < 1) wc = 1;
  if (p.GS == 32)
    k_win_fused<32><<<grid, 256, 0, st>>>(p, q.st, q.vh_pre, q.vh_suf, q.pane_ts, (WinHdr *)s.hdr, s.rows,
                                          q.tile_status, q.tile_ctr, wc);
  else
    k_win_fused<256><<<grid, 256, 0, st>>>(p, q.st, q.vh_pre, q.vh_suf, q.pane_ts, (WinHdr *)s.hdr, s.rows,
                                           q.tile_status, q.tile_ctr, wc);
  return cudaGetLastError();
}

}  // namespace sb

namespace sb {
void *p2_kernel_count(const Plan &p) {
  return p.key_mode == KM_HASH ? (void *)k_win_hash<false> : (void *)k_win_vh<false>;
}
}  // namespace sb

// ===========================================================================
// HASH keys with a declared (radix-packed) domain larger than the dense table:
// "slab mode".  After a task's scan, every pane that a closed window needs is
// compacted once from its hash table into key-range buckets (slab = key / SB,
// a counting sort by slab; PAPER.md L1350-1353 also compacts sparse GPU hash
// tables).  Window assembly then slides a *dense* per-slab state over the
// buckets: each pane entry is read twice (enter, leave) and each window-slab
// costs SB/256 shared-memory slot checks per thread plus its output rows.
namespace sb {

__device__ __forceinline__ uint32_t *ck_key(const Plan &p, uint64_t *base) { return (uint32_t *)base; }
__device__ __forceinline__ uint32_t *ck_cnt(const Plan &p, uint64_t *base) { return (uint32_t *)base + p.C; }
__device__ __forceinline__ uint64_t *ck_fld(const Plan &p, uint64_t *base, int f) { return base + p.C + (int64_t)f * p.C; }

__global__ void __launch_bounds__(256)
k_pane_compact(const Plan p, const State *__restrict__ st, const uint64_t *__restrict__ table,
               uint64_t *__restrict__ clist, int32_t *__restrict__ coff) {
  extern __shared__ __align__(16) int s_hist[];          // [S + 1] counts, then [S] cursors
  const int S = p.S, SB = p.SB;
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  int64_t lo = st->compacted_hi;                         // panes below were compacted by earlier tasks
  if (lo < J0 * p.L) lo = J0 * p.L;
  const int64_t hi = (J1 - 1) * p.L + p.K;
  const int64_t cw = p.C * (1 + p.nf);                     // clist words per pane slot
  int *cur = s_hist + S + 1;
  for (int64_t q = lo + blockIdx.x; q < hi; q += gridDim.x) {
    const int64_t slot = q & (p.R - 1);
    const uint64_t *tab = table + slot * p.slot_words;
    uint64_t *cl = clist + slot * cw;
    for (int i = threadIdx.x; i <= S; i += blockDim.x) s_hist[i] = 0;
    __syncthreads();
    for (int64_t h = threadIdx.x; h < p.C; h += blockDim.x) {
      const uint64_t k = tab[h];
      if (k != kEmpty) atomicAdd(&s_hist[(int)(k / (uint64_t)SB)], 1);
    }
    __syncthreads();
    if (threadIdx.x < 32) {                                // exclusive scan of S bucket sizes
      const int lane = threadIdx.x;
      int run = 0;
      for (int b = 0; b < S; b += 32) {
        const int v = b + lane < S ? s_hist[b + lane] : 0;
        int x = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(kFull, x, o);
          if (lane >= o) x += y;
        }
        if (b + lane < S) cur[b + lane] = run + x - v;
        run += __shfl_sync(kFull, x, 31);
      }
      if (lane == 0) cur[S] = run;
    }
    __syncthreads();
    for (int i = threadIdx.x; i <= S; i += blockDim.x) coff[slot * (S + 1) + i] = cur[i];
    __syncthreads();
    for (int64_t h = threadIdx.x; h < p.C; h += blockDim.x) {
      const uint64_t k = tab[h];
      if (k == kEmpty) continue;
      const int pos = atomicAdd(&cur[(int)(k / (uint64_t)SB)], 1);
      ck_key(p, cl)[pos] = (uint32_t)k;
      ck_cnt(p, cl)[pos] = (uint32_t)tab[p.C + h];
      FOR_F(f) ck_fld(p, cl, f)[pos] = tab[fld_off(p, f) + h];
    }
    __syncthreads();
  }
}

template <bool EMIT>
__global__ void __launch_bounds__(256)
k_win_slab(const Plan p, State *__restrict__ st, uint64_t *__restrict__ clist, const int32_t *__restrict__ coff,
           int64_t *__restrict__ counts, unsigned char *__restrict__ rows, int W) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ int scan_sm[40];
  const int S = p.S, SB = p.SB;
  int64_t *scnt = (int64_t *)smem;
  uint64_t *sf = (uint64_t *)(scnt + SB);
  double *sc = (double *)(sf + (size_t)p.nf * SB);      // TwoSum compensation of FK_SUM_F fields
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const int64_t cw = p.C * (1 + p.nf);
  const int64_t nchunks = (nw + W - 1) / W;
  const int64_t nitems = nchunks * S;
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t chunk = item / S;
    const int slab = (int)(item % S);
    const uint32_t kbase = (uint32_t)slab * (uint32_t)SB;
    const int64_t ja = J0 + chunk * W;
    const int64_t jb = ja + W < J1 ? ja + W : J1;
    __syncthreads();
    for (int s = threadIdx.x; s < SB; s += blockDim.x) {
      scnt[s] = 0;
      FOR_F(f) { sf[f * SB + s] = field_identity(p.field[f].kind); sc[f * SB + s] = 0.0; }
    }
    __syncthreads();
    // entries of one pane have distinct keys: plain read-modify-write, barrier per pane
    auto visit = [&](int64_t q, int sign, bool minmax) {
      const int64_t slot = q & (p.R - 1);
      uint64_t *cl = clist + slot * cw;
      const int a = coff[slot * (S + 1) + slab], b = coff[slot * (S + 1) + slab + 1];
      for (int e = a + threadIdx.x; e < b; e += blockDim.x) {
        const int s = (int)(ck_key(p, cl)[e] - kbase);
        if (!minmax) scnt[s] += sign * (int64_t)ck_cnt(p, cl)[e];
        FOR_F(f) {
          const int kind = p.field[f].kind;
          const uint64_t v = ck_fld(p, cl, f)[e];
          if (!minmax && kind == FK_SUM_F) {
            double e;
            sf[f * SB + s] = (uint64_t)__double_as_longlong(two_sum(__longlong_as_double((long long)sf[f * SB + s]),
                                                                    sign * __longlong_as_double((long long)v), e));
            sc[f * SB + s] += e;
          }
          else if (!minmax && kind == FK_SUM_I) sf[f * SB + s] = (uint64_t)((int64_t)sf[f * SB + s] + sign * (int64_t)v);
          else if (minmax && (kind == FK_MIN || kind == FK_MAX)) sf[f * SB + s] = field_combine(kind, sf[f * SB + s], v);
        }
      }
      __syncthreads();
    };
    for (int64_t q = ja * p.L; q < ja * p.L + p.K; ++q) visit(q, +1, false);
    for (int64_t j = ja; j < jb; ++j) {
      if (j > ja) {
        for (int64_t q = (j - 1) * p.L + p.K; q < j * p.L + p.K; ++q) visit(q, +1, false);
        for (int64_t q = (j - 1) * p.L; q < j * p.L; ++q) visit(q, -1, false);
      }
      for (int s = threadIdx.x; s < SB; s += blockDim.x)
        if (scnt[s] == 0)
          FOR_F(f)
            if (p.field[f].kind == FK_SUM_F || p.field[f].kind == FK_SUM_I) { sf[f * SB + s] = 0; sc[f * SB + s] = 0.0; }
      if (p.has_minmax) {
        for (int s = threadIdx.x; s < SB; s += blockDim.x)
          FOR_F(f)
            if (p.field[f].kind == FK_MIN || p.field[f].kind == FK_MAX) sf[f * SB + s] = field_identity(p.field[f].kind);
        __syncthreads();
        for (int64_t q = j * p.L; q < j * p.L + p.K; ++q) visit(q, 0, true);
      }
      __syncthreads();
      int my = 0;
      uint64_t fv[kMaxField];
      for (int s = threadIdx.x; s < SB; s += blockDim.x) {
        if (scnt[s] <= 0) continue;
        if (p.nhave) {
          FOR_F(f) fv[f] = p.field[f].kind == FK_SUM_F ? (uint64_t)__double_as_longlong(
              __longlong_as_double((long long)sf[f * SB + s]) + sc[f * SB + s]) : sf[f * SB + s];
          if (!having_ok(p, scnt[s], fv)) continue;
        }
        ++my;
      }
      int total;
      const int excl = group_excl_scan(my, 256, scan_sm, total);
      const int64_t ci = (j - J0) * S + slab;
      if (!EMIT) {
        if (threadIdx.x == 0) counts[ci] = total;
      } else {
        int64_t r = counts[ci] + excl;
        for (int s = threadIdx.x; s < SB; s += blockDim.x) {
          if (scnt[s] <= 0) continue;
          FOR_F(f) fv[f] = p.field[f].kind == FK_SUM_F ? (uint64_t)__double_as_longlong(
              __longlong_as_double((long long)sf[f * SB + s]) + sc[f * SB + s]) : sf[f * SB + s];
          if (p.nhave && !having_ok(p, scnt[s], fv)) continue;
          int64_t kv[kMaxKey];
          decode_key(p, (uint64_t)(kbase + (uint32_t)s), kv);
          write_row(p, rows, r++, kv, scnt[s], fv);
        }
      }
      __syncthreads();
    }
  }
}

cudaError_t launch_windows_slab(const Plan &p, const QueryDev &q, const SlotDev &s, bool emit, int grid, int W,
                                cudaStream_t st) {
  if (!emit) {
    k_pane_compact<<<148 * 4, 256, (2 * p.S + 2) * sizeof(int), st>>>(p, q.st, q.table, q.clist, q.coff);
    k_win_slab<false><<<grid, 256, p.p2_smem, st>>>(p, q.st, q.clist, q.coff, s.counts, s.rows, W);
  } else {
    k_win_slab<true><<<grid, 256, p.p2_smem, st>>>(p, q.st, q.clist, q.coff, s.counts, s.rows, W);
  }
  return cudaGetLastError();
}
void *slab_kernel(bool emit) { return emit ? (void *)k_win_slab<true> : (void *)k_win_slab<false>; }

}  // namespace sb
