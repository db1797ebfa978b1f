// k_bucket.cu -- "bucket mode": GROUP BY over a large declared key domain with
// count-based windows (BASELINE.json configs[2], C3 at G = 16K..64K groups).
//
// With G >> tuples per pane, a pane partial (window fragment, §3
// L518-684) has about as many entries as the pane has tuples, so aggregating
// panes into hash tables buys nothing and costs a global hash insert per tuple.
// Instead:
//   K1+σ+bucket (k_pane_bucket): one TMA-staged pass over the task; every
//     qualifying tuple's (key mod SB as u16, f32 values) is appended to the
//     bucket of its (pane, key slab), slab = key / SB.  Space is reserved per
//     stage with one global atomic per (pane, slab); each bucket holds at most
//     g entries (a count-window pane has g positions), so it never overflows.
//   window assembly, per (key slab, chunk of W consecutive windows), with a
//     dense shared-memory state of the slab's SB keys that slides over the
//     buckets (enter the panes a window gains, leave the ones it loses):
//       k_bkt_count  u32 counts only, tracking the number of non-empty keys:
//                    rows per (window, slab), no slot scan;
//       k_win_scan   (k_task.cu) exclusive scan → row offsets + window headers;
//       k_bkt_emit   counts + fp64 sums; per window the warps scan their slot
//                    ranges and write the rows of present keys coalesced
//                    (ballot/popc positions, per-warp-range counts tracked
//                    incrementally, so no block-wide scan per window).
// Float sums are added and subtracted in compensated fp64 (sum + TwoSum error
// word, common.cuh dd_atomic_add): the state's error does not grow with the
// magnitude of values that already left the window; a key whose count returns to
// 0 has both words reset to exactly 0.
#include <cuda_runtime.h>
#include <climits>
#include <stdint.h>

#include "common.cuh"
#include "launch_internal.h"
#include "tma.cuh"

namespace sb {

constexpr int kBkThreads = 256;
constexpr int kBkStageBytes = 16384;
constexpr int kBkStages = 3;
constexpr int kBkHist = 1024;             // (panes per stage) x S histogram entries
constexpr int kBkMaxTPT = 4;              // tuples per thread per stage (tuple_bytes >= 16)

__device__ __forceinline__ uint32_t bk_lds_u32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ int64_t bk_lds_s64(uint32_t a) {
  int64_t v;
  asm volatile("ld.shared.s64 %0, [%1];" : "=l"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ int bk_divg(const Plan &p, int x) {     // floor(x / g), 0 <= x < 2^30
  return (int)(((uint64_t)(uint32_t)x * p.g_magic) >> p.g_mshift);
}
// A bucket's fill word carries kBkDirty once it holds a value that is not a
// multiple of 2^-24 below 32 in magnitude: windows whose buckets are all clean
// slide their state in plain fp64 exactly (every partial sum of < 2^24 such
// values is a multiple of 2^-24 below 2^53·2^-24); windows touching a dirty
// bucket slide it in compensated fp64 (sum + TwoSum error word, common.cuh),
// half a slab at a time so the state still fits shared memory.
constexpr unsigned long long kBkDirty = 1ull << 62;
__device__ __forceinline__ bool bk_exact(uint32_t b) {
  if ((b & 0x7fffffffu) == 0u) return true;
  const uint32_t ex = (b >> 23) & 0xffu;
  if (ex == 0u || ex >= 132u) return false;                 // denormal, |x| >= 32, inf, NaN
  if (ex >= 126u) return true;                                // |x| >= 0.5: lowest bit >= 2^-24
  const uint32_t m = (b & 0x7fffffu) | 0x800000u;
  return (int)(__ffs(m) - 1) >= (int)(126u - ex);
}
__device__ __forceinline__ uint16_t *bk_keys(const Plan &p, unsigned char *bkt) { return (uint16_t *)bkt; }
__device__ __forceinline__ float *bk_vals(const Plan &p, unsigned char *bkt) { return (float *)(bkt + p.bk_vals); }

// ---------------------------------------------------------------------------
// K1 + σ + bucketing: one pass over the task's tuples
template <int NF>
__global__ void __launch_bounds__(kBkThreads, 2)
k_pane_bucket(const Plan p, State *__restrict__ st, const unsigned char *__restrict__ tup, int64_t n,
              unsigned long long *__restrict__ bcnt, unsigned char *__restrict__ bkt, int64_t *__restrict__ pane_ts) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int tid = threadIdx.x, lane = tid & 31;
  const int tb = p.tuple_bytes;
  const int ST = kBkStageBytes / tb;
  unsigned char *stages = smem;
  uint64_t *full = (uint64_t *)(smem + kBkStages * kBkStageBytes);
  uint64_t *empty = full + kBkStages;
  int *hist = (int *)(empty + kBkStages);
  int *base = hist + kBkHist;
  int *hdirty = base + kBkHist;                  // (pane, slab) received a value fp64 cannot slide exactly
  for (int e = tid; e < kBkHist; e += kBkThreads) { hist[e] = 0; hdirty[e] = 0; }
  const int64_t per = ((n + gridDim.x - 1) / gridDim.x + ST - 1) / ST * ST;
  const int64_t lo = (int64_t)blockIdx.x * per;
  const int64_t hi = lo + per < n ? lo + per : n;
  const int nst = hi > lo ? (int)((hi - lo + ST - 1) / ST) : 0;
  if (tid == 0) {
    for (int i = 0; i < kBkStages; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], kBkThreads / 32); }
    fence_mbar_init();
  }
  __syncthreads();
  auto issue = [&](int k) {
    const int slot = k % kBkStages;
    const int64_t cnt = (hi - lo - (int64_t)k * ST) < ST ? (hi - lo - (int64_t)k * ST) : ST;
    const uint32_t bytes = (uint32_t)(cnt * tb);
    mbar_expect_tx(&full[slot], bytes);
    bulk_g2s(stages + slot * kBkStageBytes, tup + (lo + (int64_t)k * ST) * tb, bytes, &full[slot]);
  };
  if (tid == 0)
    for (int k = 0; k < kBkStages && k < nst; ++k) issue(k);

  // CTA-relative pane coordinates: global pane = P0 + rel pane of local tuple x = (R0 + x) / g
  const int64_t gpos = st->task_pos + lo;
  const int64_t P0 = gpos / p.g;
  const int R0 = (int)(gpos - P0 * p.g);
  const int64_t mp = st->J0 * p.L - P0;                      // panes < J0·L belong to emitted windows
  const int minrel = mp <= 0 ? 0 : (mp > (1 << 30) ? (1 << 30) : (int)mp);
  const int g = (int)p.g, S = p.S, shift = p.bk_shift;
  const uint32_t smask = (1u << shift) - 1u;
  const uint32_t tsoff = 4u * p.ts_word, koff = 4u * p.key[0].word;
  const uint32_t dom = (uint32_t)p.key[0].domain;
  uint32_t foff[NF > 0 ? NF : 1];
#pragma unroll
  for (int f = 0; f < NF; ++f) foff[f] = 4u * p.field[f].word;
  const int64_t Rm = p.R - 1;
  uint16_t *keys = bk_keys(p, bkt);
  float *vals = bk_vals(p, bkt);
  const uint32_t sbase = (uint32_t)__cvta_generic_to_shared(stages);
  int err = 0;
  int64_t prev_last = (lo > 0 && lo < hi) ? *(const int64_t *)(tup + (lo - 1) * tb + tsoff) : INT64_MIN;
  const int range32 = (int)(hi - lo);
  int slot = 0;
  uint32_t phase = 0;
  for (int k = 0; k < nst; ++k) {
    mbar_wait(&full[slot], phase);
    const uint32_t sb = sbase + (uint32_t)(slot * kBkStageBytes);
    const int xs = k * ST;
    const int ntup = range32 - xs < ST ? range32 - xs : ST;
    const int pf = bk_divg(p, R0 + xs);
    const int pl = bk_divg(p, R0 + xs + ntup - 1);
    int e_[kBkMaxTPT], r_[kBkMaxTPT], q_[kBkMaxTPT];
    uint32_t ko_[kBkMaxTPT];
    uint32_t v_[kBkMaxTPT][NF > 0 ? NF : 1];
#pragma unroll
    for (int u = 0; u < kBkMaxTPT; ++u) {
      const int i = tid + u * kBkThreads;
      e_[u] = -1;
      if (i >= ntup) continue;
      const uint32_t t = sb + (uint32_t)(i * tb);
      // K1: τ non-decreasing (L347-349) and non-negative (L349-350)
      const int64_t tau = bk_lds_s64(t + tsoff);
      const int64_t up = i > 0 ? bk_lds_s64(t - tb + tsoff) : prev_last;
      if (tau < up) err |= ERR_ORDER;
      if (tau < 0) err |= ERR_TS;
      const int rel = R0 + xs + i;
      const int q = bk_divg(p, rel);
      if (q < minrel) continue;
      if (rel == q * g) pane_ts[(P0 + q) & Rm] = tau;
      if (p.npred && !s_preds(p, stages + (sb - sbase) + i * tb)) continue;
      const uint32_t key = bk_lds_u32(t + koff);
      if (key >= dom) { err |= ERR_KEY; continue; }
      const int e = (q - pf) * S + (int)(key >> shift);
      e_[u] = e;
      q_[u] = q;
      ko_[u] = key & smask;
      bool dirty = false;
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        v_[u][f] = bk_lds_u32(t + foff[f]);
        dirty |= !bk_exact(v_[u][f]);
      }
      if (dirty) hdirty[e] = 1;
      r_[u] = atomicAdd(&hist[e], 1);
    }
    prev_last = bk_lds_s64(sb + (uint32_t)((ntup - 1) * tb) + tsoff);
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[slot]);
    if (tid == 0 && k + kBkStages < nst) {
      mbar_wait(&empty[slot], phase);
      issue(k + kBkStages);
    }
    if (++slot == kBkStages) { slot = 0; phase ^= 1u; }
    __syncthreads();
    // reserve bucket space: one global atomic per (pane, slab) touched by the stage
    const int nh = (pl - pf + 1) * S;
    for (int e = tid; e < nh; e += kBkThreads) {
      const int c = hist[e];
      if (c) {
        const int q = pf + e / S;
        unsigned long long *w = &bcnt[((P0 + q) & Rm) * S + (e % S)];
        base[e] = (int)atomicAdd(w, (unsigned long long)c);     // fill count: the low 32 bits
        if (hdirty[e]) { atomicOr(w, kBkDirty); hdirty[e] = 0; }
        hist[e] = 0;
      }
    }
    __syncthreads();
#pragma unroll
    for (int u = 0; u < kBkMaxTPT; ++u) {
      if (e_[u] < 0) continue;
      const int64_t b = ((P0 + q_[u]) & Rm) * S + (e_[u] % S);
      const int64_t pos = b * g + base[e_[u]] + r_[u];
      keys[pos] = (uint16_t)ko_[u];
#pragma unroll
      for (int f = 0; f < NF; ++f) vals[(b * NF + f) * g + base[e_[u]] + r_[u]] = __uint_as_float(v_[u][f]);
    }
  }
  if (err) atomicOr(&st->error, err);
}

// ---------------------------------------------------------------------------
// Window assembly.  Sliding from window j to j+1 leaves panes [j·L, (j+1)·L) and
// enters [j·L+K, (j+1)·L+K).  With L = 1 (slide = pane, every config here) the
// bucket entries of step j+1 are loaded into registers while step j is applied
// (and, in k_bkt_emit, while window j is written), so the global-load latency
// of a step is hidden behind the previous one; kPF entries per thread and
// direction are prefetched, anything beyond is loaded in place.
constexpr int kPF = 4;                // k_bkt_count: 256 threads
constexpr int kEmitPF = 2;           // k_bkt_emit: 512 threads, two entries per thread and direction

template <int NF>
struct BkVals { float v[NF > 0 ? NF : 1]; };
template <int NF, int PF = kPF>
struct BkStep {
  int nl, ne;                          // entries leaving / entering (this slab)
  int64_t bl, be;                      // bucket index of the leaving / entering pane
  uint32_t kl[PF], ke[PF];             // prefetched keys
  BkVals<NF> vl[PF], ve[PF];
};

// bucket fill counts of step j (leave pane j, enter pane j+K; L = 1)
__device__ __forceinline__ void bk_counts(const Plan &p, const unsigned long long *__restrict__ bcnt, int64_t j, int s,
                                          int &nl, int &ne) {
  const int64_t Rm = p.R - 1;
  nl = (int)__ldg(bcnt + (j & Rm) * p.S + s);
  ne = (int)__ldg(bcnt + ((j + p.K) & Rm) * p.S + s);
}
template <int NF, bool VALS, int PF>
__device__ __forceinline__ void bk_prefetch(const Plan &p, const uint16_t *__restrict__ keys,
                                            const float *__restrict__ vals, int64_t j, int s, int nl, int ne,
                                            BkStep<NF, PF> &x) {
  const int64_t Rm = p.R - 1;
  const int S = p.S, g = (int)p.g, tid = threadIdx.x, nt = blockDim.x;
  x.bl = (j & Rm) * S + s;
  x.be = ((j + p.K) & Rm) * S + s;
  x.nl = nl;
  x.ne = ne;
#pragma unroll
  for (int u = 0; u < PF; ++u) {
    const int e = tid + u * nt;
    if (e < x.nl) {
      x.kl[u] = __ldg(keys + x.bl * g + e);
      if (VALS)
#pragma unroll
        for (int f = 0; f < NF; ++f) x.vl[u].v[f] = __ldg(vals + (x.bl * NF + f) * g + e);
    }
    if (e < x.ne) {
      x.ke[u] = __ldg(keys + x.be * g + e);
      if (VALS)
#pragma unroll
        for (int f = 0; f < NF; ++f) x.ve[u].v[f] = __ldg(vals + (x.be * NF + f) * g + e);
    }
  }
}

// window assembly, pass 1: rows per (window, slab) = keys with a non-zero count;
// chunks of about a third of the emission chunk (3 CTAs per SM)
__global__ void __launch_bounds__(256, 3)
k_bkt_count(const Plan p, const State *__restrict__ st, const unsigned long long *__restrict__ bcnt,
            const unsigned char *__restrict__ bkt, int64_t *__restrict__ counts) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ int dn[3];
  uint32_t *cnt = (uint32_t *)smem;
  const int S = p.S, SB = 1 << p.bk_shift, W = p.bk_W > 48 ? (p.bk_W + 2) / 3 : 16, g = (int)p.g;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const int64_t nitems = ((nw + W - 1) / W) * S;
  const int64_t Rm = p.R - 1;
  const uint16_t *keys = (const uint16_t *)bkt;
  const int tid = threadIdx.x, lane = tid & 31, nt = blockDim.x;
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t chunk = item / S;
    const int s = (int)(item % S);
    const int64_t ja = J0 + chunk * W;
    const int64_t jb = ja + W < J1 ? ja + W : J1;
    __syncthreads();
    for (int i = tid; i < SB; i += nt) cnt[i] = 0;
    if (tid < 3) dn[tid] = 0;
    __syncthreads();
    // +1 / -1 over entries [from, ne) of bucket b; returns this thread's change of the non-empty key count
    auto visit = [&](int64_t b, int from, int ne, bool add) -> int {
      const uint16_t *kp = keys + b * g;
      int d = 0;
      for (int e = from + tid; e < ne; e += nt) {
        const uint32_t k = __ldg(kp + e);
        if (add) d += atomicAdd(&cnt[k], 1u) == 0u;
        else d -= atomicSub(&cnt[k], 1u) == 1u;
      }
      return d;
    };
    int nnz = 0;
    int it = 0;
    // record window j's row count once every thread's updates for it are done
    auto finish = [&](int64_t j, int d) {
      d = __reduce_add_sync(kFull, (unsigned)d);
      if (lane == 0 && d) atomicAdd(&dn[it % 3], d);
      __syncthreads();
      nnz += dn[it % 3];
      if (tid == 0) {
        dn[(it + 2) % 3] = 0;
        counts[(j - J0) * S + s] = nnz;
      }
      ++it;
    };
    {
      int d = 0;
      for (int64_t q = ja * p.L; q < ja * p.L + p.K; ++q) d += visit((q & Rm) * S + s, 0, (int)__ldg(bcnt + (q & Rm) * S + s), true);
      finish(ja, d);
    }
    if (p.L == 1) {
      // three prefetch buffers in rotation: the entries of a step are loaded two
      // steps before they are applied, with no register copies in between
      BkStep<0> X0, X1, X2;
      int cnl = 0, cne = 0;                 // bucket counts of the next step to prefetch
      if (ja + 1 < jb) {
        int nl, ne;
        bk_counts(p, bcnt, ja, s, nl, ne);
        bk_prefetch<0, false>(p, keys, nullptr, ja, s, nl, ne, X0);
        if (ja + 2 < jb) {
          bk_counts(p, bcnt, ja + 1, s, nl, ne);
          bk_prefetch<0, false>(p, keys, nullptr, ja + 1, s, nl, ne, X1);
        }
        if (ja + 3 < jb) bk_counts(p, bcnt, ja + 2, s, cnl, cne);
      }
      int64_t j = ja + 1;
      auto body = [&](BkStep<0> &cur, BkStep<0> &nxt) {      // apply step j-1 → j, prefetch step j+1
        if (j + 2 < jb) {
          bk_prefetch<0, false>(p, keys, nullptr, j + 1, s, cnl, cne, nxt);
          if (j + 3 < jb) bk_counts(p, bcnt, j + 2, s, cnl, cne);
        }
        int d = 0;
#pragma unroll
        for (int u = 0; u < kPF; ++u) {
          const int e = tid + u * nt;
          if (e < cur.nl) d -= atomicSub(&cnt[cur.kl[u]], 1u) == 1u;
          if (e < cur.ne) d += atomicAdd(&cnt[cur.ke[u]], 1u) == 0u;
        }
        d += visit(cur.bl, kPF * nt, cur.nl, false) + visit(cur.be, kPF * nt, cur.ne, true);
        finish(j, d);
        ++j;
      };
      while (j < jb) {
        body(X0, X2);
        if (j >= jb) break;
        body(X1, X0);
        if (j >= jb) break;
        body(X2, X1);
      }
    } else {
      for (int64_t j = ja + 1; j < jb; ++j) {
        int d = 0;
        for (int64_t q = (j - 1) * p.L; q < j * p.L; ++q) d += visit((q & Rm) * S + s, 0, (int)__ldg(bcnt + (q & Rm) * S + s), false);
        for (int64_t q = (j - 1) * p.L + p.K; q < j * p.L + p.K; ++q)
          d += visit((q & Rm) * S + s, 0, (int)__ldg(bcnt + (q & Rm) * S + s), true);
        finish(j, d);
      }
    }
  }
}

// fp64 quotient x / c for a small positive integer c: hardware reciprocal seed,
// one Newton step, then a residual correction of the quotient (≈ correctly rounded;
// AVG is compared within 1e-5, reading A12)
__device__ __forceinline__ double bk_div(double x, double c) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(c));
  r = fma(r, fma(-c, r, 1.0), r);
  const double q = x * r;
  return fma(r, fma(-c, q, x), q);
}

// window assembly, pass 2: rows of one (slab, window chunk) item for the keys
// [half·SBe, (half+1)·SBe) of the slab.  COMP = false: the whole slab (SBe = SB)
// in plain fp64 (clean buckets: exact); COMP = true: half a slab in compensated
// fp64 (the item touches a dirty bucket).  n0[]: rows of half 0 per window, so
// half 1 continues after them.
template <int NF, int NA, bool COMP>
__device__ __forceinline__ void bk_emit_item(const Plan &p, const State *__restrict__ st,
                                             const unsigned long long *__restrict__ bcnt,
                                             const unsigned char *__restrict__ bkt, const int64_t *__restrict__ offs,
                                             unsigned char *__restrict__ rows, unsigned char *smem, int *wn, int *n0,
                                             int s, int64_t ja, int64_t jb, int SBe, int half) {
  const int S = p.S, g = (int)p.g;
  double *sum = (double *)smem;                               // [NF][SBe]
  double *cmp = sum + (size_t)NF * SBe;                       // [NF][SBe] TwoSum compensation (COMP)
  uint32_t *cnt = (uint32_t *)(smem + (size_t)(COMP ? 16 : 8) * NF * SBe);   // [SBe]
  uint16_t *slist = (uint16_t *)(cnt + SBe);                  // [SBe]: per-warp lists of present slots
  const int64_t J0 = st->J0;
  const int64_t Rm = p.R - 1;
  const uint16_t *keys = (const uint16_t *)bkt;
  const float *vals = (const float *)(bkt + p.bk_vals);
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5, nt = blockDim.x, nwarp = nt >> 5;
  const int RS = SBe / nwarp;                                 // slots per warp range (multiple of 32)
  int rs_shift = 0;
  while ((1 << rs_shift) < RS) ++rs_shift;
  const unsigned lt = (1u << lane) - 1u;
  const bool pipe = p.L == 1;
  const uint32_t klo = (uint32_t)(half * SBe);
  int akind[NA], afld[NA];
#pragma unroll
  for (int a = 0; a < NA; ++a) { akind[a] = p.agg[a].fn; afld[a] = p.agg[a].field; }
  // key k of the slab -> state slot, or -1 for the other half
  auto slot_of = [&](uint32_t k) -> int { return COMP ? ((k - klo) < (uint32_t)SBe ? (int)(k - klo) : -1) : (int)k; };
  auto upd = [&](uint32_t k0, bool add, BkVals<NF> v) {
    const int k = slot_of(k0);
    if (k < 0) return;
    if (add) {
      if (atomicAdd(&cnt[k], 1u) == 0u) atomicAdd(&wn[k >> rs_shift], 1);
    } else {
      if (atomicSub(&cnt[k], 1u) == 1u) atomicSub(&wn[k >> rs_shift], 1);
    }
#pragma unroll
    for (int f = 0; f < NF; ++f) {
      const double x = add ? (double)v.v[f] : -(double)v.v[f];
      if (COMP) dd_atomic_add(&sum[f * SBe + k], &cmp[f * SBe + k], x);
      else atomicAdd(&sum[f * SBe + k], x);
    }
  };
  __syncthreads();
  for (int i = tid; i < SBe; i += nt) {
    cnt[i] = 0;
#pragma unroll
    for (int f = 0; f < NF; ++f) {
      sum[f * SBe + i] = 0.0;
      if (COMP) cmp[f * SBe + i] = 0.0;
    }
  }
  if (tid < 32) wn[tid] = 0;
  __syncthreads();
  auto visit = [&](int64_t b, int from, int ne, bool add) {
    const uint16_t *kp = keys + b * g;
    for (int e = from + tid; e < ne; e += nt) {
      BkVals<NF> v;
#pragma unroll
      for (int f = 0; f < NF; ++f) v.v[f] = __ldg(vals + (b * NF + f) * g + e);
      upd(__ldg(kp + e), add, v);
    }
  };
  auto zero_key = [&](uint32_t k0) {                    // a key that left the window entirely: exact 0 sums
    const int k = slot_of(k0);
    if (k >= 0 && cnt[k] == 0u)
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        sum[f * SBe + k] = 0.0;
        if (COMP) cmp[f * SBe + k] = 0.0;
      }
  };
  auto zero_fix = [&](int64_t b, int from, int ne) {
    const uint16_t *kp = keys + b * g;
    for (int e = from + tid; e < ne; e += nt) zero_key(__ldg(kp + e));
  };
  auto pane_b = [&](int64_t q) { return (q & Rm) * S + s; };
  for (int64_t q = ja * p.L; q < ja * p.L + p.K; ++q) visit(pane_b(q), 0, (int)__ldg(bcnt + pane_b(q)), true);
  BkStep<NF, kEmitPF> A, B;
  int cnl = 0, cne = 0;                 // bucket counts of the step after the prefetched one
  if (pipe && ja + 1 < jb) {
    int nl, ne;
    bk_counts(p, bcnt, ja, s, nl, ne);
    bk_prefetch<NF, true>(p, keys, vals, ja, s, nl, ne, A);
    if (ja + 2 < jb) bk_counts(p, bcnt, ja + 1, s, cnl, cne);
  }
  int64_t r0n = offs[(ja - J0) * S + s];
  __syncthreads();
  for (int64_t j = ja; j < jb; ++j) {
    const int64_t r0 = r0n + (COMP && half ? n0[j - ja] : 0);
    if (j + 1 < jb) r0n = offs[(j + 1 - J0) * S + s];                                  // next window's offset
    if (pipe && j + 2 < jb) {                                                          // in flight during the emission
      bk_prefetch<NF, true>(p, keys, vals, j + 1, s, cnl, cne, B);
      if (j + 3 < jb) bk_counts(p, bcnt, j + 2, s, cnl, cne);
    }
    // ---- emit window j, slab s: warp w owns slots [w·RS, (w+1)·RS)
    const int wc = lane < nwarp ? wn[lane] : 0;
    int x = wc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(kFull, x, o);
      if (lane >= o) x += y;
    }
    const int woff = __shfl_sync(kFull, x - wc, wid);
    // column pointers at this warp's first row; rows of a window past the slot
    // capacity are not written (k_win_scan flags SABER_ENOMEM)
    const int tot = __shfl_sync(kFull, x, nwarp - 1);
    if (COMP && half == 0 && tid == 0) n0[j - ja] = tot;
    if (r0 + tot <= p.rows_cap) {
      int32_t *kcol = (int32_t *)(rows + p.col_off[0]) + r0 + woff;
      uint64_t *acol[NA];
#pragma unroll
      for (int a = 0; a < NA; ++a) acol[a] = (uint64_t *)(rows + p.col_off[1 + a]) + r0 + woff;
      // pass 1: compact this warp's present slots into its slot list (ballot/popc;
      // lane l reads slots 4l..4l+3 of each 128-slot block, list order is free)
      uint16_t *sl_w = slist + wid * RS;
      const uint4 *cw = (const uint4 *)(cnt + wid * RS) + lane;
      int n = 0;
      if (RS & 127) {                                       // small slabs: 32 slots per round
        for (int o = 0; o < RS; o += 32) {
          const uint32_t c = cnt[wid * RS + o + lane];
          const unsigned bal = __ballot_sync(kFull, c != 0u);
          if (c) sl_w[n + __popc(bal & lt)] = (uint16_t)(o + lane);
          n += __popc(bal);
        }
      } else
#pragma unroll 2
      for (int o = 0; o < RS; o += 128) {
        const uint4 c4 = cw[o >> 2];
        const uint32_t cc[4] = {c4.x, c4.y, c4.z, c4.w};
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const unsigned bal = __ballot_sync(kFull, cc[u] != 0u);
          if (cc[u]) sl_w[n + __popc(bal & lt)] = (uint16_t)(o + 4 * lane + u);
          n += __popc(bal);
        }
      }
      __syncwarp();
      // pass 2: one row per lane, consecutive rows across the warp (coalesced stores)
      const int32_t kb = (s << p.bk_shift) + (int32_t)klo + wid * RS;
#pragma unroll 4
      for (int i = lane; i < n; i += 32) {
        const int sl = sl_w[i];
        const uint32_t c = cnt[wid * RS + sl];
        kcol[i] = kb + sl;
        double sv[NF > 0 ? NF : 1];
#pragma unroll
        for (int f = 0; f < NF; ++f)
          sv[f] = COMP ? sum[f * SBe + wid * RS + sl] + cmp[f * SBe + wid * RS + sl] : sum[f * SBe + wid * RS + sl];
        const double dc = (double)c;
#pragma unroll
        for (int a = 0; a < NA; ++a) {
          double xv = 0.0;
#pragma unroll
          for (int f = 0; f < NF; ++f) xv = afld[a] == f ? sv[f] : xv;
          const uint64_t bits = akind[a] == AG_COUNT ? (uint64_t)c
                                : akind[a] == AG_SUM ? (uint64_t)__double_as_longlong(xv)
                                                     : (uint64_t)__double_as_longlong(bk_div(xv, dc));
          acol[a][i] = bits;
        }
      }
      __syncwarp();
    }
    if (j + 1 >= jb) break;
    __syncthreads();
    // ---- slide to window j+1
    if (pipe) {
#pragma unroll
      for (int u = 0; u < kEmitPF; ++u) {
        const int e = tid + u * nt;
        if (e < A.nl) upd(A.kl[u], false, A.vl[u]);
        if (e < A.ne) upd(A.ke[u], true, A.ve[u]);
      }
      visit(A.bl, kEmitPF * nt, A.nl, false);
      visit(A.be, kEmitPF * nt, A.ne, true);
    } else {
      for (int64_t q = j * p.L; q < (j + 1) * p.L; ++q) visit(pane_b(q), 0, (int)__ldg(bcnt + pane_b(q)), false);
      for (int64_t q = j * p.L + p.K; q < (j + 1) * p.L + p.K; ++q) visit(pane_b(q), 0, (int)__ldg(bcnt + pane_b(q)), true);
    }
    __syncthreads();
    // zero-fix writes sums of keys with count 0 only; the next emission reads keys
    // with count > 0 only, so no barrier separates them
    if (pipe) {
#pragma unroll
      for (int u = 0; u < kEmitPF; ++u) {
        const int e = tid + u * nt;
        if (e < A.nl) zero_key(A.kl[u]);
      }
      zero_fix(A.bl, kEmitPF * nt, A.nl);
      A = B;
    } else {
      for (int64_t q = j * p.L; q < (j + 1) * p.L; ++q) zero_fix(pane_b(q), 0, (int)__ldg(bcnt + pane_b(q)));
    }
  }
}

// COMP = false emits the clean items, COMP = true the dirty ones (two launches,
// each skipping the other kind: one register allocation per path)
template <int NF, int NA, bool COMP>
__global__ void __launch_bounds__(512, 1)
k_bkt_emit(const Plan p, const State *__restrict__ st, const unsigned long long *__restrict__ bcnt,
           const unsigned char *__restrict__ bkt, const int64_t *__restrict__ offs, unsigned char *__restrict__ rows) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ int wn[32];
  const int S = p.S, SB = 1 << p.bk_shift, W = p.bk_W;
  // dirty items: rows of half 0 per window, after the half-slab state
  int *n0 = (int *)(smem + (size_t)(SB / 2) * (6 + 16 * NF));
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const int64_t nitems = ((nw + W - 1) / W) * S;
  const int64_t Rm = p.R - 1;
  const bool always = p.s >= (1ll << 24);       // exactness bound of clean buckets: < 2^24 values per key
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t chunk = item / S;
    const int s = (int)(item % S);
    const int64_t ja = J0 + chunk * W;
    const int64_t jb = ja + W < J1 ? ja + W : J1;
    // does any bucket of the item's panes hold a value plain fp64 cannot slide exactly?
    bool dirty = always;
    for (int64_t q = ja * p.L + threadIdx.x; q < (jb - 1) * p.L + p.K; q += blockDim.x)
      dirty |= (__ldg(bcnt + (q & Rm) * S + s) & kBkDirty) != 0;
    dirty = __syncthreads_or(dirty);
    if (dirty != COMP) continue;
    if (!COMP) {
      bk_emit_item<NF, NA, false>(p, st, bcnt, bkt, offs, rows, smem, wn, n0, s, ja, jb, SB, 0);
    } else {
      for (int h = 0; h < 2; ++h)
        bk_emit_item<NF, NA, true>(p, st, bcnt, bkt, offs, rows, smem, wn, n0, s, ja, jb, SB / 2, h);
    }
  }
}

// ---------------------------------------------------------------------------
// host side
int bk_scan_smem() { return kBkStages * kBkStageBytes + 2 * kBkStages * 8 + 3 * kBkHist * 4; }
// clean items: SB·(count + slot list + nf sums); dirty items: SB/2·(count + list + nf sums + nf compensations)
int bk_emit_smem(const Plan &p) {
  const int SB = 1 << p.bk_shift;
  const int clean = SB * (6 + 8 * p.nf), dirty = (SB / 2) * (6 + 16 * p.nf) + 4 * 1024;
  return clean > dirty ? clean : dirty;
}
int bk_count_smem(const Plan &p) { return (1 << p.bk_shift) * 4; }

static void *bk_scan_kernel(const Plan &p) {
  return p.nf == 0 ? (void *)k_pane_bucket<0> : p.nf == 1 ? (void *)k_pane_bucket<1> : (void *)k_pane_bucket<2>;
}
template <int NF, bool C>
static void *bk_emit_nf(int na) {
  return na == 1 ? (void *)k_bkt_emit<NF, 1, C> : na == 2 ? (void *)k_bkt_emit<NF, 2, C>
       : na == 3 ? (void *)k_bkt_emit<NF, 3, C> : (void *)k_bkt_emit<NF, 4, C>;
}
template <bool C>
static void *bk_emit_kernel(const Plan &p) {
  return p.nf == 0 ? bk_emit_nf<0, C>(p.nagg) : p.nf == 1 ? bk_emit_nf<1, C>(p.nagg) : bk_emit_nf<2, C>(p.nagg);
}


// window assembly, pass 1 without a sliding state (one-pane slides, slabs of
// <= 4,096 keys, K <= 64): a (window, slab)'s row count is the number of keys
// present in any of its K pane buckets = popcount of the OR of the K pane
// presence bitmaps.  An item (slab, chunk of windows) builds the bitmaps of its
// panes in shared memory from the buckets' u16 key offsets (one shared atomicOr
// per entry, each entry read once) and ORs them per window; no per-window
// barrier, no count/uncount pair per entry (k_bkt_count: C3 G=1K 200 µs per GiB).
constexpr int kBrSmem = 48 * 1024;
template <int WPB>
__global__ void __launch_bounds__(256)
k_bkt_rows(const Plan p, const State *__restrict__ st, const unsigned long long *__restrict__ bcnt,
           const unsigned char *__restrict__ bkt, int64_t *__restrict__ counts) {
  extern __shared__ __align__(128) unsigned char smem[];
  uint32_t *bm = (uint32_t *)smem;                       // [panes][WPB]
  constexpr int TPW = WPB < 32 ? WPB : 32;               // threads per window
  const int S = p.S, K = (int)p.K, g = (int)p.g;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  // windows per item: what the bitmaps' shared memory holds, but about one item per CTA
  const int wmax = kBrSmem / (4 * WPB) - K + 1;
  const int64_t want = (nw + gridDim.x - 1) / gridDim.x;
  const int Wt = (int)(want < 16 ? 16 : want > wmax ? wmax : want);
  const int64_t nitems = ((nw + Wt - 1) / Wt) * S;
  const int64_t Rm = p.R - 1;
  const uint16_t *keys = (const uint16_t *)bkt;
  const int tid = threadIdx.x;
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t chunk = item / S;
    const int s = (int)(item % S);
    const int64_t ja = J0 + chunk * Wt;
    const int jn = (int)((J1 - ja) < Wt ? (J1 - ja) : Wt);
    const int np = jn + K - 1;
    __syncthreads();
    for (int i = tid; i < np * WPB; i += 256) bm[i] = 0u;
    __syncthreads();
    // a warp per pane; 16-B loads of 8 key offsets when the bucket stride allows
    const int warp = tid >> 5, lane = tid & 31;
    for (int x = warp; x < np; x += 8) {
      const int64_t b = ((ja + x) & Rm) * S + s;
      const int n = (int)__ldg(bcnt + b);
      const uint16_t *kp = keys + b * g;
      uint32_t *row = bm + x * WPB;
      if ((g & 7) == 0) {
        const uint4 *kp4 = (const uint4 *)kp;
#pragma unroll 4
        for (int v = lane; v * 8 < n; v += 32) {
          const uint4 q = __ldg(kp4 + v);
          const uint32_t w[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
          for (int h = 0; h < 8; ++h)
            if (v * 8 + h < n) {
              const uint32_t k = (w[h >> 1] >> (16 * (h & 1))) & 0xffffu;
              atomicOr(&row[k >> 5], 1u << (k & 31));
            }
        }
      } else {
#pragma unroll 4
        for (int e = lane; e < n; e += 32) {
          const uint32_t k = __ldg(kp + e);
          atomicOr(&row[k >> 5], 1u << (k & 31));
        }
      }
    }
    __syncthreads();
    constexpr int WPP = 256 / TPW;                       // windows per pass
    const int sub = tid % TPW;
    for (int w0 = 0; w0 < jn; w0 += WPP) {
      const int w = w0 + tid / TPW;
      int c = 0;
      if (w < jn)
        for (int z = sub; z < WPB; z += TPW) {
          uint32_t m = 0;
          for (int k = 0; k < K; ++k) m |= bm[(w + k) * WPB + z];
          c += __popc(m);
        }
#pragma unroll
      for (int o = TPW / 2; o; o >>= 1) c += __shfl_xor_sync(kFull, c, o);
      if (sub == 0 && w < jn) counts[(ja + w - J0) * S + s] = c;
    }
  }
}
static void *bk_rows_kernel(const Plan &p) {
  const int wpb = (1 << p.bk_shift) / 32;
  if (p.L != 1 || p.K > 64 || wpb < 8 || wpb > 128 || kBrSmem / (4 * wpb) - p.K + 1 < 16 ||
      std::getenv("SABER_NO_BKROWS"))
    return nullptr;
  return wpb == 8 ? (void *)k_bkt_rows<8> : wpb == 16 ? (void *)k_bkt_rows<16> : wpb == 32 ? (void *)k_bkt_rows<32>
       : wpb == 64 ? (void *)k_bkt_rows<64> : (void *)k_bkt_rows<128>;
}

cudaError_t bk_set_attributes(const Plan &p) {
  cudaError_t e = cudaFuncSetAttribute(bk_scan_kernel(p), cudaFuncAttributeMaxDynamicSharedMemorySize, bk_scan_smem());
  if (e) return e;
  e = cudaFuncSetAttribute((void *)k_bkt_count, cudaFuncAttributeMaxDynamicSharedMemorySize, bk_count_smem(p));
  if (e) return e;
  if (void *k = bk_rows_kernel(p)) {
    e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, kBrSmem);
    if (e) return e;
  }
  e = cudaFuncSetAttribute(bk_emit_kernel<false>(p), cudaFuncAttributeMaxDynamicSharedMemorySize, bk_emit_smem(p));
  if (e) return e;
  return cudaFuncSetAttribute(bk_emit_kernel<true>(p), cudaFuncAttributeMaxDynamicSharedMemorySize, bk_emit_smem(p));
}

int bk_scan_blocks_per_sm(const Plan &p) {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, bk_scan_kernel(p), kBkThreads, bk_scan_smem());
  return b > 0 ? b : 1;
}

cudaError_t launch_bucket_scan(const Plan &p, const QueryDev &q, const void *tuples, int64_t n, int grid,
                               cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  const int64_t stage_t = kBkStageBytes / p.tuple_bytes;
  const int64_t need = (n + stage_t - 1) / stage_t;
  const int g = (int)(need < grid ? need : grid);
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&tuples, (void *)&n, (void *)&q.table, (void *)&q.bkt,
                  (void *)&q.pane_ts};
  return cudaLaunchKernel(bk_scan_kernel(p), dim3(g), dim3(kBkThreads), args, (size_t)bk_scan_smem(), st);
}

cudaError_t launch_bucket_windows(const Plan &p, const QueryDev &q, const SlotDev &s, int nsm, cudaStream_t st) {
  const unsigned long long *bc = (const unsigned long long *)q.table;
  if (void *k = bk_rows_kernel(p)) {
    void *ra[] = {(void *)&p, (void *)&q.st, (void *)&bc, (void *)&q.bkt, (void *)&s.counts};
    cudaError_t e = cudaLaunchKernel(k, dim3(nsm * 4), dim3(256), ra, (size_t)kBrSmem, st);
    if (e) return e;
  } else {
    k_bkt_count<<<nsm * 3, 256, bk_count_smem(p), st>>>(p, q.st, bc, q.bkt, s.counts);
  }
  cudaError_t e = launch_win_scan(p, q, s, st);
  if (e) return e;
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&bc, (void *)&q.bkt, (void *)&s.counts, (void *)&s.rows};
  e = cudaLaunchKernel(bk_emit_kernel<false>(p), dim3(nsm * p.bk_ctas), dim3(p.bk_threads), args,
                       (size_t)bk_emit_smem(p), st);
  if (e) return e;
  return cudaLaunchKernel(bk_emit_kernel<true>(p), dim3(nsm * p.bk_ctas), dim3(p.bk_threads), args,
                          (size_t)bk_emit_smem(p), st);
}

}  // namespace sb
