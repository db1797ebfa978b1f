// k_winblock.cu -- window assembly for short windows over few keys (DENSE /
// GLOBAL keys, K <= 64 panes per window, a pane slot of at most a few hundred
// words): C1, C3 at G = 64, C4.  One kernel, no van Herk arrays in HBM/L2.
//
// The batch operator f_b (§3) combines the K pane partials of
// each window.  A CTA takes, in ticket order, NB consecutive K-aligned pane
// blocks; the windows starting in them need panes [b0·K, (b0+NB+1)·K - 1).  It
// stages those pane slots in shared memory with 1-D TMA bulk copies, and per
// (block, table word) computes the van Herk / Gil-Werman decomposition in place:
//   S[a] = ⊕ partial[a .. end of a's block]      (suffix, backward)
//   V[a] = S[a] ⊕ P[a+K-1],  P = ⊕ partial[start of the next block .. a+K-1]
// (V[a] = S[a] when a is block-aligned): one combine per window and word for
// count/sum/min/max alike, the same decomposition as k_vh_build + k_win_packed
// but without writing and re-reading the prefix/suffix arrays.  Then it counts
// the rows of its windows (ballots), obtains its output offset by decoupled
// look-back over earlier tickets and writes headers and rows (window-major,
// key order inside a window).
#include <cuda_runtime.h>
#include <cstdlib>
#include <stdint.h>

#include "common.cuh"
#include "launch_internal.h"
#include "tma.cuh"

namespace sb {

constexpr int kWbThreads = 256;
constexpr int kWbMaxWin = 512;          // windows per item (row counts in shared memory)
constexpr int kWbMaxRounds = 64;        // (window, key) rounds of 256 per item
constexpr int kWbMaxWords = 1024;       // table words per pane slot

template <bool FAST>
__device__ __forceinline__ uint64_t wb_combine(int kind, uint64_t a, uint64_t b) {
  if (FAST)        // counts and sums only: integer or fp64 add
    return kind == FK_SUM_F ? (uint64_t)__double_as_longlong(__longlong_as_double((long long)a) +
                                                             __longlong_as_double((long long)b))
                            : a + b;
  return kind < 0 ? a + b : field_combine(kind, a, b);
}

// fp64 x / c for a positive count c: reciprocal seed, one Newton step and a
// residual correction of the quotient (within an ulp; AVG is compared at 1e-5, A12)
__device__ __forceinline__ double wb_div(double x, double c) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(c));
  r = fma(r, fma(-c, r, 1.0), r);
  const double q = x * r;
  return fma(r, fma(-c, q, x), q);
}

// FAST: dense / global keys (one int32 key or none), only COUNT / SUM / AVG over
// sum fields, no HAVING: presence is count > 0 and rows are written directly
template <int NF, bool FAST>
__global__ void __launch_bounds__(kWbThreads)
k_win_block(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ table,
            const int64_t *__restrict__ pane_ts, WinHdr *__restrict__ hdr, unsigned char *__restrict__ rows,
            uint64_t *__restrict__ status, int *__restrict__ ticket, int NB) {
  hdr += st->hdr_base;                         // windows earlier rounds of the task wrote
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ uint64_t bar;
  __shared__ int s_t;
  __shared__ int64_t s_base;
  __shared__ int s_wcnt[kWbMaxWin];           // rows per window of the item
  __shared__ int s_roff[kWbMaxRounds * 8];    // rows per (round, warp) → exclusive offsets
  __shared__ unsigned s_rbal[kWbMaxRounds * 8];  // presence ballots per (round, warp)
  __shared__ int s_woff[kWbMaxWin];           // first row of each window inside the item
  __shared__ signed char s_kind[kWbMaxWords];  // combine of each table word: -1 count, else the field kind
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  const int64_t W = p.slot_words;             // C·(1+nf) words per pane slot
  const int64_t K = p.K, L = p.L, C = p.C, Rm = p.R - 1;
  const uint64_t epoch = (uint64_t)st->tile_epoch;
  const int64_t qlo = J0 * L, qhi = (J1 - 1) * L + K - 1;   // panes read by the task's windows
  const int64_t bfirst = qlo / K;
  const int64_t nitems = (qhi / K - bfirst + NB) / NB;       // items covering the blocks of window starts
  const int NP = (int)((NB + 1) * K - 1);                     // staged panes per item
  uint64_t *raw = (uint64_t *)smem;                           // [NP][W]
  // window values: in place over block b0's rows when NB == 1 (the prefix reads
  // only block b0+1), a separate [NB·K][W] array otherwise
  uint64_t *V = NB == 1 ? raw : raw + (int64_t)NP * W;
  const unsigned lt = (1u << lane) - 1u;
  if (tid == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
  for (int w = tid; w < W; w += kWbThreads) {
    const int f = (int)(w / C) - 1;
    s_kind[w] = (signed char)(f < 0 ? -1 : p.field[f].kind);
  }
  __syncthreads();
  uint32_t phase = 0;
  for (;;) {
    if (tid == 0) s_t = atomicAdd(ticket, 1);
    __syncthreads();
    const int64_t t = s_t;
    if (t >= nitems) break;
    const int64_t b0 = bfirst + t * NB;
    const int64_t q0 = b0 * K;                                // first staged pane
    // windows of this item: j with j·L in [max(q0, qlo), (b0+NB)·K), j < J1
    int64_t ja = (q0 + L - 1) / L;
    if (ja < J0) ja = J0;
    int64_t jb = ((b0 + NB) * K + L - 1) / L;
    if (jb > J1) jb = J1;
    const int nwin = jb > ja ? (int)(jb - ja) : 0;
    // ---- stage panes [max(q0, qlo), min(q0+NP, qhi+1)) with bulk copies (ring-contiguous runs)
    const int64_t sa = q0 > qlo ? q0 : qlo;
    const int64_t se = (q0 + NP) < (qhi + 1) ? (q0 + NP) : (qhi + 1);
    if (tid == 0) {
      uint32_t bytes = 0;
      for (int64_t q = sa; q < se;) {
        const int64_t run = ((q | Rm) + 1 - q) < (se - q) ? ((q | Rm) + 1 - q) : (se - q);   // up to the ring wrap
        int64_t done = 0;
        while (done < run) {
          const int64_t n = (run - done) * W * 8 < (1 << 20) ? (run - done) : ((1 << 20) / (W * 8));
          bytes += (uint32_t)(n * W * 8);
          done += n;
        }
        q += run;
      }
      mbar_expect_tx(&bar, bytes);
      for (int64_t q = sa; q < se;) {
        const int64_t run = ((q | Rm) + 1 - q) < (se - q) ? ((q | Rm) + 1 - q) : (se - q);
        int64_t done = 0;
        while (done < run) {
          const int64_t n = (run - done) * W * 8 < (1 << 20) ? (run - done) : ((1 << 20) / (W * 8));
          bulk_g2s(raw + (q + done - q0) * W, table + ((q + done) & Rm) * W, (uint32_t)(n * W * 8), &bar);
          done += n;
        }
        q += run;
      }
    }
    for (int i = tid; i < nwin; i += kWbThreads) s_wcnt[i] = 0;
    mbar_wait(&bar, phase);
    phase ^= 1u;
    // ---- van Herk / Gil-Werman per table word (threads over consecutive words,
    // so shared-memory accesses are conflict-free)
    // presence of a row depends only on the window count when there is no HAVING:
    // the count words are assembled first and the item's row count is published
    // to the look-back chain before the field words are, so successors rarely wait
    const bool early = NB == 1 && !p.nhave;
    if (NB == 1) {
      // in place: (A) suffix of block b0 into its own rows and prefix of block
      // b0+1 into its own rows, one thread per (word, direction); (B) V[a] =
      // S[a] ⊕ P[a+K-1] for a > b0·K, in parallel over (pane, word)
      const int64_t bs = q0, be = (bs + K - 1) < qhi ? (bs + K - 1) : qhi;
      const int64_t lo = bs > qlo ? bs : qlo;
      const int64_t pe = (bs + 2 * K - 2) < qhi ? (bs + 2 * K - 2) : qhi;   // last prefix pane needed
      const int Wi = (int)W;
      auto vh_words = [&](int wa, int wb) {          // words [wa, wb) of every staged pane
        const int Wr = wb - wa;
        for (int x = tid; x < 2 * Wr; x += kWbThreads) {
          const bool suffix = x < Wr;
          const int w = wa + (suffix ? x : x - Wr);
          const int kind = s_kind[w];
          uint64_t acc = kind < 0 ? 0ull : field_identity(kind);
          // 4 loads in flight per step (the combine chain is the only dependency)
          const int qa = suffix ? (int)(be - q0) : (int)(bs + K - q0);
          const int qe = suffix ? (int)(lo - q0) : (int)(pe - q0);     // inclusive end of the walk
          const int n = suffix ? qa - qe + 1 : qe - qa + 1;
          const int dq = suffix ? -Wi : Wi;
          uint64_t *r = raw + qa * Wi + w;
          int k = 0;
          for (; k + 4 <= n; k += 4) {
            const uint64_t v0 = r[0], v1 = r[dq], v2 = r[2 * dq], v3 = r[3 * dq];
            acc = wb_combine<FAST>(kind, acc, v0); r[0] = acc;
            acc = wb_combine<FAST>(kind, acc, v1); r[dq] = acc;
            acc = wb_combine<FAST>(kind, acc, v2); r[2 * dq] = acc;
            acc = wb_combine<FAST>(kind, acc, v3); r[3 * dq] = acc;
            r += 4 * dq;
          }
          for (; k < n; ++k) {
            acc = wb_combine<FAST>(kind, acc, r[0]);
            r[0] = acc;
            r += dq;
          }
        }
        __syncthreads();
        const int64_t a0 = lo > bs ? lo : bs + 1;                // windows starting at a0..be need a prefix
        const int64_t a1 = (pe - K + 1) < be ? (pe - K + 1) : be;
        const int nvals = a1 >= a0 ? (int)((a1 - a0 + 1) * Wr) : 0;
        // (pane, word) pairs walked incrementally: no division per element
        const int step_a = kWbThreads / Wr, step_w = kWbThreads % Wr;
        int ao = tid / Wr, w = tid - (tid / Wr) * Wr;
        const int base_a = (int)(a0 - q0), Kd = (int)(K - 1) * Wi;
        for (int x = tid; x < nvals; x += kWbThreads) {
          const int kind = s_kind[wa + w];
          uint64_t *rr = raw + (base_a + ao) * Wi + wa + w;
          *rr = wb_combine<FAST>(kind, *rr, rr[Kd]);
          ao += step_a;
          w += step_w;
          if (w >= Wr) { w -= Wr; ++ao; }
        }
      };
      if (early) {
        vh_words(0, (int)C);
        __syncthreads();
        // rows per window from the counts alone; the item total is published now
        const int Ci = (int)C;
        const int nit = nwin * Ci;
        int mine = 0;
        for (int it = tid; it < nit; it += kWbThreads) {
          const int wi = it / Ci, key = it - wi * Ci;
          const bool pres = (int64_t)(V + ((ja + wi) * L - q0) * W)[key] > 0;
          mine += pres;
          if (pres) atomicAdd(&s_wcnt[wi], 1);
        }
        mine = __reduce_add_sync(kFull, (unsigned)mine);
        if (lane == 0) s_roff[warp] = mine;
        __syncthreads();
        if (tid == 0) {
          int tot = 0;
          for (int i = 0; i < kWbThreads / 32; ++i) tot += s_roff[i];
          if (t > 0) lb_st(&status[t], lb_pack(epoch, 1, (uint64_t)tot));
        }
        vh_words((int)C, Wi);
      } else {
        vh_words(0, Wi);
      }
    } else {
      // separate V: one thread per (block, word): suffix into V, then the prefix
      // of the next block completes the windows starting inside the block
      for (int64_t x = tid; x < (int64_t)NB * W; x += kWbThreads) {
        const int bi = (int)(x / W);
        const int64_t w = x - (int64_t)bi * W;
        const int f = (int)(w / C) - 1;
        const int kind = f < 0 ? -1 : p.field[f].kind;
        const uint64_t id = kind < 0 ? 0ull : field_identity(kind);
        const int64_t bs = q0 + (int64_t)bi * K;
        const int64_t lo = bs > qlo ? bs : qlo;
        if (lo > qhi || lo >= bs + K) continue;
        const int64_t be = (bs + K - 1) < qhi ? (bs + K - 1) : qhi;
        uint64_t acc = id;
        for (int64_t q = be; q >= lo; --q) {
          acc = wb_combine<FAST>(kind, acc, raw[(q - q0) * W + w]);
          V[(q - q0) * W + w] = acc;
        }
        acc = id;
        for (int64_t a = bs + 1; a <= be; ++a) {
          const int64_t e = a + K - 1;
          if (e > qhi) break;
          acc = wb_combine<FAST>(kind, acc, raw[(e - q0) * W + w]);
          if (a >= lo) V[(a - q0) * W + w] = wb_combine<FAST>(kind, V[(a - q0) * W + w], acc);
        }
      }
    }
    __syncthreads();
    // ---- rows: (window, key) items in window-major order, 256 per round
    const int nitem = nwin * (int)C;
    const int nrounds = (nitem + kWbThreads - 1) / kWbThreads;
    const int Ci = (int)C;
    const int cshift = (Ci & (Ci - 1)) == 0 ? __ffs(Ci) - 1 : -1;  // C a power of two: shifts
    auto win_of = [&](int it) { return cshift >= 0 ? it >> cshift : it / Ci; };
    auto value = [&](int it, int64_t &c, uint64_t (&fv)[kMaxField]) -> bool {
      const int wi = win_of(it), key = it - wi * Ci;
      const uint64_t *v = V + ((ja + wi) * L - q0) * W;
      c = (int64_t)v[key];
      if constexpr (FAST) {
        return c > 0;
      } else {
        if (c <= 0) return false;
#pragma unroll
        for (int f = 0; f < NF; ++f)
          if (f < p.nf) fv[f] = v[(1 + f) * C + key];
        return !p.nhave || having_ok(p, c, fv);
      }
    };
    // pass 1: presence per item (ballots kept for pass 2), rows per window
    for (int r = 0; r < nrounds; ++r) {
      const int it = r * kWbThreads + tid;
      int64_t c = 0;
      uint64_t fv[kMaxField];
      const bool pres = it < nitem && value(it, c, fv);
      const unsigned bal = __ballot_sync(kFull, pres);
      if (lane == 0) { s_roff[r * 8 + warp] = __popc(bal); s_rbal[r * 8 + warp] = bal; }
      if (pres && !early) atomicAdd(&s_wcnt[win_of(it)], 1);
    }
    __syncthreads();
    if (warp == 0) {                                          // exclusive scan of (round, warp) counts
      const int n = nrounds * 8;
      int run = 0;
      for (int b = 0; b < n; b += 32) {
        const int v = b + lane < n ? s_roff[b + lane] : 0;
        int y = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int z = __shfl_up_sync(kFull, y, o);
          if (lane >= o) y += z;
        }
        if (b + lane < n) s_roff[b + lane] = run + y - v;
        run += __shfl_sync(kFull, y, 31);
      }
      const uint64_t total = (uint64_t)run;
      const int64_t excl = lookback_warp(status, t, epoch, total, st->row_base);
      if (lane == 0) {
        s_base = excl;
        if (t == nitems - 1) {
          st->sel_rows = excl + (int64_t)total;
          if (excl + (int64_t)total > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
        }
      }
    } else if (warp == 1) {                                   // window row offsets: scan of rows per window
      int run = 0;
      for (int b = 0; b < nwin; b += 32) {
        const int v = b + lane < nwin ? s_wcnt[b + lane] : 0;
        int y = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int z = __shfl_up_sync(kFull, y, o);
          if (lane >= o) y += z;
        }
        if (b + lane < nwin) s_woff[b + lane] = run + y - v;
        run += __shfl_sync(kFull, y, 31);
      }
    }
    __syncthreads();
    const int64_t base = s_base;
    for (int wi = tid; wi < nwin; wi += kWbThreads) {
      const int64_t j = ja + wi;
      WinHdr h;
      h.window_id = j;
      h.ts = (p.win_kind == WK_TIME) ? p.T0 + j * p.l : pane_ts[(j * L) & Rm];
      h.row_offset = base + s_woff[wi];
      h.nrows = s_wcnt[wi];
      h.flags = 0;
      hdr[j - J0] = h;
    }
    for (int r = 0; r < nrounds; ++r) {
      const int it = r * kWbThreads + tid;
      const unsigned bal = s_rbal[r * 8 + warp];
      if (!((bal >> lane) & 1u)) continue;
      int64_t c = 0;
      uint64_t fv[kMaxField];
#pragma unroll
      for (int f = 0; f < kMaxField; ++f) fv[f] = 0;
      const int64_t row = base + s_roff[r * 8 + warp] + __popc(bal & lt);
      if (FAST) {
        if (row >= p.rows_cap) continue;
        const int wi = win_of(it), key = it - wi * Ci;
        const uint64_t *v = V + ((ja + wi) * L - q0) * W;
        const int64_t cnt = (int64_t)v[key];
        if (p.nkeys) ((int32_t *)(rows + p.col_off[0]))[row] = key;
#pragma unroll
        for (int a = 0; a < kMaxAgg; ++a) {
          if (a >= p.nagg) break;
          const AggOut &o = p.agg[a];
          uint64_t x = 0;
#pragma unroll
          for (int f = 0; f < NF; ++f)
            if (f == o.field) x = v[(1 + f) * C + key];
          uint64_t bits = o.fn == AG_COUNT ? (uint64_t)cnt : x;
          if (o.fn == AG_AVG) {
            const double sum = p.field[o.field].kind == FK_SUM_F ? __longlong_as_double((long long)x)
                                                                  : (double)(int64_t)x;
            bits = (uint64_t)__double_as_longlong(wb_div(sum, (double)cnt));
          }
          ((uint64_t *)(rows + p.col_off[p.nkeys + a]))[row] = bits;
        }
        continue;
      }
      value(it, c, fv);
      int64_t kv[kMaxKey];
      decode_key(p, (uint64_t)(it - win_of(it) * Ci), kv);
      write_row(p, rows, row, kv, c, fv);
    }
    // the van Herk pass wrote `raw` with generic stores; the next ticket's bulk
    // copies (async proxy) overwrite it after the barrier
    fence_proxy_async_smem();
    __syncthreads();
  }
}

// ---------------------------------------------------------------------------
// Row counts of the register variant's windows, before any value is assembled
// (count-then-write, the shape of PAPER.md §5.4): on the FAST plan a
// (window, key) row exists iff the key's window count is > 0, i.e. iff one of the
// window's K panes counted the key.  Per pane, a ballot over its C count words
// gives a presence bitmap (C/32 words, shared memory); a window's bitmap is the
// OR of its K pane bitmaps and its row count the popcount.  A CTA takes 256
// consecutive windows per ticket, scans their row counts, and a decoupled
// look-back over the (cheap, evenly timed) tickets gives the global offsets; it
// writes every window header.  The assembly kernel then reads its windows' row
// offsets from the headers and never waits on another CTA.
constexpr int kWrWin = 512;          // windows per ticket (two per thread)
template <int NBW>
__global__ void __launch_bounds__(kWbThreads)
k_wb_rows(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ table, const int64_t *__restrict__ pane_ts,
          WinHdr *__restrict__ hdr, uint64_t *__restrict__ status, int *__restrict__ ticket,
          int64_t *__restrict__ woffs, int nz) {
  hdr += st->hdr_base;
  __shared__ unsigned s_bm[kWrWin + 64][NBW];   // pane presence bitmaps (K <= 64)
  __shared__ int s_t;
  __shared__ int s_ws[8];
  __shared__ int64_t s_base;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  const int W = (int)p.slot_words, K = (int)p.K;
  const int64_t Rm = p.R - 1;
  const uint64_t epoch = (uint64_t)st->tile_epoch;
  const int64_t nitems = (J1 - J0 + kWrWin - 1) / kWrWin;
  constexpr int U = 8;                            // panes in flight per warp
  for (;;) {
    if (tid == 0) s_t = atomicAdd(ticket, 1);
    __syncthreads();
    const int64_t t = s_t;
    if (t >= nitems) break;
    const int64_t j0 = J0 + t * kWrWin;
    const int jn = (int)((J1 - j0) < kWrWin ? (J1 - j0) : kWrWin);
    const int npanes = jn + K - 1;                    // panes [j0, j0 + npanes) (one-pane slides)
    if (p.pane_bm) {                                  // the scan's presence bitmaps (8 u32 per pane)
      const uint32_t *bm = pane_bm_words(p, table);
      for (int i = tid; i < npanes * NBW; i += kWbThreads) {
        const int x = i / NBW, z = i - x * NBW;
        s_bm[x][z] = __ldcg(bm + ((j0 + x) & Rm) * 8 + z);
      }
    } else
    for (int x0 = warp * U; x0 < npanes; x0 += (kWbThreads / 32) * U) {
      int64_t v[U][NBW];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint64_t *cw = table + ((j0 + x0 + u) & Rm) * W + lane;
#pragma unroll
        for (int z = 0; z < NBW; ++z)
          v[u][z] = x0 + u < npanes ? (int64_t)__ldcg((const unsigned long long *)cw + z * 32) : 0;
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int z = 0; z < NBW; ++z) {
          const unsigned bal = __ballot_sync(kFull, v[u][z] > 0);
          if (lane == 0 && x0 + u < npanes) s_bm[x0 + u][z] = bal;
        }
    }
    __syncthreads();
    int n0 = 0, n1 = 0;
    int pc0[NBW], pc1[NBW];                             // rows per 32-key word (key slices)
    const int w0 = 2 * tid;
#pragma unroll
    for (int z = 0; z < NBW; ++z) {
      pc0[z] = pc1[z] = 0;
      if (w0 < jn) {
        unsigned m = 0;
        for (int k = 1; k < K; ++k) m |= s_bm[w0 + k][z];          // panes shared by both windows
        pc0[z] = __popc(m | s_bm[w0][z]);
        if (w0 + 1 < jn) pc1[z] = __popc(m | s_bm[w0 + K][z]);
      }
      n0 += pc0[z];
      n1 += pc1[z];
    }
    const int n = n0 + n1;
    // block exclusive scan of the row counts
    int y = n;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int zz = __shfl_up_sync(kFull, y, o);
      if (lane >= o) y += zz;
    }
    if (lane == 31) s_ws[warp] = y;
    __syncthreads();
    if (warp == 0) {
      int v = lane < kWbThreads / 32 ? s_ws[lane] : 0, u = v;
#pragma unroll
      for (int o = 1; o < 8; o <<= 1) {
        const int zz = __shfl_up_sync(kFull, u, o);
        if (lane >= o) u += zz;
      }
      const int total = __shfl_sync(kFull, u, kWbThreads / 32 - 1);
      if (lane < kWbThreads / 32) s_ws[lane] = u - v;
      const int64_t excl = lookback_warp(status, t, epoch, (uint64_t)total, st->row_base);
      if (lane == 0) {
        s_base = excl;
        if (t == nitems - 1) {
          st->sel_rows = excl + (int64_t)total;
          if (excl + (int64_t)total > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
        }
      }
    }
    __syncthreads();
    const int64_t off = s_base + s_ws[warp] + y - n;
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      if (w0 + e >= jn) break;
      const int64_t j = j0 + w0 + e;
      WinHdr h;
      h.window_id = j;
      h.ts = (p.win_kind == WK_TIME) ? p.T0 + j * p.l : pane_ts[j & Rm];
      h.row_offset = off + (e ? n0 : 0);
      h.nrows = e ? n1 : n0;
      h.flags = 0;
      hdr[j - J0] = h;
      if (nz > 1) {                                     // first row of every key slice of the window
        int64_t r = h.row_offset;
        const int wps = NBW / nz;                       // 32-key words per slice
#pragma unroll
        for (int z = 0; z < NBW; ++z) {
          if (z % wps == 0) woffs[(j - J0) * nz + z / wps] = r;
          r += e ? pc1[z] : pc0[z];
        }
      }
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------------------
// Register variant of the FAST plan for one-pane slides (L = 1) over C = 32..256
// dense keys (C3 at G = 64): an item is one K-aligned block of K window starts.
// Warp w owns key chunk kc = w mod C/32 (lane = key within the chunk) and window
// group g = w div C/32 (WPT = K/ng consecutive window starts, ng = 256/C groups).
// The same van Herk / Gil-Werman decomposition as above, done in registers:
//   V[i] = S[i] ⊕ P[i],  S[i] = ⊕ panes [bK+i, bK+K),  P[i] = ⊕ panes [(b+1)K, (b+1)K+i)
// each thread walks its WPT panes of block b backwards (local suffixes) and its
// WPT panes of block b+1 forwards (local prefixes); the group totals go through
// shared memory, S[i] = local suffix ⊕ totals of the later groups of block b,
// P[i] = totals of the earlier groups of block b+1 ⊕ local prefix.  Nothing is
// written back into the staged panes, so the next ticket's bulk copies are issued
// as soon as every thread has read them and overlap this item's presence ballots,
// look-back and row writes.  One ballot per (window, key chunk) gives the
// presence masks; a window's rows are its keys in order (prefix popcounts).
template <int NF, int CC, int WPT>
__global__ void __launch_bounds__(kWbThreads, 3)
k_win_block_reg(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ table,
                const int64_t *__restrict__ pane_ts, WinHdr *__restrict__ hdr, unsigned char *__restrict__ rows,
                uint64_t *__restrict__ status, int *__restrict__ ticket, int NB,
                const int64_t *__restrict__ woffs) {
  (void)NB; (void)status; (void)pane_ts;
  ticket += 1;                                // [0] is k_wb_rows' ticket
  hdr += st->hdr_base;
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ uint64_t bar;
  __shared__ int s_t, s_next;
  __shared__ unsigned s_mask[64][8];          // presence: [window of the block][key chunk]
  __shared__ int64_t s_woff[64];              // first row of each window (k_wb_rows)
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  // compile-time geometry: C = CC keys, ng = 256/C window groups of WPT windows, K = ng·WPT
  // (key slices: C = p.C > CC keys are processed CC at a time, NZ items per block)
  constexpr int C = CC, nkc = CC / 32, ng = kWbThreads / CC, K = ng * WPT, W = CC * (1 + NF);
  const int NZ = (int)(p.C / CC);
  const int64_t Rm = p.R - 1;
  const int kc = warp % nkc, g = warp / nkc;
  const int64_t bfirst = J0 / K;
  const int64_t nitems = ((J1 - 1) / K - bfirst + 1) * NZ;
  const int NP = 2 * K - 1;                   // staged panes per item
  uint64_t *raw = (uint64_t *)smem;           // [NP][W]
  uint64_t *tot = raw + (size_t)NP * W;       // [2][ng][W]: group totals of blocks b and b+1
  const int64_t qhi = J1 - 1 + K - 1;         // last pane read by the task's windows
  const unsigned lt = (1u << lane) - 1u;
  auto stage = [&](int64_t t) {               // thread 0: bulk copies of item t's panes
    const int64_t q0 = (bfirst + t / NZ) * K;
    const int64_t sa = q0 > J0 ? q0 : J0;
    const int64_t se = (q0 + NP) < (qhi + 1) ? (q0 + NP) : (qhi + 1);
    if (NZ > 1) {                             // slice z: CC words of the count and of each field,
      const int z = (int)(t % NZ);            // the (NF+1)·panes copies issued by the 32 lanes of warp 0
      if (lane == 0) mbar_expect_tx(&bar, (uint32_t)((se > sa ? se - sa : 0) * W * 8));
      __syncwarp();
      for (int64_t q = sa + lane; q < se; q += 32)
#pragma unroll
        for (int f = 0; f <= NF; ++f)
          bulk_g2s(raw + (q - q0) * W + f * CC, table + (q & Rm) * p.slot_words + f * p.C + z * CC,
                   (uint32_t)(CC * 8), &bar);
      return;
    }
    if (lane) return;
    uint32_t bytes = 0;
    for (int64_t q = sa; q < se;) {
      const int64_t run = ((q | Rm) + 1 - q) < (se - q) ? ((q | Rm) + 1 - q) : (se - q);
      bytes += (uint32_t)(run * W * 8);
      q += run;
    }
    mbar_expect_tx(&bar, bytes);
    for (int64_t q = sa; q < se;) {
      const int64_t run = ((q | Rm) + 1 - q) < (se - q) ? ((q | Rm) + 1 - q) : (se - q);
      for (int64_t d = 0; d < run;) {                      // <= 1 MiB per bulk copy
        const int64_t n = (run - d) * W * 8 <= (1 << 20) ? (run - d) : ((1 << 20) / (W * 8));
        bulk_g2s(raw + (q + d - q0) * W, table + ((q + d) & Rm) * W, (uint32_t)(n * W * 8), &bar);
        d += n;
      }
      q += run;
    }
  };
  if (tid == 0) {
    mbar_init(&bar, 1);
    fence_mbar_init();
    s_t = atomicAdd(ticket, 1);
  }
  __syncthreads();
  if (warp == 0 && s_t < nitems) stage(s_t);           // warp 0 issues the bulk copies
  uint32_t phase = 0;
  for (int64_t t = s_t; t < nitems; ) {
    const int64_t q0 = (bfirst + t / NZ) * K;
    const int z = (int)(t % NZ);
    const int key = z * CC + kc * 32 + lane;
    const int64_t ja = q0 > J0 ? q0 : J0;
    const int64_t jb = (q0 + K) < J1 ? (q0 + K) : J1;
    // row offsets of the item's windows (k_wb_rows: headers, or per (window, slice)), in
    // flight during the wait
    int64_t my_off = 0;
    if (tid < K && q0 + tid >= ja && q0 + tid < jb)
      my_off = NZ > 1 ? __ldcg((const long long *)&woffs[(q0 + tid - J0) * NZ + z])
                      : __ldcg((const long long *)&hdr[q0 + tid - J0].row_offset);
    mbar_wait(&bar, phase);
    phase ^= 1u;
    // ---- local suffixes over block b and local prefixes over block b+1
    const int i0 = g * WPT;
    int64_t c[WPT];
    double f[NF][WPT];
    {
      int64_t ac = 0;
      double af[NF];
#pragma unroll
      for (int x = 0; x < NF; ++x) af[x] = 0.0;
#pragma unroll
      for (int ii = WPT - 1; ii >= 0; --ii) {
        const uint64_t *r = raw + (i0 + ii) * W + (kc * 32 + lane);
        ac += (int64_t)r[0];
        c[ii] = ac;
#pragma unroll
        for (int x = 0; x < NF; ++x) {
          af[x] += __longlong_as_double((long long)r[(1 + x) * C]);
          f[x][ii] = af[x];
        }
      }
      uint64_t *tb = tot + g * W + (kc * 32 + lane);
      tb[0] = (uint64_t)ac;
#pragma unroll
      for (int x = 0; x < NF; ++x) tb[(1 + x) * C] = (uint64_t)__double_as_longlong(af[x]);
    }
    {
      int64_t ac = 0;
      double af[NF];
#pragma unroll
      for (int x = 0; x < NF; ++x) af[x] = 0.0;
#pragma unroll
      for (int ii = 0; ii < WPT; ++ii) {
        c[ii] += ac;                                        // local prefix: panes before i in the group
#pragma unroll
        for (int x = 0; x < NF; ++x) f[x][ii] += af[x];
        const int qi = K + i0 + ii;
        if (qi < NP) {
          const uint64_t *r = raw + qi * W + (kc * 32 + lane);
          ac += (int64_t)r[0];
#pragma unroll
          for (int x = 0; x < NF; ++x) af[x] += __longlong_as_double((long long)r[(1 + x) * C]);
        }
      }
      uint64_t *tb = tot + (ng + g) * W + (kc * 32 + lane);
      tb[0] = (uint64_t)ac;
#pragma unroll
      for (int x = 0; x < NF; ++x) tb[(1 + x) * C] = (uint64_t)__double_as_longlong(af[x]);
    }
    __syncthreads();
    // every thread has read its staged panes: the next ticket's copies go now
    if (warp == 0) {
      fence_proxy_async_smem();
      int nx = 0;
      if (lane == 0) s_next = nx = atomicAdd(ticket, 1);
      nx = __shfl_sync(kFull, nx, 0);
      if (nx < nitems) stage(nx);
    }
    // ---- window values: S[i] = local suffix ⊕ later groups of b, P[i] = earlier groups of b+1 ⊕ local prefix
    {
      int64_t tc = 0;
      double tf[NF];
#pragma unroll
      for (int x = 0; x < NF; ++x) tf[x] = 0.0;
      for (int h = g + 1; h < ng; ++h) {
        const uint64_t *tb = tot + h * W + (kc * 32 + lane);
        tc += (int64_t)tb[0];
#pragma unroll
        for (int x = 0; x < NF; ++x) tf[x] += __longlong_as_double((long long)tb[(1 + x) * C]);
      }
      for (int h = 0; h < g; ++h) {
        const uint64_t *tb = tot + (ng + h) * W + (kc * 32 + lane);
        tc += (int64_t)tb[0];
#pragma unroll
        for (int x = 0; x < NF; ++x) tf[x] += __longlong_as_double((long long)tb[(1 + x) * C]);
      }
#pragma unroll
      for (int ii = 0; ii < WPT; ++ii) {
        c[ii] += tc;
#pragma unroll
        for (int x = 0; x < NF; ++x) f[x][ii] += tf[x];
      }
    }
    // ---- presence (no HAVING on the FAST plan: count > 0) of the item's windows
    unsigned pres = 0;
#pragma unroll
    for (int ii = 0; ii < WPT; ++ii) {
      const int64_t j = q0 + i0 + ii;
      const bool pr = j >= ja && j < jb && c[ii] > 0;
      pres |= (unsigned)pr << ii;
      const unsigned bal = __ballot_sync(kFull, pr);
      if (lane == 0) s_mask[i0 + ii][kc] = bal;
    }
    if (tid < K) s_woff[tid] = my_off;
    __syncthreads();
#pragma unroll
    for (int ii = 0; ii < WPT; ++ii) {
      if (!((pres >> ii) & 1u)) continue;
      const int i = i0 + ii;
      int before = 0;
#pragma unroll
      for (int z = 0; z < nkc - 1; ++z) before += z < kc ? __popc(s_mask[i][z]) : 0;
      const int64_t row = s_woff[i] + before + __popc(s_mask[i][kc] & lt);
      if (row >= p.rows_cap) continue;
      if (p.nkeys) ((int32_t *)(rows + p.col_off[0]))[row] = key;
#pragma unroll
      for (int a = 0; a < kMaxAgg; ++a) {
        if (a >= p.nagg) break;
        const AggOut &o = p.agg[a];
        double x = 0.0;
#pragma unroll
        for (int y = 0; y < NF; ++y)
          if (y == o.field) x = f[y][ii];
        uint64_t bits = o.fn == AG_COUNT ? (uint64_t)c[ii] : (uint64_t)__double_as_longlong(x);
        if (o.fn == AG_AVG) bits = (uint64_t)__double_as_longlong(wb_div(x, (double)c[ii]));
        ((uint64_t *)(rows + p.col_off[p.nkeys + a]))[row] = bits;
      }
    }
    __syncthreads();
    t = s_next;
  }
}

// ---------------------------------------------------------------------------
// host side: usable when an item's staged panes + window values fit in shared
// memory and its windows / rounds fit the per-item arrays
static int wb_nb(const Plan &p) {
  int nb = (int)((32 * p.L + p.K - 1) / p.K);     // about 32 windows per item
  return nb < 1 ? 1 : nb;
}
static bool wb_fast(const Plan &p) {
  if (p.nhave || p.has_minmax || p.nf > 2 || p.key_mode == KM_HASH) return false;
  if (p.nkeys > 1 || (p.nkeys == 1 && (p.key_pack != KP_RADIX || p.col_bytes[0] != 4))) return false;
  if (p.C & (p.C - 1)) return false;
  for (int a = 0; a < p.nagg; ++a)
    if (p.agg[a].fn != AG_COUNT && p.agg[a].fn != AG_SUM && p.agg[a].fn != AG_AVG) return false;
  return !std::getenv("SABER_NO_WBFAST");
}
// register variant: FAST plan, one-pane slides, 32..256 dense keys (power of two),
// fp64 sums only, K a multiple of the 256/C window groups with <= 16 windows per thread
// keys per item: all C, or slices of 64 (C = 128 / 256 when the whole table's
// windows would need more than 16 per thread, C3 G=256: K = 32)
static int64_t wbr_cc(const Plan &p) {
  if (!wb_fast(p) || p.L != 1 || p.key_mode == KM_HASH || p.C < 32 || p.C > 256 || (p.C & (p.C - 1))) return 0;
  if (p.slot_words != p.C * (1 + p.nf) || p.nf < 1 || std::getenv("SABER_NO_WBREG")) return 0;
  for (int f = 0; f < p.nf; ++f)
    if (p.field[f].kind != FK_SUM_F) return 0;
  if (p.K > 64) return 0;
  auto ok = [&](int64_t cc) { const int64_t ng = kWbThreads / cc, w = p.K / ng;
                              return p.K % ng == 0 && (w == 4 || w == 8 || w == 16); };
  if (ok(p.C)) return p.C;
  if (p.C > 64 && ok(64) && !std::getenv("SABER_NO_WBSLICE")) return 64;
  return 0;
}
static int wbr_wpt(const Plan &p) {
  const int64_t cc = wbr_cc(p);
  return cc ? (int)(p.K / (kWbThreads / cc)) : 0;
}
static int wbr_smem(const Plan &p) {
  const int64_t cc = wbr_cc(p);
  return (int)(((2 * p.K - 1) + 2 * (kWbThreads / cc)) * cc * (1 + p.nf) * 8);
}
int wb_smem(const Plan &p) {
  if (wbr_wpt(p)) return wbr_smem(p);
  const int nb = wb_nb(p);
  return (int)(((nb + 1) * p.K - 1 + (nb == 1 ? 0 : nb * p.K)) * p.slot_words * 8);
}
bool wb_usable(const Plan &p) {
  if (p.key_mode == KM_HASH || p.nagg == 0 || p.K > 64 || (p.slot_words & 1)) return false;   // 16-B bulk copies
  if (wbr_wpt(p)) return wbr_smem(p) <= 100 * 1024;
  const int nb = wb_nb(p);
  // the van Herk phase runs one thread per (block, word) and direction: too few
  // words leave the CTA idle (C4's 4 keys), those plans keep k_vh_build + k_win_packed
  if ((nb == 1 ? 2 * p.slot_words : nb * p.slot_words) < 64) return false;
  const int64_t nwin = (nb * p.K + p.L - 1) / p.L + 1;
  if (nwin > kWbMaxWin || (nwin * p.C + kWbThreads - 1) / kWbThreads > kWbMaxRounds) return false;
  if (p.slot_words > kWbMaxWords) return false;
  return wb_smem(p) <= 96 * 1024;
}
template <int NF, int CC>
static void *wbr_kernel(int wpt) {
  return wpt == 4 ? (void *)k_win_block_reg<NF, CC, 4> : wpt == 8 ? (void *)k_win_block_reg<NF, CC, 8>
                                                                  : (void *)k_win_block_reg<NF, CC, 16>;
}
template <int NF>
static void *wbr_kernel_c(int c, int wpt) {
  return c == 32 ? wbr_kernel<NF, 32>(wpt) : c == 64 ? wbr_kernel<NF, 64>(wpt) : c == 128 ? wbr_kernel<NF, 128>(wpt)
                                                                                 : wbr_kernel<NF, 256>(wpt);
}
static void *wb_kernel(const Plan &p) {
  if (const int wpt = wbr_wpt(p)) {
    const int cc = (int)wbr_cc(p);
    return p.nf == 1 ? wbr_kernel_c<1>(cc, wpt) : wbr_kernel_c<2>(cc, wpt);
  }
  if (wb_fast(p)) return p.nf <= 1 ? (void *)k_win_block<1, true> : (void *)k_win_block<2, true>;
  return p.nf <= 1 ? (void *)k_win_block<1, false> : p.nf <= 2 ? (void *)k_win_block<2, false>
       : p.nf <= 4 ? (void *)k_win_block<4, false> : (void *)k_win_block<8, false>;
}
cudaError_t wb_set_attributes(const Plan &p) {
  return cudaFuncSetAttribute(wb_kernel(p), cudaFuncAttributeMaxDynamicSharedMemorySize, wb_smem(p));
}
int wb_blocks_per_sm(const Plan &p) {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, wb_kernel(p), kWbThreads, wb_smem(p));
  return b > 0 ? b : 1;
}
bool wb_prepass(const Plan &p) { return wbr_wpt(p) != 0; }
cudaError_t launch_windows_block(const Plan &p, const QueryDev &q, const SlotDev &s, int grid, cudaStream_t st) {
  const int nb = wb_nb(p);
  int64_t *woffs = s.counts;
  if (wbr_wpt(p)) {     // row counts, offsets and headers first (k_wb_rows), then the values
    void (*k)(const Plan, State *, const uint64_t *, const int64_t *, WinHdr *, uint64_t *, int *, int64_t *, int) =
        p.C <= 32 ? k_wb_rows<1> : p.C <= 64 ? k_wb_rows<2> : p.C <= 128 ? k_wb_rows<4> : k_wb_rows<8>;
    const int nz = (int)(p.C / wbr_cc(p));
    k<<<grid, kWbThreads, 0, st>>>(p, q.st, q.table, q.pane_ts, (WinHdr *)s.hdr, q.tile_status, q.tile_ctr, woffs, nz);
  }
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&q.table, (void *)&q.pane_ts, (void *)&s.hdr, (void *)&s.rows,
                  (void *)&q.tile_status, (void *)&q.tile_ctr, (void *)&nb, (void *)&woffs};
  return cudaLaunchKernel(wb_kernel(p), dim3(grid), dim3(kWbThreads), args, (size_t)wb_smem(p), st);
}

}  // namespace sb
