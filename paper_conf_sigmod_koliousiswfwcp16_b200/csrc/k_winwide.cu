// k_winwide.cu -- window assembly for dense key domains with many keys
// (256 < C <= 2048 table entries, van Herk arrays built by k_vh_build*): C5a's
// 2,048 (plug, household, house) groups, C5b's 1,600 (highway, direction,
// segment) groups.
//
// The batch operator f_b (§3) of window j is, per key,
//   V[j] = S[a] ⊕ P[a+K-1]   (a = j·L; V[j] = S[a] when a ≡ 0 mod K)
// from the block-suffix / block-prefix arrays (van Herk / Gil-Werman).  A CTA
// takes one window per ticket: thread t owns keys r·256 + t (r < RR), keeps
// their combined (count, fields) in registers, HAVING (L1291-1292) decides the
// present rows, one ballot per (round, warp) gives every row's offset inside the
// window, and the window's output offset comes from decoupled look-back over
// the earlier windows of the task (tile = window).  Rows are written in key
// order, lane-consecutive (coalesced column stores), read once; k_win_fused
// instead ran a count pass and an emit pass over the same S/P words and wrote
// each thread's rows as a contiguous run (8-row stride across a warp).
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>

#include "common.cuh"
#include "launch_internal.h"

namespace sb {

constexpr int kWwThreads = 256;

template <int NF, int RR, bool PRE>
__global__ void __launch_bounds__(kWwThreads)
k_win_wide(const Plan p, State *__restrict__ st, const uint64_t *__restrict__ pre, const uint64_t *__restrict__ suf,
           const int64_t *__restrict__ pane_ts, WinHdr *__restrict__ hdr, unsigned char *__restrict__ rows,
           uint64_t *__restrict__ status, int *__restrict__ ticket, int ktab, const int64_t *__restrict__ offs) {
  hdr += st->hdr_base;                         // windows earlier rounds of the task wrote
  extern __shared__ __align__(16) int32_t s_keys[];           // ktab: decoded key columns [nkeys][C]
  __shared__ int s_cnt[RR * 8];                              // rows per (round, warp) -> exclusive offsets
  __shared__ int64_t s_base;
  __shared__ int s_t;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned lt = (1u << lane) - 1u;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const uint64_t epoch = (uint64_t)st->tile_epoch;
  const int C = (int)p.C;
  const int64_t W = p.slot_words, Rm = p.R - 1, K = p.K, L = p.L;
  if (ktab) {
    for (int s = tid; s < C; s += kWwThreads) {
      int64_t kv[kMaxKey];
      decode_key(p, (uint64_t)s, kv);
      FOR_K(i) s_keys[i * C + s] = (int32_t)kv[i];
    }
  }
  int kinds[NF];
#pragma unroll
  for (int f = 0; f < NF; ++f) kinds[f] = f < p.nf ? p.field[f].kind : FK_SUM_I;
  for (int64_t t0 = blockIdx.x;; t0 += gridDim.x) {
    if (!PRE && tid == 0) s_t = atomicAdd(ticket, 1);
    __syncthreads();
    const int64_t t = PRE ? t0 : (int64_t)s_t;
    if (t >= nw) break;
    const int64_t j = J0 + t, a = j * L;
    const bool aligned = (a % K) == 0;
    const uint64_t *sa = suf + (a & Rm) * W;
    const uint64_t *pb = pre + ((a + K - 1) & Rm) * W;
    int64_t c[RR];
    uint64_t fv[RR][NF];
    unsigned bal[RR];
    // all loads of the window first (RR·(1+NF)·2 independent 8-byte loads per thread)
    uint64_t xs[RR][1 + NF], xp[RR][1 + NF];
#pragma unroll
    for (int r = 0; r < RR; ++r) {
      const int s = r * kWwThreads + tid;
      const bool in = s < C;
#pragma unroll
      for (int f = 0; f <= NF; ++f) {
        const bool use = in && (f == 0 || f <= p.nf);
        xs[r][f] = use ? __ldg(&sa[(int64_t)f * C + s]) : 0ull;
        xp[r][f] = (use && !aligned) ? __ldg(&pb[(int64_t)f * C + s]) : 0ull;
      }
    }
#pragma unroll
    for (int r = 0; r < RR; ++r) {
      bool pres = false;
      c[r] = (int64_t)xs[r][0] + (int64_t)xp[r][0];
#pragma unroll
      for (int f = 0; f < NF; ++f)
        fv[r][f] = aligned ? xs[r][1 + f] : field_combine(kinds[f], xs[r][1 + f], xp[r][1 + f]);
      if (c[r] > 0) {
        uint64_t fa[kMaxField];
#pragma unroll
        for (int f = 0; f < kMaxField; ++f) fa[f] = f < NF ? fv[r][f] : 0;
        pres = !p.nhave || having_ok(p, c[r], fa);
      }
      bal[r] = __ballot_sync(kFull, pres);
    }
    if (lane == 0) {
#pragma unroll
      for (int r = 0; r < RR; ++r) s_cnt[r * 8 + warp] = __popc(bal[r]);
    }
    __syncthreads();
    if (warp == 0) {
      // exclusive scan of the RR·8 (round, warp) counts = key order
      int run = 0;
#pragma unroll
      for (int b = 0; b < RR * 8; b += 32) {
        const int v = b + lane < RR * 8 ? s_cnt[b + lane] : 0;
        int x = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(kFull, x, o);
          if (lane >= o) x += y;
        }
        if (b + lane < RR * 8) s_cnt[b + lane] = run + x - v;
        run += __shfl_sync(kFull, x, 31);
      }
      const uint64_t total = (uint64_t)run;
      if (PRE) {                           // offsets from k_win_wide_count + k_win_scan (headers too)
        if (lane == 0) s_base = offs[t];
      } else {
      const int64_t excl = lookback_warp(status, t, epoch, total, st->row_base);
      if (lane == 0) {
        s_base = excl;
        WinHdr h;
        h.window_id = j;
        h.ts = (p.win_kind == WK_TIME) ? p.T0 + j * p.l : pane_ts[(j * L) & Rm];
        h.row_offset = excl;
        h.nrows = (int32_t)total;
        h.flags = 0;
        hdr[t] = h;
        if (t == nw - 1) {
          st->sel_rows = excl + (int64_t)total;
          if (excl + (int64_t)total > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
        }
      }
      }
    }
    __syncthreads();
    const int64_t base = s_base;
#pragma unroll
    for (int r = 0; r < RR; ++r) {
      if ((bal[r] >> lane) & 1u) {
        const int s = r * kWwThreads + tid;
        int64_t kv[kMaxKey];
        if (ktab) {
          FOR_K(i) kv[i] = s_keys[i * C + s];
        } else {
          decode_key(p, (uint64_t)s, kv);
        }
        uint64_t fa[kMaxField];
#pragma unroll
        for (int f = 0; f < kMaxField; ++f) fa[f] = f < NF ? fv[r][f] : 0;
        write_row(p, rows, base + s_cnt[r * 8 + warp] + __popc(bal[r] & lt), kv, c[r], fa);
      }
    }
  }
}

// Row counts per window (keys with count > 0 that pass HAVING) for the
// look-back-free variant: k_win_scan turns them into offsets + headers, then
// k_win_wide<.., PRE = true> writes every window independently (grid stride).
template <int NF, int RR>
__global__ void __launch_bounds__(kWwThreads)
k_win_wide_count(const Plan p, const State *__restrict__ st, const uint64_t *__restrict__ pre,
                 const uint64_t *__restrict__ suf, int64_t *__restrict__ counts) {
  __shared__ int s_w[8];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  const int C = (int)p.C;
  const int64_t W = p.slot_words, Rm = p.R - 1, K = p.K, L = p.L;
  int kinds[NF];
#pragma unroll
  for (int f = 0; f < NF; ++f) kinds[f] = f < p.nf ? p.field[f].kind : FK_SUM_I;
  for (int64_t t = blockIdx.x; t < nw; t += gridDim.x) {
    const int64_t a = (J0 + t) * L;
    const bool aligned = (a % K) == 0;
    const uint64_t *sa = suf + (a & Rm) * W;
    const uint64_t *pb = pre + ((a + K - 1) & Rm) * W;
    int n = 0;
#pragma unroll
    for (int r = 0; r < RR; ++r) {
      const int s = r * kWwThreads + tid;
      if (s >= C) continue;
      const int64_t c = (int64_t)__ldg(&sa[s]) + (aligned ? 0 : (int64_t)__ldg(&pb[s]));
      bool pres = c > 0;
      if (pres && p.nhave) {
        uint64_t fa[kMaxField];
#pragma unroll
        for (int f = 0; f < kMaxField; ++f) fa[f] = 0;
#pragma unroll
        for (int f = 0; f < NF; ++f) {
          if (f < p.nf) {
            const uint64_t x = __ldg(&sa[(int64_t)(1 + f) * C + s]);
            fa[f] = aligned ? x : field_combine(kinds[f], x, __ldg(&pb[(int64_t)(1 + f) * C + s]));
          }
        }
        pres = having_ok(p, c, fa);
      }
      n += pres;
    }
    n = __reduce_add_sync(kFull, (unsigned)n);
    if (lane == 0) s_w[warp] = n;
    __syncthreads();
    if (tid == 0) {
      int tot = 0;
#pragma unroll
      for (int w = 0; w < 8; ++w) tot += s_w[w];
      counts[t] = tot;
    }
    __syncthreads();
  }
}

// ---------------------------------------------------------------------------
template <int NF, bool PRE>
static void *ww_rr(int rr) {
  return rr <= 2 ? (void *)k_win_wide<NF, 2, PRE> : rr <= 4 ? (void *)k_win_wide<NF, 4, PRE>
                                                             : (void *)k_win_wide<NF, 8, PRE>;
}
template <int NF>
static void *wc_rr(int rr) {
  return rr <= 2 ? (void *)k_win_wide_count<NF, 2> : rr <= 4 ? (void *)k_win_wide_count<NF, 4>
                                                             : (void *)k_win_wide_count<NF, 8>;
}
// Plans without HAVING count rows from the count words alone (half the window's
// words): count + scan + independent emission beats the per-window look-back
// (C5a 8.85 -> 8.38 ms); with HAVING the count pass re-reads every field and the
// look-back kernel stays (C5b 5.83 vs 5.89 ms).
static bool ww_pre(const Plan &p) {
  const char *v = std::getenv("SABER_WW_LOOKBACK");    // 1: always the single look-back kernel
  return !(v && *v == '1') && p.nhave == 0;
}
static void *ww_kernel(const Plan &p) {
  const int rr = (int)((p.C + kWwThreads - 1) / kWwThreads);
  if (ww_pre(p)) return p.nf <= 1 ? ww_rr<1, true>(rr) : ww_rr<2, true>(rr);
  return p.nf <= 1 ? ww_rr<1, false>(rr) : ww_rr<2, false>(rr);
}
static void *wc_kernel(const Plan &p) {
  const int rr = (int)((p.C + kWwThreads - 1) / kWwThreads);
  return p.nf <= 1 ? wc_rr<1>(rr) : wc_rr<2>(rr);
}
bool ww_usable(const Plan &p) {
  return p.key_mode != KM_HASH && p.C > 256 && p.C <= 8 * kWwThreads && p.nf <= 2 && !p.slab_mode &&
         !p.bucket_mode;
}
static int ww_smem(const Plan &p) {
  const int64_t b = p.nkeys > 1 ? p.nkeys * p.C * 4 : 0;
  return b <= 48 * 1024 ? (int)b : 0;
}
cudaError_t ww_set_attributes(const Plan &p) {
  return cudaFuncSetAttribute(ww_kernel(p), cudaFuncAttributeMaxDynamicSharedMemorySize, ww_smem(p));
}
int ww_blocks_per_sm(const Plan &p) {
  int b = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, ww_kernel(p), kWwThreads, ww_smem(p));
  return b > 0 ? b : 1;
}
cudaError_t launch_windows_wide(const Plan &p, const QueryDev &q, const SlotDev &s, int grid, cudaStream_t st) {
  int ktab = ww_smem(p) > 0 ? 1 : 0;
  const int64_t *offs = s.counts;
  if (ww_pre(p)) {
    int b = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, wc_kernel(p), kWwThreads, 0);
    void *cargs[] = {(void *)&p, (void *)&q.st, (void *)&q.vh_pre, (void *)&q.vh_suf, (void *)&s.counts};
    cudaError_t e = cudaLaunchKernel(wc_kernel(p), dim3((b > 0 ? b : 1) * 148), dim3(kWwThreads), cargs, 0, st);
    if (e) return e;
    if ((e = launch_win_scan(p, q, s, st))) return e;     // offsets + headers + sel_rows
  }
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&q.vh_pre, (void *)&q.vh_suf, (void *)&q.pane_ts,
                  (void *)&s.hdr, (void *)&s.rows, (void *)&q.tile_status, (void *)&q.tile_ctr, (void *)&ktab,
                  (void *)&offs};
  return cudaLaunchKernel(ww_kernel(p), dim3(grid), dim3(kWwThreads), args, (size_t)ww_smem(p), st);
}

}  // namespace sb
