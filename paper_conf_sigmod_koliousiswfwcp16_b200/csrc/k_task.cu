// k_task.cu -- scalar task prologue/epilogue, pane-ring initialisation, window headers, IStream carry, partition planning.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "launch_internal.h"

namespace sb {

__global__ void k_task_begin(const Plan p, State *st, const unsigned char *tup, int64_t n, int final_,
                             int has_wm, int64_t wm, int emit_on_finish, SlotMeta *meta,
                             const unsigned char *carry0, const unsigned char *carry1, int *tile_ctr,
                             int64_t *win_ts, int64_t ts_mask, int round) {
  const int lane = threadIdx.x;
  __shared__ int64_t sh[8];
  // ---- rounds (time-window aggregation, Plan::rounds > 1): this round takes the
  // longest unconsumed prefix of the task whose panes fit the ring next to the
  // panes of windows not yet emitted (J0·L ..).  If not even the next tuple fits
  // (a time gap wider than the ring), the round consumes nothing and only closes
  // the windows that tuple's arrival closes (their end <= its τ, reading A3):
  // the gap's windows are emitted -- empty ones with a header (A6) -- and the
  // ring moves past the gap for the next round
  int64_t off = 0, nn = n, closeB = INT64_MIN;
  bool short_rounds = false;
  if (p.rounds > 1) {
    if (lane == 0) {
      sh[0] = round == 0 ? 0 : st->round_off + st->round_n;
      sh[1] = st->J0;
    }
    __syncwarp();
    off = sh[0];
    const int64_t rem = n - off;
    nn = 0;
    if (rem > 0) {
      const int64_t pmax = sh[1] * p.L + p.R - 1;                 // last pane the ring can hold
      const int64_t tbeyond = p.T0 + (pmax + 1) * p.g;            // first τ past it
      const unsigned char *tr = tup + off * p.tuple_bytes;
      nn = warp_lower_bound(p, tr, rem, tr, 0, tbeyond);
      if (nn < rem) closeB = tau_at(p, tr, nn);          // the next tuple of the task has arrived
      short_rounds = round == p.rounds - 1 && nn < rem;
    }
    __syncwarp();
    tup += off * p.tuple_bytes;
    n = nn;
  }
  if (lane == 0) {
    int err = short_rounds ? ERR_CAPACITY : 0;
    const int64_t pos0 = st->pos_next;
    st->task_pos = pos0;
    st->task_n = n;
    st->round_off = off;
    st->round_n = n;
    int64_t J0 = st->J0, J1 = J0;
    // result slot bases: the first round opens the slot, later ones append
    if (round == 0) { st->slot_J0 = J0; st->row_base = 0; }
    else st->row_base = st->sel_rows;
    st->hdr_base = J0 - st->slot_J0;
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
      else if (closeB != INT64_MIN) B = closeB;                 // rounds: close by the next tuple's arrival
      else { B = st->tau_last; haveB = st->has_tau; }
      if (haveB && B - p.T0 - p.s >= 0) J1 = (B - p.T0 - p.s) / p.l + 1;
    } else {
      int64_t total = pos0 + n;   // count: W_j = [j·l, j·l+s) closes with position j·l+s-1
      if (total >= p.s) J1 = (total - p.s) / p.l + 1;
      if (n > 0) { plo = pos0 / p.g; phi = (total - 1) / p.g; }
    }
    if (J1 < J0) J1 = J0;
    st->pos_next = pos0 + n;
    if (phi > st->pane_hi) st->pane_hi = phi;
    // time windows that start after the last pane holding data (a time gap, or a
    // watermark past the data) are empty: they get headers only (reading A6,
    // k_gap_hdr) and no pane of theirs is read, so a gap never has to fit the ring
    int64_t Jn = J1;
    st->jgap_hi = 0;
    if (p.win_kind == WK_TIME && p.nagg > 0) {
      const int64_t Jd = st->pane_hi >= 0 ? st->pane_hi / p.L + 1 : 0;
      if (J1 > Jd) {
        Jn = Jd > J0 ? Jd : J0;
        st->jgap_hi = J1;
      }
    }
    st->J1 = Jn;
    // pane ring: slots of panes [J0·L, phi] and of the windows closed now must
    // coexist during this task (from the previous task's J0 when its window phase
    // may still be running)
    int64_t live_lo = (p.overlap ? st->live_J0 : J0) * p.L;
    int64_t zlo = st->zeroed_hi > live_lo ? st->zeroed_hi : live_lo;
    int64_t zhi = zlo;
    int64_t need_hi = phi;
    if (Jn > J0 && (Jn - 1) * p.L + p.K - 1 > need_hi) need_hi = (Jn - 1) * p.L + p.K - 1;
    if (need_hi >= 0 && p.nagg > 0) {
      if (need_hi - live_lo + 1 > p.R) err |= ERR_CAPACITY;
      else if (need_hi + 1 > zlo) zhi = need_hi + 1;
    }
    st->zero_lo = zlo;
    st->zero_hi = zhi;
    if (zhi > st->zeroed_hi) st->zeroed_hi = zhi;
    // the task's input tuples and the panes they span, over all its rounds (the
    // host picks the next tasks' table layout from them)
    const int64_t inp = (n > 0 && phi >= plo) ? phi - plo + 1 : 0;
    if (round == 0) { meta->in_tuples = n; meta->in_panes = inp; }
    else { meta->in_tuples += n; meta->in_panes += inp; }
    const int64_t Jend = st->jgap_hi > Jn ? st->jgap_hi : Jn;
    if (Jend - st->slot_J0 > p.win_cap) {
      // more windows than the slot's headers hold: a sticky error, and nothing is
      // written past the slot
      err |= ERR_RESULT;
      st->J1 = J0;
      st->jgap_hi = 0;
    }
    meta->first_window = st->slot_J0;
    meta->nwindows = st->J1 - st->slot_J0;
    if (err) st->error |= err;
    st->tile_epoch += 1;
    st->sel_rows = st->row_base;
    tile_ctr[0] = 0;
    tile_ctr[1] = 0;
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
  // IStream count windows: header ts = τ at position j·l (reading A7); k_select
  // records it for covered positions, the first task also for the positions of
  // its first windows before its cover (a partition's halo, first_window > 0)
  if (p.win_kind == WK_COUNT && st->first_task && n > 0) {
    const int64_t cend = cover_lo < pos0 + n ? cover_lo : pos0 + n;
    for (int64_t jj = (pos0 + p.l - 1) / p.l + lane; jj * p.l < cend; jj += 32)
      win_ts[jj & ts_mask] = tau_at(p, tup, jj * p.l - pos0);
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
// initialise the pane slots [zero_lo, zero_hi) of the ring: one CTA per slot at a
// time, one contiguous segment (hash keys, counts, each field) after the other,
// so no per-word division decides the identity value
__global__ void __launch_bounds__(256) k_zero_panes(const Plan p, const State *st, uint64_t *table, int sgrid,
                                                    int64_t sper) {
  const int64_t lo = st->zero_lo, hi = st->zero_hi;
  if (hi <= lo) return;
  const int64_t W = p.slot_words;
  if (sper > 0) {
    // the scan (k_pane_cnt) initialises every pane wholly inside one CTA's tuples;
    // here only the panes holding a CTA boundary b_c = task_pos + min(c·per, n),
    // c = 0..sgrid (the task's ends included): floor((b_c-1)/g) and floor(b_c/g)
    const int64_t pos = st->task_pos, n = st->task_n;
    for (int64_t x = blockIdx.x; x < 2 * ((int64_t)sgrid + 1); x += gridDim.x) {
      const int64_t c = x >> 1;
      const int64_t b = pos + (c * sper < n ? c * sper : n) - (x & 1);
      if (b < 0) continue;
      const int64_t pane = b / p.g;
      if (pane < lo || pane >= hi) continue;
      const int64_t slot = pane & (p.R - 1);
      for (int64_t w = threadIdx.x; w < W; w += blockDim.x) table[slot * W + w] = 0;
      if (p.pane_bm && threadIdx.x < 8) pane_bm_words(p, table)[slot * 8 + threadIdx.x] = 0;
    }
    return;
  }
  if (p.pane_bm) {                                   // presence bitmaps of the new panes
    uint32_t *bm = pane_bm_words(p, table);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (hi - lo) * 8;
         i += (int64_t)gridDim.x * blockDim.x)
      bm[((lo + (i >> 3)) & (p.R - 1)) * 8 + (i & 7)] = 0;
  }
  bool flat = p.bucket_mode || (p.key_mode != KM_HASH && !p.has_minmax);
  if (flat && (W & 1) == 0) {
    // every word's identity is 0: 16-byte stores over the ring-contiguous runs
    const int64_t Rm = p.R - 1;
    const int64_t s0 = lo & Rm, n = hi - lo;
    const int64_t n1 = (s0 + n <= p.R) ? n : p.R - s0;         // panes before the ring wrap
    uint4 *d1 = (uint4 *)(table + s0 * W), *d2 = (uint4 *)table;
    const int64_t v1 = n1 * W / 2, v2 = (n - n1) * W / 2;
    const uint4 z = make_uint4(0, 0, 0, 0);
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < v1 + v2; i += (int64_t)gridDim.x * blockDim.x) {
      if (i < v1) d1[i] = z; else d2[i - v1] = z;
    }
    return;
  }
  for (int64_t pane = lo + blockIdx.x; pane < hi; pane += gridDim.x) {
    uint64_t *slot = table + (pane & (p.R - 1)) * W;
    if (p.bucket_mode) {
      for (int64_t w = threadIdx.x; w < W; w += blockDim.x) slot[w] = 0;
      continue;
    }
    const int64_t co = cnt_off(p);
    for (int64_t w = threadIdx.x; w < co; w += blockDim.x) slot[w] = kEmpty;          // hash keys
    for (int64_t w = threadIdx.x; w < p.C; w += blockDim.x) slot[co + w] = 0;         // counts
    for (int f = 0; f < p.nf; ++f) {
      const uint64_t v = field_identity(p.field[f].kind);
      uint64_t *d = slot + fld_off(p, f);
      for (int64_t w = threadIdx.x; w < p.C; w += blockDim.x) d[w] = v;
    }
  }
}

// Window headers and row offsets of a task from its per-(window, slab) row
// counts (HASH / slab / bucket modes): tiles of kScanTW windows take tickets,
// scan their counts in the CTA, get the tile's base by decoupled look-back over
// earlier tiles (st->tile_epoch keeps stale status words of earlier tasks out),
// then rewrite counts as exclusive row offsets and write the headers.
constexpr int kScanThreads = 256, kScanPer = 4, kScanTW = kScanThreads * kScanPer;

__global__ void __launch_bounds__(kScanThreads)
k_win_scan(const Plan p, State *st, const int64_t *__restrict__ pane_ts, int64_t *__restrict__ counts,
           WinHdr *__restrict__ hdr, SlotMeta *meta, uint64_t *__restrict__ status, int *__restrict__ ticket) {
  hdr += st->hdr_base;                         // windows earlier rounds of the task wrote
  __shared__ int64_t wsum[kScanThreads / 32];
  __shared__ int64_t s_base;
  __shared__ int s_t;
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  const uint64_t epoch = (uint64_t)st->tile_epoch;
  const int S = p.S;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t ntiles = (nw + kScanTW - 1) / kScanTW;
  if (nw <= 0) {
    if (blockIdx.x == 0 && tid == 0) { meta->nrows = st->row_base; st->sel_rows = st->row_base; }
    return;
  }
  for (;;) {
    if (tid == 0) s_t = atomicAdd(ticket, 1);
    __syncthreads();
    const int64_t t = s_t;
    if (t >= ntiles) break;
    const int64_t a = t * kScanTW + (int64_t)tid * kScanPer;
    int64_t wt[kScanPer];
    int64_t local = 0;
#pragma unroll
    for (int k = 0; k < kScanPer; ++k) {
      wt[k] = 0;
      if (a + k < nw)
        for (int s = 0; s < S; ++s) wt[k] += counts[(a + k) * S + s];
      local += wt[k];
    }
    int64_t x = local;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t y = (int64_t)__shfl_up_sync(kFull, (unsigned long long)x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) wsum[wid] = x;
    __syncthreads();
    if (wid == 0) {
      const int64_t w = lane < kScanThreads / 32 ? wsum[lane] : 0;
      int64_t y = w;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t z = (int64_t)__shfl_up_sync(kFull, (unsigned long long)y, o);
        if (lane >= o) y += z;
      }
      if (lane < kScanThreads / 32) wsum[lane] = y - w;
      const uint64_t total = (uint64_t)__shfl_sync(kFull, (unsigned long long)y, 31);   // the tile total
      const int64_t excl = lookback_warp(status, t, epoch, total, st->row_base);
      if (lane == 31) {
        s_base = excl;
        if (t == ntiles - 1) {
          const int64_t rows = excl + (int64_t)total;
          meta->nrows = rows;
          st->sel_rows = rows;
          if (rows > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
        }
      }
    }
    __syncthreads();
    int64_t run = s_base + wsum[wid] + x - local;
#pragma unroll
    for (int k = 0; k < kScanPer; ++k) {
      const int64_t j = a + k;
      if (j >= nw) break;
      WinHdr h;
      h.window_id = J0 + j;
      h.ts = (p.win_kind == WK_TIME) ? p.T0 + (J0 + j) * p.l : pane_ts[((J0 + j) * p.L) & (p.R - 1)];
      h.row_offset = run;
      h.nrows = (int32_t)wt[k];
      h.flags = 0;
      hdr[j] = h;
      for (int s = 0; s < S; ++s) {
        const int64_t c = counts[j * S + s];
        counts[j * S + s] = run;
        run += c;
      }
    }
    __syncthreads();
  }
}

__global__ void k_task_end(const Plan p, State *st, SlotMeta *meta) {
  if (threadIdx.x) return;
  meta->first_window = st->slot_J0;
  meta->nwindows = st->J1 - st->slot_J0;
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
    if (!p.overlap) meta->nrows = st->sel_rows;     // written by the window pass (fused) or k_win_scan
    meta->ntuples = 0;
  }
  if (p.slab_mode && st->J1 > st->J0) {
    const int64_t c = (st->J1 - 1) * p.L + p.K;
    if (c > st->compacted_hi) st->compacted_hi = c;
  }
  // the window ends of this task had their block prefixes built (k_vh_build_tile)
  if (p.nagg > 0 && st->J1 > st->J0) {
    const int64_t e = (st->J1 - 1) * p.L + p.K;
    if (e > st->vh_pre_hi) st->vh_pre_hi = e;
  }
  st->live_J0 = st->J0;
  st->J0 = st->jgap_hi > st->J1 ? st->jgap_hi : st->J1;
  meta->nwindows = st->J0 - st->slot_J0;
}

// headers of the empty windows [J1, jgap_hi) of a time gap (k_task_begin):
// nrows = 0, row_offset = the slot's row count so far (reading A6)
__global__ void k_gap_hdr(const Plan p, const State *st, WinHdr *hdr, SlotMeta *meta) {
  const int64_t a = st->J1, b = st->jgap_hi;
  if (b <= a) return;
  const int64_t rows = st->sel_rows;
  for (int64_t j = a + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < b; j += (int64_t)gridDim.x * blockDim.x) {
    WinHdr h;
    h.window_id = j;
    h.ts = p.T0 + j * p.l;
    h.row_offset = rows;
    h.nrows = 0;
    h.flags = 0;
    hdr[j - st->slot_J0] = h;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) meta->nrows = rows;
}

// overlap plans: close the window phase of a slot that ran on its State snapshot
__global__ void k_win_end(State *st, const State *wst, SlotMeta *meta) {
  if (threadIdx.x) return;
  meta->nrows = wst->sel_rows;
  if (wst->error) {
    meta->error |= wst->error;
    atomicOr(&st->error, wst->error);
  }
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

__global__ void k_init_state(State *st, int64_t base_index, int64_t first_window, int64_t L, int64_t epoch0) {
  if (threadIdx.x) return;
  State s = {};
  s.tile_epoch = epoch0;          // look-back epochs stay unique across resets
  s.pos_next = base_index;
  s.J0 = first_window;
  s.J1 = first_window;
  s.zeroed_hi = first_window * L;
  s.pane_hi = -1;
  s.first_task = 1;
  s.carry_pos = base_index;
  s.compacted_hi = first_window * L;
  s.live_J0 = first_window;
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

}  // namespace sb

namespace sb {

cudaError_t launch_task_begin(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int64_t n,
                              int final_, int has_wm, int64_t wm, int emit_on_finish, cudaStream_t st, int round) {
  k_task_begin<<<1, 32, 0, st>>>(p, q.st, (const unsigned char *)tuples, n, final_, has_wm, wm, emit_on_finish,
                                 s.meta, q.carry[0], q.carry[1], q.tile_ctr, q.win_ts, q.ts_mask, round);
  return cudaGetLastError();
}
cudaError_t launch_zero_panes(const Plan &p, const QueryDev &q, cudaStream_t st, int64_t n, int scan_grid) {
  int g = 0;
  const int64_t per = n > 0 && p.nagg > 0 && !p.bucket_mode ? p1_selfzero_per(p, n, scan_grid, &g) : 0;
  k_zero_panes<<<148 * 4, 256, 0, st>>>(p, q.st, q.table, g, per);
  return cudaGetLastError();
}
cudaError_t launch_win_scan(const Plan &p, const QueryDev &q, const SlotDev &s, cudaStream_t st) {
  // reset the ticket counter (k_task_begin already did for this task; the slab
  // and hash paths launch no other ticketed kernel before this one)
  k_win_scan<<<148 * 2, kScanThreads, 0, st>>>(p, q.st, q.pane_ts, s.counts, (WinHdr *)s.hdr, s.meta,
                                               q.tile_status, q.tile_ctr);
  return cudaGetLastError();
}
cudaError_t launch_task_end(const Plan &p, const QueryDev &q, const SlotDev &s, cudaStream_t st) {
  if (p.win_kind == WK_TIME && p.nagg > 0) {
    k_gap_hdr<<<148, 256, 0, st>>>(p, q.st, (WinHdr *)s.hdr, s.meta);
    cudaError_t e = cudaGetLastError();
    if (e) return e;
  }
  k_task_end<<<1, 32, 0, st>>>(p, q.st, s.meta);
  return cudaGetLastError();
}
cudaError_t launch_win_end(const QueryDev &q, const SlotDev &s, cudaStream_t st) {
  k_win_end<<<1, 32, 0, st>>>(q.st, s.wst, s.meta);
  return cudaGetLastError();
}
cudaError_t launch_carry(const Plan &p, const QueryDev &q, const void *tuples, cudaStream_t st) {
  k_carry<<<148, 256, 0, st>>>(p, q.st, (const uint4 *)tuples, (const uint4 *)q.carry[0], (const uint4 *)q.carry[1],
                               (uint4 *)q.carry[0], (uint4 *)q.carry[1]);
  return cudaGetLastError();
}
cudaError_t launch_init_state(const Plan &p, const QueryDev &q, int64_t base_index, int64_t epoch0, cudaStream_t s) {
  k_init_state<<<1, 32, 0, s>>>(q.st, base_index, p.first_window, p.L, epoch0);
  return cudaGetLastError();
}
cudaError_t launch_partition_plan(int ts_word, int tuple_words, int win_kind, int64_t s, int64_t l, int64_t T0,
                                  const void *tuples, int64_t begin, int64_t n, int64_t *dev_out2, cudaStream_t st) {
  k_partition_plan<<<1, 32, 0, st>>>(ts_word, tuple_words * 4, win_kind, s, l, T0, (const unsigned char *)tuples,
                                     begin, n, dev_out2);
  return cudaGetLastError();
}

}  // namespace sb
