// k_select.cu -- σ/π with stream compaction (IStream): PAPER.md §5.4 L1315-1327.
//
// The paper evaluates the predicate into a binary vector in work-group memory
// and prefix-sums it into contiguous output addresses per fragment, offset by
// the fragment's start.  Here one single-pass kernel writes every selected row
// once, straight to its final place:
//   k_select  persistent CTAs take tiles (one 32 KiB TMA stage of the virtual
//             input [carry ++ task], positions [cover_lo, cover_hi)) by ticket,
//             in stream order.  Per tile: σ per tuple, warp ballots + a CTA scan
//             give the tile's row count, which is published at once to a
//             decoupled look-back chain; the exclusive prefix of the tile is
//             resolved one tile LATER (after the CTA has counted its next tile),
//             so predecessors have long published and the look-back rarely
//             waits; then the projected rows go to base + rank.  The tile stays
//             in its shared-memory slot until written; three slots per CTA keep
//             one tile counting, one writing and one loading.
// Only positions [cover_lo, cover_hi) -- tuples whose first window closed in
// this task, position identity (reading A9) -- are emitted.  Window headers
// (row offset of each window's first new tuple) are recorded on the way and
// finished by k_sel_hdr.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "launch_internal.h"
#include "tma.cuh"

namespace sb {

constexpr int kSelThreads = 256, kSelWarps = 8;
constexpr int kSelStageBytes = 32768;
constexpr int kSelStages = 3;
constexpr int kSelMaxIter = kSelStageBytes / 16 / kSelThreads;   // tuples per thread per stage (16-B tuples)

__device__ __forceinline__ int64_t sel_s_int(const unsigned char *t, int word, int type) {
  return type == T_I32 ? (int64_t) * (const int32_t *)(t + 4 * word) : *(const int64_t *)(t + 4 * word);
}
__device__ __forceinline__ double sel_s_flt(const unsigned char *t, int word, int type) {
  return type == T_F32 ? (double)*(const float *)(t + 4 * word) : *(const double *)(t + 4 * word);
}

__global__ void __launch_bounds__(kSelThreads, 2)
k_select(const Plan p, State *__restrict__ st, const unsigned char *__restrict__ task,
         const unsigned char *__restrict__ carry0, const unsigned char *__restrict__ carry1,
         unsigned char *__restrict__ rows, uint64_t *__restrict__ status, int *__restrict__ ticket,
         int64_t *__restrict__ ihdr, int64_t *__restrict__ win_ts, int64_t ts_mask) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ int s_tile[kSelStages];
  __shared__ int64_t s_prev[kSelStages];                 // τ of the tuple before each slot's tile
  __shared__ int s_cnt[kSelMaxIter][kSelWarps];
  __shared__ int s_off[2][kSelMaxIter][kSelWarps];
  __shared__ unsigned s_bal[2][kSelMaxIter][kSelWarps];
  __shared__ int s_total[2];
  __shared__ int64_t s_base;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int tb = p.tuple_bytes;
  const int ST = kSelStageBytes / tb;                     // tuples per tile
  const int NIT = ST / kSelThreads;                       // tuples per thread per tile
  unsigned char *stages = smem;
  uint64_t *full = (uint64_t *)(smem + kSelStages * kSelStageBytes);
  const int64_t cl = st->cover_lo, ch = st->cover_hi;
  const int64_t tpos = st->task_pos, cpos = st->carry_pos;
  const int64_t J0 = st->J0, J1 = st->J1;
  const uint64_t epoch = (uint64_t)st->tile_epoch;
  const unsigned char *carry = st->carry_sel ? carry1 : carry0;
  const int64_t n = ch - cl;
  const int64_t ntiles = (n + ST - 1) / ST;
  const int ow = p.out_row_words;
  const unsigned ltmask = (1u << lane) - 1u;
  auto tau_pos = [&](int64_t pos) -> int64_t {           // τ at a virtual-input position
    return *(const int64_t *)((pos < tpos ? carry + (pos - cpos) * tb : task + (pos - tpos) * tb) + 4 * p.ts_word);
  };
  auto grab = [&](int slot) {                             // next ticket into a free slot (thread 0)
    const int t = atomicAdd(ticket, 1);
    s_tile[slot] = t;
    if (t >= ntiles) return;
    const int64_t a = cl + (int64_t)t * ST, b = (a + ST < ch) ? a + ST : ch;
    s_prev[slot] = a > cpos ? tau_pos(a - 1) : INT64_MIN;
    mbar_expect_tx(&full[slot], (uint32_t)((b - a) * tb));
    unsigned char *dst = stages + slot * kSelStageBytes;
    if (a < tpos) {
      const int64_t e = b < tpos ? b : tpos;
      bulk_g2s(dst, carry + (a - cpos) * tb, (uint32_t)((e - a) * tb), &full[slot]);
      if (b > tpos) bulk_g2s(dst + (e - a) * tb, task, (uint32_t)((b - tpos) * tb), &full[slot]);
    } else {
      bulk_g2s(dst, task + (a - tpos) * tb, (uint32_t)((b - a) * tb), &full[slot]);
    }
  };
  if (tid == 0) {
    for (int i = 0; i < kSelStages; ++i) mbar_init(&full[i], 1);
    fence_mbar_init();
    for (int i = 0; i < kSelStages; ++i) grab(i);
  }
  __syncthreads();
  int err = 0;

  // write tile tp (slot sp, ballots/offsets set bp) at its resolved base
  auto write_tile = [&](int sp, int bp, int64_t tp, int total) {
    if (wid == 0) {
      const int64_t base = lookback_warp(status, tp, epoch, (uint64_t)total, 0, true);
      if (lane == 0) {
        s_base = base;
        if (tp == ntiles - 1) {
          st->sel_rows = base + total;
          if (base + total > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
        }
      }
    }
    __syncthreads();
    const int64_t base = s_base;
    const unsigned char *sb = stages + sp * kSelStageBytes;
    const int64_t a0 = cl + tp * ST;
    const int ns = (int)((ch - a0) < ST ? (ch - a0) : ST);
    // π: projected words of the selected tuples, compacted in stream order
#pragma unroll
    for (int j = 0; j < kSelMaxIter; ++j) {
      if (j >= NIT) continue;
      const unsigned bal = s_bal[bp][j][wid];
      if (!((bal >> lane) & 1u)) continue;
      const int i = j * kSelThreads + tid;
      const int64_t r = base + s_off[bp][j][wid] + __popc(bal & ltmask);
      if (r >= p.rows_cap) continue;
      const uint32_t *src = (const uint32_t *)(sb + i * tb);
      uint32_t *dst = (uint32_t *)(rows + r * (int64_t)ow * 4);
      if ((ow & 3) == 0) {
        for (int c = 0; c < ow; c += 4)
          *(uint4 *)(dst + c) = make_uint4(src[p.proj_word[c]], src[p.proj_word[c + 1]], src[p.proj_word[c + 2]],
                                           src[p.proj_word[c + 3]]);
      } else {
        for (int c = 0; c < ow; ++c) dst[c] = src[p.proj_word[c]];
      }
    }
    // window headers (reading A9: window j's rows are the selected tuples of
    // W_j \ W_{j-1}, a position segment): the global rank of the first row of
    // every window whose segment starts in this tile
    auto rank_at = [&](int x) -> int64_t {                // rows before local index x
      const int jx = x / kSelThreads, tx = x - jx * kSelThreads;
      return base + s_off[bp][jx][tx >> 5] + __popc(s_bal[bp][jx][tx >> 5] & ((1u << (tx & 31)) - 1u));
    };
    if (p.win_kind == WK_COUNT) {
      const int64_t sl = p.l, ss = p.s;
      for (int64_t jj = (a0 + sl - 1) / sl + tid; jj * sl < a0 + ns; jj += kSelThreads)    // τ at window starts (A7)
        win_ts[jj & ts_mask] = *(const int64_t *)(sb + (jj * sl - a0) * tb + 4 * p.ts_word);
      const int64_t jf = a0 <= ss ? 1 : (a0 - ss + sl - 1) / sl + 1;
      if (a0 == 0 && tid == 0 && J0 == 0) ihdr[0] = rank_at(0);
      for (int64_t jj = jf + tid; (jj - 1) * sl + ss < a0 + ns; jj += kSelThreads)
        if (jj >= J0 && jj < J1) ihdr[jj - J0] = rank_at((int)((jj - 1) * sl + ss - a0));
    } else {
      const int64_t sl = p.l, B0 = p.T0 + p.s;
      auto seg = [&](int64_t tau) -> int64_t { return tau < B0 ? 0 : (tau - B0) / sl + 1; };
      for (int x = tid; x < ns; x += kSelThreads) {
        const int64_t pos = a0 + x;
        const int64_t tau = *(const int64_t *)(sb + x * tb + 4 * p.ts_word);
        int64_t jfrom;
        if (pos == cl) jfrom = J0;
        else {
          const int64_t up = x > 0 ? *(const int64_t *)(sb + (x - 1) * tb + 4 * p.ts_word) : s_prev[sp];
          if (up == tau) continue;
          jfrom = seg(up) + 1;
        }
        int64_t jto = seg(tau);
        if (jto > J1 - 1) jto = J1 - 1;
        if (jfrom < J0) jfrom = J0;
        if (jfrom <= jto) {
          const int64_t v = rank_at(x);
          for (int64_t jj = jfrom; jj <= jto; ++jj) ihdr[jj - J0] = v;
        }
      }
      // windows whose segments are empty at the end of the cover start after every row
      if (tp == ntiles - 1 && tid == 0) {
        const int64_t tl = *(const int64_t *)(sb + (ns - 1) * tb + 4 * p.ts_word);
        for (int64_t jj = seg(tl) + 1 > J0 ? seg(tl) + 1 : J0; jj < J1; ++jj) ihdr[jj - J0] = base + total;
      }
    }
    __syncthreads();                                      // the slot is read completely
  };

  int pend_slot = -1, pend_set = 0, pend_total = 0;
  int64_t pend_tile = -1;
  for (int k = 0;; ++k) {
    const int slot = k % kSelStages;
    const int64_t t = s_tile[slot];
    if (t >= ntiles) break;
    mbar_wait(&full[slot], (uint32_t)((k / kSelStages) & 1));
    const unsigned char *sb = stages + slot * kSelStageBytes;
    const int64_t a = cl + t * ST;
    const int ns = (int)((ch - a) < ST ? (ch - a) : ST);
    const int set = k & 1;
#pragma unroll
    for (int j = 0; j < kSelMaxIter; ++j) {
      if (j >= NIT) continue;
      const int i = j * kSelThreads + tid;
      bool s = i < ns;
      if (s) {
        const unsigned char *tp = sb + i * tb;
        const int64_t tau = *(const int64_t *)(tp + 4 * p.ts_word);
        const int64_t up = i > 0 ? *(const int64_t *)(tp - tb + 4 * p.ts_word) : s_prev[slot];
        if (tau < up) err |= ERR_ORDER;
        if (tau < 0) err |= ERR_TS;
        if (p.win_kind == WK_TIME) s &= tau >= p.T0;
        for (int q = 0; q < p.npred && s; ++q) {
          const Pred &pr = p.pred[q];
          s = (pr.type == T_F32 || pr.type == T_F64) ? cmp_op(sel_s_flt(tp, pr.word, pr.type), pr.op, pr.fval)
                                                      : cmp_op(sel_s_int(tp, pr.word, pr.type), pr.op, pr.ival);
        }
      }
      const unsigned bal = __ballot_sync(kFull, s);
      if (lane == 0) { s_cnt[j][wid] = __popc(bal); s_bal[set][j][wid] = bal; }
    }
    __syncthreads();
    if (wid == 0) {                                       // scan of the (j, warp) counts in stream order
      int run = 0;
      for (int b0 = 0; b0 < NIT * kSelWarps; b0 += 32) {
        const int idx = b0 + lane;
        const int v = idx < NIT * kSelWarps ? s_cnt[idx / kSelWarps][idx % kSelWarps] : 0;
        int x = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int y = __shfl_up_sync(kFull, x, o);
          if (lane >= o) x += y;
        }
        if (idx < NIT * kSelWarps) s_off[set][idx / kSelWarps][idx % kSelWarps] = run + x - v;
        run += __shfl_sync(kFull, x, 31);
      }
      if (lane == 0) {
        s_total[set] = run;
        // publish the tile's count now; its prefix is resolved after the next tile
        lb_st(&status[t], lb_pack(epoch, t == 0 ? 2 : 1, (uint64_t)run));
      }
    }
    __syncthreads();
    if (pend_tile >= 0) {
      write_tile(pend_slot, pend_set, pend_tile, pend_total);
      if (tid == 0) grab(pend_slot);                      // refill the written slot
      __syncthreads();
    }
    pend_slot = slot;
    pend_set = set;
    pend_total = s_total[set];
    pend_tile = t;
  }
  if (pend_tile >= 0) write_tile(pend_slot, pend_set, pend_tile, pend_total);
  if (err) atomicOr(&st->error, err);
}

// window headers of the task: row_offset of window j = global rank of its first
// new tuple; nrows = next window's offset - own (the last: the task's total)
__global__ void __launch_bounds__(256)
k_sel_hdr(const Plan p, const State *__restrict__ st, const int64_t *__restrict__ ihdr,
          const int64_t *__restrict__ win_ts, int64_t ts_mask, WinHdr *__restrict__ hdr) {
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  const bool empty = st->cover_hi <= st->cover_lo;
  const int64_t total = empty ? 0 : st->sel_rows;
  auto off = [&](int64_t i) -> int64_t { return (empty || i >= nw) ? total : ihdr[i]; };
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nw; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = J0 + i;
    const int64_t o = off(i);
    WinHdr h;
    h.window_id = j;
    h.ts = p.win_kind == WK_TIME ? p.T0 + j * p.l : win_ts[j & ts_mask];
    h.row_offset = o;
    h.nrows = (int32_t)(off(i + 1) - o);
    h.flags = 0;
    hdr[i] = h;
  }
}

void *sel_kernel(const Plan &p) { return (void *)k_select; }

int sel_smem_bytes() { return kSelStages * kSelStageBytes + kSelStages * 8; }

int64_t sel_tiles(const Plan &p, int64_t cover) { return (cover + kSelStageBytes / p.tuple_bytes - 1) / (kSelStageBytes / p.tuple_bytes); }

cudaError_t launch_select(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int grid,
                          cudaStream_t st) {
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&tuples, (void *)&q.carry[0], (void *)&q.carry[1],
                  (void *)&s.rows, (void *)&q.tile_status, (void *)&q.tile_ctr, (void *)&q.ihdr_tmp,
                  (void *)&q.win_ts, (void *)&q.ts_mask};
  cudaError_t e = cudaLaunchKernel(sel_kernel(p), dim3(grid), dim3(kSelThreads), args, (size_t)sel_smem_bytes(), st);
  if (e) return e;
  k_sel_hdr<<<148, 256, 0, st>>>(p, q.st, q.ihdr_tmp, q.win_ts, q.ts_mask, (WinHdr *)s.hdr);
  return cudaGetLastError();
}

}  // namespace sb
