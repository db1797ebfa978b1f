// k_select.cu -- σ/π with stream compaction (IStream): PAPER.md §5.4 L1315-1327.
//
// The paper evaluates the predicate into a binary vector in work-group memory
// and prefix-sums it into contiguous output addresses per fragment, offset by
// the fragment's start.  Here:
//   k_select      every CTA streams a contiguous range of the task through
//                 shared memory with 1-D TMA bulk copies (3 stages in flight),
//                 evaluates σ per tuple, ranks the selected tuples with warp
//                 ballots + a CTA scan per stage, and writes the projected rows,
//                 compacted and in stream order, into its own staging segment
//                 (starting at its range offset); its row count goes to cta_cnt;
//   k_select_fix  each CTA segment is moved to its exclusive offset (a scan of
//                 the per-CTA counts) -- no serial look-back chain between CTAs.
// Only positions [cover_lo, cover_hi) -- tuples whose first window closed in
// this task, position identity (reading A9) -- are emitted; the virtual input is
// [carry (uncovered tail of earlier tasks) ++ task].
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "launch_internal.h"
#include "tma.cuh"

namespace sb {

constexpr int kSelThreads = 256, kSelWarps = 8;
#ifndef SB_SEL_STAGE_KB
#define SB_SEL_STAGE_KB 32
#endif
#ifndef SB_SEL_STAGES
#define SB_SEL_STAGES 3
#endif
#ifndef SB_SEL_BPS
#define SB_SEL_BPS 2
#endif
constexpr int kSelStageBytes = SB_SEL_STAGE_KB * 1024;
constexpr int kSelStages = SB_SEL_STAGES;
constexpr int kSelMaxIter = kSelStageBytes / 16 / kSelThreads;   // tuples per thread per stage (16-B tuples)

__device__ __forceinline__ int64_t sel_s_int(const unsigned char *t, int word, int type) {
  return type == T_I32 ? (int64_t) * (const int32_t *)(t + 4 * word) : *(const int64_t *)(t + 4 * word);
}
__device__ __forceinline__ double sel_s_flt(const unsigned char *t, int word, int type) {
  return type == T_F32 ? (double)*(const float *)(t + 4 * word) : *(const double *)(t + 4 * word);
}

__global__ void __launch_bounds__(kSelThreads, SB_SEL_BPS)
k_select(const Plan p, State *__restrict__ st, const unsigned char *__restrict__ task,
         const unsigned char *__restrict__ carry0, const unsigned char *__restrict__ carry1,
         unsigned char *__restrict__ stage_rows, int64_t *__restrict__ cta_cnt,
         int64_t *__restrict__ ihdr, int64_t *__restrict__ win_ts, int64_t ts_mask) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ int s_cnt[kSelMaxIter][kSelWarps];
  __shared__ unsigned s_bal[kSelMaxIter][kSelWarps];
  __shared__ int s_off[kSelMaxIter][kSelWarps];
  __shared__ int s_total;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int tb = p.tuple_bytes;
  const int ST = kSelStageBytes / tb;                     // tuples per stage
  const int NIT = ST / kSelThreads;                       // tuples per thread per stage
  unsigned char *stages = smem;
  uint64_t *full = (uint64_t *)(smem + kSelStages * kSelStageBytes);
  uint64_t *empty = full + kSelStages;
  const int64_t cl = st->cover_lo, ch = st->cover_hi;
  const int64_t tpos = st->task_pos, cpos = st->carry_pos;
  const int64_t J0 = st->J0, J1 = st->J1;
  const unsigned char *carry = st->carry_sel ? carry1 : carry0;
  // contiguous, stage-aligned range of this CTA within [cover_lo, cover_hi)
  const int64_t n = ch - cl;
  const int64_t per = ((n + gridDim.x - 1) / gridDim.x + ST - 1) / ST * ST;
  const int64_t lo = cl + (int64_t)blockIdx.x * per;
  const int64_t hi = lo + per < ch ? lo + per : ch;
  const int nst = hi > lo ? (int)((hi - lo + ST - 1) / ST) : 0;
  if (tid == 0) {
    for (int i = 0; i < kSelStages; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], kSelWarps); }
    fence_mbar_init();
  }
  __syncthreads();
  auto issue = [&](int k) {          // copy stage k of [carry ++ task]
    const int slot = k % kSelStages;
    const int64_t a = lo + (int64_t)k * ST, b = (a + ST < hi) ? a + ST : hi;
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
  if (tid == 0)
    for (int k = 0; k < kSelStages && k < nst; ++k) issue(k);
  const int ow = p.out_row_words;
  const unsigned ltmask = (1u << lane) - 1u;
  unsigned char *out = stage_rows + (lo - cl) * (int64_t)ow * 4;   // this CTA's staging segment
  int64_t written = 0;
  int err = 0;
  int64_t prev_tau = INT64_MIN;                    // τ of the tuple before the CTA range
  if (lo < hi && lo > cpos) {
    const int64_t pp = lo - 1;
    prev_tau = *(const int64_t *)((pp < tpos ? carry + (pp - cpos) * tb : task + (pp - tpos) * tb) + 4 * p.ts_word);
  }
  for (int k = 0; k < nst; ++k) {
    const int slot = k % kSelStages;
    const uint32_t phase = (uint32_t)((k / kSelStages) & 1);
    mbar_wait(&full[slot], phase);
    const unsigned char *sb = stages + slot * kSelStageBytes;
    const int64_t a = lo + (int64_t)k * ST;
    const int ns = (int)((hi - a) < ST ? (hi - a) : ST);
    unsigned bal[kSelMaxIter];
#pragma unroll
    for (int j = 0; j < kSelMaxIter; ++j) {
      bal[j] = 0;
      if (j >= NIT) continue;
      const int i = j * kSelThreads + tid;
      bool s = i < ns;
      if (s) {
        const unsigned char *tp = sb + i * tb;
        const int64_t tau = *(const int64_t *)(tp + 4 * p.ts_word);
        const int64_t up = i > 0 ? *(const int64_t *)(tp - tb + 4 * p.ts_word) : prev_tau;
        if (tau < up) err |= ERR_ORDER;
        if (tau < 0) err |= ERR_TS;
        if (p.win_kind == WK_TIME) s &= tau >= p.T0;
        for (int q = 0; q < p.npred && s; ++q) {
          const Pred &pr = p.pred[q];
          s = (pr.type == T_F32 || pr.type == T_F64) ? cmp_op(sel_s_flt(tp, pr.word, pr.type), pr.op, pr.fval)
                                                      : cmp_op(sel_s_int(tp, pr.word, pr.type), pr.op, pr.ival);
        }
      }
      bal[j] = __ballot_sync(kFull, s);
      if (lane == 0) { s_cnt[j][wid] = __popc(bal[j]); s_bal[j][wid] = bal[j]; }
    }
    const int64_t prev_tau_stage = prev_tau;
    prev_tau = *(const int64_t *)(sb + (ns - 1) * tb + 4 * p.ts_word);
    __syncthreads();
    if (wid == 0) {                                      // scan of the (j, warp) counts in stream order
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
        if (idx < NIT * kSelWarps) s_off[idx / kSelWarps][idx % kSelWarps] = run + x - v;
        run += __shfl_sync(kFull, x, 31);
      }
      if (lane == 0) s_total = run;
    }
    __syncthreads();
    // window headers (reading A9: window j's rows are the selected tuples of
    // W_j \ W_{j-1}, a position segment): record, for every window whose segment
    // starts in this stage, the CTA-relative rank of its first row
    const int64_t a0 = lo + (int64_t)k * ST;
    auto rank_at = [&](int x) -> int64_t {        // selected tuples of the CTA before local index x
      const int jx = x / kSelThreads, tx = x - jx * kSelThreads;
      return written + s_off[jx][tx >> 5] + __popc(s_bal[jx][tx >> 5] & ((1u << (tx & 31)) - 1u));
    };
    const int64_t pack_cta = (int64_t)blockIdx.x << 44;
    if (p.win_kind == WK_COUNT) {
      const int64_t sl = p.l, ss = p.s;
      // τ at window starts j·l inside the stage (header ts, reading A7)
      for (int64_t jj = (a0 + sl - 1) / sl + tid; jj * sl < a0 + ns; jj += kSelThreads)
        win_ts[jj & ts_mask] = *(const int64_t *)(sb + (jj * sl - a0) * tb + 4 * p.ts_word);
      // segment starts: position 0 (window 0) and (j-1)·l + s (window j >= 1)
      int64_t jf = a0 <= ss ? 1 : (a0 - ss + sl - 1) / sl + 1;
      if (a0 == 0 && tid == 0 && J0 == 0) ihdr[0] = pack_cta | rank_at(0);
      for (int64_t jj = jf + tid; (jj - 1) * sl + ss < a0 + ns; jj += kSelThreads)
        if (jj >= J0 && jj < J1) ihdr[jj - J0] = pack_cta | rank_at((int)((jj - 1) * sl + ss - a0));
    } else {
      const int64_t sl = p.l, B0 = p.T0 + p.s;
      auto seg = [&](int64_t tau) -> int64_t { return tau < B0 ? 0 : (tau - B0) / sl + 1; };
      for (int x = tid; x < ns; x += kSelThreads) {
        const int64_t pos = a0 + x;
        const int64_t tau = *(const int64_t *)(sb + x * tb + 4 * p.ts_word);
        int64_t jfrom;
        if (pos == cl) jfrom = J0;
        else {
          const int64_t up = x > 0 ? *(const int64_t *)(sb + (x - 1) * tb + 4 * p.ts_word) : prev_tau_stage;
          if (up == tau) continue;
          jfrom = seg(up) + 1;
        }
        int64_t jto = seg(tau);
        if (jto > J1 - 1) jto = J1 - 1;
        if (jfrom < J0) jfrom = J0;
        if (jfrom <= jto) {
          const int64_t v = pack_cta | rank_at(x);
          for (int64_t jj = jfrom; jj <= jto; ++jj) ihdr[jj - J0] = v;
        }
      }
    }
    // π: projected words of the selected tuples, compacted in stream order
#pragma unroll
    for (int j = 0; j < kSelMaxIter; ++j) {
      if (j >= NIT) continue;
      if (!((bal[j] >> lane) & 1u)) continue;
      const int i = j * kSelThreads + tid;
      const int64_t r = written + s_off[j][wid] + __popc(bal[j] & ltmask);
      const uint32_t *src = (const uint32_t *)(sb + i * tb);
      uint32_t *dst = (uint32_t *)(out + r * (int64_t)ow * 4);
      if ((ow & 3) == 0) {
        for (int c = 0; c < ow; c += 4)
          *(uint4 *)(dst + c) = make_uint4(src[p.proj_word[c]], src[p.proj_word[c + 1]], src[p.proj_word[c + 2]],
                                           src[p.proj_word[c + 3]]);
      } else {
        for (int c = 0; c < ow; ++c) dst[c] = src[p.proj_word[c]];
      }
    }
    written += s_total;
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[slot]);
    if (tid == 0 && k + kSelStages < nst) {
      mbar_wait(&empty[slot], phase);
      issue(k + kSelStages);
    }
  }
  if (tid == 0) {
    cta_cnt[blockIdx.x] = written;
    // time windows whose segments are empty at the end of the cover start at
    // the cover's end: they begin after every row of the last CTA
    if (p.win_kind == WK_TIME && lo < hi && hi == ch) {
      const int64_t sl = p.l, B0 = p.T0 + p.s;
      const int64_t jfrom = (prev_tau < B0 ? 0 : (prev_tau - B0) / sl + 1) + 1;
      for (int64_t jj = jfrom > J0 ? jfrom : J0; jj < J1; ++jj) ihdr[jj - J0] = ((int64_t)blockIdx.x << 44) | written;
    }
  }
  if (err) atomicOr(&st->error, err);
}

// move every CTA's staged rows to its exclusive offset in the result slot
__global__ void __launch_bounds__(256)
k_select_fix(const Plan p, State *__restrict__ st, const unsigned char *__restrict__ stage_rows,
             const int64_t *__restrict__ cta_cnt, int ncta, unsigned char *__restrict__ rows,
             int64_t *__restrict__ cta_base) {
  __shared__ int64_t s_part[8];
  __shared__ int64_t s_base;
  const int b = blockIdx.x;
  if (b >= ncta) return;
  const int64_t cl = st->cover_lo, ch = st->cover_hi;
  const int tb = p.tuple_bytes;
  const int ST = kSelStageBytes / tb;
  const int64_t n = ch - cl;
  const int64_t per = ((n + ncta - 1) / ncta + ST - 1) / ST * ST;
  // exclusive prefix of the counts of CTAs < b (block reduction)
  int64_t x = 0;
  for (int i = threadIdx.x; i < b; i += blockDim.x) x += cta_cnt[i];
#pragma unroll
  for (int o = 16; o; o >>= 1) x += (int64_t)__shfl_xor_sync(kFull, (unsigned long long)x, o);
  if ((threadIdx.x & 31) == 0) s_part[threadIdx.x >> 5] = x;
  __syncthreads();
  if (threadIdx.x == 0) {
    int64_t s = 0;
    for (int w = 0; w < 8; ++w) s += s_part[w];
    s_base = s;
    cta_base[b] = s;
    if (b == ncta - 1) {
      st->sel_rows = s + cta_cnt[b];
      if (s + cta_cnt[b] > p.rows_cap) atomicOr(&st->error, ERR_RESULT);
    }
  }
  __syncthreads();
  const int64_t base = s_base, cnt = cta_cnt[b];
  const int64_t rb = (int64_t)p.out_row_words * 4;
  const int64_t nbytes = cnt * rb;
  if (base + cnt > p.rows_cap) return;
  const unsigned char *src = stage_rows + (int64_t)b * per * rb;
  unsigned char *dst = rows + base * rb;
  if ((rb & 15) == 0) {
    for (int64_t i = threadIdx.x; i < nbytes / 16; i += blockDim.x)
      ((uint4 *)dst)[i] = ((const uint4 *)src)[i];
  } else {
    for (int64_t i = threadIdx.x; i < nbytes / 4; i += blockDim.x)
      ((uint32_t *)dst)[i] = ((const uint32_t *)src)[i];
  }
}

// window headers of the task: row_offset of window j = global rank of its first
// new tuple; nrows = next window's offset - own (the last: the task's total)
__global__ void __launch_bounds__(256)
k_sel_hdr(const Plan p, const State *__restrict__ st, const int64_t *__restrict__ ihdr,
          const int64_t *__restrict__ cta_base, const int64_t *__restrict__ win_ts, int64_t ts_mask,
          WinHdr *__restrict__ hdr) {
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  const bool empty = st->cover_hi <= st->cover_lo;
  const int64_t total = empty ? 0 : st->sel_rows;
  auto off = [&](int64_t i) -> int64_t {
    if (empty || i >= nw) return total;
    const int64_t v = ihdr[i];
    return cta_base[v >> 44] + (v & ((1ll << 44) - 1));
  };
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

int sel_smem_bytes() { return kSelStages * kSelStageBytes + 2 * kSelStages * 8; }

cudaError_t launch_select(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int grid,
                          cudaStream_t st) {
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&tuples, (void *)&q.carry[0], (void *)&q.carry[1],
                  (void *)&q.sel_stage, (void *)&q.cta_cnt, (void *)&q.ihdr_tmp, (void *)&q.win_ts,
                  (void *)&q.ts_mask};
  cudaError_t e = cudaLaunchKernel(sel_kernel(p), dim3(grid), dim3(kSelThreads), args, (size_t)sel_smem_bytes(), st);
  if (e) return e;
  k_select_fix<<<grid, 256, 0, st>>>(p, q.st, q.sel_stage, q.cta_cnt, grid, s.rows, q.cta_base);
  if ((e = cudaGetLastError())) return e;
  k_sel_hdr<<<148, 256, 0, st>>>(p, q.st, q.ihdr_tmp, q.cta_base, q.win_ts, q.ts_mask, (WinHdr *)s.hdr);
  return cudaGetLastError();
}

}  // namespace sb
