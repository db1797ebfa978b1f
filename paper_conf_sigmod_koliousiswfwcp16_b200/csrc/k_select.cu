// k_select.cu -- σ/π with stream compaction (IStream), §5.4 L1315-1327.
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"
#include "launch_internal.h"

namespace sb {

constexpr int kSelThreads = 256;
constexpr int kSelPer = 8;            // tuples per thread per tile
constexpr int kSelTile = kSelThreads * kSelPer;

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

}  // namespace sb

namespace sb {

void *sel_kernel(const Plan &p) {
  switch (p.tuple_words) {
    case 4: return (void *)k_select<4>;
    case 8: return (void *)k_select<8>;
    case 12: return (void *)k_select<12>;
    default: return (void *)k_select<16>;
  }
}

cudaError_t launch_select(const Plan &p, const QueryDev &q, const SlotDev &s, const void *tuples, int grid,
                          cudaStream_t st) {
  void *args[] = {(void *)&p, (void *)&q.st, (void *)&tuples, (void *)&q.carry[0], (void *)&q.carry[1],
                  (void *)&q.tile_status, (void *)&q.tile_ctr, (void *)&s.rows};
  return cudaLaunchKernel(sel_kernel(p), dim3(grid), dim3(kSelThreads), args, 0, st);
}

}  // namespace sb
