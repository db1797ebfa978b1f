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

// one thread per (block of K panes, slot)
__global__ void __launch_bounds__(256)
k_vh_build(const Plan p, const State *__restrict__ st, const uint64_t *__restrict__ table,
           uint64_t *__restrict__ pre, uint64_t *__restrict__ suf) {
  const int64_t J0 = st->J0, J1 = st->J1;
  if (J1 <= J0) return;
  const int64_t lo = J0 * p.L, hi = (J1 - 1) * p.L + p.K - 1;
  const int64_t b0 = lo / p.K, b1 = hi / p.K;
  const int64_t items = (b1 - b0 + 1) * p.C;
  const int64_t co = cnt_off(p);
  for (int64_t it = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; it < items; it += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = b0 + it / p.C;
    const int64_t slot = it % p.C;
    const int64_t bs = b * p.K, be = (bs + p.K - 1 < hi) ? bs + p.K - 1 : hi;
    for (int f = -1; f < p.nf; ++f) {
      const int64_t src = (f < 0 ? co : fld_off(p, f)) + slot;
      const int64_t dst = (f < 0 ? 0 : vh_off(p, f)) + slot;
      const uint64_t id = f < 0 ? 0ull : field_identity(p.field[f].kind);
      if (bs >= lo) {                       // prefix arrays are only read for blocks starting >= lo
        uint64_t acc = id;
        for (int64_t q = bs; q <= be; ++q) {
          const int64_t r = (q & (p.R - 1)) * p.slot_words;
          acc = combine_cnt_or_field(p, f, acc, table[r + src]);
          pre[(q & (p.R - 1)) * p.slot_words + dst] = acc;
        }
      }
      uint64_t acc = id;
      const int64_t qlo = bs > lo ? bs : lo;
      for (int64_t q = be; q >= qlo; --q) {
        const int64_t r = (q & (p.R - 1)) * p.slot_words;
        acc = combine_cnt_or_field(p, f, acc, table[r + src]);
        suf[(q & (p.R - 1)) * p.slot_words + dst] = acc;
      }
    }
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
      for (int f = 0; f < p.nf; ++f) {
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
      for (int f = 0; f < p.nf; ++f) {
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
  const int64_t J0 = st->J0, J1 = st->J1, nw = J1 - J0;
  if (nw <= 0) return;
  const int64_t maxprobe = (int64_t)st->max_probe;
  const int64_t span = (SB + maxprobe + 1) < p.C ? (SB + maxprobe + 1) : p.C;
  const int64_t nchunks = (nw + W - 1) / W;
  const int64_t nitems = nchunks * S;
  if (threadIdx.x == 0) s_err = 0;
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t chunk = item / S;
    const uint32_t slot0 = (uint32_t)((item % S) * SB);
    const int64_t ja = J0 + chunk * W;
    const int64_t jb = ja + W < J1 ? ja + W : J1;
    __syncthreads();
    for (int h = threadIdx.x; h < ST; h += blockDim.x) {
      skeys[h] = kEmpty;
      scnt[h] = 0;
      for (int f = 0; f < p.nf; ++f) sf[f * ST + h] = field_identity(p.field[f].kind);
    }
    __syncthreads();
    auto find = [&](uint64_t k) -> int {
      uint32_t h = (uint32_t)(fmix64(k) >> 32) & (uint32_t)(ST - 1);
      volatile uint64_t *vk = skeys;
      for (int probe = 0; probe < ST; ++probe) {
        uint64_t cur = vk[h];
        if (cur == k) return (int)h;
        if (cur == kEmpty) {
          uint64_t old = atomicCAS((unsigned long long *)&skeys[h], kEmpty, k);
          if (old == kEmpty || old == k) return (int)h;
        }
        h = (h + 1) & (uint32_t)(ST - 1);
      }
      s_err = 1;
      return -1;
    };
    // mode 0: add (+1) / subtract (-1) invertible fields; mode 2: min/max only
    auto visit_pane = [&](int64_t q, int sign, bool minmax) {
      const uint64_t *b = table + (q & (p.R - 1)) * p.slot_words;
      for (int64_t o = threadIdx.x; o < span; o += blockDim.x) {
        const uint32_t h = (slot0 + (uint32_t)o) & Cm;
        const uint64_t k = b[h];
        if (k == kEmpty) continue;
        const uint32_t home = (uint32_t)fmix64(k) & Cm;
        if (((home - slot0) & Cm) >= (uint32_t)SB) continue;
        const int s = find(k);
        if (s < 0) continue;
        if (!minmax) {
          atomicAdd((unsigned long long *)&scnt[s], (unsigned long long)(sign * (int64_t)b[p.C + h]));
        }
        for (int f = 0; f < p.nf; ++f) {
          const int kind = p.field[f].kind;
          const uint64_t v = b[fld_off(p, f) + h];
          if (!minmax && kind == FK_SUM_F) atomicAdd((double *)&sf[f * ST + s], sign * __longlong_as_double((long long)v));
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
      for (int h = threadIdx.x; h < ST; h += blockDim.x)
        if (scnt[h] == 0)
          for (int f = 0; f < p.nf; ++f)
            if (p.field[f].kind == FK_SUM_F || p.field[f].kind == FK_SUM_I) sf[f * ST + h] = 0;
      if (p.has_minmax) {
        for (int h = threadIdx.x; h < ST; h += blockDim.x)
          for (int f = 0; f < p.nf; ++f)
            if (p.field[f].kind == FK_MIN || p.field[f].kind == FK_MAX) sf[f * ST + h] = field_identity(p.field[f].kind);
        __syncthreads();
        for (int64_t q = j * p.L; q < j * p.L + p.K; ++q) visit_pane(q, 0, true);
      }
      __syncthreads();
      int my = 0;
      uint64_t fv[kMaxField];
      for (int h = threadIdx.x; h < ST; h += blockDim.x) {
        if (skeys[h] == kEmpty || scnt[h] <= 0) continue;
        for (int f = 0; f < p.nf; ++f) fv[f] = sf[f * ST + h];
        if (having_ok(p, scnt[h], fv)) ++my;
      }
      int total;
      int excl = group_excl_scan(my, 256, scan_sm, total);
      const int64_t ci = (j - J0) * S + (item % S);
      if (!EMIT) {
        if (threadIdx.x == 0) counts[ci] = total;
      } else {
        int64_t r = counts[ci] + excl;
        for (int h = threadIdx.x; h < ST; h += blockDim.x) {
          if (skeys[h] == kEmpty || scnt[h] <= 0) continue;
          for (int f = 0; f < p.nf; ++f) fv[f] = sf[f * ST + h];
          if (!having_ok(p, scnt[h], fv)) continue;
          int64_t kv[kMaxKey];
          decode_key(p, skeys[h], kv);
          write_row(p, rows, r++, kv, scnt[h], fv);
        }
      }
      __syncthreads();
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

}  // namespace sb

namespace sb {
void *p2_kernel_count(const Plan &p) {
  return p.key_mode == KM_HASH ? (void *)k_win_hash<false> : (void *)k_win_vh<false>;
}
}  // namespace sb
